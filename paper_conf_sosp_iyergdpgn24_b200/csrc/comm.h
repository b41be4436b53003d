// Inter-split transfer primitives (e3.h "comm").  Product
// code only.
//
// A Link is one direction between this rank and a peer rank.  Messages on a
// link are matched in order; each is a fixed number of bytes.  post() is
// asynchronous: a send starts once `ready` (an event on the producer's
// stream) has completed, a recv lands in the buffer; query(no) reports
// whether message `no` has completed and, for a receive, hands back an event
// that a consumer stream may wait on.
//   NCCL      ncclSend / ncclRecv on a 2-rank communicator split off the
//             world communicator, on the link's own stream
//   LOOPBACK  both ranks in this process: a hub channel matches the i-th send
//             with the i-th recv and enqueues a device-to-device copy
#pragma once

#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>
#include <memory>
#include <string>

#include "../../include/e3.h"

namespace e3 {

struct Chan;
struct Hub;
typedef struct ncclComm *ncclCommPtr;

constexpr int kLinkEvents = 16;   // per-link event ring (>= messages in flight)

struct Link {
  int peer = -1;          // world rank of the other end
  bool send = false;
  int64_t posted = 0;     // messages posted on this link
  // NCCL
  ncclCommPtr comm = nullptr;
  int peer_in_comm = 0;
  cudaStream_t stream = nullptr;
  cudaEvent_t ev[kLinkEvents] = {};
  // LOOPBACK
  Chan *chan = nullptr;

  ~Link();
  e3_status post(void *buf, size_t bytes, cudaEvent_t ready);
  // done: message `no` (< posted) completed; ev (recv only, when done): an
  // event recorded after the data landed
  e3_status query(int64_t no, bool *done, cudaEvent_t *ev);
  e3_status check_async();   // NCCL asynchronous errors -> E3_ENCCL
};

// Creates the link for (this rank -> peer) or (peer -> this rank).  NCCL:
// `link_color` is the canonical index of the link in the plan; every world
// rank must call comm_split_link with the same sequence of colors
// (members: sender and receiver; everybody else passes member = false).
e3_status comm_make_link(e3_comm *c, int link_color, bool member, bool send, int peer, std::unique_ptr<Link> *out);
int comm_rank(const e3_comm *c);
int comm_world(const e3_comm *c);
int comm_device(const e3_comm *c);
int comm_transport(const e3_comm *c);

}  // namespace e3
