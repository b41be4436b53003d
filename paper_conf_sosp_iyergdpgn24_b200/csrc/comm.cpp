// Communicators and links of the inter-split transfer (comm.h; e3.h "comm").
//
// NCCL is resolved at run time (dlopen of libnccl.so.2 -- the copy torch
// already loaded when it is in the process), so libe3.so links no NCCL and
// still loads on a host without one; every entry point then reports E3_ENCCL.
#include <dlfcn.h>
#include <nccl.h>

#include <chrono>
#include <cstring>
#include <deque>
#include <map>
#include <mutex>
#include <new>
#include <utility>

#include "comm.h"
#include "common.cuh"

namespace e3 {

namespace {

struct NcclApi {
  bool ok = false;
  std::string why;
  ncclResult_t (*get_unique_id)(ncclUniqueId *) = nullptr;
  ncclResult_t (*init_rank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*split)(ncclComm_t, int, int, ncclComm_t *, ncclConfig_t *) = nullptr;
  ncclResult_t (*send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*destroy)(ncclComm_t) = nullptr;
  ncclResult_t (*async_error)(ncclComm_t, ncclResult_t *) = nullptr;
  const char *(*error_string)(ncclResult_t) = nullptr;
};

const NcclApi &nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_LOCAL);
    if (!h) {
      api.why = std::string("libnccl.so.2 not loadable: ") + dlerror();
      return;
    }
    auto sym = [&](const char *n) { return dlsym(h, n); };
    api.get_unique_id = reinterpret_cast<decltype(api.get_unique_id)>(sym("ncclGetUniqueId"));
    api.init_rank = reinterpret_cast<decltype(api.init_rank)>(sym("ncclCommInitRank"));
    api.split = reinterpret_cast<decltype(api.split)>(sym("ncclCommSplit"));
    api.send = reinterpret_cast<decltype(api.send)>(sym("ncclSend"));
    api.recv = reinterpret_cast<decltype(api.recv)>(sym("ncclRecv"));
    api.destroy = reinterpret_cast<decltype(api.destroy)>(sym("ncclCommDestroy"));
    api.async_error = reinterpret_cast<decltype(api.async_error)>(sym("ncclCommGetAsyncError"));
    api.error_string = reinterpret_cast<decltype(api.error_string)>(sym("ncclGetErrorString"));
    api.ok = api.get_unique_id && api.init_rank && api.split && api.send && api.recv && api.destroy &&
             api.async_error && api.error_string;
    if (!api.ok) api.why = "libnccl.so.2 lacks ncclCommSplit / ncclSend / ncclRecv (need NCCL >= 2.18)";
  });
  return api;
}

e3_status nccl_fail(ncclResult_t r, const char *what) {
  const NcclApi &a = nccl();
  set_error(std::string("NCCL error at ") + what + ": " + (a.error_string ? a.error_string(r) : "?"));
  return E3_ENCCL;
}

#define E3_NCCL_TRY(expr)                                  \
  do {                                                     \
    ncclResult_t _r = (expr);                              \
    if (_r != ncclSuccess) return nccl_fail(_r, #expr);    \
  } while (0)

e3_status need_nccl() {
  if (!nccl().ok) {
    set_error(nccl().why);
    return E3_ENCCL;
  }
  return E3_OK;
}

}  // namespace

// ------------------------------------------------------------ loopback hub
struct Chan {
  std::mutex mu;
  struct S {
    const void *buf;
    size_t bytes;
    cudaEvent_t ready;
  };
  struct R {
    void *buf;
    size_t bytes;
  };
  std::deque<S> sends;
  std::deque<R> recvs;
  int64_t matched = 0;
  cudaStream_t stream = nullptr;
  cudaEvent_t done[kLinkEvents] = {};

  e3_status match() {   // mu held
    while (!sends.empty() && !recvs.empty()) {
      const S s = sends.front();
      const R r = recvs.front();
      sends.pop_front();
      recvs.pop_front();
      if (s.bytes != r.bytes) {
        set_error("loopback link: send and recv sizes differ");
        return E3_EINVAL;
      }
      if (s.ready) E3_CUDA_TRY(cudaStreamWaitEvent(stream, s.ready, 0));
      E3_CUDA_TRY(cudaMemcpyAsync(r.buf, s.buf, s.bytes, cudaMemcpyDeviceToDevice, stream));
      E3_CUDA_TRY(cudaEventRecord(done[matched % kLinkEvents], stream));
      ++matched;
    }
    return E3_OK;
  }
  ~Chan() {
    for (auto &e : done)
      if (e) cudaEventDestroy(e);
    if (stream) cudaStreamDestroy(stream);
  }
};

struct Hub {
  int device = 0;
  std::mutex mu;
  std::map<std::pair<int, int>, std::unique_ptr<Chan>> chans;

  e3_status get(int src, int dst, Chan **out) {
    std::lock_guard<std::mutex> g(mu);
    auto &c = chans[{src, dst}];
    if (!c) {
      auto ch = std::make_unique<Chan>();
      E3_CUDA_TRY(cudaStreamCreateWithFlags(&ch->stream, cudaStreamNonBlocking));
      for (auto &e : ch->done) E3_CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
      c = std::move(ch);
    }
    *out = c.get();
    return E3_OK;
  }
};

// ------------------------------------------------------------------- link
Link::~Link() {
  if (comm && nccl().ok) nccl().destroy(reinterpret_cast<ncclComm_t>(comm));
  for (auto &e : ev)
    if (e) cudaEventDestroy(e);
  if (stream) cudaStreamDestroy(stream);
}

e3_status Link::post(void *buf, size_t bytes, cudaEvent_t ready) {
  if (chan) {
    std::lock_guard<std::mutex> g(chan->mu);
    if (send) chan->sends.push_back({buf, bytes, ready});
    else chan->recvs.push_back({buf, bytes});
    ++posted;
    return chan->match();
  }
  const NcclApi &a = nccl();
  auto c = reinterpret_cast<ncclComm_t>(comm);
  if (send) {
    if (ready) E3_CUDA_TRY(cudaStreamWaitEvent(stream, ready, 0));
    E3_NCCL_TRY(a.send(buf, bytes, ncclUint8, peer_in_comm, c, stream));
  } else {
    E3_NCCL_TRY(a.recv(buf, bytes, ncclUint8, peer_in_comm, c, stream));
  }
  E3_CUDA_TRY(cudaEventRecord(ev[posted % kLinkEvents], stream));
  ++posted;
  return E3_OK;
}

e3_status Link::query(int64_t no, bool *done, cudaEvent_t *e) {
  *done = false;
  cudaEvent_t x = nullptr;
  if (chan) {
    std::lock_guard<std::mutex> g(chan->mu);
    if (no >= chan->matched) return E3_OK;
    x = chan->done[no % kLinkEvents];
  } else {
    if (no >= posted) return E3_OK;
    x = ev[no % kLinkEvents];
  }
  const cudaError_t r = cudaEventQuery(x);
  if (r == cudaErrorNotReady) {
    cudaGetLastError();
    return E3_OK;
  }
  E3_CUDA_TRY(r);
  *done = true;
  if (e) *e = x;
  return E3_OK;
}

e3_status Link::check_async() {
  if (!comm) return E3_OK;
  ncclResult_t st = ncclSuccess;
  E3_NCCL_TRY(nccl().async_error(reinterpret_cast<ncclComm_t>(comm), &st));
  if (st != ncclSuccess && st != ncclInProgress) return nccl_fail(st, "link communicator (asynchronous)");
  return E3_OK;
}

}  // namespace e3

struct e3_comm {
  int rank = 0, world = 1, device = 0;
  int transport = E3_TRANSPORT_NCCL;
  ncclComm_t world_comm = nullptr;
  std::shared_ptr<e3::Hub> hub;
};

namespace e3 {

int comm_rank(const e3_comm *c) { return c ? c->rank : 0; }
int comm_world(const e3_comm *c) { return c ? c->world : 1; }
int comm_device(const e3_comm *c) { return c ? c->device : 0; }
int comm_transport(const e3_comm *c) { return c ? c->transport : E3_TRANSPORT_LOOPBACK; }

e3_status comm_make_link(e3_comm *c, int color, bool member, bool send, int peer, std::unique_ptr<Link> *out) {
  out->reset();
  std::unique_ptr<Link> L;
  if (member) {
    L = std::make_unique<Link>();
    L->peer = peer;
    L->send = send;
  }
  if (c->transport == E3_TRANSPORT_LOOPBACK) {
    if (!member) return E3_OK;
    const int src = send ? c->rank : peer, dst = send ? peer : c->rank;
    e3_status r = c->hub->get(src, dst, &L->chan);
    if (r != E3_OK) return r;
    *out = std::move(L);
    return E3_OK;
  }
  e3_status r = need_nccl();
  if (r != E3_OK) return r;
  ncclComm_t nc = nullptr;
  E3_NCCL_TRY(nccl().split(c->world_comm, member ? color : NCCL_SPLIT_NOCOLOR, send ? 0 : 1, &nc, nullptr));
  if (!member) return E3_OK;
  L->comm = reinterpret_cast<ncclCommPtr>(nc);
  L->peer_in_comm = send ? 1 : 0;
  E3_CUDA_TRY(cudaStreamCreateWithFlags(&L->stream, cudaStreamNonBlocking));
  for (auto &e : L->ev) E3_CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  *out = std::move(L);
  return E3_OK;
}

}  // namespace e3

using namespace e3;

extern "C" {

e3_status e3_comm_unique_id(uint8_t id[E3_COMM_ID_BYTES]) {
  E3_CHECK_ARG(id, "null id");
  e3_status r = need_nccl();
  if (r != E3_OK) return r;
  static_assert(sizeof(ncclUniqueId) == E3_COMM_ID_BYTES, "NCCL unique id size");
  ncclUniqueId u;
  E3_NCCL_TRY(nccl().get_unique_id(&u));
  std::memcpy(id, &u, sizeof u);
  return E3_OK;
}

e3_status e3_comm_init(const uint8_t id[E3_COMM_ID_BYTES], int rank, int world, int device, e3_comm **out) {
  E3_CHECK_ARG(id && out && world >= 1 && rank >= 0 && rank < world && device >= 0, "bad comm arguments");
  e3_status r = need_nccl();
  if (r != E3_OK) return r;
  E3_CUDA_TRY(cudaSetDevice(device));
  ncclUniqueId u;
  std::memcpy(&u, id, sizeof u);
  ncclComm_t nc = nullptr;
  E3_NCCL_TRY(nccl().init_rank(&nc, world, u, rank));
  e3_comm *c = new (std::nothrow) e3_comm();
  if (!c) return E3_ECUDA;
  c->rank = rank;
  c->world = world;
  c->device = device;
  c->transport = E3_TRANSPORT_NCCL;
  c->world_comm = nc;
  *out = c;
  return E3_OK;
}

e3_status e3_comm_init_loopback(int world, int device, e3_comm **out) {
  E3_CHECK_ARG(out && world >= 1 && world <= E3_MAX_REPLICA_SLOTS && device >= 0, "bad loopback arguments");
  auto hub = std::make_shared<Hub>();
  hub->device = device;
  for (int i = 0; i < world; ++i) {
    e3_comm *c = new (std::nothrow) e3_comm();
    if (!c) return E3_ECUDA;
    c->rank = i;
    c->world = world;
    c->device = device;
    c->transport = E3_TRANSPORT_LOOPBACK;
    c->hub = hub;
    out[i] = c;
  }
  return E3_OK;
}

e3_status e3_comm_rank(const e3_comm *c, int32_t *rank, int32_t *world) {
  E3_CHECK_ARG(c && rank && world, "null argument");
  *rank = c->rank;
  *world = c->world;
  return E3_OK;
}

e3_status e3_comm_destroy(e3_comm *c) {
  if (!c) return E3_OK;
  if (c->world_comm && nccl().ok) nccl().destroy(c->world_comm);
  delete c;
  return E3_OK;
}

}  // extern "C"
