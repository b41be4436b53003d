// Public survivor queue + re-batching top-up (e3.h).
//
// A device FIFO ring of rows ("a queue that holds the partial results",
// PAPER.md:970-972).  head and tail are row counters kept in device memory so
// that pushes whose size is only known on the device (survivor counts) can be
// enqueued without a host round trip; e3_rebatch synchronises the stream to
// read them (the pipeline instead mirrors them on the host, see pipeline.cu).
#include <new>

#include "common.cuh"
#include "kernels.h"

struct e3_queue {
  int device = 0;
  int64_t row_bytes = 0;
  int64_t cap = 0;
  uint8_t *rows = nullptr;
  int64_t *ids = nullptr;
  int64_t *ctr = nullptr;     // device [2]: head, tail
  int *overflow = nullptr;    // device flag
  bool poisoned = false;
};

using namespace e3;

extern "C" {

e3_status e3_queue_create(int device, int64_t row_bytes, int32_t cap_rows, e3_queue **q) {
  E3_CHECK_ARG(q && row_bytes > 0 && cap_rows > 0, "bad arguments");
  E3_CHECK_ARG(row_bytes % 16 == 0, "row_bytes must be a multiple of 16");
  E3_CUDA_TRY(cudaSetDevice(device));
  e3_queue *Q = new (std::nothrow) e3_queue();
  if (!Q) return E3_ECUDA;
  Q->device = device;
  Q->row_bytes = row_bytes;
  Q->cap = cap_rows;
  cudaError_t e = cudaMalloc(&Q->rows, (size_t)row_bytes * cap_rows);
  if (e == cudaSuccess) e = cudaMalloc(&Q->ids, (size_t)cap_rows * 8);
  if (e == cudaSuccess) e = cudaMalloc(&Q->ctr, 2 * 8);
  if (e == cudaSuccess) e = cudaMalloc(&Q->overflow, sizeof(int));
  if (e == cudaSuccess) e = cudaMemset(Q->ctr, 0, 16);
  if (e == cudaSuccess) e = cudaMemset(Q->overflow, 0, sizeof(int));
  if (e != cudaSuccess) {
    e3_queue_destroy(Q);
    return cuda_fail(e, "e3_queue_create");
  }
  *q = Q;
  return E3_OK;
}

e3_status e3_queue_destroy(e3_queue *q) {
  if (!q) return E3_OK;
  cudaFree(q->rows);
  cudaFree(q->ids);
  cudaFree(q->ctr);
  cudaFree(q->overflow);
  delete q;
  return E3_OK;
}

e3_status e3_queue_push(e3_queue *q, void *stream, const void *rows, const int64_t *ids, const int32_t *n_dev,
                        int32_t max_rows) {
  E3_CHECK_ARG(q && rows && ids && n_dev && max_rows >= 0, "bad arguments");
  if (q->poisoned) {
    set_error("queue poisoned");
    return E3_ESTATE;
  }
  E3_CHECK_ARG((reinterpret_cast<uintptr_t>(rows) & 15) == 0, "rows must be 16-byte aligned");
  e3_status r = ring_push_copy(rows, ids, n_dev, max_rows, q->rows, q->ids, q->cap, q->ctr + 1, q->ctr, q->overflow,
                               q->row_bytes, reinterpret_cast<cudaStream_t>(stream));
  if (r == E3_ECUDA) q->poisoned = true;
  return r;
}

static e3_status read_state(e3_queue *q, cudaStream_t st, int64_t *head, int64_t *tail) {
  int64_t c[2];
  int ovf = 0;
  E3_CUDA_TRY(cudaMemcpyAsync(c, q->ctr, 16, cudaMemcpyDeviceToHost, st));
  E3_CUDA_TRY(cudaMemcpyAsync(&ovf, q->overflow, sizeof(int), cudaMemcpyDeviceToHost, st));
  E3_CUDA_TRY(cudaStreamSynchronize(st));
  if (ovf) {
    set_error("queue overflow: a push exceeded the ring capacity");
    return E3_ECAPACITY;
  }
  *head = c[0];
  *tail = c[1];
  return E3_OK;
}

e3_status e3_queue_count(e3_queue *q, int32_t *host_count) {
  E3_CHECK_ARG(q && host_count, "bad arguments");
  int64_t h, t;
  E3_CUDA_TRY(cudaDeviceSynchronize());
  e3_status r = read_state(q, nullptr, &h, &t);
  if (r != E3_OK) return r;
  *host_count = (int32_t)(t - h);
  return E3_OK;
}

e3_status e3_rebatch(e3_queue *q, void *stream, int32_t B, int32_t flush, void *x_out, int64_t *id_out,
                     int32_t *n_valid_dev, int32_t *emitted) {
  E3_CHECK_ARG(q && x_out && id_out && n_valid_dev && emitted && B > 0, "bad arguments");
  if (q->poisoned) {
    set_error("queue poisoned");
    return E3_ESTATE;
  }
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  int64_t h, t;
  e3_status r = read_state(q, st, &h, &t);
  if (r != E3_OK) return r;
  const int64_t count = t - h;
  *emitted = 0;
  if (count < B && !(flush && count > 0)) return E3_OK;
  const int n = count >= B ? B : (int)count;   // never more than B
  r = ring_pop_copy(q->rows, q->ids, q->cap, h, n, B, q->row_bytes, x_out, id_out, 0, st);
  if (r != E3_OK) {
    q->poisoned = true;
    return r;
  }
  const int64_t new_head = h + n;
  E3_CUDA_TRY(cudaMemcpyAsync(q->ctr, &new_head, 8, cudaMemcpyHostToDevice, st));
  r = fill_valid(n_valid_dev, n, st);
  if (r != E3_OK) return r;
  E3_CUDA_TRY(cudaStreamSynchronize(st));   // new_head lives on this stack frame
  *emitted = 1;
  return E3_OK;
}

}  // extern "C"
