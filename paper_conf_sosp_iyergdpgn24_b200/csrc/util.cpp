// Error plumbing, device queries and TMA tensor-map encoding.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <string>

#include "common.cuh"

namespace e3 {

static thread_local std::string g_last_error;

void set_error(const std::string &msg) { g_last_error = msg; }

e3_status cuda_fail(cudaError_t e, const char *what) {
  set_error(std::string("CUDA error ") + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ") at " + what);
  return E3_ECUDA;
}

PFN_encodeTiled encode_tiled_fn() {
  static PFN_encodeTiled fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_encodeTiled>(p);
  });
  return fn;
}

static e3_status encode(CUtensorMap *m, int rank, const void *base, const cuuint64_t *dims, const cuuint64_t *strides,
                        const cuuint32_t *box, CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  PFN_encodeTiled fn = encode_tiled_fn();
  if (!fn) {
    set_error("cuTensorMapEncodeTiled unavailable (no CUDA driver?)");
    return E3_ECUDA;
  }
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, (cuuint32_t)rank, const_cast<void *>(base), dims, strides, box,
                  estr, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    char buf[160];
    snprintf(buf, sizeof buf, "cuTensorMapEncodeTiled failed (%d): rank %d box %u x %u", (int)r, rank, box[0],
             box[1]);
    set_error(buf);
    return E3_ECUDA;
  }
  return E3_OK;
}

e3_status make_tmap_2d(CUtensorMap *m, const void *base, uint64_t rows, uint64_t cols, uint64_t row_pitch_elems,
                       uint32_t box_rows, uint32_t box_cols) {
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {row_pitch_elems * 2};
  cuuint32_t box[2] = {box_cols, box_rows};
  return encode(m, 2, base, dims, strides, box);
}

e3_status make_tmap_2d_sw64(CUtensorMap *m, const void *base, uint64_t rows, uint64_t cols, uint64_t row_pitch_elems,
                            uint32_t box_rows, uint32_t box_cols) {
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {row_pitch_elems * 2};
  cuuint32_t box[2] = {box_cols, box_rows};
  return encode(m, 2, base, dims, strides, box, CU_TENSOR_MAP_SWIZZLE_64B);
}

e3_status make_tmap_3d(CUtensorMap *m, const void *base, uint64_t d0, uint64_t d1, uint64_t d2, uint64_t pitch1,
                       uint64_t pitch2, uint32_t b0, uint32_t b1, uint32_t b2) {
  cuuint64_t dims[3] = {d0, d1, d2};
  cuuint64_t strides[2] = {pitch1 * 2, pitch2 * 2};
  cuuint32_t box[3] = {b0, b1, b2};
  return encode(m, 3, base, dims, strides, box);
}

bool pdl_enabled() {
  static const bool on = [] {
    const char *e = getenv("E3_NO_PDL");
    return !(e && e[0] == '1');
  }();
  return on;
}

int num_sms(int device) {
  int n = 0;
  if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, device) != cudaSuccess || n <= 0) n = 148;
  return n;
}

}  // namespace e3

extern "C" const char *e3_last_error(void) { return e3::g_last_error.c_str(); }
extern "C" const char *e3_version(void) { return "e3-b200 0.1 (sm_100a)"; }
