// common.cuh — libstg internals: status/error plumbing, device allocation,
// kernel launch accounting.  Product code only (no oracle code is reachable).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <atomic>
#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <string>
#include <utility>

#include "../../include/stg.h"

namespace stg {

// ---------------------------------------------------------------- errors
void set_error(const char* fmt, ...);
stg_status fail(stg_status s, const char* fmt, ...);
stg_status cuda_fail(cudaError_t e, const char* what, const char* file, int line);

#define STG_CUDA(call)                                                          \
  do {                                                                          \
    cudaError_t e_ = (call);                                                    \
    if (e_ != cudaSuccess) return ::stg::cuda_fail(e_, #call, __FILE__, __LINE__); \
  } while (0)

#define STG_TRY(call)                          \
  do {                                         \
    stg_status s_ = (call);                    \
    if (s_ != STG_OK) return s_;               \
  } while (0)

// Checks for a sticky/async error from earlier work and for a launch error.
stg_status check_launch(const char* what);

// Counts every kernel launched by this library (reported by
// stg_kernel_launch_count and used by bench.py's "gpu_launches").
extern std::atomic<int64_t> g_launches;
inline void count_launch(int n = 1) { g_launches.fetch_add(n, std::memory_order_relaxed); }

// ---------------------------------------------------------------- memory
void* dmalloc(size_t bytes, cudaStream_t s);
void dfree(void* p, cudaStream_t s);

template <class T>
struct DArray {
  T* p = nullptr;
  size_t n = 0;
  DArray() = default;
  DArray(const DArray&) = delete;
  DArray& operator=(const DArray&) = delete;
  DArray(DArray&& o) noexcept : p(o.p), n(o.n) { o.p = nullptr; o.n = 0; }
  DArray& operator=(DArray&& o) noexcept {
    if (this != &o) { reset(); p = o.p; n = o.n; o.p = nullptr; o.n = 0; }
    return *this;
  }
  ~DArray() { reset(); }
  void reset() {
    if (p) dfree(p, nullptr);
    p = nullptr; n = 0;
  }
  // (re)allocates to hold at least `count` elements; contents undefined
  stg_status alloc(size_t count, cudaStream_t s = nullptr) {
    if (count <= n && p) return STG_OK;
    reset();
    size_t c = count ? count : 1;
    p = static_cast<T*>(dmalloc(c * sizeof(T), s));
    if (!p) return fail(STG_ERR_NO_MEMORY, "device allocation of %zu bytes failed", c * sizeof(T));
    n = c;
    return STG_OK;
  }
  T* get() const { return p; }
};

// A grow-only scratch arena (bump allocator reset per use).
struct Scratch {
  DArray<unsigned char> buf;
  size_t off = 0;
  void reset() { off = 0; }
};

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

int num_sms();

// 2-D TMA descriptor of a row-major fp32 matrix [rows × cols] (row stride ld
// elements, 16-byte aligned), box [box_rows × box_cols] with 128-byte swizzle
// (box_cols·4 <= 128; atom32: 32-byte swizzle atoms = the UMMA MN-major
// SWIZZLE_128B_BASE32B layout).  Encoded through the driver entry point.
stg_status make_tmap_f32(CUtensorMap* out, const float* base, uint64_t rows, uint64_t cols, uint64_t ld,
                         uint32_t box_cols, uint32_t box_rows, bool atom32 = false);
// Output (store) map of the per-warp box stores: box [box_rows × box_cols] with
// the swizzle whose span equals the box row (box_cols·4 = 32 or 64 bytes), see
// tc::box_off.
stg_status make_tmap_f32_store(CUtensorMap* out, float* base, uint64_t rows, uint64_t cols, uint64_t ld,
                               uint32_t box_cols, uint32_t box_rows);
// 3-D store map of a contiguous [planes][rows][cols] fp32 tensor, box [1][box_rows][box_cols]
stg_status make_tmap_f32_store3(CUtensorMap* out, float* base, uint64_t planes, uint64_t rows, uint64_t cols,
                                uint32_t box_cols, uint32_t box_rows);

// The timing surrogate head fused into the GRU kernels (per-step Algorithm-1
// driver): forward y_t, w_o, b_o, 1/V_total; per-CTA partials of Σ e² (lpart),
// Σ g·ReLU(H') and Σ g (gpart [nb][H+1]); per row hg = {g, bits(H' > 0)} for
// the backward, which adds dℓ/dH' = g·w_o ⊙ [H' > 0] to its upstream gradient.
struct HeadArgs {
  const float* y;
  const float* w_o;
  const float* b_o;
  float inv_v;
  double* lpart;
  float* gpart;
  float2* hg;
};

// ---------------------------------------------------------------- profiler
// Per-phase device time with CUDA events on the launching stream (bench.py and
// the Fig. 9 breakdown).  Off by default; zero cost when off.
enum Phase { PH_AGG_FWD = 0, PH_AGG_BWD, PH_SNAPSHOT, PH_XW, PH_GRU_FWD, PH_GRU_BWD, PH_DW, PH_HEAD, PH_DL,
             PH_SNAP_STEP, PH_SNAP_XPOSE, PH_COUNT };   // (the last two are sub-phases of PH_SNAPSHOT)
bool prof_on();
cudaEvent_t prof_event();
void prof_push(int phase, cudaEvent_t a, cudaEvent_t b);
struct ProfScope {
  int phase;
  cudaStream_t s;
  cudaEvent_t a = nullptr;
  ProfScope(int ph, cudaStream_t st) : phase(ph), s(st) {
    if (prof_on()) { a = prof_event(); cudaEventRecord(a, s); }
  }
  ~ProfScope() {
    if (a) { cudaEvent_t b = prof_event(); cudaEventRecord(b, s); prof_push(phase, a, b); }
  }
};

}  // namespace stg
