// common.cu — error strings, allocator hook, launch counter.
#include <mutex>
#include <unordered_map>

#include "common.cuh"

#include <mutex>
#include <vector>

namespace stg {

static thread_local std::string t_err;
std::atomic<int64_t> g_launches{0};

static stg_alloc_fn g_alloc = nullptr;
static stg_free_fn g_free = nullptr;
static void* g_ctx = nullptr;

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  t_err = buf;
}

stg_status fail(stg_status s, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  t_err = buf;
  return s;
}

stg_status cuda_fail(cudaError_t e, const char* what, const char* file, int line) {
  return fail(STG_ERR_CUDA, "%s failed at %s:%d: %s (%s)", what, file, line, cudaGetErrorName(e),
              cudaGetErrorString(e));
}

stg_status check_launch(const char* what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(STG_ERR_CUDA, "kernel launch %s: %s", what, cudaGetErrorString(e));
  return STG_OK;
}

// Blocks from the allocator hook remember the free function they came from, so
// a block outlives a later stg_set_allocator call safely.
struct HookBlock {
  stg_free_fn free_fn;
  void* ctx;
};
static std::mutex g_hook_mu;
static std::unordered_map<void*, HookBlock> g_hook_blocks;
static bool g_detached = false;     // stg_allocator_detach: hook blocks are never freed

void* dmalloc(size_t bytes, cudaStream_t s) {
  stg_alloc_fn a;
  stg_free_fn f;
  void* ctx;
  {
    std::lock_guard<std::mutex> lk(g_hook_mu);
    a = g_alloc; f = g_free; ctx = g_ctx;
  }
  if (a) {
    // A pooled block may have been released by its previous owner with work still
    // pending on another stream, and the library may use this block on any of its
    // streams: wait for the device first (cudaMalloc's ordering; allocations are
    // grow-only and rare, never inside a captured graph)
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(s, &cs) != cudaSuccess) cudaGetLastError();
    if (cs == cudaStreamCaptureStatusNone) cudaDeviceSynchronize();
    void* p = a(bytes, (stg_stream_t)s, ctx);
    if (p) {
      std::lock_guard<std::mutex> lk(g_hook_mu);
      g_hook_blocks[p] = HookBlock{f, ctx};
    }
    return p;
  }
  void* p = nullptr;
  if (cudaMalloc(&p, bytes) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return p;
}

void dfree(void* p, cudaStream_t s) {
  if (!p) return;
  HookBlock hb{nullptr, nullptr};
  bool hooked = false;
  {
    std::lock_guard<std::mutex> lk(g_hook_mu);
    auto it = g_hook_blocks.find(p);
    if (it != g_hook_blocks.end()) {
      hb = it->second;
      hooked = true;
      g_hook_blocks.erase(it);
    }
  }
  if (hooked && !hb.free_fn) return;   // detached (process teardown): the owner's pool is gone
  if (hb.free_fn) {
    // cudaFree's ordering: no kernel of any stream may still use the block when
    // it returns to the caller's pool
    cudaDeviceSynchronize();
    hb.free_fn(p, (stg_stream_t)s, hb.ctx);
    return;
  }
  cudaFree(p);
}

int num_sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

struct Prof {
  std::mutex mu;
  bool on = false;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> pending[PH_COUNT];
  std::vector<cudaEvent_t> pool;
  double total[PH_COUNT] = {};
  int64_t count[PH_COUNT] = {};
};
static Prof& prof() {
  static Prof p;
  return p;
}
bool prof_on() { return prof().on; }
cudaEvent_t prof_event() {
  Prof& p = prof();
  std::lock_guard<std::mutex> lk(p.mu);
  if (!p.pool.empty()) {
    cudaEvent_t e = p.pool.back();
    p.pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}
void prof_push(int phase, cudaEvent_t a, cudaEvent_t b) {
  Prof& p = prof();
  std::lock_guard<std::mutex> lk(p.mu);
  p.pending[phase].emplace_back(a, b);
}

typedef CUresult (*PFN_encodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

stg_status make_tmap_f32(CUtensorMap* out, const float* base, uint64_t rows, uint64_t cols, uint64_t ld,
                         uint32_t box_cols, uint32_t box_rows, bool atom32) {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess || !p ||
        q != cudaDriverEntryPointSuccess) {
      cudaGetLastError();
      return fail(STG_ERR_CUDA, "cuTensorMapEncodeTiled entry point unavailable");
    }
    fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  if (box_cols * 4 > 128 || (ld * 4) % 16 || ((uintptr_t)base) % 16)
    return fail(STG_ERR_INVALID_ARG, "make_tmap_f32: box %u cols / ld %llu / base alignment", box_cols,
                (unsigned long long)ld);
  const cuuint64_t dims[2] = {cols, rows};
  const cuuint64_t strides[1] = {ld * 4};
  const cuuint32_t box[2] = {box_cols, box_rows};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(out, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE,
                  atom32 ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B : CU_TENSOR_MAP_SWIZZLE_128B,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(STG_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return STG_OK;
}

stg_status make_tmap_f32_store(CUtensorMap* out, float* base, uint64_t rows, uint64_t cols, uint64_t ld,
                               uint32_t box_cols, uint32_t box_rows) {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess || !p)
      return fail(STG_ERR_CUDA, "cuTensorMapEncodeTiled entry point unavailable");
    fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  if ((box_cols * 4 != 64 && box_cols * 4 != 32) || (ld * 4) % 16 || ((uintptr_t)base) % 16)
    return fail(STG_ERR_INVALID_ARG, "store map: box of %u cols / ld / base alignment", box_cols);
  const cuuint64_t dims[2] = {cols, rows};
  const cuuint64_t strides[1] = {ld * 4};
  const cuuint32_t box[2] = {box_cols, box_rows};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(out, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, base, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  box_cols * 4 == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B,
                  CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(STG_ERR_CUDA, "cuTensorMapEncodeTiled (store) failed (%d)", (int)r);
  return STG_OK;
}

stg_status make_tmap_f32_store3(CUtensorMap* out, float* base, uint64_t planes, uint64_t rows, uint64_t cols,
                                uint32_t box_cols, uint32_t box_rows) {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess || !p)
      return fail(STG_ERR_CUDA, "cuTensorMapEncodeTiled entry point unavailable");
    fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  if ((box_cols * 4 != 64 && box_cols * 4 != 32) || (cols * 4) % 16 || ((uintptr_t)base) % 16)
    return fail(STG_ERR_INVALID_ARG, "store map 3d: box of %u cols / alignment", box_cols);
  const cuuint64_t dims[3] = {cols, rows, planes};
  const cuuint64_t strides[2] = {cols * 4, rows * cols * 4};
  const cuuint32_t box[3] = {box_cols, box_rows, 1};
  const cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(out, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, base, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  box_cols * 4 == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B,
                  CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(STG_ERR_CUDA, "cuTensorMapEncodeTiled (store 3d) failed (%d)", (int)r);
  return STG_OK;
}

}  // namespace stg

extern "C" {

stg_status stg_profile_enable(int32_t on) {
  stg::prof().on = on != 0;
  return STG_OK;
}

stg_status stg_profile_read(int32_t phase, double* total_ms, int64_t* count, int32_t reset) {
  using namespace stg;
  if (phase < 0 || phase >= PH_COUNT) return fail(STG_ERR_OUT_OF_RANGE, "stg_profile_read: phase %d", phase);
  Prof& p = prof();
  std::lock_guard<std::mutex> lk(p.mu);
  for (auto& pr : p.pending[phase]) {
    if (cudaEventSynchronize(pr.second) != cudaSuccess) return fail(STG_ERR_CUDA, "stg_profile_read: event sync");
    float ms = 0.f;
    cudaEventElapsedTime(&ms, pr.first, pr.second);
    p.total[phase] += ms;
    p.count[phase] += 1;
    p.pool.push_back(pr.first);
    p.pool.push_back(pr.second);
  }
  p.pending[phase].clear();
  if (total_ms) *total_ms = p.total[phase];
  if (count) *count = p.count[phase];
  if (reset) { p.total[phase] = 0.0; p.count[phase] = 0; }
  return STG_OK;
}

const char* stg_last_error(void) { return stg::t_err.c_str(); }

int32_t stg_version(void) { return 100; }

int64_t stg_kernel_launch_count(void) { return stg::g_launches.load(); }

stg_status stg_allocator_detach(void) {
  std::lock_guard<std::mutex> lk(stg::g_hook_mu);
  for (auto& e : stg::g_hook_blocks) e.second.free_fn = nullptr;   // freed later: skipped
  stg::g_detached = true;
  stg::g_alloc = nullptr;
  stg::g_free = nullptr;
  stg::g_ctx = nullptr;
  return STG_OK;
}

stg_status stg_set_allocator(stg_alloc_fn alloc, stg_free_fn free_fn, void* ctx) {
  if ((alloc == nullptr) != (free_fn == nullptr))
    return stg::fail(STG_ERR_INVALID_ARG, "stg_set_allocator: alloc and free must both be set or both NULL");
  std::lock_guard<std::mutex> lk(stg::g_hook_mu);
  stg::g_alloc = alloc;
  stg::g_free = free_fn;
  stg::g_ctx = ctx;
  return STG_OK;
}

}  // extern "C"

extern "C" {
// Byte copy on a stream (kind: 0 = device->device, 1 = host->device, 2 = device->host).
// Used by the Python binding to read back borrowed view arrays.
stg_status stg_memcpy(void* dst, const void* src, size_t bytes, int32_t kind, stg_stream_t stream) {
  if (!bytes) return STG_OK;
  if (!dst || !src) return stg::fail(STG_ERR_INVALID_ARG, "stg_memcpy: NULL pointer");
  cudaMemcpyKind k = kind == 1 ? cudaMemcpyHostToDevice : (kind == 2 ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice);
  cudaError_t e = cudaMemcpyAsync(dst, src, bytes, k, (cudaStream_t)stream);
  if (e != cudaSuccess) return stg::fail(STG_ERR_CUDA, "stg_memcpy: %s", cudaGetErrorString(e));
  return STG_OK;
}
}
