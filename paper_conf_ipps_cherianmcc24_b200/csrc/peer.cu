// peer.cu — sharded mode over peer memory (SURVEY §8(e) "sharded mode";
// north_star: destination-row blocks with the source rows exchanged over NVLink
// each timestep).  One process per GPU; every rank owns the rows of its block
// of a row matrix in a CUDA-IPC-visible allocation, and the other ranks read
// those rows with plain (NVLink peer) loads:
//   * stg_gcn_aggregate_peer (aggregate.cu) gathers neighbour rows straight
//     from their owners' blocks — the all-gather fused into the aggregation;
//   * stg_allgather_rows materialises the whole matrix (explicit all-gather);
//   * stg_reduce_scatter_rows sums every rank's partial rows of the caller's
//     block in rank order (the backward's partial dP, deterministic).
// No NCCL on the data path; cross-rank ordering is the caller's (include/stg.h).
#include <climits>
#include <cstring>

#include "graph.cuh"

namespace stg {
namespace {

struct RowTable {
  const float* base[STG_MAX_PEERS];   // block k shifted back by bounds[k] rows
  int32_t bnd[STG_MAX_PEERS];         // first row of block k (INT_MAX past the last)
};

__device__ __forceinline__ const float* owner_row(const RowTable& t, int32_t u, int64_t ld) {
  int k = 0;
#pragma unroll
  for (int i = 1; i < STG_MAX_PEERS; ++i) k += (u >= t.bnd[i]) ? 1 : 0;
  return t.base[k] + (int64_t)u * ld;
}

// full[u, :] = owner block row u: one warp per row, float4 lanes (W % 4 == 0)
// or scalar lanes; rows grid-strided.
__global__ void __launch_bounds__(256) k_allgather_rows(const RowTable t, int64_t ld, int32_t V, int32_t W,
                                                        float* __restrict__ full, int64_t ldf, int vec4) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; u < V; u += nw) {
    const float* src = owner_row(t, (int32_t)u, ld);
    float* dst = full + u * ldf;
    if (vec4) {
      for (int c = lane; c < (W >> 2); c += 32)
        __stcs(reinterpret_cast<float4*>(dst) + c, __ldcs(reinterpret_cast<const float4*>(src) + c));
    } else {
      for (int c = lane; c < W; c += 32) dst[c] = src[c];
    }
  }
}

// out[i, :] = Σ_q part_q[rb + i, :] in rank order q = 0..world-1
__global__ void __launch_bounds__(256) k_reduce_scatter_rows(const RowTable t, int32_t world, int64_t ld,
                                                             int32_t rb, int32_t R, int32_t W,
                                                             float* __restrict__ out, int64_t ldo, int vec4) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < R; i += nw) {
    const int64_t row = (int64_t)(rb + i) * ld;
    float* dst = out + i * ldo;
    if (vec4) {
      for (int c = lane; c < (W >> 2); c += 32) {
        float4 acc = __ldcs(reinterpret_cast<const float4*>(t.base[0] + row) + c);
        for (int q = 1; q < world; ++q) {
          const float4 v = __ldcs(reinterpret_cast<const float4*>(t.base[q] + row) + c);
          acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
        }
        __stcs(reinterpret_cast<float4*>(dst) + c, acc);
      }
    } else {
      for (int c = lane; c < W; c += 32) {
        float acc = t.base[0][row + c];
        for (int q = 1; q < world; ++q) acc += t.base[q][row + c];
        dst[c] = acc;
      }
    }
  }
}

unsigned rows_grid(int64_t rows) {
  const int64_t warps = rows > 0 ? rows : 1;
  return (unsigned)std::min<int64_t>(ceil_div(warps, 8), (int64_t)num_sms() * 8);
}

}  // namespace
}  // namespace stg

extern "C" {

stg_status stg_peer_alloc(int64_t bytes, void** dptr, stg_ipc_handle* handle) {
  static_assert(sizeof(cudaIpcMemHandle_t) <= sizeof(stg_ipc_handle), "IPC handle size");
  if (bytes < 1 || !dptr || !handle) return stg::fail(STG_ERR_INVALID_ARG, "stg_peer_alloc: bad arguments");
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, (size_t)bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return stg::fail(STG_ERR_NO_MEMORY, "stg_peer_alloc: cudaMalloc(%lld): %s", (long long)bytes,
                     cudaGetErrorString(e));
  }
  cudaMemset(p, 0, (size_t)bytes);                 // zero-initialised (exchange counters start at 0)
  cudaIpcMemHandle_t h;
  e = cudaIpcGetMemHandle(&h, p);
  if (e != cudaSuccess) {
    cudaFree(p);
    return stg::cuda_fail(e, "cudaIpcGetMemHandle", __FILE__, __LINE__);
  }
  memset(handle, 0, sizeof(*handle));
  memcpy(handle->reserved, &h, sizeof(h));
  *dptr = p;
  return STG_OK;
}

stg_status stg_peer_free(void* dptr) {
  if (!dptr) return STG_OK;
  STG_CUDA(cudaFree(dptr));
  return STG_OK;
}

stg_status stg_peer_open(const stg_ipc_handle* handle, void** dptr) {
  if (!handle || !dptr) return stg::fail(STG_ERR_INVALID_ARG, "stg_peer_open: bad arguments");
  cudaIpcMemHandle_t h;
  memcpy(&h, handle->reserved, sizeof(h));
  void* p = nullptr;
  STG_CUDA(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
  *dptr = p;
  return STG_OK;
}

stg_status stg_peer_close(void* dptr) {
  if (!dptr) return STG_OK;
  STG_CUDA(cudaIpcCloseMemHandle(dptr));
  return STG_OK;
}

static stg_status make_table(const stg_peer_rows* t, int32_t W, stg::RowTable* out, int32_t* V) {
  using stg::fail;
  if (!t || t->world < 1 || t->world > STG_MAX_PEERS || !t->bounds || !t->blocks)
    return fail(STG_ERR_INVALID_ARG, "peer rows: world must be in [1,%d] with bounds and blocks", STG_MAX_PEERS);
  if (W < 1 || t->ld < W) return fail(STG_ERR_INVALID_ARG, "peer rows: need 1 <= W <= ld");
  if (t->bounds[0] != 0) return fail(STG_ERR_INVALID_ARG, "peer rows: bounds[0] must be 0");
  for (int k = 0; k < STG_MAX_PEERS; ++k) {
    out->base[k] = nullptr;
    out->bnd[k] = k == 0 ? 0 : INT_MAX;
  }
  for (int k = 0; k < t->world; ++k) {
    const int32_t b = t->bounds[k], e = t->bounds[k + 1];
    if (e < b) return fail(STG_ERR_INVALID_ARG, "peer rows: bounds decrease at %d", k);
    if (e > b && !t->blocks[k]) return fail(STG_ERR_INVALID_ARG, "peer rows: block %d is NULL", k);
    if (k > 0) out->bnd[k] = b;
    out->base[k] = reinterpret_cast<const float*>(reinterpret_cast<uintptr_t>(t->blocks[k]) -
                                                  (uintptr_t)((int64_t)b * t->ld * 4));
  }
  *V = t->bounds[t->world];
  return STG_OK;
}

stg_status stg_allgather_rows(const stg_peer_rows* src, int32_t W, float* full, int64_t ldf, stg_stream_t stream) {
  stg::RowTable tab;
  int32_t V = 0;
  STG_TRY(make_table(src, W, &tab, &V));
  if (!full || ldf < W) return stg::fail(STG_ERR_INVALID_ARG, "stg_allgather_rows: bad output");
  if (V == 0) return STG_OK;
  bool vec4 = W % 4 == 0 && src->ld % 4 == 0 && ldf % 4 == 0 && (uintptr_t)full % 16 == 0;
  for (int k = 0; k < src->world; ++k) vec4 = vec4 && (uintptr_t)src->blocks[k] % 16 == 0;
  stg::k_allgather_rows<<<stg::rows_grid(V), 256, 0, (cudaStream_t)stream>>>(tab, src->ld, V, W, full, ldf,
                                                                            vec4 ? 1 : 0);
  stg::count_launch();
  return stg::check_launch("stg_allgather_rows");
}

stg_status stg_reduce_scatter_rows(int32_t world, const int32_t* bounds, const float* const* partials, int64_t ld,
                                   int32_t rank, int32_t W, float* out, int64_t ldout, stg_stream_t stream) {
  using stg::fail;
  if (world < 1 || world > STG_MAX_PEERS || !bounds || !partials || rank < 0 || rank >= world)
    return fail(STG_ERR_INVALID_ARG, "stg_reduce_scatter_rows: bad world/rank");
  const int32_t rb = bounds[rank], R = bounds[rank + 1] - rb;
  if (rb < 0 || R < 0) return fail(STG_ERR_INVALID_ARG, "stg_reduce_scatter_rows: bad bounds");
  if (W < 1 || ld < W || ldout < W) return fail(STG_ERR_INVALID_ARG, "stg_reduce_scatter_rows: bad shapes");
  if (R == 0) return STG_OK;                       // an empty block
  if (!out) return fail(STG_ERR_INVALID_ARG, "stg_reduce_scatter_rows: NULL output");
  stg::RowTable tab;
  bool vec4 = W % 4 == 0 && ld % 4 == 0 && ldout % 4 == 0 && (uintptr_t)out % 16 == 0;
  for (int q = 0; q < STG_MAX_PEERS; ++q) {
    tab.base[q] = q < world ? partials[q] : nullptr;
    tab.bnd[q] = 0;
    if (q < world) {
      if (!partials[q]) return fail(STG_ERR_INVALID_ARG, "stg_reduce_scatter_rows: partials[%d] is NULL", q);
      vec4 = vec4 && (uintptr_t)partials[q] % 16 == 0;
    }
  }
  stg::k_reduce_scatter_rows<<<stg::rows_grid(R), 256, 0, (cudaStream_t)stream>>>(tab, world, ld, rb, R, W, out,
                                                                                 ldout, vec4 ? 1 : 0);
  stg::count_launch();
  return stg::check_launch("stg_reduce_scatter_rows");
}

}  // extern "C"
