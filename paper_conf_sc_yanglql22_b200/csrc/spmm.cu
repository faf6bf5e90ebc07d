// spmm.cu -- g-SpMM on the sampled sub-graph CSR (section III-C4;
// SURVEY.md 8(f) NEXT #2): the GraphSAGE-mean message passing of Eq. (1) that consumes
// the hot path's outputs (row_ptr, sub_col, X).
//
// forward   Y[t, :] = 1/deg(t) * sum_{e in row t} X[sub_col[e], :]   ("the forward of
//           g-SpMM can be done directly on the CSR matrix", L186)
// backward  dX[c, :] += dY[t, :] / deg(t) for every edge t -> c, computed on the same CSR
//           with atomic adds instead of a transpose (L186); sub-graph nodes sampled exactly
//           once (duplicate count 1, produced by Append Unique) receive a plain store
//           instead of an atomic (L186-192).
// One warp per target row, lanes over 16 B slices of the feature row; fp32 accumulate in
// edge order (deterministic forward).
#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr int SPMM_THREADS = 256;
#ifndef SPMM_UNR_FWD
#define SPMM_UNR_FWD 8  // edges in flight per lane, forward (A/B: 1 0.52, 4 0.66, 8 0.735 of HBM)
#endif
#ifndef SPMM_UNR_BWD
#define SPMM_UNR_BWD 4  // backward (atomics): 1 0.60, 4 0.62, 8 0.575
#endif

__device__ __forceinline__ int64_t count_or_cap(const int64_t* d, int64_t cap) {
  if (!d) return cap;
  const int64_t v = *d;
  return v < 0 ? 0 : (v > cap ? cap : v);
}

// D4 = feature columns / 4 (float4 slices per row)
// Edges whose column lies outside [0, n_x) (e.g. the -1 a relabel writes for an invalid id after
// WG_DEVERR_ID_RANGE) are skipped in both directions: no out-of-bounds read or write.
__global__ void __launch_bounds__(SPMM_THREADS) spmm_mean_fwd_kernel(const int64_t* row_ptr, int64_t cap_rows,
                                                                     const int64_t* d_rows, const int32_t* col,
                                                                     const float4* X, int64_t n_x, int D4, float4* Y) {
  const int64_t n = count_or_cap(d_rows, cap_rows);
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (SPMM_THREADS / 32);
  for (int64_t t = ((int64_t)blockIdx.x * SPMM_THREADS + threadIdx.x) / 32; t < n; t += warps) {
    const int64_t b = row_ptr[t], e = row_ptr[t + 1];
    const float inv = e > b ? 1.0f / (float)(e - b) : 0.0f;
    for (int c = lane; c < D4; c += 32) {
      float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
      // SPMM_UNR_FWD edges at a time: their column ids, then their X slices, are all in flight before the
      // first is added; the rest (fewer than SPMM_UNR_FWD: every row of a fanout-5 hop) in a plain loop the
      // compiler unrolls.  The sum stays in edge order (deterministic).
      int64_t k = b;
      for (; k + SPMM_UNR_FWD <= e; k += SPMM_UNR_FWD) {
        int64_t r[SPMM_UNR_FWD];
        float4 x[SPMM_UNR_FWD];
#pragma unroll
        for (int u = 0; u < SPMM_UNR_FWD; ++u) r[u] = col[k + u];
#pragma unroll
        for (int u = 0; u < SPMM_UNR_FWD; ++u)
          x[u] = (r[u] >= 0 && r[u] < n_x) ? __ldg(&X[r[u] * D4 + c]) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
        for (int u = 0; u < SPMM_UNR_FWD; ++u) {
          if (r[u] < 0 || r[u] >= n_x) continue;
          acc.x += x[u].x;
          acc.y += x[u].y;
          acc.z += x[u].z;
          acc.w += x[u].w;
        }
      }
      for (; k < e; ++k) {
        const int64_t r = col[k];
        if (r < 0 || r >= n_x) continue;
        const float4 x = __ldg(&X[r * D4 + c]);
        acc.x += x.x;
        acc.y += x.y;
        acc.z += x.z;
        acc.w += x.w;
      }
      Y[t * D4 + c] = make_float4(acc.x * inv, acc.y * inv, acc.z * inv, acc.w * inv);
    }
  }
}

__global__ void __launch_bounds__(SPMM_THREADS) spmm_mean_bwd_kernel(const int64_t* row_ptr, int64_t cap_rows,
                                                                     const int64_t* d_rows, const int32_t* col,
                                                                     const int32_t* dup, const float4* dY, int D4,
                                                                     float4* dX, int64_t n_x) {
  const int64_t n = count_or_cap(d_rows, cap_rows);
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (SPMM_THREADS / 32);
  for (int64_t t = ((int64_t)blockIdx.x * SPMM_THREADS + threadIdx.x) / 32; t < n; t += warps) {
    const int64_t b = row_ptr[t], e = row_ptr[t + 1];
    if (e == b) continue;
    const float inv = 1.0f / (float)(e - b);
    for (int c = lane; c < D4; c += 32) {
      float4 g = dY[t * D4 + c];
      g = make_float4(g.x * inv, g.y * inv, g.z * inv, g.w * inv);
      int64_t k = b;
      for (; k + SPMM_UNR_BWD <= e; k += SPMM_UNR_BWD) {  // ids and duplicate counts of SPMM_UNR_BWD edges in flight
        int64_t r[SPMM_UNR_BWD];
        int dc[SPMM_UNR_BWD];
#pragma unroll
        for (int u = 0; u < SPMM_UNR_BWD; ++u) r[u] = col[k + u];
#pragma unroll
        for (int u = 0; u < SPMM_UNR_BWD; ++u) dc[u] = (dup && r[u] >= 0 && r[u] < n_x) ? dup[r[u]] : 0;
#pragma unroll
        for (int u = 0; u < SPMM_UNR_BWD; ++u) {
          if (r[u] < 0 || r[u] >= n_x) continue;
          if (dc[u] == 1)
            dX[r[u] * D4 + c] = g;  // the only contribution this row receives
          else
            atomicAdd(&dX[r[u] * D4 + c], g);
        }
      }
      for (; k < e; ++k) {
        const int64_t r = col[k];
        if (r < 0 || r >= n_x) continue;
        if (dup && dup[r] == 1)
          dX[r * D4 + c] = g;  // the only contribution this row receives
        else
          atomicAdd(&dX[r * D4 + c], g);
      }
    }
  }
}

}  // namespace wg

using namespace wg;

extern "C" {

wg_status wg_spmm_mean_forward(const int64_t* d_row_ptr, int64_t n_rows, const int64_t* d_n_rows,
                               const int32_t* d_sub_col, const float* d_x, int64_t n_x_rows, int64_t dim, float* d_y,
                               wg_stream_t stream) {
  if (n_rows < 0 || n_x_rows < 0 || dim <= 0 || dim % 4 != 0 || (n_rows > 0 && (!d_row_ptr || !d_sub_col || !d_x || !d_y)))
    return fail(WG_ERR_INVALID_ARG, "bad arguments (dim must be a positive multiple of 4)");
  if (n_rows == 0) return WG_OK;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  int64_t blocks = (n_rows * 32 + SPMM_THREADS - 1) / SPMM_THREADS;
  blocks = blocks > (int64_t)sms * 8 ? (int64_t)sms * 8 : blocks;
  spmm_mean_fwd_kernel<<<(unsigned)blocks, SPMM_THREADS, 0, (cudaStream_t)stream>>>(
      d_row_ptr, n_rows, d_n_rows, d_sub_col, reinterpret_cast<const float4*>(d_x), n_x_rows, (int)(dim / 4),
      reinterpret_cast<float4*>(d_y));
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? WG_OK : fail(WG_ERR_CUDA, cudaGetErrorString(e));
}

wg_status wg_spmm_mean_backward(const int64_t* d_row_ptr, int64_t n_rows, const int64_t* d_n_rows,
                                const int32_t* d_sub_col, const int32_t* d_dup_count, const float* d_dy,
                                int64_t dim, float* d_dx, int64_t n_x_rows, wg_stream_t stream) {
  if (n_rows < 0 || n_x_rows < 0 || dim <= 0 || dim % 4 != 0 ||
      (n_rows > 0 && (!d_row_ptr || !d_sub_col || !d_dy || !d_dx)))
    return fail(WG_ERR_INVALID_ARG, "bad arguments (dim must be a positive multiple of 4)");
  cudaStream_t st = (cudaStream_t)stream;
  cudaError_t e = cudaMemsetAsync(d_dx, 0, (size_t)n_x_rows * dim * sizeof(float), st);
  if (e != cudaSuccess) return fail(WG_ERR_CUDA, cudaGetErrorString(e));
  if (n_rows == 0) return WG_OK;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  int64_t blocks = (n_rows * 32 + SPMM_THREADS - 1) / SPMM_THREADS;
  blocks = blocks > (int64_t)sms * 8 ? (int64_t)sms * 8 : blocks;
  spmm_mean_bwd_kernel<<<(unsigned)blocks, SPMM_THREADS, 0, st>>>(
      d_row_ptr, n_rows, d_n_rows, d_sub_col, d_dup_count, reinterpret_cast<const float4*>(d_dy), (int)(dim / 4),
      reinterpret_cast<float4*>(d_dx), n_x_rows);
  e = cudaGetLastError();
  return e == cudaSuccess ? WG_OK : fail(WG_ERR_CUDA, cudaGetErrorString(e));
}

}  // extern "C"
