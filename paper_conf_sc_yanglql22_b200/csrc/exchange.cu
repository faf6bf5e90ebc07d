// exchange.cu -- helper kernels of the distributed-memory (NCCL) global gather, the
// comparison baseline of PAPER.md L178-180 (Fig. 4 left, Fig. 10):
//   step 1  bucket the requested ids by home GPU           -> wg_bucket_by_owner
//   step 2  send counts, then ids (all-to-all)              -> caller (NCCL via torch.distributed)
//   step 3  local gather on every GPU                       -> wg_gather (own shard only)
//   step 4  send the features back (all-to-all)            -> caller
//   step 5  local reorder into input order                  -> wg_rows_permute
// The product path (wg_gather) replaces all five with one kernel of P2P loads (L182).
#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr int EX_THREADS = 256;

__global__ void __launch_bounds__(EX_THREADS) bucket_count_kernel(ShardView s, const int64_t* ids, int64_t cap,
                                                                  const int64_t* d_n, unsigned long long* counts,
                                                                  unsigned* ctrl) {
  __shared__ unsigned long long sc[WG_MAX_WORLD];
  if (threadIdx.x < WG_MAX_WORLD) sc[threadIdx.x] = 0;
  __syncthreads();
  int64_t n = cap;
  if (d_n) n = min(max(*d_n, (int64_t)0), cap);
  for (int64_t i = (int64_t)blockIdx.x * EX_THREADS + threadIdx.x; i < n; i += (int64_t)gridDim.x * EX_THREADS) {
    const int64_t v = ids[i];
    if (v < 0 || v >= s.n) {
      latch_error(&ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
      continue;
    }
    int o;
    int64_t l;
    owner_local(s, v, o, l);
    atomicAdd(&sc[o], 1ull);
  }
  __syncthreads();
  if (threadIdx.x < s.world && sc[threadIdx.x]) atomicAdd(&counts[threadIdx.x], sc[threadIdx.x]);
}

// counts[] complete; cursors[] zeroed.  out[offset(o) + slot] = v, perm[i] = that position.
__global__ void __launch_bounds__(EX_THREADS) bucket_scatter_kernel(ShardView s, const int64_t* ids, int64_t cap,
                                                                    const int64_t* d_n,
                                                                    const unsigned long long* counts,
                                                                    unsigned long long* cursors, int64_t* out,
                                                                    int64_t* perm) {
  __shared__ unsigned long long off[WG_MAX_WORLD];
  if (threadIdx.x == 0) {
    unsigned long long run = 0;
    for (int o = 0; o < s.world; ++o) {
      off[o] = run;
      run += counts[o];
    }
  }
  __syncthreads();
  int64_t n = cap;
  if (d_n) n = min(max(*d_n, (int64_t)0), cap);
  for (int64_t i = (int64_t)blockIdx.x * EX_THREADS + threadIdx.x; i < n; i += (int64_t)gridDim.x * EX_THREADS) {
    const int64_t v = ids[i];
    if (v < 0 || v >= s.n) {
      perm[i] = -1;
      continue;
    }
    int o;
    int64_t l;
    owner_local(s, v, o, l);
    const int64_t pos = (int64_t)(off[o] + atomicAdd(&cursors[o], 1ull));
    out[pos] = v;
    perm[i] = pos;
  }
}

// dst[i][:] = src[perm[i]][:] (perm[i] < 0 -> zeros), 16 B chunks when possible
template <typename V>
__global__ void __launch_bounds__(EX_THREADS) rows_permute_kernel(const uint8_t* src, uint8_t* dst, const int64_t* perm,
                                                                  int64_t n, int64_t row_bytes) {
  const int64_t cpr = row_bytes / (int64_t)sizeof(V);
  const int64_t total = n * cpr;
  for (int64_t c = (int64_t)blockIdx.x * EX_THREADS + threadIdx.x; c < total; c += (int64_t)gridDim.x * EX_THREADS) {
    const int64_t row = c / cpr, k = c - row * cpr;
    const int64_t p = perm[row];
    V v{};
    if (p >= 0) v = reinterpret_cast<const V*>(src + p * row_bytes)[k];
    reinterpret_cast<V*>(dst + row * row_bytes)[k] = v;
  }
}

}  // namespace wg

using namespace wg;

extern "C" {

wg_status wg_bucket_by_owner(wg_dsm_t h, const int64_t* d_ids, int64_t n_ids, const int64_t* d_n_ids,
                             int64_t* d_counts, int64_t* d_bucketed_ids, int64_t* d_perm, wg_stream_t stream) {
  if (!h || n_ids < 0 || !d_counts || (n_ids > 0 && (!d_ids || !d_bucketed_ids || !d_perm)))
    return fail(WG_ERR_INVALID_ARG, "bad arguments");
  cudaSetDevice(h->device);
  cudaStream_t st = (cudaStream_t)stream;
  // counts and cursors (W each) live back to back in the caller's d_counts[2 * W]
  WG_CUDA_TRY(cudaMemsetAsync(d_counts, 0, 2 * sizeof(int64_t) * h->world, st));
  if (n_ids == 0) return WG_OK;
  int64_t blocks = (n_ids + EX_THREADS - 1) / EX_THREADS;
  blocks = blocks > (int64_t)h->sm_count * 8 ? (int64_t)h->sm_count * 8 : blocks;
  auto* cnt = reinterpret_cast<unsigned long long*>(d_counts);
  bucket_count_kernel<<<(unsigned)blocks, EX_THREADS, 0, st>>>(h->view, d_ids, n_ids, d_n_ids, cnt, h->ws.ctrl);
  bucket_scatter_kernel<<<(unsigned)blocks, EX_THREADS, 0, st>>>(h->view, d_ids, n_ids, d_n_ids, cnt,
                                                                 cnt + h->world, d_bucketed_ids, d_perm);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? WG_OK : fail(WG_ERR_CUDA, cudaGetErrorString(e));
}

wg_status wg_rows_permute(const void* d_src, void* d_dst, const int64_t* d_perm, int64_t n, int64_t row_bytes,
                          wg_stream_t stream) {
  if (n < 0 || row_bytes <= 0 || (n > 0 && (!d_src || !d_dst || !d_perm))) return fail(WG_ERR_INVALID_ARG, "bad arguments");
  if (n == 0) return WG_OK;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaStream_t st = (cudaStream_t)stream;
  const bool v16 = row_bytes % 16 == 0 && (uintptr_t)d_src % 16 == 0 && (uintptr_t)d_dst % 16 == 0;
  const int64_t vb = v16 ? 16 : 1;
  int64_t blocks = (n * (row_bytes / vb) + EX_THREADS - 1) / EX_THREADS;
  blocks = blocks > (int64_t)sms * 16 ? (int64_t)sms * 16 : blocks;
  if (v16)
    rows_permute_kernel<uint4><<<(unsigned)blocks, EX_THREADS, 0, st>>>(
        static_cast<const uint8_t*>(d_src), static_cast<uint8_t*>(d_dst), d_perm, n, row_bytes);
  else
    rows_permute_kernel<uint8_t><<<(unsigned)blocks, EX_THREADS, 0, st>>>(
        static_cast<const uint8_t*>(d_src), static_cast<uint8_t*>(d_dst), d_perm, n, row_bytes);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? WG_OK : fail(WG_ERR_CUDA, cudaGetErrorString(e));
}

}  // extern "C"
