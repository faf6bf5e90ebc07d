// gen.cu -- GPU version of the synthetic input generators in synth/graph.py and
// synth/features.py (fixture, not the method).  Same formulas, evaluated with
// explicitly rounded IEEE operations (__dsqrt_rn, __dmul_rn, __ddiv_rn: no FMA
// contraction), so every row equals the numpy generator's row bit for bit
// (checked by tests/test_gpu_synth.py).  Used to fill large DSM shards directly on
// the device (products / papers100M / MAG240M shapes).
#include <climits>
#include <cuda_runtime.h>
#include <stdint.h>

#include <cub/device/device_segmented_sort.cuh>

namespace {

__device__ __forceinline__ unsigned long long splitmix64(unsigned long long x) {
  unsigned long long z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ double unit(unsigned long long hv) {
  return __dmul_rn((double)(hv >> 11), 0x1p-53);  // exact scaling by 2^-53
}

__global__ void raw_degree_kernel(int64_t n, int rank, int world, double d_min, int64_t d_max,
                                  unsigned long long gs, int64_t n_local, int64_t* deg) {
  for (int64_t l = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; l < n_local; l += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long v = (unsigned long long)(rank + l * world);
    const unsigned long long hv = splitmix64(splitmix64(splitmix64(gs) ^ 0ull) ^ v);
    const double x = __dsub_rn(1.0, unit(hv));
    const double t = __dsqrt_rn(x);
    const double p = __dmul_rn(t, __dsqrt_rn(t));
    double val = floor(__ddiv_rn(d_min, p));
    if (val > (double)d_max) val = (double)d_max;
    deg[l] = (int64_t)val;
  }
}

// warp per local row: slot j of row v -> w(v, j)
__global__ void fill_raw_kernel(int64_t n, int rank, int world, unsigned long long gs, int64_t n_local,
                                const int64_t* raw_off, int64_t* raw_col) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x / 32);
  const unsigned long long h1 = splitmix64(splitmix64(gs) ^ 1ull);
  for (int64_t l = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / 32; l < n_local; l += warps) {
    const unsigned long long v = (unsigned long long)(rank + l * world);
    const unsigned long long hv = splitmix64(h1 ^ v);
    const int64_t b = raw_off[l], e = raw_off[l + 1];
    for (int64_t j = b + lane; j < e; j += 32) {
      const double u = unit(splitmix64(hv ^ (unsigned long long)(j - b)));
      const double c = __dmul_rn(__dmul_rn(u, u), __dsqrt_rn(u));
      int64_t w = (int64_t)floor(__dmul_rn((double)n, c));
      if (w > n - 1) w = n - 1;
      raw_col[j] = w;
    }
  }
}

// warp per row over the sorted raw row: keep first of each run, drop self-loops
__global__ void dedup_count_kernel(int rank, int world, int64_t n_local, const int64_t* raw_off,
                                   const int64_t* sorted, int64_t* deg) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x / 32);
  for (int64_t l = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / 32; l < n_local; l += warps) {
    const int64_t v = rank + l * world;
    const int64_t b = raw_off[l], e = raw_off[l + 1];
    int64_t cnt = 0;
    for (int64_t j0 = b; j0 < e; j0 += 32) {
      const int64_t j = j0 + lane;
      bool keep = false;
      if (j < e) {
        const int64_t a = sorted[j];
        keep = (j == b || sorted[j - 1] != a) && a != v;
      }
      cnt += __popc(__ballot_sync(0xffffffffu, keep));
    }
    if (lane == 0) deg[l] = cnt;
  }
}

__global__ void compact_kernel(int rank, int world, int64_t n_local, const int64_t* raw_off, const int64_t* sorted,
                               const int64_t* row_ptr, int64_t* col) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x / 32);
  for (int64_t l = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / 32; l < n_local; l += warps) {
    const int64_t v = rank + l * world;
    const int64_t b = raw_off[l], e = raw_off[l + 1];
    int64_t out = row_ptr[l];
    for (int64_t j0 = b; j0 < e; j0 += 32) {
      const int64_t j = j0 + lane;
      bool keep = false;
      int64_t a = 0;
      if (j < e) {
        a = sorted[j];
        keep = (j == b || sorted[j - 1] != a) && a != v;
      }
      const unsigned m = __ballot_sync(0xffffffffu, keep);
      if (keep) col[out + __popc(m & ((1u << lane) - 1u))] = a;
      out += __popc(m);
    }
  }
}

// Element c of local row l is written at feat + l*stride + c*elt when that byte offset is below
// body_bytes, else at tail + l*tail_pitch + (c*elt - body_bytes) (the DSM's split row layout).
__global__ void features_kernel(unsigned long long feat_seed, int rank, int world, int64_t n_local, int64_t dim,
                                int dtype, int64_t stride, uint8_t* feat, int64_t body_bytes, int64_t tail_pitch,
                                uint8_t* tail) {
  const int64_t total = n_local * dim;
  const unsigned long long h0 = splitmix64(feat_seed);
  const int64_t elt = dtype == 0 ? 4 : 2;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t l = i / dim, c = i - l * dim;
    const unsigned long long v = (unsigned long long)(rank + l * world);
    const unsigned long long hv = splitmix64(splitmix64(h0 ^ v) ^ (unsigned long long)c);
    const int64_t b = c * elt;
    uint8_t* dst = b < body_bytes ? feat + l * stride + b : tail + l * tail_pitch + (b - body_bytes);
    if (dtype == 0)
      *reinterpret_cast<uint32_t*>(dst) = 0x3F800000u | (uint32_t)(hv >> 41);
    else if (dtype == 1)
      *reinterpret_cast<uint16_t*>(dst) = (uint16_t)(0x3C00u | (uint32_t)(hv >> 54));
    else
      *reinterpret_cast<uint16_t*>(dst) = (uint16_t)(0x3F80u | (uint32_t)(hv >> 57));
  }
}

unsigned grid_for(int64_t work, int per_block) {
  int64_t b = (work + per_block - 1) / per_block;
  if (b < 1) b = 1;
  if (b > 148 * 32) b = 148 * 32;
  return (unsigned)b;
}

}  // namespace

extern "C" {

int gen_raw_degree(int64_t n, int rank, int world, double d_min, int64_t d_max, uint64_t gs, int64_t n_local,
                   int64_t* deg, void* stream) {
  raw_degree_kernel<<<grid_for(n_local, 256), 256, 0, (cudaStream_t)stream>>>(n, rank, world, d_min, d_max, gs,
                                                                              n_local, deg);
  return (int)cudaGetLastError();
}

int gen_fill_raw(int64_t n, int rank, int world, uint64_t gs, int64_t n_local, const int64_t* raw_off,
                 int64_t* raw_col, void* stream) {
  fill_raw_kernel<<<grid_for(n_local * 32, 256), 256, 0, (cudaStream_t)stream>>>(n, rank, world, gs, n_local,
                                                                                 raw_off, raw_col);
  return (int)cudaGetLastError();
}

// Sort each segment [off[s] - base, off[s+1] - base) of keys_in into keys_out
// (chunk-relative int32 offsets, num_items < 2^31).  temp may be NULL to query.
int gen_segmented_sort(void* temp, size_t* temp_bytes, const int64_t* keys_in, int64_t* keys_out, int num_items,
                       int num_segments, const int* offsets, void* stream) {
  cudaError_t e = cub::DeviceSegmentedSort::SortKeys(temp, *temp_bytes, keys_in, keys_out, num_items, num_segments,
                                                     offsets, offsets + 1, (cudaStream_t)stream);
  return (int)e;
}

int gen_dedup_count(int rank, int world, int64_t n_local, const int64_t* raw_off, const int64_t* sorted,
                    int64_t* deg, void* stream) {
  dedup_count_kernel<<<grid_for(n_local * 32, 256), 256, 0, (cudaStream_t)stream>>>(rank, world, n_local, raw_off,
                                                                                    sorted, deg);
  return (int)cudaGetLastError();
}

int gen_compact(int rank, int world, int64_t n_local, const int64_t* raw_off, const int64_t* sorted,
                const int64_t* row_ptr, int64_t* col, void* stream) {
  compact_kernel<<<grid_for(n_local * 32, 256), 256, 0, (cudaStream_t)stream>>>(rank, world, n_local, raw_off, sorted,
                                                                                row_ptr, col);
  return (int)cudaGetLastError();
}

int gen_features(uint64_t feat_seed, int rank, int world, int64_t n_local, int64_t dim, int dtype, int64_t stride,
                 uint8_t* feat, int64_t body_bytes, int64_t tail_pitch, uint8_t* tail, void* stream) {
  if (!tail) body_bytes = INT64_MAX;
  features_kernel<<<grid_for(n_local * dim, 256), 256, 0, (cudaStream_t)stream>>>(
      feat_seed, rank, world, n_local, dim, dtype, stride, feat, body_bytes, tail_pitch, tail);
  return (int)cudaGetLastError();
}

}  // extern "C"
