// gather.cu -- global gather over the DSM: "a single gather
// kernel in each GPU"; NVLink/NVSwitch carry the remote reads.
//
// The output X[R][row_bytes] is treated as a flat stream of 16-byte chunks; thread
// t copies chunk c -> (row c / cpr, column c % cpr), cpr = row_bytes / 16.  Adjacent
// threads therefore read adjacent 16 B pieces of the same source row (full 32 B
// sectors, one row = one contiguous burst from local HBM or a peer) and write fully
// coalesced 128 B lines.  Each thread keeps UNROLL independent 16 B loads in flight
// (ld.global.nc.L1::no_allocate: every byte is read exactly once), so a grid of
// ~8 x 256 threads per SM keeps ~0.5 MB in flight chip-wide -- enough to cover
// local-HBM and NVLink latency.  Rows whose size is not a multiple of 16 use the
// same scheme with 4- or 2-byte chunks.
#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr int GATHER_THREADS = 256;
constexpr int GATHER_UNROLL = 4;

// n / d for n < 2^31 via multiply-high (Granlund-Montgomery; d >= 1).
struct FastDiv {
  unsigned d, mul, shift;
  __host__ explicit FastDiv(unsigned d_) : d(d_) {
    shift = 0;
    while ((1u << shift) < d) ++shift;
    unsigned long long m = ((1ull << (32 + shift)) + d - 1) / d;
    mul = (unsigned)m;  // the implicit bit 2^32 is added back in div()
    if (d == 1) { mul = 0; shift = 0; }
  }
  __device__ __forceinline__ unsigned div(unsigned n) const {
    if (d == 1) return n;
    // q = floor((n * (2^32 + mul)) / 2^(32+shift)) computed without overflow
    const unsigned t = __umulhi(n, mul);
    return (unsigned)(((unsigned long long)t + n) >> shift);
  }
};

template <typename V>
__device__ __forceinline__ V ld_feat(const void* p);
template <>
__device__ __forceinline__ uint4 ld_feat<uint4>(const void* p) { return ld_nc_na_v4(p); }
template <>
__device__ __forceinline__ unsigned ld_feat<unsigned>(const void* p) { return ld_nc_na_u32(p); }
template <>
__device__ __forceinline__ unsigned short ld_feat<unsigned short>(const void* p) { return ld_nc_na_u16(p); }

struct GatherArgs {
  ShardView s;
  const int64_t* ids;
  int64_t cap;
  const int64_t* d_n;
  uint8_t* out;
  unsigned* ctrl;
  FastDiv cpr;  // chunks per row
};

template <typename V>
__global__ void __launch_bounds__(GATHER_THREADS) gather_kernel(const GatherArgs a) {
  int64_t n = a.cap;
  if (a.d_n) {
    n = *a.d_n;
    if (n > a.cap || n < 0) {
      if (threadIdx.x == 0 && blockIdx.x == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      n = n < 0 ? 0 : a.cap;
    }
  }
  const unsigned cpr = a.cpr.d;
  const unsigned total = (unsigned)(n * cpr);  // < 2^31 (checked on the host)
  const unsigned stride = gridDim.x * GATHER_THREADS;
  V* __restrict__ out = reinterpret_cast<V*>(a.out);
  for (unsigned c0 = blockIdx.x * GATHER_THREADS + threadIdx.x; c0 < total; c0 += stride * GATHER_UNROLL) {
    V val[GATHER_UNROLL];
    unsigned dst[GATHER_UNROLL];
#pragma unroll
    for (int j = 0; j < GATHER_UNROLL; ++j) {
      const unsigned c = c0 + (unsigned)j * stride;
      dst[j] = c;
      if (c < total) {
        const unsigned row = a.cpr.div(c);
        const unsigned colc = c - row * cpr;
        const int64_t v = a.ids[row];
        if (v >= 0 && v < a.s.n) {
          int o;
          int64_t l;
          owner_local(a.s, v, o, l);
          val[j] = ld_feat<V>(a.s.feat[o] + l * a.s.feat_stride + (int64_t)colc * sizeof(V));
        } else {
          if (colc == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
          val[j] = V{};
        }
      }
    }
#pragma unroll
    for (int j = 0; j < GATHER_UNROLL; ++j)
      if (dst[j] < total) out[dst[j]] = val[j];
  }
}

cudaError_t launch_gather(wg_dsm* h, const int64_t* ids, int64_t cap, const int64_t* d_n, void* out,
                          cudaStream_t st) {
  const int64_t rb = h->row_bytes;
  int vb = (rb % 16 == 0 && ((uintptr_t)out % 16) == 0) ? 16 : (rb % 4 == 0 && ((uintptr_t)out % 4) == 0) ? 4 : 2;
  GatherArgs a{h->view, ids, cap, d_n, static_cast<uint8_t*>(out), h->ws.ctrl, FastDiv((unsigned)(rb / vb))};
  const int64_t total = cap * (rb / vb);
  int64_t blocks = (total + GATHER_THREADS * GATHER_UNROLL - 1) / (GATHER_THREADS * GATHER_UNROLL);
  // one full wave: resident blocks per SM (from the occupancy calculator) x SMs
  static int occ[3] = {0, 0, 0};
  const int which = vb == 16 ? 0 : (vb == 4 ? 1 : 2);
  if (!occ[which]) {
    int nb = 0;
    if (vb == 16)
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<uint4>, GATHER_THREADS, 0);
    else if (vb == 4)
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<unsigned>, GATHER_THREADS, 0);
    else
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<unsigned short>, GATHER_THREADS, 0);
    occ[which] = nb > 0 ? nb : 4;
  }
  const int64_t max_blocks = (int64_t)h->sm_count * occ[which];
  blocks = blocks < 1 ? 1 : (blocks > max_blocks ? max_blocks : blocks);
  if (vb == 16)
    gather_kernel<uint4><<<(unsigned)blocks, GATHER_THREADS, 0, st>>>(a);
  else if (vb == 4)
    gather_kernel<unsigned><<<(unsigned)blocks, GATHER_THREADS, 0, st>>>(a);
  else
    gather_kernel<unsigned short><<<(unsigned)blocks, GATHER_THREADS, 0, st>>>(a);
  return cudaGetLastError();
}

}  // namespace wg
