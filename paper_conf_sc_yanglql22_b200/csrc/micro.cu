// micro.cu -- characterisation kernels: the DSM's dependent-access latency (Table I,
// L66-80: P2P vs unified memory over 8-128 GB) and the two ceilings the latency-bound prep
// kernels are measured against ("the measured random-32 B-sector rate" for the
// sampler, "L2 atomic throughput" for append-unique).
#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

// One thread chases a dependent chain of 8 B loads through the first span of a shard: the next
// address is the multiply-high of (value * golden) with the slot count -- two dependent IMADs
// (~8 cycles, 4 ns at 1.965 GHz) between a load's return and the next load's issue.
__global__ void dsm_chase_kernel(const uint8_t* base, unsigned long long n_slots, long long accesses,
                                 unsigned long long* sink) {
  unsigned long long x = 0x243F6A8885A308D3ull, acc = 0;
  for (long long i = 0; i < accesses; ++i) {
    const unsigned long long slot = __umul64hi(x, n_slots);  // uniform in [0, n) for a random x
    const unsigned long long v = *reinterpret_cast<const volatile unsigned long long*>(base + slot * 64);
    acc += v;
    x = (v + (unsigned long long)i) * 0x9E3779B97F4A7C15ull;  // the next address depends on the value
  }
  *sink = acc;
}

// Random-read rate: every thread issues RR_ILP independent loads of `width` bytes (8 or 32) at
// random `width`-aligned offsets of [0, span), `rounds` times; addresses come from a Weyl sequence of
// the access index (not from loaded values), so all loads of a round are in flight together -- the
// transaction-bound regime of the sampler's row_ptr / col_idx accesses.
constexpr int RR_ILP = 8;
template <int W>
__global__ void __launch_bounds__(256) random_read_kernel(const uint8_t* base, unsigned long long n_slots, int rounds,
                                                          unsigned long long* sink) {
  const unsigned long long tid = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
  for (int r = 0; r < rounds; ++r) {
    unsigned long long v[RR_ILP];
#pragma unroll
    for (int k = 0; k < RR_ILP; ++k) {
      // Weyl sequence of the access index: one multiply, high bits spread uniformly over the span
      const unsigned long long h = ((unsigned long long)r * gridDim.x * blockDim.x * RR_ILP + tid * RR_ILP + k) *
                                   0x9E3779B97F4A7C15ull;
      const uint8_t* p = base + __umul64hi(h, n_slots) * W;
      if (W == 32) {
        const uint4 a = ld_nc_na_v4(p), b = ld_nc_na_v4(p + 16);
        v[k] = (unsigned long long)(a.x ^ b.w);
      } else {
        v[k] = __ldcg(reinterpret_cast<const unsigned long long*>(p));
      }
    }
#pragma unroll
    for (int k = 0; k < RR_ILP; ++k) acc += v[k];
  }
  if (acc == 0x1234567ull) *sink = acc;  // keeps the loads live; practically never stores
}

// L2 atomic throughput on a table of `slots` 8 B words (sized like an append-unique hash table):
// every thread issues RR_ILP independent 64-bit atomics (op 0: CAS that always fails to swap, i.e.
// a compare of a probe; op 1: CAS claiming the word; op 2: atomicMin) at random slots, `rounds` times.
__global__ void __launch_bounds__(256) atomic_kernel(unsigned long long* table, unsigned long long slots, int op,
                                                     int rounds, unsigned long long* sink) {
  const unsigned long long tid = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
  for (int r = 0; r < rounds; ++r) {
    unsigned long long v[RR_ILP];
#pragma unroll
    for (int k = 0; k < RR_ILP; ++k) {
      const unsigned long long h = ((unsigned long long)r * gridDim.x * blockDim.x * RR_ILP + tid * RR_ILP + k) *
                                   0x9E3779B97F4A7C15ull;
      unsigned long long* w = table + __umul64hi(h, slots);
      if (op == 0)
        v[k] = atomicCAS(w, ~0ull, h);          // never matches (the table holds no ~0): a probe
      else if (op == 1)
        v[k] = atomicCAS(w, *reinterpret_cast<volatile unsigned long long*>(w), h | 1ull);
      else
        v[k] = atomicMin(w, h);
    }
#pragma unroll
    for (int k = 0; k < RR_ILP; ++k) acc += v[k];
  }
  if (acc == 0x1234567ull) *sink = acc;
}

static int full_grid(int per_sm_blocks) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms * per_sm_blocks;
}

}  // namespace wg

using namespace wg;

extern "C" {

wg_status wg_dsm_chase(wg_dsm_t h, int32_t rank, int64_t span_bytes, int64_t accesses, uint64_t* d_sink,
                       wg_stream_t stream) {
  if (!h || rank < 0 || rank >= h->world || accesses < 1 || !d_sink) return fail(WG_ERR_INVALID_ARG, "bad arguments");
  const int64_t shard = h->n_local_of[rank] * h->feat_stride;
  if (span_bytes < 64 || span_bytes > shard) return fail(WG_ERR_INVALID_ARG, "span outside the rank's feature shard");
  cudaSetDevice(h->device);
  dsm_chase_kernel<<<1, 1, 0, (cudaStream_t)stream>>>(h->view.feat[rank], (unsigned long long)(span_bytes / 64),
                                                      (long long)accesses, reinterpret_cast<unsigned long long*>(d_sink));
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(WG_ERR_CUDA, cudaGetErrorString(e));
  return WG_OK;
}

wg_status wg_micro_random_read(const void* d_buf, int64_t span_bytes, int32_t width, int32_t rounds,
                               int32_t blocks_per_sm, uint64_t* d_sink, int64_t* loads_issued, wg_stream_t stream) {
  if (!d_buf || !d_sink || (width != 8 && width != 32) || span_bytes < width || rounds < 1 || blocks_per_sm < 1 ||
      blocks_per_sm > 8)
    return fail(WG_ERR_INVALID_ARG, "bad arguments");
  const int grid = full_grid(blocks_per_sm);
  const unsigned long long slots = (unsigned long long)(span_bytes / width);
  cudaStream_t st = (cudaStream_t)stream;
  if (width == 8)
    random_read_kernel<8><<<grid, 256, 0, st>>>(static_cast<const uint8_t*>(d_buf), slots, rounds,
                                                reinterpret_cast<unsigned long long*>(d_sink));
  else
    random_read_kernel<32><<<grid, 256, 0, st>>>(static_cast<const uint8_t*>(d_buf), slots, rounds,
                                                 reinterpret_cast<unsigned long long*>(d_sink));
  if (loads_issued) *loads_issued = (int64_t)grid * 256 * RR_ILP * rounds;
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? WG_OK : fail(WG_ERR_CUDA, cudaGetErrorString(e));
}

wg_status wg_micro_atomics(uint64_t* d_table, int64_t slots, int32_t op, int32_t rounds, int32_t blocks_per_sm,
                           uint64_t* d_sink, int64_t* ops_issued, wg_stream_t stream) {
  if (!d_table || !d_sink || slots < 1 || op < 0 || op > 2 || rounds < 1 || blocks_per_sm < 1 || blocks_per_sm > 8)
    return fail(WG_ERR_INVALID_ARG, "bad arguments");
  const int grid = full_grid(blocks_per_sm);
  atomic_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(reinterpret_cast<unsigned long long*>(d_table),
                                                         (unsigned long long)slots, op, rounds,
                                                         reinterpret_cast<unsigned long long*>(d_sink));
  if (ops_issued) *ops_issued = (int64_t)grid * 256 * RR_ILP * rounds;
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? WG_OK : fail(WG_ERR_CUDA, cudaGetErrorString(e));
}

}  // extern "C"
