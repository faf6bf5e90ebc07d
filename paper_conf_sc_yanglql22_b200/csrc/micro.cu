// micro.cu -- DSM characterisation (Table I: dependent-access latency
// of P2P vs unified memory over 8-128 GB): one thread chases a dependent chain of 8 B
// loads through the first `span_bytes` of a rank's feature shard (local HBM or a peer
// over NVLink).  Each address is a hash of the value just loaded, so every access waits
// for the previous one and lands on a random 64 B-aligned row of the span.
#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

__global__ void dsm_chase_kernel(const uint8_t* base, unsigned long long n_slots, long long accesses,
                                 unsigned long long* sink) {
  unsigned long long x = 0x9E3779B97F4A7C15ull, acc = 0;
  for (long long i = 0; i < accesses; ++i) {
    const unsigned long long slot = __umul64hi(fmix64(x ^ (unsigned long long)i), n_slots);  // uniform in [0, n)
    const unsigned long long v = *reinterpret_cast<const volatile unsigned long long*>(base + slot * 64);
    acc += v;
    x = v + acc;  // the next address depends on the value just loaded
  }
  *sink = acc;
}

}  // namespace wg

using namespace wg;

extern "C" wg_status wg_dsm_chase(wg_dsm_t h, int32_t rank, int64_t span_bytes, int64_t accesses,
                                  uint64_t* d_sink, wg_stream_t stream) {
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
