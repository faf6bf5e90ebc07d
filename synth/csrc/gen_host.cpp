// gen_host.cpp -- host C++ version of synth/graph.py rows() (fixture, not the method):
// regenerates the adjacency rows of arbitrary nodes fast enough for whole
// products/papers-shaped batches.  Same formulas as graph.py; compiled with
// -ffp-contract=off so every double op is a single correctly rounded IEEE op.
// tests/test_synth.py checks it against the numpy generator.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <vector>

static inline uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static inline double unit(uint64_t hv) { return (double)(hv >> 11) * 0x1p-53; }

extern "C" {

// Raw degree of node v (graph.py raw_degree).
int64_t genh_raw_degree(int64_t n, double d_min, int64_t d_max, uint64_t gs, int64_t v) {
  (void)n;
  const uint64_t hv = splitmix64(splitmix64(splitmix64(gs) ^ 0ull) ^ (uint64_t)v);
  const double x = 1.0 - unit(hv);
  const double t = std::sqrt(x);
  const double p = t * std::sqrt(t);
  double val = std::floor(d_min / p);
  if (val > (double)d_max) val = (double)d_max;
  return (int64_t)val;
}

// Rows of nodes vs[0..k): first call with col == NULL to get ptr (sizes), then again
// with col allocated to ptr[k] entries.  Returns 0.
int genh_rows(int64_t n, double d_min, int64_t d_max, uint64_t gs, const int64_t* vs, int64_t k, int64_t* ptr,
              int64_t* col) {
  const uint64_t h1 = splitmix64(splitmix64(gs) ^ 1ull);
  std::vector<int64_t> buf;
  ptr[0] = 0;
  for (int64_t i = 0; i < k; ++i) {
    const int64_t v = vs[i];
    const int64_t d = genh_raw_degree(n, d_min, d_max, gs, v);
    const uint64_t hv = splitmix64(h1 ^ (uint64_t)v);
    buf.resize((size_t)d);
    for (int64_t j = 0; j < d; ++j) {
      const double u = unit(splitmix64(hv ^ (uint64_t)j));
      const double c = (u * u) * std::sqrt(u);
      int64_t w = (int64_t)std::floor((double)n * c);
      if (w > n - 1) w = n - 1;
      buf[(size_t)j] = w;
    }
    std::sort(buf.begin(), buf.end());
    int64_t m = 0;
    int64_t base = ptr[i];
    for (int64_t j = 0; j < d; ++j) {
      if ((j == 0 || buf[(size_t)j] != buf[(size_t)j - 1]) && buf[(size_t)j] != v) {
        if (col) col[base + m] = buf[(size_t)j];
        ++m;
      }
    }
    ptr[i + 1] = base + m;
  }
  return 0;
}

// Feature bits of nodes vs[0..k) (features.py feature_bits), dtype 0 fp32 / 1 fp16 /
// 2 bf16, written densely: out row i = dim elements of elt bytes.
int genh_features(uint64_t feat_seed, const int64_t* vs, int64_t k, int64_t dim, int dtype, void* out) {
  const uint64_t h0 = splitmix64(feat_seed);
  for (int64_t i = 0; i < k; ++i) {
    const uint64_t hv0 = splitmix64(h0 ^ (uint64_t)vs[i]);
    for (int64_t c = 0; c < dim; ++c) {
      const uint64_t hv = splitmix64(hv0 ^ (uint64_t)c);
      if (dtype == 0)
        ((uint32_t*)out)[i * dim + c] = 0x3F800000u | (uint32_t)(hv >> 41);
      else if (dtype == 1)
        ((uint16_t*)out)[i * dim + c] = (uint16_t)(0x3C00u | (uint32_t)(hv >> 54));
      else
        ((uint16_t*)out)[i * dim + c] = (uint16_t)(0x3F80u | (uint32_t)(hv >> 57));
    }
  }
  return 0;
}

}  // extern "C"
