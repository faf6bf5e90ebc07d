// wg_internal.cuh -- internal definitions shared by the libwg.so translation units.
// (Product code; shares nothing with oracle/.)
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "wg.h"

namespace wg {

// ------------------------------------------------------------------ errors
void set_error(const std::string& msg);
wg_status fail(wg_status s, const std::string& msg);
#define WG_CUDA_TRY(expr)                                                                  \
  do {                                                                                     \
    cudaError_t e_ = (expr);                                                               \
    if (e_ != cudaSuccess)                                                                 \
      return ::wg::fail(WG_ERR_CUDA, std::string(#expr) + ": " + cudaGetErrorString(e_));  \
  } while (0)

// ------------------------------------------------------------------ shard view
// The "memory pointer table": one base pointer per rank, passed
// BY VALUE as a kernel parameter (constant bank; no global load per access).
struct ShardView {
  const int64_t* row_ptr[WG_MAX_WORLD];
  const void* col[WG_MAX_WORLD];      // col_idx entries: int64, or uint32 with WG_DSM_COL32
  const uint8_t* feat[WG_MAX_WORLD];  // feature rows (their first body_bytes bytes), pitch feat_stride
  const uint8_t* tail[WG_MAX_WORLD];  // split layout: bytes [body_bytes, row_bytes) of every row, pitch tail_pitch
  int64_t n;            // num_nodes
  int64_t feat_stride;  // bytes between feature rows in a shard (multiple of 16)
  int64_t tail_pitch;   // 0 = no split: whole rows live in feat
  int64_t body_bytes;   // bytes of a row stored in feat (= row bytes when not split)
  int32_t world;
  int32_t log2w;        // log2(world) if world is a power of two, else -1
  int32_t csr_rank;     // WG_DSM_CSR_REPLICATED: this rank, whose slab holds the whole CSR; -1: CSR row-sharded
  int32_t col32;        // WG_DSM_COL32: col_idx entries are uint32
};

// Neighbour id at entry e of rank o's col_idx shard (8 B, or 4 B with WG_DSM_COL32).
template <bool COL32>
__device__ __forceinline__ int64_t ld_col(const ShardView& s, int o, int64_t e) {
  if (COL32) return (int64_t)static_cast<const uint32_t*>(s.col[o])[e];
  return static_cast<const int64_t*>(s.col[o])[e];
}

// Owner rank and local row of node v in the feature table (hash partition o(v) = v mod W,
// l(v) = v div W; A11).
__device__ __forceinline__ void owner_local(const ShardView& s, int64_t v, int& o, int64_t& l) {
  if (s.log2w >= 0) {
    o = (int)(v & (int64_t)(s.world - 1));
    l = v >> s.log2w;
  } else {
    o = (int)(v % s.world);
    l = v / s.world;
  }
}
// Where v's CSR row lives: with the paper's placement next to its feature row ("edges are stored
// together with the source node", L110); with WG_DSM_CSR_REPLICATED in this rank's own full copy.
__device__ __forceinline__ void csr_owner_local(const ShardView& s, int64_t v, int& o, int64_t& l) {
  if (s.csr_rank >= 0) {
    o = s.csr_rank;
    l = v;
  } else {
    owner_local(s, v, o, l);
  }
}

// ------------------------------------------------------------------ workspace
// Device-side scratch owned by the handle.  Everything that must be "fresh" per
// call is either epoch-tagged (hash table) or reset by the last block of the
// kernel that used it (scan status + done counters), so no memset is needed per
// call and every op is CUDA-graph capturable.
struct __align__(16) HashSlot {
  unsigned long long key;  // (epoch << 40) | node id
  unsigned long long val;  // ((EPOCH_MAX - epoch) << 40) | first position
};
struct Workspace {
  HashSlot* hslots = nullptr;            // [hcap] append-unique hash table (hash.cuh)
  unsigned long long* hslots2 = nullptr;  // compact format: [hcap] 8 B words, the odd epoch cycles' table
  int64_t hcap = 0;                      // slots (a multiple of 8, < 2^31); each call uses a prefix
  int compact = 0;                       // 8 B slots {epoch8, key28, pos28} (hash.cuh), else 16 B slots
  // direct table (hash.cuh, graphs small enough that a word per NODE beats a hashed slot per key): two
  // uint32 arrays of num_nodes words {255 - compact_epoch, first position}; the epochs of 255-epoch cycle c
  // use dtab[c & 1] (hash.cuh);
  // the fused hop's sampler inserts into it, so a hop has no insert pass and no slot_of round trip
  int direct = 0;
  unsigned* dtab[2] = {nullptr, nullptr};
  int pad32 = 0;                         // padded sampler slots hold uint32 ids (num_nodes < 2^32)
  unsigned long long* status_sample = nullptr;  // decoupled look-back tile status
  unsigned long long* status_unique = nullptr;
  int64_t status_cap = 0;
  int32_t* excl[4] = {nullptr, nullptr, nullptr, nullptr};  // ring of [max_keys] exclusive scans of
                                         // first-occurrence flags (a relabel on a side stream may
                                         // still read one while the next hops write the others)
  int32_t* slot_of = nullptr;            // [max_keys] hash slot of every position of the current call
  int64_t* nbrs_pad = nullptr;           // [max_keys] sampler output, padded slots k*M + i
  int32_t* pos_pad = nullptr;            // [max_keys] adjacency positions of the padded slots
  int32_t* cnt = nullptr;                // [max_keys] per-target sample counts min(M, deg)
  unsigned* ctrl = nullptr;              // [16] control words (see CTRL_*)
  int64_t max_keys = 0;
};
enum { CTRL_ERR = 0, CTRL_EPOCH = 1, CTRL_DONE_SAMPLE = 2, CTRL_DONE_UNIQUE = 3, CTRL_WORDS = 16 };
constexpr unsigned EPOCH_MAX = (1u << 23) - 1;
// compact hash table (8 B slots): epochs 1..255 cycle; the table is cleared when a cycle restarts
constexpr unsigned CEPOCHS = 255;
__host__ __device__ inline unsigned compact_epoch(unsigned e) { return e % CEPOCHS + 1u; }
// Direct table eligibility: positions fit its 24-bit field and the two tables stay small (products:
// 2 x 9.8 MB).  Above that (papers100M: 2 x 444 MB, whose 700k random words per hop would each cost a
// line) the hashed formats touch fewer lines.  WG_DSM_HASHED forces the hashed formats.
constexpr int DPOS_BITS = 24;
#ifndef WG_DIRECT_MAX_NODES
#define WG_DIRECT_MAX_NODES (int64_t(1) << 24)
#endif
constexpr int EXCL_RING = 4;
// Hash-table sizing (measured on B200): a call uses a prefix of
// HASH_FACTOR x its own key bound slots (at least HASH_MIN_SLOTS), so small hops touch few lines.
#ifndef WG_HASH_FACTOR_PCT
#define WG_HASH_FACTOR_PCT 200
#endif
#ifndef WG_HASH_MIN_LOG2
#define WG_HASH_MIN_LOG2 20
#endif
constexpr double HASH_FACTOR = WG_HASH_FACTOR_PCT / 100.0;
constexpr int64_t HASH_MIN_SLOTS = int64_t(1) << WG_HASH_MIN_LOG2;
constexpr int64_t HASH_MAX_SLOTS = (int64_t(1) << 31) - 8;  // slot indices are stored as int32 (slot_of)

}  // namespace wg

// ------------------------------------------------------------------ host handle
struct wg_dsm {
  int rank = 0, world = 1, device = 0;
  int64_t n = 0, n_local = 0, e_local = 0, feat_dim = 0, elt = 4, row_bytes = 0, feat_stride = 0;
  int64_t body_bytes = 0, tail_pitch = 0;  // split feature layout (see wg_dsm_feat_layout)
  int64_t n_local_of[WG_MAX_WORLD] = {0};
  int64_t e_local_of[WG_MAX_WORLD] = {0};
  void* slab = nullptr;                 // this rank's allocation
  size_t slab_bytes = 0;
  void* peer_base[WG_MAX_WORLD] = {nullptr};
  bool peer_opened[WG_MAX_WORLD] = {false};  // opened through cudaIpcOpenMemHandle
  wg::ShardView view{};
  wg::Workspace ws{};
  wg_allgather_fn allgather = nullptr;
  void* ctx = nullptr;
  int sm_count = 148;
  int excl_next = 0;                    // next excl ring slot (host-side, per call)
  cudaEvent_t fork_event = nullptr;     // relabel fork onto a side stream
  wg_dsm* parent = nullptr;             // set for a workspace fork (wg_dsm_fork): shards are the parent's
  int live_forks = 0;                   // forks of this handle not yet destroyed
  int gather_bps = 0;                   // wg_dsm_set_gather_occupancy (0 = occupancy maximum)
  uint32_t flags = 0;                   // wg_dsm_desc.flags
  // wg_dsm_set_stage_events: events recorded after each kernel of an op (diagnostics, eager launches)
  cudaEvent_t stage_ev[8] = {nullptr};
  int stage_n = 0, stage_i = 0;
};

namespace wg {
// Programmatic dependent launch (sm_90+): kernels of one op chain are launched with
// ProgrammaticStreamSerialization, start their blocks while the previous kernel drains and
// wait for its results with griddepcontrol.wait (pdl_wait) before touching memory
// (correctness never depends on it: a kernel launched without the attribute waits anyway).
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                              Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

// Slots of the append-unique hash-table prefix a call with this key bound uses: HASH_FACTOR x the
// bound (a multiple of 8 slots = one 128 B line of compact words), at least HASH_MIN_SLOTS.
inline int64_t table_prefix(const wg_dsm* h, int64_t key_bound) {
  int64_t hc = (int64_t)(HASH_FACTOR * (double)key_bound) + 8;
  hc = hc < HASH_MIN_SLOTS ? HASH_MIN_SLOTS : hc;
  hc = (hc + 7) / 8 * 8;
  return hc < h->ws.hcap ? hc : h->ws.hcap;
}

// Record the next stage event (if any are set) on st, after the kernel just enqueued there.
inline void stage_mark(wg_dsm* h, cudaStream_t st) {
  if (h->stage_i < h->stage_n) cudaEventRecord(h->stage_ev[h->stage_i++], st);
}

// padded sampler slots: int64 ids, or uint32 ids when every id fits (half the bytes)
__device__ __forceinline__ void st_pad(int64_t* p, int pad32, int64_t i, int64_t v) {
  if (pad32)
    reinterpret_cast<uint32_t*>(p)[i] = (uint32_t)v;
  else
    p[i] = v;
}
__device__ __forceinline__ int64_t ld_pad(const int64_t* p, int pad32, int64_t i) {
  return pad32 ? (int64_t)reinterpret_cast<const uint32_t*>(p)[i] : p[i];
}

// Whether the fused hop's sampler inserts the keys itself (the direct key table: no insert pass).
bool hop_inserts_in_sampler(const wg_dsm* h);

// launchers (stream-ordered); arguments already validated by the ABI layer
cudaError_t launch_sample(wg_dsm* h, const int64_t* targets, int64_t cap, const int64_t* d_n, int fanout,
                          uint64_t seed, const uint64_t* d_seed, int hop, int64_t* out_row_ptr,
                          int64_t* out_nbrs, int32_t* out_pos, int64_t* d_num_edges, cudaStream_t st);
cudaError_t launch_append_unique(wg_dsm* h, const int64_t* T, int64_t capT, const int64_t* d_nT,
                                 const int64_t* nbrs, int64_t capE, const int64_t* d_nE, int64_t* U,
                                 int64_t* d_nU, int32_t* sub_col, int32_t* dup, cudaStream_t st);
cudaError_t launch_hop(wg_dsm* h, const int64_t* T, int64_t capT, const int64_t* d_nT, int fanout, uint64_t seed,
                       const uint64_t* d_seed, int hop, int64_t* out_row_ptr, int64_t* out_nbrs, int32_t* out_pos,
                       int64_t* d_num_edges, int64_t* U, int64_t* d_nU, int32_t* sub_col, int32_t* dup,
                       cudaStream_t st, cudaStream_t side);
cudaError_t launch_gather(wg_dsm* h, const int64_t* ids, int64_t cap, const int64_t* d_n, const int64_t* d_begin,
                          void* out, int64_t out_pitch, cudaStream_t st);
}  // namespace wg
