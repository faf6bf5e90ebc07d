// dsm.cu -- the multi-GPU distributed shared memory (section III-B)
// and the C-ABI entry points of include/wg.h.
//
// Each rank allocates ONE slab on its GPU holding its shards
//   [ row_ptr int64[n_local+1] | col_idx int64[e_local] | feat[n_local][stride] | tail[n_local][tail_pitch] ]
// The tail region exists only for the split feature layout (feat_geometry below).
// (256-byte aligned sub-offsets; cudaMalloc of >= 2 MB uses 2 MB pages, so TLB reach
// covers the shards with few entries), exports a CUDA IPC handle, allgathers a fixed
// record {pid, device pointer, IPC handle, geometry} through the caller's callback
// (L100), opens every peer's handle with cudaIpcOpenMemHandle (L100-106) -- a peer
// in the SAME process (in-process virtual ranks) is used directly -- and keeps the
// per-rank base pointers as the "memory pointer table" (L106), which travels to
// every kernel by value inside ShardView.
#include <unistd.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

static thread_local std::string g_last_error;

void set_error(const std::string& msg) { g_last_error = msg; }
wg_status fail(wg_status s, const std::string& msg) {
  g_last_error = msg;
  return s;
}

static int64_t round_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

static int64_t local_rows(int64_t n, int rank, int world) {
  return n > rank ? (n - rank + world - 1) / world : 0;
}

// Feature-row layout.  The B200 L2 fills whole 128 B lines on a miss (measured:
// profiles/r01/fetch_granularity.md -- a random 32 B row costs 128 B of DRAM, a 400 B row at
// a 64 B-aligned pitch costs 4 lines = 512 B, cudaLimitMaxL2FetchGranularity has no effect).
// A row whose size is not a multiple of 128 B (but a multiple of 16 B, > 128 B) is therefore
// SPLIT: its first floor(row/128)*128 bytes (the body) live in the feature shard at a pitch of
// exactly that many bytes, so a body is whole lines and costs no over-fetch; the remaining
// row % 128 bytes (the tail) live densely in a separate tail region (pitch = tail bytes), small
// enough to stay in L2 (products-shaped: 2.45M x 16 B = 39 MB) and read with an evict_last hint.
// Otherwise rows stay whole at a pitch rounded up to 64 B.  WG_DSM_WHOLE_ROWS disables the split.
static void feat_geometry(int64_t row_bytes, bool split, int64_t* body, int64_t* stride, int64_t* tail_pitch) {
  const int64_t t = row_bytes % 128;
  if (split && row_bytes > 128 && t != 0 && t % 16 == 0) {
    *body = row_bytes - t;
    *stride = *body;
    *tail_pitch = t;
  } else {
    *body = row_bytes;
    *stride = round_up(row_bytes, 64);
    *tail_pitch = 0;
  }
}

struct PeerRecord {
  int64_t pid;
  uint64_t dev_ptr;
  int64_t slab_bytes;
  int64_t n_local;
  int64_t e_local;
  int64_t off_col;
  int64_t off_feat;
  int64_t off_tail;
  int64_t num_nodes;
  int64_t feat_stride;
  int64_t tail_pitch;
  int32_t world;
  int32_t rank;
  uint32_t flags;
  int32_t pad_;
  char uuid[16];  // the rank's GPU (cudaDeviceProp::uuid): ordinals differ between processes
  cudaIpcMemHandle_t handle;
};

static wg_status barrier(wg_dsm* h) {
  if (h->world == 1) return WG_OK;
  if (h->allgather(nullptr, nullptr, 0, h->ctx) != 0) return fail(WG_ERR_COLLECTIVE, "barrier: allgather callback failed");
  return WG_OK;
}

static void free_workspace(wg_dsm* h) {
  Workspace& w = h->ws;
  cudaFree(w.hslots);
  cudaFree(w.hslots2);
  cudaFree(w.dtab[0]);
  cudaFree(w.dtab[1]);
  cudaFree(w.status_sample);
  cudaFree(w.status_unique);
  for (int k = 0; k < EXCL_RING; ++k) cudaFree(w.excl[k]);
  cudaFree(w.slot_of);
  cudaFree(w.nbrs_pad);
  cudaFree(w.pos_pad);
  cudaFree(w.cnt);
  cudaFree(w.ctrl);
  w = Workspace{};
}

static wg_status alloc_workspace(wg_dsm* h, int64_t max_keys) {
  Workspace& w = h->ws;
  if (max_keys < 1) max_keys = 1;
  // Table size = HASH_FACTOR (2) x the capacity bound (a multiple of 8 slots).  Trade-off measured on B200:
  // a larger table shortens the warp-max linear-probe chains (single-batch latency), a smaller
  // one packs the touched slots into fewer DRAM lines, which matters when several batches (one
  // table each) are in flight and compete for the 126 MB L2.  Slot indices must fit int32 (slot_of).
  int64_t cap = (int64_t)(HASH_FACTOR * (double)max_keys) + 8;
  cap = std::min<int64_t>(std::max<int64_t>(1024, (cap + 7) / 8 * 8), HASH_MAX_SLOTS);
  w.hcap = cap;
  w.max_keys = max_keys;
  w.status_cap = max_keys / 32 + 2;  // sampler tiles hold >= 32 targets, flag tiles 1024 positions
  if (cudaMalloc(&w.status_sample, w.status_cap * 8) != cudaSuccess ||
      cudaMalloc(&w.status_unique, w.status_cap * 8) != cudaSuccess ||
      cudaMalloc(&w.excl[0], max_keys * 4) != cudaSuccess || cudaMalloc(&w.excl[1], max_keys * 4) != cudaSuccess ||
      cudaMalloc(&w.excl[2], max_keys * 4) != cudaSuccess || cudaMalloc(&w.excl[3], max_keys * 4) != cudaSuccess ||
      cudaMalloc(&w.slot_of, max_keys * 4) != cudaSuccess || cudaMalloc(&w.nbrs_pad, max_keys * 8) != cudaSuccess ||
      cudaMalloc(&w.pos_pad, max_keys * 4) != cudaSuccess || cudaMalloc(&w.cnt, max_keys * 4) != cudaSuccess ||
      cudaMalloc(&w.ctrl, CTRL_WORDS * 4) != cudaSuccess) {
    cudaGetLastError();
    free_workspace(h);
    return fail(WG_ERR_OOM, "workspace allocation failed");
  }
  // compact 8 B slots (hash.cuh) when node ids and positions fit 28 bits (WG_DSM_WIDE_HASH: 16 B slots)
  w.compact = !(h->flags & WG_DSM_WIDE_HASH) && h->n <= (int64_t(1) << 28) && max_keys < (int64_t(1) << 28) ? 1 : 0;
  // direct table (a word per node, hash.cuh) for small graphs unless a hashed format is asked for
  w.direct = !(h->flags & (WG_DSM_WIDE_HASH | WG_DSM_HASHED)) && h->n <= WG_DIRECT_MAX_NODES &&
                     max_keys < (int64_t(1) << DPOS_BITS)
                 ? 1
                 : 0;
  if (w.direct) {  // no hash table at all: every append-unique of this workspace keys the direct tables
    w.hcap = 0;
    const size_t db = (size_t)((h->n + 3) / 4) * 16;  // whole 16 B units (dtab_clear_ahead)
    for (int t = 0; t < 2; ++t) {
      if (cudaMalloc(&w.dtab[t], db) != cudaSuccess) {
        cudaGetLastError();
        free_workspace(h);
        return fail(WG_ERR_OOM, "workspace allocation failed (direct table)");
      }
      WG_CUDA_TRY(cudaMemset(w.dtab[t], 0xff, db));  // every word empty
    }
  }
  w.pad32 = !(h->flags & WG_DSM_PAD64) && h->n < (int64_t(1) << 32) ? 1 : 0;
  if (w.direct) {
  } else if (w.compact) {
    // two tables of 8 B words, alternating per 255-epoch cycle (hash.cuh); every word stale (epoch 0)
    if (cudaMalloc(&w.hslots, cap * 8) != cudaSuccess || cudaMalloc(&w.hslots2, cap * 8) != cudaSuccess) {
      cudaGetLastError();
      free_workspace(h);
      return fail(WG_ERR_OOM, "workspace allocation failed (hash table)");
    }
    WG_CUDA_TRY(cudaMemset(w.hslots, 0, cap * 8));
    WG_CUDA_TRY(cudaMemset(w.hslots2, 0, cap * 8));
  } else {
    if (cudaMalloc(&w.hslots, cap * sizeof(HashSlot)) != cudaSuccess) {
      cudaGetLastError();
      free_workspace(h);
      return fail(WG_ERR_OOM, "workspace allocation failed (hash table)");
    }
    WG_CUDA_TRY(cudaMemset(w.hslots, 0xff, cap * sizeof(HashSlot)));                   // val = all ones
    WG_CUDA_TRY(cudaMemset2D(w.hslots, sizeof(HashSlot), 0, sizeof(unsigned long long), cap));  // key = 0 (empty)
  }
  // The kernels read the padded sampler slots speculatively (a key is loaded together with its
  // slot's count and discarded for a padding slot): zero them once so no read is of never-written
  // memory (compute-sanitizer initcheck clean).
  WG_CUDA_TRY(cudaMemset(w.nbrs_pad, 0, max_keys * 8));
  WG_CUDA_TRY(cudaMemset(w.pos_pad, 0, max_keys * 4));
  WG_CUDA_TRY(cudaMemset(w.status_sample, 0, w.status_cap * 8));
  WG_CUDA_TRY(cudaMemset(w.status_unique, 0, w.status_cap * 8));
  unsigned ctrl[CTRL_WORDS] = {0};
  ctrl[CTRL_EPOCH] = 1;
  WG_CUDA_TRY(cudaMemcpy(w.ctrl, ctrl, sizeof(ctrl), cudaMemcpyHostToDevice));
  return WG_OK;
}

static void release(wg_dsm* h) {
  if (h->fork_event) cudaEventDestroy(h->fork_event);
  if (h->parent) {  // a workspace fork owns only its workspace
    free_workspace(h);
    h->parent->live_forks -= 1;
    delete h;
    return;
  }
  for (int r = 0; r < h->world; ++r)
    if (h->peer_opened[r]) cudaIpcCloseMemHandle(h->peer_base[r]);
  free_workspace(h);
  if (h->slab) cudaFree(h->slab);
  delete h;
}

}  // namespace wg

using namespace wg;

extern "C" {

const char* wg_last_error(void) { return g_last_error.c_str(); }
const char* wg_version(void) { return "wholegraph-b200 0.1 (sm_100a)"; }

wg_status wg_dsm_create(const wg_dsm_desc* d, wg_dsm_t* out) {
  if (!out) return fail(WG_ERR_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (!d) return fail(WG_ERR_INVALID_ARG, "desc is NULL");
  if (d->world_size < 1 || d->world_size > WG_MAX_WORLD || d->rank < 0 || d->rank >= d->world_size)
    return fail(WG_ERR_INVALID_ARG, "rank/world_size out of range");
  if (d->num_nodes < 0 || d->num_nodes >= (int64_t(1) << 40) || d->local_num_edges < 0 || d->feat_dim < 0 ||
      d->max_batch_keys < 0 || d->max_batch_keys >= (int64_t(1) << 31))
    return fail(WG_ERR_INVALID_ARG, "sizes out of range (num_nodes < 2^40, max_batch_keys < 2^31)");
  if (d->feat_dtype < WG_F32 || d->feat_dtype > WG_BF16) return fail(WG_ERR_INVALID_ARG, "feat_dtype");
  if (d->world_size > 1 && !d->allgather) return fail(WG_ERR_INVALID_ARG, "allgather callback required for W > 1");
  if ((d->flags & ~(WG_DSM_WHOLE_ROWS | WG_DSM_WIDE_HASH | WG_DSM_PAD64 | WG_DSM_CSR_REPLICATED | WG_DSM_COL32 |
                    WG_DSM_HASHED)) ||
      d->reserved)
    return fail(WG_ERR_INVALID_ARG, "unknown flags");
  if ((d->flags & WG_DSM_COL32) && d->num_nodes > (int64_t(1) << 32))
    return fail(WG_ERR_INVALID_ARG, "WG_DSM_COL32 needs num_nodes <= 2^32");

  WG_CUDA_TRY(cudaSetDevice(d->device));
  int major = 0, minor = 0, sms = 0;
  WG_CUDA_TRY(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, d->device));
  WG_CUDA_TRY(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, d->device));
  WG_CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, d->device));
  if (major * 10 + minor < 100) return fail(WG_ERR_UNSUPPORTED, "needs an sm_100 (Blackwell) device");

  wg_dsm* h = new wg_dsm();
  h->rank = d->rank;
  h->world = d->world_size;
  h->device = d->device;
  h->n = d->num_nodes;
  h->feat_dim = d->feat_dim;
  h->elt = d->feat_dtype == WG_F32 ? 4 : 2;
  h->row_bytes = h->feat_dim * h->elt;
  h->flags = d->flags;
  feat_geometry(h->row_bytes, !(h->flags & WG_DSM_WHOLE_ROWS), &h->body_bytes, &h->feat_stride, &h->tail_pitch);
  h->allgather = d->allgather;
  h->ctx = d->ctx;
  h->sm_count = sms;
  h->n_local = local_rows(h->n, h->rank, h->world);
  h->e_local = d->local_num_edges;

  // ---- this rank's slab (the CSR part holds all n rows with WG_DSM_CSR_REPLICATED)
  const bool csr_rep = (h->flags & WG_DSM_CSR_REPLICATED) != 0;
  const int64_t csr_rows = csr_rep ? h->n : h->n_local;
  const int64_t off_col = round_up((csr_rows + 1) * 8, 256);
  const int64_t col_bytes = (h->flags & WG_DSM_COL32) ? 4 : 8;
  const int64_t off_feat = round_up(off_col + h->e_local * col_bytes, 256);
  const int64_t off_tail = round_up(off_feat + h->n_local * h->feat_stride, 256);
  h->slab_bytes = (size_t)round_up(off_tail + h->n_local * h->tail_pitch, 256);
  if (cudaMalloc(&h->slab, h->slab_bytes) != cudaSuccess) {
    cudaGetLastError();
    h->slab = nullptr;
    release(h);
    return fail(WG_ERR_OOM, "shard allocation of " + std::to_string(h->slab_bytes) + " bytes failed");
  }
  if (cudaEventCreateWithFlags(&h->fork_event, cudaEventDisableTiming) != cudaSuccess) {
    cudaGetLastError();
    h->fork_event = nullptr;
    release(h);
    return fail(WG_ERR_CUDA, "cudaEventCreate failed");
  }
  wg_status st = alloc_workspace(h, d->max_batch_keys);
  if (st != WG_OK) {
    std::string m = g_last_error;
    release(h);
    return fail(st, m);
  }

  // ---- export + allgather the IPC handles (L100)
  PeerRecord mine;
  std::memset(&mine, 0, sizeof(mine));
  mine.pid = (int64_t)getpid();
  mine.dev_ptr = (uint64_t)(uintptr_t)h->slab;
  mine.slab_bytes = (int64_t)h->slab_bytes;
  mine.n_local = h->n_local;
  mine.e_local = h->e_local;
  mine.off_col = off_col;
  mine.off_feat = off_feat;
  mine.off_tail = off_tail;
  mine.num_nodes = h->n;
  mine.feat_stride = h->feat_stride;
  mine.tail_pitch = h->tail_pitch;
  mine.world = h->world;
  mine.rank = h->rank;
  mine.flags = h->flags;
  {
    cudaDeviceProp prop;
    WG_CUDA_TRY(cudaGetDeviceProperties(&prop, h->device));
    std::memcpy(mine.uuid, prop.uuid.bytes, 16);
  }
  PeerRecord all[WG_MAX_WORLD];
  std::memset(all, 0, sizeof(all));
  if (h->world > 1) {
    if (cudaIpcGetMemHandle(&mine.handle, h->slab) != cudaSuccess) {
      cudaGetLastError();
      release(h);
      return fail(WG_ERR_PEER_ACCESS, "cudaIpcGetMemHandle failed");
    }
    if (h->allgather(&mine, all, sizeof(PeerRecord), h->ctx) != 0) {
      release(h);
      return fail(WG_ERR_COLLECTIVE, "allgather of IPC handles failed");
    }
  } else {
    all[0] = mine;
  }
  for (int r = 0; r < h->world; ++r) {
    if (all[r].rank != r || all[r].world != h->world || all[r].num_nodes != h->n ||
        all[r].feat_stride != h->feat_stride || all[r].tail_pitch != h->tail_pitch || all[r].flags != h->flags) {
      release(h);
      return fail(WG_ERR_INVALID_ARG, "ranks disagree on world_size / num_nodes / feat_dim / flags");
    }
  }

  // ---- open peers (L100-106) and build the memory pointer table (L106)
  for (int r = 0; r < h->world; ++r) {
    h->n_local_of[r] = all[r].n_local;
    h->e_local_of[r] = all[r].e_local;
    if (r == h->rank) {
      h->peer_base[r] = h->slab;
    } else if (all[r].pid == mine.pid) {
      h->peer_base[r] = (void*)(uintptr_t)all[r].dev_ptr;  // same process: plain device pointer
    } else {
      // one process per GPU (L98): a peer slab on ANOTHER visible GPU needs P2P access (NVLink) from ours
      int peer_dev = -1, ndev = 0;
      cudaGetDeviceCount(&ndev);
      for (int dv = 0; dv < ndev && peer_dev < 0; ++dv) {
        cudaDeviceProp pp;
        if (cudaGetDeviceProperties(&pp, dv) == cudaSuccess && std::memcmp(pp.uuid.bytes, all[r].uuid, 16) == 0)
          peer_dev = dv;
      }
      cudaGetLastError();
      if (peer_dev >= 0 && peer_dev != h->device) {
        int can = 0;
        cudaDeviceCanAccessPeer(&can, h->device, peer_dev);
        if (!can) {
          release(h);
          return fail(WG_ERR_PEER_ACCESS, "device " + std::to_string(h->device) + " cannot access rank " +
                                              std::to_string(r) + "'s device " + std::to_string(peer_dev) +
                                              " peer-to-peer (cudaDeviceCanAccessPeer == 0)");
        }
      }
      void* p = nullptr;
      cudaError_t e = cudaIpcOpenMemHandle(&p, all[r].handle, cudaIpcMemLazyEnablePeerAccess);
      if (e != cudaSuccess) {
        cudaGetLastError();
        release(h);
        return fail(WG_ERR_PEER_ACCESS, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
      }
      h->peer_base[r] = p;
      h->peer_opened[r] = true;
    }
    uint8_t* b = static_cast<uint8_t*>(h->peer_base[r]);
    h->view.row_ptr[r] = reinterpret_cast<const int64_t*>(b);
    h->view.col[r] = b + all[r].off_col;
    h->view.feat[r] = b + all[r].off_feat;
    h->view.tail[r] = h->tail_pitch ? b + all[r].off_tail : nullptr;
  }
  h->view.n = h->n;
  h->view.feat_stride = h->feat_stride;
  h->view.tail_pitch = h->tail_pitch;
  h->view.body_bytes = h->body_bytes;
  h->view.world = h->world;
  h->view.log2w = -1;
  for (int k = 0; k <= 3; ++k)
    if ((1 << k) == h->world) h->view.log2w = k;
  h->view.csr_rank = csr_rep ? h->rank : -1;
  h->view.col32 = (h->flags & WG_DSM_COL32) ? 1 : 0;
  // Zero this rank's row_ptr so an unfilled shard reads as degree 0.
  if (cudaMemset(h->slab, 0, (csr_rows + 1) * 8) != cudaSuccess) {
    cudaGetLastError();
    release(h);
    return fail(WG_ERR_CUDA, "memset row_ptr");
  }
  if (cudaDeviceSynchronize() != cudaSuccess || barrier(h) != WG_OK) {
    release(h);
    return fail(WG_ERR_COLLECTIVE, "create: final barrier failed");
  }
  *out = h;
  return WG_OK;
}

wg_status wg_dsm_local_view(wg_dsm_t h, int64_t** row_ptr, int64_t** col, void** feat, int64_t* n_local_rows,
                            int64_t* stride) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  if (row_ptr) *row_ptr = const_cast<int64_t*>(h->view.row_ptr[h->rank]);
  if (col) *col = const_cast<int64_t*>(static_cast<const int64_t*>(h->view.col[h->rank]));
  if (feat) *feat = const_cast<uint8_t*>(h->view.feat[h->rank]);
  if (n_local_rows) *n_local_rows = h->n_local;
  if (stride) *stride = h->feat_stride;
  return WG_OK;
}

wg_status wg_dsm_feat_layout(wg_dsm_t h, int64_t* body_bytes, int64_t* body_pitch, void** d_tail,
                             int64_t* tail_pitch) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  if (body_bytes) *body_bytes = h->body_bytes;
  if (body_pitch) *body_pitch = h->feat_stride;
  if (d_tail) *d_tail = const_cast<uint8_t*>(h->view.tail[h->rank]);
  if (tail_pitch) *tail_pitch = h->tail_pitch;
  return WG_OK;
}

wg_status wg_dsm_shard_info(wg_dsm_t h, int32_t r, int64_t* n_local_rows, int64_t* local_num_edges) {
  if (!h || r < 0 || r >= h->world) return fail(WG_ERR_INVALID_ARG, "bad handle or rank");
  if (n_local_rows) *n_local_rows = h->n_local_of[r];
  if (local_num_edges) *local_num_edges = h->e_local_of[r];
  return WG_OK;
}

wg_status wg_dsm_set_gather_occupancy(wg_dsm_t h, int32_t blocks_per_sm) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  if (blocks_per_sm < 0) return fail(WG_ERR_INVALID_ARG, "blocks_per_sm < 0");
  h->gather_bps = blocks_per_sm;
  return WG_OK;
}

wg_status wg_dsm_fork(wg_dsm_t parent, int64_t max_batch_keys, wg_dsm_t* out) {
  if (!out) return fail(WG_ERR_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (!parent || parent->parent) return fail(WG_ERR_INVALID_ARG, "parent must be a DSM created by wg_dsm_create");
  if (max_batch_keys < 0 || max_batch_keys >= (int64_t(1) << 31)) return fail(WG_ERR_INVALID_ARG, "max_batch_keys");
  WG_CUDA_TRY(cudaSetDevice(parent->device));
  wg_dsm* h = new wg_dsm();
  *h = *parent;  // geometry, pointer table, callbacks
  h->ws = Workspace{};
  h->fork_event = nullptr;
  h->stage_n = 0;
  h->parent = parent;
  h->live_forks = 0;
  h->excl_next = 0;
  for (int r = 0; r < WG_MAX_WORLD; ++r) h->peer_opened[r] = false;  // mappings stay owned by the parent
  h->slab = nullptr;
  parent->live_forks += 1;
  if (cudaEventCreateWithFlags(&h->fork_event, cudaEventDisableTiming) != cudaSuccess) {
    cudaGetLastError();
    h->fork_event = nullptr;
    release(h);
    return fail(WG_ERR_CUDA, "cudaEventCreate failed");
  }
  wg_status st = alloc_workspace(h, max_batch_keys ? max_batch_keys : parent->ws.max_keys);
  if (st != WG_OK) {
    std::string m = g_last_error;
    release(h);
    return fail(st, m);
  }
  *out = h;
  return WG_OK;
}

wg_status wg_dsm_destroy(wg_dsm_t h) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  cudaSetDevice(h->device);
  cudaDeviceSynchronize();
  if (h->parent) {  // a fork: not collective
    release(h);
    return WG_OK;
  }
  if (h->live_forks > 0) return fail(WG_ERR_INVALID_ARG, "destroy the handle's forks first");
  wg_status s1 = barrier(h);  // nobody reads a peer any more
  for (int r = 0; r < h->world; ++r)
    if (h->peer_opened[r]) {
      cudaIpcCloseMemHandle(h->peer_base[r]);
      h->peer_opened[r] = false;
    }
  wg_status s2 = barrier(h);  // nobody maps ours any more
  release(h);
  if (s1 != WG_OK) return s1;
  return s2;
}

wg_status wg_sample_neighbors(wg_dsm_t h, const int64_t* d_targets, int64_t n_targets, const int64_t* d_n_targets,
                              int32_t fanout, uint64_t seed, const uint64_t* d_seed, int32_t hop,
                              int64_t* d_out_row_ptr, int64_t* d_out_nbrs, int32_t* d_out_pos,
                              int64_t* d_out_num_edges, wg_stream_t stream) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  if (fanout < 1) return fail(WG_ERR_INVALID_ARG, "fanout must be >= 1");
  if (fanout > WG_MAX_FANOUT) return fail(WG_ERR_UNSUPPORTED, "fanout > 1024");
  if (n_targets < 0 || (n_targets > 0 && !d_targets) || !d_out_row_ptr || (n_targets > 0 && !d_out_nbrs))
    return fail(WG_ERR_INVALID_ARG, "null pointer or negative size");
  if (hop < 0) return fail(WG_ERR_INVALID_ARG, "hop must be >= 0");
  if (n_targets * (int64_t)fanout > h->ws.max_keys)
    return fail(WG_ERR_CAPACITY, "n_targets * fanout exceeds max_batch_keys");
  if (n_targets * (int64_t)fanout >= (int64_t(1) << 40)) return fail(WG_ERR_INVALID_ARG, "too many edges");
  cudaSetDevice(h->device);
  cudaError_t e = launch_sample(h, d_targets, n_targets, d_n_targets, fanout, seed, d_seed, hop, d_out_row_ptr,
                                d_out_nbrs, d_out_pos, d_out_num_edges, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(WG_ERR_CUDA, std::string("sample launch: ") + cudaGetErrorString(e));
  return WG_OK;
}

wg_status wg_append_unique(wg_dsm_t h, const int64_t* d_targets, int64_t n_targets, const int64_t* d_n_targets,
                           const int64_t* d_nbrs, int64_t n_nbrs, const int64_t* d_n_nbrs, int64_t* d_out_unique,
                           int64_t* d_out_num_unique, int32_t* d_out_sub_col, int32_t* d_out_dup_count,
                           wg_stream_t stream) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  if (n_targets < 0 || n_nbrs < 0) return fail(WG_ERR_INVALID_ARG, "negative size");
  if ((n_targets > 0 && !d_targets) || (n_nbrs > 0 && (!d_nbrs || !d_out_sub_col)) ||
      (n_targets + n_nbrs > 0 && !d_out_unique))
    return fail(WG_ERR_INVALID_ARG, "null pointer");
  if (n_targets + n_nbrs > h->ws.max_keys)
    return fail(WG_ERR_CAPACITY, "n_targets + n_nbrs exceeds max_batch_keys");
  cudaSetDevice(h->device);
  cudaError_t e = launch_append_unique(h, d_targets, n_targets, d_n_targets, d_nbrs, n_nbrs, d_n_nbrs, d_out_unique,
                                       d_out_num_unique, d_out_sub_col, d_out_dup_count, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(WG_ERR_CUDA, std::string("append_unique launch: ") + cudaGetErrorString(e));
  return WG_OK;
}

wg_status wg_sample_hop(wg_dsm_t h, const int64_t* d_targets, int64_t n_targets, const int64_t* d_n_targets,
                        int32_t fanout, uint64_t seed, const uint64_t* d_seed, int32_t hop, int64_t* d_out_row_ptr,
                        int64_t* d_out_nbrs, int32_t* d_out_pos, int64_t* d_out_num_edges, int64_t* d_out_unique,
                        int64_t* d_out_num_unique, int32_t* d_out_sub_col, int32_t* d_out_dup_count,
                        wg_stream_t stream, wg_stream_t side_stream) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  if (fanout < 1) return fail(WG_ERR_INVALID_ARG, "fanout must be >= 1");
  if (fanout > WG_MAX_FANOUT) return fail(WG_ERR_UNSUPPORTED, "fanout > 1024");
  if (n_targets < 0 || hop < 0 || !d_out_row_ptr || !d_out_num_edges ||
      (n_targets > 0 && (!d_targets || !d_out_nbrs || !d_out_unique || !d_out_sub_col)))
    return fail(WG_ERR_INVALID_ARG, "null pointer or negative size");
  const int64_t n_nbrs = n_targets * (int64_t)fanout;
  if (n_targets + n_nbrs > h->ws.max_keys) return fail(WG_ERR_CAPACITY, "n_targets*(1+fanout) exceeds max_batch_keys");
  cudaSetDevice(h->device);
  cudaError_t e = launch_hop(h, d_targets, n_targets, d_n_targets, fanout, seed, d_seed, hop, d_out_row_ptr,
                             d_out_nbrs, d_out_pos, d_out_num_edges, d_out_unique, d_out_num_unique, d_out_sub_col,
                             d_out_dup_count, (cudaStream_t)stream, (cudaStream_t)side_stream);
  if (e != cudaSuccess) return fail(WG_ERR_CUDA, std::string("hop launch: ") + cudaGetErrorString(e));
  return WG_OK;
}

wg_status wg_gather_rows(wg_dsm_t h, const int64_t* d_ids, int64_t n_ids, const int64_t* d_begin,
                         const int64_t* d_end, void* d_out, int64_t out_pitch, wg_stream_t stream) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  if (n_ids < 0 || (n_ids > 0 && (!d_ids || !d_out))) return fail(WG_ERR_INVALID_ARG, "null pointer or negative size");
  if (h->row_bytes == 0) return fail(WG_ERR_INVALID_ARG, "DSM has no feature table");
  if (h->row_bytes % 2 != 0) return fail(WG_ERR_UNSUPPORTED, "odd row size");
  // a pitched output may cover the row's padding in the shard (whole layout) or up to the next 32 B
  // (split layout: the tail chunk is zero-filled past the row)
  const int64_t max_pitch = h->tail_pitch ? round_up(h->row_bytes, 32) : h->feat_stride;
  if (out_pitch != 0 && out_pitch != h->row_bytes &&
      (out_pitch < h->row_bytes || out_pitch % 16 != 0 || out_pitch > max_pitch))
    return fail(WG_ERR_INVALID_ARG, "out_pitch must be 0, row_bytes, or a multiple of 16 in [row_bytes, row pitch]");
  const int64_t cw = out_pitch > h->row_bytes ? out_pitch : h->row_bytes;
  if (n_ids * (cw / 2) >= (int64_t(1) << 31)) return fail(WG_ERR_UNSUPPORTED, "gather too large for one launch");
  cudaSetDevice(h->device);
  if (n_ids == 0 && !d_end) return WG_OK;
  cudaError_t e = launch_gather(h, d_ids, n_ids, d_end, d_begin, d_out, out_pitch, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(WG_ERR_CUDA, std::string("gather launch: ") + cudaGetErrorString(e));
  return WG_OK;
}

wg_status wg_gather(wg_dsm_t h, const int64_t* d_ids, int64_t n_ids, const int64_t* d_n_ids, void* d_out,
                    wg_stream_t stream) {
  return wg_gather_rows(h, d_ids, n_ids, nullptr, d_n_ids, d_out, 0, stream);
}

wg_status wg_device_error(wg_dsm_t h, uint32_t* code, int32_t clear) {
  if (!h || !code) return fail(WG_ERR_INVALID_ARG, "null argument");
  cudaSetDevice(h->device);
  WG_CUDA_TRY(cudaDeviceSynchronize());
  WG_CUDA_TRY(cudaMemcpy(code, h->ws.ctrl + CTRL_ERR, 4, cudaMemcpyDeviceToHost));
  if (clear) WG_CUDA_TRY(cudaMemset(h->ws.ctrl + CTRL_ERR, 0, 4));
  return WG_OK;
}

wg_status wg_dsm_reset_workspace(wg_dsm_t h, wg_stream_t stream) {
  if (!h) return fail(WG_ERR_INVALID_ARG, "handle is NULL");
  cudaSetDevice(h->device);
  cudaStream_t st = (cudaStream_t)stream;
  if (h->ws.direct) {
    for (int t = 0; t < 2; ++t) WG_CUDA_TRY(cudaMemsetAsync(h->ws.dtab[t], 0xff, (size_t)((h->n + 3) / 4) * 16, st));
  }
  if (h->ws.direct) {
  } else if (h->ws.compact) {
    WG_CUDA_TRY(cudaMemsetAsync(h->ws.hslots, 0, h->ws.hcap * 8, st));
    WG_CUDA_TRY(cudaMemsetAsync(h->ws.hslots2, 0, h->ws.hcap * 8, st));
  } else {
    WG_CUDA_TRY(cudaMemsetAsync(h->ws.hslots, 0xff, h->ws.hcap * sizeof(HashSlot), st));
    WG_CUDA_TRY(cudaMemset2DAsync(h->ws.hslots, sizeof(HashSlot), 0, sizeof(unsigned long long), h->ws.hcap, st));
  }
  static const unsigned one = 1;
  WG_CUDA_TRY(cudaMemcpyAsync(h->ws.ctrl + CTRL_EPOCH, &one, 4, cudaMemcpyHostToDevice, st));
  return WG_OK;
}

wg_status wg_dsm_set_stage_events(wg_dsm_t h, void* const* events, int32_t n) {
  if (!h || n < 0 || n > 8 || (n > 0 && !events)) return fail(WG_ERR_INVALID_ARG, "bad arguments (n <= 8)");
  for (int i = 0; i < 8; ++i) h->stage_ev[i] = i < n ? (cudaEvent_t)events[i] : nullptr;
  h->stage_n = n;
  h->stage_i = 0;
  return WG_OK;
}

wg_status wg_dsm_debug_set_epoch(wg_dsm_t h, uint32_t epoch) {
  if (!h || epoch == 0 || epoch >= EPOCH_MAX) return fail(WG_ERR_INVALID_ARG, "bad handle or epoch");
  cudaSetDevice(h->device);
  WG_CUDA_TRY(cudaDeviceSynchronize());
  WG_CUDA_TRY(cudaMemcpy(h->ws.ctrl + CTRL_EPOCH, &epoch, 4, cudaMemcpyHostToDevice));
  // the direct tables hold words of the old epoch sequence: empty them (the next op's table must be
  // clean, hash.cuh)
  if (h->ws.direct)
    for (int t = 0; t < 2; ++t) WG_CUDA_TRY(cudaMemset(h->ws.dtab[t], 0xff, (size_t)((h->n + 3) / 4) * 16));
  if (h->ws.compact && !h->ws.direct) {  // likewise the compact tables (the next cycle's table must be clean)
    WG_CUDA_TRY(cudaMemset(h->ws.hslots, 0, h->ws.hcap * 8));
    WG_CUDA_TRY(cudaMemset(h->ws.hslots2, 0, h->ws.hcap * 8));
  }
  return WG_OK;
}

wg_status wg_dsm_unique_format(wg_dsm_t h, int32_t* format, int32_t* hop_insert_pass) {
  if (!h || !format) return fail(WG_ERR_INVALID_ARG, "null argument");
  *format = h->ws.direct ? WG_UNIQUE_DIRECT : h->ws.compact ? WG_UNIQUE_COMPACT : WG_UNIQUE_WIDE;
  if (hop_insert_pass) *hop_insert_pass = wg::hop_inserts_in_sampler(h) ? 0 : 1;
  return WG_OK;
}

}  // extern "C"
