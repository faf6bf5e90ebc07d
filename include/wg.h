/*
 * wg.h -- C ABI of the B200-native WholeGraph mini-batch preparation path.
 *
 * WholeGraph (Yang, Liu, Qi, Lai, SC'22; /root/reference/PAPER.md) prepares a
 * GNN mini-batch on every GPU from a graph and a feature table held in a
 * multi-GPU distributed shared memory (DSM).  Citations "L<n>" are PAPER.md
 * lines; "A<n>" are the readings of ambiguous passages listed in DESIGN.md
 * (section "Readings") and SURVEY.md 8(c).
 *
 * Conventions for every call below
 *  - Pointers prefixed d_ are DEVICE pointers on the handle's device; the caller
 *    owns them (e.g. torch tensors).  The handle owns the shards, the peer
 *    mappings and an internal workspace (hash table, scan state, error word).
 *  - Every op is stream-ordered and asynchronous: it enqueues kernels on
 *    `stream` (a cudaStream_t; NULL = legacy default stream) and returns without
 *    synchronising the host.  Calls on one handle must be issued on one stream
 *    at a time (they share the workspace).  All ops are CUDA-graph capturable.
 *  - Sizes n_* are HOST capacities (upper bounds, used to size launches and to
 *    bound writes).  The optional d_n_* are DEVICE int64 scalars holding the
 *    actual count produced by a previous call (e.g. d_out_num_edges), so hops
 *    chain without a host sync; NULL means "use n_* exactly".  An actual count
 *    larger than its capacity is clamped to the capacity and latches
 *    WG_DEVERR_CAPACITY.
 *  - Global node ids are int64 in [0, num_nodes) ("8 bytes to store each edge",
 *    L236; A12).  Sub-graph (local) ids are int32.
 *  - Argument errors are detected on the host and returned immediately
 *    (nothing is enqueued).  Data errors found by kernels (an id out of range, a
 *    duplicate target, a capacity overflow) are OR-ed into a device error word
 *    read by wg_device_error(); the op still writes defined outputs.
 *  - There is no CPU fallback: every op runs in the library's sm_100a kernels,
 *    and wg_dsm_create returns WG_ERR_UNSUPPORTED on devices below sm_100.
 */
#ifndef WG_H_
#define WG_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define WG_MAX_WORLD 8          /* ranks (GPUs) per DSM: one HGX B200 box */
#define WG_MAX_FANOUT 1024      /* largest M: <= 32 uses the warp sampler, above a block per target */

typedef struct wg_dsm* wg_dsm_t; /* opaque host handle, one per rank process */
typedef void* wg_stream_t;       /* a cudaStream_t */

typedef enum {
  WG_OK = 0,
  WG_ERR_INVALID_ARG = 1,  /* bad pointer / size / fanout; nothing enqueued */
  WG_ERR_CUDA = 2,         /* a CUDA runtime call failed; see wg_last_error() */
  WG_ERR_OOM = 3,          /* device allocation failed */
  WG_ERR_PEER_ACCESS = 4,  /* IPC export/import of a peer shard failed */
  WG_ERR_CAPACITY = 5,     /* request exceeds the workspace sized at create */
  WG_ERR_UNSUPPORTED = 6,  /* device below sm_100, or fanout > WG_MAX_FANOUT */
  WG_ERR_COLLECTIVE = 7    /* the allgather callback returned non-zero */
} wg_status;

typedef enum { WG_F32 = 0, WG_F16 = 1, WG_BF16 = 2 } wg_dtype;

/* Bits of the latched device error word (wg_device_error). */
#define WG_DEVERR_ID_RANGE   0x1u  /* a node id outside [0, num_nodes): treated as degree 0 / skipped
                                       (a col_idx entry of 0xFFFFFFFF in a uint32 shard with the direct key
                                       table reads as "no sample"; the error is latched either way) */
#define WG_DEVERR_DUP_TARGET 0x2u  /* wg_append_unique: duplicate target (A8) */
#define WG_DEVERR_CAPACITY   0x4u  /* a device count exceeded its host capacity, or the hash table filled */
#define WG_DEVERR_DEGREE     0x8u  /* a degree >= 2^32 (A3 requires N < 2^32) */
#define WG_DEVERR_EPOCH      0x10u /* hash-table epoch space exhausted: call wg_dsm_reset_workspace */

/* wg_dsm_desc.flags (layout / placement choices of one DSM; results never depend on the layout
 * flags, only on the graph, the table and the inputs). */
#define WG_DSM_WHOLE_ROWS     0x1u  /* feature rows stored whole (never split into body + tail, see
                                       wg_dsm_feat_layout) */
#define WG_DSM_WIDE_HASH      0x2u  /* 16 B append-unique hash slots even when node ids and positions fit
                                       the compact 8 B format (the format used for num_nodes >= 2^28) */
#define WG_DSM_PAD64          0x4u  /* int64 padded sampler slots even when every id fits 32 bits */
#define WG_DSM_CSR_REPLICATED 0x8u  /* hybrid placement: every rank holds the WHOLE
                                       CSR (row_ptr int64[num_nodes+1], col_idx int64[local_num_edges =
                                       all E]) and samples locally; only the feature table is row-sharded
                                       (o(v) = v mod W) and read over NVLink.  Results are identical. */
#define WG_DSM_COL32          0x10u /* col_idx entries stored as uint32 (needs num_nodes <= 2^32): half the
                                       bytes of every sampled line; wg_dsm_local_view's d_col_idx then points
                                       to uint32 entries (ids in every op stay int64) */
#define WG_DSM_HASHED         0x20u /* append-unique keys in a hash table even when the direct table fits
                                       (see wg_dsm_unique_format) */

/* Key-table formats of Append Unique ("the key of our GPU hash table is nodeID";
 * wg_dsm_unique_format).  DIRECT (num_nodes <= 2^24, max_batch_keys < 2^24, no WG_DSM_HASHED /
 * WG_DSM_WIDE_HASH): the "table" is indexed by the node id itself -- one 32-bit word per node holding
 * the key's first position, two such arrays per workspace (2 x 4 B x num_nodes); the fused hop's
 * sampler inserts every key (no insert pass).  COMPACT: 8 B hashed slots (ids and positions < 2^28),
 * two tables alternating per 255-epoch cycle.  WIDE: 16 B hashed slots.  Both hashed formats run a
 * separate insert pass.
 * Results never depend on the format. */
#define WG_UNIQUE_WIDE    0
#define WG_UNIQUE_COMPACT 1
#define WG_UNIQUE_DIRECT  2

/* Allgather of host bytes across the W ranks of the DSM ("an
 * AllGather pattern communication is performed so that each process can get all
 * the CUDA IPC handles").  recv receives world_size * bytes_per_rank bytes in
 * rank order.  bytes_per_rank == 0 must act as a barrier.  Return 0 on success.
 * Used only inside wg_dsm_create / wg_dsm_destroy (setup), never on the hot path. */
typedef int (*wg_allgather_fn)(const void* send, void* recv, size_t bytes_per_rank, void* ctx);

typedef struct {
  int32_t rank;             /* this process's rank in [0, world_size) */
  int32_t world_size;       /* W, 1 <= W <= WG_MAX_WORLD */
  int32_t device;           /* CUDA device ordinal this rank drives ("one process
                               usually controls one single GPU", L98) */
  int32_t feat_dtype;       /* wg_dtype; only sets the element size (rows move as bytes, A14) */
  int64_t num_nodes;        /* n; node v lives on rank o(v) = v mod W at local row
                               l(v) = v div W (hash partition, L110; A11) */
  int64_t local_num_edges;  /* CSR entries of the rows THIS rank owns ("edges are
                               stored together with the source node", L110) */
  int64_t feat_dim;         /* feature columns per node (0 = no feature table) */
  int64_t max_batch_keys;   /* workspace sizing: the largest n_targets + n_nbrs
                               passed to wg_append_unique and the largest
                               n_targets passed to wg_sample_neighbors */
  wg_allgather_fn allgather;
  void* ctx;                /* passed through to allgather */
  uint32_t flags;           /* WG_DSM_* above (0 = the paper's placement, measured-best layout) */
  uint32_t reserved;        /* must be 0 */
} wg_dsm_desc;

/* Create the DSM (section III-B).  COLLECTIVE over the W ranks.
 * Each rank allocates its shard slab on its device -- row_ptr int64[n_local+1] (int64[num_nodes+1]
 * with WG_DSM_CSR_REPLICATED), col_idx int64[local_num_edges] (uint32 with WG_DSM_COL32), features
 * [n_local][row stride] (+ a tail region for the
 * split row layout, see wg_dsm_feat_layout) -- exports a CUDA IPC handle, allgathers the
 * handles (L100), opens every peer's handle (L100-106; same-process peers are used
 * directly) and keeps the W base pointers as the "memory pointer table" (L106),
 * passed by value to every kernel.  n_local = number of v in [0,n) with v mod W == rank.
 * The shard contents are undefined until the caller fills them through
 * wg_dsm_local_view and all ranks pass a barrier.
 * Errors: WG_ERR_INVALID_ARG, WG_ERR_UNSUPPORTED, WG_ERR_OOM, WG_ERR_PEER_ACCESS,
 * WG_ERR_COLLECTIVE, WG_ERR_CUDA.  On error *out is NULL and nothing leaks. */
wg_status wg_dsm_create(const wg_dsm_desc* desc, wg_dsm_t* out);

/* Device pointers of THIS rank's shard, for filling it (any stream; the caller
 * synchronises and barriers before other ranks read).  Any output may be NULL.
 * d_row_ptr: int64[n_local_rows + 1] local offsets (int64[num_nodes + 1] with
 * WG_DSM_CSR_REPLICATED); d_col_idx: the local CSR entries as int64, or as uint32 with
 * WG_DSM_COL32 (reinterpret the pointer); n_local_rows = feature rows of this rank.
 * feat_row_stride_bytes is the row pitch of the feature shard, which holds the first
 * body_bytes bytes of every row (wg_dsm_feat_layout; the whole row unless the layout is split). */
wg_status wg_dsm_local_view(wg_dsm_t h, int64_t** d_row_ptr, int64_t** d_col_idx, void** d_feat,
                            int64_t* n_local_rows, int64_t* feat_row_stride_bytes);

/* Feature-row layout of the shards (identical on every rank).  The B200 L2 fills whole
 * 128 B lines on a miss, so a row of R bytes with R > 128, R % 128 != 0 and R % 16 == 0 is
 * SPLIT: its first body_bytes = R - R % 128 bytes are stored in the feature shard
 * (wg_dsm_local_view's d_feat) at body_pitch = body_bytes, i.e. whole lines, and its last
 * R % 128 bytes at d_tail + l * tail_pitch (tail_pitch = R % 128) in a dense tail region of
 * THIS rank's slab.  Otherwise body_bytes = R, body_pitch = R rounded up to 64, d_tail = NULL
 * and tail_pitch = 0.  Fillers write bytes [0, body_bytes) of local row l at
 * d_feat + l * body_pitch and bytes [body_bytes, R) at d_tail + l * tail_pitch.  The layout is
 * invisible to every op (wg_gather returns whole rows).  The WG_DSM_WHOLE_ROWS flag at create
 * disables the split (A/B).  Any output may be NULL. */
wg_status wg_dsm_feat_layout(wg_dsm_t h, int64_t* body_bytes, int64_t* body_pitch, void** d_tail,
                             int64_t* tail_pitch);

/* Geometry of rank r's shard (any r): local feature rows and local CSR entries (with
 * WG_DSM_CSR_REPLICATED: the whole CSR's entries; its rows are num_nodes). */
wg_status wg_dsm_shard_info(wg_dsm_t h, int32_t r, int64_t* n_local_rows, int64_t* local_num_edges);

/* A second handle on the SAME shards with its own workspace (hash table, scan
 * state, error word), so independent batches can be prepared concurrently on
 * different streams (each handle's calls stay on one stream at a time).  Not
 * collective; no memory is mapped or copied.  max_batch_keys = 0 copies the
 * parent's.  Destroy forks (wg_dsm_destroy, not collective for a fork) before
 * their parent. */
wg_status wg_dsm_fork(wg_dsm_t parent, int64_t max_batch_keys, wg_dsm_t* out);

/* Destroy (COLLECTIVE): barrier (no rank still reads a peer), close the peer
 * mappings, barrier (no peer still maps ours), free the shard and workspace.
 * The caller must have synchronised every stream that used the handle. */
wg_status wg_dsm_destroy(wg_dsm_t h);

/* Multi-GPU sampling op, one hop (Algorithm 1).
 * For target k (in input order) with N = deg(d_targets[k]) read from the owner's
 * row_ptr (local HBM or a peer's over NVLink):
 *   - if fanout >= N: all N neighbours, in CSR order ("all of N neighbors are
 *     sampled", L118; A5);
 *   - else: fanout neighbours drawn without replacement by Algorithm 1 with draw
 *     r_i = floor(x_i * (N-i) / 2^32), x_i = word (i & 3) of Philox4x32-10 at
 *     counter (i>>2, hop, lo32(node), hi32(node)) under key (lo32(seed),
 *     hi32(seed)) (A2, A3), output in draw order i = 0..fanout-1 (A5).
 * Outputs: d_out_row_ptr int64[n_targets+1] = exclusive prefix of min(fanout, N)
 * (the sub-graph CSR row pointer, L166); d_out_nbrs int64[cap n_targets*fanout]
 * = sampled global ids; d_out_pos int32[same] (nullable) = positions in the
 * adjacency list; d_out_num_edges (nullable) = device int64 total.
 * seed: the per-batch rng_seed; if d_seed is non-NULL the seed is read from that
 * device uint64 instead (so a captured CUDA graph can be replayed with new seeds).
 * Requires 1 <= fanout <= WG_MAX_FANOUT (WG_ERR_UNSUPPORTED above) and n_targets * fanout
 * <= max_batch_keys (the padded per-target slots live in the workspace).  fanout <= 32:
 * a warp lane group per target with a sort-free form of Algorithm 1; fanout > 32: a
 * block of next_pow2(fanout) threads per target running Algorithm 1 as listed, with
 * a bitonic block sort as parallel_sort (L118-120).  Both give identical results. */
wg_status wg_sample_neighbors(wg_dsm_t h, const int64_t* d_targets, int64_t n_targets,
                              const int64_t* d_n_targets, int32_t fanout, uint64_t seed,
                              const uint64_t* d_seed, int32_t hop, int64_t* d_out_row_ptr,
                              int64_t* d_out_nbrs, int32_t* d_out_pos, int64_t* d_out_num_edges,
                              wg_stream_t stream);

/* Append Unique op: U = the targets first, in input order,
 * with their index as sub-graph id (L160, L166), then every neighbour id not seen
 * before, numbered continuously after the targets in order of first appearance
 * in d_nbrs (A7; the paper's hash-bucket order is nondeterministic).  A
 * neighbour equal to a target takes the target's id (A9).  Duplicate targets
 * latch WG_DEVERR_DUP_TARGET (A8).
 * Outputs: d_out_unique int64[cap n_targets+n_nbrs]; d_out_num_unique device
 * int64 (nullable); d_out_sub_col int32[n_nbrs] = sub-graph id of each sampled
 * neighbour (with d_out_row_ptr of the sampling op this is the sub-graph CSR,
 * L166); d_out_dup_count int32[cap n_targets+n_nbrs] (nullable) = how many
 * times each sub-graph node was sampled as a neighbour (the duplicate count, L186).
 * Requires n_targets + n_nbrs <= max_batch_keys and < 2^31. */
wg_status wg_append_unique(wg_dsm_t h, const int64_t* d_targets, int64_t n_targets,
                           const int64_t* d_n_targets, const int64_t* d_nbrs, int64_t n_nbrs,
                           const int64_t* d_n_nbrs, int64_t* d_out_unique, int64_t* d_out_num_unique,
                           int32_t* d_out_sub_col, int32_t* d_out_dup_count, wg_stream_t stream);

/* One whole hop of mini-batch preparation = wg_sample_neighbors followed by
 * wg_append_unique on its output ("stacking multiple
 * single-layer sub-graph sampling"), with identical results, fused for B200: the
 * sampling kernel writes padded per-target slots without any scan, the insert
 * pass of Append Unique reads them directly, and ONE single-pass scan both
 * compacts the sampler output into the CSR (row_ptr, neighbours, positions) and
 * numbers the first occurrences -- four kernels, no host sync (three with the
 * direct key table, wg_dsm_unique_format: the sampler inserts every key itself and
 * there is no insert pass).  The relabel
 * (which fills d_out_sub_col / d_out_dup_count) is launched on side_stream when
 * it is non-NULL (forked from `stream` with an event); the caller must make its
 * consumers wait for side_stream, and must join it before issuing a fifth
 * append-unique on the handle (the workspace keeps a ring of 4 scan buffers).
 * Arguments are those of the two calls; n_nbrs = n_targets * fanout and the
 * neighbour count is d_out_num_edges (required here).  Requires
 * n_targets * (1 + fanout) <= max_batch_keys. */
wg_status wg_sample_hop(wg_dsm_t h, const int64_t* d_targets, int64_t n_targets, const int64_t* d_n_targets,
                        int32_t fanout, uint64_t seed, const uint64_t* d_seed, int32_t hop, int64_t* d_out_row_ptr,
                        int64_t* d_out_nbrs, int32_t* d_out_pos, int64_t* d_out_num_edges, int64_t* d_out_unique,
                        int64_t* d_out_num_unique, int32_t* d_out_sub_col, int32_t* d_out_dup_count,
                        wg_stream_t stream, wg_stream_t side_stream);

/* Global gather: d_out[i][:] = the feature row of node
 * d_ids[i], in input order, read from the owner's shard (local HBM or a peer's
 * over NVLink) by one kernel ("a single gather kernel in each GPU", L182).  Rows
 * are copied as raw bytes: d_out is dense, row i at i * feat_dim * elt_size.
 * Repeated ids are allowed. */
wg_status wg_gather(wg_dsm_t h, const int64_t* d_ids, int64_t n_ids, const int64_t* d_n_ids,
                    void* d_out, wg_stream_t stream);

/* ---- Distributed-memory global gather: the comparison baseline (PAPER.md L178-180,
 * Fig. 4 left, Fig. 10).  The caller drives the five steps with NCCL all-to-alls:
 *   1 wg_bucket_by_owner  2 all-to-all counts + ids  3 wg_gather on the received ids
 *   (all owned by this rank)  4 all-to-all features  5 wg_rows_permute.
 * wg_bucket_by_owner: d_counts int64[2*W] (first W = ids per owner rank; the rest is
 * scratch), d_bucketed_ids int64[n_ids] = the ids grouped by owner (rank 0's first; order
 * within a group unspecified), d_perm int64[n_ids] = position of input i in the grouped
 * array (-1 for an invalid id, which also latches WG_DEVERR_ID_RANGE).
 * wg_rows_permute: d_dst[i] = d_src[d_perm[i]] for rows of row_bytes (zeros for -1). */
wg_status wg_bucket_by_owner(wg_dsm_t h, const int64_t* d_ids, int64_t n_ids, const int64_t* d_n_ids,
                             int64_t* d_counts, int64_t* d_bucketed_ids, int64_t* d_perm, wg_stream_t stream);
wg_status wg_rows_permute(const void* d_src, void* d_dst, const int64_t* d_perm, int64_t n, int64_t row_bytes,
                          wg_stream_t stream);

/* ---- GNN layer op consuming the prepared mini-batch (III-C4) ----
 * g-SpMM with mean aggregation (GraphSAGE-mean message passing, Eq. (1)) on the
 * sub-graph CSR produced by one hop: rows = targets (d_row_ptr int64[n_rows+1], e.g.
 * wg_sample_hop's d_out_row_ptr), columns = sub-graph ids (d_sub_col int32), features
 * d_x float32 [*, dim] row-major (e.g. the gathered X viewed as float32; dim % 4 == 0).
 * forward:  d_y[t, :] = mean over the row's edges of d_x[sub_col[e], :] (0 for an empty
 *           row), fp32 accumulation in edge order.
 * backward: d_dx[c, :] = sum over edges t->c of d_dy[t, :] / deg(t), computed on the same
 *           CSR with atomic adds (no transpose, L186); rows with d_dup_count == 1 (the
 *           Append Unique duplicate count; nullable) are written with a plain store
 *           (L186-192).  d_dx [n_x_rows, dim] is zeroed by the call.
 * d_x has n_x_rows rows; an edge whose sub-graph id lies outside [0, n_x_rows) (the -1 of an
 * invalid id) is skipped in both directions.  d_n_rows: optional device count (as for the other ops). */
wg_status wg_spmm_mean_forward(const int64_t* d_row_ptr, int64_t n_rows, const int64_t* d_n_rows,
                               const int32_t* d_sub_col, const float* d_x, int64_t n_x_rows, int64_t dim, float* d_y,
                               wg_stream_t stream);
wg_status wg_spmm_mean_backward(const int64_t* d_row_ptr, int64_t n_rows, const int64_t* d_n_rows,
                                const int32_t* d_sub_col, const int32_t* d_dup_count, const float* d_dy,
                                int64_t dim, float* d_dx, int64_t n_x_rows, wg_stream_t stream);

/* DSM characterisation, the analogue of PAPER.md Table I (L66-80): one GPU thread
 * performs `accesses` dependent 8 B loads at random 64 B-aligned offsets within the
 * first span_bytes of rank `rank`'s feature shard (local HBM when rank is this rank,
 * a peer's HBM over NVLink otherwise); each address is the multiply-high of the previously
 * loaded value (times a constant) with the slot count: two dependent integer multiplies
 * (~4 ns) between a load's return and the next load.  The caller times the launch (e.g. with CUDA events) and divides by
 * `accesses`.  d_sink: one device uint64 receiving a checksum (keeps the loads live).
 * Errors: WG_ERR_INVALID_ARG if span_bytes exceeds that shard. */
wg_status wg_dsm_chase(wg_dsm_t h, int32_t rank, int64_t span_bytes, int64_t accesses, uint64_t* d_sink,
                       wg_stream_t stream);

/* Ceilings of the latency-bound prep kernels, measured on the box itself.
 * wg_micro_random_read: blocks_per_sm x SMs blocks of 256 threads, each thread `rounds` times issuing
 * 8 independent loads of `width` (8 or 32) bytes at hash-random width-aligned offsets of
 * [d_buf, d_buf + span_bytes) -- the random-sector rate bounding the sampler (S1-S2: row_ptr pairs and
 * col_idx entries at random rows).  wg_micro_atomics: the same shape of independent 64-bit atomics on
 * random words of d_table[slots] -- op 0 = a CAS that never swaps (a probe), 1 = a CAS that swaps, 2 =
 * atomicMin -- the L2 atomic rate bounding append-unique's insert pass (S3).  *loads_issued / *ops_issued
 * (nullable) receive the operation count of the launch; the caller times it (CUDA events) on `stream`.
 * d_sink: one device uint64 that keeps the results live.  d_table's contents are overwritten.
 * Errors: WG_ERR_INVALID_ARG (null pointer, width not 8/32, span < width, rounds < 1,
 * blocks_per_sm outside [1, 8], op outside [0, 2]). */
wg_status wg_micro_random_read(const void* d_buf, int64_t span_bytes, int32_t width, int32_t rounds,
                               int32_t blocks_per_sm, uint64_t* d_sink, int64_t* loads_issued, wg_stream_t stream);
wg_status wg_micro_atomics(uint64_t* d_table, int64_t slots, int32_t op, int32_t rounds, int32_t blocks_per_sm,
                           uint64_t* d_sink, int64_t* ops_issued, wg_stream_t stream);

/* wg_gather restricted to rows [*d_begin, *d_end) of d_ids / d_out (device int64 scalars;
 * d_begin NULL = 0, d_end NULL = n_ids; both clamped to [0, n_ids]).  Row i is written at
 * d_out + i * pitch, pitch = out_pitch (0 = dense, row_bytes).  A pitched output (a multiple
 * of 16 in (row_bytes, row pitch of the shard]) lets rows that are not a multiple of 32 B
 * move as whole 32 B vectors: bytes [row_bytes, pitch) of each output row are unspecified.  Because every hop's unique list is a prefix of the
 * next one (targets first, L160, L168-174), the rows a batch will gather become known hop by
 * hop: a caller may gather rows [|U_{h-1}|, |U_h|) while hop h+1 is still sampling. */
wg_status wg_gather_rows(wg_dsm_t h, const int64_t* d_ids, int64_t n_ids, const int64_t* d_begin,
                         const int64_t* d_end, void* d_out, int64_t out_pitch, wg_stream_t stream);

/* Occupancy of this handle's gather launches (wg_gather, wg_gather_rows): at most blocks_per_sm
 * resident 256-thread blocks per SM; 0 (the default) = the occupancy maximum, which keeps the most
 * bytes in flight and is fastest for a gather running alone.  When several batches are prepared
 * concurrently on one GPU (wg_dsm_fork), a smaller value leaves register file and warp slots to the
 * latency-bound sampling / append-unique kernels of the other streams so they overlap the gather
 * (measured in DESIGN.md).  Read when a gather is enqueued (so a captured CUDA graph keeps the value
 * it was captured with); results never depend on it.  Errors: WG_ERR_INVALID_ARG if h is NULL or
 * blocks_per_sm < 0. */
wg_status wg_dsm_set_gather_occupancy(wg_dsm_t h, int32_t blocks_per_sm);

/* Read (and optionally clear) the latched device error word.  Synchronises the
 * handle's device. */
wg_status wg_device_error(wg_dsm_t h, uint32_t* code, int32_t clear);

/* Clear the append-unique hash table (and the direct tables) and restart its epoch counter.  Stream-ordered.
 * Needed only with the wide 16 B table format (node ids or positions >= 2^28, or
 * WG_DSM_WIDE_HASH) after WG_DEVERR_EPOCH, i.e. after ~8M append-unique calls; the compact
 * 8 B format cycles through 255 epochs and clears itself when a cycle restarts. */
wg_status wg_dsm_reset_workspace(wg_dsm_t h, wg_stream_t stream);

/* The Append Unique key-table format of h's workspace: WG_UNIQUE_WIDE / _COMPACT / _DIRECT; and
 * (hop_insert_pass, nullable) 1 if wg_sample_hop runs a separate insert pass (the hashed formats), 0 if
 * its sampler inserts the keys (the direct format).  Errors: WG_ERR_INVALID_ARG if h or format is
 * NULL. */
wg_status wg_dsm_unique_format(wg_dsm_t h, int32_t* format, int32_t* hop_insert_pass);

/* Diagnostics (per-kernel device times): while set, wg_sample_hop records events[0..n)
 * in order after its kernels -- sampler, insert, flag scan, relabel (the relabel's on the side stream
 * when one is given; without an insert pass (wg_dsm_unique_format): sampler, flag scan, relabel) --
 * and wg_append_unique after insert, flag scan, relabel.  events are cudaEvent_t
 * handles owned by the caller; n = 0 clears.  Use with eager launches (not inside a graph capture).
 * Errors: WG_ERR_INVALID_ARG if n is outside [0, 8] or events is NULL with n > 0. */
wg_status wg_dsm_set_stage_events(wg_dsm_t h, void* const* events, int32_t n);

/* Test hook: set the hash-table epoch counter of h's workspace (synchronous), e.g. near the end
 * of the wide format's 2^23 epochs or of the compact format's 255-epoch cycle, so tests reach
 * WG_DEVERR_EPOCH and the cycle restart in a few calls.  Errors: WG_ERR_INVALID_ARG if epoch is
 * 0 or >= 2^23. */
wg_status wg_dsm_debug_set_epoch(wg_dsm_t h, uint32_t epoch);

/* Thread-local message describing the last non-OK status. */
const char* wg_last_error(void);

/* Library version string. */
const char* wg_version(void);

#ifdef __cplusplus
}
#endif

#endif /* WG_H_ */
