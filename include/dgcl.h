/* dgcl.h — C ABI of the B200-native DGCL halo-exchange library (libdgcl.so).
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:n" = line n):
 *   DGCL's data-parallel hot path: executing a communication plan for GNN embedding passing.
 *   - graphAllgather forward (§4.2): after the call every GPU d holds, in its halo, the
 *     embedding row of every remote vertex it requires (V^r_d of §4.1).
 *   - its backward (§2; §6.1; §6.2): gradients of the halo rows
 *     flow back along the reversed plan and are summed into the owner rows in a fixed order, with
 *     no atomics.
 *   - the plan is built once by SPST (Algorithm 1 + 2, §5.2) over a link-cost model of
 *     the topology (§5.1) and reused by every layer.
 *
 * Conventions (every function):
 *   - returns dgcl_status; no exception crosses the ABI; dgcl_last_error(ctx) explains failures;
 *   - one context per rank, used by one host thread;
 *   - host pointers are read during the call only and never retained unless stated;
 *   - device pointers are caller-owned unless stated; the library never frees caller memory;
 *   - `stream` arguments are cudaStream_t passed as void* (0 = legacy default stream);
 *   - embeddings are fp32 rows; pitches are in ELEMENTS (floats); dims[l] >= 1.
 *
 * Row layouts:
 *   local rows   loc[v] = number of w < v with part[w] == part[v]  (ascending global id, §4.1)
 *   halo rows    halo_d[i] = embedding of R_d[i], R_d in the order the caller gave to
 *                dgcl_build_plan (the paper leaves the re-indexed order open)
 *   LOOPBACK contexts (all `world` virtual ranks on one GPU; test/bench, §8(d) "1-GPU loopback"):
 *                emb / emb_grad are [N x pitch] partition-major: rank r's local rows start at row
 *                sum_{q<r} n_local[q];  halo / halo_grad are [sum_d |R_d| x pitch], rank d's block
 *                starts at row sum_{q<d} |R_q|.
 */
#ifndef DGCL_H_
#define DGCL_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  DGCL_OK = 0,
  DGCL_EINVAL = 1,   /* bad argument (range, duplicate, alignment, pitch < dim, ...) */
  DGCL_ESTATE = 2,   /* call out of order (e.g. dispatch before build_plan/register) */
  DGCL_ECUDA = 3,    /* a CUDA runtime/driver call failed (or no usable GPU) */
  DGCL_ENOMEM = 4,   /* host or device allocation failed / workspace too small */
  DGCL_ETIMEOUT = 5, /* a device-side flag wait exceeded the watchdog (a peer never arrived) */
  DGCL_EPLAN = 6     /* planning failed: some requesting GPU is unreachable in the topology */
} dgcl_status;

typedef struct dgcl_ctx dgcl_ctx;

/* Loopback flags (dgcl_init_loopback). */
#define DGCL_LOOPBACK_FUSED 0    /* one executor launch runs every virtual rank's program */
#define DGCL_LOOPBACK_PER_RANK 1 /* one launch per virtual rank on its own stream, with the full
                                    ready/done flag protocol of the multi-GPU path (test mode) */

/* Topology D(V', E') of §5.1: ordered GPU pairs (i, j) map to lists of
 * physical hops; hop h costs hop_ticks[h] (> 0) per embedding row.  A pair with an empty hop list
 * has no link.  link_ptr is CSR over pair index i*world + j (size world*world + 1). */
typedef struct {
  int32_t n_hops;
  const int64_t *hop_ticks; /* [n_hops] */
  const int64_t *link_ptr;  /* [world*world + 1] */
  const int32_t *link_hops; /* [link_ptr[world*world]] hop ids */
} dgcl_topology;

typedef struct {
  int32_t world;
  int32_t n_stages;            /* forward stages K (<= world-1) */
  int64_t n_vertices_planned;  /* |{u : D_u non-empty}| */
  int64_t n_deliveries;        /* sum_d |R_d| */
  int64_t n_tree_edges;        /* sum_u |T_u| edges (>= n_deliveries; excess = relay hops) */
  int64_t n_relay_rows;        /* tree edges into GPUs that did not request the vertex */
  int64_t model_cost_ticks;    /* t(S) of §5.1 in ticks */
  int64_t table_bytes;         /* device bytes of send/receive index tables (Fig. 11) */
  double planner_seconds;      /* SPST wall time, one host thread (Table 8) */
  double lowering_seconds;
  int32_t n_fwd_groups;        /* (stage, src, dst, buffer-kind) tuples */
  int32_t n_bwd_groups;
  int64_t n_multicast_rows;    /* rows sent through the NVSwitch multicast (option "multicast") */
} dgcl_plan_stats;

/* ---- lifecycle ---------------------------------------------------------------------------- */

/* One rank of a `world`-GPU job (§6.3 one process per GPU).
 * part: host [n_vertices], part[v] in [0, world), copied.  dims: host [n_layers], fp32 elements per
 * row of each layer; one plan serves every layer.  cuda_device < 0 makes a host-only
 * planning context (every device call then returns DGCL_ESTATE).  Builds loc / n_local (§4.1).
 * Errors: EINVAL (rank >= world, world < 1 or > 16, n_layers < 1, dims[l] < 1, part out of range),
 * ECUDA (cudaSetDevice failed). */
dgcl_status dgcl_init(int32_t rank, int32_t world, int32_t cuda_device, int64_t n_vertices,
                      const int32_t *part, int32_t n_layers, const int32_t *dims, dgcl_ctx **out);

/* All `world` virtual ranks in one context on one GPU (the 1-GPU loopback configuration).
 * flags: DGCL_LOOPBACK_FUSED or DGCL_LOOPBACK_PER_RANK.  Same errors as dgcl_init. */
dgcl_status dgcl_init_loopback(int32_t world, int32_t cuda_device, int64_t n_vertices,
                               const int32_t *part, int32_t n_layers, const int32_t *dims,
                               int32_t flags, dgcl_ctx **out);

/* Optional, before dgcl_build_plan; default = uniform NVSwitch (link i->j = {egress_i, ingress_j},
 * 900 GB/s each, 111 ticks per row).  Copied.  EINVAL for bad hop ids / ticks, ESTATE after plan. */
dgcl_status dgcl_set_topology(dgcl_ctx *ctx, const dgcl_topology *topo);

/* Build the communication plan (buildCommInfo; Algorithm 1).
 * Collective in the sense that every rank must pass ALL ranks' required lists (the Python wrapper
 * all-gathers them) and the same seed, so every rank computes the identical plan without a master.
 * req_ptr: host [world+1]; req_ids: host [req_ptr[world]]; R_d = req_ids[req_ptr[d]:req_ptr[d+1]]
 * in GPU d's halo row order.  Host work only (no device memory is touched).
 * Errors: EINVAL (id out of range, id owned by the requester, duplicate id in one list),
 * EPLAN (unreachable GPU), ESTATE (called twice), ENOMEM. */
dgcl_status dgcl_build_plan(dgcl_ctx *ctx, const int64_t *req_ptr, const int64_t *req_ids,
                            uint64_t seed);

/* Build the plan from saved trees instead of running SPST (checkpoint/resume of the planning
 * step: the plan is made once before training, and SPST costs seconds to minutes at
 * scale, Table 8).  The trees are the tuples dgcl_plan_export returns — edge e =
 * (u[e], parent[e], child[e], stage[e]), all host arrays of n_edges entries, the edges of one
 * vertex contiguous and in root-to-leaf order (a parent is u's owner or an earlier child).  The
 * same relation checks as dgcl_build_plan, then the plan invariants of the oracle:
 * every vertex some GPU requests has exactly one tree, rooted at its owner, reaching every
 * requester over existing links, stage = tree depth <= world-1, no leaf that did not request
 * it; t(S) is recomputed (dgcl_plan_info).  Errors: as dgcl_build_plan; EPLAN for an invalid
 * tree (dgcl_last_error says which edge / vertex); EINVAL for NULL arrays with n_edges > 0. */
dgcl_status dgcl_build_plan_from_trees(dgcl_ctx *ctx, const int64_t *req_ptr,
                                       const int64_t *req_ids, int64_t n_edges, const int64_t *u,
                                       const int32_t *parent, const int32_t *child,
                                       const int32_t *stage);

/* Device workspace.  The caller allocates ONE device buffer of at least *bytes bytes, 256-B
 * aligned (PyTorch does), keeps it alive until dgcl_destroy, and registers it.  The library carves
 * out halos (one per layer), relay staging, backward gradient slots and flag words, zeroes the flag
 * words (synchronously) and uploads the plan tables (library-owned device memory).
 * Errors: ESTATE (no plan / host-only ctx), EINVAL (misaligned), ENOMEM (too small), ECUDA. */
dgcl_status dgcl_workspace_bytes(dgcl_ctx *ctx, size_t *bytes);
dgcl_status dgcl_register_workspace(dgcl_ctx *ctx, void *dev, size_t bytes);

/* Where the halo of `layer` lives inside the registered workspace: byte offset, rows (|R_me|, or
 * sum_d |R_d| for loopback), pitch in elements (dims[layer] rounded up to a multiple of 4). */
dgcl_status dgcl_halo_view(dgcl_ctx *ctx, int32_t layer, size_t *offset, int64_t *rows,
                           int64_t *pitch);

/* Per-rank row counts: n_local[world], n_halo[world] (= |R_d|).  Host arrays filled by the call. */
dgcl_status dgcl_rank_rows(dgcl_ctx *ctx, int64_t *n_local, int64_t *n_halo);

/* Peer mapping over NVLink (CUDA IPC; the B200 form of §6.2 method (1)).
 * export: writes this rank's opaque blob (IPC handle of the workspace allocation + offset) into
 * blob (capacity *len on entry; bytes written on return; DGCL_IPC_BLOB_BYTES always suffices).
 * import: blobs = world blobs of len_each bytes, in rank order (own entry ignored); maps every
 * peer workspace.  The caller must barrier all ranks after import and before the first dispatch.
 * Errors: ESTATE (no workspace), EINVAL (bad blob), ECUDA (peer mapping impossible). */
#define DGCL_IPC_BLOB_BYTES 256
dgcl_status dgcl_ipc_export(dgcl_ctx *ctx, void *blob, size_t *len);
dgcl_status dgcl_ipc_import(dgcl_ctx *ctx, const void *blobs, size_t len_each);

/* ---- the hot path ------------------------------------------------------------------------- */

/* graphAllgather forward for `layer` (plan tuples of §6.1).
 * emb: device [n_local x emb_pitch] (loopback: [N x emb_pitch], partition-major), caller-owned,
 * local, read-only during the call.  halo: NULL or the registered view for `layer` (EINVAL
 * otherwise).  Enqueues on `stream`, returns without a host sync; a collective (every rank calls it
 * with the same layer sequence).  After the stream reaches this point:
 *   halo[i][0:dim] == emb_global[R_me[i]][0:dim]   bit-exactly.
 * Errors: EINVAL (layer, pitch < dim), ESTATE (not registered / not imported), ETIMEOUT (an
 * earlier call's watchdog fired; the context is unusable), ECUDA (launch failed). */
dgcl_status dgcl_dispatch_forward(dgcl_ctx *ctx, int32_t layer, const float *emb,
                                  int64_t emb_pitch, float *halo, void *stream);

/* Backward of graphAllgather for `layer`: the adjoint (stages reversed, send/receive tables
 * swapped), without atomics (§6.2).
 * halo_grad: device [|R_me| x hg_pitch] (loopback [sum_d |R_d| x hg_pitch]), caller-owned, local.
 * emb_grad: device in/out [n_local x eg_pitch] (loopback [N x eg_pitch]).  On completion
 *   emb_grad[loc u] = ((emb_grad_in[loc u] + val(y1)) + val(y2)) + ...
 * over u's tree children y1 < y2 < ... (ascending GPU id), where a child's val is its own halo
 * gradient (if it requested u) followed by its own children's vals, ascending (R6).
 * For single-stage (direct) plans this is  emb_grad_in + G_c1 + G_c2 + ... , c ascending.
 * Rows of vertices nobody requested are untouched.  Same errors as dispatch_forward. */
dgcl_status dgcl_dispatch_backward(dgcl_ctx *ctx, int32_t layer, const float *halo_grad,
                                   int64_t hg_pitch, float *emb_grad, int64_t eg_pitch,
                                   void *stream);

/* End-to-end variants with HOST buffers (pinned or pageable): copy the input rows host->device
 * into library-owned staging (one buffer per layer and input), dispatch on `stream`, copy the
 * result device->host, then synchronize `stream`.  The two copies run on library-owned copy
 * streams, ordered against `stream` by events, so with option "host_async" = 1 (no synchronize;
 * the host result is complete once `stream` is synchronized, and the host buffers must stay
 * valid until then) the input copy of the next call overlaps the output copy of this one.
 * forward:  host_emb [rows x pitch] -> host_halo [halo rows x pitch] (pitch = the halo view pitch)
 * backward: host_halo_grad [halo rows x pitch] and host_emb_grad in/out [rows x pitch].
 * Errors: as the device variants, plus ENOMEM for staging. */
dgcl_status dgcl_forward_host(dgcl_ctx *ctx, int32_t layer, const float *host_emb,
                              float *host_halo, void *stream);
dgcl_status dgcl_backward_host(dgcl_ctx *ctx, int32_t layer, const float *host_halo_grad,
                               float *host_emb_grad, void *stream);

/* ---- introspection ----------------------------------------------------------------------- */

dgcl_status dgcl_plan_info(dgcl_ctx *ctx, dgcl_plan_stats *info);

/* Forward rows per (stage k in 1..n_stages, src, dst): rows[((k-1)*world + src)*world + dst];
 * caller provides n_stages*world*world int64.  Relay rows included (bytes = rows*dim*4). */
dgcl_status dgcl_plan_counts(dgcl_ctx *ctx, int64_t *rows);

/* Tree edges of the plan (§5.1 T_u) as (u, parent, child, stage) in planning order.
 * Two-call pattern: pass NULL arrays to get *n_edges, then arrays of that size. */
dgcl_status dgcl_plan_export(dgcl_ctx *ctx, int64_t *n_edges, int64_t *u, int32_t *parent,
                             int32_t *child, int32_t *stage);

/* Options (before dgcl_register_workspace unless noted):
 *   "timeout_ms"     device watchdog for flag waits (default 20000; any time)
 *   "item_bytes"     target bytes of gathered operands per work item (default/max 98304)
 *   "tma"            1 (default): bulk-copy (cp.async.bulk) gather executor when rows are 16-B
 *                    aligned; 0: the register (LDG/STG) executor
 *   "ctas_per_sm"    executor CTAs per SM (default: occupancy, max 4)
 *   "threads"        executor CTA size (128..512, multiple of 32; default 512)
 *   "gather4"        1 (default): TMA tile::gather4 (four rows per instruction) for short-run
 *                    row gathers (embeddings, halos, relay staging, halo gradients), rows <= 1 KB
 *   "stage_fold"     1 (default): backward folds bulk-copy all their operand rows into shared
 *                    memory (segments of consecutive rows) before adding them; 0: consumers
 *                    gather the operands with plain loads
 *   "pipeline_blocks" relay plans: vertex blocks of the stage chaining (1..8, default 1): stage k
 *                    of a block waits only for stage k-1 of the same block, so consecutive stages
 *                    may overlap; 1 = one done counter per (stage, source) as in §6.1.  Measured
 *                    slower with more blocks on one B200 (smaller groups and items)
 *   "leaf_split"     relay plans: 1 (default) the deliveries of stages >= 2 that no later stage
 *                    forwards count on done counters of their own (nothing but the forward
 *                    completion waits on them) and follow the stage's forwarded rows, so stage k+1
 *                    starts once stage k's forwarded rows landed; 2 stage 1 too; 0 off
 *   "relay_lead_kb"  relay plans with the leaf split: the forwarded rows of every stage run ahead
 *                    of the leaves — after stage k's forwarded items come about this many KB of
 *                    leaf rows (any stage <= k), then stage k+1's forwarded items, the remaining
 *                    leaves last (default 196608; -1 = stage-major build order)
 *   "dual_producer"  1 (default): launches of plain copies (no waits, no signals, no gather4,
 *                    round-robin items) run two producer warps per CTA that split the items;
 *                    0: one producer (any time)
 *   "dual_claims"    1 (default): dual producers also for launches whose items are claimed
 *                    dynamically (each producer claims its own batches; stage uses from a shared
 *                    counter); 0: such launches keep one producer (any time)
 *   "owner_major"    fused loopback: 1 (default) the forward COPY items of one owner's groups (its
 *                    embeddings to each receiver) run together, owner after owner — the write
 *                    front is a few long runs of halo rows and the owner's rows stay in L2 for
 *                    its receivers; 0: chunk c of every (owner, receiver) group together
 *   "align_sources"  1 (default): the forward COPY groups that read one rank's embeddings (one per
 *                    receiver) are cut into items at common source rows, so the copies of a row
 *                    to its receivers run close together (L2 reuse; rows <= 1 KB); 0: independent
 *                    cuts
 *   "fanout"         0 (default) / 1: forward stage 1 as one fan-out item stream per owner — each
 *                    embedding row read once and stored into every first-hop receiver's row
 *                    (kernel-level communication fusion) — instead of one COPY group
 *                    per (owner, receiver).  Same result; measured slower on one B200 (the
 *                    per-pair groups write long contiguous destination runs with TMA stores)
 *   "atomic_backward" 0 (default) / 1: ABLATION ONLY (the paper's "Atomic" baseline, Table 9
 *                    P:2531-2537): a fused loopback with a single-stage plan runs the backward as
 *                    requesters adding their halo-gradient rows into the owners' rows with atomic
 *                    reductions (TMA bulk reduce-add).  The sum is the same but its order is not
 *                    fixed, so results may differ from the fixed-order fold in the last bits
 *   "direct_reduce"  1 (default): fused loopback with a single-stage plan folds the requesters'
 *                    halo gradients in place (no slot round trip); 0: push + owner reduce
 *   "direct_copy_rows" COPY items whose runs average fewer rows are gathered by the consumer
 *                    warps with plain loads (default 0 = never)
 *   "trace"          1: record per-item timelines of every launch (dgcl_trace_read); default 0
 *   "l2_policy"      L2 eviction hints of the bulk-copy executor, bit mask (any time): 1 data stores
 *                    evict_first (default), 2 COPY source reads evict_last, 4 COPY source reads
 *                    evict_first, 8 FOLD operand reads evict_first
 *   "claim_batch"    bulk-copy executor item assignment (any time): -1 (default) auto = dynamic
 *                    claiming in batches of 4 for relay forwards, of 2 for jobs of <= 4 ranks,
 *                    round-robin otherwise; 0 round-robin everywhere; k >= 1 batches of k
 *   "sys_scope"      loopback contexts: 1 = use the multi-GPU system-scope flag protocol (A/B;
 *                    default 0: device scope, exact when every rank is on this GPU)
 *   "multicast"      NVSwitch multicast of high-fan-out rows (see dgcl_multicast_open): 0 off
 *                    (default), 1 rows every peer requested, k >= 2 rows >= k GPUs requested
 *   "sm_budget"      SMs one executor launch may use (default 0 = all; any time): leaves SMs free
 *                    for kernels that overlap the exchange (dgcl_stream_wait_arrival)
 *   "signal_all"     fused loopback: every item publishes its done count, so arrival waits work
 *                    (default 0: only counts some item of the launch waits on)
 *   "small_launch_bytes" launches moving fewer bytes (rows x row size) run the register
 *                    executor instead of the bulk-copy pipeline (latency; default 4 MiB, 0 = never)
 *   "host_async"     0 (default) / 1: dgcl_forward_host / dgcl_backward_host return before the
 *                    device->host copy completes (any time)
 *   "geometry"       bulk-copy launch geometry: 0 (default) auto per launch, 1 WIDE (1 CTA per
 *                    SM, 4 x 48 KB stages), 2 DUAL (2 CTAs per SM, 2 x 47 KB stages)
 *   "bulk_store", "bulk_store_peer"  TMA stores for packed contiguous destinations in local HBM
 *                    (default 1) / peer memory (default 0)
 * Options other than "timeout_ms", "debug_skip_rank" and "host_async" must be set before
 * dgcl_register_workspace (ESTATE otherwise).
 *   "debug_skip_rank" fault injection for DGCL_LOOPBACK_PER_RANK contexts: never launch that
 *                    virtual rank's program, so its peers' flag waits hit the watchdog (any time;
 *                    -1 = off)
 * EINVAL for an unknown key or bad value. */
dgcl_status dgcl_set_option(dgcl_ctx *ctx, const char *key, int64_t value);

/* Per-item timeline of the LAST launch of program (layer, dir = 0 forward / 1 backward, rank =
 * the virtual rank for per-rank loopback contexts, ignored otherwise), recorded when option
 * "trace" was set before dgcl_register_workspace (ESTATE otherwise).  One record per work item
 * in launch order: %globaltimer ns when the executor reached it, when its source waits (stage
 * chaining, ready words) were satisfied, and when its rows were stored; the SM that ran it.
 * recs == NULL: *n = number of records.  Synchronizes the device. */
typedef struct dgcl_trace_rec {
  uint64_t t_start, t_ready, t_done;
  uint32_t sm, tag;  /* op | dir << 4 | exec rank << 8 | dst rank << 16 | stage << 24 (5 bits)
                        | vertex block << 29 (option "pipeline_blocks") */
} dgcl_trace_rec;
dgcl_status dgcl_trace_read(dgcl_ctx *ctx, int32_t layer, int32_t dir, int32_t rank,
                            dgcl_trace_rec *recs, int64_t *n);

/* Device start barrier over the ranks (timing protocol of SURVEY.md §8(d) / a13; PAPER.md times
 * communication "after warm-up", averaged over 10 runs): a one-warp kernel on
 * `stream` in which this rank releases arrived[rank] = n into every peer's flag region (n = this
 * context's barrier call count) and acquire-waits until every peer's arrived word reaches n.  Work
 * queued after it on `stream` starts only once all ranks have reached the same barrier call.  A
 * collective: every rank calls it the same number of times.  Loopback contexts run all virtual
 * ranks in the one warp.  world == 1: no-op.  Errors: DGCL_ESTATE before registration / import;
 * a peer that never arrives trips the watchdog (dgcl_check -> DGCL_ETIMEOUT). */
dgcl_status dgcl_device_barrier(dgcl_ctx *ctx, void *stream);

/* Arrival wait for overlapping work (the paper runs graph operations
 * after graphAllgather returns, P:1554-1566 — this lets them start per source instead).
 * Enqueues on `stream` a one-warp kernel that acquire-waits until rank `dst` (this rank; any
 * virtual rank in loopback; -1 = this rank) has received, in the most recent dgcl_dispatch_forward
 * call, every row that comes from rank `src` (single-stage plans: src's stage-1 done counter), or
 * — for relay plans, or src = -1 — every incoming row of every stage.  Work queued after it on
 * `stream` may read those halo rows while the exchange is still running on the dispatch stream.
 * Use with option "sm_budget" < the SM count so that the overlapped kernels find free SMs.
 * Fused loopback contexts need option "signal_all" (set before registration).  Errors: EINVAL
 * for a bad (dst, src), ESTATE before registration / without signal_all; a row that never
 * arrives trips the watchdog (dgcl_check -> DGCL_ETIMEOUT).  No forward call yet: no-op. */
dgcl_status dgcl_stream_wait_arrival(dgcl_ctx *ctx, int32_t dst, int32_t src, void *stream);

/* ---- NVSwitch multicast (the switch-level form of the paper's
 * communication fusion, and of "forward to multiple destinations") ----
 * With option "multicast" (1: rows every peer requested; k >= 2: rows >= k GPUs requested; set
 * before dgcl_build_plan or re-lowered on set; single-stage plans only) the owner of such a row
 * stores it ONCE through a multicast address (multimem.st): the NVSwitch replicates the write into
 * every GPU's copy of a multicast region bound at the same offset (row mc_off[owner] + j), one
 * multimem reduction bumps the owner's multicast done counter on every GPU, and each requester
 * copies the row from its own region into its halo row (unpack, local HBM).  Owner egress drops
 * from |D_u| row copies to one; the ingress bound is unchanged.  The backward keeps the fixed-order
 * reduce (multimem.ld_reduce has no fixed order).  Setup, after dgcl_ipc_import, collective:
 *   dgcl_multicast_open  rank 0 creates the object (cuMulticastCreate, POSIX fd handle) and returns
 *                        *fd; every other rank passes that fd (received over a Unix socket:
 *                        the Python setup does it) and imports it;
 *   dgcl_multicast_add   every rank adds its device;    -- barrier --
 *   dgcl_multicast_bind  every rank binds its memory and maps the unicast + multicast views.
 * Loopback contexts emulate the multicast (one store per virtual rank's region copy, in the
 * workspace).  Errors: ECUDA when the device has no multicast support (probe with
 * dgcl_multicast_supported) or a driver call fails; ESTATE on a wrong order; dispatch refuses a
 * multi-GPU context whose plan multicasts before dgcl_multicast_bind. */
dgcl_status dgcl_multicast_supported(int32_t cuda_device, int32_t *supported);
dgcl_status dgcl_multicast_bytes(dgcl_ctx *ctx, size_t *bytes, int64_t *rows);
dgcl_status dgcl_multicast_open(dgcl_ctx *ctx, int32_t *fd);
dgcl_status dgcl_multicast_add(dgcl_ctx *ctx);
dgcl_status dgcl_multicast_bind(dgcl_ctx *ctx);
/* Verification aid: a one-device multicast object on `cuda_device` (bytes of region), stores and
 * a reduction through the multicast address, checked through the unicast view.  Writes a one-line
 * result into msg.  DGCL_ECUDA if unsupported. */
dgcl_status dgcl_debug_multicast_selftest(int32_t cuda_device, int64_t bytes, char *msg,
                                          size_t msg_len);
/* Verification aid (loopback contexts, host only, no device needed): runs the work items of
 * (layer, direction) — the fused program, or every virtual rank's program — through the flag
 * protocol of P:1447-1466 on the host: items in list order, each only once the counters it waits
 * on reached their targets, signals applied at its end.  Checks that every wait target equals the
 * rows ever signalled on its counter, that the programs cannot deadlock, that every source row
 * written in the same launch (halo / relay staging / slots / multicast copy) is read only by an
 * item that waits on its writer's counter, that no row is written twice, and (forward) that
 * every halo row is written.  mutate 1..4 checks a deliberately broken copy instead (the
 * checker's negative tests: 1 an item stops waiting, 2 an item moves before its producers, 3 a
 * data item repeats, 4 a producer stops signalling).  DGCL_EPLAN with the first violation in msg,
 * else DGCL_OK. */
dgcl_status dgcl_debug_check_protocol(dgcl_ctx *ctx, int32_t layer, int32_t direction,
                                      int32_t mutate, char *msg, size_t msg_len);

/* Number of executor kernel launches issued so far by this context. */
dgcl_status dgcl_launch_count(dgcl_ctx *ctx, uint64_t *count);

/* Device watchdog result: DGCL_ETIMEOUT if a flag wait expired (the context is then unusable),
 * DGCL_ECUDA on a sticky CUDA error, else DGCL_OK.  Does not synchronize the device. */
dgcl_status dgcl_check(dgcl_ctx *ctx);

const char *dgcl_last_error(dgcl_ctx *ctx);
const char *dgcl_strerror(dgcl_status status);

/* Unmaps peers, frees library-owned memory (tables, staging, streams), never the caller's
 * workspace.  Synchronizes the device first.  NULL is a no-op. */
dgcl_status dgcl_destroy(dgcl_ctx *ctx);

/* ---- verification aids (not on the dispatch path) --------------------------------------- */

/* Runs the lowered plan tables of a LOOPBACK context with a host interpreter (single thread, same
 * item order and fp32 fold order as the device executor), for CPU tests of planning + lowering
 * without a GPU.  Never called by dgcl_dispatch_*; there is no CPU fallback on the product path.
 * Buffers use the loopback layouts above with pitch = the halo view pitch of `layer`. */
dgcl_status dgcl_debug_hostsim_forward(dgcl_ctx *ctx, int32_t layer, const float *emb,
                                       float *halo);
dgcl_status dgcl_debug_hostsim_backward(dgcl_ctx *ctx, int32_t layer, const float *halo_grad,
                                        float *emb_grad);

#ifdef __cplusplus
}
#endif
#endif /* DGCL_H_ */
