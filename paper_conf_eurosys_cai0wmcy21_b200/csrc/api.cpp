// api.cpp — the C ABI (include/dgcl.h): context, plan, workspace, IPC, dispatch.
//
// PAPER.md references: API §4.2, buildCommInfo, client-side decentralised
// coordination §6.1, CUDA-VM peer method §6.2, process model §6.3
// (P:1535-1548).  B200 design: one process per GPU; each GPU's workspace (halos, relay staging,
// backward slots, flag words) is mapped by every peer over NVLink 5 / NVSwitch with CUDA IPC; one
// persistent executor launch per layer and direction runs every stage, chained by device flags.

#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <new>
#include <string>
#include <unordered_map>
#include <vector>

#include <map>

#include "dgcl.h"
#include "hostsim.h"
#include "plan.h"

using namespace dgcl;

namespace {

constexpr size_t kAlign = 256;
inline size_t align_up(size_t x, size_t a = kAlign) { return (x + a - 1) / a * a; }
inline int64_t pitch_of(int dim) { return (dim + 3) / 4 * 4; }

struct Program {
  // one launch: items for one (layer, direction, executing rank or -1 = fused loopback)
  std::vector<DevItem> items;
  std::vector<DevRun> runs;
  std::vector<uint32_t> sterms;  // staged FOLD items: operand row of every term
  size_t dev_off = 0;  // offset (in items) into the device item pool
  int op_mask = 0;     // kMaskCopy / kMaskFold / kMaskDirect / kMaskStaged items present
  bool fold_wide = false;  // FOLD rows average >= 4 terms
  int geo = 0;             // bulk-copy launch geometry: 0 = kGeoWide, 1 = kGeoDual, 2 = kGeoWide3
  int64_t bytes = 0;       // operand rows moved (rows x 16-B-rounded row, + fold terms)
  int g4_kinds = 0;        // source kinds of its gather4 items (tensor maps the launch needs)
  bool tree = false;       // carries tree-order FOLD programs (kTermRankTree)
  TraceRec *d_trace = nullptr;  // option "trace": per-item timeline of the last launch
  mutable uint64_t claims = 0;  // dynamic item claiming: the counter's value before the next launch
  bool relay_fwd = false;       // a forward program with stage chaining (waits on counters)
  bool simple_copy = false;     // COPY items only, no waits / signals
  int64_t max_meta = 0;         // largest producer metadata of one COPY item (runs / row window)
};

}  // namespace

struct dgcl_ctx {
  int rank = 0, world = 1, device = -1;
  bool loopback = false;
  int lb_flags = 0;
  int64_t n = 0;
  std::vector<int32_t> part;
  std::vector<int64_t> loc, n_local, row_off;
  int n_layers = 0;
  std::vector<int32_t> dims;
  std::vector<int64_t> pitch;  // halo pitch per layer (elements)
  int64_t max_pitch = 0;

  Topology topo;
  bool planned = false;
  Relation rel;
  Plan plan;
  Lowered low;
  std::vector<int64_t> halo_off;  // loopback: first halo row of each rank

  // workspace layout: per rank, byte offsets relative to that rank's base
  std::vector<size_t> off_flags, off_slot, ws_need;
  std::vector<std::vector<size_t>> off_halo, off_relay;  // [layer][rank]
  char *ws = nullptr;
  size_t ws_bytes = 0;
  std::vector<char *> base;  // per rank: workspace base (peer-mapped in multi-GPU mode)
  std::vector<char *> ipc_opened;
  bool registered = false, imported = false;

  // device tables
  DevGroup *d_groups = nullptr;
  DevWait *d_waits = nullptr;
  int32_t *d_idx = nullptr;
  int64_t *d_term_ptr = nullptr;
  uint32_t *d_terms = nullptr;
  DevItem *d_items = nullptr;
  DevRun *d_runs = nullptr;
  uint32_t *d_sterms = nullptr;
  uint64_t *d_claims = nullptr;  // one item-claim counter per program (dynamic claiming)
  // dynamic item claiming (bulk-copy executor): -1 auto (batches of 4 for relay forwards, of 2
  // for jobs of <= 4 ranks, else round-robin), 0 round-robin everywhere, k >= 1 batches of k
  int claim_batch = -1;
  bool lsu_gather = false;  // short-run COPY items gathered by consumer cp.async (A/B option)
  int64_t run_bytes = 0;
  bool bulk_store_local = true;   // TMA stores into local HBM (loopback)
  bool bulk_store_peer = false;   // TMA stores into peer memory over NVLink (not yet validated)
  std::vector<Program> progs;  // index prog_index(layer, dir, r)
  std::vector<int32_t> host_gids[2];  // group order of the host interpreter per direction
  bool direct_reduce = true;          // fused loopback + single-stage plan: in-place reduce
  bool atomic_backward = false;       // ablation: loopback backward with atomic adds
  bool fanout = false;                // forward stage 1 as per-owner fan-out items (option)
  // NVSwitch multicast (option "multicast": 0 off, 1 rows requested by every peer, k >= 2 rows
  // requested by >= k GPUs).  Multi-GPU: a multicast object over every rank's device with this
  // region bound at the same offset; loopback: emulated (one copy per virtual rank, workspace)
  int multicast = 0;
  std::vector<size_t> off_mc;   // loopback: each virtual rank's region copy in the workspace
  std::vector<size_t> mc_layer_off;  // byte offset of each layer's rows in the region
  size_t mc_bytes = 0;          // region bytes (flag page + every layer's rows)
  CUmemGenericAllocationHandle mc_handle = 0, mc_mem = 0;  // multicast object, bound memory
  bool mc_have_handle = false, mc_have_mem = false, mc_added = false;
  char *mc_va = nullptr, *mc_uc = nullptr;  // multicast / unicast mappings of the region
  size_t mc_map_bytes = 0;      // granularity-rounded size of the mappings
  bool align_sources = true;          // forward COPY items of one source rank cut at common rows
  int pipeline_blocks = 1;            // relay plans: vertex blocks of the stage chaining
  int leaf_split = 1;                 // relay plans: leaf deliveries after each stage's forwards
                                      // (A/B r2ab: 1 best; dgx1_like 0.721 -> 0.694 ms)
#ifndef DGCL_DUAL_PRODUCER_DEFAULT
#define DGCL_DUAL_PRODUCER_DEFAULT 1  // (build-time A/B of the sustained bench)
#endif
  bool dual_producer = DGCL_DUAL_PRODUCER_DEFAULT;  // simple launches: two producer warps
#ifndef DGCL_DUAL_CLAIMS_DEFAULT
#define DGCL_DUAL_CLAIMS_DEFAULT 1  // (A/B r2tk: Web-Google-4 forward on WIDE 0.416 -> 0.293 ms)
#endif
  bool dual_claims = DGCL_DUAL_CLAIMS_DEFAULT;  // ... also when their items are claimed dynamically
  int owner_major = 1;                // fused loopback forwards: one owner's groups at a time
                                      // (A/B r2sh: Reddit fwd602 -1 %, Com-Orkut -2.5 %,
                                      // Web-Google dgx1_like -6 %)
  int64_t relay_lead_kb = 196608;     // relay forwards: leaves between stages' forwarded items
                                      // (A/B r2sc/r2sd: ring 0.862 -> 0.853 ms, others neutral)
  int64_t direct_copy_rows = 0;       // COPY items with shorter average runs: consumer gathers
  bool use_gather4 = true;            // TMA gather4 for short-run embedding gathers
  bool stage_fold = true;             // FOLD operand rows bulk-copied into the stage
  bool hostsim_items = false;         // debug host interpreter: run the work items, not groups
  bool spst_fast = true;              // uniform switch: SPST's closed form (parallel), not the loop
  int geometry = 0;                   // bulk-copy geometry: 0 auto per program, 1 WIDE, 2 DUAL
  int sm_budget = 0;                  // SMs an executor launch may use (0 = all): the rest stay
                                      // free for kernels overlapping the exchange (NEXT-2)
  bool signal_all = false;            // fused loopback: publish every done count (arrival waits)
  int l2_policy = 1;                  // L2 eviction hints (executor_tma.cu): stores evict_first
                                      // (Com-Orkut forward 1.69 -> 1.63 ms, others neutral)
  bool force_sys_scope = false;       // loopback with the multi-GPU (.sys) flag scope (A/B)
  bool threads_set = false, ctas_set = false;  // user overrides of the CTA shape
  int sm_count = 148;  // SMs of the device (B200 until queried), for cutting small stages
  // (geo, block, instance mask or -1) -> co-resident CTAs per SM
  std::map<std::tuple<int, int, int>, int> tma_ctas;
  int n_prog_ranks = 1;        // programs per (layer, dir)

  uint64_t seq = 0, epoch[2] = {0, 0};
  uint64_t barrier_seq = 0;  // dgcl_device_barrier calls
  int *err_host = nullptr, *err_dev = nullptr;
  int threads = 512, ctas_per_sm = 0, grid = 0, n_sm = 0, use_tma = 1;
  int64_t item_bytes = kTmaBufBytes, timeout_ms = 20000;
  std::vector<cudaStream_t> rank_streams;
  std::vector<cudaEvent_t> rank_events;
  cudaEvent_t fork_event = nullptr;
  // host-buffer entry points: device staging per (buffer, layer), each with the event of its
  // last device-side use, and two copy streams so that the host->device copy of one call runs
  // while the device->host copy of the previous one is in flight (PCIe is full duplex)
  struct Stage {
    void *ptr = nullptr;
    size_t bytes = 0;
    cudaEvent_t free = nullptr;  // recorded after the last kernel / copy that reads it
  };
  std::map<int, Stage> stages;  // key: kind * 4096 + layer (kind 0 emb, 1 halo grad, 2 emb grad)
  cudaStream_t h2d_stream = nullptr, d2h_stream = nullptr;
  bool host_async = false;  // host calls return before the device->host copy completes
  int64_t small_launch_bytes = 4 << 20;  // launches moving less use the register executor
  bool trace = false;                    // per-item timelines (dgcl_trace_read)
  uint64_t launches = 0;
  int debug_skip_rank = -1;  // fault injection (per-rank loopback): never launch this rank
  bool dead = false;
  std::string err;

  int prog_index(int layer, int dir, int r) const { return (layer * 2 + dir) * n_prog_ranks + r; }
};

namespace {

dgcl_status fail(dgcl_ctx *c, dgcl_status s, const char *fmt, ...) {
  if (c) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    std::vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    c->err = buf;
  }
  return s;
}

#define CUDA_TRY(c, call)                                                                   \
  do {                                                                                      \
    cudaError_t e_ = (call);                                                                \
    if (e_ != cudaSuccess)                                                                  \
      return fail((c), DGCL_ECUDA, "%s failed: %s", #call, cudaGetErrorString(e_));         \
  } while (0)

dgcl_status init_common(int32_t rank, int32_t world, int32_t dev, int64_t n, const int32_t *part,
                        int32_t n_layers, const int32_t *dims, bool loopback, int flags,
                        dgcl_ctx **out) {
  if (!out) return DGCL_EINVAL;
  *out = nullptr;
  if (world < 1 || world > kMaxRanks || rank < 0 || rank >= world || n < 0 || n_layers < 1 ||
      !dims || (n > 0 && !part))
    return DGCL_EINVAL;
  if (loopback && flags != DGCL_LOOPBACK_FUSED && flags != DGCL_LOOPBACK_PER_RANK)
    return DGCL_EINVAL;
  dgcl_ctx *c = new (std::nothrow) dgcl_ctx();
  if (!c) return DGCL_ENOMEM;
  c->rank = rank;
  c->world = world;
  c->device = dev;
  c->loopback = loopback;
  c->lb_flags = flags;
  c->n = n;
  c->n_layers = n_layers;
  for (int l = 0; l < n_layers; ++l) {
    if (dims[l] < 1 || dims[l] > (1 << 24)) {
      delete c;
      return DGCL_EINVAL;
    }
    c->dims.push_back(dims[l]);
    c->pitch.push_back(pitch_of(dims[l]));
    c->max_pitch = std::max(c->max_pitch, pitch_of(dims[l]));
  }
  c->part.assign(part, part + n);
  c->loc.assign(n, 0);
  c->n_local.assign(world, 0);
  for (int64_t v = 0; v < n; ++v) {  // §4.1 re-indexing: ascending global id per partition
    const int32_t p = part[v];
    if (p < 0 || p >= world) {
      delete c;
      return DGCL_EINVAL;
    }
    c->loc[v] = c->n_local[p]++;
  }
  c->row_off.assign(world + 1, 0);
  for (int d = 0; d < world; ++d) c->row_off[d + 1] = c->row_off[d] + c->n_local[d];
  c->topo = Topology::uniform_nvswitch(world);
  if (dev >= 0) {
    cudaError_t e = cudaSetDevice(dev);
    if (e == cudaSuccess)
      e = cudaDeviceGetAttribute(&c->sm_count, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) {
      delete c;
      return DGCL_ECUDA;
    }
  }
  *out = c;
  return DGCL_OK;
}

bool has_device(dgcl_ctx *c) { return c->device >= 0; }

int mc_min_fanout(const dgcl_ctx *c) {
  if (c->multicast <= 0 || c->world < 2) return 0;
  return c->multicast == 1 ? c->world - 1 : c->multicast;
}

void relower(dgcl_ctx *c) {
  lower_plan(c->rel, c->plan, c->part.data(), c->loc, &c->low, c->pipeline_blocks,
             c->atomic_backward, c->fanout && !mc_min_fanout(c), mc_min_fanout(c),
             c->leaf_split);
}

void compute_layout(dgcl_ctx *c) {
  const int m = c->world;
  const Lowered &L = c->low;
  c->off_flags.assign(m, 0);
  c->off_slot.assign(m, 0);
  c->ws_need.assign(m, 0);
  c->off_halo.assign(c->n_layers, std::vector<size_t>(m, 0));
  c->off_relay.assign(c->n_layers, std::vector<size_t>(m, 0));
  if (c->loopback) {
    // one allocation, buffer-major: every layer's halo of all ranks is one contiguous array
    size_t off = 0;
    for (int r = 0; r < m; ++r) c->off_flags[r] = off + (size_t)r * kFlagBytes;
    off += (size_t)m * kFlagBytes;
    for (int l = 0; l < c->n_layers; ++l) {
      for (int r = 0; r < m; ++r)
        c->off_halo[l][r] = off + (size_t)c->halo_off[r] * c->pitch[l] * 4;
      off = align_up(off + (size_t)c->halo_off[m] * c->pitch[l] * 4);
    }
    // relay staging: every layer's rows of all ranks contiguous too (one tensor map per layer)
    for (int l = 0; l < c->n_layers; ++l) {
      size_t rows = 0;
      for (int r = 0; r < m; ++r) {
        c->off_relay[l][r] = off + rows * c->pitch[l] * 4;
        rows += (size_t)L.n_relay[r];
      }
      off = align_up(off + rows * c->pitch[l] * 4);
    }
    for (int r = 0; r < m; ++r) {
      c->off_slot[r] = off;
      off = align_up(off + (size_t)L.n_slot[r] * c->max_pitch * 4);
    }
    for (int r = 0; r < m; ++r) c->ws_need[r] = off;
  } else {
    for (int r = 0; r < m; ++r) {
      size_t off = 0;
      c->off_flags[r] = 0;
      off = kFlagBytes;
      for (int l = 0; l < c->n_layers; ++l) {
        c->off_halo[l][r] = off;
        off = align_up(off + (size_t)L.n_halo[r] * c->pitch[l] * 4);
      }
      for (int l = 0; l < c->n_layers; ++l) {
        c->off_relay[l][r] = off;
        off = align_up(off + (size_t)L.n_relay[r] * c->pitch[l] * 4);
      }
      c->off_slot[r] = off;
      off = align_up(off + (size_t)L.n_slot[r] * c->max_pitch * 4);
      c->ws_need[r] = off;
    }
  }
  // multicast region: [flag page][layer 0 rows][layer 1 rows] ... (same layout on every rank)
  c->mc_layer_off.assign(c->n_layers, 0);
  c->mc_bytes = 0;
  c->off_mc.assign(m, 0);
  if (L.mc_total > 0) {
    size_t o = kMcFlagBytes;
    for (int l = 0; l < c->n_layers; ++l) {
      c->mc_layer_off[l] = o;
      o = align_up(o + (size_t)L.mc_total * c->pitch[l] * 4);
    }
    c->mc_bytes = o;
    if (c->loopback) {  // emulation: every virtual rank's copy after the workspace
      size_t off = c->ws_need[0];
      for (int r = 0; r < m; ++r) {
        c->off_mc[r] = off;
        off = align_up(off + c->mc_bytes);
      }
      for (int r = 0; r < m; ++r) c->ws_need[r] = off;
    }
  }
}

// counters some group of the given program waits on (fused loopback: only those need a signal)
std::vector<uint8_t> needed_counters(const Lowered &L, const std::vector<int32_t> &gids) {
  std::vector<uint8_t> need((size_t)kMaxRanks * kCtrSpace, 0);
  for (int32_t gi : gids) {
    const DevGroup &g = L.groups[gi];
    for (int w = 0; w < g.wait_n; ++w)
      need[(size_t)g.exec_rank * kCtrSpace + L.waits[g.wait_off + w].ctr] = 1;
  }
  return need;
}

void build_programs(dgcl_ctx *c) {
  const Lowered &L = c->low;
  const int m = c->world;
  const bool fused = c->loopback && c->lb_flags == DGCL_LOOPBACK_FUSED;
  c->n_prog_ranks = fused ? 1 : m;
  c->progs.assign((size_t)c->n_layers * 2 * c->n_prog_ranks, Program());
  const int ng = (int)L.groups.size();
  // forward stage 1 as one fan-out group per owner (each row read once, stored into all its
  // first-hop receivers) instead of one COPY group per (owner, receiver); per layer below
  const bool fan_avail = c->fanout && L.fanout_end > L.atomic_end && L.n_blocks == 1;
  auto is_stage1_copy = [&](const DevGroup &g) {
    return g.dir == DIR_FWD && g.op == OP_COPY && g.stage == 1 && g.src_kind == K_EMB;
  };
  for (int dir = 0; dir < 2; ++dir) {
    std::vector<std::vector<int32_t>> gids(c->n_prog_ranks), gids_fan(c->n_prog_ranks);
    for (int r = 0; r < c->n_prog_ranks; ++r) {
      const bool want_rank = c->loopback || r == c->rank;
      if (!fused && !want_rank) continue;
      if (!fused && m > 1) {
        for (int gi = 0; gi < ng; ++gi)
          if (L.groups[gi].op == OP_READY && L.groups[gi].exec_rank == r) gids[r].push_back(gi);
      }
      gids_fan[r] = gids[r];
      if (dir == DIR_FWD && fan_avail)
        for (int gi = L.atomic_end; gi < L.fanout_end; ++gi)
          if (fused || L.groups[gi].exec_rank == r) gids_fan[r].push_back(gi);
      for (int gi = 0; gi < ng; ++gi) {
        const DevGroup &g = L.groups[gi];
        if (g.op == OP_READY || g.op == OP_WAIT || g.dir != dir) continue;
        if (gi >= L.direct_begin && gi < L.tree_end) continue;
        if (!fused && g.exec_rank != r) continue;
        gids[r].push_back(gi);
        if (!(fan_avail && is_stage1_copy(g))) gids_fan[r].push_back(gi);
      }
      if (!fused && dir == DIR_FWD && m > 1) {
        for (int gi = 0; gi < ng; ++gi)
          if (L.groups[gi].op == OP_WAIT && L.groups[gi].exec_rank == r) {
            gids[r].push_back(gi);
            gids_fan[r].push_back(gi);
          }
      }
    }
    // fused loopback, single-stage plan: the owner folds its requesters' halo gradients in place
    // (ablation, option "atomic_backward": requesters add their rows into the owners' rows with
    // atomic reductions instead)
    const bool atomic = fused && dir == DIR_BWD && c->atomic_backward && L.n_stages <= 1 &&
                        L.atomic_end > L.direct_end;
    const bool direct = !atomic && fused && dir == DIR_BWD && c->direct_reduce &&
                        L.n_stages <= 1 && L.direct_end > L.direct_begin;
    // relay plans: each owner row folds its whole tree in the reversed plan's order in one pass
    const bool tree = fused && dir == DIR_BWD && c->direct_reduce && L.n_stages >= 2 &&
                      L.tree_end > L.fanout_end;
    if (direct || atomic || tree) {
      gids[0].clear();
      const int b = atomic ? L.direct_end : tree ? L.fanout_end : L.direct_begin;
      const int e = atomic ? L.atomic_end : tree ? L.tree_end : L.direct_end;
      for (int gi = b; gi < e; ++gi) gids[0].push_back(gi);
    }
    // the host interpreter runs the fused-order program of this direction
    c->host_gids[dir].clear();
    if (direct || atomic || tree) {
      c->host_gids[dir] = gids[0];
    } else {
      if (dir == DIR_FWD && fan_avail)
        for (int gi = L.atomic_end; gi < L.fanout_end; ++gi) c->host_gids[dir].push_back(gi);
      for (int gi = 0; gi < ng; ++gi) {
        const DevGroup &g = L.groups[gi];
        if (g.op == OP_READY || g.op == OP_WAIT || g.dir != dir) continue;
        if (gi >= L.direct_begin && gi < L.tree_end) continue;
        if (fan_avail && is_stage1_copy(g)) continue;
        c->host_gids[dir].push_back(gi);
      }
    }
    for (int l = 0; l < c->n_layers; ++l) {
      const int64_t row_bytes = (int64_t)c->dims[l] * 4, row16 = (row_bytes + 15) / 16 * 16;
      // fan-out items stage a row plus its destination words: rows up to half a DUAL stage
      const bool fan = fan_avail && dir == DIR_FWD &&
                       2 * (row16 + 128) <= kGeoDual.stage_bytes - kStageHdrBytes;
      auto build = [&](Program &P, int r, int geo) {
        const std::vector<int32_t> &G = fan ? gids_fan[r] : gids[r];
        const std::vector<uint8_t> need = needed_counters(L, G);
        P.geo = geo;
        ItemLimits lim = item_limits(geometry_of(geo), c->item_bytes,
                                     (int64_t)c->sm_count * geometry_of(geo).ctas_per_sm);
        lim.align_sources = c->align_sources;
        lim.lsu_gather = c->lsu_gather && c->use_tma;
        lim.owner_major = fused ? c->owner_major : 0;
        build_items(L, G, row_bytes, lim, !fused || c->signal_all, need, &P.items, &P.runs,
                    c->direct_copy_rows,
                    c->stage_fold ? &P.sterms : nullptr);
        if (dir == DIR_FWD && c->relay_lead_kb >= 0)
          lead_relay_items(L, &P.items, row_bytes, c->relay_lead_kb * 1024);
        P.op_mask = 0;
        int64_t fold_rows = 0, fold_terms = 0;
        for (const DevItem &it : P.items) {
          if (it.op == OP_FOLD && (it.flags & kItemStaged)) {
            P.op_mask |= kMaskStaged;
          } else if (it.op == OP_FOLD && it.term_mode == kTermRankTree) {
            P.op_mask |= kMaskTree;
          } else if (it.op == OP_FOLD) {
            P.op_mask |= kMaskFold;
            fold_rows += it.rows;
            fold_terms += it.nterms;
          }
          if (it.op == OP_COPY) P.op_mask |= (it.flags & kItemDirect) ? kMaskDirect : kMaskCopy;
          if (it.op == OP_COPY && (it.flags & kItemLsu)) P.op_mask |= kMaskLsu;
          if (it.op == OP_COPY && it.dst_kind == K_MCAST) P.op_mask |= kMaskMcast;
          if (it.op == OP_FANOUT) P.op_mask |= kMaskFanout;
        }
        P.fold_wide = fold_rows > 0 && fold_terms >= 4 * fold_rows;
        // dual producers (executor_tma.cu) need plain copies whose runs fit half a meta slot
        P.simple_copy = !P.items.empty();
        P.max_meta = 0;
        for (const DevItem &it : P.items) {
          if ((it.op != OP_COPY && it.op != OP_FOLD) || it.wait_n > 0 ||
              (it.flags & (kItemSignal | kItemDirect | kItemLsu | kItemAtomic)) ||
              it.dst_kind == K_MCAST)
            P.simple_copy = false;
          if (it.op == OP_COPY)  // runs (16 B each), or a gather4 item's 16-B-aligned row window
            P.max_meta = std::max<int64_t>(P.max_meta, (it.flags & kItemGather4)
                                                           ? (int64_t)it.rows * 4 + 32
                                                           : (int64_t)it.nterms * 16);
          else if (it.op == OP_FOLD && (it.flags & kItemStaged))  // its segments
            P.max_meta = std::max<int64_t>(P.max_meta, (int64_t)(it.src >> kSegShift) * 16);
        }
        P.relay_fwd = false;
        for (const DevItem &it : P.items)
          if (it.dir == DIR_FWD && it.op == OP_COPY && it.wait_n > 0) P.relay_fwd = true;
        P.g4_kinds = 0;
        P.tree = false;
        for (const DevItem &it : P.items)
          if (it.op == OP_FOLD && it.term_mode == kTermRankTree) P.tree = true;
        for (const DevItem &it : P.items)
          if (it.op == OP_COPY && (it.flags & kItemGather4)) P.g4_kinds |= 1 << it.src_kind;
        P.bytes = 0;
        for (const DevItem &it : P.items)
          if (it.op == OP_COPY || it.op == OP_FOLD)
            P.bytes += (int64_t)(it.rows + (it.op == OP_FOLD ? it.nterms : 0)) * row16;
          else if (it.op == OP_FANOUT)
            P.bytes += (int64_t)(it.rows + it.nterms) * row16;
      };
      for (int r = 0; r < c->n_prog_ranks; ++r) {
        Program &P = c->progs[c->prog_index(l, dir, r)];
        // WIDE: 4 x 48 KB stages for launches that get two producers, 3 x 64 KB (WIDE3) for
        // launches that keep one (waits, signals, READY / WAIT items)
        auto build_wide = [&](Program &Q, int rr) {
          build(Q, rr, 0);
          bool one = false;
          for (const DevItem &it : Q.items)
            one = one || it.wait_n > 0 || (it.flags & kItemSignal) || it.op == OP_READY ||
                  it.op == OP_WAIT;
          if (one) build(Q, rr, 2);
        };
        if (c->geometry) {
          if (c->geometry == 1)
            build_wide(P, r);
          else
            build(P, r, c->geometry - 1);
          continue;
        }
        // auto: DUAL (two producer warps per SM) unless the launch is bulk-copy friendly —
        // copies only, >= 8 KB per bulk operation (long runs of rows) — or carries unstaged folds
        // (consumer gathers, which want more consumer warps); see TmaGeometry
        build(P, r, 1);
        int64_t ops = 0, bytes = 0;
        bool waits = false;
        for (const DevItem &it : P.items) {
          waits = waits || (it.wait_n > 0 && (it.op == OP_COPY || it.op == OP_FOLD));
          if (it.op == OP_FANOUT) {  // one bulk copy per item
            bytes += (int64_t)it.rows * row16;
            ops += 1;
          }
          if (it.op != OP_COPY) continue;
          bytes += (int64_t)it.rows * row16;
          ops += (it.flags & kItemGather4) ? (it.rows + 3) / 4 : it.nterms;
        }
        const bool copy_only = (P.op_mask & ~(kMaskCopy | kMaskFanout)) == 0;
        // (relay forwards chained on flags now run DUAL too: 1.08 -> 1.01 ms on the Web-Google
        // ring plan, 0.83 -> 0.81 dgx1_like, no bimodality with device-scope flags, A/B r2j/r2k)
        if (std::getenv("DGCL_DEBUG_GEO"))
          std::fprintf(stderr, "geo: layer %d dir %d rank %d copy_only %d ops %lld bytes %lld per op %.0f\n",
                       l, dir, r, (int)copy_only, (long long)ops, (long long)bytes,
                       ops ? (double)bytes / ops : 0.0);
        // (copy launches without waits or signals — two producers, 4 x 48 KB stages — run WIDE from 3.5 KB
        // per bulk operation: Web-Google-8 forward 4.1 KB / op 0.425 DUAL vs 0.419 WIDE,
        // Web-Google-2 0.186 vs 0.182, Reddit fwd256 0.313 vs 0.311, Com-Orkut 2.8 KB / op 1.43
        // vs 1.53, A/B r2tg; with waits / signals (relay forwards, per-rank programs: one
        // producer) from 28 KB, r2sj)
        // (the launch gets dual producers only without waits and signals, and with claims only
        // under option dual_claims (default on) — Web-Google-4 forward on WIDE with claims and
        // one producer: 0.414 ms vs 0.292 DUAL, r2th; with dual producers 0.2925, r2tk)
        bool sigs = false;
        for (const DevItem &it : P.items) sigs = sigs || (it.flags & kItemSignal);
        const bool claims = (c->claim_batch > 0 || (c->claim_batch < 0 && m <= 4)) &&
                            !(c->dual_producer && c->dual_claims);
        const int64_t wide_op = (waits || sigs || claims) ? 28672 : 3584;
        if ((copy_only && ops > 0 && bytes >= wide_op * ops) || (P.op_mask & (kMaskFold | kMaskTree)))
          build_wide(P, r);
      }
      // per-rank loopback: the ranks' launches run concurrently on one device and their CTAs wait
      // on each other's flags, so together they must be co-resident.  A WIDE CTA (one per SM by
      // shared memory) cannot share an SM with a DUAL one: every rank of a (layer, direction)
      // takes the geometry of the largest program (launch() likewise picks one executor for all)
      if (c->loopback && !fused && c->n_prog_ranks > 1) {
        int big = 0;
        for (int r = 1; r < c->n_prog_ranks; ++r)
          if (c->progs[c->prog_index(l, dir, r)].bytes > c->progs[c->prog_index(l, dir, big)].bytes)
            big = r;
        const int geo = c->progs[c->prog_index(l, dir, big)].geo;
        for (int r = 0; r < c->n_prog_ranks; ++r) {
          Program &P = c->progs[c->prog_index(l, dir, r)];
          if (P.geo != geo) build(P, r, geo);
        }
      }
    }
  }
}

template <typename T>
dgcl_status upload(dgcl_ctx *c, T **dptr, const std::vector<T> &v) {
  if (*dptr) cudaFree(*dptr);
  *dptr = nullptr;
  // + 64 zeroed bytes: the executor bulk-copies 16-B aligned windows of these pools, whose last
  // window may extend up to 15 bytes past the final element
  const size_t bytes = v.size() * sizeof(T) + 64;
  CUDA_TRY(c, cudaMalloc((void **)dptr, bytes));
  CUDA_TRY(c, cudaMemset(*dptr, 0, bytes));
  if (!v.empty()) CUDA_TRY(c, cudaMemcpy(*dptr, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice));
  return DGCL_OK;
}

// CTA size of a program's bulk-copy launch: the geometry's, except that unstaged folds
// (consumer-side gathers, latency-bound) get more consumer warps — 1024 threads for fold-only
// launches with many terms per row, 512 otherwise — and the user's "threads" option wins
int tma_block(const dgcl_ctx *c, const Program &pg) {
  if (c->threads_set) return c->threads;
  const TmaGeometry &G = geometry_of(pg.geo);
  if (pg.geo != 1 && (pg.op_mask & (kMaskFold | kMaskTree)))
    return pg.op_mask == kMaskFold && pg.fold_wide && !pg.tree ? 1024 : 512;
  return G.threads;
}

// occupancy key of a program's launch: its own instance when it runs alone on the device; the
// worst case over instances when per-rank loopback launches share the device concurrently
int occ_mask(const dgcl_ctx *c, const Program &pg) {
  return (c->loopback && c->lb_flags == DGCL_LOOPBACK_PER_RANK) ? -1 : pg.op_mask;
}

dgcl_status check_dead(dgcl_ctx *c) {
  if (c->dead) return fail(c, DGCL_ETIMEOUT, "context unusable after a device watchdog timeout");
  if (c->err_host && *(volatile int *)c->err_host != 0) {
    c->dead = true;
    return fail(c, DGCL_ETIMEOUT, "device watchdog: a flag wait timed out (code %d)",
                *(volatile int *)c->err_host);
  }
  return DGCL_OK;
}

inline bool al16(const void *p) { return ((uintptr_t)p & 15) == 0; }

// CUDA driver entry points, resolved through the runtime (libdgcl does not link libcuda)
template <typename F>
F drv(const char *name) {
  void *p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess)
    return nullptr;
  return (F)p;
}

// ---- NVSwitch multicast objects (cuMulticast*): the driver calls behind dgcl_multicast_* ----
struct McDriver {
  CUresult (*getAttr)(int *, CUdevice_attribute, CUdevice) = nullptr;
  CUresult (*gran)(size_t *, const CUmulticastObjectProp *, CUmulticastGranularity_flags) = nullptr;
  CUresult (*create)(CUmemGenericAllocationHandle *, const CUmulticastObjectProp *) = nullptr;
  CUresult (*addDevice)(CUmemGenericAllocationHandle, CUdevice) = nullptr;
  CUresult (*bindMem)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t,
                      size_t, unsigned long long) = nullptr;
  CUresult (*unbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t) = nullptr;
  CUresult (*memCreate)(CUmemGenericAllocationHandle *, size_t, const CUmemAllocationProp *,
                        unsigned long long) = nullptr;
  CUresult (*memRelease)(CUmemGenericAllocationHandle) = nullptr;
  CUresult (*reserve)(CUdeviceptr *, size_t, size_t, CUdeviceptr, unsigned long long) = nullptr;
  CUresult (*addrFree)(CUdeviceptr, size_t) = nullptr;
  CUresult (*map)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle,
                  unsigned long long) = nullptr;
  CUresult (*unmap)(CUdeviceptr, size_t) = nullptr;
  CUresult (*setAccess)(CUdeviceptr, size_t, const CUmemAccessDesc *, size_t) = nullptr;
  CUresult (*exportH)(void *, CUmemGenericAllocationHandle, CUmemAllocationHandleType,
                      unsigned long long) = nullptr;
  CUresult (*importH)(CUmemGenericAllocationHandle *, void *, CUmemAllocationHandleType) = nullptr;
  bool ok = false;
  McDriver() {
    getAttr = drv<decltype(getAttr)>("cuDeviceGetAttribute");
    gran = drv<decltype(gran)>("cuMulticastGetGranularity");
    create = drv<decltype(create)>("cuMulticastCreate");
    addDevice = drv<decltype(addDevice)>("cuMulticastAddDevice");
    bindMem = drv<decltype(bindMem)>("cuMulticastBindMem");
    unbind = drv<decltype(unbind)>("cuMulticastUnbind");
    memCreate = drv<decltype(memCreate)>("cuMemCreate");
    memRelease = drv<decltype(memRelease)>("cuMemRelease");
    reserve = drv<decltype(reserve)>("cuMemAddressReserve");
    addrFree = drv<decltype(addrFree)>("cuMemAddressFree");
    map = drv<decltype(map)>("cuMemMap");
    unmap = drv<decltype(unmap)>("cuMemUnmap");
    setAccess = drv<decltype(setAccess)>("cuMemSetAccess");
    exportH = drv<decltype(exportH)>("cuMemExportToShareableHandle");
    importH = drv<decltype(importH)>("cuMemImportFromShareableHandle");
    ok = getAttr && gran && create && addDevice && bindMem && unbind && memCreate && memRelease &&
         reserve && addrFree && map && unmap && setAccess && exportH && importH;
  }
};
const McDriver &mcd() {
  static McDriver d;
  return d;
}

bool mc_supported(int dev) {
  const McDriver &D = mcd();
  int v = 0;
  return D.ok && D.getAttr(&v, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, (CUdevice)dev) == CUDA_SUCCESS &&
         v != 0;
}

CUmulticastObjectProp mc_prop(int n_devices, size_t bytes) {
  CUmulticastObjectProp p;
  std::memset(&p, 0, sizeof(p));
  p.numDevices = (unsigned)n_devices;
  p.size = bytes;
  p.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  return p;
}

// bind `bytes` of new device memory of `dev` to multicast object h at offset 0 and map it twice:
// unicast (*uc) and through the multicast address (*mc)
CUresult mc_bind_map(int dev, CUmemGenericAllocationHandle h, size_t bytes,
                     CUmemGenericAllocationHandle *mem, char **uc, char **mc) {
  const McDriver &D = mcd();
  CUmemAllocationProp ap;
  std::memset(&ap, 0, sizeof(ap));
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = dev;
  CUresult r = D.memCreate(mem, bytes, &ap, 0);
  if (r != CUDA_SUCCESS) return r;
  if ((r = D.bindMem(h, 0, *mem, 0, bytes, 0)) != CUDA_SUCCESS) return r;
  CUmemAccessDesc acc;
  std::memset(&acc, 0, sizeof(acc));
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = dev;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CUdeviceptr a = 0, b = 0;
  if ((r = D.reserve(&a, bytes, 0, 0, 0)) != CUDA_SUCCESS) return r;
  if ((r = D.map(a, bytes, 0, *mem, 0)) != CUDA_SUCCESS) return r;
  if ((r = D.setAccess(a, bytes, &acc, 1)) != CUDA_SUCCESS) return r;
  *uc = (char *)a;
  if ((r = D.reserve(&b, bytes, 0, 0, 0)) != CUDA_SUCCESS) return r;
  if ((r = D.map(b, bytes, 0, h, 0)) != CUDA_SUCCESS) return r;
  if ((r = D.setAccess(b, bytes, &acc, 1)) != CUDA_SUCCESS) return r;
  *mc = (char *)b;
  return CUDA_SUCCESS;
}

void mc_teardown(int dev, CUmemGenericAllocationHandle h, bool have_h, CUmemGenericAllocationHandle mem,
                 bool have_mem, char *uc, char *mc, size_t bytes) {
  const McDriver &D = mcd();
  if (!D.ok) return;
  if (mc) {
    D.unmap((CUdeviceptr)mc, bytes);
    D.addrFree((CUdeviceptr)mc, bytes);
  }
  if (uc) {
    D.unmap((CUdeviceptr)uc, bytes);
    D.addrFree((CUdeviceptr)uc, bytes);
  }
  if (have_h && have_mem) D.unbind(h, (CUdevice)dev, 0, bytes);
  if (have_mem) D.memRelease(mem);
  if (have_h) D.memRelease(h);
}

// 2-D tensor map over `rows` packed rows of row_bytes (<= 1 KB) starting at `base`: box = one row,
// for cp.async.bulk.tensor ... tile::gather4.  The driver entry point is resolved through the
// runtime (no libcuda link).  Returns false if the map cannot be built (the launch then uses
// per-run bulk copies).
bool encode_rows_tmap(dgcl_ctx *c, unsigned char *out, const void *base, int64_t rows,
                      int row_bytes) {
  typedef CUresult (*Encode)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                             const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                             const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  static Encode fn = nullptr;
  if (!fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) !=
            cudaSuccess ||
        !p || q != cudaDriverEntryPointSuccess)
      return false;
    fn = (Encode)p;
  }
  (void)c;
  const cuuint64_t dims[2] = {(cuuint64_t)(row_bytes / 4), (cuuint64_t)rows};
  const cuuint64_t strides[1] = {(cuuint64_t)row_bytes};
  const cuuint32_t box[2] = {(cuuint32_t)(row_bytes / 4), 1};
  const cuuint32_t estr[2] = {1, 1};
  CUtensorMap map;
  const CUresult r = fn(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void *>(base), dims,
                        strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return false;
  static_assert(sizeof(CUtensorMap) == 128, "tensor map size");
  std::memcpy(out, &map, sizeof(map));
  return true;
}

// the context's device is current for the launches (and the caller's restored afterwards)
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

dgcl_status launch(dgcl_ctx *c, int layer, int dir, const float *in, int64_t in_pitch,
                   float *out, int64_t out_pitch, cudaStream_t stream) {
  DeviceGuard guard(c->device);
  const int m = c->world;
  ExecParams P;
  std::memset(&P, 0, sizeof(P));
  const int64_t hp = c->pitch[layer] * 4;  // bytes
  bool v16 = (hp % 16) == 0;
  for (int r = 0; r < m; ++r) {
    char *b = c->base[r];
    P.flags[r] = (uint64_t *)(b + c->off_flags[r]);
    P.buf[K_HALO][r] = {b + c->off_halo[layer][r], hp};
    P.buf[K_RELAY][r] = {b + c->off_relay[layer][r], hp};
    P.buf[K_SLOT][r] = {b + c->off_slot[r], hp};
  }
  if (dir == DIR_FWD && c->low.mc_total > 0) {
    const size_t lo = c->mc_layer_off[layer];
    for (int r = 0; r < m; ++r) {
      if (c->loopback) {
        char *b = c->base[r] + c->off_mc[r];
        P.buf[K_MCUC][r] = {b + lo, hp};
        P.mcuc_flags[r] = (uint64_t *)b;
      } else if (r == c->rank) {
        P.buf[K_MCUC][r] = {c->mc_uc + lo, hp};
        P.buf[K_MCAST][r] = {c->mc_va + lo, hp};
        P.mcuc_flags[r] = (uint64_t *)c->mc_uc;
        P.mc_flags = (uint64_t *)c->mc_va;
      }
    }
    P.mc_emulate = c->loopback ? 1 : 0;
  }
  const int in_kind = dir == DIR_FWD ? K_EMB : K_HGRAD;
  for (int r = 0; r < m; ++r) {
    if (!c->loopback && r != c->rank) continue;
    const int64_t in_row = c->loopback ? (dir == DIR_FWD ? c->row_off[r] : c->halo_off[r]) : 0;
    P.buf[in_kind][r] = {(char *)(in + in_row * in_pitch), in_pitch * 4};
    if (dir == DIR_BWD) {
      const int64_t out_row = c->loopback ? c->row_off[r] : 0;
      P.buf[K_EGRAD][r] = {(char *)(out + out_row * out_pitch), out_pitch * 4};
    }
  }
  if ((in_pitch * 4) % 16 || !al16(in)) v16 = false;
  if (dir == DIR_BWD && ((out_pitch * 4) % 16 || !al16(out))) v16 = false;
  P.groups = c->d_groups;
  P.waits = c->d_waits;
  P.idx = c->d_idx;
  P.term_ptr = c->d_term_ptr;
  P.terms = c->d_terms;
  P.world = m;
  P.row_bytes = c->dims[layer] * 4;
  P.vec16 = v16 ? 1 : 0;
  P.n_chunks = v16 ? (P.row_bytes + 15) / 16 : c->dims[layer];
  const FastDiv fd = make_fastdiv((uint32_t)P.n_chunks);
  P.div_mul = fd.mul;
  P.div_shift = fd.shift;
  P.epoch[0] = c->epoch[0];
  P.epoch[1] = c->epoch[1];
  P.seq = c->seq;
  P.timeout_ns = (uint64_t)c->timeout_ms * 1000000ull;
  P.err = c->err_dev;
  P.row16 = (P.row_bytes + 15) / 16 * 16;
  P.runs = c->d_runs;
  P.sterms = c->d_sterms;
  P.bulk_store = (c->loopback ? c->bulk_store_local : c->bulk_store_peer) ? 1 : 0;
  P.l2_policy = c->l2_policy;
  // every rank on this device (loopback): the flag protocol needs only device scope
  P.sys_scope = (c->loopback && !c->force_sys_scope) ? 0 : 1;
  // bulk-copy path: 16-B rows and every gathered item fits one shared-memory stage (checked
  // again per program against its geometry in launch_program)
  P.use_tma = (v16 && c->use_tma && P.row16 <= kTmaOperandBytes) ? 1 : 0;
  // TMA row gather (gather4) for items whose source rows come in short runs: one 2-D tensor
  // map per source kind over the packed rows this process reads — the caller's embeddings
  // (forward) or halo gradients (backward), and the workspace's halo / relay staging of this
  // layer (relay forwarding).  In loopback every kind's rows of all ranks are one array (the
  // caller's buffer, the buffer-major workspace); a rank's first row is its tensor row offset.
  // Encoded per launch for the kinds its program uses (Program::g4_kinds).
  auto encode_g4 = [&](ExecParams &Q, int kinds) {
    Q.gather4_mask = 0;
    if (!Q.use_tma || !c->use_gather4 || Q.row16 > kGather4MaxRowBytes || Q.row16 % 32) return;
    const int me = c->loopback ? 0 : c->rank;
    for (int k = 0; k < kG4Kinds; ++k) {
      if (!((kinds >> k) & 1)) continue;
      const BufRef &B0 = Q.buf[k][me];
      if (!B0.ptr || B0.pitch != Q.row16) continue;
      int64_t rows = 0;
      if (k == in_kind)
        rows = c->loopback ? (dir == DIR_FWD ? c->n : c->halo_off[m])
                           : (dir == DIR_FWD ? c->n_local[c->rank] : c->rel.n_halo[c->rank]);
      else if (k == K_HALO)
        rows = c->loopback ? c->halo_off[m] : c->rel.n_halo[c->rank];
      else if (k == K_RELAY)
        for (int r = 0; r < m; ++r)
          rows += (c->loopback || r == c->rank) ? c->low.n_relay[r] : 0;
      if (rows <= 0 || rows >= INT32_MAX || !encode_rows_tmap(c, Q.tmap[k], B0.ptr, rows, Q.row16))
        continue;
      Q.gather4_mask |= 1 << k;
      for (int r = 0; r < m; ++r)
        Q.tmap_row_off[k][r] = c->loopback ? (int32_t)((Q.buf[k][r].ptr - B0.ptr) / Q.row16) : 0;
    }
  };
  // one program's launch: its items, kernel instance, CTA shape and bulk-copy geometry
  auto launch_program = [&](const Program &pg, int grid_div, cudaStream_t st,
                            int64_t sel_bytes) -> int {
    ExecParams Pp = P;
    Pp.items = c->d_items + pg.dev_off;
    Pp.op_mask = pg.op_mask;
    Pp.fold_wide = pg.fold_wide ? 1 : 0;
    Pp.n_items = (int32_t)pg.items.size();
    Pp.trace = pg.d_trace;
    const TmaGeometry &G = geometry_of(pg.geo);
    const int tblock = tma_block(c, pg);
    const auto occ = c->tma_ctas.find({pg.geo, tblock, occ_mask(c, pg)});
    const int tctas = occ == c->tma_ctas.end() ? 0 : occ->second;
    // (sm_budget: the grid covers only that many SMs, still co-resident; the other SMs run
    // whatever the caller overlaps with the exchange)
    const int sms = c->sm_budget > 0 ? std::min(c->sm_budget, c->n_sm) : c->n_sm;
    int block = c->threads, grid_all = sms * c->ctas_per_sm;
    // latency-bound launches (a few MB) skip the bulk-copy pipeline: the register executor's
    // single round trip per item is shorter (tiny config: 10 vs 14-19 us per launch)
    // (sel_bytes: per-rank loopback decides for all ranks of a launch together, co-residency)
    const bool small = sel_bytes < c->small_launch_bytes;
    if (Pp.use_tma && !small && Pp.row16 <= G.stage_bytes - kStageHdrBytes && tctas > 0) {
      block = tblock;
      grid_all = sms * tctas;
      Pp.tma_stages = G.stages;
      Pp.tma_buf = G.stage_bytes;
      Pp.meta_bytes = G.meta_bytes;
    } else {
      Pp.use_tma = 0;
    }
    encode_g4(Pp, pg.g4_kinds);
    const int grid = (int)std::min<int64_t>(std::max(1, grid_all / grid_div), Pp.n_items);
    // auto: batches of 4 for relay forwards (stage boundaries wait for the slowest CTA: Web-Google
    // dgx1_like 0.815 -> 0.730 ms, ring 1.017 -> 0.969, Reddit dgx1_like 0.516 -> 0.482), of 2
    // for jobs of <= 4 ranks (per-SM speed spread: Web-Google-2 fwd 0.211 -> 0.185, bwd 0.275 ->
    // 0.255), none for the 8-way single-stage launches (Reddit fwd602 0.741 -> 0.765 with 4: the
    // claims cost more than the spread), A/B r2n
    const int cb = c->claim_batch >= 0 ? c->claim_batch
                   : pg.relay_fwd     ? 4
                   : m <= 4           ? 2
                                      : 0;
    uint64_t claimed = 0;
    if (Pp.use_tma && cb > 0 && c->d_claims) {
      Pp.claim = c->d_claims + (&pg - c->progs.data());
      Pp.claim_base = pg.claims;
      Pp.claim_batch = cb;
      claimed = (uint64_t)cb * ((uint64_t)(Pp.n_items + cb - 1) / cb + (uint64_t)grid);
    }
    // two producer warps for simple copy launches on the WIDE geometry (option dual_producer)
    // (each producer's metadata slots are half size: an item's runs must fit meta_bytes / 2)
    // (DUAL-geometry launches of bulk-copy runs only — already two producers per SM — gain
    // nothing: Reddit fwd256 0.311 -> 0.312 / 0.318 -> 0.322, A/B r2sx / r2sz; WIDE and gather4
    // launches do: fwd602 0.718 -> 0.695, Web-Google-8 0.437 -> 0.428)
    // staged folds (fused in-place / tree-order backward): the producer bounds them too (ncu
    // r2tb: ~600 dependent instructions per item)
    const bool dual_copy = Pp.op_mask == kMaskCopy && (pg.geo != 1 || pg.g4_kinds != 0);
    const bool dual_fold = Pp.op_mask == kMaskStaged || Pp.op_mask == (kMaskTree | kMaskStaged);
    Pp.dual_prod = (c->dual_producer && Pp.use_tma && pg.simple_copy && (dual_copy || dual_fold) &&
                    pg.max_meta <= Pp.meta_bytes / 2 && (!Pp.claim || c->dual_claims) &&
                    !Pp.trace && !Pp.use_ready && block >= 4 * 32)
                       ? 1 : 0;
    // (with claims each of the two producers ends with one failing claim)
    if (Pp.claim && Pp.dual_prod)
      claimed = (uint64_t)cb * ((uint64_t)(Pp.n_items + cb - 1) / cb + 2 * (uint64_t)grid);
    const int rc = launch_executor(Pp, grid, block, st);
    if (rc == 0) pg.claims += claimed;  // (a launch that never ran added nothing on the device)
    return rc;
  };
  const bool fused = c->loopback && c->lb_flags == DGCL_LOOPBACK_FUSED;
  P.use_ready = (!fused && m > 1) ? 1 : 0;
  if (fused || !c->loopback) {
    const int r = fused ? 0 : c->rank;
    const Program &pg = c->progs[c->prog_index(layer, dir, fused ? 0 : (c->loopback ? r : r))];
    if (pg.items.empty()) return DGCL_OK;
    int e = launch_program(pg, 1, stream, pg.bytes);
    if (e != 0) return fail(c, DGCL_ECUDA, "executor launch failed: %s",
                            cudaGetErrorString((cudaError_t)e));
    c->launches++;
    return DGCL_OK;
  }
  // loopback, one launch per virtual rank on its own stream (full flag protocol)
  CUDA_TRY(c, cudaEventRecord(c->fork_event, stream));
  int64_t sel_bytes = 0;  // one executor for every rank's launch: the largest program decides
  for (int r = 0; r < m; ++r) sel_bytes = std::max(sel_bytes, c->progs[c->prog_index(layer, dir, r)].bytes);
  for (int r = 0; r < m; ++r) {
    const Program &pg = c->progs[c->prog_index(layer, dir, r)];
    CUDA_TRY(c, cudaStreamWaitEvent(c->rank_streams[r], c->fork_event, 0));
    if (!pg.items.empty() && r != c->debug_skip_rank) {
      int e = launch_program(pg, m, c->rank_streams[r], sel_bytes);
      if (e != 0) return fail(c, DGCL_ECUDA, "executor launch failed: %s",
                              cudaGetErrorString((cudaError_t)e));
      c->launches++;
    }
    CUDA_TRY(c, cudaEventRecord(c->rank_events[r], c->rank_streams[r]));
    CUDA_TRY(c, cudaStreamWaitEvent(stream, c->rank_events[r], 0));
  }
  return DGCL_OK;
}

dgcl_status ready_to_dispatch(dgcl_ctx *c, int32_t layer) {
  if (!c) return DGCL_EINVAL;
  if (!has_device(c)) return fail(c, DGCL_ESTATE, "host-only context");
  if (!c->registered) return fail(c, DGCL_ESTATE, "workspace not registered");
  if (!c->loopback && c->world > 1 && !c->imported)
    return fail(c, DGCL_ESTATE, "peers not imported");
  if (layer < 0 || layer >= c->n_layers) return fail(c, DGCL_EINVAL, "bad layer %d", layer);
  if (!c->loopback && c->low.mc_total > 0 && !c->mc_uc)
    return fail(c, DGCL_ESTATE, "multicast planned but the region is not bound (dgcl_multicast_bind)");
  return check_dead(c);
}

}  // namespace

extern "C" {

dgcl_status dgcl_init(int32_t rank, int32_t world, int32_t cuda_device, int64_t n_vertices,
                      const int32_t *part, int32_t n_layers, const int32_t *dims, dgcl_ctx **out) {
  return init_common(rank, world, cuda_device, n_vertices, part, n_layers, dims, false, 0, out);
}

dgcl_status dgcl_init_loopback(int32_t world, int32_t cuda_device, int64_t n_vertices,
                               const int32_t *part, int32_t n_layers, const int32_t *dims,
                               int32_t flags, dgcl_ctx **out) {
  return init_common(0, world, cuda_device, n_vertices, part, n_layers, dims, true, flags, out);
}

dgcl_status dgcl_set_topology(dgcl_ctx *c, const dgcl_topology *t) {
  if (!c || !t || !t->hop_ticks || !t->link_ptr || t->n_hops < 0) return DGCL_EINVAL;
  if (c->planned) return fail(c, DGCL_ESTATE, "topology must be set before dgcl_build_plan");
  const int m = c->world;
  Topology T;
  T.m = m;
  for (int h = 0; h < t->n_hops; ++h) {
    if (t->hop_ticks[h] <= 0) return fail(c, DGCL_EINVAL, "hop %d: ticks must be > 0", h);
    T.w.push_back(t->hop_ticks[h]);
  }
  if (t->link_ptr[0] != 0) return fail(c, DGCL_EINVAL, "link_ptr[0] != 0");
  T.link_ptr.assign(t->link_ptr, t->link_ptr + (size_t)m * m + 1);
  for (size_t p = 0; p < (size_t)m * m; ++p) {
    if (T.link_ptr[p + 1] < T.link_ptr[p]) return fail(c, DGCL_EINVAL, "link_ptr decreasing");
    if (p / m == p % m && T.link_ptr[p + 1] != T.link_ptr[p])
      return fail(c, DGCL_EINVAL, "self link %zu", p / m);
  }
  const int64_t nh = T.link_ptr[(size_t)m * m];
  if (nh > 0 && !t->link_hops) return DGCL_EINVAL;
  for (int64_t q = 0; q < nh; ++q) {
    if (t->link_hops[q] < 0 || t->link_hops[q] >= t->n_hops)
      return fail(c, DGCL_EINVAL, "link hop id out of range");
    T.link_hops.push_back(t->link_hops[q]);
  }
  c->topo = T;
  return DGCL_OK;
}

}  // extern "C"

namespace {

// build_plan / build_plan_from_trees: the relation, then a plan from SPST (trees == nullptr) or
// from the caller's saved trees, then lowering, workspace layout and the launch programs
dgcl_status plan_common(dgcl_ctx *c, const int64_t *req_ptr, const int64_t *req_ids,
                        uint64_t seed, int64_t n_edges, const int64_t *tu, const int32_t *tp,
                        const int32_t *tc, const int32_t *ts, bool trees) {
  if (!c || !req_ptr) return DGCL_EINVAL;
  if (c->planned) return fail(c, DGCL_ESTATE, "plan already built");
  if (req_ptr[c->world] > 0 && !req_ids) return DGCL_EINVAL;
  if (trees && (n_edges < 0 || (n_edges > 0 && (!tu || !tp || !tc || !ts)))) return DGCL_EINVAL;
  try {
    std::string e = build_relation(c->n, c->world, c->part.data(), req_ptr, req_ids, &c->rel);
    if (!e.empty()) return fail(c, DGCL_EINVAL, "%s", e.c_str());
    for (int d = 0; d < c->world; ++d)
      if (req_ptr[d + 1] - req_ptr[d] > INT32_MAX) return fail(c, DGCL_EINVAL, "halo too large");
    e = trees ? import_plan(c->topo, c->part.data(), c->rel, n_edges, tu, tp, tc, ts, &c->plan)
              : spst_plan(c->topo, c->part.data(), c->rel, seed, &c->plan, c->spst_fast);
    if (!e.empty()) return fail(c, DGCL_EPLAN, "%s", e.c_str());
    if (c->plan.n_stages >= kMaxStages) return fail(c, DGCL_EPLAN, "too many stages");
    relower(c);
    c->halo_off.assign(c->world + 1, 0);
    for (int d = 0; d < c->world; ++d) c->halo_off[d + 1] = c->halo_off[d] + c->rel.n_halo[d];
    compute_layout(c);
    for (int d = 0; d < c->world; ++d)  // direct-reduce terms hold 28-bit halo rows
      if (c->rel.n_halo[d] > (int64_t)kTermRowMask) c->direct_reduce = false;
    build_programs(c);
  } catch (const std::bad_alloc &) {
    return fail(c, DGCL_ENOMEM, "host allocation failed while planning");
  }
  c->planned = true;
  return DGCL_OK;
}

}  // namespace

extern "C" {

dgcl_status dgcl_build_plan(dgcl_ctx *c, const int64_t *req_ptr, const int64_t *req_ids,
                            uint64_t seed) {
  return plan_common(c, req_ptr, req_ids, seed, 0, nullptr, nullptr, nullptr, nullptr, false);
}

dgcl_status dgcl_build_plan_from_trees(dgcl_ctx *c, const int64_t *req_ptr,
                                       const int64_t *req_ids, int64_t n_edges, const int64_t *u,
                                       const int32_t *parent, const int32_t *child,
                                       const int32_t *stage) {
  return plan_common(c, req_ptr, req_ids, 0, n_edges, u, parent, child, stage, true);
}

dgcl_status dgcl_workspace_bytes(dgcl_ctx *c, size_t *bytes) {
  if (!c || !bytes) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  *bytes = c->ws_need[c->loopback ? 0 : c->rank];
  return DGCL_OK;
}

dgcl_status dgcl_register_workspace(dgcl_ctx *c, void *dev, size_t bytes) {
  if (!c) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  if (!has_device(c)) return fail(c, DGCL_ESTATE, "host-only context");
  if (c->registered) return fail(c, DGCL_ESTATE, "workspace already registered");
  if (!dev || ((uintptr_t)dev % kAlign)) return fail(c, DGCL_EINVAL, "workspace must be 256-B aligned");
  const size_t need = c->ws_need[c->loopback ? 0 : c->rank];
  if (bytes < need) return fail(c, DGCL_ENOMEM, "workspace %zu < %zu bytes", bytes, need);
  CUDA_TRY(c, cudaSetDevice(c->device));
  c->ws = (char *)dev;
  c->ws_bytes = bytes;
  c->base.assign(c->world, nullptr);
  if (c->loopback)
    for (int r = 0; r < c->world; ++r) c->base[r] = c->ws;
  else
    c->base[c->rank] = c->ws;
  // zero every flag region this context owns (monotonic counters start at 0)
  if (c->loopback) {
    CUDA_TRY(c, cudaMemset(c->ws, 0, (size_t)c->world * kFlagBytes));
    for (int r = 0; r < c->world && c->mc_bytes; ++r)
      CUDA_TRY(c, cudaMemset(c->ws + c->off_mc[r], 0, kMcFlagBytes));
  } else {
    CUDA_TRY(c, cudaMemset(c->ws, 0, kFlagBytes));
  }
  // device tables
  dgcl_status s;
  if ((s = upload(c, &c->d_groups, c->low.groups)) != DGCL_OK) return s;
  if ((s = upload(c, &c->d_waits, c->low.waits)) != DGCL_OK) return s;
  if ((s = upload(c, &c->d_idx, c->low.idx)) != DGCL_OK) return s;
  if ((s = upload(c, &c->d_term_ptr, c->low.term_ptr)) != DGCL_OK) return s;
  if ((s = upload(c, &c->d_terms, c->low.terms)) != DGCL_OK) return s;
  std::vector<DevItem> all;
  std::vector<DevRun> all_runs;
  std::vector<uint32_t> all_sterms;
  for (Program &p : c->progs) {
    p.dev_off = all.size();
    const int64_t run_base = (int64_t)all_runs.size();
    const int64_t sterm_base = (int64_t)all_sterms.size();
    for (DevItem it : p.items) {
      // program-relative -> pool indices
      if (it.op == OP_COPY) it.tp += run_base;
      if (it.op == OP_FOLD && (it.flags & kItemStaged)) {
        it.src += run_base;  // low bits: first segment
        it.t0 += sterm_base;
      }
      all.push_back(it);
    }
    all_runs.insert(all_runs.end(), p.runs.begin(), p.runs.end());
    all_sterms.insert(all_sterms.end(), p.sterms.begin(), p.sterms.end());
  }
  if ((s = upload(c, &c->d_items, all)) != DGCL_OK) return s;
  if ((s = upload(c, &c->d_runs, all_runs)) != DGCL_OK) return s;
  if ((s = upload(c, &c->d_sterms, all_sterms)) != DGCL_OK) return s;
  if ((s = upload(c, &c->d_claims, std::vector<uint64_t>(c->progs.size(), 0))) != DGCL_OK) return s;
  c->run_bytes = (int64_t)(all_runs.size() * sizeof(DevRun) + all_sterms.size() * 4);
  if (c->trace)
    for (Program &p : c->progs)
      if (!p.items.empty()) {
        CUDA_TRY(c, cudaMalloc((void **)&p.d_trace, p.items.size() * sizeof(TraceRec)));
        CUDA_TRY(c, cudaMemset(p.d_trace, 0, p.items.size() * sizeof(TraceRec)));
      }
  // watchdog word in mapped host memory
  CUDA_TRY(c, cudaHostAlloc((void **)&c->err_host, 64, cudaHostAllocMapped));
  std::memset(c->err_host, 0, 64);
  CUDA_TRY(c, cudaHostGetDevicePointer((void **)&c->err_dev, c->err_host, 0));
  // launch geometry: persistent grid of co-resident CTAs
  CUDA_TRY(c, cudaDeviceGetAttribute(&c->n_sm, cudaDevAttrMultiProcessorCount, c->device));
  int occ = 0;
  int e = executor_occupancy(c->threads, &occ);
  if (e != 0) return fail(c, DGCL_ECUDA, "occupancy query failed");
  // bulk-copy executor: co-resident CTAs per SM for every (geometry, CTA size) a program uses
  for (const Program &pg : c->progs) {
    const int block = tma_block(c, pg);
    const int mk = occ_mask(c, pg);
    if (c->tma_ctas.count({pg.geo, block, mk})) continue;
    const TmaGeometry &G = geometry_of(pg.geo);
    int n = 0;
    e = executor_tma_occupancy(mk, block, tma_smem_bytes(G), &n);
    if (e != 0) return fail(c, DGCL_ECUDA, "occupancy query failed");
    n = std::min(n, G.ctas_per_sm);
    if (c->ctas_set) n = std::min(n, c->ctas_per_sm);
    c->tma_ctas[{pg.geo, block, mk}] = n;
  }
  if (c->ctas_per_sm <= 0) c->ctas_per_sm = std::min(occ, 4);
  c->ctas_per_sm = std::max(1, std::min(c->ctas_per_sm, occ));
  c->grid = c->n_sm * c->ctas_per_sm;
  if (c->loopback && c->lb_flags == DGCL_LOOPBACK_PER_RANK) {
    c->rank_streams.assign(c->world, nullptr);
    c->rank_events.assign(c->world, nullptr);
    for (int r = 0; r < c->world; ++r) {
      CUDA_TRY(c, cudaStreamCreateWithFlags(&c->rank_streams[r], cudaStreamNonBlocking));
      CUDA_TRY(c, cudaEventCreateWithFlags(&c->rank_events[r], cudaEventDisableTiming));
    }
    CUDA_TRY(c, cudaEventCreateWithFlags(&c->fork_event, cudaEventDisableTiming));
  }
  CUDA_TRY(c, cudaDeviceSynchronize());
  c->registered = true;
  return DGCL_OK;
}

dgcl_status dgcl_halo_view(dgcl_ctx *c, int32_t layer, size_t *offset, int64_t *rows,
                           int64_t *pitch) {
  if (!c || !offset || !rows || !pitch) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  if (layer < 0 || layer >= c->n_layers) return fail(c, DGCL_EINVAL, "bad layer");
  const int r = c->loopback ? 0 : c->rank;
  *offset = c->off_halo[layer][r];
  *rows = c->loopback ? c->halo_off[c->world] : c->rel.n_halo[c->rank];
  *pitch = c->pitch[layer];
  return DGCL_OK;
}

dgcl_status dgcl_rank_rows(dgcl_ctx *c, int64_t *n_local, int64_t *n_halo) {
  if (!c || !n_local || !n_halo) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  for (int d = 0; d < c->world; ++d) {
    n_local[d] = c->n_local[d];
    n_halo[d] = c->rel.n_halo[d];
  }
  return DGCL_OK;
}

namespace {
struct IpcBlob {
  uint64_t magic;
  int32_t rank, world;
  uint64_t offset;   // workspace start within the exported allocation
  uint64_t bytes;
  cudaIpcMemHandle_t handle;
};
constexpr uint64_t kBlobMagic = 0x44474C4349504331ull;  // "DGCLIPC1"
static_assert(sizeof(IpcBlob) <= DGCL_IPC_BLOB_BYTES, "blob size");
}  // namespace

dgcl_status dgcl_ipc_export(dgcl_ctx *c, void *blob, size_t *len) {
  if (!c || !blob || !len) return DGCL_EINVAL;
  if (!c->registered) return fail(c, DGCL_ESTATE, "workspace not registered");
  if (*len < sizeof(IpcBlob)) return fail(c, DGCL_EINVAL, "blob capacity too small");
  IpcBlob b;
  std::memset(&b, 0, sizeof(b));
  b.magic = kBlobMagic;
  b.rank = c->rank;
  b.world = c->world;
  b.bytes = c->ws_bytes;
  // allocation base of the (possibly sub-allocated, e.g. PyTorch caching allocator) workspace;
  // the driver entry point is resolved through the runtime so libdgcl does not link libcuda
  typedef CUresult (*GetRange)(CUdeviceptr *, size_t *, CUdeviceptr);
  void *fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CUDA_TRY(c, cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q));
  if (!fn || q != cudaDriverEntryPointSuccess)
    return fail(c, DGCL_ECUDA, "cuMemGetAddressRange entry point unavailable");
  CUdeviceptr base = 0;
  size_t sz = 0;
  CUresult cr = ((GetRange)fn)(&base, &sz, (CUdeviceptr)c->ws);
  if (cr != CUDA_SUCCESS) return fail(c, DGCL_ECUDA, "cuMemGetAddressRange failed (%d)", (int)cr);
  b.offset = (uint64_t)((CUdeviceptr)c->ws - base);
  CUDA_TRY(c, cudaIpcGetMemHandle(&b.handle, (void *)base));
  std::memcpy(blob, &b, sizeof(b));
  *len = sizeof(b);
  return DGCL_OK;
}

dgcl_status dgcl_ipc_import(dgcl_ctx *c, const void *blobs, size_t len_each) {
  if (!c || !blobs) return DGCL_EINVAL;
  if (!c->registered) return fail(c, DGCL_ESTATE, "workspace not registered");
  if (c->loopback) return fail(c, DGCL_ESTATE, "loopback contexts have no peers");
  if (c->imported) return fail(c, DGCL_ESTATE, "already imported");
  if (len_each < sizeof(IpcBlob)) return fail(c, DGCL_EINVAL, "blob too small");
  CUDA_TRY(c, cudaSetDevice(c->device));
  for (int r = 0; r < c->world; ++r) {
    if (r == c->rank) continue;
    IpcBlob b;
    std::memcpy(&b, (const char *)blobs + (size_t)r * len_each, sizeof(b));
    if (b.magic != kBlobMagic || b.rank != r || b.world != c->world)
      return fail(c, DGCL_EINVAL, "bad IPC blob for rank %d", r);
    if (b.bytes < c->ws_need[r]) return fail(c, DGCL_EINVAL, "peer %d workspace too small", r);
    void *p = nullptr;
    CUDA_TRY(c, cudaIpcOpenMemHandle(&p, b.handle, cudaIpcMemLazyEnablePeerAccess));
    c->ipc_opened.push_back((char *)p);
    c->base[r] = (char *)p + b.offset;
  }
  c->imported = true;
  return DGCL_OK;
}

dgcl_status dgcl_dispatch_forward(dgcl_ctx *c, int32_t layer, const float *emb, int64_t emb_pitch,
                                  float *halo, void *stream) {
  dgcl_status s = ready_to_dispatch(c, layer);
  if (s != DGCL_OK) return s;
  if (emb_pitch < c->dims[layer]) return fail(c, DGCL_EINVAL, "emb_pitch < dim");
  const char *view = c->base[c->loopback ? 0 : c->rank] + c->off_halo[layer][c->loopback ? 0 : c->rank];
  if (halo && (const char *)halo != view) return fail(c, DGCL_EINVAL, "halo is not the registered view");
  const int64_t rows = c->loopback ? c->n : c->n_local[c->rank];
  if (rows > 0 && !emb) return fail(c, DGCL_EINVAL, "emb is NULL");
  if (c->world == 1) return DGCL_OK;
  c->seq++;
  c->epoch[DIR_FWD]++;
  return launch(c, layer, DIR_FWD, emb, emb_pitch, nullptr, 0, (cudaStream_t)stream);
}

dgcl_status dgcl_dispatch_backward(dgcl_ctx *c, int32_t layer, const float *halo_grad,
                                   int64_t hg_pitch, float *emb_grad, int64_t eg_pitch,
                                   void *stream) {
  dgcl_status s = ready_to_dispatch(c, layer);
  if (s != DGCL_OK) return s;
  if (hg_pitch < c->dims[layer] || eg_pitch < c->dims[layer])
    return fail(c, DGCL_EINVAL, "pitch < dim");
  const int64_t hrows = c->loopback ? c->halo_off[c->world] : c->rel.n_halo[c->rank];
  const int64_t rows = c->loopback ? c->n : c->n_local[c->rank];
  if ((hrows > 0 && !halo_grad) || (rows > 0 && !emb_grad))
    return fail(c, DGCL_EINVAL, "NULL buffer");
  if (c->world == 1) return DGCL_OK;
  c->seq++;
  c->epoch[DIR_BWD]++;
  return launch(c, layer, DIR_BWD, halo_grad, hg_pitch, emb_grad, eg_pitch, (cudaStream_t)stream);
}

static dgcl_status get_stage(dgcl_ctx *c, int kind, int layer, size_t bytes,
                             dgcl_ctx::Stage **out) {
  dgcl_ctx::Stage &S = c->stages[kind * 4096 + layer];
  if (!S.free) CUDA_TRY(c, cudaEventCreateWithFlags(&S.free, cudaEventDisableTiming));
  if (S.bytes < bytes) {
    // the old buffer may still be in use by queued work: wait for it before freeing
    if (S.ptr) {
      CUDA_TRY(c, cudaEventSynchronize(S.free));
      cudaFree(S.ptr);
    }
    S.ptr = nullptr;
    S.bytes = 0;
    if (cudaMalloc(&S.ptr, std::max<size_t>(bytes, 256)) != cudaSuccess)
      return fail(c, DGCL_ENOMEM, "staging allocation of %zu bytes failed", bytes);
    S.bytes = bytes;
  }
  if (!c->h2d_stream) {
    CUDA_TRY(c, cudaStreamCreateWithFlags(&c->h2d_stream, cudaStreamNonBlocking));
    CUDA_TRY(c, cudaStreamCreateWithFlags(&c->d2h_stream, cudaStreamNonBlocking));
  }
  *out = &S;
  return DGCL_OK;
}

// `to` waits for the work queued so far on `from`
static dgcl_status stream_after(dgcl_ctx *c, cudaStream_t to, cudaStream_t from) {
  cudaEvent_t e;
  CUDA_TRY(c, cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  CUDA_TRY(c, cudaEventRecord(e, from));
  CUDA_TRY(c, cudaStreamWaitEvent(to, e, 0));
  cudaEventDestroy(e);  // released once the recorded work completes
  return DGCL_OK;
}

// host -> staging on the copy stream, after the staging buffer's last reader; `st` waits for it
static dgcl_status stage_in(dgcl_ctx *c, dgcl_ctx::Stage *S, const void *host, size_t bytes,
                            cudaStream_t st) {
  if (!bytes) return DGCL_OK;
  CUDA_TRY(c, cudaStreamWaitEvent(c->h2d_stream, S->free, 0));
  CUDA_TRY(c, cudaMemcpyAsync(S->ptr, host, bytes, cudaMemcpyHostToDevice, c->h2d_stream));
  return stream_after(c, st, c->h2d_stream);
}

// device -> host on the second copy stream once `st`'s work is done; `st` then waits for the copy
// (so synchronizing the caller's stream means the host result is there), `src_free` is recorded
// after it, and in synchronous mode the call waits
static dgcl_status stage_out(dgcl_ctx *c, void *host, const void *dev, size_t bytes,
                             cudaStream_t st, cudaEvent_t src_free) {
  dgcl_status s = stream_after(c, c->d2h_stream, st);
  if (s != DGCL_OK) return s;
  if (bytes)
    CUDA_TRY(c, cudaMemcpyAsync(host, dev, bytes, cudaMemcpyDeviceToHost, c->d2h_stream));
  if (src_free) CUDA_TRY(c, cudaEventRecord(src_free, c->d2h_stream));
  if ((s = stream_after(c, st, c->d2h_stream)) != DGCL_OK) return s;
  if (!c->host_async) CUDA_TRY(c, cudaStreamSynchronize(st));
  return check_dead(c);
}

dgcl_status dgcl_device_barrier(dgcl_ctx *c, void *stream) {
  if (!c) return DGCL_EINVAL;
  if (!has_device(c)) return fail(c, DGCL_ESTATE, "host-only context");
  if (!c->registered) return fail(c, DGCL_ESTATE, "workspace not registered");
  if (!c->loopback && c->world > 1 && !c->imported) return fail(c, DGCL_ESTATE, "peers not imported");
  dgcl_status s = check_dead(c);
  if (s != DGCL_OK) return s;
  if (c->world == 1) return DGCL_OK;
  DeviceGuard guard(c->device);
  ExecParams P;
  std::memset(&P, 0, sizeof(P));
  for (int r = 0; r < c->world; ++r) P.flags[r] = (uint64_t *)(c->base[r] + c->off_flags[r]);
  P.world = c->world;
  P.seq = ++c->barrier_seq;
  P.sys_scope = c->loopback ? 0 : 1;
  P.timeout_ns = (uint64_t)c->timeout_ms * 1000000ull;
  P.err = c->err_dev;
  // a fused loopback context is one launch stream: its virtual ranks arrive together
  const int first = c->loopback ? 0 : c->rank, count = c->loopback ? c->world : 1;
  const int e = launch_barrier(P, first, count, stream);
  if (e != 0) return fail(c, DGCL_ECUDA, "barrier launch failed: %s", cudaGetErrorString((cudaError_t)e));
  return DGCL_OK;
}

dgcl_status dgcl_multicast_supported(int32_t cuda_device, int32_t *supported) {
  if (!supported) return DGCL_EINVAL;
  *supported = mc_supported(cuda_device) ? 1 : 0;
  return DGCL_OK;
}

dgcl_status dgcl_multicast_bytes(dgcl_ctx *c, size_t *bytes, int64_t *rows) {
  if (!c || !bytes) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  *bytes = c->mc_bytes;
  if (rows) *rows = c->low.mc_total;
  return DGCL_OK;
}

dgcl_status dgcl_multicast_open(dgcl_ctx *c, int32_t *fd) {
  if (!c || !fd) return DGCL_EINVAL;
  if (!c->registered) return fail(c, DGCL_ESTATE, "workspace not registered");
  if (c->loopback) return fail(c, DGCL_ESTATE, "loopback contexts emulate the multicast");
  if (c->mc_bytes == 0) return fail(c, DGCL_ESTATE, "no multicast rows planned (option multicast)");
  if (c->mc_have_handle) return fail(c, DGCL_ESTATE, "multicast object already open");
  if (!mc_supported(c->device))
    return fail(c, DGCL_ECUDA, "device %d does not support multicast objects", c->device);
  DeviceGuard guard(c->device);
  const McDriver &D = mcd();
  CUmulticastObjectProp prop = mc_prop(c->world, c->mc_bytes);
  size_t g = 0;
  CUresult r = D.gran(&g, &prop, CU_MULTICAST_GRANULARITY_MINIMUM);
  if (r != CUDA_SUCCESS || g == 0) return fail(c, DGCL_ECUDA, "cuMulticastGetGranularity (%d)", (int)r);
  c->mc_map_bytes = (c->mc_bytes + g - 1) / g * g;
  prop.size = c->mc_map_bytes;
  if (c->rank == 0) {
    if ((r = D.create(&c->mc_handle, &prop)) != CUDA_SUCCESS)
      return fail(c, DGCL_ECUDA, "cuMulticastCreate (%d)", (int)r);
    c->mc_have_handle = true;
    int out = -1;
    if ((r = D.exportH(&out, c->mc_handle, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0)) != CUDA_SUCCESS)
      return fail(c, DGCL_ECUDA, "cuMemExportToShareableHandle (%d)", (int)r);
    *fd = out;
  } else {
    if ((r = D.importH(&c->mc_handle, (void *)(intptr_t)*fd, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR)) !=
        CUDA_SUCCESS)
      return fail(c, DGCL_ECUDA, "cuMemImportFromShareableHandle (%d)", (int)r);
    c->mc_have_handle = true;
  }
  return DGCL_OK;
}

dgcl_status dgcl_multicast_add(dgcl_ctx *c) {
  if (!c) return DGCL_EINVAL;
  if (!c->mc_have_handle) return fail(c, DGCL_ESTATE, "dgcl_multicast_open first");
  if (c->mc_added) return fail(c, DGCL_ESTATE, "device already added");
  DeviceGuard guard(c->device);
  const CUresult r = mcd().addDevice(c->mc_handle, (CUdevice)c->device);
  if (r != CUDA_SUCCESS) return fail(c, DGCL_ECUDA, "cuMulticastAddDevice (%d)", (int)r);
  c->mc_added = true;
  return DGCL_OK;
}

dgcl_status dgcl_multicast_bind(dgcl_ctx *c) {
  if (!c) return DGCL_EINVAL;
  if (!c->mc_added) return fail(c, DGCL_ESTATE, "dgcl_multicast_add first (on every rank)");
  if (c->mc_uc) return fail(c, DGCL_ESTATE, "already bound");
  DeviceGuard guard(c->device);
  const CUresult r = mc_bind_map(c->device, c->mc_handle, c->mc_map_bytes, &c->mc_mem, &c->mc_uc,
                                 &c->mc_va);
  c->mc_have_mem = c->mc_mem != 0;
  if (r != CUDA_SUCCESS) return fail(c, DGCL_ECUDA, "multicast bind / map (%d)", (int)r);
  CUDA_TRY(c, cudaMemset(c->mc_uc, 0, kMcFlagBytes));
  CUDA_TRY(c, cudaDeviceSynchronize());
  return DGCL_OK;
}

dgcl_status dgcl_debug_multicast_selftest(int32_t cuda_device, int64_t bytes, char *msg,
                                          size_t msg_len) {
  auto say = [&](const char *fmt, int v) {
    if (msg && msg_len) std::snprintf(msg, msg_len, fmt, v);
  };
  if (bytes < 4096) bytes = 4096;
  if (!mc_supported(cuda_device)) {
    say("multicast not supported on device %d", cuda_device);
    return DGCL_ECUDA;
  }
  if (cudaSetDevice(cuda_device) != cudaSuccess) return DGCL_ECUDA;
  const McDriver &D = mcd();
  CUmulticastObjectProp prop = mc_prop(1, (size_t)bytes);
  size_t g = 0;
  CUresult r = D.gran(&g, &prop, CU_MULTICAST_GRANULARITY_MINIMUM);
  if (r != CUDA_SUCCESS) { say("cuMulticastGetGranularity %d", (int)r); return DGCL_ECUDA; }
  const size_t sz = ((size_t)bytes + g - 1) / g * g;
  prop.size = sz;
  CUmemGenericAllocationHandle h = 0, mem = 0;
  char *uc = nullptr, *mc = nullptr;
  dgcl_status st = DGCL_OK;
  if ((r = D.create(&h, &prop)) != CUDA_SUCCESS) { say("cuMulticastCreate %d", (int)r); return DGCL_ECUDA; }
  if ((r = D.addDevice(h, (CUdevice)cuda_device)) != CUDA_SUCCESS) {
    say("cuMulticastAddDevice %d", (int)r);
    st = DGCL_ECUDA;
  } else if ((r = mc_bind_map(cuda_device, h, sz, &mem, &uc, &mc)) != CUDA_SUCCESS) {
    say("bind / map %d", (int)r);
    st = DGCL_ECUDA;
  } else {
    // region = [flag 4 KB | data]: chunk i of the data through the multicast address
    const int n16 = (int)((sz - 4096) / 16 < 65536 ? (sz - 4096) / 16 : 65536);
    std::vector<int32_t> hostv((size_t)n16 * 4);
    uint64_t flag = 0;
    if (cudaMemset(uc, 0, sz) != cudaSuccess ||
        launch_mc_selftest(mc + 4096, (uint64_t *)mc, n16, nullptr) != 0 ||
        cudaDeviceSynchronize() != cudaSuccess ||
        cudaMemcpy(hostv.data(), uc + 4096, hostv.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess ||
        cudaMemcpy(&flag, uc, 8, cudaMemcpyDeviceToHost) != cudaSuccess) {
      say("kernel / copy failed (%d)", (int)cudaGetLastError());
      st = DGCL_ECUDA;
    } else {
      int bad = 0;
      for (int i = 0; i < n16; ++i)
        bad += hostv[4 * i] != i || hostv[4 * i + 1] != (i ^ 0x5a5a5a5a) || hostv[4 * i + 2] != ~i ||
               hostv[4 * i + 3] != 7;
      if (bad || flag != 5) {
        say("wrong data through the unicast view (%d bad chunks)", bad);
        st = DGCL_EPLAN;
      } else {
        say("ok: %d chunks stored through the multicast address, reduction seen", n16);
      }
    }
  }
  mc_teardown(cuda_device, h, true, mem, mem != 0, uc, mc, sz);
  return st;
}

dgcl_status dgcl_stream_wait_arrival(dgcl_ctx *c, int32_t dst, int32_t src, void *stream) {
  if (!c) return DGCL_EINVAL;
  if (!has_device(c)) return fail(c, DGCL_ESTATE, "host-only context");
  if (!c->registered) return fail(c, DGCL_ESTATE, "workspace not registered");
  if (!c->loopback && c->world > 1 && !c->imported) return fail(c, DGCL_ESTATE, "peers not imported");
  if (dst < 0) dst = c->rank;
  if (dst >= c->world || src < -1 || src >= c->world || src == dst)
    return fail(c, DGCL_EINVAL, "bad (dst %d, src %d)", dst, src);
  if (!c->loopback && dst != c->rank) return fail(c, DGCL_EINVAL, "dst must be this rank");
  if (c->loopback && c->lb_flags == DGCL_LOOPBACK_FUSED && !c->signal_all)
    return fail(c, DGCL_ESTATE, "fused loopback publishes arrivals only with option signal_all");
  dgcl_status s = check_dead(c);
  if (s != DGCL_OK) return s;
  if (c->world == 1 || c->epoch[DIR_FWD] == 0) return DGCL_OK;
  // the forward-completion wait list of dst: every incoming counter of every stage; a
  // single-stage plan's entry for src is exactly "all rows from src have landed"
  const Lowered &L = c->low;
  int32_t off = -1, n = 0;
  for (const DevGroup &g : L.groups)
    if (g.op == OP_WAIT && g.exec_rank == dst) {
      off = g.wait_off;
      n = g.wait_n;
    }
  if (off < 0) return fail(c, DGCL_EPLAN, "no completion list for rank %d", dst);
  // multicast: the rows of src that came through the multicast region land with dst's unpack
  int32_t mc_w = -1;
  if (!L.mc_unpack_wait.empty()) {
    if (src >= 0) {
      mc_w = L.mc_unpack_wait[(size_t)dst * c->world + src];
    } else {
      for (int s2 = 0; s2 < c->world; ++s2) {  // every source: one wait launch per unpack
        const int32_t w = L.mc_unpack_wait[(size_t)dst * c->world + s2];
        if (w >= 0) {
          dgcl_status st = dgcl_stream_wait_arrival(c, dst, s2, stream);
          if (st != DGCL_OK) return st;
        }
      }
    }
  }
  if (src >= 0 && L.n_stages <= 1) {
    const int32_t want = (int32_t)ctr_index(DIR_FWD, 1, src, 0);
    int32_t hit = -1;
    for (int32_t w = off; w < off + n; ++w)
      if (L.waits[w].ctr == want) hit = w;
    off = hit;
    n = hit < 0 ? 0 : 1;  // (hit < 0: nothing comes from src directly)
  }
  if (n == 0 && mc_w < 0) return DGCL_OK;
  DeviceGuard guard(c->device);
  ExecParams P;
  std::memset(&P, 0, sizeof(P));
  for (int r = 0; r < c->world; ++r) P.flags[r] = (uint64_t *)(c->base[r] + c->off_flags[r]);
  P.world = c->world;
  P.waits = c->d_waits;
  P.epoch[DIR_FWD] = c->epoch[DIR_FWD];
  P.timeout_ns = (uint64_t)c->timeout_ms * 1000000ull;
  P.err = c->err_dev;
  P.sys_scope = c->loopback ? 0 : 1;
  int e = n > 0 ? launch_wait(P, dst, off, n, stream) : 0;
  if (e == 0 && mc_w >= 0) e = launch_wait(P, dst, mc_w, 1, stream);
  if (e != 0) return fail(c, DGCL_ECUDA, "wait launch failed: %s", cudaGetErrorString((cudaError_t)e));
  return DGCL_OK;
}

dgcl_status dgcl_forward_host(dgcl_ctx *c, int32_t layer, const float *host_emb, float *host_halo,
                              void *stream) {
  dgcl_status s = ready_to_dispatch(c, layer);
  if (s != DGCL_OK) return s;
  const int64_t p = c->pitch[layer];
  const int64_t rows = c->loopback ? c->n : c->n_local[c->rank];
  const int64_t hrows = c->loopback ? c->halo_off[c->world] : c->rel.n_halo[c->rank];
  cudaStream_t st = (cudaStream_t)stream;
  dgcl_ctx::Stage *E;
  if ((s = get_stage(c, 0, layer, rows * p * 4, &E)) != DGCL_OK) return s;
  if ((s = stage_in(c, E, host_emb, rows * p * 4, st)) != DGCL_OK) return s;
  if ((s = dgcl_dispatch_forward(c, layer, (const float *)E->ptr, p, nullptr, stream)) != DGCL_OK)
    return s;
  CUDA_TRY(c, cudaEventRecord(E->free, st));
  const char *view = c->base[c->loopback ? 0 : c->rank] + c->off_halo[layer][c->loopback ? 0 : c->rank];
  // (the next call writing this halo is queued on `st` after this copy: stage_out makes `st` wait)
  return stage_out(c, host_halo, view, hrows * p * 4, st, nullptr);
}

dgcl_status dgcl_backward_host(dgcl_ctx *c, int32_t layer, const float *host_halo_grad,
                               float *host_emb_grad, void *stream) {
  dgcl_status s = ready_to_dispatch(c, layer);
  if (s != DGCL_OK) return s;
  const int64_t p = c->pitch[layer];
  const int64_t rows = c->loopback ? c->n : c->n_local[c->rank];
  const int64_t hrows = c->loopback ? c->halo_off[c->world] : c->rel.n_halo[c->rank];
  cudaStream_t st = (cudaStream_t)stream;
  dgcl_ctx::Stage *G, *E;
  if ((s = get_stage(c, 1, layer, hrows * p * 4, &G)) != DGCL_OK) return s;
  if ((s = get_stage(c, 2, layer, rows * p * 4, &E)) != DGCL_OK) return s;
  if ((s = stage_in(c, G, host_halo_grad, hrows * p * 4, st)) != DGCL_OK) return s;
  if ((s = stage_in(c, E, host_emb_grad, rows * p * 4, st)) != DGCL_OK) return s;
  if ((s = dgcl_dispatch_backward(c, layer, (const float *)G->ptr, p, (float *)E->ptr, p,
                                  stream)) != DGCL_OK)
    return s;
  CUDA_TRY(c, cudaEventRecord(G->free, st));
  return stage_out(c, host_emb_grad, E->ptr, rows * p * 4, st, E->free);
}

dgcl_status dgcl_plan_info(dgcl_ctx *c, dgcl_plan_stats *info) {
  if (!c || !info) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  std::memset(info, 0, sizeof(*info));
  info->world = c->world;
  info->n_stages = c->plan.n_stages;
  info->n_vertices_planned = (int64_t)c->plan.order.size();
  info->n_deliveries = c->rel.d_ptr[c->rel.n];
  info->n_tree_edges = c->low.n_tree_edges;
  info->n_relay_rows = c->low.n_relay_edges;
  info->model_cost_ticks = c->plan.cost;
  int64_t item_bytes = 0;
  for (const Program &p : c->progs) item_bytes += (int64_t)(p.items.size() * sizeof(DevItem));
  info->table_bytes = c->low.table_bytes() + item_bytes;
  info->planner_seconds = c->plan.seconds;
  info->lowering_seconds = c->low.seconds;
  int nf = 0, nb = 0;
  for (const DevGroup &g : c->low.groups) {
    if (g.op == OP_READY || g.op == OP_WAIT) continue;
    (g.dir == DIR_FWD ? nf : nb)++;
  }
  info->n_fwd_groups = nf;
  info->n_bwd_groups = nb;
  info->n_multicast_rows = c->low.mc_total;
  return DGCL_OK;
}

dgcl_status dgcl_plan_counts(dgcl_ctx *c, int64_t *rows) {
  if (!c || !rows) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  const int m = c->world, K = c->plan.n_stages;
  for (int k = 1; k <= K; ++k)
    for (int s = 0; s < m; ++s)
      for (int d = 0; d < m; ++d)
        rows[((size_t)(k - 1) * m + s) * m + d] = c->low.rows(DIR_FWD, k, s, d);
  // multicast deliveries are stage-1 rows s -> d too (their counters are the multicast ones)
  for (size_t i = 0; i < c->low.mc_unpack_wait.size(); ++i)
    if (c->low.mc_unpack_wait[i] >= 0) {
      const int d = (int)(i / m), s = (int)(i % m);
      rows[(size_t)s * m + d] += c->low.waits[c->low.mc_unpack_wait[i]].amount;
    }
  return DGCL_OK;
}

dgcl_status dgcl_plan_export(dgcl_ctx *c, int64_t *n_edges, int64_t *u, int32_t *parent,
                             int32_t *child, int32_t *stage) {
  if (!c || !n_edges) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  const int64_t NE = (int64_t)c->plan.e_parent.size();
  if (!u && !parent && !child && !stage) {
    *n_edges = NE;
    return DGCL_OK;
  }
  if (!u || !parent || !child || !stage || *n_edges < NE) return DGCL_EINVAL;
  for (size_t i = 0; i < c->plan.order.size(); ++i)
    for (int64_t e = c->plan.e_ptr[i]; e < c->plan.e_ptr[i + 1]; ++e) {
      u[e] = c->plan.order[i];
      parent[e] = c->plan.e_parent[e];
      child[e] = c->plan.e_child[e];
      stage[e] = c->plan.e_stage[e];
    }
  *n_edges = NE;
  return DGCL_OK;
}

dgcl_status dgcl_set_option(dgcl_ctx *c, const char *key, int64_t value) {
  if (!c || !key) return DGCL_EINVAL;
  const std::string k(key);
  if (k == "timeout_ms") {
    if (value < 1) return fail(c, DGCL_EINVAL, "timeout_ms must be >= 1");
    c->timeout_ms = value;
    return DGCL_OK;
  }
  if (k == "geometry") {  // bulk-copy launch geometry: 0 auto, 1 WIDE, 2 DUAL (TmaGeometry)
    if (value < 0 || value > 2) return fail(c, DGCL_EINVAL, "geometry must be 0, 1 or 2");
    if (c->registered) return fail(c, DGCL_ESTATE, "geometry must be set before registration");
    c->geometry = (int)value;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "spst_fast") {  // before dgcl_build_plan: 0 = always run Algorithm 1's loop
    if (c->planned) return fail(c, DGCL_ESTATE, "spst_fast must be set before dgcl_build_plan");
    c->spst_fast = value != 0;
    return DGCL_OK;
  }
  if (k == "claim_batch") {  // dynamic item claiming: -1 auto, 0 off, k >= 1 batch size; any time
    if (value < -1 || value > 64) return fail(c, DGCL_EINVAL, "claim_batch in -1..64");
    c->claim_batch = (int)value;
    return DGCL_OK;
  }
  if (k == "sys_scope") {  // loopback: 1 = the multi-GPU system-scope flag protocol (A/B)
    c->force_sys_scope = value != 0;
    return DGCL_OK;
  }
  if (k == "l2_policy") {  // L2 eviction hints, bit mask (executor_tma.cu); any time
    if (value < 0 || value > 15) return fail(c, DGCL_EINVAL, "l2_policy in 0..15");
    c->l2_policy = (int)value;
    return DGCL_OK;
  }
  if (k == "sm_budget") {  // SMs per executor launch (0 = all); any time
    if (value < 0) return fail(c, DGCL_EINVAL, "sm_budget must be >= 0");
    c->sm_budget = (int)value;
    return DGCL_OK;
  }
  if (k == "trace") {  // per-item timelines of every launch (dgcl_trace_read)
    c->trace = value != 0;
    return DGCL_OK;
  }
  if (k == "small_launch_bytes") {  // below: register executor (latency), 0 = always bulk-copy
    if (value < 0) return fail(c, DGCL_EINVAL, "small_launch_bytes must be >= 0");
    c->small_launch_bytes = value;
    return DGCL_OK;
  }
  if (k == "host_async") {  // host-buffer calls return once queued (see dgcl_forward_host)
    c->host_async = value != 0;
    return DGCL_OK;
  }
  if (k == "dual_producer") {  // simple copy launches: two producer warps (any time)
    c->dual_producer = value != 0;
    return DGCL_OK;
  }
  if (k == "dual_claims") {  // dual producers also for launches with dynamic claims (any time)
    c->dual_claims = value != 0;
    return DGCL_OK;
  }
  if (k == "hostsim_items") {  // verification aid: the host interpreter runs the work items
    c->hostsim_items = value != 0;
    return DGCL_OK;
  }
  if (k == "debug_skip_rank") {
    if (value < -1 || value >= c->world) return fail(c, DGCL_EINVAL, "debug_skip_rank");
    c->debug_skip_rank = (int)value;
    return DGCL_OK;
  }
  if (c->registered) return fail(c, DGCL_ESTATE, "option %s must be set before registration", key);
  if (k == "item_bytes") {
    if (value < 16) return fail(c, DGCL_EINVAL, "item_bytes too small");
    c->item_bytes = value;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "tma") {
    c->use_tma = value != 0;
    return DGCL_OK;
  }
  if (k == "direct_copy_rows") {
    if (value < 0) return fail(c, DGCL_EINVAL, "direct_copy_rows must be >= 0");
    c->direct_copy_rows = value;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "gather4") {  // TMA gather4 (four rows per instruction) for short-run row gathers
    c->use_gather4 = value != 0;
    return DGCL_OK;
  }
  if (k == "bulk_store") {  // TMA stores for local (loopback) destinations
    c->bulk_store_local = value != 0;
    return DGCL_OK;
  }
  if (k == "bulk_store_peer") {  // TMA stores into peer memory (multi-GPU)
    c->bulk_store_peer = value != 0;
    return DGCL_OK;
  }
  if (k == "stage_fold") {  // bulk-copy FOLD operand rows into the stage (bulk-copy executor)
    c->stage_fold = value != 0;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "owner_major") {  // fused loopback forwards: items of one owner's groups at a time
    if (value < 0 || value > 2) return fail(c, DGCL_EINVAL, "owner_major in 0..2");
    c->owner_major = (int)value;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "relay_lead_kb") {  // relay forwards: KB of leaves between stages (-1: build order)
    if (value < -1 || value > (1 << 30)) return fail(c, DGCL_EINVAL, "relay_lead_kb in -1..2^30");
    c->relay_lead_kb = value;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "leaf_split") {  // relay plans: 0 off, 1 stages >= 2, 2 every stage (see lower_plan)
    if (value < 0 || value > 2) return fail(c, DGCL_EINVAL, "leaf_split in 0..2");
    c->leaf_split = (int)value;
    if (c->planned) {
      relower(c);
      compute_layout(c);
      build_programs(c);
    }
    return DGCL_OK;
  }
  if (k == "pipeline_blocks") {  // relay plans: stage chaining per vertex block (1..8)
    if (value < 1 || value > kMaxBlocks) return fail(c, DGCL_EINVAL, "pipeline_blocks in 1..%d", kMaxBlocks);
    c->pipeline_blocks = (int)value;
    if (c->planned) {
      relower(c);
      compute_layout(c);
      build_programs(c);
    }
    return DGCL_OK;
  }
  if (k == "signal_all") {  // fused loopback: every item publishes its done count
    c->signal_all = value != 0;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "lsu_gather") {  // short-run COPY items: consumer cp.async gathers (bulk-copy executor)
    c->lsu_gather = value != 0;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "align_sources") {  // forward COPY groups of one source rank: common item boundaries
    c->align_sources = value != 0;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "multicast") {  // NVSwitch multicast of high-fan-out rows (0 off, 1 all peers, k >= 2)
    if (value < 0 || value > kMaxRanks) return fail(c, DGCL_EINVAL, "multicast in 0..%d", kMaxRanks);
    c->multicast = (int)value;
    if (c->planned) {
      relower(c);
      compute_layout(c);
      build_programs(c);
    }
    return DGCL_OK;
  }
  if (k == "fanout") {  // forward stage 1: per-owner fan-out items (1) or per-pair COPY items (0)
    c->fanout = value != 0;
    if (c->planned) {  // its groups are lowered only when asked for
      relower(c);
      compute_layout(c);
      build_programs(c);
    }
    return DGCL_OK;
  }
  if (k == "atomic_backward") {  // ablation: loopback single-stage backward with atomic adds
    c->atomic_backward = value != 0;
    if (c->planned) {  // its groups are lowered only when asked for
      relower(c);
      compute_layout(c);
      build_programs(c);
    }
    return DGCL_OK;
  }
  if (k == "direct_reduce") {
    c->direct_reduce = value != 0;
    if (c->planned) build_programs(c);
    return DGCL_OK;
  }
  if (k == "ctas_per_sm") {
    if (value < 1 || value > 32) return fail(c, DGCL_EINVAL, "ctas_per_sm out of range");
    c->ctas_per_sm = (int)value;
    c->ctas_set = true;
    return DGCL_OK;
  }
  if (k == "threads") {
    if (value < 128 || value > 512 || value % 32) return fail(c, DGCL_EINVAL, "threads");
    c->threads = (int)value;
    c->threads_set = true;
    return DGCL_OK;
  }
  return fail(c, DGCL_EINVAL, "unknown option %s", key);
}

dgcl_status dgcl_trace_read(dgcl_ctx *c, int32_t layer, int32_t dir, int32_t rank,
                            dgcl_trace_rec *recs, int64_t *n) {
  if (!c || !n) return DGCL_EINVAL;
  if (!c->registered || !c->trace) return fail(c, DGCL_ESTATE, "tracing is off (option \"trace\")");
  if (layer < 0 || layer >= c->n_layers || dir < 0 || dir > 1) return DGCL_EINVAL;
  const bool fused = c->loopback && c->lb_flags == DGCL_LOOPBACK_FUSED;
  if (fused) rank = 0;
  else if (!c->loopback) rank = c->rank;
  if (rank < 0 || rank >= c->n_prog_ranks) return DGCL_EINVAL;
  const Program &pg = c->progs[c->prog_index(layer, dir, rank)];
  const int64_t cnt = (int64_t)pg.items.size();
  if (!recs) {
    *n = cnt;
    return DGCL_OK;
  }
  if (*n < cnt) return fail(c, DGCL_EINVAL, "trace buffer holds %lld < %lld records",
                            (long long)*n, (long long)cnt);
  static_assert(sizeof(dgcl_trace_rec) == sizeof(TraceRec), "trace record layout");
  CUDA_TRY(c, cudaSetDevice(c->device));
  CUDA_TRY(c, cudaDeviceSynchronize());
  if (cnt) CUDA_TRY(c, cudaMemcpy(recs, pg.d_trace, cnt * sizeof(TraceRec), cudaMemcpyDeviceToHost));
  *n = cnt;
  return DGCL_OK;
}

dgcl_status dgcl_launch_count(dgcl_ctx *c, uint64_t *count) {
  if (!c || !count) return DGCL_EINVAL;
  *count = c->launches;
  return DGCL_OK;
}

dgcl_status dgcl_check(dgcl_ctx *c) {
  if (!c) return DGCL_EINVAL;
  dgcl_status s = check_dead(c);
  if (s != DGCL_OK) return s;
  if (has_device(c)) {
    cudaError_t e = cudaPeekAtLastError();
    if (e != cudaSuccess) return fail(c, DGCL_ECUDA, "sticky CUDA error: %s", cudaGetErrorString(e));
  }
  return DGCL_OK;
}

const char *dgcl_last_error(dgcl_ctx *c) { return c ? c->err.c_str() : "null context"; }

const char *dgcl_strerror(dgcl_status s) {
  switch (s) {
    case DGCL_OK: return "ok";
    case DGCL_EINVAL: return "invalid argument";
    case DGCL_ESTATE: return "invalid call order / state";
    case DGCL_ECUDA: return "CUDA error";
    case DGCL_ENOMEM: return "out of memory";
    case DGCL_ETIMEOUT: return "device flag wait timed out";
    case DGCL_EPLAN: return "planning failed (unreachable GPU)";
  }
  return "unknown status";
}

dgcl_status dgcl_destroy(dgcl_ctx *c) {
  if (!c) return DGCL_OK;
  if (has_device(c)) {
    cudaSetDevice(c->device);
    cudaDeviceSynchronize();
    for (char *p : c->ipc_opened) cudaIpcCloseMemHandle(p);
    cudaFree(c->d_groups);
    cudaFree(c->d_waits);
    cudaFree(c->d_idx);
    cudaFree(c->d_term_ptr);
    cudaFree(c->d_terms);
    cudaFree(c->d_items);
    cudaFree(c->d_runs);
    cudaFree(c->d_sterms);
    cudaFree(c->d_claims);
    for (Program &p : c->progs)
      if (p.d_trace) cudaFree(p.d_trace);
    for (auto &kv : c->stages) {
      if (kv.second.ptr) cudaFree(kv.second.ptr);
      if (kv.second.free) cudaEventDestroy(kv.second.free);
    }
    if (c->h2d_stream) cudaStreamDestroy(c->h2d_stream);
    if (c->d2h_stream) cudaStreamDestroy(c->d2h_stream);
    if (c->err_host) cudaFreeHost(c->err_host);
    for (cudaStream_t s : c->rank_streams)
      if (s) cudaStreamDestroy(s);
    for (cudaEvent_t e : c->rank_events)
      if (e) cudaEventDestroy(e);
    if (c->fork_event) cudaEventDestroy(c->fork_event);
    mc_teardown(c->device, c->mc_handle, c->mc_have_handle, c->mc_mem, c->mc_have_mem, c->mc_uc,
                c->mc_va, c->mc_map_bytes);
  }
  delete c;
  return DGCL_OK;
}

dgcl_status dgcl_debug_hostsim_forward(dgcl_ctx *c, int32_t layer, const float *emb, float *halo) {
  if (!c || !emb || !halo) return DGCL_EINVAL;
  if (!c->planned || !c->loopback) return fail(c, DGCL_ESTATE, "needs a planned loopback context");
  if (layer < 0 || layer >= c->n_layers) return DGCL_EINVAL;
  if (c->hostsim_items && c->lb_flags == DGCL_LOOPBACK_FUSED) {
    const Program &P = c->progs[c->prog_index(layer, DIR_FWD, 0)];
    if (!hostsim_run_items(c->low, P.items, P.runs, P.sterms, c->row_off, c->halo_off,
                           c->pitch[layer], c->dims[layer], emb, halo, nullptr, nullptr))
      return fail(c, DGCL_EPLAN, "malformed work item");
    return DGCL_OK;
  }
  hostsim_run(c->low, c->host_gids[DIR_FWD], c->row_off, c->halo_off, c->pitch[layer],
              c->dims[layer], emb, halo, nullptr, nullptr);
  return DGCL_OK;
}

dgcl_status dgcl_debug_hostsim_backward(dgcl_ctx *c, int32_t layer, const float *halo_grad,
                                        float *emb_grad) {
  if (!c || !halo_grad || !emb_grad) return DGCL_EINVAL;
  if (!c->planned || !c->loopback) return fail(c, DGCL_ESTATE, "needs a planned loopback context");
  if (layer < 0 || layer >= c->n_layers) return DGCL_EINVAL;
  if (c->hostsim_items && c->lb_flags == DGCL_LOOPBACK_FUSED) {
    const Program &P = c->progs[c->prog_index(layer, DIR_BWD, 0)];
    if (!hostsim_run_items(c->low, P.items, P.runs, P.sterms, c->row_off, c->halo_off,
                           c->pitch[layer], c->dims[layer], nullptr, nullptr, halo_grad, emb_grad))
      return fail(c, DGCL_EPLAN, "malformed work item");
    return DGCL_OK;
  }
  hostsim_run(c->low, c->host_gids[DIR_BWD], c->row_off, c->halo_off, c->pitch[layer],
              c->dims[layer], nullptr, nullptr, halo_grad, emb_grad);
  return DGCL_OK;
}

}  // extern "C"

// ---- verification aid: the flag protocol of one launch, checked on the host ----
// Runs the programs of (layer, direction) — the fused loopback program, or every virtual rank's
// program — as a scheduler would: each program's items in list order, an item only once every
// counter it waits on has reached its target, signals applied when the item ends.  Reports the
// first violation: a wait target that differs from the rows ever signalled on its counter, a
// deadlock (no program can advance), a source row read before it was written or by an item that
// does not wait on its writer's counter (a race on the GPU), a destination row written twice,
// or (forward) a halo row never written.  If every program completes here, the executor cannot
// deadlock either: a CTA takes its items in list order, so the item that ran first here among
// the unfinished ones has all its waits satisfied and nothing of its own CTA before it.
dgcl_status dgcl_debug_check_protocol(dgcl_ctx *c, int32_t layer, int32_t direction,
                                      int32_t mutate, char *msg, size_t msg_len) {
  if (!c || (direction != DIR_FWD && direction != DIR_BWD)) return DGCL_EINVAL;
  if (!c->planned) return fail(c, DGCL_ESTATE, "no plan");
  if (layer < 0 || layer >= c->n_layers) return fail(c, DGCL_EINVAL, "bad layer");
  if (!c->loopback) return fail(c, DGCL_EINVAL, "loopback contexts only (every rank's program)");
  const Lowered &L = c->low;
  const int m = c->world;
  char buf[512];
  auto bad = [&](const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    std::vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    if (msg && msg_len) std::snprintf(msg, msg_len, "%s", buf);
    return fail(c, DGCL_EPLAN, "%s", buf);
  };
  std::vector<Program> PP;
  for (int r = 0; r < c->n_prog_ranks; ++r) PP.push_back(c->progs[c->prog_index(layer, direction, r)]);
  // the checker's own negative tests: a deliberately broken copy of the programs
  if (mutate) {
    Program *pw = nullptr;
    size_t iw = 0;
    for (Program &p : PP)
      for (size_t i = 0; i < p.items.size() && !pw; ++i)
        if (p.items[i].wait_n > 0 && p.items[i].op != OP_WAIT) {
          pw = &p;
          iw = i;
        }
    if (!pw && mutate != 3) return fail(c, DGCL_EINVAL, "no waiting item to mutate");
    if (mutate == 1) {         // a stage-chained item that no longer waits (a race)
      pw->items[iw].wait_n = 0;
    } else if (mutate == 2) {  // the same item moved before its producers (a deadlock)
      const DevItem I = pw->items[iw];
      pw->items.erase(pw->items.begin() + iw);
      pw->items.insert(pw->items.begin(), I);
    } else if (mutate == 3) {  // a data item repeated (a row written twice)
      bool done = false;
      for (Program &p : PP)
        for (size_t i = 0; i < p.items.size() && !done; ++i)
          if (p.items[i].op == OP_COPY || p.items[i].op == OP_FANOUT || p.items[i].op == OP_FOLD) {
            p.items.push_back(p.items[i]);
            done = true;
          }
      if (!done) return fail(c, DGCL_EINVAL, "no data item to mutate");
    } else if (mutate == 4) {  // a producer of a waited counter that no longer signals
      const int32_t ctr = c->low.waits[pw->items[iw].wait_off].ctr;
      bool done = false;
      for (Program &p : PP)
        for (DevItem &I : p.items)
          if (!done && (I.flags & kItemSignal) && I.sig_ctr == ctr) {
            I.flags &= (uint8_t)~kItemSignal;
            done = true;
          }
    } else {
      return fail(c, DGCL_EINVAL, "mutate in 0..4");
    }
  }
  std::vector<const Program *> P;
  for (const Program &p : PP) P.push_back(&p);
  auto key = [](int rank, int64_t ctr) { return (uint64_t)rank * kCtrSpace + (uint64_t)ctr; };
  // rows of buffer (kind, rank) written in this launch: -2 not yet, -1 by an item that does not
  // signal, else the writer's counter index (on that rank)
  constexpr int32_t kUnwritten = -2, kNoSignal = -1;
  std::vector<std::vector<int32_t>> wr((size_t)K_NKINDS * m);
  auto rows_of = [&](int kind, int r) -> int64_t {
    switch (kind) {
      case K_HALO: return c->rel.n_halo[r];
      case K_RELAY: return L.n_relay[r];
      case K_SLOT: return L.n_slot[r];
      case K_MCUC: return L.mc_total;
      default: return 0;
    }
  };
  for (int k = 0; k < K_NKINDS; ++k)
    for (int r = 0; r < m; ++r) wr[(size_t)k * m + r].assign(rows_of(k, r), kUnwritten);
  auto tracked = [&](int kind) { return kind == K_HALO || kind == K_RELAY || kind == K_SLOT || kind == K_MCUC; };
  // every (receiver, counter, rows) signal of an item
  auto signals = [&](const DevItem &I, auto &&emit) {
    if (!(I.flags & kItemSignal) || I.sig_ctr < 0) return;
    if (I.op == OP_FANOUT) {
      int64_t cnt[kMaxRanks] = {0};
      for (int64_t t = I.t0; t + 1 < I.t0 + I.nterms; t += 2) ++cnt[L.terms[t] >> 28];
      for (int d = 0; d < m; ++d)
        if (cnt[d]) emit(d, (int64_t)I.sig_ctr, cnt[d]);
    } else if (I.dst_kind == K_MCAST) {
      for (int d = 0; d < m; ++d) emit(d, (int64_t)I.sig_ctr, (int64_t)I.rows);
    } else {
      emit((int)I.dst_rank, (int64_t)I.sig_ctr, (int64_t)I.rows);
    }
  };
  std::unordered_map<uint64_t, int64_t> total, val;
  for (const Program *p : P)
    for (const DevItem &I : p->items)
      signals(I, [&](int d, int64_t ctr, int64_t n) { total[key(d, ctr)] += n; });
  for (size_t pi = 0; pi < P.size(); ++pi)
    for (size_t i = 0; i < P[pi]->items.size(); ++i) {
      const DevItem &I = P[pi]->items[i];
      for (int w = I.wait_off; w < I.wait_off + I.wait_n; ++w) {
        const auto it = total.find(key(I.exec_rank, L.waits[w].ctr));
        const int64_t have = it == total.end() ? 0 : it->second;
        if (have != L.waits[w].amount)
          return bad("program %zu item %zu (group %d): waits for %lld rows on counter %d of rank %d, "
                     "%lld are ever signalled", pi, i, I.group, (long long)L.waits[w].amount,
                     L.waits[w].ctr, I.exec_rank, (long long)have);
      }
    }
  auto waits_ok = [&](const DevItem &I) {
    for (int w = I.wait_off; w < I.wait_off + I.wait_n; ++w) {
      const auto it = val.find(key(I.exec_rank, L.waits[w].ctr));
      if ((it == val.end() ? 0 : it->second) < L.waits[w].amount) return false;
    }
    return true;
  };
  auto waits_on = [&](const DevItem &I, int32_t ctr) {
    for (int w = I.wait_off; w < I.wait_off + I.wait_n; ++w)
      if (L.waits[w].ctr == ctr) return true;
    return false;
  };
  // one source row read / destination row written by item I
  auto read = [&](const DevItem &I, int kind, int r, int64_t row, size_t pi, size_t i) -> bool {
    if (!tracked(kind)) return true;
    auto &v = wr[(size_t)kind * m + r];
    if (row < 0 || row >= (int64_t)v.size()) {
      bad("program %zu item %zu (group %d): source row %lld of kind %d rank %d out of range", pi, i,
          I.group, (long long)row, kind, r);
      return false;
    }
    const int32_t w = v[row];
    if (w == kUnwritten || w == kNoSignal || r != I.exec_rank || !waits_on(I, w)) {
      bad("program %zu item %zu (group %d, stage %d): reads row %lld of kind %d rank %d %s", pi, i,
          I.group, L.groups[I.group].stage, (long long)row, kind, r,
          w == kUnwritten ? "before it is written"
          : w == kNoSignal ? "whose writer signals no counter"
                           : "without waiting on its writer's counter");
      return false;
    }
    return true;
  };
  auto write = [&](const DevItem &I, int kind, int r, int64_t row, int32_t ctr, size_t pi,
                   size_t i) -> bool {
    if (!tracked(kind)) return true;
    auto &v = wr[(size_t)kind * m + r];
    if (row < 0 || row >= (int64_t)v.size() || v[row] != kUnwritten) {
      bad("program %zu item %zu (group %d): destination row %lld of kind %d rank %d %s", pi, i,
          I.group, (long long)row, kind, r,
          row < 0 || row >= (int64_t)v.size() ? "out of range" : "written twice");
      return false;
    }
    v[row] = ctr;
    return true;
  };
  auto run = [&](const DevItem &I, const Program &p, size_t pi, size_t i) -> bool {
    const int32_t sctr = (I.flags & kItemSignal) ? I.sig_ctr : kNoSignal;
    if (I.op == OP_COPY) {
      for (int64_t q = I.tp; q < I.tp + I.nterms; ++q) {
        const DevRun &R = p.runs[q];
        for (int64_t j = 0; j < R.len; ++j) {
          if (!read(I, I.src_kind, I.exec_rank, R.src + j, pi, i)) return false;
          if (I.dst_kind == K_MCAST) {
            for (int d = 0; d < m; ++d)
              if (!write(I, K_MCUC, d, R.dst + j, sctr, pi, i)) return false;
          } else if (!write(I, I.dst_kind, I.dst_rank, R.dst + j, sctr, pi, i)) {
            return false;
          }
        }
      }
    } else if (I.op == OP_FANOUT) {
      for (int64_t t = I.t0; t + 1 < I.t0 + I.nterms; t += 2) {
        const uint32_t w = L.terms[t];
        if (!write(I, (w & kFanRelay) ? K_RELAY : K_HALO, (int)(w >> 28), (int64_t)(w & kFanRowMask),
                   sctr, pi, i))
          return false;
      }
    } else if (I.op == OP_FOLD) {  // (sources not traced: the parity tests cover the folds)
      for (int64_t j = 0; j < I.rows; ++j) {
        const int64_t row = I.dst >= 0 ? I.dst + j : (int64_t)L.idx[~I.dst + j];
        if (!write(I, I.dst_kind, I.dst_rank, row, sctr, pi, i)) return false;
      }
    }
    signals(I, [&](int d, int64_t ctr, int64_t n) { val[key(d, ctr)] += n; });
    return true;
  };
  std::vector<size_t> cur(P.size(), 0);
  size_t left = 0;
  for (const Program *p : P) left += p->items.size();
  while (left > 0) {
    bool progress = false;
    for (size_t pi = 0; pi < P.size(); ++pi) {
      const auto &items = P[pi]->items;
      while (cur[pi] < items.size() && waits_ok(items[cur[pi]])) {
        if (!run(items[cur[pi]], *P[pi], pi, cur[pi])) return DGCL_EPLAN;
        ++cur[pi];
        --left;
        progress = true;
      }
    }
    if (!progress) {
      for (size_t pi = 0; pi < P.size(); ++pi)
        if (cur[pi] < P[pi]->items.size()) {
          const DevItem &I = P[pi]->items[cur[pi]];
          return bad("deadlock: program %zu item %zu (group %d, stage %d) waits forever", pi,
                     cur[pi], I.group, L.groups[I.group].stage);
        }
    }
  }
  if (direction == DIR_FWD)
    for (int r = 0; r < m; ++r) {
      const auto &v = wr[(size_t)K_HALO * m + r];
      for (size_t row = 0; row < v.size(); ++row)
        if (v[row] == kUnwritten) return bad("halo row %zu of rank %d is never written", row, r);
    }
  if (msg && msg_len) std::snprintf(msg, msg_len, "ok: %zu programs, %zu counters", P.size(), total.size());
  return DGCL_OK;
}
