// internal.h — shared (host + device) definitions of libdgcl.
//
// The lowered plan is a list of GROUPS: one per send tuple (d_i, d_j, k, T^s_ij, T^r_ij) of §6.1
// (PAPER.md P:1401-1420), further split by the buffer kinds the rows come from / go to.  Groups
// are cut into fixed-size row ranges (ITEMS) which the persistent executor kernel walks in stage
// order.  Stage chaining uses monotonically increasing per-(direction, stage, source) row counters
// in the receiver's flag region — the "done" flags of §6.1 — and a per-source
// "ready" word, so no flag is ever reset and no host round-trip happens between stages.
#pragma once

#include <cstddef>
#include <cstdint>

namespace dgcl {

constexpr int kMaxRanks = 16;
constexpr int kMaxStages = 16;  // stage indices 1..15 (<= world-1)

// buffer kinds
enum Kind : int32_t {
  K_EMB = 0,    // user embeddings (local rows), read-only
  K_HALO = 1,   // per-layer halo (workspace), written by peers
  K_RELAY = 2,  // per-layer relay staging (workspace): rows a GPU forwards but did not request
  K_HGRAD = 3,  // user halo gradients, read-only
  K_SLOT = 4,   // backward gradient slots (workspace), written by tree children
  K_EGRAD = 5,  // user embedding gradients (in/out)
  K_MCAST = 6,  // multicast region through the NVSwitch multicast address (multimem stores)
  K_MCUC = 7,   // this GPU's own copy of the multicast region (unicast reads)
  K_NKINDS = 8
};

// source kinds a COPY item may gather with tile::gather4 (tensor map per kind, ExecParams::tmap)
constexpr int kG4Kinds = 4;
static_assert(K_EMB == 0 && K_HALO == 1 && K_RELAY == 2 && K_HGRAD == 3, "gather4 kinds");

enum Op : int32_t {
  OP_COPY = 0,   // dst[dst_row(i)] = src[src_row(i)]
  OP_FOLD = 1,   // dst[dst_row(i)] = fold(init ? dst : -, terms(i)) in order, fp32 adds
  OP_READY = 2,  // write ready[exec_rank] = seq into every peer's flag region
  OP_WAIT = 3,   // wait on the group's wait list (forward completion)
  OP_END = 4,    // (device only) end-of-stream marker from the producer warp to the consumers
  OP_FLUSH = 5,  // (device only) publish the done counts accumulated since the last flush
  OP_FANOUT = 6  // forward stage 1, per owner: read each embedding row once and store it into
                 // every requester's halo (or relay) row: dests(i) = terms[term_ptr[i]..)
};

// OP_FANOUT destinations (terms pool): word pairs (dest, source row); dest bits 31..28 = receiving
// rank, bit 27 = relay staging (else halo), bits 26..0 = row in that buffer
constexpr uint32_t kFanRelay = 1u << 27;
constexpr uint32_t kFanRowMask = (1u << 27) - 1;
// DevItem::ready_rank of an item that writes to several ranks (OP_FANOUT): wait for every peer
constexpr int8_t kReadyAll = -2;

enum Dir : int32_t { DIR_FWD = 0, DIR_BWD = 1 };

// flag region layout (uint64 words) at the start of every rank's workspace: done counters per
// (direction, stage, vertex block, source rank) — relay plans split their vertices into blocks
// so that stage k of block b waits only for stage k-1 of block b (stages overlap) — then the
// ready words
constexpr int kMaxBlocks = 8;
constexpr int64_t ctr_index(int dir, int stage, int src, int block = 0) {
  return (((int64_t)dir * kMaxStages + stage) * kMaxBlocks + block) * kMaxRanks + src;
}
constexpr int64_t kReadyBase = 2 * kMaxStages * kMaxBlocks * kMaxRanks;  // ready[src] words
constexpr int64_t kBarrierBase = kReadyBase + kMaxRanks;  // device start barrier: arrived[src]
constexpr int64_t kFlagWords = kBarrierBase + kMaxRanks;
// multicast done counters mc_done[owner] live in the multicast region's flag page, not in the
// flag region: counter indices kMcCtrBase + owner (DevGroup::sig_ctr, DevWait::ctr)
constexpr int64_t kMcCtrBase = kFlagWords;
constexpr int64_t kMcFlagBytes = 4096;  // flag page at the start of the multicast region
constexpr int64_t kCtrSpace = kFlagWords + kMaxRanks;  // counter indices of one rank
constexpr int64_t kFlagBytes = 40960;  // region reserved (>= kFlagWords * 8)
static_assert(kFlagWords * 8 <= kFlagBytes, "flag region");

// term encodings for OP_FOLD
//   kTermLocal:     bit 31 set => SLOT(exec) row, else HGRAD(exec) row
//   kTermRankHgrad: bits 31..28 = rank r, bits 27..0 = row of HGRAD(r)  (loopback direct reduce:
//                   every virtual rank's halo gradients live on the same device)
constexpr uint32_t kTermSlot = 0x80000000u;
constexpr int32_t kTermLocal = 0;
constexpr int32_t kTermRankHgrad = 1;
constexpr uint32_t kTermRowMask = 0x0FFFFFFFu;
//   kTermRankTree:  a postfix program: every term pushes an operand, then performs `adds` stack
//                   adds (pop two, push below + top); bits 31..28 = rank r, 27..24 = adds,
//                   23..0 = row of HGRAD(r).  The starting value (fold_init) is the stack
//                   bottom.  The loopback tree-order backward of relay plans: each owner row
//                   folds its whole tree in the reversed plan's order in one pass.
//                   Staged items keep the adds in the staged-term words (stage row | adds << 24)
constexpr int32_t kTermRankTree = 2;
constexpr uint32_t kTreeRowMask = 0x00FFFFFFu;
constexpr int kTreeAddShift = 24;
constexpr int kTreeMaxDepth = 8;  // register stack slots (bottom included); deeper trees: staged

struct DevGroup {
  int32_t op;
  int32_t dir;
  int32_t exec_rank;   // the GPU executing the group (all reads are local to it)
  int32_t dst_rank;    // the GPU whose buffer is written (a peer over NVLink, or itself)
  int32_t stage;       // forward stage k, or backward stage b (RED = K + 1)
  int32_t src_kind;    // OP_COPY source buffer kind
  int32_t dst_kind;
  int32_t fold_init;   // OP_FOLD: start from the destination row (RED)
  int32_t sig_ctr;     // counter index (ctr_index) on dst_rank to add n_rows to, or -1
  int32_t ready_rank;  // wait ready[ready_rank] >= seq before writing (-1: none)
  int32_t wait_off;    // waits[wait_off .. wait_off + wait_n) on exec_rank's counters
  int32_t wait_n;
  int32_t term_mode;   // OP_FOLD terms: kTermLocal (SLOT/HGRAD of exec) or kTermRankHgrad
  int32_t atomic_add;  // OP_COPY: add the rows into the destination with atomics (ablation)
  int32_t block;       // vertex block (relay plans: stage chaining per block), 0..n_blocks-1
  int32_t pad3;
  int64_t n_rows;
  int64_t src_idx;     // offset into idx pool, or -1 => rows src_base + i
  int64_t src_base;
  int64_t dst_idx;     // offset into idx pool, or -1 => rows dst_base + i
  int64_t dst_base;
  int64_t term_ptr;    // OP_FOLD: offset into term_ptr pool (n_rows + 1 entries)
};

// One work item = a row range of one group, self-contained (64 B, one descriptor load): the
// executor never dereferences the group table on the hot path.
struct alignas(16) DevItem {
  uint8_t op, dir, exec_rank, dst_rank;
  uint8_t src_kind, dst_kind, fold_init, term_mode;
  int8_t ready_rank;   // wait ready[ready_rank] >= seq before writing (-1: none)
  uint8_t flags;       // kItemSignal: add `rows` to the receiver's counter sig_ctr afterwards
  int16_t wait_n;      // waits[wait_off .. +wait_n) on exec_rank's counters (source readiness)
  int32_t rows;
  int32_t sig_ctr;
  int32_t wait_off;
  int64_t src;         // >= 0: first source row (rows are consecutive); < 0: ~(idx pool offset)
  int64_t dst;         // same encoding for the destination rows
  int64_t tp;          // OP_FOLD: term_ptr pool index of the first row (rows + 1 entries)
                       // OP_COPY: index of the item's first DevRun in the run pool
  int64_t t0;          // OP_FOLD: term_ptr[tp] (index of the first term)
  int32_t nterms;      // OP_FOLD: terms of the item; OP_COPY: runs of the item
  int32_t group;       // originating group (diagnostics / watchdog codes)
};
static_assert(sizeof(DevItem) == 64, "DevItem is one 64-B descriptor");
constexpr uint8_t kItemSignal = 1;
constexpr uint8_t kItemDirect = 2;  // COPY: consumers gather rows themselves (short row runs)
constexpr uint8_t kItemGather4 = 4; // COPY with short source runs (kind < kG4Kinds): TMA gather4
// FOLD whose operand rows are all bulk-copied into the stage (bulk-copy executor only; the
// register executor ignores the flag): src = (segments << 40) | first segment in the run pool,
// t0 = first staged term (shared-memory row of each term, per-program pool `sterms`)
constexpr uint8_t kItemStaged = 8;
// COPY whose rows are ADDED into the destination with atomic reductions (the paper's atomic
// backward baseline, Table 9; ablation only: the order of the adds is not fixed)
constexpr uint8_t kItemAtomic = 16;
// COPY with short source runs (option "lsu_gather", bulk-copy executor): the consumer threads
// gather the rows into the stage with 16-B cp.async (LDGSTS, many in flight, no per-instruction
// issue loop on the producer), then the stage is stored as usual (TMA bulk stores); the
// producer stages only the source-row window, after the rows
constexpr uint8_t kItemLsu = 32;
constexpr int kSegShift = 40;
constexpr int kGather4MaxRowBytes = 1024;  // one tensor box (<= 256 fp32) per row

struct DevWait {
  int32_t ctr;         // counter index on the executing rank
  int32_t pad;
  int64_t amount;      // rows per call; target = epoch[dir] * amount
};

struct BufRef {
  char *ptr;
  int64_t pitch;       // bytes
};

struct alignas(64) ExecParams {
  // 2-D tensor maps (CUtensorMap, 128 B) over the packed rows of the source buffers of this
  // launch — embeddings, halos, relay staging, halo gradients (index = buffer kind) — for the
  // row-gather TMA (cp.async.bulk.tensor ... tile::gather4: four arbitrary rows per instruction)
  alignas(64) unsigned char tmap[kG4Kinds][128];
  int32_t gather4_mask;                       // bit k: tmap[k] valid for this launch
  int32_t tmap_row_off[kG4Kinds][kMaxRanks];  // first tensor row of each rank's rows of kind k
  BufRef buf[K_NKINDS][kMaxRanks];
  uint64_t *flags[kMaxRanks];  // flag region of every rank (peer-mapped in multi-GPU mode)
  const DevGroup *groups;
  const DevItem *items;
  const DevWait *waits;
  const int32_t *idx;
  const int64_t *term_ptr;
  const uint32_t *terms;
  int32_t n_items;
  int32_t world;
  int32_t row_bytes;   // dims[layer] * 4: bytes moved per row
  int32_t n_chunks;    // 16-byte chunks per row (vector path) or 4-byte words (scalar path)
  uint32_t div_mul;    // fast division by n_chunks: q = (umulhi(x, mul) + x) >> shift
  int32_t div_shift;
  int32_t vec16;       // 1: 16-byte path (all bases and pitches 16-B aligned)
  int32_t use_ready;   // per-rank programs: honour ready words before writing to a peer
  uint64_t epoch[2];   // completed+current calls per direction (counter targets)
  uint64_t seq;        // global call sequence number (ready words)
  uint64_t timeout_ns;
  int *err;            // host-mapped error word (0 = ok)
  int32_t use_tma;     // 1: bulk-copy (TMA) gather into shared memory, then store from smem
  int32_t row16;       // row bytes rounded up to 16 (bulk-copy size per row)
  int32_t tma_buf;     // bytes per shared-memory stage buffer (launch geometry, TmaGeometry)
  int32_t tma_stages;  // stage buffers per CTA (<= kMaxTmaStages)
  int32_t meta_bytes;  // bytes per producer metadata slot
  int32_t bulk_store;  // 1: contiguous COPY destinations are written with bulk (TMA) stores
  const struct DevRun *runs;  // COPY items: maximal runs of consecutive (source, destination) rows
  int32_t op_mask;     // kinds of data items in this launch (kMaskCopy | kMaskFold | kMaskDirect |
                       // kMaskStaged):
                       // selects a kernel instance that carries only the code it needs
  int32_t fold_wide;   // FOLD rows average >= 4 terms (selects the 1024-thread fold instance)
  const uint32_t *sterms;  // staged FOLD items: operand row (in the stage) of every term
  struct TraceRec *trace;  // option "trace": one record per item of this launch, or nullptr
  int32_t l2_policy;       // option "l2_policy": L2 eviction hints of the bulk-copy executor
  int32_t sys_scope;       // 1: flags / fences at system scope (peers are other GPUs); 0: .gpu
  // bulk-copy executor, dynamic item claiming (option "claim_batch"): a launch-wide counter
  // (nullptr = round-robin).  Every CTA claims batches of claim_batch list positions until a
  // claim fails, so a launch adds exactly claim_batch * (ceil(n_items / claim_batch) + grid) to
  // the counter; claim_base = its value at launch (kept by the host, never reset)
  uint64_t *claim;
  uint64_t claim_base;
  int32_t claim_batch;
  // multicast (option "multicast"): the multicast flag page (multimem reductions), every rank's
  // unicast flag page (acquire waits; loopback: each virtual rank's copy), and whether the
  // multicast is emulated by one store / reduction per rank (loopback: no multicast object)
  uint64_t *mc_flags;
  uint64_t *mcuc_flags[kMaxRanks];
  int32_t mc_emulate;
  // 1: a simple copy launch (COPY items only: no waits, no signals, every item's runs or row
  // window within half a metadata slot, round-robin, copy-only instance) runs two producer warps
  // (gather4 items are issued by their own producer, without the helper hand-over)
  int32_t dual_prod;
};

// Per-item timeline (%globaltimer ns), written when tracing is on: the executor reached the item,
// its source waits were satisfied (stage chaining), its rows were stored; and what it was.
struct TraceRec {
  uint64_t t_start, t_ready, t_done;
  uint32_t sm, tag;  /* op | dir << 4 | exec << 8 | dst << 16 | stage << 24 | block << 29 */
};
static_assert(sizeof(TraceRec) == 32, "trace record");
#ifdef __CUDACC__
#define DGCL_HD __host__ __device__
#else
#define DGCL_HD
#endif
DGCL_HD inline uint32_t trace_tag(const DevItem &I, int stage, int block) {
  return (uint32_t)I.op | (uint32_t)I.dir << 4 | (uint32_t)I.exec_rank << 8 |
         (uint32_t)I.dst_rank << 16 | (uint32_t)(stage & 31) << 24 | (uint32_t)(block & 7) << 29;
}
constexpr int32_t kMaskCopy = 1, kMaskFold = 2, kMaskDirect = 4, kMaskStaged = 8, kMaskFanout = 16,
                  kMaskTree = 32,  // unstaged tree-order FOLD items (their own instance)
                  kMaskLsu = 64,   // COPY items gathered by consumer cp.async (option lsu_gather;
                                   // only the catch-all instance carries that code)
                  kMaskMcast = 128;  // COPY items into the multicast region (likewise)

// A run of `len` rows whose source rows src.. and destination rows dst.. are both consecutive;
// `pos` is the first row's index inside its item.  One bulk copy moves a run when the pitches
// equal the 16-B-rounded row.  For a staged FOLD item the run is a SEGMENT: `len` consecutive
// rows src.. of buffer (kind = dst >> 8, rank = dst & 255) copied to operand rows pos.. .
struct DevRun {
  int32_t src, dst, len, pos;
};

// Bulk-copy executor (executor_tma.cu) shared-memory geometry and the item limits it implies.
// Dynamic shared memory of a CTA:
//   [0,256) mbarriers | meta slots (4 x meta_bytes, producer-private row runs / segments) |
//   descriptor ring (8 x 64 B) | stages (stages x stage_bytes) | 1152 B done counts + barrier
// and one stage = [0,64) item header | [64,128) info | [128,2176) term_ptr window (FOLD) |
//   [2176,4096) destination-row window | [4096, stage_bytes) operand rows + staged terms.
// Two geometries, chosen per launch (per program) by the host:
//   WIDE: 1 CTA per SM, 4 x 48 KB stages — large items; best for long row runs of big rows
//         (write-dominated forward of Reddit-shaped rows: 0.94 vs 0.75 of HBM peak)
//   DUAL: 2 CTAs per SM, 2 x 47 KB stages — two producer warps per SM; best when the producer's
//         per-item work dominates (short runs, staged folds: backward 0.70 -> 0.95-1.0 of peak)
// (measured on the Reddit / Web-Google / Com-Orkut loopbacks)
struct TmaGeometry {
  int32_t stages, stage_bytes, meta_bytes, threads, ctas_per_sm, max_item_rows;
};
#ifndef DGCL_WIDE_STAGES  // (build-time A/B of the WIDE geometry; 3 x 64 KB until the dual
#define DGCL_WIDE_STAGES 4  //  producers: 4 x 48 KB then won, Reddit fwd602 0.696 -> 0.685, r2tf)
#define DGCL_WIDE_STAGE_KB 48
#endif
constexpr TmaGeometry kGeoWide = {DGCL_WIDE_STAGES, DGCL_WIDE_STAGE_KB * 1024, 8 * 1024, 256, 1, 464};
// WIDE with 3 x 64 KB stages for launches that keep one producer (waits / signals: relay and
// per-rank programs) — larger items, less producer work per byte (per-rank Reddit fwd602: 4 x 48
// KB 1.13 ms vs 3 x 64 KB 0.82)
constexpr TmaGeometry kGeoWide3 = {3, 64 * 1024, 8 * 1024, 256, 1, 464};
#ifndef DGCL_DUAL_STAGES  // (build-time A/B of the DUAL geometry, tools/build_variant.sh)
#define DGCL_DUAL_STAGES 2
#define DGCL_DUAL_STAGE_KB 47
#define DGCL_DUAL_CTAS 2
#define DGCL_DUAL_META_KB 4
#endif
constexpr TmaGeometry kGeoDual = {DGCL_DUAL_STAGES, DGCL_DUAL_STAGE_KB * 1024,
                                  DGCL_DUAL_META_KB * 1024, 256, DGCL_DUAL_CTAS,
                                  DGCL_DUAL_META_KB * 1024 / 16 < 240 ? DGCL_DUAL_META_KB * 1024 / 16
                                                                       : 240};
constexpr int kMaxTmaStages = 4;
constexpr int kStageHdrBytes = 4096;
constexpr int kTmaBufBytes = kGeoWide3.stage_bytes;         // largest stage
constexpr int kTmaOperandBytes = kTmaBufBytes - kStageHdrBytes;
constexpr size_t tma_smem_bytes(const TmaGeometry &g) {
  return 256 + 4 * (size_t)g.meta_bytes + 8 * 64 + (size_t)g.stages * g.stage_bytes + 1152;
}
static_assert(tma_smem_bytes(kGeoWide) <= 227 * 1024, "WIDE: one CTA per SM");
static_assert(tma_smem_bytes(kGeoWide3) <= 227 * 1024, "WIDE3: one CTA per SM");
static_assert(kGeoWide.stage_bytes <= kGeoWide3.stage_bytes && kGeoDual.stage_bytes <= kGeoWide3.stage_bytes,
              "kTmaBufBytes is the largest stage");
// launch geometry by index: 0 WIDE (4 x 48 KB, dual-producer launches), 1 DUAL, 2 WIDE3
inline const TmaGeometry &geometry_of(int g) { return g == 1 ? kGeoDual : g == 2 ? kGeoWide3 : kGeoWide; }
static_assert(tma_smem_bytes(kGeoDual) * DGCL_DUAL_CTAS <= 227 * 1024, "DUAL: CTAs per SM");
static_assert(kGeoWide.max_item_rows * 16 <= kGeoWide.meta_bytes &&
                  kGeoDual.max_item_rows * 16 <= kGeoDual.meta_bytes,
              "a meta slot holds an item's 16-B runs");
constexpr int kMaxItemRows = 464;        // <= (1920 B dst window) / 4 B - slack
constexpr int kMaxFoldRows = 240;        // (2048 B term_ptr window) / 8 B - slack
constexpr int kMaxItemTerms = 2040;      // (8 KB terms window) / 4 B - slack

// fast unsigned division by a runtime constant d >= 1, exact for x < 2^31
struct FastDiv {
  uint32_t mul;
  int32_t shift;
};
inline FastDiv make_fastdiv(uint32_t d) {
  int l = 0;
  while ((1ull << l) < d) ++l;  // l = ceil(log2 d)
  FastDiv f;
  f.shift = l;
  f.mul = (uint32_t)(((1ull << 32) * ((1ull << l) - d)) / d + 1);
  return f;
}
inline uint32_t fastdiv_host(uint32_t x, FastDiv f) {
  uint32_t hi = (uint32_t)(((uint64_t)x * f.mul) >> 32);
  return (uint32_t)(((uint64_t)hi + x) >> f.shift);
}

// launch wrapper implemented in executor.cu; returns a cudaError_t value
int launch_executor(const ExecParams &p, int grid, int block, void *stream);
int executor_occupancy(int block, int *ctas_per_sm);                          // register path
// device start barrier: ranks first .. first+count-1 of this process (threads of one warp) each
// release arrived[rank] = p.seq into every peer's flag region, then acquire-wait on every peer's
int launch_barrier(const ExecParams &p, int first, int count, void *stream);
// arrival wait (overlap): one thread acquire-waits on rank `exec`'s counters
// p.waits[off .. off + n) >= p.epoch[DIR_FWD] * amount, then the kernel ends
int launch_wait(const ExecParams &p, int exec, int off, int n, void *stream);
// multicast self-test kernel (dgcl_debug_multicast_selftest): multimem stores + one reduction
int launch_mc_selftest(void *mc, uint64_t *mcflag, int n16, void *stream);
// bulk-copy path: the instance for op_mask (< 0: the worst case over instances)
int executor_tma_occupancy(int op_mask, int block, size_t smem_bytes, int *ctas_per_sm);

}  // namespace dgcl
