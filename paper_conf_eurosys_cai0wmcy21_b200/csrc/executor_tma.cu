// executor_tma.cu — the bulk-copy (TMA) plan executor, warp-specialised (sm_100a).
//
// Same semantics as executor.cu (items / counters, see internal.h), different data movement.
// PAPER.md §6.1-6.2: the sender packs rows by its send table and writes them into
// the receiver's buffer.  Here the "pack" is a gather of whole rows into shared memory by the
// Tensor Memory Accelerator (one cp.async.bulk per run of consecutive rows, or tile::gather4 for
// four scattered rows), and the "send" is a bulk (TMA) store or a coalesced 16-B store stream from
// shared memory to the destination rows (a peer's halo over NVLink 5, or local HBM).
//
// Per CTA (WIDE: one per SM, 4 x 48 KB stages; DUAL: two per SM, 2 x 47 KB; descriptor ring, run windows):
//   warp 0 (producer) walks the CTA's items in order with a metadata pipeline — descriptors
//     bulk-copied 6 items ahead, row runs / source rows 3 items ahead — so no dependent global
//     load is on its critical path.  Per data item it resolves the source waits (stage chaining)
//     and the destination's ready word, claims a stage, writes the item header, arms the stage's
//     "full" mbarrier with the byte count and issues the row gathers plus the consumers' tables;
//     before it could block on a wait it inserts a FLUSH marker so pending done counts go out;
//   (launches without waits or signals: warps 0 and 1 are two producers splitting the items —
//    ExecParams::dual_prod; copy launches otherwise use warp 1 as a gather4 helper)
//   the other warps (consumers) take stages in order: store (COPY) or fold-and-store (FOLD), count the
//     item's rows in shared memory (published at FLUSH / END: fence.sys, then one
//     red.release.sys per (source, receiver)) and release the stage.  An END header stops them.
// Up to ~180 KB of gathers are in flight per SM, hiding HBM / NVLink latency without registers.

#include "device_common.cuh"

namespace dgcl {

using namespace dev;

namespace {

#ifndef DGCL_HELPER
#define DGCL_HELPER 1  // copy launches: this many helper warps issue a share of each item's gathers
#endif
// diagnostic builds (tools/build_variant.sh): DGCL_DIAG_NO_GATHER — COPY items store whatever the
// stage holds (no row gathers); DGCL_DIAG_NO_STORE — COPY items gather but store nothing
#ifndef DGCL_DIAG_NO_GATHER
#define DGCL_DIAG_NO_GATHER 0
#endif
#ifndef DGCL_DIAG_NO_STORE
#define DGCL_DIAG_NO_STORE 0
#endif
#ifndef DGCL_FAN_BULK_ROW
#define DGCL_FAN_BULK_ROW 1024
#endif
#ifndef DGCL_STORE_SPLIT
#define DGCL_STORE_SPLIT 4  // bulk stores per COPY stage (A/B r2sg/r2sh; 15 rotating before)
#endif
// DGCL_STORE_FIXED 1: the same consumer warps store every stage, so each of them has one bulk
// store in flight and a CTA writes at most kStoreSplit runs at a time; HBM writes fewer, longer
// runs (tools/store_bench.cu: one 60-KB store stream per SM 7.06 TB/s, 15 concurrent 4-KB pieces
// 6.26 TB/s); 0: warps rotate per stage
#ifndef DGCL_ROW_BULK
#define DGCL_ROW_BULK 1024  // > 0: COPY rows of >= this many bytes to scattered destinations
                            // (relay stages) go out as one bulk store per row; 0: consumer STG
                            // (A/B r2so: relay forwards 1-1.5 % faster)
#endif
#ifndef DGCL_STG_SHARE
#define DGCL_STG_SHARE 0  // percent of a bulk-store COPY stage stored with STG instead (A/B)
#endif
#ifndef DGCL_STORE_FIXED
#define DGCL_STORE_FIXED 1
#endif
constexpr int kStoreSplit = DGCL_STORE_SPLIT;  // bulk stores per COPY item (<= consumer warps)
constexpr int kFanBulkRowBytes = DGCL_FAN_BULK_ROW;  // fan-out rows stored by bulk stores
constexpr int kMetaSlots = 4;         // run windows prefetched kMetaAhead items ahead
constexpr int kMetaAhead = 3;
constexpr int kDescAhead = 6;         // descriptors prefetched further ahead (ring of kDescSlots)
constexpr int kHdrInfo = 64;         // stage: int32 info words after the 64-B item header
constexpr int kTabTp = 128;          // stage: term_ptr window (FOLD)
constexpr int kTabDst = 2176;        // stage: destination-row window
constexpr int kDescSlots = 8;        // producer descriptor ring
static_assert(kDescAhead > kMetaAhead && kDescAhead < kDescSlots && kMetaAhead < kMetaSlots,
              "prefetch distances");
// shared-memory carve-up (internal.h, tma_smem_bytes): offsets depend on the launch geometry
constexpr size_t kMetaOff = 256;     // after the mbarriers (full, empty, meta, desc)
// dual-producer mode (ExecParams::dual_prod): 2 producer warps, each with half of the descriptor
// ring and the metadata region cut into kDualMetaSlots half-size slots per producer
constexpr int kDualMetaSlots = 4;
constexpr int kDualDescAhead = 3, kDualMetaAhead = 2;  // (a descriptor lands before its runs are asked for)
constexpr int kMetaBarriers = 2 * kDualMetaSlots;  // (single mode uses the first kMetaSlots)
static_assert((2 * kMaxTmaStages + kMetaBarriers + kDescSlots) * 8 <= 256, "mbarrier region");
static_assert(kDescSlots == 2 * 4 && kDualDescAhead < 4 && kDualMetaAhead < kDualMetaSlots,
              "dual-producer rings");
static_assert(kMetaSlots * 8 * 64 <= 4 * 8 * 1024 && kDescSlots == 8, "layout of tma_smem_bytes");
constexpr size_t kSmemMax = tma_smem_bytes(kGeoWide) > tma_smem_bytes(kGeoWide3)
                                ? tma_smem_bytes(kGeoWide) : tma_smem_bytes(kGeoWide3);

// k-th stage use of a ring of ns (2, 3 or 4) stages: slot and use count without a division
__device__ __forceinline__ void ring_pos(uint32_t k, uint32_t ns, uint32_t &slot, uint32_t &use) {
  use = ns == 2 ? (k >> 1) : ns == 4 ? (k >> 2) : (__umulhi(k, 0xAAAAAAABu) >> 1);
  slot = k - use * ns;
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ bool mbar_test(uint64_t *b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      " selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(smem_u32(b)), "r"(parity)
      : "memory");
  return ok != 0;
}
#ifndef DGCL_WAIT_HINT
#define DGCL_WAIT_HINT 0  // ns: try_wait suspend-time hint of the spin waits (0: none)
#endif
#ifndef DGCL_WAIT_SLEEP
#define DGCL_WAIT_SLEEP 0  // ns: nanosleep between failed try_waits (0: none)
#endif
__device__ __forceinline__ bool mbar_test_hint(uint64_t *b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n"
      " selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(smem_u32(b)), "r"(parity), "r"((uint32_t)DGCL_WAIT_HINT)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  if (DGCL_WAIT_HINT) {
    while (!mbar_test_hint(b, parity)) {
    }
    return;
  }
  while (!mbar_test(b, parity)) {
    if (DGCL_WAIT_SLEEP) __nanosleep(DGCL_WAIT_SLEEP);
  }
}
__device__ __forceinline__ void bulk_g2s(void *sdst, const void *gsrc, uint32_t bytes,
                                         uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
          "r"(smem_u32(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
// L2 eviction priority hints (option "l2_policy", ExecParams::l2_policy): a 64-bit cache policy
// made once per thread by createpolicy, attached to the data bulk copies / stores
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void bulk_g2s_h(void *sdst, const void *gsrc, uint32_t bytes,
                                           uint64_t *bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1], %2, [%3], %4;" ::"r"(smem_u32(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void bulk_s2g_h(void *gdst, const void *ssrc, uint32_t bytes,
                                           uint64_t pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(
                   gdst),
               "r"(smem_u32(ssrc)), "r"(bytes), "l"(pol)
               : "memory");
}
// data movement with an optional policy (pol == 0: no hint)
__device__ __forceinline__ void g2s(void *sdst, const void *gsrc, uint32_t bytes, uint64_t *bar,
                                    uint64_t pol);
__device__ __forceinline__ void bulk_s2g(void *gdst, const void *ssrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst),
               "r"(smem_u32(ssrc)), "r"(bytes)
               : "memory");
}
// TMA bulk reduction: dst[i] += src[i] (fp32, element-wise atomic in L2) for `bytes` (16-B multiple)
__device__ __forceinline__ void bulk_s2g_add_f32(void *gdst, const void *ssrc, uint32_t bytes) {
  asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(
                   gdst),
               "r"(smem_u32(ssrc)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void g2s(void *sdst, const void *gsrc, uint32_t bytes, uint64_t *bar,
                                    uint64_t pol) {
  if (pol)
    bulk_g2s_h(sdst, gsrc, bytes, bar, pol);
  else
    bulk_g2s(sdst, gsrc, bytes, bar);
}
__device__ __forceinline__ void s2g(void *gdst, const void *ssrc, uint32_t bytes, uint64_t pol) {
  if (pol)
    bulk_s2g_h(gdst, ssrc, bytes, pol);
  else
    bulk_s2g(gdst, ssrc, bytes);
}
__device__ __forceinline__ void bulk_commit() {
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_all() {
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
// generic-proxy accesses (acquired flags, smem reads) before async-proxy bulk copies
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}
__device__ __forceinline__ int4 lds_v4(const uint8_t *p) {
  return *reinterpret_cast<const int4 *>(p);
}

// Barrier over the consumer warps only (the producer never joins): lane 0 of each warp arrives,
// the last one advances the generation.
__device__ __forceinline__ void consumer_barrier(unsigned *count, volatile unsigned *gen,
                                                 unsigned nwarps, int lane) {
  __syncwarp();
  if (lane == 0) {
    const unsigned g = *gen;
    __threadfence_block();
    if (atomicAdd(count, 1u) == nwarps - 1) {
      *count = 0;
      __threadfence_block();
      atomicAdd((unsigned *)gen, 1u);
    } else {
      while (*gen == g) {
      }
    }
    __threadfence_block();
  }
  __syncwarp();
}

// non-blocking: are all counter waits of I already satisfied?
__device__ __forceinline__ bool waits_ready(const ExecParams &P, const DevItem &I) {
  for (int w = 0; w < I.wait_n; ++w) {
    const DevWait W = P.waits[I.wait_off + w];
    if (ld_acquire(ctr_ptr(P, I.exec_rank, W.ctr), P.sys_scope) <
        P.epoch[I.dir] * (uint64_t)W.amount)
      return false;
  }
  return true;
}

// 16-B aligned window [a, e) of `n` elements of size `sz` starting at element `off`
struct Win {
  int64_t a;       // first element copied (aligned down)
  uint32_t bytes;  // multiple of 16
  int32_t skew;    // off - a
};
__device__ __forceinline__ Win window(int64_t off, int64_t n, int sz) {
  const int64_t per = 16 / sz;
  Win w;
  w.a = off / per * per;
  const int64_t e = (off + n + per - 1) / per * per;
  w.bytes = (uint32_t)((e - w.a) * sz);
  w.skew = (int32_t)(off - w.a);
  return w;
}

// named barriers between the producer warp and its helper (ids 1 and 2; __syncthreads is 0)
__device__ __forceinline__ void named_arrive(int id, int n) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ void named_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}

// COPY item gathered four rows per TMA instruction (tile::gather4 through the launch's tensor map)
__device__ __forceinline__ bool uses_gather4(const ExecParams &P, const DevItem &I) {
  return (I.flags & kItemGather4) && I.op == OP_COPY && I.src < 0 && I.src_kind < kG4Kinds &&
         ((P.gather4_mask >> I.src_kind) & 1);
}

__device__ __forceinline__ void tma_gather4(void *sdst, const void *tmap, int32_t col, int32_t r0,
                                            int32_t r1, int32_t r2, int32_t r3, uint64_t *bar,
                                            uint64_t pol = 0) {
  if (pol) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
        ".L2::cache_hint [%0], [%1, {%2, %3, %4, %5, %6}], [%7], %8;" ::"r"(smem_u32(sdst)),
        "l"(tmap), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
    return;
  }
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(smem_u32(sdst)),
      "l"(tmap), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(smem_u32(bar))
      : "memory");
}

// staged FOLD item: operand rows bulk-copied into the stage (destination rows first when the
// fold starts from them, then one row per term), followed by the staged-term window
__device__ __forceinline__ bool is_staged(const DevItem &I) {
  return I.op == OP_FOLD && (I.flags & kItemStaged);
}
__device__ __forceinline__ uint32_t staged_rows(const DevItem &I) {
  return (I.fold_init ? (uint32_t)I.rows : 0u) + (uint32_t)I.nterms;
}
__device__ __forceinline__ uint32_t n_segments(const DevItem &I) {
  return (uint32_t)(I.src >> kSegShift);
}

// producer lane 0: bulk-copy the metadata the producer needs to issue item I's gathers (the
// caller has fenced generic accesses to the slot against the async proxy)
template <bool kLsu>
__device__ __forceinline__ void issue_meta(const ExecParams &P, const DevItem &I, uint8_t *meta,
                                           uint64_t *bar) {
  // COPY (bulk path): the item's row runs, or its source rows for a gather4 item.  FOLD and
  // direct COPY items need nothing here (the consumers gather their operands); the barrier phase
  // then completes on the arrive alone.
  if (uses_gather4(P, I)) {
    const Win ws = window(~I.src, I.rows, 4);
    mbar_expect_tx(bar, ws.bytes);
    bulk_g2s(meta, P.idx + ws.a, ws.bytes, bar);
    return;
  }
  if (is_staged(I)) {  // the item's segments
    const uint32_t tx = n_segments(I) * (uint32_t)sizeof(DevRun);
    mbar_expect_tx(bar, tx);
    bulk_g2s(meta, P.runs + (I.src & ((1ll << kSegShift) - 1)), tx, bar);
    return;
  }
  const uint32_t tx = (I.op == OP_COPY && !(I.flags & (kItemDirect | (kLsu ? kItemLsu : 0))))
                          ? (uint32_t)I.nterms * (uint32_t)sizeof(DevRun)
                          : 0u;
  mbar_expect_tx(bar, tx);
  if (tx) bulk_g2s(meta, P.runs + I.tp, tx, bar);
}

// bytes bulk-copied into the operand area of a stage (gathered rows, or a FOLD's terms window)
template <bool kLsu>
__device__ __forceinline__ uint32_t operand_bytes(const ExecParams &P, const DevItem &I) {
  if (I.op == OP_COPY) {
    if (uses_gather4(P, I)) return (uint32_t)((I.rows + 3) / 4 * 4) * (uint32_t)P.row16;
    if (kLsu && (I.flags & kItemLsu)) return I.src < 0 ? window(~I.src, I.rows, 4).bytes : 0u;
    if (!(I.flags & kItemDirect)) return (uint32_t)I.rows * (uint32_t)P.row16;
    return I.src < 0 ? window(~I.src, I.rows, 4).bytes : 0u;  // source-row window only
  }
  if (is_staged(I)) return staged_rows(I) * (uint32_t)P.row16 + window(I.t0, I.nterms, 4).bytes;
  if (I.op == OP_FANOUT) return (uint32_t)I.rows * (uint32_t)P.row16 + window(I.t0, I.nterms, 4).bytes;
  return window(I.t0, I.nterms, 4).bytes;
}

// gathers [gb, ge) of a gather4 COPY item, one per lane and round (row indices from its meta slot)
__device__ __forceinline__ void issue_gather4(const ExecParams &P, const DevItem &I, uint8_t *st,
                                              const uint8_t *meta, uint64_t *full, int lane, int gb,
                                              int ge, uint64_t pol) {
  const uint32_t r16 = (uint32_t)P.row16;
  uint8_t *ops = st + kStageHdrBytes;
  const int32_t *sidx = reinterpret_cast<const int32_t *>(meta) +
                        (int32_t)(~I.src - window(~I.src, I.rows, 4).a);
  const int32_t base = P.tmap_row_off[I.src_kind][I.exec_rank];
  const void *tmap = P.tmap[I.src_kind];
  for (int g = gb + lane; g < ge; g += 32) {
    const int r = 4 * g, last = I.rows - 1;
    tma_gather4(ops + (size_t)r * r16, tmap, 0, base + sidx[r], base + sidx[min(r + 1, last)],
                base + sidx[min(r + 2, last)], base + sidx[min(r + 3, last)], full, pol);
  }
}

// producer warp: header, consumer tables and row gathers of data item I (in registers; Ism = its
// descriptor in shared memory, copied as the stage header) into `st`.  The caller waited for the
// stage to be free and fenced the consumers' generic reads of it against the async proxy.
// With kHelp, gather4 items are handed to the helper warp through the mailbox mb (stage and
// meta-slot offsets) after the stage's transaction bytes are armed; the two warps then each issue
// half of the gathers.
template <bool kLsu, bool kHelp>
__device__ __forceinline__ void issue_item(const ExecParams &P, const DevItem &I,
                                           const DevItem *Ism, uint8_t *st, const uint8_t *meta,
                                           uint64_t *full, int lane, uint32_t item_index,
                                           uint64_t pol_copy, uint64_t pol_fold, uint32_t *mb,
                                           bool *mb_busy, const uint8_t *stages_base,
                                           const uint8_t *metas_base) {
  const uint32_t r16 = (uint32_t)P.row16;
  // consumer tables: term_ptr window (FOLD) and destination rows (when not consecutive)
  Win wtp = {0, 0, 0}, wdst = {0, 0, 0};
  if (I.op == OP_FOLD) wtp = window(I.tp, I.rows + 1, 8);
  if (I.dst < 0) wdst = window(~I.dst, I.rows, 4);
  if (lane < 4) reinterpret_cast<int4 *>(st)[lane] = reinterpret_cast<const int4 *>(Ism)[lane];
  if (lane == 4) {
    int32_t *info = reinterpret_cast<int32_t *>(st + kHdrInfo);
    info[0] = wtp.skew;
    info[1] = wdst.skew;
    info[2] = (int32_t)item_index;  // (trace records)
  }
  __syncwarp();  // header and info written before lane 0's arrive publishes the stage
  const bool diag_ng = DGCL_DIAG_NO_GATHER && I.op == OP_COPY;
  if (lane == 0)
    mbar_expect_tx(full, (diag_ng ? 0u : operand_bytes<kLsu>(P, I)) + wtp.bytes + wdst.bytes);
  __syncwarp();
  if (lane == 0) {
    if (wtp.bytes) bulk_g2s(st + kTabTp, P.term_ptr + wtp.a, wtp.bytes, full);
    if (wdst.bytes) bulk_g2s(st + kTabDst, P.idx + wdst.a, wdst.bytes, full);
  }
  uint8_t *ops = st + kStageHdrBytes;
  if (diag_ng) return;
  if (I.op == OP_FANOUT) {
    // consecutive source rows: one bulk copy (packed rows), then the destination words
    const BufRef S = P.buf[I.src_kind][I.exec_rank];
    if (S.pitch == (int64_t)r16) {
      if (lane == 0) g2s(ops, S.ptr + I.src * S.pitch, (uint32_t)I.rows * r16, full, pol_copy);
    } else {
      for (int r = lane; r < I.rows; r += 32)
        g2s(ops + (size_t)r * r16, S.ptr + (I.src + r) * S.pitch, r16, full, pol_copy);
    }
    if (lane == 0) {
      const Win wt = window(I.t0, I.nterms, 4);
      bulk_g2s(ops + (size_t)I.rows * r16, P.terms + wt.a, wt.bytes, full);
    }
    return;
  }
  if (I.op == OP_COPY && (I.flags & kItemDirect)) {
    // short runs: stage only the source-row window; the consumers gather the rows
    if (lane == 0 && I.src < 0) {
      const Win ws = window(~I.src, I.rows, 4);
      bulk_g2s(ops, P.idx + ws.a, ws.bytes, full);
    }
  } else if (kLsu && I.op == OP_COPY && (I.flags & kItemLsu)) {
    // consumer cp.async gathers: the source-row window goes after the item's rows
    if (lane == 0 && I.src < 0) {
      const Win ws = window(~I.src, I.rows, 4);
      bulk_g2s(ops + (size_t)I.rows * r16, P.idx + ws.a, ws.bytes, full);
    }
  } else if (uses_gather4(P, I)) {
    // four rows per instruction (the last group repeats the item's last row; the stage holds
    // the padding rows, the consumers never store them)
    const int ng = (I.rows + 3) / 4;
    const bool hand = kHelp && ng >= 4;  // (helper h takes share h + 1 of 1 + DGCL_HELPER)
    constexpr int kNB = 32 * (1 + (kHelp ? DGCL_HELPER : 0));  // producer + helper threads
    if (hand) {  // the helper warps take shares of the groups (see executor_tma_kernel)
      if (*mb_busy) named_sync(2, kNB);  // (they have read the previous hand-over)
      if (lane == 0) {
        mb[0] = (uint32_t)(st - (stages_base));
        mb[1] = (uint32_t)(meta - metas_base);
        mb[2] = 0;
      }
      __syncwarp();
      named_arrive(1, kNB);
      *mb_busy = true;
    }
    issue_gather4(P, I, st, meta, full, lane, 0, hand ? ng / (1 + DGCL_HELPER) : ng, pol_copy);
  } else if (I.op == OP_COPY) {
    // one bulk copy per run of consecutive source rows when rows are packed (pitch == row16)
    const char *sbase = P.buf[I.src_kind][I.exec_rank].ptr;
    const int64_t spitch = P.buf[I.src_kind][I.exec_rank].pitch;
    const DevRun *runs = reinterpret_cast<const DevRun *>(meta);
    if (spitch == (int64_t)r16) {
      for (int q = lane; q < I.nterms; q += 32) {
        const DevRun R = runs[q];
        g2s(ops + (size_t)R.pos * r16, sbase + (int64_t)R.src * spitch, (uint32_t)R.len * r16,
            full, pol_copy);
      }
    } else {
      for (int q = lane; q < I.nterms; q += 32) {
        const DevRun R = runs[q];
        for (int j = 0; j < R.len; ++j)
          g2s(ops + (size_t)(R.pos + j) * r16, sbase + (int64_t)(R.src + j) * spitch, r16, full,
              pol_copy);
      }
    }
  } else if (is_staged(I)) {
    // staged FOLD: one bulk copy per segment of consecutive operand rows, then the staged terms
    const DevRun *segs = reinterpret_cast<const DevRun *>(meta);
    const int ns = (int)n_segments(I);
    for (int q = lane; q < ns; q += 32) {
      const DevRun R = segs[q];
      const BufRef B = P.buf[R.dst >> 8][R.dst & 255];
      if (B.pitch == (int64_t)r16) {
        g2s(ops + (size_t)R.pos * r16, B.ptr + (int64_t)R.src * B.pitch, (uint32_t)R.len * r16,
            full, pol_fold);
      } else {
        for (int j = 0; j < R.len; ++j)
          g2s(ops + (size_t)(R.pos + j) * r16, B.ptr + (int64_t)(R.src + j) * B.pitch, r16, full,
              pol_fold);
      }
    }
    if (lane == 0) {
      const Win wt = window(I.t0, I.nterms, 4);
      if (wt.bytes) bulk_g2s(ops + (size_t)staged_rows(I) * r16, P.sterms + wt.a, wt.bytes, full);
    }
  } else if (lane == 0) {
    // OP_FOLD: only the terms window is staged (into the operand area); the consumers gather
    // the operand rows themselves, many loads in flight per warp
    const Win wt = window(I.t0, I.nterms, 4);
    if (wt.bytes) bulk_g2s(ops, P.terms + wt.a, wt.bytes, full);
  }
}

// consumers: store a gathered COPY item (whole 16-B chunks: the destinations are library-owned
// rows whose pitch covers the rounded-up row)
__device__ __forceinline__ void store_copy(const ExecParams &P, const DevItem &I, const uint8_t *st,
                                           uint32_t tid, uint32_t T) {
  char *dbase = P.buf[I.dst_kind][I.dst_rank].ptr;
  const int64_t dpitch = P.buf[I.dst_kind][I.dst_rank].pitch;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t r16 = (uint32_t)P.row16;
  const uint32_t total = (uint32_t)I.rows * nch;
  const uint8_t *ops = st + kStageHdrBytes;
  if (I.dst >= 0) {
    char *d0 = dbase + I.dst * dpitch;
    for (uint32_t e0 = tid; e0 < total; e0 += T * kUnroll) {
#pragma unroll
      for (int j = 0; j < kUnroll; ++j) {
        const uint32_t e = e0 + j * T;
        if (e < total) {
          const uint32_t r = fdiv(e, P);
          const uint32_t col = e - r * nch;
          st_v4(d0 + (int64_t)r * dpitch + col * 16, lds_v4(ops + r * r16 + col * 16));
        }
      }
    }
  } else {
    const int32_t *tab = reinterpret_cast<const int32_t *>(st + kTabDst) +
                         reinterpret_cast<const int32_t *>(st + kHdrInfo)[1];
    for (uint32_t e0 = tid; e0 < total; e0 += T * kUnroll) {
#pragma unroll
      for (int j = 0; j < kUnroll; ++j) {
        const uint32_t e = e0 + j * T;
        if (e < total) {
          const uint32_t r = fdiv(e, P);
          const uint32_t col = e - r * nch;
          st_v4(dbase + (int64_t)tab[r] * dpitch + col * 16, lds_v4(ops + r * r16 + col * 16));
        }
      }
    }
  }
}

// consumers: COPY item into the multicast region (NVSwitch multicast):
// every 16-B chunk goes out once through the multicast address (multimem.st) and lands in every
// GPU's copy of the region; the destination rows are consecutive
__device__ __forceinline__ void store_copy_mc(const ExecParams &P, const DevItem &I,
                                              const uint8_t *st, uint32_t tid, uint32_t T) {
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t r16 = (uint32_t)P.row16;
  const uint32_t total = (uint32_t)I.rows * nch;
  const uint8_t *ops = st + kStageHdrBytes;
  for (uint32_t e = tid; e < total; e += T) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    mc_store16(P, I.exec_rank, I.dst + r, col, lds_v4(ops + r * r16 + col * 16));
  }
}

// consumers: FANOUT item — the staged rows stored into all their receivers' rows (halo or relay
// staging, library-owned: whole 16-B chunks).  Flat (destination pair, chunk) index space over the
// consumer threads, kUnroll independent chunks per thread in flight (as store_copy); with
// signalling on, the thread holding a pair's chunk 0 counts it for its receiver (published at the
// next FLUSH / END)
__device__ __forceinline__ void store_fanout(const ExecParams &P, const DevItem &I,
                                             const uint8_t *st, uint32_t tid, uint32_t T,
                                             uint32_t *s_pend, uint64_t pol_st) {
  const uint32_t r16 = (uint32_t)P.row16;
  const uint8_t *ops = st + kStageHdrBytes;
  const uint32_t *pw = reinterpret_cast<const uint32_t *>(ops + (size_t)I.rows * r16) +
                       window(I.t0, I.nterms, 4).skew;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)(I.nterms >> 1) * nch;
  const bool sig = (I.flags & kItemSignal) != 0;
  const uint32_t src0 = (uint32_t)I.src;
  if (P.bulk_store && r16 >= (uint32_t)kFanBulkRowBytes) {
    // rows of >= 1 KB: one bulk (TMA) store per (row, receiver) pair, issued by every consumer
    // thread for its pairs; the stage is released once the stores have read it
    const uint32_t np = (uint32_t)(I.nterms >> 1);
    for (uint32_t j = tid; j < np; j += T) {
      const uint32_t d = pw[2 * j], r = pw[2 * j + 1] - src0;
      const BufRef D = P.buf[(d & kFanRelay) ? K_RELAY : K_HALO][d >> 28];
      s2g(D.ptr + (int64_t)(d & kFanRowMask) * D.pitch, ops + r * r16, r16, pol_st);
      if (sig) atomicAdd(&s_pend[I.exec_rank * kMaxRanks + (d >> 28)], 1u);
    }
    if (tid < np) {
      bulk_commit();
      bulk_wait_read();
    }
    return;
  }
  for (uint32_t e0 = tid; e0 < total; e0 += T * kUnroll) {
#pragma unroll
    for (int q = 0; q < kUnroll; ++q) {
      const uint32_t e = e0 + q * T;
      if (e < total) {
        const uint32_t j = fdiv(e, P);
        const uint32_t col = e - j * nch;
        const uint32_t d = pw[2 * j], r = pw[2 * j + 1] - src0;
        const BufRef D = P.buf[(d & kFanRelay) ? K_RELAY : K_HALO][d >> 28];
        st_v4(D.ptr + (int64_t)(d & kFanRowMask) * D.pitch + col * 16,
              lds_v4(ops + r * r16 + col * 16));
        if (sig && col == 0) atomicAdd(&s_pend[I.exec_rank * kMaxRanks + (d >> 28)], 1u);
      }
    }
  }
}

// consumers: COPY item ADDED into its destination rows (ablation, option "atomic_backward"): every
// consumer thread takes whole rows, one TMA bulk reduce-add (fp32 add in L2, atomic per element)
// for the row's 16-B chunks and fp32 atomics for a partial last chunk (the destination is the
// caller's emb_grad: nothing past the row is touched)
__device__ __forceinline__ void store_copy_atomic(const ExecParams &P, const DevItem &I,
                                                  const uint8_t *st, uint32_t tid, uint32_t T) {
  const BufRef D = P.buf[I.dst_kind][I.dst_rank];
  const int32_t *tab = I.dst < 0 ? reinterpret_cast<const int32_t *>(st + kTabDst) +
                                       reinterpret_cast<const int32_t *>(st + kHdrInfo)[1]
                                 : nullptr;
  const uint32_t r16 = (uint32_t)P.row16;
  const uint8_t *ops = st + kStageHdrBytes;
  const uint32_t body = (uint32_t)P.row_bytes & ~15u;
  const int tailw = (P.row_bytes - (int)body) / 4;
  bool issued = false;
  for (uint32_t r = tid; r < (uint32_t)I.rows; r += T) {
    const int64_t drow = tab ? (int64_t)tab[r] : I.dst + r;
    char *dp = D.ptr + drow * D.pitch;
    if (body) {
      bulk_s2g_add_f32(dp, ops + r * r16, body);
      issued = true;
    }
    for (int w = 0; w < tailw; ++w)
      atomicAdd(reinterpret_cast<float *>(dp + body) + w,
                reinterpret_cast<const float *>(ops + r * r16 + body)[w]);
  }
  if (issued) {
    bulk_commit();
    bulk_wait_read();  // the stage may be reused once the reductions have read it
  }
}

// consumers: LSU item — gather the item's rows into the stage with 16-B cp.async (every consumer
// thread many chunks in flight), then make them visible to the async proxy for the bulk stores
__device__ __forceinline__ void gather_lsu(const ExecParams &P, const DevItem &I, uint8_t *st,
                                           uint32_t tid, uint32_t T) {
  const uint32_t r16 = (uint32_t)P.row16;
  uint8_t *ops = st + kStageHdrBytes;
  const char *sbase = P.buf[I.src_kind][I.exec_rank].ptr;
  const int64_t spitch = P.buf[I.src_kind][I.exec_rank].pitch;
  const int32_t *sidx = I.src < 0 ? reinterpret_cast<const int32_t *>(ops + (size_t)I.rows * r16) +
                                        window(~I.src, I.rows, 4).skew
                                  : nullptr;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  for (uint32_t e = tid; e < total; e += T) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    const int64_t srow = sidx ? (int64_t)sidx[r] : I.src + r;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(ops + r * r16 + col * 16)),
                 "l"(sbase + srow * spitch + (int64_t)col * 16)
                 : "memory");
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  fence_proxy_async_smem();  // (this thread's shared-memory writes -> the TMA stores' reads)
}

// consumers: COPY item with short runs — gather each row chunk straight from memory (8 loads in
// flight per thread) and store it; whole 16-B chunks (library-owned destination rows)
__device__ __forceinline__ void store_copy_direct(const ExecParams &P, const DevItem &I,
                                                  const uint8_t *st, uint32_t tid, uint32_t T) {
  constexpr int kU = 4;
  const char *sbase = P.buf[I.src_kind][I.exec_rank].ptr;
  const int64_t spitch = P.buf[I.src_kind][I.exec_rank].pitch;
  char *dbase = P.buf[I.dst_kind][I.dst_rank].ptr;
  const int64_t dpitch = P.buf[I.dst_kind][I.dst_rank].pitch;
  const int32_t *sidx = I.src < 0 ? reinterpret_cast<const int32_t *>(st + kStageHdrBytes) +
                                        window(~I.src, I.rows, 4).skew
                                  : nullptr;
  const int32_t *didx = I.dst < 0 ? reinterpret_cast<const int32_t *>(st + kTabDst) +
                                        reinterpret_cast<const int32_t *>(st + kHdrInfo)[1]
                                  : nullptr;
  const bool nc = readonly_kind(I.src_kind);
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  for (uint32_t e0 = tid; e0 < total; e0 += T * kU) {
    int4 v[kU];
#pragma unroll
    for (int j = 0; j < kU; ++j) {
      const uint32_t e = e0 + j * T;
      if (e < total) {
        const uint32_t r = fdiv(e, P);
        const uint32_t col = e - r * nch;
        const int64_t srow = sidx ? (int64_t)sidx[r] : I.src + r;
        const char *sp = sbase + srow * spitch + (int64_t)col * 16;
        v[j] = nc ? ld_nc_v4(sp) : ld_cg_v4(sp);
      }
    }
#pragma unroll
    for (int j = 0; j < kU; ++j) {
      const uint32_t e = e0 + j * T;
      if (e < total) {
        const uint32_t r = fdiv(e, P);
        const uint32_t col = e - r * nch;
        const int64_t drow = didx ? (int64_t)didx[r] : I.dst + r;
        st_v4(dbase + drow * dpitch + (int64_t)col * 16, v[j]);
      }
    }
  }
}

// consumers: fold a gathered FOLD item (operands in list order) and store it; the row's last
// chunk is stored partially (the destination may be the caller's emb_grad)
template <int kE>
__device__ __forceinline__ void store_fold_multi(const ExecParams &P, const DevItem &I, const uint8_t *st,
                                           uint32_t tid, uint32_t T) {
  const BufRef D = P.buf[I.dst_kind][I.dst_rank];
  const int32_t *info = reinterpret_cast<const int32_t *>(st + kHdrInfo);
  const int64_t *tp = reinterpret_cast<const int64_t *>(st + kTabTp) + info[0];
  const int32_t *tab = reinterpret_cast<const int32_t *>(st + kTabDst) + info[1];
  const uint32_t *tm = reinterpret_cast<const uint32_t *>(st + kStageHdrBytes) +
                       window(I.t0, I.nterms, 4).skew;  // the item's terms, staged by the producer
  const int init = I.fold_init;
  const int mode = I.term_mode;
  const int exec = I.exec_rank;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  const int tail = P.row_bytes - (int)(nch - 1) * 16;
  // operand j of the current row at chunk col: halo-gradient rows are read-only inputs (nc),
  // slots were written during the launch (cg)
  auto operand = [&](uint32_t term, uint32_t col, int nb) -> int4 {
    const bool slot = mode == kTermLocal && (term & kTermSlot) != 0;
    const BufRef &B = mode == kTermRankHgrad ? P.buf[K_HGRAD][term >> 28]
                      : slot                 ? P.buf[K_SLOT][exec]
                                             : P.buf[K_HGRAD][exec];
    const uint32_t row = mode == kTermRankHgrad ? (term & kTermRowMask) : (term & ~kTermSlot);
    const char *p = B.ptr + (int64_t)row * B.pitch + (int64_t)col * 16;
    if (nb == 16) return slot ? ld_cg_v4(p) : ld_nc_v4(p);
    return slot ? ld_part<false>(p, nb) : ld_part<true>(p, nb);
  };
  // kE independent output chunks per thread; every round issues one operand load per chunk (kE
  // loads in flight) and then adds them, so each chunk's terms are still added in list order
  const int j0 = init ? 0 : 1;  // first term still to add after the starting value
  auto dst_of = [&](uint32_t r, uint32_t col) -> char * {
    const int64_t drow = I.dst >= 0 ? I.dst + r : (int64_t)tab[r];
    return D.ptr + drow * D.pitch + (int64_t)col * 16;
  };
  for (uint32_t e0 = tid; e0 < total; e0 += T * kE) {
    float4 acc[kE];
    uint32_t rc[kE];  // (row << 16) | chunk, 0xffffffff when past the end
    int cnt[kE];
    int rounds = 0;
#pragma unroll
    for (int q = 0; q < kE; ++q) {
      const uint32_t e = e0 + q * T;
      cnt[q] = 0;
      rc[q] = 0xffffffffu;
      if (e < total) {
        const uint32_t r = fdiv(e, P);
        const uint32_t col = e - r * nch;
        rc[q] = (r << 16) | col;
        const int nb = col + 1 == nch ? tail : 16;
        cnt[q] = (int)(tp[r + 1] - tp[r]);
        if (init) {
          char *dp = dst_of(r, col);
          acc[q] = as_f4(nb == 16 ? ld_cg_v4(dp) : ld_part<false>(dp, nb));
        } else {
          acc[q] = as_f4(operand(tm[tp[r] - I.t0], col, nb));
        }
        rounds = max(rounds, cnt[q] - j0);
      }
    }
    for (int t = 0; t < rounds; ++t) {
      int4 v[kE];
#pragma unroll
      for (int q = 0; q < kE; ++q) {
        if (j0 + t < cnt[q]) {
          const uint32_t r = rc[q] >> 16, col = rc[q] & 0xffffu;
          v[q] = operand(tm[tp[r] - I.t0 + j0 + t], col, col + 1 == nch ? tail : 16);
        }
      }
#pragma unroll
      for (int q = 0; q < kE; ++q)
        if (j0 + t < cnt[q]) add4(acc[q], v[q]);
    }
#pragma unroll
    for (int q = 0; q < kE; ++q) {
      if (rc[q] == 0xffffffffu) continue;
      const uint32_t r = rc[q] >> 16, col = rc[q] & 0xffffu;
      const int nb = col + 1 == nch ? tail : 16;
      char *dp = dst_of(r, col);
      if (nb == 16)
        st_v4(dp, as_i4(acc[q]));
      else
        st_part(dp, as_i4(acc[q]), nb);
    }
  }
}

// consumers: staged FOLD item — every operand row is in the stage; add each output chunk's terms
// in list order (init row first when the fold starts from the destination) and store it
__device__ __forceinline__ void store_fold_staged(const ExecParams &P, const DevItem &I,
                                                  const uint8_t *st, uint32_t tid, uint32_t T) {
  const BufRef D = P.buf[I.dst_kind][I.dst_rank];
  const int32_t *info = reinterpret_cast<const int32_t *>(st + kHdrInfo);
  const int64_t *tp = reinterpret_cast<const int64_t *>(st + kTabTp) + info[0];
  const int32_t *tab = reinterpret_cast<const int32_t *>(st + kTabDst) + info[1];
  const uint32_t r16 = (uint32_t)P.row16;
  const uint8_t *ops = st + kStageHdrBytes;
  const uint32_t *stt = reinterpret_cast<const uint32_t *>(ops + (size_t)staged_rows(I) * r16) +
                        window(I.t0, I.nterms, 4).skew;
  const int init = I.fold_init;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  const int tail = P.row_bytes - (int)(nch - 1) * 16;
  const int64_t tbase = tp[0];
  if (I.term_mode == kTermRankTree) {
    // postfix programs over the staged rows (loopback tree-order backward), one chunk per thread
    for (uint32_t e = tid; e < total; e += T) {
      const uint32_t r = fdiv(e, P);
      const uint32_t col = e - r * nch;
      const uint8_t *oc = ops + col * 16;
      const int j = (int)(tp[r] - tbase), je = (int)(tp[r + 1] - tbase);
      const float4 acc =
          fold_tree(as_f4(lds_v4(oc + r * r16)), stt + j, je - j,
                    [&](uint32_t s) { return as_f4(lds_v4(oc + (s & kTreeRowMask) * r16)); });
      const int64_t drow = I.dst >= 0 ? I.dst + r : (int64_t)tab[r];
      char *dp = D.ptr + drow * D.pitch + (int64_t)col * 16;
      if (col + 1 < nch || tail == 16)
        st_v4(dp, as_i4(acc));
      else
        st_part(dp, as_i4(acc), tail);
    }
    return;
  }
  for (uint32_t e = tid; e < total; e += T) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    const uint8_t *oc = ops + col * 16;
    int j = (int)(tp[r] - tbase);
    const int je = (int)(tp[r + 1] - tbase);
    float4 acc;
    if (init) {
      acc = as_f4(lds_v4(oc + r * r16));
    } else {
      acc = as_f4(lds_v4(oc + stt[j] * r16));
      ++j;
    }
    for (; j + 4 <= je; j += 4) {
      const int4 v0 = lds_v4(oc + stt[j] * r16), v1 = lds_v4(oc + stt[j + 1] * r16);
      const int4 v2 = lds_v4(oc + stt[j + 2] * r16), v3 = lds_v4(oc + stt[j + 3] * r16);
      add4(acc, v0);
      add4(acc, v1);
      add4(acc, v2);
      add4(acc, v3);
    }
    for (; j < je; ++j) add4(acc, lds_v4(oc + stt[j] * r16));
    const int64_t drow = I.dst >= 0 ? I.dst + r : (int64_t)tab[r];
    char *dp = D.ptr + drow * D.pitch + (int64_t)col * 16;
    if (col + 1 < nch || tail == 16)
      st_v4(dp, as_i4(acc));
    else
      st_part(dp, as_i4(acc), tail);
  }
}

// consumers: unstaged tree-order FOLD (kTermRankTree): each output chunk evaluates its row's
// postfix program, operands gathered from the requesters' halo-gradient rows
__device__ __forceinline__ void store_fold_tree(const ExecParams &P, const DevItem &I,
                                                const uint8_t *st, uint32_t tid, uint32_t T) {
  const BufRef D = P.buf[I.dst_kind][I.dst_rank];
  const int32_t *info = reinterpret_cast<const int32_t *>(st + kHdrInfo);
  const int64_t *tp = reinterpret_cast<const int64_t *>(st + kTabTp) + info[0];
  const int32_t *tab = reinterpret_cast<const int32_t *>(st + kTabDst) + info[1];
  const uint32_t *tm = reinterpret_cast<const uint32_t *>(st + kStageHdrBytes) +
                       window(I.t0, I.nterms, 4).skew;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  const int tail = P.row_bytes - (int)(nch - 1) * 16;
  for (uint32_t e = tid; e < total; e += T) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    const int nb = col + 1 == nch ? tail : 16;
    const int64_t drow = I.dst >= 0 ? I.dst + r : (int64_t)tab[r];
    char *dp = D.ptr + drow * D.pitch + (int64_t)col * 16;
    const float4 init = as_f4(nb == 16 ? ld_cg_v4(dp) : ld_part<false>(dp, nb));
    const float4 acc = fold_tree(init, tm + (tp[r] - I.t0), (int)(tp[r + 1] - tp[r]),
                                 [&](uint32_t w) {
                                   const BufRef &B = P.buf[K_HGRAD][w >> 28];
                                   const char *p = B.ptr + (int64_t)(w & kTreeRowMask) * B.pitch +
                                                   (int64_t)col * 16;
                                   return as_f4(nb == 16 ? ld_nc_v4(p) : ld_part<true>(p, nb));
                                 });
    if (nb == 16)
      st_v4(dp, as_i4(acc));
    else
      st_part(dp, as_i4(acc), nb);
  }
}

// consumers: FOLD item with many terms per row — one output chunk at a time, its terms loaded in
// batches of 8 independent loads, then added in list order
template <int kBatch>
__device__ __forceinline__ void store_fold_rows(const ExecParams &P, const DevItem &I,
                                             const uint8_t *st, uint32_t tid, uint32_t T) {
  const BufRef D = P.buf[I.dst_kind][I.dst_rank];
  const int32_t *info = reinterpret_cast<const int32_t *>(st + kHdrInfo);
  const int64_t *tp = reinterpret_cast<const int64_t *>(st + kTabTp) + info[0];
  const int32_t *tab = reinterpret_cast<const int32_t *>(st + kTabDst) + info[1];
  const uint32_t *tm = reinterpret_cast<const uint32_t *>(st + kStageHdrBytes) +
                       window(I.t0, I.nterms, 4).skew;
  const int init = I.fold_init;
  const int mode = I.term_mode;
  const int exec = I.exec_rank;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  const int tail = P.row_bytes - (int)(nch - 1) * 16;
  auto operand = [&](uint32_t term, uint32_t col, int nb) -> int4 {
    const bool slot = mode == kTermLocal && (term & kTermSlot) != 0;
    const BufRef &B = mode == kTermRankHgrad ? P.buf[K_HGRAD][term >> 28]
                      : slot                 ? P.buf[K_SLOT][exec]
                                             : P.buf[K_HGRAD][exec];
    const uint32_t row = mode == kTermRankHgrad ? (term & kTermRowMask) : (term & ~kTermSlot);
    const char *p = B.ptr + (int64_t)row * B.pitch + (int64_t)col * 16;
    if (nb == 16) return slot ? ld_cg_v4(p) : ld_nc_v4(p);
    return slot ? ld_part<false>(p, nb) : ld_part<true>(p, nb);
  };
  for (uint32_t e = tid; e < total; e += T) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    const int nb = col + 1 == nch ? tail : 16;
    const int64_t ta = tp[r], tb = tp[r + 1];
    const uint32_t *rt = tm + (ta - I.t0);
    const int cnt = (int)(tb - ta);
    const int64_t drow = I.dst >= 0 ? I.dst + r : (int64_t)tab[r];
    char *dp = D.ptr + drow * D.pitch + (int64_t)col * 16;
    float4 acc;
    int j = 0;
    if (init) {
      acc = as_f4(nb == 16 ? ld_cg_v4(dp) : ld_part<false>(dp, nb));
    } else {
      acc = as_f4(operand(rt[0], col, nb));
      j = 1;
    }
    while (j < cnt) {
      int4 v[kBatch];
      const int n = cnt - j < kBatch ? cnt - j : kBatch;
#pragma unroll
      for (int q = 0; q < kBatch; ++q)
        if (q < n) v[q] = operand(rt[j + q], col, nb);
#pragma unroll
      for (int q = 0; q < kBatch; ++q)
        if (q < n) add4(acc, v[q]);
      j += n;
    }
    if (nb == 16)
      st_v4(dp, as_i4(acc));
    else
      st_part(dp, as_i4(acc), nb);
  }
}

template <int kMask, int kMaxThreads = 512>
__global__ void __launch_bounds__(kMaxThreads, 1)
    executor_tma_kernel(const __grid_constant__ ExecParams P) {
  extern __shared__ __align__(128) uint8_t dsmem[];
  const uint32_t NS = (uint32_t)P.tma_stages;
  const size_t stage_bytes = (size_t)P.tma_buf, meta_bytes = (size_t)P.meta_bytes;
  const size_t kDescOff = kMetaOff + kMetaSlots * meta_bytes;
  const size_t kStageOff = kDescOff + kDescSlots * 64;
  const size_t kPendOff = kStageOff + NS * stage_bytes;  // 1 KB counts + 3 words
  uint64_t *full = reinterpret_cast<uint64_t *>(dsmem);
  uint64_t *empty = full + kMaxTmaStages;
  uint64_t *metab = empty + kMaxTmaStages;
  uint64_t *descb = metab + kMetaBarriers;
  uint8_t *metas = dsmem + kMetaOff;
  DevItem *descs = reinterpret_cast<DevItem *>(dsmem + kDescOff);
  uint8_t *stages = dsmem + kStageOff;
  // rows stored since the last flush per (source, receiver), their counter family, and the
  // consumer barrier words: carved from the dynamic region (no static shared memory)
  uint32_t *s_pend = reinterpret_cast<uint32_t *>(dsmem + kPendOff);
  int &s_pend_base = *reinterpret_cast<int *>(dsmem + kPendOff + 1024);
  unsigned &s_bar_count = *reinterpret_cast<unsigned *>(dsmem + kPendOff + 1028);
  volatile unsigned &s_bar_gen = *reinterpret_cast<volatile unsigned *>(dsmem + kPendOff + 1032);
  // producer-private: per executing rank, the wait list last found satisfied (counters are
  // monotonic and their targets fixed for the launch, so it stays satisfied: later items of the
  // same (direction, stage, rank) skip the flag reads)
  int32_t *s_wait_ok = reinterpret_cast<int32_t *>(dsmem + kPendOff + 1040);
  // producer-private (dynamic claiming): the launch index of the item in each descriptor slot
  uint32_t *s_claim = reinterpret_cast<uint32_t *>(dsmem + kPendOff + 1104);
  // producer -> helper hand-over: stage offset, meta-slot offset, end flag
  uint32_t *s_mb = reinterpret_cast<uint32_t *>(dsmem + kPendOff + 1136);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // copy-only instances: warp 1 helps the producer issue gather4 instructions (the issue loop of
  // a TMA instruction is serialised per lane: the producer was the bound of the small-row
  // forwards, profiles/r2k_orkut_fwd_source.md)
  constexpr bool kHelp = DGCL_HELPER && (kMask & kMaskCopy) &&
                         !(kMask & (kMaskFold | kMaskStaged | kMaskTree | kMaskFanout | kMaskLsu |
                                    kMaskMcast | kMaskDirect));
  constexpr int kProdWarps = kHelp ? 1 + DGCL_HELPER : 1;
  // dual producers (P.dual_prod): copy-only instances use the helper warp, staged-fold instances
  // take warp 1 from the consumers
  constexpr bool kDualCap =
      kHelp || kMask == kMaskStaged || kMask == (kMaskTree | kMaskStaged);
  const int prod_warps = (kDualCap && P.dual_prod) ? 2 : kProdWarps;
  const int n_cons_warps = (int)(blockDim.x >> 5) - prod_warps;
  // L2 hints (option "l2_policy"): bit 0 data stores evict_first (write-once halo / relay /
  // slot rows), bit 1 COPY / FANOUT source reads evict_last (a row sent to several receivers is
  // read again soon), bit 2 COPY source reads evict_first, bit 3 FOLD operand reads evict_first
  const int lp = P.l2_policy;
  const uint64_t pol_st = (lp & 1) ? policy_evict_first() : 0;
  const uint64_t pol_copy = (lp & 2) ? policy_evict_last() : (lp & 4) ? policy_evict_first() : 0;
  const uint64_t pol_fold = (lp & 8) ? policy_evict_first() : 0;
  for (int i = threadIdx.x; i < kMaxRanks * kMaxRanks; i += blockDim.x) s_pend[i] = 0;
  if (threadIdx.x == 0) {
    s_mb[0] = 0;  // (dual producers with claims: next stage use, finished producers)
    s_mb[1] = 0;
    s_pend_base = 0;
    s_bar_count = 0;
    s_bar_gen = 0;
    for (int r = 0; r < kMaxRanks; ++r) s_wait_ok[r] = -1;
    for (int s = 0; s < (int)NS; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], n_cons_warps);
    }
    for (int s = 0; s < kMetaBarriers; ++s) mbar_init(&metab[s], 1);
    for (int s = 0; s < kDescSlots; ++s) mbar_init(&descb[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (kDualCap && P.dual_prod && warp <= 1) {
    // --------------------- dual producers (simple copy launches) -----------------------------
    // A launch of plain COPY items or staged FOLD items — no waits, no signals, no tracing,
    // round-robin items (the host sets dual_prod only then) — has no FLUSH markers, so item m
    // of this CTA
    // simply takes stage use k = m.  Warps 0 and 1 then split the items (m = w, w + 2, ...),
    // each with its own descriptor slots [4w, 4w + 4) and metadata slots (half-size), and issue
    // their items' bulk copies / gather4s independently (no helper hand-over); the consumers
    // still take the stages in k order.
    // (ncu r2sk: on the Reddit dim-602 forward one producer warp was busy ~100 % of the time,
    // ~450 dependent instructions per item — the launch's bound.)
    // With dynamic claiming (P.claim) the producers claim their own batches and take stage uses
    // from a shared counter (s_mb[0]; the helper mailbox is unused here), so item order and
    // stage order need not agree; the second producer to run out of items emits END (s_mb[1]).
    const int pw = warp;
    const uint32_t G = gridDim.x;
    const bool claims = P.claim != nullptr;
    const uint32_t nmine = claims ? 0xffffffffu
                           : blockIdx.x < (uint32_t)P.n_items
                               ? ((uint32_t)P.n_items - blockIdx.x + G - 1) / G
                               : 0;
    const size_t mb2 = meta_bytes / 2;
    auto dslot = [&](uint32_t j) { return (uint32_t)(4 * pw) + (j & 3u); };
    auto mslot = [&](uint32_t j) { return (uint32_t)(kDualMetaSlots * pw) + (j % kDualMetaSlots); };
    uint64_t bnext = 0;
    uint32_t bleft = 0;
    auto req_desc = [&](uint32_t j) -> bool {  // lane 0: my j-th item (claims: false = none left)
      const uint32_t sl = dslot(j);
      uint64_t idx;
      if (claims) {
        if (bleft == 0) {
          const uint64_t b0 = atomicAdd(reinterpret_cast<unsigned long long *>(P.claim),
                                        (unsigned long long)P.claim_batch) - P.claim_base;
          if (b0 >= (uint64_t)P.n_items) return false;
          bnext = b0;
          bleft = (uint32_t)min((uint64_t)P.claim_batch, (uint64_t)P.n_items - b0);
        }
        idx = bnext++;
        --bleft;
      } else {
        idx = blockIdx.x + (uint64_t)((uint32_t)pw + 2u * j) * G;
      }
      s_claim[sl] = (uint32_t)idx;
      mbar_expect_tx(&descb[sl], (uint32_t)sizeof(DevItem));
      bulk_g2s(descs + sl, P.items + idx, (uint32_t)sizeof(DevItem), &descb[sl]);
      return true;
    };
    auto desc_wait = [&](uint32_t j) -> const DevItem & {
      mbar_wait(&descb[dslot(j)], (j >> 2) & 1u);
      return descs[dslot(j)];
    };
    auto meta_at = [&](uint32_t j) { return metas + (size_t)mslot(j) * mb2; };
    auto meta_req = [&](uint32_t j) {  // lane 0, descriptor j ready
      issue_meta<false>(P, descs[dslot(j)], meta_at(j), &metab[mslot(j)]);
    };
    // my items: round-robin m = pw, pw + 2, ... < nmine; claims: until a claim fails
    uint32_t nj = 0;
    if (!claims)
      while ((uint32_t)pw + 2u * nj < nmine) ++nj;
    else
      nj = 0xffffffffu;
    auto request = [&](uint32_t j) {  // warp-collective: request my j-th item (claims: learn the end)
      int ok = 1;
      if (lane == 0) ok = req_desc(j) ? 1 : 0;
      ok = __shfl_sync(0xffffffffu, ok, 0);
      if (!ok && j < nj) nj = j;
    };
    fence_proxy_async_smem();
    for (uint32_t j = 0; j < (uint32_t)kDualDescAhead && j < nj; ++j) request(j);
    for (uint32_t j = 0; j < (uint32_t)kDualMetaAhead && j < nj; ++j) {
      desc_wait(j);
      if (lane == 0) meta_req(j);
    }
    bool dummy = false;
    for (uint32_t j = 0; j < nj; ++j) {
      const DevItem I = desc_wait(j);
      mbar_wait(&metab[mslot(j)], (j / kDualMetaSlots) & 1u);
      uint32_t k = (uint32_t)pw + 2u * j;  // stage use (round-robin: my item's position)
      if (claims) {
        if (lane == 0) k = atomicAdd(&s_mb[0], 1u);
        k = __shfl_sync(0xffffffffu, k, 0);
      }
      uint32_t stage, use;
      ring_pos(k, NS, stage, use);
      if (use > 0) mbar_wait(&empty[stage], (use - 1) & 1u);
      fence_proxy_async_smem();
      issue_item<false, false>(P, I, &descs[dslot(j)], stages + (size_t)stage * stage_bytes,
                               meta_at(j), &full[stage], lane, s_claim[dslot(j)], pol_copy,
                               pol_fold, s_mb, &dummy, stages, metas);
      __syncwarp();
      // prefetch (the fence above covers the slots read so far)
      if (j + kDualDescAhead < nj) request(j + kDualDescAhead);
      if (j + kDualMetaAhead < nj) {
        desc_wait(j + kDualMetaAhead);
        if (lane == 0) meta_req(j + kDualMetaAhead);
      }
      __syncwarp();
    }
    // END after every item: round-robin at stage use nmine (by the producer whose turn it is);
    // claims: the second producer to finish takes the next stage use
    bool emit = false;
    uint32_t kend = nmine;
    if (claims) {
      int last = 0;
      if (lane == 0 && atomicAdd(&s_mb[1], 1u) == 1u) {
        last = 1;
        kend = atomicAdd(&s_mb[0], 1u);
      }
      last = __shfl_sync(0xffffffffu, last, 0);
      kend = __shfl_sync(0xffffffffu, kend, 0);
      emit = last != 0;
    } else {
      emit = (nmine & 1u) == (uint32_t)pw;
    }
    if (emit) {
      uint32_t stage, use;
      ring_pos(kend, NS, stage, use);
      if (use > 0) mbar_wait(&empty[stage], (use - 1) & 1u);
      if (lane == 0) {
        reinterpret_cast<DevItem *>(stages + (size_t)stage * stage_bytes)->op = OP_END;
        mbar_arrive(&full[stage]);
      }
      __syncwarp();
    }
  } else if (kHelp && warp >= 1 && warp <= DGCL_HELPER) {
    // ------------------------------- helper warps --------------------------------------------
    constexpr int kNB = 32 * (1 + DGCL_HELPER);
    const uint64_t pol_h = pol_copy;
    for (;;) {
      named_sync(1, kNB);  // a hand-over (or the end) from the producer
      const uint32_t so = s_mb[0], mo = s_mb[1], end = s_mb[2];
      __syncwarp();
      named_arrive(2, kNB);  // mailbox read
      if (end) break;
      uint8_t *st = stages + so;
      const DevItem I = *reinterpret_cast<const DevItem *>(st);
      fence_proxy_async_smem();
      const int ng = (I.rows + 3) / 4;
      issue_gather4(P, I, st, metas + mo, &full[so / stage_bytes], lane,
                    ng * warp / (1 + DGCL_HELPER), ng * (warp + 1) / (1 + DGCL_HELPER), pol_h);
    }
  } else if (warp == 0) {
    // ------------------------------- producer warp -------------------------------------------
    // item q of this CTA is P.items[blockIdx.x + q * gridDim.x]; its descriptor is bulk-copied
    // into ring slot q % kDescSlots kDescAhead items ahead, its row runs into meta slot
    // q % kMetaSlots kMetaAhead items ahead, so their latency never stalls the issue loop
    const uint32_t G = gridDim.x;
    // Items are taken in list order: round-robin (item q of this CTA at list position
    // blockIdx.x + q * G), or — with P.claim — in batches of P.claim_batch consecutive positions
    // claimed from a launch-wide counter (claims hand out positions in increasing order, so every
    // CTA's queue stays in list = stage order and the earliest unfinished item can always run:
    // deadlock-free like round-robin; CTAs that drew cheaper items take more, which removes the
    // per-SM speed spread at stage boundaries).  nmine: this CTA's item count (dynamic: known
    // once a claim fails).
    uint32_t nmine = P.claim ? 0xffffffffu
                             : blockIdx.x < (uint32_t)P.n_items
                                   ? ((uint32_t)P.n_items - blockIdx.x + G - 1) / G
                                   : 0;
    uint64_t bnext = 0;
    uint32_t bleft = 0;                        // (lane 0) unissued positions of the batch
    auto request_desc = [&](uint32_t q) -> bool {  // lane 0, after a proxy fence
      const uint32_t s = q % kDescSlots;
      uint64_t idx;
      if (P.claim) {
        if (bleft == 0) {
          const uint64_t b0 = atomicAdd(reinterpret_cast<unsigned long long *>(P.claim),
                                        (unsigned long long)P.claim_batch) - P.claim_base;
          if (b0 >= (uint64_t)P.n_items) return false;
          bnext = b0;
          bleft = (uint32_t)min((uint64_t)P.claim_batch, (uint64_t)P.n_items - b0);
        }
        idx = bnext++;
        --bleft;
        s_claim[s] = (uint32_t)idx;
      } else {
        idx = blockIdx.x + (uint64_t)q * G;
      }
      mbar_expect_tx(&descb[s], (uint32_t)sizeof(DevItem));
      bulk_g2s(descs + s, P.items + idx, (uint32_t)sizeof(DevItem), &descb[s]);
      return true;
    };
    auto req = [&](uint32_t q) {  // warp-collective: request q, learn the end when claiming
      int ok_q = 1;
      if (lane == 0) ok_q = request_desc(q) ? 1 : 0;
      if (P.claim) {
        ok_q = __shfl_sync(0xffffffffu, ok_q, 0);
        if (!ok_q && q < nmine) nmine = q;
      }
    };
    auto desc_ready = [&](uint32_t q) -> const DevItem & {
      mbar_wait(&descb[q % kDescSlots], (q / kDescSlots) & 1u);
      return descs[q % kDescSlots];
    };
    uint32_t k = 0;  // stages issued (data items and markers)
    uint32_t m = 0;  // this CTA's item sequence
    bool ok = true;
    uint32_t ready_ok = 0;  // lane 0: destinations whose ready word reached seq (bit per rank)
    auto known_sources = [&](const DevItem &I) {
      return I.wait_n == 0 || s_wait_ok[I.exec_rank] == I.wait_off;
    };
    bool mb_busy = false;  // a hand-over to the helper is outstanding (not yet read)
    bool pend = false;  // signalling items issued since the last FLUSH
    int pend_key = -1;  // their counter family: ctr_index(dir, stage, 0)
    auto emit_marker = [&](uint8_t op) {  // header-only stage: FLUSH or END
      uint32_t stage, use;
      ring_pos(k, NS, stage, use);
      if (use > 0) mbar_wait(&empty[stage], (use - 1) & 1u);
      if (lane == 0) {
        reinterpret_cast<DevItem *>(stages + (size_t)stage * stage_bytes)->op = op;
        mbar_arrive(&full[stage]);
      }
      __syncwarp();
      ++k;
    };
    auto meta_of = [&](uint32_t q) { return metas + (size_t)(q % kMetaSlots) * meta_bytes; };
    // One proxy fence per item: generic reads of the descriptor ring, the meta slots and (by the
    // consumers, ordered by the empty barrier) the stage come before every bulk copy into them.
    // Prefetches are issued after the item, so the item's fence covers them too.
    fence_proxy_async_smem();
    for (uint32_t q = 0; q < (uint32_t)kDescAhead && q < nmine; ++q) req(q);
    for (uint32_t q = 0; q < (uint32_t)kMetaAhead && q < nmine; ++q) {
      const DevItem Iq = desc_ready(q);
      if (lane == 0) issue_meta<(kMask & kMaskLsu) != 0>(P, Iq, meta_of(q), &metab[q % kMetaSlots]);
    }
    for (; m < nmine; ++m) {
      const DevItem I = desc_ready(m);  // registers: no shared-memory reload per field
      const DevItem *Ism = &descs[m % kDescSlots];
      bool fenced = false;
      const uint32_t gidx = P.claim ? s_claim[m % kDescSlots] : blockIdx.x + m * G;  // (launch)
      if (P.trace && lane == 0) {
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        P.trace[gidx].t_start = globaltimer();
        P.trace[gidx].sm = smid;
        P.trace[gidx].tag = trace_tag(I, P.groups[I.group].stage, P.groups[I.group].block);
      }
      if (I.op == OP_READY) {
        // (the item's metadata phase completed on its arrive: observe it, synccheck-clean)
        mbar_wait(&metab[m % kMetaSlots], (m / kMetaSlots) & 1u);
        // my buffers of every layer are free for this call: tell every peer
        if (lane == 0)
          for (int s = 0; s < P.world; ++s)
            if (s != I.exec_rank)
              st_release(P.flags[s] + kReadyBase + I.exec_rank, P.seq, P.sys_scope);
      } else if (I.op == OP_WAIT) {
        mbar_wait(&metab[m % kMetaSlots], (m / kMetaSlots) & 1u);
        // forward completion: the launch ends only once every incoming row landed
        if (pend) {
          emit_marker(OP_FLUSH);
          pend = false;
        }
        int w = 1;
        if (lane == 0 && !known_sources(I)) w = wait_item_sources(P, I, 200000 + I.group) ? 1 : 0;
        ok = __shfl_sync(0xffffffffu, w, 0) != 0;
        if (!ok) break;
      } else if (I.op == OP_COPY || I.op == OP_FOLD || I.op == OP_FANOUT) {
        // Done counts are published in batches (FLUSH markers): before this producer could
        // block on a wait, whenever the counter family (direction, stage) changes, and before
        // an item that signals nothing (relay forwards: a stage's leaves follow its forwarded
        // rows, whose counts the next stage waits on — holding them back until this CTA blocks
        // would delay that stage by the whole leaf phase)
        const bool sig = (I.flags & kItemSignal) != 0;
        const int key = sig ? I.sig_ctr - I.exec_rank : -1;
        if (pend) {
          int ready = 1;
          if (lane == 0) {
            ready = known_sources(I) || waits_ready(P, I) ? 1 : 0;
            if (ready && P.use_ready && I.ready_rank >= 0 && !((ready_ok >> I.ready_rank) & 1u))
              ready = ld_acquire(P.flags[I.exec_rank] + kReadyBase + I.ready_rank, P.sys_scope) >=
                      P.seq;
            if (ready && P.use_ready && I.ready_rank == kReadyAll)
              for (int s = 0; s < P.world && ready; ++s)
                if (s != I.exec_rank && !((ready_ok >> s) & 1u))
                  ready = ld_acquire(P.flags[I.exec_rank] + kReadyBase + s, P.sys_scope) >= P.seq;
          }
          ready = __shfl_sync(0xffffffffu, ready, 0);
          if (!ready || key != pend_key) {
            emit_marker(OP_FLUSH);
            pend = false;
          }
        }
        int w = 1, acq = 0;
        if (lane == 0) {
          // sources final (stage chaining) and the destination's buffers free (ready word)
          if (!known_sources(I)) {
            w = wait_item_sources(P, I, 100000 + I.group) ? 1 : 0;
            if (w) s_wait_ok[I.exec_rank] = I.wait_off;
            acq = 1;
          }
          if (w && P.use_ready && I.ready_rank >= 0 && !((ready_ok >> I.ready_rank) & 1u)) {
            w = wait_geq(P.flags[I.exec_rank] + kReadyBase + I.ready_rank, P.seq, P,
                         1000 + I.group) ? 1 : 0;
            if (w) ready_ok |= 1u << I.ready_rank;
          }
          if (w && P.use_ready && I.ready_rank == kReadyAll)  // fan-out: every receiver
            for (int s = 0; s < P.world && w; ++s)
              if (s != I.exec_rank && !((ready_ok >> s) & 1u)) {
                w = wait_geq(P.flags[I.exec_rank] + kReadyBase + s, P.seq, P, 1000 + I.group) ? 1 : 0;
                if (w) ready_ok |= 1u << s;
              }
        }
        ok = __shfl_sync(0xffffffffu, w, 0) != 0;
        if (!ok) break;
        // acquired peers' rows -> bulk reads (a wait list found satisfied earlier was fenced then:
        // this warp's later bulk reads follow that fence in program order)
        if (__shfl_sync(0xffffffffu, acq, 0)) fence_proxy_async_global();
        mbar_wait(&metab[m % kMetaSlots], (m / kMetaSlots) & 1u);
        uint32_t stage, use;
        ring_pos(k, NS, stage, use);
        if (use > 0) mbar_wait(&empty[stage], (use - 1) & 1u);
        if (P.trace && lane == 0) P.trace[gidx].t_ready = globaltimer();
        fence_proxy_async_smem();
        fenced = true;
        issue_item<(kMask & kMaskLsu) != 0, kHelp>(P, I, Ism, stages + (size_t)stage * stage_bytes,
                                                   meta_of(m), &full[stage], lane, gidx, pol_copy,
                                                   pol_fold, s_mb, &mb_busy, stages, metas);
        ++k;
        if (sig) {
          pend = true;
          pend_key = key;
        }
      }
      __syncwarp();
      // prefetch: descriptor kDescAhead items ahead, row runs / segments kMetaAhead items ahead
      if (!fenced && (m + kMetaAhead < nmine)) fence_proxy_async_smem();
      if (m + kDescAhead < nmine) req(m + kDescAhead);
      if (m + kMetaAhead < nmine) {
        const uint32_t q = m + kMetaAhead;
        const DevItem In = desc_ready(q);
        if (lane == 0) issue_meta<(kMask & kMaskLsu) != 0>(P, In, meta_of(q), &metab[q % kMetaSlots]);
      }
    }
    if (!ok) {
      // watchdog abort: descriptor / metadata copies still in flight land before the CTA leaves
      // (item m aborted before its own prefetches: requested so far are descriptors < m +
      // kDescAhead and metadata < m + kMetaAhead)
      for (uint32_t q = m; q < m + kDescAhead && q < nmine; ++q)
        mbar_wait(&descb[q % kDescSlots], (q / kDescSlots) & 1u);
      for (uint32_t q = m; q < m + kMetaAhead && q < nmine; ++q)
        mbar_wait(&metab[q % kMetaSlots], (q / kMetaSlots) & 1u);
    }
    if (kHelp) {  // release the helpers
      constexpr int kNB = 32 * (1 + DGCL_HELPER);
      if (mb_busy) named_sync(2, kNB);
      if (lane == 0) s_mb[2] = 1;
      __syncwarp();
      named_arrive(1, kNB);
      named_sync(2, kNB);
    }
    // END marker: consumers drain every issued stage, publish pending counts, then stop
    emit_marker(OP_END);
  } else {
    // ------------------------------- consumer warps ------------------------------------------
    const uint32_t tid = threadIdx.x - 32 * prod_warps, T = blockDim.x - 32 * prod_warps;
    const int cw = warp - prod_warps;
    for (uint32_t k = 0;; ++k) {
      uint32_t stage, use;
      ring_pos(k, NS, stage, use);
      mbar_wait(&full[stage], use & 1u);
      const uint8_t *st = stages + (size_t)stage * stage_bytes;
      const DevItem I = *reinterpret_cast<const DevItem *>(st);
      if (I.op == OP_END || I.op == OP_FLUSH) {
        // publish the rows stored since the last flush: every thread's stores and bulk stores
        // are visible system-wide before one release-add per (source, receiver).  (Every thread
        // waits for its own bulk groups: per-row, fan-out and atomic stores are issued by any
        // consumer lane, not only lane 0; the wait is a no-op for a thread with none pending.)
        bulk_wait_all();
        fence_proxy_async_global();
        fence_scope(P.sys_scope);
        consumer_barrier(&s_bar_count, &s_bar_gen, (unsigned)n_cons_warps, lane);
        // (strided: there are fewer consumer threads than (source, receiver) entries)
        for (uint32_t i = tid; i < (uint32_t)(kMaxRanks * kMaxRanks); i += T) {
          const uint32_t amt = s_pend[i];
          if (amt) {
            const int ex = (int)(i / kMaxRanks), dst = (int)(i % kMaxRanks);
            if (s_pend_base >= kMcCtrBase)  // multicast sends: every GPU's copy of ex's counter
              mc_publish(P, ex, amt);
            else
              red_release_add(P.flags[dst] + s_pend_base + ex, amt, P.sys_scope);
            s_pend[i] = 0;
          }
        }
        consumer_barrier(&s_bar_count, &s_bar_gen, (unsigned)n_cons_warps, lane);
        if (I.op == OP_END) break;
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[stage]);
        continue;
      }
      // kMask: the item kinds this instance was compiled for (the host picks the instance from
      // the launch's items, so e.g. a forward launch carries no fold code / registers)
      if ((kMask & kMaskCopy) && I.op == OP_COPY && !(I.flags & kItemDirect)) {
        const BufRef DB = P.buf[I.dst_kind][I.dst_rank];
        if ((kMask & kMaskLsu) && (I.flags & kItemLsu)) {  // rows gathered by every consumer
                                                            // thread, then stored as usual
          gather_lsu(P, I, const_cast<uint8_t *>(st), tid, T);
          consumer_barrier(&s_bar_count, &s_bar_gen, (unsigned)n_cons_warps, lane);
        }
        if (DGCL_DIAG_NO_STORE) {
        } else if ((kMask & kMaskMcast) && I.dst_kind == K_MCAST) {
          store_copy_mc(P, I, st, tid, T);
        } else if (I.flags & kItemAtomic) {
          store_copy_atomic(P, I, st, tid, T);
        } else if (P.bulk_store && I.dst >= 0 && DB.pitch == (int64_t)P.row16) {
          // consecutive packed destination rows: kStoreSplit bulk (TMA) stores move the item,
          // issued by consumer warps 0 .. kStoreSplit-1 (DGCL_STORE_FIXED; else rotating
          // (k * kStoreSplit + j) % n_cons_warps); the other warps move on
          const int split = kStoreSplit < n_cons_warps ? kStoreSplit : n_cons_warps;
          const int first =
              DGCL_STORE_FIXED ? 0 : (int)((k * (uint32_t)split) % (uint32_t)n_cons_warps);
          const int j = (cw - first + n_cons_warps) % n_cons_warps;
          // (DGCL_STG_SHARE > 0: the last share of the rows is stored by the other consumer warps
          // with LDS + STG, off the TMA unit)
          const int64_t rows_tma =
              DGCL_STG_SHARE && n_cons_warps > split ? (int64_t)I.rows * (100 - DGCL_STG_SHARE) / 100
                                                     : (int64_t)I.rows;
          if (j < split && lane == 0) {
            const int64_t lo = rows_tma * j / split;
            const int64_t hi = rows_tma * (j + 1) / split;
            if (hi > lo) {
              s2g(DB.ptr + (I.dst + lo) * DB.pitch, st + kStageHdrBytes + lo * P.row16,
                  (uint32_t)((hi - lo) * P.row16), pol_st);
              bulk_commit();
              bulk_wait_read();  // the stage may be reused once the bulk store has read it
            }
          } else if (DGCL_STG_SHARE && j >= split && rows_tma < I.rows) {
            const uint32_t nch = (uint32_t)P.n_chunks;
            const uint32_t t2 = (uint32_t)(j - split) * 32 + lane;
            const uint32_t T2 = (uint32_t)(n_cons_warps - split) * 32;
            const uint32_t e_end = (uint32_t)I.rows * nch;
            char *d0 = DB.ptr + I.dst * DB.pitch;
            const uint8_t *ops = st + kStageHdrBytes;
            for (uint32_t e = (uint32_t)rows_tma * nch + t2; e < e_end; e += T2) {
              const uint32_t r = fdiv(e, P);
              const uint32_t col = e - r * nch;
              st_v4(d0 + (int64_t)r * DB.pitch + col * 16, lds_v4(ops + r * P.row16 + col * 16));
            }
          }
        } else if (DGCL_ROW_BULK && P.bulk_store && I.dst < 0 && DB.pitch == (int64_t)P.row16 &&
                   P.row16 >= DGCL_ROW_BULK) {
          // scattered destination rows (relay stages): one bulk store per row, rows spread over
          // the consumer threads
          const int32_t *tab = reinterpret_cast<const int32_t *>(st + kTabDst) +
                               reinterpret_cast<const int32_t *>(st + kHdrInfo)[1];
          for (uint32_t r = tid; r < (uint32_t)I.rows; r += T)
            s2g(DB.ptr + (int64_t)tab[r] * DB.pitch, st + kStageHdrBytes + r * P.row16,
                (uint32_t)P.row16, pol_st);
          if (tid < (uint32_t)I.rows) {
            bulk_commit();
            bulk_wait_read();
          }
        } else {
          store_copy(P, I, st, tid, T);
        }
      } else if ((kMask & kMaskFanout) && I.op == OP_FANOUT) {
        store_fanout(P, I, st, tid, T, s_pend, pol_st);
        if ((I.flags & kItemSignal) && tid == 0) s_pend_base = I.sig_ctr - I.exec_rank;
      } else if ((kMask & kMaskDirect) && I.op == OP_COPY) {
        store_copy_direct(P, I, st, tid, T);
      } else if ((kMask & kMaskStaged) && is_staged(I)) {
        store_fold_staged(P, I, st, tid, T);
      } else if ((kMask & kMaskTree) && I.op == OP_FOLD && I.term_mode == kTermRankTree) {
        // (unstaged tree programs have their own kernel instance: the register stack would
        // crowd the other fold paths)
        store_fold_tree(P, I, st, tid, T);
      } else if ((kMask & kMaskFold) && I.op == OP_FOLD) {
        // many terms per row: batch a row's terms; few: batch across output chunks
        if (I.nterms >= 4 * I.rows)
          store_fold_rows<(kMaxThreads > 512 ? 4 : 8)>(P, I, st, tid, T);
        else
          store_fold_multi<(kMaxThreads > 512 ? 3 : 6)>(P, I, st, tid, T);
      }
      if (P.trace && tid == 0)  // this warp's share of the item is stored
        P.trace[reinterpret_cast<const int32_t *>(st + kHdrInfo)[2]].t_done = globaltimer();
      if ((I.flags & kItemSignal) && tid == 0 && I.op != OP_FANOUT) {
        // counted now, published by the next FLUSH / END marker (done flags)
        atomicAdd(&s_pend[I.exec_rank * kMaxRanks + I.dst_rank], (uint32_t)I.rows);
        s_pend_base = I.sig_ctr - I.exec_rank;
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[stage]);  // this warp is done reading the stage
    }
    bulk_wait_all();  // every thread's bulk stores complete before the CTA retires
  }
}

}  // namespace

namespace {

template <int kMask, int kThreads = 512>
int launch_mask(const ExecParams &p, int grid, int block, cudaStream_t s) {
  // kernel attributes are per device (context): set once per device this process launches on
  static unsigned long long attr_set = 0;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return (int)e;
  const unsigned long long bit = 1ull << (dev & 63);
  if (!(attr_set & bit)) {
    e = cudaFuncSetAttribute(executor_tma_kernel<kMask, kThreads>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemMax);
    if (e != cudaSuccess) return (int)e;
    attr_set |= bit;
  }
  const TmaGeometry g = {p.tma_stages, p.tma_buf, p.meta_bytes, block, 0, 0};
  executor_tma_kernel<kMask, kThreads><<<grid, block, tma_smem_bytes(g), s>>>(p);
  return (int)cudaGetLastError();
}

constexpr int kAll = kMaskCopy | kMaskFold | kMaskDirect | kMaskStaged | kMaskFanout | kMaskTree |
                     kMaskLsu | kMaskMcast;

}  // namespace

int launch_tma_executor(const ExecParams &p, int grid, int block, void *stream) {
  cudaStream_t s = (cudaStream_t)stream;
  switch (p.op_mask) {
    case kMaskCopy: return launch_mask<kMaskCopy>(p, grid, block, s);
    // forward with fan-out stage 1 (uniform plans), plus relay copies (relay plans)
    case kMaskFanout: return launch_mask<kMaskFanout>(p, grid, block, s);
    case kMaskFanout | kMaskCopy: return launch_mask<kMaskFanout | kMaskCopy>(p, grid, block, s);
    // loopback tree-order backward (relay plans): staged programs, plus unstaged ones
    case kMaskTree: return launch_mask<kMaskTree>(p, grid, block, s);
    case kMaskTree | kMaskStaged: return launch_mask<kMaskTree | kMaskStaged>(p, grid, block, s);
    case kMaskFold:
      // fold-only launches of unstaged folds are latency-bound gathers by the consumer warps:
      // the host may run them with 1024 threads (31 consumer warps, <= 64 registers) for twice
      // the loads in flight per SM (rows with many terms, WIDE geometry)
      if (block == 1024) return launch_mask<kMaskFold, 1024>(p, grid, 1024, s);
      return launch_mask<kMaskFold>(p, grid, block, s);
    case kMaskCopy | kMaskFold: return launch_mask<kMaskCopy | kMaskFold>(p, grid, block, s);
    // staged folds (backward reduce / partial-sum pushes with every operand row bulk-copied)
    case kMaskStaged: return launch_mask<kMaskStaged>(p, grid, block, s);
    case kMaskCopy | kMaskStaged: return launch_mask<kMaskCopy | kMaskStaged>(p, grid, block, s);
    default: return launch_mask<kAll>(p, grid, block, s);
  }
}

namespace {
template <int kMask, int kThreads = 512>
int occupancy_of(int block, size_t smem_bytes, int *ctas_per_sm) {
  cudaError_t e = cudaFuncSetAttribute(executor_tma_kernel<kMask, kThreads>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemMax);
  if (e == cudaSuccess)
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm,
                                                      executor_tma_kernel<kMask, kThreads>, block,
                                                      smem_bytes);
  return (int)e;
}
}  // namespace

// co-resident CTAs per SM (the persistent grid must be fully resident: CTAs wait on flags other
// CTAs set) of the instance launch_tma_executor picks for op_mask, or (op_mask < 0) of the
// worst-case instance — for launches that share the device with other programs' launches
int tma_executor_occupancy(int op_mask, int block, size_t smem_bytes, int *ctas_per_sm) {
  switch (op_mask) {
    case kMaskCopy: return occupancy_of<kMaskCopy>(block, smem_bytes, ctas_per_sm);
    case kMaskFanout: return occupancy_of<kMaskFanout>(block, smem_bytes, ctas_per_sm);
    case kMaskFanout | kMaskCopy:
      return occupancy_of<kMaskFanout | kMaskCopy>(block, smem_bytes, ctas_per_sm);
    case kMaskTree: return occupancy_of<kMaskTree>(block, smem_bytes, ctas_per_sm);
    case kMaskTree | kMaskStaged:
      return occupancy_of<kMaskTree | kMaskStaged>(block, smem_bytes, ctas_per_sm);
    case kMaskFold:
      if (block == 1024) return occupancy_of<kMaskFold, 1024>(1024, smem_bytes, ctas_per_sm);
      return occupancy_of<kMaskFold>(block, smem_bytes, ctas_per_sm);
    case kMaskCopy | kMaskFold:
      return occupancy_of<kMaskCopy | kMaskFold>(block, smem_bytes, ctas_per_sm);
    case kMaskStaged: return occupancy_of<kMaskStaged>(block, smem_bytes, ctas_per_sm);
    case kMaskCopy | kMaskStaged:
      return occupancy_of<kMaskCopy | kMaskStaged>(block, smem_bytes, ctas_per_sm);
    default: break;
  }
  int e = occupancy_of<kAll>(block == 1024 ? 512 : block, smem_bytes, ctas_per_sm);
  if (e != 0 || block != 1024) return e;
  return occupancy_of<kMaskFold, 1024>(1024, smem_bytes, ctas_per_sm);
}

}  // namespace dgcl
