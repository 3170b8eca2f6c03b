// executor.cu — the register-path (LDG/STG) plan executor and the launch entry points.
//
// PAPER.md: communication kernel that packs by send table and writes into the peer's buffer (§6.1
// P:1458-1462, §6.2), 16-byte packing, ready/done flags,
// non-atomic backward.  Design:
//   * one CTA works on one ITEM (a row range of one group) at a time; the item list is in stage
//     order and CTAs walk it round-robin (item = blockIdx.x + i * gridDim.x).  The grid is sized to
//     be co-resident (SMs x occupancy), so a CTA blocked on a stage-k wait never keeps a stage-(k-1)
//     item from running: deadlock-free without a host round-trip per stage;
//   * rows are copied as a flat (row, 16-B chunk) index space: consecutive threads move consecutive
//     16-B chunks, so loads from a gathered row and stores into the destination rows coalesce
//     whatever the dim; kUnroll independent 16-B loads per thread are in flight before the stores;
//   * user inputs (embeddings, halo gradients) are read with ld.global.nc.L1::no_allocate,
//     workspace rows written during the launch (halo / relay / slots) with ld.global.cg;
//   * stores go straight to the destination GPU's final row (a peer pointer over NVLink 5); after
//     an item every thread fences at system scope, then one thread adds the item's rows to the
//     receiver's monotonic counter with red.release.sys; waiters use ld.acquire.sys;
//   * the backward fold adds terms in list order with __fadd_rn (no FMA, no atomics).
// This path serves rows that are not 16-B aligned (4-byte variant) and is kept as the tma=0
// option; the default for aligned rows is the bulk-copy executor in executor_tma.cu.

#include "device_common.cuh"

namespace dgcl {

using namespace dev;

namespace {

constexpr int kMaxFoldPrefetch = 4;
#ifndef DGCL_REG_MINB
#define DGCL_REG_MINB 2  // 2 x 512 threads per SM (64 registers): twice the loads in flight
#endif
#ifndef DGCL_COPY_UNROLL
#define DGCL_COPY_UNROLL 2  // A/B on B200: 2 beat 4 and 8 (fewest spills at 64 registers per thread)
#endif
constexpr int kCopyUnroll = DGCL_COPY_UNROLL;  // 16-B loads in flight per thread (whole-chunk copies)

__device__ __forceinline__ const int32_t *idx_of(const ExecParams &P, int64_t enc) {
  return enc < 0 ? P.idx + ~enc : nullptr;
}

// ---- OP_COPY, 16-byte path ----------------------------------------------------------------
template <bool kNC>
__device__ __forceinline__ void copy_rows_v16(const ExecParams &P, const DevItem &I) {
  const char *sbase = P.buf[I.src_kind][I.exec_rank].ptr;
  const int64_t spitch = P.buf[I.src_kind][I.exec_rank].pitch;
  char *dbase = P.buf[I.dst_kind][I.dst_rank].ptr;
  const int64_t dpitch = P.buf[I.dst_kind][I.dst_rank].pitch;
  const int32_t *sidx = idx_of(P, I.src), *didx = idx_of(P, I.dst);
  const int64_t sb = I.src, db = I.dst;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  const int tail = P.row_bytes - (int)(nch - 1) * 16;  // bytes in each row's last chunk (1..16)
  const uint32_t T = blockDim.x;
#pragma unroll 1
  for (uint32_t e0 = threadIdx.x; e0 < total; e0 += T * kUnroll) {
    int4 v[kUnroll];
    char *dp[kUnroll];
    int nb[kUnroll];
#pragma unroll
    for (int j = 0; j < kUnroll; ++j) {
      const uint32_t e = e0 + j * T;
      nb[j] = 0;
      if (e < total) {
        const uint32_t r = fdiv(e, P);
        const uint32_t col = e - r * nch;
        const char *sp = sbase + row_of(sidx, sb, r) * spitch + (int64_t)col * 16;
        dp[j] = dbase + row_of(didx, db, r) * dpitch + (int64_t)col * 16;
        nb[j] = col + 1 == nch ? tail : 16;
        v[j] = nb[j] == 16 ? (kNC ? ld_nc_v4(sp) : ld_cg_v4(sp)) : ld_part<kNC>(sp, nb[j]);
      }
    }
#pragma unroll
    for (int j = 0; j < kUnroll; ++j) {
      if (nb[j] == 16)
        st_v4(dp[j], v[j]);
      else if (nb[j] > 0)
        st_part(dp[j], v[j], nb[j]);
    }
  }
}

// whole-chunk rows (row_bytes % 16 == 0): destinations kept as (row, chunk) 32-bit pairs instead
// of pointers until the store loop, so the kUnroll vectors in flight fit 64 registers unspilled
template <bool kNC>
__device__ __forceinline__ void copy_rows_full(const ExecParams &P, const DevItem &I) {
  const char *sbase = P.buf[I.src_kind][I.exec_rank].ptr;
  const int64_t spitch = P.buf[I.src_kind][I.exec_rank].pitch;
  char *dbase = P.buf[I.dst_kind][I.dst_rank].ptr;
  const int64_t dpitch = P.buf[I.dst_kind][I.dst_rank].pitch;
  const int32_t *sidx = idx_of(P, I.src), *didx = idx_of(P, I.dst);
  const int64_t sb = I.src, db = I.dst;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  const uint32_t T = blockDim.x;
#pragma unroll 1
  for (uint32_t e0 = threadIdx.x; e0 < total; e0 += T * kCopyUnroll) {
    int4 v[kCopyUnroll];
    int32_t drow[kCopyUnroll];
    uint32_t dcol[kCopyUnroll];
#pragma unroll
    for (int j = 0; j < kCopyUnroll; ++j) {
      const uint32_t e = e0 + j * T;
      drow[j] = -1;
      if (e < total) {
        const uint32_t r = fdiv(e, P);
        dcol[j] = e - r * nch;
        drow[j] = (int32_t)row_of(didx, db, r);
        const char *sp = sbase + row_of(sidx, sb, r) * spitch + (int64_t)dcol[j] * 16;
        v[j] = kNC ? ld_nc_v4(sp) : ld_cg_v4(sp);
      }
    }
#pragma unroll
    for (int j = 0; j < kCopyUnroll; ++j)
      if (drow[j] >= 0) st_v4(dbase + (int64_t)drow[j] * dpitch + (int64_t)dcol[j] * 16, v[j]);
  }
}

// ---- OP_COPY into the multicast region: every chunk once through the multicast address ----
__device__ __forceinline__ void copy_rows_mc(const ExecParams &P, const DevItem &I) {
  const char *sbase = P.buf[I.src_kind][I.exec_rank].ptr;
  const int64_t spitch = P.buf[I.src_kind][I.exec_rank].pitch;
  const int32_t *sidx = idx_of(P, I.src);
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  for (uint32_t e = threadIdx.x; e < total; e += blockDim.x) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    mc_store16(P, I.exec_rank, I.dst + r, col,
               ld_nc_v4(sbase + row_of(sidx, I.src, r) * spitch + (int64_t)col * 16));
  }
}

// ---- OP_COPY with atomic adds (ablation, option "atomic_backward"): one fp32 atomic per word --
__device__ __forceinline__ void copy_rows_atomic(const ExecParams &P, const DevItem &I) {
  const char *sbase = P.buf[I.src_kind][I.exec_rank].ptr;
  const int64_t spitch = P.buf[I.src_kind][I.exec_rank].pitch;
  char *dbase = P.buf[I.dst_kind][I.dst_rank].ptr;
  const int64_t dpitch = P.buf[I.dst_kind][I.dst_rank].pitch;
  const int32_t *sidx = idx_of(P, I.src), *didx = idx_of(P, I.dst);
  const uint32_t dim = (uint32_t)P.row_bytes / 4;
  const uint32_t total = (uint32_t)I.rows * dim;
  for (uint32_t e = threadIdx.x; e < total; e += blockDim.x) {
    const uint32_t r = e / dim, w = e - r * dim;
    const float v = *reinterpret_cast<const float *>(sbase + row_of(sidx, I.src, r) * spitch +
                                                     (int64_t)w * 4);
    atomicAdd(reinterpret_cast<float *>(dbase + row_of(didx, I.dst, r) * dpitch) + w, v);
  }
}

// ---- OP_COPY, 4-byte path (unaligned pitches) ---------------------------------------------
template <bool kNC>
__device__ __forceinline__ void copy_rows_b32(const ExecParams &P, const DevItem &I) {
  const char *sbase = P.buf[I.src_kind][I.exec_rank].ptr;
  const int64_t spitch = P.buf[I.src_kind][I.exec_rank].pitch;
  char *dbase = P.buf[I.dst_kind][I.dst_rank].ptr;
  const int64_t dpitch = P.buf[I.dst_kind][I.dst_rank].pitch;
  const int32_t *sidx = idx_of(P, I.src), *didx = idx_of(P, I.dst);
  const int64_t sb = I.src, db = I.dst;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  const uint32_t T = blockDim.x;
#pragma unroll 1
  for (uint32_t e0 = threadIdx.x; e0 < total; e0 += T * kUnroll) {
    int v[kUnroll];
    char *dp[kUnroll];
#pragma unroll
    for (int j = 0; j < kUnroll; ++j) {
      const uint32_t e = e0 + j * T;
      dp[j] = nullptr;
      if (e < total) {
        const uint32_t r = fdiv(e, P);
        const uint32_t col = e - r * nch;
        const char *sp = sbase + row_of(sidx, sb, r) * spitch + (int64_t)col * 4;
        dp[j] = dbase + row_of(didx, db, r) * dpitch + (int64_t)col * 4;
        v[j] = kNC ? ld_nc_b32(sp) : ld_cg_b32(sp);
      }
    }
#pragma unroll
    for (int j = 0; j < kUnroll; ++j)
      if (dp[j]) st_b32(dp[j], v[j]);
  }
}

// load 16 bytes (or the row's valid tail) of term row `term` at column chunk `col`
template <bool V16>
__device__ __forceinline__ int4 ld_term(const ExecParams &P, int exec, int mode, uint32_t term,
                                        uint32_t col, int nb) {
  const bool slot = mode == kTermLocal && (term & kTermSlot) != 0;
  const BufRef &B = mode == kTermRankHgrad ? P.buf[K_HGRAD][term >> 28]
                    : slot                 ? P.buf[K_SLOT][exec]
                                           : P.buf[K_HGRAD][exec];
  const uint32_t row = mode == kTermRankHgrad ? (term & kTermRowMask) : (term & ~kTermSlot);
  const char *p = B.ptr + (int64_t)row * B.pitch + (int64_t)col * (V16 ? 16 : 4);
  if (V16 && nb == 16) return slot ? ld_cg_v4(p) : ld_nc_v4(p);
  return slot ? ld_part<false>(p, V16 ? nb : 4) : ld_part<true>(p, V16 ? nb : 4);
}

// ---- OP_FOLD: dst = ((init + t0) + t1) + ... ----------------------------------------------
template <bool V16>
__device__ __forceinline__ void fold_rows(const ExecParams &P, const DevItem &I) {
  const BufRef D = P.buf[I.dst_kind][I.dst_rank];
  const int32_t *didx = idx_of(P, I.dst);
  const int64_t db = I.dst;
  const int64_t *tp = P.term_ptr + I.tp;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)I.rows * nch;
  const int tail = V16 ? P.row_bytes - (int)(nch - 1) * 16 : 4;
  const int exec = I.exec_rank, mode = I.term_mode;
  for (uint32_t e = threadIdx.x; e < total; e += blockDim.x) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    const int nb = V16 ? (col + 1 == nch ? tail : 16) : 4;
    char *dp = D.ptr + row_of(didx, db, r) * D.pitch + (int64_t)col * (V16 ? 16 : 4);
    if (mode == kTermRankTree) {  // loopback tree-order backward: postfix program per row
      const int64_t t0 = __ldg(tp + r), t1 = __ldg(tp + r + 1);
      const float4 acc = fold_tree(
          as_f4(V16 && nb == 16 ? ld_cg_v4(dp) : ld_part<false>(dp, V16 ? nb : 4)),
          P.terms + t0, (int)(t1 - t0), [&](uint32_t w) {
            const BufRef &B = P.buf[K_HGRAD][w >> 28];
            const char *p = B.ptr + (int64_t)(w & kTreeRowMask) * B.pitch +
                            (int64_t)col * (V16 ? 16 : 4);
            return as_f4(V16 && nb == 16 ? ld_nc_v4(p) : ld_part<true>(p, V16 ? nb : 4));
          });
      if (V16 && nb == 16)
        st_v4(dp, as_i4(acc));
      else
        st_part(dp, as_i4(acc), V16 ? nb : 4);
      continue;
    }
    int64_t t = __ldg(tp + r);
    const int64_t t1 = __ldg(tp + r + 1);
    float4 acc;
    if (I.fold_init) {
      acc = as_f4(V16 && nb == 16 ? ld_cg_v4(dp) : ld_part<false>(dp, V16 ? nb : 4));
    } else {
      acc = as_f4(ld_term<V16>(P, exec, mode, __ldg(P.terms + t), col, nb));
      ++t;
    }
    while (t < t1) {
      // issue up to kMaxFoldPrefetch independent loads, then add them in list order
      int4 buf[kMaxFoldPrefetch];
      const int n = (int)(t1 - t < kMaxFoldPrefetch ? t1 - t : kMaxFoldPrefetch);
#pragma unroll
      for (int j = 0; j < kMaxFoldPrefetch; ++j)
        if (j < n) buf[j] = ld_term<V16>(P, exec, mode, __ldg(P.terms + t + j), col, nb);
#pragma unroll
      for (int j = 0; j < kMaxFoldPrefetch; ++j)
        if (j < n) add4(acc, buf[j]);
      t += n;
    }
    const int4 out = as_i4(acc);
    if (V16 && nb == 16)
      st_v4(dp, out);
    else
      st_part(dp, out, V16 ? nb : 4);
  }
}

// ---- OP_FANOUT: flat (destination pair, chunk) space — each pair (dest word, source row) copies
// the source row into one receiver's row (halo / relay staging, library-owned: whole chunks) ----
template <bool V16>
__device__ __forceinline__ void fanout_rows(const ExecParams &P, const DevItem &I,
                                            uint32_t *s_cnt) {
  const BufRef S = P.buf[I.src_kind][I.exec_rank];
  const uint32_t *pw = P.terms + I.t0;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)(I.nterms >> 1) * nch;
  const bool sig = (I.flags & kItemSignal) != 0;
  for (uint32_t e = threadIdx.x; e < total; e += blockDim.x) {
    const uint32_t j = fdiv(e, P);
    const uint32_t col = e - j * nch;
    const uint32_t d = __ldg(pw + 2 * j), r = __ldg(pw + 2 * j + 1);
    const BufRef D = P.buf[(d & kFanRelay) ? K_RELAY : K_HALO][d >> 28];
    const char *sp = S.ptr + (int64_t)r * S.pitch;
    char *dp = D.ptr + (int64_t)(d & kFanRowMask) * D.pitch;
    if (V16)
      st_v4(dp + col * 16, ld_nc_v4(sp + col * 16));
    else
      st_part(dp + col * 4, ld_part<true>(sp + col * 4, 4), 4);
    if (sig && col == 0) atomicAdd(&s_cnt[d >> 28], 1u);
  }
}

// Done counts are published lazily: an item's (counter, rows) goes into a small per-CTA table, and
// the table is flushed (every thread fences at system scope, then one red.release.sys per counter)
// only before this CTA could block on a wait, when the table is full, and at the end.  A CTA never
// waits while holding unpublished counts, so the co-resident grid stays deadlock-free; a fence per
// item (a store drain every 64 KB) held the path at ~0.25 of HBM peak.
constexpr int kPendMax = 16;

// kCopy: the instance per launch kind — 0 general; for launches whose data items are all COPY
// (op_mask == kMaskCopy) 1 = whole 16-B chunks (or 4-B rows): no fold / fan-out / ragged-tail
// code, spill-free under the 64-register cap; 2 = ragged 16-B rows (e.g. dim 602: 2408 B) without
// the fold / fan-out code (the general instance spills far more there); 3 = fold-only launches
// (owner reduces, tree-order folds: no copy / fan-out code)
template <bool V16, int kCopy>
__global__ void __launch_bounds__(512, DGCL_REG_MINB) executor_kernel(const __grid_constant__ ExecParams P) {
  __shared__ int s_abort, s_flush, s_npend;
  __shared__ uint64_t *s_pend_ctr[kPendMax];
  __shared__ uint64_t s_pend_rows[kPendMax];
  __shared__ DevItem s_item;
  // per executing rank: the wait list last found satisfied (monotonic counters, fixed targets)
  __shared__ int32_t s_wait_ok[kMaxRanks];
  __shared__ uint32_t s_ready_ok;
  __shared__ uint32_t s_cnt[kMaxRanks];  // fan-out rows per receiver of the current item
  if (threadIdx.x < kMaxRanks) s_cnt[threadIdx.x] = 0;
  if (threadIdx.x < kMaxRanks) s_wait_ok[threadIdx.x] = -1;
  if (threadIdx.x == 0) s_ready_ok = 0, s_npend = 0;
  auto flush = [&]() {  // all threads: publish the pending done counts
    fence_scope(P.sys_scope);  // this thread's row stores are visible (peers: system-wide) ...
    __syncthreads();         // ... for every thread of the CTA ...
    if (threadIdx.x == 0) {  // ... before a receiver can observe the counts
      for (int i = 0; i < s_npend; ++i)
        release_rows(s_pend_ctr[i], s_pend_rows[i], true, P.sys_scope);
      s_npend = 0;
    }
    __syncthreads();
  };
  for (int it = blockIdx.x; it < P.n_items; it += gridDim.x) {
    if (threadIdx.x < 4)
      reinterpret_cast<int4 *>(&s_item)[threadIdx.x] =
          __ldg(reinterpret_cast<const int4 *>(P.items + it) + threadIdx.x);
    __syncthreads();
    const DevItem I = s_item;
    if (threadIdx.x == 0) {  // could this item block (an uncached wait)?  Or is the table full?
      bool may_block = s_npend == kPendMax;
      if (P.use_ready && I.ready_rank >= 0 && !((s_ready_ok >> I.ready_rank) & 1u))
        may_block = true;
      if (P.use_ready && I.ready_rank == kReadyAll)
        for (int s = 0; s < P.world; ++s)
          if (s != I.exec_rank && !((s_ready_ok >> s) & 1u)) may_block = true;
      if (I.wait_n > 0 && s_wait_ok[I.exec_rank] != I.wait_off) may_block = true;
      // (an item that signals nothing: publish the counts of the signalling items before it)
      if ((I.op == OP_COPY || I.op == OP_FOLD || I.op == OP_FANOUT) && !(I.flags & kItemSignal))
        may_block = true;
      s_flush = may_block && s_npend > 0;
    }
    __syncthreads();
    if (s_flush) flush();
    if (threadIdx.x == 0) {
      bool ok = true;
      if (P.trace) {
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        P.trace[it].t_start = globaltimer();
        P.trace[it].sm = smid;
        P.trace[it].tag = trace_tag(I, P.groups[I.group].stage, P.groups[I.group].block);
      }
      if (I.op == OP_READY) {
        // my buffers of every layer are free for this call: tell every peer
        for (int s = 0; s < P.world; ++s)
          if (s != I.exec_rank) st_release(P.flags[s] + kReadyBase + I.exec_rank, P.seq, P.sys_scope);
      }
      if (P.use_ready && I.ready_rank >= 0 && !((s_ready_ok >> I.ready_rank) & 1u)) {
        ok = wait_geq(P.flags[I.exec_rank] + kReadyBase + I.ready_rank, P.seq, P,
                      1000 + I.group);
        if (ok) s_ready_ok |= 1u << I.ready_rank;
      }
      if (P.use_ready && I.ready_rank == kReadyAll)  // fan-out: every receiver's buffers free
        for (int s = 0; s < P.world && ok; ++s)
          if (s != I.exec_rank && !((s_ready_ok >> s) & 1u)) {
            ok = wait_geq(P.flags[I.exec_rank] + kReadyBase + s, P.seq, P, 1000 + I.group);
            if (ok) s_ready_ok |= 1u << s;
          }
      if (ok && I.wait_n > 0 && s_wait_ok[I.exec_rank] != I.wait_off) {
        ok = wait_item_sources(P, I, 100000 + I.group);
        if (ok) s_wait_ok[I.exec_rank] = I.wait_off;
      }
      s_abort = ok ? 0 : 1;
      if (P.trace) P.trace[it].t_ready = globaltimer();
    }
    __syncthreads();
    if (s_abort) return;  // the watchdog fired; the error word is set, leave the launch
    if (kCopy == 3) {  // fold-only instance
      if (I.op == OP_FOLD) fold_rows<V16>(P, I);
    } else if (kCopy == 0 && I.op == OP_COPY && I.dst_kind == K_MCAST) {
      copy_rows_mc(P, I);
    } else if (I.op == OP_COPY && (I.flags & kItemAtomic)) {
      copy_rows_atomic(P, I);
    } else if (I.op == OP_COPY) {
      const bool nc = readonly_kind(I.src_kind);
      if (V16) {
        // the copy-only instance runs whole-chunk rows only (the ragged loop, inlined, made the
        // whole kernel spill at 64 registers)
        const bool full = kCopy == 1 || (kCopy == 0 && (P.row_bytes & 15) == 0);
        if (nc) full ? copy_rows_full<true>(P, I) : copy_rows_v16<true>(P, I);
        else full ? copy_rows_full<false>(P, I) : copy_rows_v16<false>(P, I);
      } else {
        if (nc) copy_rows_b32<true>(P, I);
        else copy_rows_b32<false>(P, I);
      }
    } else if (kCopy != 0) {
    } else if (I.op == OP_FOLD) {
      fold_rows<V16>(P, I);
    } else if (I.op == OP_FANOUT) {
      fanout_rows<V16>(P, I, s_cnt);
    }
    if (P.trace) {
      __syncthreads();
      if (threadIdx.x == 0) P.trace[it].t_done = globaltimer();
    }
    if (kCopy == 0 && (I.flags & kItemSignal) && I.dst_kind == K_MCAST) {  // multicast: at once
      fence_scope(1);
      __syncthreads();
      if (threadIdx.x == 0) mc_publish(P, I.exec_rank, (uint64_t)I.rows);
    } else if ((I.flags & kItemSignal) && I.op == OP_FANOUT) {
      fence_scope(P.sys_scope);
      __syncthreads();
      if (threadIdx.x < (unsigned)P.world && s_cnt[threadIdx.x]) {
        release_rows(P.flags[threadIdx.x] + I.sig_ctr, (uint64_t)s_cnt[threadIdx.x], true,
                     P.sys_scope);
        s_cnt[threadIdx.x] = 0;
      }
    } else if ((I.flags & kItemSignal) && threadIdx.x == 0) {  // deferred (see kPendMax)
      uint64_t *ctr = P.flags[I.dst_rank] + I.sig_ctr;
      int i = 0;
      while (i < s_npend && s_pend_ctr[i] != ctr) ++i;
      if (i == s_npend) s_pend_ctr[s_npend++] = ctr, s_pend_rows[i] = 0;
      s_pend_rows[i] += (uint64_t)I.rows;
    }
    __syncthreads();
  }
  if (s_npend > 0) flush();
}

// Device start barrier (timing protocol: every timed call starts when all ranks
// have arrived, so per-call times measure the exchange, not the ranks' launch skew).  Thread t
// plays rank first + t; the ranks of a per-rank loopback context are threads of one warp, whose
// spins make independent progress.
__global__ void barrier_kernel(const __grid_constant__ ExecParams P, int first, int count) {
  const int r = first + (int)threadIdx.x;
  if ((int)threadIdx.x >= count) return;
  for (int s = 0; s < P.world; ++s)
    if (s != r) st_release(P.flags[s] + kBarrierBase + r, P.seq, P.sys_scope);
  for (int s = 0; s < P.world; ++s)
    if (s != r && !wait_geq(P.flags[r] + kBarrierBase + s, P.seq, P, 3000000 + s)) return;
}

// Arrival wait: later work on the stream sees the rows counted by these counters (acquire).
__global__ void wait_kernel(const __grid_constant__ ExecParams P, int exec, int off, int n) {
  if (threadIdx.x != 0) return;
  for (int w = off; w < off + n; ++w) {
    const DevWait W = P.waits[w];
    if (!wait_geq(ctr_ptr(P, exec, W.ctr), P.epoch[DIR_FWD] * (uint64_t)W.amount, P, 4000000 + w))
      return;
  }
}

// multicast self-test: chunk i of the region = (i, i ^ 0x5a5a5a5a, ~i, 7) through the multicast
// address, then the flag word += 5 by one multimem reduction (release)
__global__ void mc_selftest_kernel(char *mc, uint64_t *mcflag, int n16) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n16) mm_st_v4(mc + (int64_t)i * 16, make_int4(i, i ^ 0x5a5a5a5a, ~i, 7));
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence_system();
    mm_red_release_add(mcflag, 5);
  }
}

}  // namespace

int launch_mc_selftest(void *mc, uint64_t *mcflag, int n16, void *stream) {
  mc_selftest_kernel<<<(n16 + 255) / 256, 256, 0, (cudaStream_t)stream>>>((char *)mc, mcflag, n16);
  return (int)cudaGetLastError();
}

int launch_wait(const ExecParams &p, int exec, int off, int n, void *stream) {
  wait_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(p, exec, off, n);
  return (int)cudaGetLastError();
}

int launch_barrier(const ExecParams &p, int first, int count, void *stream) {
  if (count <= 0) return 0;
  barrier_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(p, first, count);
  return (int)cudaGetLastError();
}

// executor_tma.cu
int launch_tma_executor(const ExecParams &p, int grid, int block, void *stream);
int tma_executor_occupancy(int op_mask, int block, size_t smem_bytes, int *ctas_per_sm);

int launch_executor(const ExecParams &p, int grid, int block, void *stream) {
  if (grid <= 0) return 0;
  if (p.use_tma) return launch_tma_executor(p, grid, block, stream);
  cudaStream_t s = (cudaStream_t)stream;
  // copy-only: every data item is a COPY (bulk-path or consumer-gather kind: the register path
  // runs both the same way); fold-only: no COPY of any kind and no FANOUT (the kCopy == 3
  // instance runs OP_FOLD items only, so a direct COPY must never reach it)
  // (multicast and lsu launches take the general instance, kMaskMcast / kMaskLsu)
  const int copies = kMaskCopy | kMaskDirect;
  const int folds = kMaskFold | kMaskStaged | kMaskTree;
  const bool copy_only = p.op_mask != 0 && (p.op_mask & ~copies) == 0;
  const bool whole = !p.vec16 || (p.row_bytes & 15) == 0;
  const bool fold_only = p.op_mask != 0 && (p.op_mask & ~folds) == 0;
  if (p.vec16 && copy_only && whole)
    executor_kernel<true, 1><<<grid, block, 0, s>>>(p);
  else if (p.vec16 && copy_only)
    executor_kernel<true, 2><<<grid, block, 0, s>>>(p);
  else if (p.vec16 && fold_only)
    executor_kernel<true, 3><<<grid, block, 0, s>>>(p);
  else if (p.vec16)
    executor_kernel<true, 0><<<grid, block, 0, s>>>(p);
  else if (copy_only)
    executor_kernel<false, 1><<<grid, block, 0, s>>>(p);
  else
    executor_kernel<false, 0><<<grid, block, 0, s>>>(p);
  return (int)cudaGetLastError();
}

int executor_tma_occupancy(int op_mask, int block, size_t smem_bytes, int *ctas_per_sm) {
  return tma_executor_occupancy(op_mask, block, smem_bytes, ctas_per_sm);
}

int executor_occupancy(int block, int *ctas_per_sm) {
  int a = 0, b = 0;
  cudaError_t ce = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, executor_kernel<true, 0>, block, 0);
  if (ce != cudaSuccess) return (int)ce;
  ce = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, executor_kernel<false, 0>, block, 0);
  if (ce != cudaSuccess) return (int)ce;
  *ctas_per_sm = a < b ? a : b;
  return 0;
}

}  // namespace dgcl
