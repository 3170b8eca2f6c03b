// executor.cu — the sm_100a plan executor: fused gather -> NVLink push, relay forwarding, backward
// partial-sum push and the fixed-order owner reduce, all in one persistent kernel per launch.
//
// PAPER.md: communication kernel that packs by send table and writes into the peer's buffer (§6.1
// P:1458-1462, §6.2), 16-byte packing, ready/done flags,
// non-atomic backward.  B200 design:
//   * one CTA works on one ITEM (a row range of one group) at a time; the item list is in stage
//     order and CTAs walk it round-robin (item = blockIdx.x + i * gridDim.x).  The grid is sized to
//     be co-resident (SMs x occupancy), so a CTA blocked on a stage-k wait never keeps a stage-(k-1)
//     item from running: deadlock-free without a host round-trip per stage;
//   * rows are copied as a flat (row, 16-B chunk) index space: consecutive threads move consecutive
//     16-B chunks, so loads from a gathered row and stores into the peer's contiguous halo rows are
//     coalesced whatever the dim; U independent 16-B loads per thread are in flight before stores;
//   * gathered user inputs (embeddings, halo gradients) are read with ld.global.nc.L1::no_allocate;
//     workspace rows written during the launch (halo / relay / slots) with ld.global.cg (L2);
//   * stores go straight to the destination GPU's final row (peer pointer over NVLink 5); after an
//     item, every thread fences at system scope, then one thread adds the item's rows to the
//     receiver's monotonic counter with red.release.sys; waiters use ld.acquire.sys;
//   * the backward fold adds terms in list order with __fadd_rn (no FMA contraction, no atomics).

#include <cuda_runtime.h>

#include <cstdint>

#include "internal.h"

namespace dgcl {

namespace {

constexpr int kUnroll = 4;
constexpr int kMaxFoldPrefetch = 4;

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_release_sys_add(uint64_t *p, uint64_t v) {
  asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ int4 ld_nc_v4(const void *p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ int4 ld_cg_v4(const void *p) {
  int4 r;
  asm volatile("ld.global.cg.v4.s32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ void st_v4(void *p, const int4 &v) {
  asm volatile("st.global.v4.s32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}
__device__ __forceinline__ int ld_nc_b32(const void *p) {
  int r;
  asm volatile("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ int ld_cg_b32(const void *p) {
  int r;
  asm volatile("ld.global.cg.b32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ void st_b32(void *p, int v) {
  asm volatile("st.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// partial 16-B chunk (the row's tail, nb in {4, 8, 12}): predicated 4-byte accesses, no local arrays
template <bool kNC>
__device__ __forceinline__ int4 ld_part(const char *p, int nb) {
  int4 r = make_int4(0, 0, 0, 0);
  r.x = kNC ? ld_nc_b32(p) : ld_cg_b32(p);
  if (nb > 4) r.y = kNC ? ld_nc_b32(p + 4) : ld_cg_b32(p + 4);
  if (nb > 8) r.z = kNC ? ld_nc_b32(p + 8) : ld_cg_b32(p + 8);
  return r;
}
__device__ __forceinline__ void st_part(char *p, const int4 &v, int nb) {
  st_b32(p, v.x);
  if (nb > 4) st_b32(p + 4, v.y);
  if (nb > 8) st_b32(p + 8, v.z);
}

// read-only user inputs (embeddings, halo gradients) take the non-coherent path
__device__ __forceinline__ bool readonly_kind(int kind) { return kind == K_EMB || kind == K_HGRAD; }

// Spin until *p >= target (acquire, system scope), bounded by the watchdog.
__device__ bool wait_geq(const uint64_t *p, uint64_t target, const ExecParams &P, int code) {
  if (ld_acquire_sys(p) >= target) return true;
  const uint64_t t0 = globaltimer();
  for (uint32_t it = 1;; ++it) {
    __nanosleep(64);
    if (ld_acquire_sys(p) >= target) return true;
    if ((it & 255) == 0) {
      if (*(volatile int *)P.err != 0) return false;  // another CTA/peer already failed
      if (globaltimer() - t0 > P.timeout_ns) {
        atomicCAS(P.err, 0, code);
        __threadfence_system();
        return false;
      }
    }
  }
}

__device__ __forceinline__ uint32_t fdiv(uint32_t x, const ExecParams &P) {
  return (__umulhi(x, P.div_mul) + x) >> P.div_shift;
}

__device__ __forceinline__ int64_t row_of(const int32_t *idx, int64_t base, int64_t i) {
  return idx ? (int64_t)__ldg(idx + i) : base + i;
}

// ---- OP_COPY, 16-byte path ----------------------------------------------------------------
template <bool kNC>
__device__ __forceinline__ void copy_rows_v16(const ExecParams &P, const DevGroup &G,
                                              int32_t rb, int32_t re) {
  const char *sbase = P.buf[G.src_kind][G.exec_rank].ptr;
  const int64_t spitch = P.buf[G.src_kind][G.exec_rank].pitch;
  char *dbase = P.buf[G.dst_kind][G.dst_rank].ptr;
  const int64_t dpitch = P.buf[G.dst_kind][G.dst_rank].pitch;
  const int32_t *sidx = G.src_idx >= 0 ? P.idx + G.src_idx + rb : nullptr;
  const int32_t *didx = G.dst_idx >= 0 ? P.idx + G.dst_idx + rb : nullptr;
  const int64_t sb = G.src_base + rb, db = G.dst_base + rb;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)(re - rb) * nch;
  const int tail = P.row_bytes - (int)(nch - 1) * 16;  // bytes in each row's last chunk (1..16)
  const uint32_t T = blockDim.x;
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

// ---- OP_COPY, 4-byte path (unaligned pitches) ---------------------------------------------
template <bool kNC>
__device__ __forceinline__ void copy_rows_b32(const ExecParams &P, const DevGroup &G,
                                              int32_t rb, int32_t re) {
  const char *sbase = P.buf[G.src_kind][G.exec_rank].ptr;
  const int64_t spitch = P.buf[G.src_kind][G.exec_rank].pitch;
  char *dbase = P.buf[G.dst_kind][G.dst_rank].ptr;
  const int64_t dpitch = P.buf[G.dst_kind][G.dst_rank].pitch;
  const int32_t *sidx = G.src_idx >= 0 ? P.idx + G.src_idx + rb : nullptr;
  const int32_t *didx = G.dst_idx >= 0 ? P.idx + G.dst_idx + rb : nullptr;
  const int64_t sb = G.src_base + rb, db = G.dst_base + rb;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)(re - rb) * nch;
  const uint32_t T = blockDim.x;
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

__device__ __forceinline__ float4 as_f4(const int4 &v) {
  return make_float4(__int_as_float(v.x), __int_as_float(v.y), __int_as_float(v.z),
                     __int_as_float(v.w));
}
__device__ __forceinline__ void add4(float4 &a, const int4 &b) {
  a.x = __fadd_rn(a.x, __int_as_float(b.x));
  a.y = __fadd_rn(a.y, __int_as_float(b.y));
  a.z = __fadd_rn(a.z, __int_as_float(b.z));
  a.w = __fadd_rn(a.w, __int_as_float(b.w));
}

// load 16 bytes (or the row's valid tail) of term row `term` at column chunk `col`
template <bool V16>
__device__ __forceinline__ int4 ld_term(const ExecParams &P, int exec, uint32_t term, uint32_t col,
                                        int nb) {
  const bool slot = (term & kTermSlot) != 0;
  const BufRef &B = slot ? P.buf[K_SLOT][exec] : P.buf[K_HGRAD][exec];
  const char *p = B.ptr + (int64_t)(term & ~kTermSlot) * B.pitch + (int64_t)col * (V16 ? 16 : 4);
  if (V16 && nb == 16) return slot ? ld_cg_v4(p) : ld_nc_v4(p);
  return slot ? ld_part<false>(p, V16 ? nb : 4) : ld_part<true>(p, V16 ? nb : 4);
}

// ---- OP_FOLD: dst = ((init + t0) + t1) + ... ----------------------------------------------
template <bool V16>
__device__ __forceinline__ void fold_rows(const ExecParams &P, const DevGroup &G, int32_t rb,
                                          int32_t re) {
  const BufRef D = P.buf[G.dst_kind][G.dst_rank];
  const int32_t *didx = G.dst_idx >= 0 ? P.idx + G.dst_idx + rb : nullptr;
  const int64_t db = G.dst_base + rb;
  const int64_t *tp = P.term_ptr + G.term_ptr + rb;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t total = (uint32_t)(re - rb) * nch;
  const int tail = V16 ? P.row_bytes - (int)(nch - 1) * 16 : 4;
  const int exec = G.exec_rank;
  for (uint32_t e = threadIdx.x; e < total; e += blockDim.x) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    const int nb = V16 ? (col + 1 == nch ? tail : 16) : 4;
    char *dp = D.ptr + row_of(didx, db, r) * D.pitch + (int64_t)col * (V16 ? 16 : 4);
    int64_t t = __ldg(tp + r);
    const int64_t t1 = __ldg(tp + r + 1);
    float4 acc;
    if (G.fold_init) {
      acc = as_f4(V16 && nb == 16 ? ld_cg_v4(dp) : ld_part<false>(dp, V16 ? nb : 4));
    } else {
      acc = as_f4(ld_term<V16>(P, exec, __ldg(P.terms + t), col, nb));
      ++t;
    }
    while (t < t1) {
      // issue up to kMaxFoldPrefetch independent loads, then add them in list order
      int4 buf[kMaxFoldPrefetch];
      const int n = (int)(t1 - t < kMaxFoldPrefetch ? t1 - t : kMaxFoldPrefetch);
#pragma unroll
      for (int j = 0; j < kMaxFoldPrefetch; ++j)
        if (j < n) buf[j] = ld_term<V16>(P, exec, __ldg(P.terms + t + j), col, nb);
#pragma unroll
      for (int j = 0; j < kMaxFoldPrefetch; ++j)
        if (j < n) add4(acc, buf[j]);
      t += n;
    }
    const int4 out = make_int4(__float_as_int(acc.x), __float_as_int(acc.y), __float_as_int(acc.z),
                               __float_as_int(acc.w));
    if (V16 && nb == 16)
      st_v4(dp, out);
    else
      st_part(dp, out, V16 ? nb : 4);
  }
}

template <bool V16>
__global__ void __launch_bounds__(512, 1) executor_kernel(const __grid_constant__ ExecParams P) {
  __shared__ int s_abort;
  for (int it = blockIdx.x; it < P.n_items; it += gridDim.x) {
    const DevItem item = P.items[it];
    const DevGroup &G = P.groups[item.group];
    if (threadIdx.x == 0) {
      bool ok = true;
      const int op = G.op;
      if (op == OP_READY) {
        // my buffers of every layer are free for this call: tell every peer
        for (int s = 0; s < P.world; ++s)
          if (s != G.exec_rank) st_release_sys(P.flags[s] + kReadyBase + G.exec_rank, P.seq);
      }
      if (P.use_ready && G.ready_rank >= 0)
        ok = wait_geq(P.flags[G.exec_rank] + kReadyBase + G.ready_rank, P.seq, P,
                      1000 + item.group);
      for (int w = 0; ok && w < G.wait_n; ++w) {
        const DevWait W = P.waits[G.wait_off + w];
        ok = wait_geq(P.flags[G.exec_rank] + W.ctr, P.epoch[G.dir] * (uint64_t)W.amount, P,
                      100000 + item.group);
      }
      s_abort = ok ? 0 : 1;
    }
    __syncthreads();
    if (s_abort) return;  // the watchdog fired; the error word is set, leave the launch
    if (G.op == OP_COPY) {
      const bool nc = readonly_kind(G.src_kind);
      if (V16) {
        if (nc) copy_rows_v16<true>(P, G, item.row_begin, item.row_end);
        else copy_rows_v16<false>(P, G, item.row_begin, item.row_end);
      } else {
        if (nc) copy_rows_b32<true>(P, G, item.row_begin, item.row_end);
        else copy_rows_b32<false>(P, G, item.row_begin, item.row_end);
      }
    } else if (G.op == OP_FOLD) {
      fold_rows<V16>(P, G, item.row_begin, item.row_end);
    }
    if (item.flags & kItemSignal) {
      __threadfence_system();  // this thread's row stores are visible system-wide ...
      __syncthreads();         // ... for every thread of the CTA ...
      if (threadIdx.x == 0)    // ... before the receiver can observe the count (done flag)
        red_release_sys_add(P.flags[G.dst_rank] + G.sig_ctr,
                            (uint64_t)(item.row_end - item.row_begin));
    }
    __syncthreads();
  }
}


// =============================================================================================
// Bulk-copy (TMA) executor: thread 0 gathers every source row of an item into shared memory
// with cp.async.bulk (one instruction per row, completion counted on an mbarrier), while all
// threads store the PREVIOUS item from the other shared-memory stage with coalesced 16-B stores
// (to a peer over NVLink or to local HBM).  Two 96 KB stages per CTA keep ~96 KB of gathers in
// flight per SM without spending registers on them.
// =============================================================================================

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
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
        " selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(smem_u32(b)), "r"(parity)
        : "memory");
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
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async;" ::: "memory");
}
__device__ __forceinline__ int4 lds_v4(const uint8_t *p) {
  return *reinterpret_cast<const int4 *>(p);
}

__device__ __forceinline__ bool is_data_op(int op) { return op == OP_COPY || op == OP_FOLD; }

// non-blocking: are all counter waits of G already satisfied?
__device__ __forceinline__ bool waits_ready(const ExecParams &P, const DevGroup &G) {
  for (int w = 0; w < G.wait_n; ++w) {
    const DevWait W = P.waits[G.wait_off + w];
    if (ld_acquire_sys(P.flags[G.exec_rank] + W.ctr) < P.epoch[G.dir] * (uint64_t)W.amount)
      return false;
  }
  return true;
}

// thread 0: gather the item's source rows (COPY) or fold operands (FOLD) into `buf`
__device__ void issue_item_loads(const ExecParams &P, const DevGroup &G, const DevItem &item,
                                 uint8_t *buf, uint64_t *bar) {
  fence_proxy_async();  // order earlier generic accesses (acquires, smem reads) before the bulk copies
  const int32_t rb = item.row_begin;
  const int rows = item.row_end - rb;
  const uint32_t r16 = (uint32_t)P.row16;
  if (G.op == OP_COPY) {
    const char *sbase = P.buf[G.src_kind][G.exec_rank].ptr;
    const int64_t spitch = P.buf[G.src_kind][G.exec_rank].pitch;
    const int32_t *sidx = G.src_idx >= 0 ? P.idx + G.src_idx + rb : nullptr;
    const int64_t sb = G.src_base + rb;
    mbar_expect_tx(bar, (uint32_t)rows * r16);
    for (int r = 0; r < rows; ++r)
      bulk_g2s(buf + (size_t)r * r16, sbase + row_of(sidx, sb, r) * spitch, r16, bar);
  } else {
    const int64_t *tp = P.term_ptr + G.term_ptr + rb;
    const int init = G.fold_init;
    const int64_t t0 = tp[0];
    const uint32_t nslots = (uint32_t)(tp[rows] - t0) + (init ? rows : 0);
    mbar_expect_tx(bar, nslots * r16);
    const BufRef D = P.buf[G.dst_kind][G.dst_rank];
    const int32_t *didx = G.dst_idx >= 0 ? P.idx + G.dst_idx + rb : nullptr;
    const int64_t db = G.dst_base + rb;
    const BufRef SL = P.buf[K_SLOT][G.exec_rank];
    const BufRef HG = P.buf[K_HGRAD][G.exec_rank];
    uint32_t slot = 0;
    for (int r = 0; r < rows; ++r) {
      if (init)
        bulk_g2s(buf + (size_t)(slot++) * r16, D.ptr + row_of(didx, db, r) * D.pitch, r16, bar);
      for (int64_t t = tp[r]; t < tp[r + 1]; ++t) {
        const uint32_t term = P.terms[t];
        const BufRef &B = (term & kTermSlot) ? SL : HG;
        bulk_g2s(buf + (size_t)(slot++) * r16, B.ptr + (int64_t)(term & ~kTermSlot) * B.pitch,
                 r16, bar);
      }
    }
  }
}

// all threads: store a gathered COPY item from shared memory
__device__ __forceinline__ void store_copy_item(const ExecParams &P, const DevGroup &G,
                                                const DevItem &item, const uint8_t *buf) {
  char *dbase = P.buf[G.dst_kind][G.dst_rank].ptr;
  const int64_t dpitch = P.buf[G.dst_kind][G.dst_rank].pitch;
  const int32_t rb = item.row_begin;
  const int32_t *didx = G.dst_idx >= 0 ? P.idx + G.dst_idx + rb : nullptr;
  const int64_t db = G.dst_base + rb;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t r16 = (uint32_t)P.row16;
  const uint32_t total = (uint32_t)(item.row_end - rb) * nch;
  const uint32_t T = blockDim.x;
  if (!didx) {
    // contiguous destination rows: the item is one strided 2-D block
    for (uint32_t e0 = threadIdx.x; e0 < total; e0 += T * kUnroll) {
#pragma unroll
      for (int j = 0; j < kUnroll; ++j) {
        const uint32_t e = e0 + j * T;
        if (e < total) {
          const uint32_t r = fdiv(e, P);
          const uint32_t col = e - r * nch;
          st_v4(dbase + (db + r) * dpitch + (int64_t)col * 16, lds_v4(buf + r * r16 + col * 16));
        }
      }
    }
  } else {
    for (uint32_t e0 = threadIdx.x; e0 < total; e0 += T * kUnroll) {
#pragma unroll
      for (int j = 0; j < kUnroll; ++j) {
        const uint32_t e = e0 + j * T;
        if (e < total) {
          const uint32_t r = fdiv(e, P);
          const uint32_t col = e - r * nch;
          st_v4(dbase + (int64_t)__ldg(didx + r) * dpitch + (int64_t)col * 16,
                lds_v4(buf + r * r16 + col * 16));
        }
      }
    }
  }
}

// all threads: fold a gathered FOLD item from shared memory, in list order, and store it
__device__ __forceinline__ void fold_item_smem(const ExecParams &P, const DevGroup &G,
                                               const DevItem &item, const uint8_t *buf) {
  const BufRef D = P.buf[G.dst_kind][G.dst_rank];
  const int32_t rb = item.row_begin;
  const int32_t *didx = G.dst_idx >= 0 ? P.idx + G.dst_idx + rb : nullptr;
  const int64_t db = G.dst_base + rb;
  const int64_t *tp = P.term_ptr + G.term_ptr + rb;
  const int64_t t0 = __ldg(tp);
  const int init = G.fold_init;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t r16 = (uint32_t)P.row16;
  const uint32_t total = (uint32_t)(item.row_end - rb) * nch;
  const int tail = P.row_bytes - (int)(nch - 1) * 16;
  for (uint32_t e = threadIdx.x; e < total; e += blockDim.x) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    const int64_t ta = __ldg(tp + r), tb = __ldg(tp + r + 1);
    const uint32_t base = (uint32_t)(ta - t0) + (init ? r : 0);
    const uint32_t cnt = (uint32_t)(tb - ta) + (init ? 1 : 0);
    const uint8_t *p = buf + (size_t)base * r16 + col * 16;
    float4 acc = as_f4(lds_v4(p));
    for (uint32_t j = 1; j < cnt; ++j) add4(acc, lds_v4(p + (size_t)j * r16));
    const int4 out = make_int4(__float_as_int(acc.x), __float_as_int(acc.y),
                               __float_as_int(acc.z), __float_as_int(acc.w));
    char *dp = D.ptr + row_of(didx, db, r) * D.pitch + (int64_t)col * 16;
    const int nb = col + 1 == nch ? tail : 16;
    if (nb == 16)
      st_v4(dp, out);
    else
      st_part(dp, out, nb);
  }
}

__global__ void __launch_bounds__(512, 1) executor_tma_kernel(const __grid_constant__ ExecParams P) {
  extern __shared__ __align__(128) uint8_t dsmem[];
  uint64_t *bars = reinterpret_cast<uint64_t *>(dsmem);
  uint8_t *bufs = dsmem + 128;
  __shared__ int s_abort, s_issued;
  if (threadIdx.x == 0) {
    mbar_init(&bars[0], 1);
    mbar_init(&bars[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  uint32_t phase[2] = {0u, 0u};
  int prefetched = -1;  // thread 0 only: the item whose loads are already in flight
  int k = 0;
  for (int it = blockIdx.x; it < P.n_items; it += gridDim.x, ++k) {
    const int slot = k & 1;
    uint8_t *buf = bufs + (size_t)slot * P.tma_buf;
    const DevItem item = P.items[it];
    const DevGroup &G = P.groups[item.group];
    if (threadIdx.x == 0) {
      bool ok = true;
      int issued = 0;
      const int op = G.op;
      if (op == OP_READY) {
        for (int s = 0; s < P.world; ++s)
          if (s != G.exec_rank) st_release_sys(P.flags[s] + kReadyBase + G.exec_rank, P.seq);
      }
      if (prefetched == it) {
        issued = 1;
      } else {
        for (int w = 0; ok && w < G.wait_n; ++w) {
          const DevWait W = P.waits[G.wait_off + w];
          ok = wait_geq(P.flags[G.exec_rank] + W.ctr, P.epoch[G.dir] * (uint64_t)W.amount, P,
                        100000 + item.group);
        }
        if (ok && is_data_op(op)) {
          issue_item_loads(P, G, item, buf, &bars[slot]);
          issued = 1;
        }
      }
      if (ok && P.use_ready && G.ready_rank >= 0)
        ok = wait_geq(P.flags[G.exec_rank] + kReadyBase + G.ready_rank, P.seq, P,
                      1000 + item.group);
      // prefetch this CTA's next item into the other stage if its sources are final already
      const int nxt = it + gridDim.x;
      if (ok && nxt < P.n_items) {
        const DevItem ni = P.items[nxt];
        const DevGroup &NG = P.groups[ni.group];
        if (is_data_op(NG.op) && waits_ready(P, NG)) {
          issue_item_loads(P, NG, ni, bufs + (size_t)(slot ^ 1) * P.tma_buf, &bars[slot ^ 1]);
          prefetched = nxt;
        }
      }
      s_abort = ok ? 0 : 1;
      s_issued = issued;
    }
    __syncthreads();
    if (s_abort) {
      // drain bulk copies that target this CTA's shared memory before leaving
      if (s_issued) mbar_wait(&bars[slot], phase[slot]);
      if (threadIdx.x == 0 && prefetched == it + (int)gridDim.x)
        mbar_wait(&bars[slot ^ 1], phase[slot ^ 1]);
      __syncthreads();
      return;
    }
    if (is_data_op(G.op)) {
      mbar_wait(&bars[slot], phase[slot]);
      phase[slot] ^= 1u;
      if (G.op == OP_COPY)
        store_copy_item(P, G, item, buf);
      else
        fold_item_smem(P, G, item, buf);
    }
    if (item.flags & kItemSignal) {
      __threadfence_system();
      __syncthreads();
      if (threadIdx.x == 0)
        red_release_sys_add(P.flags[G.dst_rank] + G.sig_ctr,
                            (uint64_t)(item.row_end - item.row_begin));
    }
    __syncthreads();
  }
}

}  // namespace

constexpr size_t kTmaSmem = 128 + 2 * (size_t)kTmaBufBytes;

int launch_executor(const ExecParams &p, int grid, int block, void *stream) {
  if (grid <= 0) return 0;
  cudaStream_t s = (cudaStream_t)stream;
  if (p.use_tma) {
    static bool attr = false;
    if (!attr) {
      cudaError_t e = cudaFuncSetAttribute(executor_tma_kernel,
                                           cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           (int)kTmaSmem);
      if (e != cudaSuccess) return (int)e;
      attr = true;
    }
    executor_tma_kernel<<<grid, block, kTmaSmem, s>>>(p);
  } else if (p.vec16)
    executor_kernel<true><<<grid, block, 0, s>>>(p);
  else
    executor_kernel<false><<<grid, block, 0, s>>>(p);
  return (int)cudaGetLastError();
}

int executor_occupancy(int block, int *ctas_per_sm, int *tma_ctas_per_sm) {
  int a = 0, b = 0, t = 0;
  cudaError_t et = cudaFuncSetAttribute(executor_tma_kernel,
                                        cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTmaSmem);
  if (et != cudaSuccess) return (int)et;
  et = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&t, executor_tma_kernel, block, kTmaSmem);
  if (et != cudaSuccess) return (int)et;
  *tma_ctas_per_sm = t;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, executor_kernel<true>, block, 0);
  if (e != cudaSuccess) return (int)e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, executor_kernel<false>, block, 0);
  if (e != cudaSuccess) return (int)e;
  *ctas_per_sm = a < b ? a : b;
  return 0;
}

}  // namespace dgcl
