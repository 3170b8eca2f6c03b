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

}  // namespace

int launch_executor(const ExecParams &p, int grid, int block, void *stream) {
  if (grid <= 0) return 0;
  cudaStream_t s = (cudaStream_t)stream;
  if (p.vec16)
    executor_kernel<true><<<grid, block, 0, s>>>(p);
  else
    executor_kernel<false><<<grid, block, 0, s>>>(p);
  return (int)cudaGetLastError();
}

int executor_occupancy(int block, int *ctas_per_sm) {
  int a = 0, b = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, executor_kernel<true>, block, 0);
  if (e != cudaSuccess) return (int)e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, executor_kernel<false>, block, 0);
  if (e != cudaSuccess) return (int)e;
  *ctas_per_sm = a < b ? a : b;
  return 0;
}

}  // namespace dgcl
