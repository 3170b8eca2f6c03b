// executor_tma.cu — the bulk-copy (TMA) plan executor, warp-specialised (sm_100a).
//
// Same semantics as executor.cu (groups / items / counters, see internal.h), different data
// movement.  PAPER.md §6.1-6.2: the sender packs rows by its send table and writes
// them into the receiver's buffer; here the "pack" is a gather of whole rows into shared memory by
// the Tensor Memory Accelerator, and the "send" is a coalesced 16-B store stream from shared
// memory to the destination rows (a peer's halo over NVLink 5, or local HBM in loopback).
//
// Per CTA (one per SM, 512 threads, 4 x 48 KB shared-memory stages):
//   warp 0 (producer): walks the CTA's items in order; for each data item it resolves the item's
//     source waits (stage chaining, acquire on the receiver-side counters), waits for a free stage
//     (mbarrier "empty"), arms the stage's "full" mbarrier with the item's byte count and issues one
//     cp.async.bulk per gathered row (lanes issue rows lane, lane+32, ...);
//   warps 1-15 (consumers): wait for the stage to fill, store (COPY) or fold-and-store (FOLD) from
//     shared memory, publish the item (fence.sys + red.release.sys on the receiver's counter) and
//     release the stage.
// Up to 4 items (192 KB) of gathers are in flight per SM while the consumers drain older ones, so
// HBM / NVLink latency is hidden without holding data in registers.

#include "device_common.cuh"

namespace dgcl {

using namespace dev;

namespace {

constexpr int kStages = 4;
constexpr int kStageBytes = kTmaBufBytes;
constexpr size_t kSmemBytes = 128 + (size_t)kStages * kStageBytes;

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
// wait for phase `parity` of barrier b; gives up (returns false) once *abort is set
__device__ __forceinline__ bool mbar_wait(uint64_t *b, uint32_t parity, volatile int *abort) {
  for (uint32_t it = 0;; ++it) {
    if (mbar_test(b, parity)) return true;
    if ((it & 63) == 63 && *abort) return false;
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
// Barrier over the consumer warps that gives up once *abort is set (a hardware bar.sync could
// hang forever if some consumer left on a watchdog abort).  Returns false on abort.
__device__ __forceinline__ bool consumer_barrier(unsigned *count, volatile unsigned *gen,
                                                 unsigned nwarps, volatile int *abort, int lane) {
  __syncwarp();
  int ok = 1;
  if (lane == 0) {
    const unsigned g = *gen;
    __threadfence_block();
    if (atomicAdd(count, 1u) == nwarps - 1) {
      *count = 0;
      __threadfence_block();
      atomicAdd((unsigned *)gen, 1u);
    } else {
      while (*gen == g) {
        if (*abort) {
          ok = 0;
          break;
        }
      }
    }
    __threadfence_block();
  }
  ok = __shfl_sync(0xffffffffu, ok, 0);
  return ok != 0;
}
__device__ __forceinline__ int4 lds_v4(const uint8_t *p) {
  return *reinterpret_cast<const int4 *>(p);
}
__device__ __forceinline__ bool is_data_op(int op) { return op == OP_COPY || op == OP_FOLD; }

// bytes of gathered operands of a data item (must equal the sum of the bulk copies issued)
__device__ __forceinline__ uint32_t item_bytes(const ExecParams &P, const DevGroup &G,
                                               const DevItem &it) {
  const int rows = it.row_end - it.row_begin;
  if (G.op == OP_COPY) return (uint32_t)rows * (uint32_t)P.row16;
  const int64_t *tp = P.term_ptr + G.term_ptr + it.row_begin;
  return ((uint32_t)(tp[rows] - tp[0]) + (G.fold_init ? rows : 0)) * (uint32_t)P.row16;
}

// producer lanes: gather the item's rows into `buf` (lane handles rows lane, lane + 32, ...)
__device__ __forceinline__ void issue_rows(const ExecParams &P, const DevGroup &G,
                                           const DevItem &item, uint8_t *buf, uint64_t *bar,
                                           int lane) {
  const int32_t rb = item.row_begin;
  const int rows = item.row_end - rb;
  const uint32_t r16 = (uint32_t)P.row16;
  if (G.op == OP_COPY) {
    const char *sbase = P.buf[G.src_kind][G.exec_rank].ptr;
    const int64_t spitch = P.buf[G.src_kind][G.exec_rank].pitch;
    const int32_t *sidx = G.src_idx >= 0 ? P.idx + G.src_idx + rb : nullptr;
    const int64_t sb = G.src_base + rb;
    for (int r = lane; r < rows; r += 32)
      bulk_g2s(buf + (size_t)r * r16, sbase + row_of(sidx, sb, r) * spitch, r16, bar);
  } else {
    const int64_t *tp = P.term_ptr + G.term_ptr + rb;
    const int init = G.fold_init;
    const int64_t t0 = __ldg(tp);
    const BufRef D = P.buf[G.dst_kind][G.dst_rank];
    const int32_t *didx = G.dst_idx >= 0 ? P.idx + G.dst_idx + rb : nullptr;
    const int64_t db = G.dst_base + rb;
    const BufRef SL = P.buf[K_SLOT][G.exec_rank];
    const BufRef HG = P.buf[K_HGRAD][G.exec_rank];
    for (int r = lane; r < rows; r += 32) {
      const int64_t ta = __ldg(tp + r), tb = __ldg(tp + r + 1);
      uint32_t slot = (uint32_t)(ta - t0) + (init ? r : 0);
      if (init)
        bulk_g2s(buf + (size_t)(slot++) * r16, D.ptr + row_of(didx, db, r) * D.pitch, r16, bar);
      for (int64_t t = ta; t < tb; ++t) {
        const uint32_t term = __ldg(P.terms + t);
        const BufRef &B = (term & kTermSlot) ? SL : HG;
        bulk_g2s(buf + (size_t)(slot++) * r16, B.ptr + (int64_t)(term & ~kTermSlot) * B.pitch,
                 r16, bar);
      }
    }
  }
}

// consumers: store a gathered COPY item from shared memory (whole 16-B chunks: the destinations
// are library-owned rows whose pitch covers the rounded-up row)
__device__ __forceinline__ void store_copy(const ExecParams &P, const DevGroup &G,
                                           const DevItem &item, const uint8_t *buf, uint32_t tid,
                                           uint32_t T) {
  char *dbase = P.buf[G.dst_kind][G.dst_rank].ptr;
  const int64_t dpitch = P.buf[G.dst_kind][G.dst_rank].pitch;
  const int32_t rb = item.row_begin;
  const int32_t *didx = G.dst_idx >= 0 ? P.idx + G.dst_idx + rb : nullptr;
  const int64_t db = G.dst_base + rb;
  const uint32_t nch = (uint32_t)P.n_chunks;
  const uint32_t r16 = (uint32_t)P.row16;
  const uint32_t total = (uint32_t)(item.row_end - rb) * nch;
  for (uint32_t e0 = tid; e0 < total; e0 += T * kUnroll) {
#pragma unroll
    for (int j = 0; j < kUnroll; ++j) {
      const uint32_t e = e0 + j * T;
      if (e < total) {
        const uint32_t r = fdiv(e, P);
        const uint32_t col = e - r * nch;
        st_v4(dbase + row_of(didx, db, r) * dpitch + (int64_t)col * 16,
              lds_v4(buf + r * r16 + col * 16));
      }
    }
  }
}

// consumers: fold a gathered FOLD item from shared memory, operands in list order, and store it
// (the row's last chunk is stored partially: the destination may be the caller's emb_grad)
__device__ __forceinline__ void store_fold(const ExecParams &P, const DevGroup &G,
                                           const DevItem &item, const uint8_t *buf, uint32_t tid,
                                           uint32_t T) {
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
  for (uint32_t e = tid; e < total; e += T) {
    const uint32_t r = fdiv(e, P);
    const uint32_t col = e - r * nch;
    const int64_t ta = __ldg(tp + r), tb = __ldg(tp + r + 1);
    const uint32_t base = (uint32_t)(ta - t0) + (init ? r : 0);
    const uint32_t cnt = (uint32_t)(tb - ta) + (init ? 1 : 0);
    const uint8_t *p = buf + (size_t)base * r16 + col * 16;
    float4 acc = as_f4(lds_v4(p));
    for (uint32_t j = 1; j < cnt; ++j) add4(acc, lds_v4(p + (size_t)j * r16));
    char *dp = D.ptr + row_of(didx, db, r) * D.pitch + (int64_t)col * 16;
    const int nb = col + 1 == nch ? tail : 16;
    if (nb == 16)
      st_v4(dp, as_i4(acc));
    else
      st_part(dp, as_i4(acc), nb);
  }
}

__global__ void __launch_bounds__(512, 1)
    executor_tma_kernel(const __grid_constant__ ExecParams P) {
  extern __shared__ __align__(128) uint8_t dsmem[];
  uint64_t *full = reinterpret_cast<uint64_t *>(dsmem);
  uint64_t *empty = full + kStages;
  uint8_t *bufs = dsmem + 128;
  __shared__ volatile int s_abort;
  __shared__ unsigned s_bar_count;
  __shared__ volatile unsigned s_bar_gen;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n_cons_warps = (int)(blockDim.x >> 5) - 1;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], n_cons_warps);
    }
    s_abort = 0;
    s_bar_count = 0;
    s_bar_gen = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == 0) {
    // ------------------------------- producer warp -------------------------------------------
    uint32_t k = 0;
    for (int it = blockIdx.x; it < P.n_items; it += gridDim.x) {
      const DevItem item = P.items[it];
      const DevGroup &G = P.groups[item.group];
      const int op = G.op;
      if (op == OP_READY) {
        // my buffers of every layer are free for this call: tell every peer
        if (lane == 0)
          for (int s = 0; s < P.world; ++s)
            if (s != G.exec_rank) st_release_sys(P.flags[s] + kReadyBase + G.exec_rank, P.seq);
        __syncwarp();
        continue;
      }
      if (!is_data_op(op)) continue;
      int ok = 1;
      if (lane == 0) ok = wait_group_sources(P, G, 100000 + item.group) ? 1 : 0;
      ok = __shfl_sync(0xffffffffu, ok, 0);
      if (!ok) s_abort = 1;
      if (s_abort) break;
      const uint32_t stage = k % kStages, use = k / kStages;
      if (use > 0 && !mbar_wait(&empty[stage], (use - 1) & 1u, &s_abort)) break;
      if (lane == 0) mbar_expect_tx(&full[stage], item_bytes(P, G, item));
      __syncwarp();
      fence_proxy_async();  // acquired sources / released stage -> async-proxy bulk copies
      issue_rows(P, G, item, bufs + (size_t)stage * kStageBytes, &full[stage], lane);
      ++k;
    }
    if (s_abort) {
      // drain: never leave with bulk copies still writing this CTA's shared memory
      for (uint32_t s = 0; s < kStages && s < k; ++s) {
        const uint32_t uses = (k - 1 - s) / kStages + 1;  // issues on stage s
        while (!mbar_test(&full[s], (uses - 1) & 1u)) {
        }
      }
    }
  } else {
    // ------------------------------- consumer warps ------------------------------------------
    const uint32_t tid = threadIdx.x - 32, T = blockDim.x - 32;
    uint32_t k = 0;
    for (int it = blockIdx.x; it < P.n_items; it += gridDim.x) {
      const DevItem item = P.items[it];
      const DevGroup &G = P.groups[item.group];
      const int op = G.op;
      if (op == OP_WAIT) {
        // forward completion: the halo is complete when the launch ends
        if (tid == 0 && !wait_group_sources(P, G, 200000 + item.group)) s_abort = 1;
        continue;
      }
      if (!is_data_op(op)) continue;
      const uint32_t stage = k % kStages, use = k / kStages;
      const unsigned nw = (unsigned)n_cons_warps;
      if (P.use_ready && G.ready_rank >= 0) {
        // the destination GPU's buffers must be free for this call before we write them
        if (tid == 0 &&
            !wait_geq(P.flags[G.exec_rank] + kReadyBase + G.ready_rank, P.seq, P,
                      1000 + item.group))
          s_abort = 1;
        if (!consumer_barrier(&s_bar_count, &s_bar_gen, nw, &s_abort, lane)) return;
      }
      if (!mbar_wait(&full[stage], use & 1u, &s_abort)) return;
      const uint8_t *buf = bufs + (size_t)stage * kStageBytes;
      if (op == OP_COPY)
        store_copy(P, G, item, buf, tid, T);
      else
        store_fold(P, G, item, buf, tid, T);
      if (item.flags & kItemSignal) {
        __threadfence_system();  // this thread's stores are visible system-wide ...
        // ... for every consumer thread ...
        if (!consumer_barrier(&s_bar_count, &s_bar_gen, nw, &s_abort, lane)) return;
        release_rows(P.flags[G.dst_rank] + G.sig_ctr, (uint64_t)(item.row_end - item.row_begin),
                     tid == 0);  // ... before the receiver can observe the count (done flag)
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[stage]);  // this warp is done reading the stage
      ++k;
    }
  }
}

}  // namespace

int launch_tma_executor(const ExecParams &p, int grid, int block, void *stream) {
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(executor_tma_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)kSmemBytes);
    if (e != cudaSuccess) return (int)e;
    attr = true;
  }
  executor_tma_kernel<<<grid, block, kSmemBytes, (cudaStream_t)stream>>>(p);
  return (int)cudaGetLastError();
}

int tma_executor_occupancy(int block, int *ctas_per_sm) {
  cudaError_t e = cudaFuncSetAttribute(executor_tma_kernel,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)kSmemBytes);
  if (e != cudaSuccess) return (int)e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, executor_tma_kernel, block,
                                                    kSmemBytes);
  return (int)e;
}

}  // namespace dgcl
