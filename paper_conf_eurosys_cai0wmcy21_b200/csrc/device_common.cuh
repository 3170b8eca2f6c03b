// device_common.cuh — PTX helpers shared by the executor kernels (sm_100a).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "internal.h"

namespace dgcl {
namespace dev {

constexpr int kUnroll = 4;

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
// The flag protocol's scope: system (.sys) when peers are other GPUs (NVLink peer memory, CUDA
// IPC), device (.gpu) when every rank lives on this GPU (loopback) — ExecParams::sys_scope.  The
// narrower scope is exact there and makes fences / releases far cheaper (MEMBAR.GPU vs .SYS).
__device__ __forceinline__ uint64_t ld_acquire_gpu(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu(uint64_t *p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_release_gpu_add(uint64_t *p, uint64_t v) {
  asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire(const uint64_t *p, int sys) {
  return sys ? ld_acquire_sys(p) : ld_acquire_gpu(p);
}
__device__ __forceinline__ void st_release(uint64_t *p, uint64_t v, int sys) {
  if (sys)
    st_release_sys(p, v);
  else
    st_release_gpu(p, v);
}
__device__ __forceinline__ void red_release_add(uint64_t *p, uint64_t v, int sys) {
  if (sys)
    red_release_sys_add(p, v);
  else
    red_release_gpu_add(p, v);
}
// this thread's earlier stores are visible at the protocol's scope before its later ones
__device__ __forceinline__ void fence_scope(int sys) {
  if (sys)
    __threadfence_system();
  else
    __threadfence();
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

// partial 16-B chunk (a row's tail, nb in {4, 8, 12}): predicated 4-byte accesses
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

__device__ __forceinline__ float4 as_f4(const int4 &v) {
  return make_float4(__int_as_float(v.x), __int_as_float(v.y), __int_as_float(v.z),
                     __int_as_float(v.w));
}
__device__ __forceinline__ int4 as_i4(const float4 &a) {
  return make_int4(__float_as_int(a.x), __float_as_int(a.y), __float_as_int(a.z),
                   __float_as_int(a.w));
}
// one IEEE round-to-nearest fp32 add per lane (never contracted, never reassociated)
__device__ __forceinline__ void add4(float4 &a, const int4 &b) {
  a.x = __fadd_rn(a.x, __int_as_float(b.x));
  a.y = __fadd_rn(a.y, __int_as_float(b.y));
  a.z = __fadd_rn(a.z, __int_as_float(b.z));
  a.w = __fadd_rn(a.w, __int_as_float(b.w));
}

// kTermRankTree: one output chunk of a postfix fold program — every word pushes load(word), then
// replaces the top two by (below + top) (word >> 24) & 15 times; the stack bottom is the starting
// value.  The top of the stack lives in a register and only the entries below it in a small
// local array, so a word with adds >= 1 consumes the register top without memory traffic: a
// direct (relay-free) tree, ((L + o1) + o2) ..., runs entirely in registers, and only relay
// subtrees (a word with no adds pushes) touch local memory.
template <typename Load>
__device__ __forceinline__ float4 fold_tree(float4 init, const uint32_t *prog, int n, Load load) {
  float4 below[kTreeMaxDepth];
  int nb = 0;
  float4 top = init;
  for (int j = 0; j < n; ++j) {
    const uint32_t w = prog[j];
    float4 t = load(w);
    uint32_t a = (w >> kTreeAddShift) & 15u;
    if (a == 0) {  // push: the old top goes below
      below[nb++] = top;
      top = t;
      continue;
    }
    t.x = __fadd_rn(top.x, t.x);  // the first add consumes the register top
    t.y = __fadd_rn(top.y, t.y);
    t.z = __fadd_rn(top.z, t.z);
    t.w = __fadd_rn(top.w, t.w);
    for (; a > 1; --a) {
      const float4 b = below[--nb];
      t.x = __fadd_rn(b.x, t.x);
      t.y = __fadd_rn(b.y, t.y);
      t.z = __fadd_rn(b.z, t.z);
      t.w = __fadd_rn(b.w, t.w);
    }
    top = t;
  }
  return top;
}

// Spin until *p >= target (acquire, system scope), bounded by the watchdog.
static __device__ __noinline__ bool wait_geq(const uint64_t *p, uint64_t target, const ExecParams &P,
                                      int code) {
  if (ld_acquire(p, P.sys_scope) >= target) return true;
  const uint64_t t0 = globaltimer();
  for (uint32_t it = 1;; ++it) {
    __nanosleep(64);
    if (ld_acquire(p, P.sys_scope) >= target) return true;
    if ((it & 255) == 0) {
      if (*(volatile int *)P.err != 0) return false;  // another CTA / peer already failed
      if (globaltimer() - t0 > P.timeout_ns) {
        atomicCAS(P.err, 0, code);
        __threadfence_system();
        return false;
      }
    }
  }
}

// counter index -> word: the flag region, or (multicast done counters) the multicast flag page
__device__ __forceinline__ uint64_t *ctr_ptr(const ExecParams &P, int rank, int64_t ctr) {
  return ctr < kMcCtrBase ? P.flags[rank] + ctr : P.mcuc_flags[rank] + (ctr - kMcCtrBase);
}

// NVSwitch multicast: one store through the multicast address lands in every bound GPU's copy
__device__ __forceinline__ void mm_st_v4(void *p, const int4 &v) {
  asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p),
               "f"(__int_as_float(v.x)), "f"(__int_as_float(v.y)), "f"(__int_as_float(v.z)),
               "f"(__int_as_float(v.w))
               : "memory");
}
__device__ __forceinline__ void mm_red_release_add(uint64_t *p, uint64_t v) {
  asm volatile("multimem.red.release.sys.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// a 16-B chunk of multicast region row `row` (layer pitch): every GPU's copy
__device__ __forceinline__ void mc_store16(const ExecParams &P, int exec, int64_t row,
                                           uint32_t col, const int4 &v) {
  if (P.mc_emulate) {
    for (int r = 0; r < P.world; ++r)
      st_v4(P.buf[K_MCUC][r].ptr + row * P.buf[K_MCUC][r].pitch + (int64_t)col * 16, v);
  } else {
    mm_st_v4(P.buf[K_MCAST][exec].ptr + row * P.buf[K_MCAST][exec].pitch + (int64_t)col * 16, v);
  }
}
// owner's multicast done counter += rows on every GPU (the caller fenced its stores)
__device__ __forceinline__ void mc_publish(const ExecParams &P, int owner, uint64_t rows) {
  if (P.mc_emulate) {
    for (int r = 0; r < P.world; ++r) red_release_add(P.mcuc_flags[r] + owner, rows, P.sys_scope);
  } else {
    mm_red_release_add(P.mc_flags + owner, rows);
  }
}

// counter waits of an item (all of them, blocking): its source rows are final
__device__ __forceinline__ bool wait_item_sources(const ExecParams &P, const DevItem &I,
                                                  int code) {
  bool ok = true;
  for (int w = 0; ok && w < I.wait_n; ++w) {
    const DevWait W = P.waits[I.wait_off + w];
    ok = wait_geq(ctr_ptr(P, I.exec_rank, W.ctr), P.epoch[I.dir] * (uint64_t)W.amount, P, code);
  }
  return ok;
}

// fast division by n_chunks (exact for x < 2^31)
__device__ __forceinline__ uint32_t fdiv(uint32_t x, const ExecParams &P) {
  return (__umulhi(x, P.div_mul) + x) >> P.div_shift;
}

__device__ __forceinline__ int64_t row_of(const int32_t *idx, int64_t base, int64_t i) {
  return idx ? (int64_t)__ldg(idx + i) : base + i;
}

// receiver-visible completion of an item: every thread's stores, then one counter add
__device__ __forceinline__ void release_rows(uint64_t *ctr, uint64_t rows, bool leader, int sys) {
  if (leader) red_release_add(ctr, rows, sys);
}

}  // namespace dev
}  // namespace dgcl
