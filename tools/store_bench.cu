// store_bench.cu — per-SM write-path ceilings on this B200 (diagnostic tool, not the product):
// how fast can one persistent CTA per SM push data from shared memory (or registers) to HBM?
//   tma   : bulk (TMA) stores cp.async.bulk.global.shared of `piece` bytes, `split` warps each
//           issuing one store per chunk, up to `depth` commit groups in flight per warp
//   stg   : every thread st.global.v4 from registers (fill-like), grid-stride
//   lds   : every thread ld.shared.v4 + st.global.v4 (the executor's non-bulk store path)
//   mix   : warps [0, split) TMA stores, the others LDS+STG, each its share of every chunk
// Destinations: contiguous chunks of `chunk` bytes handed round-robin to CTAs (like the
// executor's items), so each CTA writes chunk-sized contiguous pieces at scattered offsets.
// build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/store_bench.cu -o build/store_bench
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void bulk_s2g(void *g, const void *s, uint32_t bytes, uint64_t pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(g),
               "r"(smem_u32(s)), "r"(bytes), "l"(pol)
               : "memory");
}
__device__ __forceinline__ uint64_t pol_ef() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}

template <int kMode>  // 0 tma, 1 stg, 2 lds, 3 mix
__global__ void __launch_bounds__(512, 1) store_kernel(char *out, size_t total, int chunk, int split,
                                                        int depth, int hint, int off) {
  extern __shared__ __align__(128) uint8_t sm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nw = blockDim.x >> 5;
  for (int i = threadIdx.x; i < chunk / 16; i += blockDim.x)
    reinterpret_cast<int4 *>(sm)[i] = make_int4(i, i + 1, i + 2, i + 3);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  const uint64_t pol = hint ? pol_ef() : 0;
  const size_t nchunks = total / chunk - 1;
  int inflight = 0;
  for (size_t c = blockIdx.x; c < nchunks; c += gridDim.x) {
    char *dst = out + c * chunk + off;
    const bool tma_w = kMode == 0 || (kMode == 3 && warp < split);
    if (tma_w) {
      const int parts = kMode == 0 ? split : split;
      if (warp < parts && lane == 0) {
        // tma share: mode 0 -> whole chunk over `split` warps; mode 3 -> first half of the chunk
        const int span = kMode == 0 ? chunk : chunk / 2;
        const int lo = (int)((int64_t)span * warp / parts) & ~15;
        const int hi = warp + 1 == parts ? span : (int)((int64_t)span * (warp + 1) / parts) & ~15;
        if (hi > lo) {
          if (hint)
            bulk_s2g(dst + lo, sm + lo, hi - lo, pol);
          else
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + lo),
                         "r"(smem_u32(sm + lo)), "r"(hi - lo)
                         : "memory");
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          if (++inflight >= depth) {
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            inflight = 0;
          }
        }
      }
    } else {
      // register / lds stores by the remaining threads
      const int first = kMode == 3 ? chunk / 2 : 0;
      const int t0 = kMode == 3 ? threadIdx.x - split * 32 : threadIdx.x;
      const int T = kMode == 3 ? blockDim.x - split * 32 : blockDim.x;
      for (int o = first + t0 * 16; o < chunk; o += T * 16) {
        int4 v = kMode == 1 ? make_int4(o, o, o, o) : *reinterpret_cast<const int4 *>(sm + o);
        *reinterpret_cast<int4 *>(dst + o) = v;
      }
    }
  }
  if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main(int argc, char **argv) {
  const size_t total = (size_t)4 << 30;
  char *out;
  cudaMalloc(&out, total);
  cudaMemset(out, 0, total);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto run = [&](const char *name, auto kern, int chunk, int split, int depth, int hint, int ctas, int off = 0) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    float best = 1e9f;
    for (int rep = 0; rep < 6; ++rep) {
      cudaEventRecord(a);
      kern<<<sms * ctas, 512, chunk, 0>>>(out, total, chunk, split, depth, hint, off);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (rep > 0 && ms < best) best = ms;
    }
    cudaError_t e = cudaGetLastError();
    printf("%-4s chunk %6d split %2d depth %d hint %d ctas/SM %d off %3d: %7.0f GB/s %s\n", name,
           chunk, split, depth, hint, ctas, off, (total - chunk) / (best * 1e6),
           e ? cudaGetErrorString(e) : "");
  };
  if (argc > 1) {  // alignment study: chunk = 25 rows of a 2416-B pitch, start offsets
    for (int off : {0, 16, 32, 64, 128})
      for (int split : {1, 4})
        run("tma", store_kernel<0>, 60400, split, 1, 1, 1, off);
    for (int off : {0, 16})
      run("stg", store_kernel<1>, 60400, 0, 1, 1, 1, off);
    return 0;
  }
  for (int hint = 0; hint < 2; ++hint) {
    run("stg", store_kernel<1>, 61440, 0, 1, hint, 1);
    run("lds", store_kernel<2>, 61440, 0, 1, hint, 1);
    for (int split : {1, 4, 15, 16})
      for (int depth : {1, 2, 4})
        run("tma", store_kernel<0>, 61440, split, depth, hint, 1);
    run("tma", store_kernel<0>, 16384, 8, 2, hint, 1);
    run("tma", store_kernel<0>, 16384, 8, 4, hint, 1);
    run("tma", store_kernel<0>, 61440, 15, 2, hint, 2);
    for (int split : {4, 8})
      run("mix", store_kernel<3>, 61440, split, 2, hint, 1);
  }
  return 0;
}
