// pipe_bench.cu — per-SM copy-pipeline ceilings on this B200 (diagnostic tool, not the product):
// one persistent CTA per SM moves 4 GiB of `chunk`-byte pieces from a source (L2-resident when
// small, as the re-read rows of a high-fan-out forward; DRAM when large) to a destination.
//   mode 0 tma/tma : producer bulk-loads a chunk into one of S stages, `split` fixed consumer
//                    warps bulk-store it (the executor's scheme)
//   mode 1 tma/stg : same loads, every consumer thread LDS + STG
//   mode 2 ldg/stg : no shared memory, every thread LDG.128 x4 -> STG.128 x4
//   mode 3 fan-out : a chunk is bulk-loaded once and bulk-stored to `split` destination regions
//                    (one consumer warp each), as a fan-out of one owner's rows to its receivers
// build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/pipe_bench.cu -o build/pipe_bench
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t *b, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mb_expect(uint64_t *b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mb_arrive(uint64_t *b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(b)) : "memory");
}
__device__ __forceinline__ void mb_wait(uint64_t *b, uint32_t ph) {
  uint32_t ok = 0;
  while (!ok)
    asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
                 : "=r"(ok) : "r"(sa(b)), "r"(ph) : "memory");
}

template <int kMode>
__global__ void __launch_bounds__(256) pipe(const char *src, size_t src_bytes, char *dst,
                                                size_t total, int chunk, int S, int split) {
  extern __shared__ __align__(128) uint8_t sm[];
  uint64_t *full = reinterpret_cast<uint64_t *>(sm), *empty = full + 8;
  uint8_t *stg = sm + 128;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, ncw = (blockDim.x >> 5) - 1;
  const size_t nch = (kMode == 3 ? total / split : total) / chunk, G = gridDim.x;
  const size_t nsrc = src_bytes / chunk;
  if (kMode == 2) {
    for (size_t c = blockIdx.x; c < nch; c += G) {
      const int4 *s = reinterpret_cast<const int4 *>(src + (c % nsrc) * chunk);
      int4 *d = reinterpret_cast<int4 *>(dst + c * chunk);
      const int n = chunk / 16;
      for (int i = threadIdx.x; i < n; i += 4 * blockDim.x) {
        int4 v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (i + u * (int)blockDim.x < n) v[u] = __ldcg(s + i + u * blockDim.x);
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (i + u * (int)blockDim.x < n) d[i + u * blockDim.x] = v[u];
      }
    }
    return;
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mb_init(&full[s], 1);
      mb_init(&empty[s], ncw);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == 0) {
    if (lane == 0) {
      uint32_t i = 0;
      for (size_t c = blockIdx.x; c < nch; c += G, ++i) {
        const uint32_t s = i % S, use = i / S;
        if (use) mb_wait(&empty[s], (use - 1) & 1);
        mb_expect(&full[s], chunk);
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         sa(stg + (size_t)s * chunk)),
                     "l"(src + (c % nsrc) * chunk), "r"(chunk), "r"(sa(&full[s]))
                     : "memory");
      }
    }
    return;
  }
  const int cw = warp - 1;
  const int tid = threadIdx.x - 32, T = blockDim.x - 32;
  uint32_t i = 0;
  for (size_t c = blockIdx.x; c < nch; c += G, ++i) {
    const uint32_t s = i % S, use = i / S;
    uint8_t *st = stg + (size_t)s * chunk;
    mb_wait(&full[s], use & 1);
    if (kMode == 3) {
      if (cw < split && lane == 0) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(
                         dst + (size_t)cw * nch * chunk + c * chunk),
                     "r"(sa(st)), "r"(chunk) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      }
    } else if (kMode == 1) {
      for (int o = tid * 16; o < chunk; o += T * 16)
        *reinterpret_cast<int4 *>(dst + c * chunk + o) = *reinterpret_cast<const int4 *>(st + o);
    } else if (cw < split && lane == 0) {
      const int lo = (int)((int64_t)chunk * cw / split) & ~15, hi = cw + 1 == split ? chunk : (int)((int64_t)chunk * (cw + 1) / split) & ~15;
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + c * chunk + lo),
                   "r"(sa(st + lo)), "r"(hi - lo) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
    }
    __syncwarp();
    if (lane == 0) mb_arrive(&empty[s]);
  }
  if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main() {
  const size_t total = (size_t)4 << 30;
  char *src, *dst;
  cudaMalloc(&src, total);
  cudaMalloc(&dst, total);
  cudaMemset(src, 1, total);
  cudaMemset(dst, 0, total);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto run = [&](const char *name, auto kern, size_t src_bytes, int chunk, int S, int split, int ctas = 1) {
    const size_t smem = 128 + (size_t)S * chunk;
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    float best = 1e9f;
    for (int rep = 0; rep < 5; ++rep) {
      cudaEventRecord(a);
      kern<<<sms * ctas, 256, smem>>>(src, src_bytes, dst, total, chunk, S, split);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (rep && ms < best) best = ms;
    }
    cudaError_t e = cudaGetLastError();
    printf("%-12s x%d src %5zu MB chunk %6d stages %d split %d: %6.0f GB/s written (%6.0f r+w) %s\n", name, ctas,
           src_bytes >> 20, chunk, S, split, total / (best * 1e6),
           (src_bytes >= total ? 2.0 : 1.0) * total / (best * 1e6), e ? cudaGetErrorString(e) : "");
  };
  for (int S : {2, 3})
    for (int fan : {4, 7}) run("fan-out", pipe<3>, total, 61440, S, fan);
  for (size_t sb : {(size_t)48 << 20, total}) {
    run("ldg/stg", pipe<2>, sb, 61440, 0, 0, 1);
    run("ldg/stg", pipe<2>, sb, 61440, 0, 0, 8);
    for (int S : {3, 2})
      for (int split : {1, 4, 7}) run("tma/tma", pipe<0>, sb, 61440, S, split);
    run("tma/tma", pipe<0>, sb, 45056, 4, 4);
    run("tma/tma", pipe<0>, sb, 30720, 6, 4);
    run("tma/stg", pipe<1>, sb, 61440, 3, 0);
  }
  return 0;
}
