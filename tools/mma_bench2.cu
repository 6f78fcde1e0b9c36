// mma_bench2.cu -- standalone: tcgen05.mma (kind::f16, cta_group::1) issue
// throughput with the warp-converged elect.sync pattern the conv kernel uses
// (operands in uniform registers), vs. N, M, A source (smem / TMEM), number
// of issuing warps (separate accumulators) and unroll depth.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mma_bench2 mma_bench2.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}
__device__ __forceinline__ bool elect_one() {
  uint32_t pred = 0;
  asm volatile("{\n.reg .pred P;\nelect.sync _|P, 0xffffffff;\nselp.b32 %0, 1, 0, P;\n}\n" : "=r"(pred));
  return pred != 0;
}
__device__ __forceinline__ void mma_ss(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
               "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(d),
               "r"(a), "l"(b), "r"(idesc), "r"(acc));
}

// each issuing warp: `iters` rounds of 4 MMAs (one 64-channel K-step), into
// its own accumulator columns; commit + wait at the end only
__global__ void bench(int iters, int n, int m, int atmem, unsigned long long* out, int aoff = 0, int rot = 0) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bars[8];
  const int warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < 8; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[i])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tslot;
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(m >> 4) << 24);
  const uint32_t cols_per = atmem ? 256u / nw : 512u / nw;
  const uint32_t d = tm + (uint32_t)warp * cols_per;
  const uint32_t at = tm + 256u + (uint32_t)warp * 8u;  // A in TMEM (only with atmem: nw*n <= 256)
  const uint64_t ad = desc(smem_u32(sm) + warp * 16384 + aoff), bd = desc(smem_u32(sm + 65536));
  long long t0 = clock64();
  const bool el = elect_one();
  for (int i = 0; i < iters; ++i) {
    if (el) {
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        if (atmem) mma_ts(d, at + 2u * k, bd + 2 * k, idesc, (i | k) ? 1u : 0u);
        else mma_ss(d, ad + 2 * k + (rot ? (uint64_t)(8 * (i % 3)) : 0), bd + 2 * k, idesc, (i | k) ? 1u : 0u);
      }
    }
    __syncwarp();
  }
  if (el)
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bars[warp]))
                 : "memory");
  __syncwarp();
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W_%=;\n}\n" ::"r"(
                   smem_u32(&bars[warp]))
               : "memory");
  long long t1 = clock64();
  if (blockIdx.x == 0 && (threadIdx.x & 31) == 0) out[warp] = t1 - t0;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm));
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 64);
  cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  // A window alignment study (halo mode starts A windows at any 128-B row)
  for (int n : {32, 64, 128, 256})
    for (int aoff : {0, 128, 384, 1152})
      for (int rot : {0, 1}) {
        const int iters = 1024;
        bench<<<148, 32, 140 * 1024>>>(iters, n, 128, 0, d, aoff, rot);
        bench<<<148, 32, 140 * 1024>>>(iters, n, 128, 0, d, aoff, rot);
        cudaError_t e = cudaDeviceSynchronize();
        unsigned long long h[8];
        cudaMemcpy(h, d, 64, cudaMemcpyDeviceToHost);
        printf("N=%3d A start +%4d B %s: %.1f cyc/MMA (floor %.0f) %s\n", n, aoff, rot ? "(rotating +0/128/256 B)" : "                       ",
               (double)h[0] / (iters * 4.0), 128.0 * n / 256.0, cudaGetErrorString(e));
      }
  return 0;
}
