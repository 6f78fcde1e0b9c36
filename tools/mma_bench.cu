// mma_bench.cu -- standalone: issue cost of tcgen05.mma.cta_group::1.kind::f16
// from one thread (M=128, K=16, N in {32..256}), with a tcgen05.commit to an
// mbarrier every `g` MMAs (and a wait on it, like a pipeline stage), vs without.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mma_bench mma_bench.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <vector>

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

__global__ void mma_kernel(int iters, int n, int g, int wait_each, unsigned long long* out, int m = 128, int atmem = 0) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bars[4];
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[i])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tslot;
  const int issuers = blockDim.x / 32;
  if ((threadIdx.x & 31) == 0) {
    const int w = threadIdx.x >> 5;
    uint64_t& bar = bars[w];
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(m >> 4) << 24);
    const uint64_t ad = desc(smem_u32(sm)), bd = desc(smem_u32(sm + 16384));
    uint32_t ph = 0;
    int gc = 0;
    long long t0 = clock64();
    for (int i = w; i < iters; i += issuers) {
      uint32_t acc = i > w;
      if (atmem)
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(
                         tm + (uint32_t)(w * (256 / issuers))),
                     "r"(tm + 256u + 8u * (uint32_t)(i & 3)), "l"(bd + 2 * (i & 3)), "r"(idesc), "r"(acc));
      else
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(
                         tm + (uint32_t)(w * (256 / issuers))),
                     "l"(ad + 2 * (i & 3)), "l"(bd + 2 * (i & 3)), "r"(idesc), "r"(acc));
      if (g > 0 && ++gc == g) {
        gc = 0;
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar))
                     : "memory");
        if (wait_each) {
          asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
                           smem_u32(&bar)),
                       "r"(ph)
                       : "memory");
          ph ^= 1;
        }
      }
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar))
                 : "memory");
    long long t1 = clock64();
    asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
                     smem_u32(&bar)),
                 "r"(ph)
                 : "memory");
    long long t2 = clock64();
    if (blockIdx.x == 0 && w == 0) { out[0] = t1 - t0; out[1] = t2 - t0; }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm));
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 16);
  cudaFuncSetAttribute(mma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  for (int issuers : {1, 2, 4})
  for (int n : {64, 128, 256})
    for (int g : {0, 4}) for (int we : {0, 1}) {
      if (g == 0 && we) continue;
      if (n * issuers > 256) continue;
      int iters = 2048;
      mma_kernel<<<148, 32 * issuers, 70 * 1024>>>(iters, n, g, we, d);
      mma_kernel<<<148, 32 * issuers, 70 * 1024>>>(iters, n, g, we, d);
      cudaDeviceSynchronize();
      unsigned long long h[2];
      cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
      double ideal = 128.0 * n / 256.0;
      printf("issuers %d N=%3d commit every %d %s: issue %.1f cyc/MMA, complete %.1f cyc/MMA (ideal %.0f) %s\n", issuers, n, g,
             we ? "+wait" : "     ", (double)h[0] / iters, (double)h[1] / iters, ideal,
             cudaGetErrorString(cudaGetLastError()));
    }
  // operand-source study: M = 64 vs 128 (A bytes halve), A from smem vs TMEM
  for (int atmem : {0, 1})
    for (int m : {64, 128})
      for (int n : {16, 32, 64, 128, 256}) {
        int iters = 2048;
        mma_kernel<<<148, 32, 70 * 1024>>>(iters, n, 0, 0, d, m, atmem);
        mma_kernel<<<148, 32, 70 * 1024>>>(iters, n, 0, 0, d, m, atmem);
        cudaDeviceSynchronize();
        unsigned long long h[2];
        cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
        printf("A from %s M=%3d N=%3d: complete %.1f cyc/MMA (floor %.0f) %s\n", atmem ? "TMEM" : "smem", m, n,
               (double)h[1] / iters, 128.0 * n / 256.0, cudaGetErrorString(cudaGetLastError()));
      }
  return 0;
}
