// tcgen05.mma issue rate from a warp-uniform loop with an elected lane (the
// conv kernel's issue pattern), cta_group::1 M=128 and cta_group::2 M=256,
// N = 16..256, K = 16 per instruction.  Prints cycles per MMA (issue of
// `iters` MMAs + completion).   nvcc -gencode arch=compute_100a,code=sm_100a
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

template <int CG>
__global__ void bench(int iters, int n, unsigned long long* out, int aoff = 0) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bar;
  uint32_t rank = 0;
  if (CG == 2) asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  if (threadIdx.x < 32) {
    if (CG == 1) {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(&tslot)));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    } else {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(&tslot)));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (CG == 2) {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tslot;
  const int M = 128 * CG;
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
  const uint64_t ad = desc(smem_u32(sm) + (uint32_t)aoff), bd = desc(smem_u32(sm + 32768));
  if (threadIdx.x < 32 && rank == 0) {
    const uint32_t on = elect_one() ? 1u : 0u;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const uint32_t acc = i > 0;
      const uint64_t a = ad + 2 * (i & 3), b = bd + 2 * (i & 3);
      if (CG == 1)
        asm volatile("{\n.reg .pred p, q;\nsetp.ne.b32 p, %4, 0;\nsetp.ne.b32 q, %5, 0;\n"
                     "@q tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tm),
                     "l"(a), "l"(b), "r"(idesc), "r"(acc), "r"(on));
      else
        asm volatile("{\n.reg .pred p, q;\nsetp.ne.b32 p, %4, 0;\nsetp.ne.b32 q, %5, 0;\n"
                     "@q tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tm),
                     "l"(a), "l"(b), "r"(idesc), "r"(acc), "r"(on));
    }
    if (CG == 1)
      asm volatile("{\n.reg .pred q;\nsetp.ne.b32 q, %1, 0;\n"
                   "@q tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n}\n" ::"r"(
                       smem_u32(&bar)), "r"(on) : "memory");
    else
      asm volatile("{\n.reg .pred q;\nsetp.ne.b32 q, %1, 0;\n"
                   "@q tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %2;\n}\n" ::"r"(
                       smem_u32(&bar)), "r"(on), "h"((uint16_t)3) : "memory");
    long long t1 = clock64();
    asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W_%=;\n}\n" ::"r"(
                     smem_u32(&bar)) : "memory");
    long long t2 = clock64();
    if (blockIdx.x == 0 && threadIdx.x == 0) { out[0] = t1 - t0; out[1] = t2 - t0; }
  } else if (CG == 2 && threadIdx.x < 32 && rank == 1) {
    asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W_%=;\n}\n" ::"r"(
                     smem_u32(&bar)) : "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (CG == 2) asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (threadIdx.x < 32) {
    if (CG == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tm));
    else asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 256;" ::"r"(tm));
  }
}

// the conv kernel's situation: TMEM address and B descriptor the compiler
// cannot prove warp-uniform (loaded from smem).  mode 1: warp-uniform loop,
// predicated issue by the elected lane; mode 2: the whole loop in a lane-0 branch
__global__ void bench_nu(int iters, int n, unsigned long long* out, int mode) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint64_t sdesc[2];
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    sdesc[0] = desc(smem_u32(sm));
    sdesc[1] = desc(smem_u32(sm + 32768));
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tslot;
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
  const uint64_t ad = sdesc[0], bd = sdesc[1];
  __shared__ __align__(8) uint64_t spinbar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&spinbar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x >= 32) {
    // mode 3: the other warps spin on an mbarrier until the issuing warp is done
    if (mode == 3)
      asm volatile("{\n.reg .pred p;\nS_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra S_%=;\n}\n" ::"r"(
                       smem_u32(&spinbar)) : "memory");
  } else {
    const int lane = threadIdx.x & 31;
    long long t0 = clock64();
    if (mode == 1 || mode == 3) {
      const uint32_t on = elect_one() ? 1u : 0u;
      for (int i = 0; i < iters; ++i) {
        const uint32_t acc = i > 0;
        const uint64_t a = ad + 2 * (i & 3), b = bd + 2 * (i & 3);
        asm volatile("{\n.reg .pred p, q;\nsetp.ne.b32 p, %4, 0;\nsetp.ne.b32 q, %5, 0;\n"
                     "@q tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tm + (uint32_t)(i & 1) * 64u),
                     "l"(a), "l"(b), "r"(idesc), "r"(acc), "r"(on));
      }
      asm volatile("{\n.reg .pred q;\nsetp.ne.b32 q, %1, 0;\n"
                   "@q tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n}\n" ::"r"(
                       smem_u32(&bar)), "r"(on) : "memory");
    } else if (lane == 0) {
      for (int i = 0; i < iters; ++i) {
        const uint32_t acc = i > 0;
        const uint64_t a = ad + 2 * (i & 3), b = bd + 2 * (i & 3);
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                     "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tm + (uint32_t)(i & 1) * 64u),
                     "l"(a), "l"(b), "r"(idesc), "r"(acc));
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar))
                   : "memory");
    }
    __syncwarp();
    long long t1 = clock64();
    asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W_%=;\n}\n" ::"r"(
                     smem_u32(&bar)) : "memory");
    long long t2 = clock64();
    if (blockIdx.x == 0 && threadIdx.x == 0) { out[0] = t1 - t0; out[1] = t2 - t0; }
    if (threadIdx.x == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&spinbar)) : "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tm));
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 16);
  cudaFuncSetAttribute(bench<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  cudaFuncSetAttribute(bench<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  const int iters = 4096;
  for (int cg : {1, 2})
    for (int n : {16, 32, 64, 128, 256}) {
      if (cg == 2 && n < 32) continue;
      for (int rep = 0; rep < 2; ++rep) {
        if (cg == 1) {
          bench<1><<<148, 128, 80 * 1024>>>(iters, n, d, 0);
        } else {
          cudaLaunchConfig_t cfg = {};
          cfg.gridDim = dim3(148);
          cfg.blockDim = dim3(128);
          cfg.dynamicSmemBytes = 80 * 1024;
          cudaLaunchAttribute at[1];
          at[0].id = cudaLaunchAttributeClusterDimension;
          at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
          cfg.attrs = at; cfg.numAttrs = 1;
          cudaLaunchKernelEx(&cfg, bench<2>, iters, n, d, 0);
        }
      }
      cudaError_t e = cudaDeviceSynchronize();
      unsigned long long h[2];
      cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
      const int M = 128 * cg;
      const double floor_ = 128.0 * n / 256.0;  // cycles per MMA per SM pair member (guide formula)
      printf("cta_group::%d M=%d N=%3d: issue %.1f cyc/MMA, complete %.1f cyc/MMA (floor %.0f) -> %.0f flop/cyc/SM  %s\n",
             cg, M, n, (double)h[0] / iters, (double)h[1] / iters, floor_,
             2.0 * M * n * 16 / ((double)h[1] / iters) / cg, cudaGetErrorString(e));
    }
  cudaFuncSetAttribute(bench_nu, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  for (int mode : {1, 2, 3})
    for (int n : {32, 128}) {
      bench_nu<<<148, 384, 80 * 1024>>>(iters, n, d, mode);
      bench_nu<<<148, 384, 80 * 1024>>>(iters, n, d, mode);
      cudaError_t e = cudaDeviceSynchronize();
      unsigned long long h[2];
      cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
      printf("non-uniform operands, %s N=%3d: issue %.1f complete %.1f cyc/MMA  %s\n",
             mode == 1 ? "elected+predicated" : mode == 2 ? "lane-0 branch     " : "elected + 11 spinning warps", n, (double)h[0] / iters, (double)h[1] / iters,
             cudaGetErrorString(e));
    }
  // A window starting at a 128-byte row inside the swizzle atom (the conv's
  // halo-mode shifted windows): same loop, A start offset 0 / 128 / 384 B
  for (int aoff : {0, 128, 384, 1024 + 256})
    for (int n : {32, 128, 256}) {
      bench<1><<<148, 128, 80 * 1024>>>(iters, n, d, aoff);
      bench<1><<<148, 128, 80 * 1024>>>(iters, n, d, aoff);
      cudaError_t e = cudaDeviceSynchronize();
      unsigned long long h[2];
      cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
      printf("A offset %4d B  N=%3d: complete %.1f cyc/MMA  %s\n", aoff, n, (double)h[1] / iters, cudaGetErrorString(e));
    }
  return 0;
}
