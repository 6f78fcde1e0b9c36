// MMA issue loop shaped like the conv kernel's (descriptors that change per
// K-step, an mbarrier wait per stage): which code shape keeps ptxas on the
// uniform datapath?  variant 0: asm-internal wait loop + elect-predicated MMA
// (the conv kernel as of r01); 1: vote-uniform wait loop + elect inside the
// MMA asm; 2: vote-uniform wait + elect-predicated.   cycles per MMA, N=32.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | (uint64_t)1 << 16 | (uint64_t)(1024 >> 4) << 32 | (uint64_t)1 << 46 |
         (uint64_t)2 << 61;
}
__device__ __forceinline__ bool elect_one() {
  uint32_t pred = 0;
  asm volatile("{\n.reg .pred P;\nelect.sync _|P, 0xffffffff;\nselp.b32 %0, 1, 0, P;\n}\n" : "=r"(pred));
  return pred != 0;
}
__device__ __forceinline__ void wait_asm(uint32_t bar, uint32_t ph) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(bar),
               "r"(ph) : "memory");
}
__device__ __forceinline__ uint32_t try_wait(uint32_t bar, uint32_t ph) {
  uint32_t ok;
  asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.b32 %0, 1, 0, p;\n}\n"
               : "=r"(ok) : "r"(bar), "r"(ph) : "memory");
  return ok;
}
__device__ __forceinline__ void wait_vote(uint32_t bar, uint32_t ph) {
  while (!__all_sync(0xffffffffu, try_wait(bar, ph))) {
  }
}
__device__ __forceinline__ void mma_pred(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc, uint32_t on) {
  asm volatile("{\n.reg .pred p, q;\nsetp.ne.b32 p, %4, 0;\nsetp.ne.b32 q, %5, 0;\n"
               "@q tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
               "l"(a), "l"(b), "r"(idesc), "r"(acc), "r"(on));
}
__device__ __forceinline__ void mma_elect(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n.reg .pred p, q;\nsetp.ne.b32 p, %4, 0;\nelect.sync _|q, 0xffffffff;\n"
               "@q tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
               "l"(a), "l"(b), "r"(idesc), "r"(acc));
}

__global__ void bench(int tiles, int taps, int n, int variant, unsigned long long* out) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bar, done;
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&done)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&bar)) : "memory");  // phase 0 done
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tslot;
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
  const uint32_t a0 = smem_u32(sm), b0 = smem_u32(sm + 65536);
  // warp index via shfl from lane 0: provably warp-uniform for ptxas (as
  // CUTLASS's canonical_warp_idx_sync), so the role branch is not divergent
  const int warp_u = variant >= 3 ? __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0) : (int)(threadIdx.x >> 5);
  if (variant >= 8 && variant < 10 && threadIdx.x < 32) {
    long long t0 = clock64();
    int cnt = 0;
    if (threadIdx.x == 0) {
      for (int tile = 0; tile < tiles; ++tile) {
        const uint32_t d = tm + (uint32_t)(tile & 1) * 64u;
        wait_asm(smem_u32(&bar), 0);
        const uint64_t ad0 = desc(a0), bd0 = desc(b0);
        if (variant == 8) {
#pragma unroll
          for (int t = 0; t < 9; ++t) {
            const uint64_t ad = ad0 + (uint64_t)((t / 3) * 65 + (t % 3) * 8), bd = bd0 + (uint64_t)(t & 3) * (uint64_t)(n * 8);
            asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                         ::"r"(d), "l"(ad), "l"(bd), "r"(idesc), "r"((uint32_t)(t > 0)));
            asm volatile("tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, 1;" ::"r"(d), "l"(ad + 2), "l"(bd + 2), "r"(idesc));
            cnt += 2;
          }
        } else {
          uint64_t aoff = 0;
          for (int t = 0; t < taps; ++t) {
            const uint64_t ad = ad0 + aoff, bd = bd0 + (uint64_t)(t & 3) * (uint64_t)(n * 8);
            asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                         ::"r"(d), "l"(ad), "l"(bd), "r"(idesc), "r"((uint32_t)(t > 0)));
            asm volatile("tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, 1;" ::"r"(d), "l"(ad + 2), "l"(bd + 2), "r"(idesc));
            aoff += (t % 3 == 2) ? 49u : 8u;
            cnt += 2;
          }
        }
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&done)) : "memory");
    }
    __syncwarp();
    long long t1 = clock64();
    wait_asm(smem_u32(&done), 0);
    long long t2 = clock64();
    if (blockIdx.x == 0 && threadIdx.x == 0) { out[0] = t1 - t0; out[1] = t2 - t0; out[2] = cnt; }
  } else if ((variant >= 3 && variant < 8 && warp_u == 0) || (variant >= 10 && warp_u == 0) || (variant < 3 && threadIdx.x < 32)) {
    const uint32_t on = elect_one() ? 1u : 0u;
    long long t0 = clock64();
    int cnt = 0;
    for (int tile = 0; tile < tiles; ++tile) {
      const uint32_t d = (variant >= 10 ? 0u : tm) + (uint32_t)(tile & 1) * 64u;
      if (variant == 0 || variant == 3 || variant >= 10) wait_asm(smem_u32(&bar), 0); else wait_vote(smem_u32(&bar), 0);
      uint64_t aoff = 0;
      uint32_t accum = 0;
      const uint64_t ad0 = desc(a0), bd0 = desc(b0);
      if (variant == 11) {
        // runtime tap loop, TMEM base a compile-time 0
        for (int t = 0; t < taps; ++t) {
          const uint64_t ad = ad0 + aoff, bd = bd0 + (uint64_t)(t & 3) * (uint64_t)(n * 8);
          mma_pred(d, ad, bd, idesc, accum, on);
          mma_pred(d, ad + 2, bd + 2, idesc, 1u, on);
          accum = 1;
          aoff += (t % 3 == 2) ? 65u : 8u;
          cnt += 2;
        }
        continue;
      }
      if (variant >= 6) {
        // fully unrolled 3x3: every descriptor = per-chunk base + compile-time offset
#pragma unroll
        for (int t = 0; t < 9; ++t) {
          const uint64_t ad = ad0 + (uint64_t)((t / 3) * 65 + (t % 3) * 8), bd = bd0 + (uint64_t)(t & 3) * (uint64_t)(n * 8);
          if (variant == 7) {
            mma_elect(d, ad, bd, idesc, t > 0);
            mma_elect(d, ad + 2, bd + 2, idesc, 1u);
          } else {
            mma_pred(d, ad, bd, idesc, t > 0, on);
            mma_pred(d, ad + 2, bd + 2, idesc, 1u, on);
          }
          cnt += 2;
        }
        continue;
      }
      for (int t = 0; t < taps; ++t) {
        const uint64_t ad = ad0 + aoff, bd = bd0 + (uint64_t)(t & 3) * (uint64_t)(n * 8);
        if (variant == 1 || variant == 4) {
          mma_elect(d, ad, bd, idesc, accum);
          mma_elect(d, ad + 2, bd + 2, idesc, 1u);
        } else {
          mma_pred(d, ad, bd, idesc, accum, on);
          mma_pred(d, ad + 2, bd + 2, idesc, 1u, on);
        }
        accum = 1;
        aoff += (t % 3 == 2) ? 1040u / 16u * 16u / 16u * 0 + 65u : 8u;  // row / column step (in 16-byte units)
        cnt += 2;
      }
    }
    if (on) asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&done)) : "memory");
    __syncwarp();
    long long t1 = clock64();
    wait_asm(smem_u32(&done), 0);
    long long t2 = clock64();
    if (blockIdx.x == 0 && threadIdx.x == 0) { out[0] = t1 - t0; out[1] = t2 - t0; out[2] = cnt; }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tm));
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 32);
  cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int variant : {0, 6, 10, 11})
    for (int n : {32, 128}) {
      bench<<<148, 128, 140 * 1024>>>(64, 9, n, variant, d);
      bench<<<148, 128, 140 * 1024>>>(64, 9, n, variant, d);
      cudaError_t e = cudaDeviceSynchronize();
      unsigned long long h[3];
      cudaMemcpy(h, d, 24, cudaMemcpyDeviceToHost);
      printf("variant %d N=%3d: issue %.1f complete %.1f cyc/MMA  %s\n", variant, n, (double)h[0] / h[2],
             (double)h[1] / h[2], cudaGetErrorString(e));
    }
  return 0;
}
