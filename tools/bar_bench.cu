// bar_bench.cu -- standalone: cost of the producer/consumer mbarrier ring used
// by the conv kernel (no TMA, no MMA): warp 0 arrives on full[st] after
// waiting empty[st]; warp 1 waits full[st] and arrives on empty[st] (plain
// arrive or tcgen05.commit).  All counters incremental (no divisions).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bar_bench bar_bench.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void wait_try(uint32_t bar, uint32_t par) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(bar),
               "r"(par)
               : "memory");
}
__device__ __forceinline__ void wait_test(uint32_t bar, uint32_t par) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.test_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(bar),
               "r"(par)
               : "memory");
}
__device__ __forceinline__ void arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}

__global__ void ring_kernel(int iters, int ST, int mode, int use_commit, unsigned long long* out) {
  __shared__ __align__(8) uint64_t full[16], empty[16], never;
  __shared__ uint32_t tslot;
  if (threadIdx.x == 0) {
    for (int i = 0; i < ST; ++i) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[i])));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&empty[i])));
    }
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&never)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (threadIdx.x >= 32 && threadIdx.x < 64 && use_commit) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(smem_u32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  long long t0 = clock64();
  if (warp == 0 && lane == 0) {
    uint32_t st = 0, ph = 0;
    for (int i = 0; i < iters; ++i) {
      if (mode == 1) wait_test(smem_u32(&empty[st]), ph ^ 1); else wait_try(smem_u32(&empty[st]), ph ^ 1);
      arrive(smem_u32(&full[st]));
      if (++st == (uint32_t)ST) { st = 0; ph ^= 1; }
    }
  } else if (warp == 1 && lane == 0) {
    uint32_t st = 0, ph = 0;
    for (int i = 0; i < iters; ++i) {
      if (mode == 1) wait_test(smem_u32(&full[st]), ph); else wait_try(smem_u32(&full[st]), ph);
      if (use_commit)
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                         smem_u32(&empty[st]))
                     : "memory");
      else
        arrive(smem_u32(&empty[st]));
      if (++st == (uint32_t)ST) { st = 0; ph ^= 1; }
    }
    if (blockIdx.x == 0) out[0] = clock64() - t0;
    arrive(smem_u32(&never));  // release the spinning warps
  } else if (warp >= 2) {
    // extra warps spinning on a barrier (like epilogue warps waiting for an accumulator)
    if (mode == 2) { uint32_t ok = 0; while (!ok) { asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\nselp.b32 %0, 1, 0, p;\n}\n" : "=r"(ok) : "r"(smem_u32(&never)) : "memory"); if (!ok) __nanosleep(200); } }
    else wait_try(smem_u32(&never), 0);
  }
  __syncthreads();
  if (threadIdx.x >= 32 && threadIdx.x < 64 && use_commit)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tslot));
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 8);
  for (int extra : {0, 4, 10})
  for (int commit : {1})
    for (int mode : {0, 2})
      for (int ST : {4}) {
        int iters = 4096;
        ring_kernel<<<148, 64 + 32 * extra>>>(iters, ST, mode, commit, d);
        ring_kernel<<<148, 64 + 32 * extra>>>(iters, ST, mode, commit, d);
        cudaDeviceSynchronize();
        unsigned long long h;
        cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
        printf("extra spinning warps %2d, spin %s ST=%d: %.1f cycles / iteration  %s\n", extra,
               mode == 2 ? "try+nanosleep" : "try_wait     ", ST, (double)h / iters, cudaGetErrorString(cudaGetLastError()));
      }
  return 0;
}
