// tma_bench.cu -- standalone micro-benchmark: per-SM TMA load throughput for
// the box shapes the conv kernel uses.  One CTA per SM; thread 0 keeps
// `depth` TMA loads in flight through a ring of smem slots (mbarrier per slot)
// and streams `iters` boxes; reports bytes / cycle / SM and GB/s chip-wide.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_bench tma_bench.cu
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

typedef CUresult (*PFN_encodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                     const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                     CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void tma_kernel(const __grid_constant__ CUtensorMap m, int iters, int depth, uint32_t box_bytes,
                           int n1, int n2, unsigned long long* cycles, int lanes_mode) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)raw + 1023) & ~(uintptr_t)1023);
  uint64_t* bars = (uint64_t*)(sm + depth * box_bytes);
  if (threadIdx.x == 0) {
    for (int i = 0; i < depth; ++i)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bars + i)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  // `issuers` warps (lane 0 each) share the ring: warp w handles slots w, w+issuers, ...
  // warps mode: lane 0 of each warp issues; lanes mode: lanes 0..k-1 of warp 0
  const int issuers = lanes_mode ? lanes_mode : blockDim.x / 32;
  int w;
  if (lanes_mode) { if (threadIdx.x >= lanes_mode) return; w = threadIdx.x; }
  else { if ((threadIdx.x & 31) != 0) return; w = threadIdx.x >> 5; }
  long long t0 = clock64();
  uint32_t ph = 0;
  for (int it = w; it < iters; it += issuers) {
    int slot = it % depth;
    if (it >= depth) {
      uint32_t par = ((it / depth) - 1) & 1;
      asm volatile(
          "{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
              smem_u32(bars + slot)),
          "r"(par)
          : "memory");
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bars + slot)), "r"(box_bytes)
                 : "memory");
    int c1 = (blockIdx.x * 7 + it) % n1, c2 = (it / n1) % n2;
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(
            smem_u32(sm + slot * box_bytes)),
        "l"((uint64_t)&m), "r"(smem_u32(bars + slot)), "r"(0), "r"(c1), "r"(c2)
        : "memory");
  }
  for (int it = iters + w; it < iters + depth; it += issuers) {
    int slot = it % depth;
    uint32_t par = ((it / depth) - 1) & 1;
    asm volatile(
        "{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
            smem_u32(bars + slot)),
        "r"(par)
        : "memory");
  }
  (void)ph;
  if (w == 0) cycles[blockIdx.x] = clock64() - t0;
}

int main() {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  PFN_encodeTiled enc = (PFN_encodeTiled)p;
  // 2048 channels x 64 x 64 pixels bf16 activation (like a deep NHWC layer), 16 MB
  const int C = 2048, W = 512, H = 64;
  void* buf;
  cudaMalloc(&buf, (size_t)C * W * H * 2);
  cudaMemset(buf, 0, (size_t)C * W * H * 2);
  unsigned long long* cyc;
  cudaMalloc(&cyc, 148 * 8);
  cudaFuncSetAttribute(tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
  struct Cfg { const char* name; int b1, b2; uint32_t C_dim; int es1 = 1; };
  std::vector<Cfg> cfgs = {{"box {64,128,1} 16KB", 128, 1, (uint32_t)C},
                           {"box {64,32,1} 4KB", 32, 1, (uint32_t)C},
                           {"box {64,64,2} 16KB", 64, 2, (uint32_t)C},
                           {"box {64,128,2} 32KB", 128, 2, (uint32_t)C},
                           {"box {64,128,1} 16KB C=40", 128, 1, 40u},
                           {"box {64,256/2,1} 16KB es2", 256, 1, (uint32_t)C, 2},
                           {"box {64,256/2,1} es2 C=40", 256, 1, 40u, 2},
                           {"box {64,64,8} 64KB", 64, 8, (uint32_t)C}};
  for (auto& c : cfgs) {
    for (int depth : {8}) for (int lm : {0}) for (int issuers : {1, 2, 4}) {
      if (issuers > depth) continue;
      if (!lm && issuers > 4) continue;
      CUtensorMap m;
      cuuint64_t dims[3] = {c.C_dim, (cuuint64_t)W, (cuuint64_t)H};
      cuuint64_t strides[2] = {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2};
      cuuint32_t box[3] = {64, (cuuint32_t)c.b1, (cuuint32_t)c.b2};
      cuuint32_t es[3] = {1, (cuuint32_t)c.es1, 1};
      CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, buf, dims, strides, box, es,
                       CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) { printf("encode failed %d\n", r); continue; }
      uint32_t bytes = 128u * (c.b1 / c.es1) * c.b2;
      if ((size_t)depth * bytes > 200 * 1024) continue;
      size_t smem = 1024 + depth * bytes + depth * 8;
      int iters = 400;
      int n1 = W / c.b1 > 0 ? W - c.b1 + 1 : 1, n2 = H - c.b2 + 1;
      const int thr = lm ? 32 : 32 * issuers, lmode = lm ? issuers : 0;
      tma_kernel<<<148, thr, smem>>>(m, 20 * issuers, depth, bytes, n1, n2, cyc, lmode);  // warm
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      cudaEventRecord(e0);
      tma_kernel<<<148, thr, smem>>>(m, iters, depth, bytes, n1, n2, cyc, lmode);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      std::vector<unsigned long long> h(148);
      cudaMemcpy(h.data(), cyc, 148 * 8, cudaMemcpyDeviceToHost);
      double avg = 0;
      for (auto v : h) avg += v;
      avg /= 148;
      printf("%-40s depth %d %s %d: %6.1f B/cycle/SM, %7.1f GB/s chip (%.1f us), err=%s\n", c.name, depth, lm ? "lanes" : "warps", issuers,
             (double)bytes * iters / avg, (double)bytes * iters * 148 / (ms * 1e-3) / 1e9, ms * 1e3,
             cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
