// FP32 CUDA-core peak on this GPU (the denominator of the fp32 path's
// roofline: "the measured FP32 SIMT peak for fp32").  Every
// thread runs 8 independent FFMA chains (enough ILP to cover the 4-cycle FMA
// latency at 4 warps per scheduler); 2 FLOP per FFMA.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fp32_peak tools/fp32_peak.cu && /tmp/fp32_peak
#include <cstdio>
#include <cuda_runtime.h>

__global__ void ffma_kernel(float* out, int iters, float a, float b) {
  float x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      x0 = fmaf(x0, a, b); x1 = fmaf(x1, a, b); x2 = fmaf(x2, a, b); x3 = fmaf(x3, a, b);
      x4 = fmaf(x4, a, b); x5 = fmaf(x5, a, b); x6 = fmaf(x6, a, b); x7 = fmaf(x7, a, b);
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

int main() {
  int sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int threads = 512, blocks = sms * 4, iters = 4096;
  float* out;
  cudaMalloc(&out, sizeof(float) * threads * blocks);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e30f;
  for (int r = 0; r < 6; ++r) {
    cudaEventRecord(e0);
    ffma_kernel<<<blocks, threads>>>(out, iters, 0.999f, 0.001f);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (r > 0 && ms < best) best = ms;
  }
  const double flop = 2.0 * 8 * 16 * (double)iters * threads * blocks;
  printf("{\"fp32_tflops\": %.2f, \"sms\": %d, \"clock_mhz_attr\": %d, \"nominal_tflops_at_attr_clock\": %.2f, "
         "\"ms\": %.3f}\n",
         flop / (best * 1e-3) / 1e12, sms, clk / 1000, 2.0 * 128 * sms * (clk * 1e3) / 1e12, best);
  return 0;
}
