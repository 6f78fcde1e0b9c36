// launch_floor.cu -- diagnostic: the per-kernel floor of a chain of dependent
// kernels replayed from one CUDA graph on this GPU (what a batch-1 DAG step of
// ~120 dependent operators pays before any work), with and without
// programmatic dependent launch (PDL), for 1 / 148 / 296 CTAs of 128 / 384
// threads, optionally with a dynamic smem request like conv_tc's (212 KB).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/launch_floor tools/launch_floor.cu && /tmp/launch_floor
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_empty(int* p) {
  if (p && threadIdx.x == 0 && blockIdx.x == 0) p[0] += 1;
}
__global__ void k_pdl(int* p) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (p && threadIdx.x == 0 && blockIdx.x == 0) p[0] += 1;
}

static float run(int n, int grid, int block, size_t smem, bool pdl) {
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  int* d;
  cudaMalloc(&d, 4);
  if (smem > 48 * 1024) {
    cudaFuncSetAttribute(k_empty, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_pdl, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  }
  cudaGraph_t g;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeRelaxed);
  for (int i = 0; i < n; ++i) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl ? 1 : 0;
    if (pdl) cudaLaunchKernelEx(&cfg, k_pdl, d);
    else cudaLaunchKernelEx(&cfg, k_empty, d);
  }
  cudaStreamEndCapture(s, &g);
  cudaGraphExec_t ge;
  if (cudaGraphInstantiate(&ge, g, 0) != cudaSuccess) { printf("instantiate failed\n"); return -1; }
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) cudaGraphLaunch(ge, s);
  float best = 1e30f;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(a, s);
    cudaGraphLaunch(ge, s);
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (ms < best) best = ms;
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
  cudaGraphExecDestroy(ge);
  cudaGraphDestroy(g);
  cudaFree(d);
  cudaStreamDestroy(s);
  return best * 1000.f / n;
}

int main() {
  const int n = 200;
  for (int pdl = 0; pdl < 2; ++pdl)
    for (int grid : {1, 148, 296})
      for (int block : {128, 384})
        for (size_t smem : {(size_t)0, (size_t)212 * 1024}) {
          float us = run(n, grid, block, smem, pdl != 0);
          printf("pdl=%d grid=%3d block=%3d smem=%6zu: %.2f us per kernel\n", pdl, grid, block, smem, us);
        }
  return 0;
}
