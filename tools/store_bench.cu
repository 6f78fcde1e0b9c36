// store_bench.cu -- diagnostic: write bandwidth of the conv epilogue's store
// patterns on this GPU.  128 threads per CTA, one CTA per SM (148), each CTA
// writes `tiles` tiles of 128 pixel rows x NB bytes (row pitch = NB, i.e. a
// dense NHWC tensor):
//   scatter16 / scatter32: thread = one pixel row, 16- / 32-byte vector stores
//     along its own row (the direct-store epilogue, conv_tc epi 2)
//   coalesced: consecutive threads store consecutive 16 bytes of the tile
//     (what a warp-staged copy-out or a bulk store would issue)
//   nb_kernel: the same bytes as one cp.async.bulk (smem -> global) per warp
//     row block
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/store_bench tools/store_bench.cu && /tmp/store_bench
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

template <int NB>
__global__ void __launch_bounds__(128) scatter16(uint4* out, int tiles) {
  for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
    char* base = reinterpret_cast<char*>(out) + (size_t)t * 128 * NB + (size_t)threadIdx.x * NB;
#pragma unroll
    for (int c = 0; c < NB; c += 16) *reinterpret_cast<uint4*>(base + c) = make_uint4(t, c, 1, 2);
  }
}

template <int NB>
__global__ void __launch_bounds__(128) scatter32(uint4* out, int tiles) {
  for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
    char* base = reinterpret_cast<char*>(out) + (size_t)t * 128 * NB + (size_t)threadIdx.x * NB;
#pragma unroll
    for (int c = 0; c < NB; c += 32)
      asm volatile("st.global.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(base + c), "r"(t), "r"(c), "r"(1),
                   "r"(2), "r"(3), "r"(4), "r"(5), "r"(6)
                   : "memory");
  }
}

template <int NB>
__global__ void __launch_bounds__(128) coalesced(uint4* out, int tiles) {
  for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
    uint4* base = reinterpret_cast<uint4*>(reinterpret_cast<char*>(out) + (size_t)t * 128 * NB);
#pragma unroll
    for (int i = threadIdx.x; i < 128 * NB / 16; i += 128) base[i] = make_uint4(t, i, 1, 2);
  }
}

template <int NB>
__global__ void __launch_bounds__(128) bulk(uint4* out, int tiles) {
  __shared__ __align__(128) uint4 buf[128 * NB / 16];
  for (int i = threadIdx.x; i < 128 * NB / 16; i += 128) buf[i] = make_uint4(i, 0, 1, 2);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
    if (lane == 0) {
      char* dst = reinterpret_cast<char*>(out) + (size_t)t * 128 * NB + (size_t)warp * 32 * NB;
      const uint32_t src = static_cast<uint32_t>(__cvta_generic_to_shared(buf)) + warp * 32 * NB;
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src), "r"(32 * NB)
                   : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group.read 4;" ::: "memory");
    }
    __syncwarp();
  }
  if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

template <typename K>
static void run(const char* name, K k, int nb, uint4* d, int tiles) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) k<<<148, 128>>>(d, tiles);
  cudaEventRecord(a);
  const int reps = 10;
  for (int i = 0; i < reps; ++i) k<<<148, 128>>>(d, tiles);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  const double bytes = (double)tiles * 128 * nb;
  printf("%-10s NB=%4d: %7.2f us per launch, %6.0f GB/s, %.2f us per tile per CTA\n", name, nb, ms * 1e3 / reps,
         bytes * reps / (ms * 1e-3) / 1e9, ms * 1e3 / reps / ((double)tiles / 148));
}

int main() {
  const int tiles = 148 * 64;
  uint4* d;
  cudaMalloc(&d, (size_t)tiles * 128 * 512);
  run("scatter16", scatter16<128>, 128, d, tiles);
  run("scatter32", scatter32<128>, 128, d, tiles);
  run("coalesced", coalesced<128>, 128, d, tiles);
  run("bulk", bulk<128>, 128, d, tiles);
  run("scatter16", scatter16<256>, 256, d, tiles);
  run("scatter32", scatter32<256>, 256, d, tiles);
  run("coalesced", coalesced<256>, 256, d, tiles);
  run("bulk", bulk<256>, 256, d, tiles);
  run("scatter16", scatter16<64>, 64, d, tiles);
  run("scatter32", scatter32<64>, 64, d, tiles);
  run("coalesced", coalesced<64>, 64, d, tiles);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
  return 0;
}
