// conv_simt.cu -- fp32 implicit-GEMM convolution on CUDA cores (FFMA).
// The fp32 path exists for the 1e-4 parity bar (north star); TF32 tensor
// cores would not meet it (SURVEY §7 "fp32 parity at 1e-4 rules out TF32").
// 64 pixels x 64 out-channels per CTA, K = R*S*C in steps of 16, 256 threads,
// 4 x 4 outputs per thread, double-buffered smem tiles.
#include "kernels.cuh"

namespace hios {

constexpr int SBM = 64, SBN = 64, SBK = 16;

__global__ void __launch_bounds__(256) conv_simt_kernel(const ConvSimtArgs a) {
  pdl_enter();
  __shared__ float As[2][SBK][SBM + 4];
  __shared__ float Bs[2][SBK][SBN + 4];
  const int t = threadIdx.x, tx = t & 15, ty = t >> 4;
  const int m0 = blockIdx.x * SBM, n0 = blockIdx.y * SBN;
  const int M = a.P * a.Q, RSC = a.R * a.S * a.C;
  // each thread loads 4 A elements and 4 B elements per K step: k = e % 16, row = e / 16
  int am[4], aih[4], aiw[4];
  bool avalid[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int e = t + i * 256, row = e >> 4;
    const int m = m0 + row;
    avalid[i] = m < M;
    const int p = avalid[i] ? m / a.Q : 0, q = avalid[i] ? m % a.Q : 0;
    am[i] = m;
    aih[i] = p * a.sh - a.ph;
    aiw[i] = q * a.sw - a.pw;
  }
  float acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;

  float ra[4], rb[4];
  auto gload = [&](int k0) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int e = t + i * 256, k = e & 15, row = e >> 4;
      const int kg = k0 + k;
      float v = 0.f;
      if (avalid[i] && kg < RSC) {
        const int rs = kg / a.C, c = kg - rs * a.C;
        const int r = rs / a.S, s = rs - r * a.S;
        const int h = aih[i] + r * a.dh, w = aiw[i] + s * a.dw;
        if (h >= 0 && h < a.H && w >= 0 && w < a.W) v = __ldg(a.x + ((size_t)h * a.W + w) * a.ldx + c);
      }
      ra[i] = v;
      const int n = n0 + row;
      rb[i] = (n < a.K && kg < RSC) ? __ldg(a.w + (size_t)n * RSC + kg) : 0.f;
    }
  };
  auto sstore = [&](int buf) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int e = t + i * 256, k = e & 15, row = e >> 4;
      As[buf][k][row] = ra[i];
      Bs[buf][k][row] = rb[i];
    }
  };
  gload(0);
  sstore(0);
  __syncthreads();
  int buf = 0;
  for (int k0 = 0; k0 < RSC; k0 += SBK) {
    const bool more = k0 + SBK < RSC;
    if (more) gload(k0 + SBK);
#pragma unroll
    for (int kk = 0; kk < SBK; ++kk) {
      float av[4], bv[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) av[i] = As[buf][kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) bv[j] = Bs[buf][kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    if (more) {
      sstore(buf ^ 1);
      __syncthreads();
      buf ^= 1;
    }
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int m = m0 + ty * 4 + i;
    if (m >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = n0 + tx * 4 + j;
      if (n >= a.K) continue;
      float y = acc[i][j] * a.scale[n] + a.shift[n];
      if (a.relu) y = fmaxf(y, 0.f);
      a.out[(size_t)m * a.ldo + n] = y;
      for (int d_ = 0; d_ < a.out2.n; ++d_) a.out2.p[d_][(size_t)m * a.out2.ld[d_] + n] = y;
    }
  }
}

void launch_conv_simt(const ConvSimtArgs& a, cudaStream_t st) {
  dim3 grid((a.P * a.Q + SBM - 1) / SBM, (a.K + SBN - 1) / SBN);
  launch_pdl(conv_simt_kernel, grid, dim3(256), 0, st, a);
}

}  // namespace hios
