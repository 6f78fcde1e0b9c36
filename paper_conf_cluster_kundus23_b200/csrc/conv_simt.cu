// conv_simt.cu -- fp32 implicit-GEMM convolution on CUDA cores (FFMA), the
// fp32 path (the north star's 1e-4 parity bar; TF32 tensor cores would not
// meet it).
//
// GEMM view M = output pixels, N = output channels, K = R*S*C walked as
// (tap (r, s), 16-channel chunk): for a fixed tap, the 16 channels of one input
// pixel are contiguous in NHWC, so an A-tile row is 4 float4 loads and no
// per-element index arithmetic (no div/mod in the K loop).  Weights are laid
// out [K][R*S][Cp] with Cp = C rounded up to 16 and zero-padded, so a B-tile
// row is 4 aligned float4 loads too.  CTA tile 128 x 128 x 16, 256 threads,
// 8 x 8 outputs per thread: per k, two LDS.128 of A and two of B feed 64 FFMA
// (FFMA-bound, not shared-memory bound); double-buffered shared tiles with the
// next chunk's global loads in flight under the current chunk's FFMAs.
// Roofline: 2*K*C*R*S*P*Q FLOP at the measured FP32 CUDA-core peak
// (tools/fp32_peak.cu: 72.5 TFLOP/s on B200).
#include "kernels.cuh"

namespace hios {

constexpr int SBK = 16, SPAD = 4;

// BT x BT CTA tile (BT = 128: 8 x 8 outputs per thread; BT = 64: 4 x 4, for
// convs whose 128-tiles would leave most SMs idle -- small spatial extents)
template <int BT>
__global__ void __launch_bounds__(256) conv_simt_kernel(const ConvSimtArgs a) {
  constexpr int SBM = BT, SBN = BT, TT = BT / 16, HALF = BT / 2;  // TT outputs per thread per dim
  pdl_enter();
  __shared__ __align__(16) float As[2][SBK][SBM + SPAD];
  __shared__ __align__(16) float Bs[2][SBK][SBN + SPAD];
  const int t = threadIdx.x, tx = t & 15, ty = t >> 4;
  const int m0 = blockIdx.x * SBM, n0 = blockIdx.y * SBN;
  const int M = a.P * a.Q, RS = a.R * a.S, Cp = (a.C + 15) & ~15, nch = Cp >> 4;
  // loads: 128 rows x 16 k = 512 float4 per operand, two per thread: rows
  // t >> 2 and 64 + (t >> 2), channel quad (t & 3) * 4
  constexpr int NL = BT / 64;  // float4 loads per operand per thread
  const int lrow = t >> 2, lq = (t & 3) * 4;
  int ih[NL], iw[NL];
  bool mval[NL];
#pragma unroll
  for (int i = 0; i < NL; ++i) {
    const int m = m0 + lrow + 64 * i;
    mval[i] = m < M;
    const int p = mval[i] ? m / a.Q : 0, q = mval[i] ? m - (m / a.Q) * a.Q : 0;
    ih[i] = p * a.sh - a.ph;
    iw[i] = q * a.sw - a.pw;
  }
  bool nval[NL];
  const float* wrow[NL];
#pragma unroll
  for (int i = 0; i < NL; ++i) {
    const int n = n0 + lrow + 64 * i;
    nval[i] = n < a.K;
    wrow[i] = a.w + (size_t)(nval[i] ? n : 0) * RS * Cp;
  }
  float acc[TT][TT];
#pragma unroll
  for (int i = 0; i < TT; ++i)
#pragma unroll
    for (int j = 0; j < TT; ++j) acc[i][j] = 0.f;

  float4 ra[NL], rb[NL];
  auto gload = [&](int rs, int c0) {
    const int r = rs / a.S, s = rs - r * a.S;  // once per 16-channel chunk
    const int c = c0 + lq;
#pragma unroll
    for (int i = 0; i < NL; ++i) {
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      const int h = ih[i] + r * a.dh, w = iw[i] + s * a.dw;
      if (mval[i] && h >= 0 && h < a.H && w >= 0 && w < a.W) {
        const float* px = a.x + ((size_t)h * a.W + w) * a.ldx;
        if (c + 4 <= a.C) {
          v = __ldg(reinterpret_cast<const float4*>(px + c));
        } else {
          if (c < a.C) v.x = __ldg(px + c);
          if (c + 1 < a.C) v.y = __ldg(px + c + 1);
          if (c + 2 < a.C) v.z = __ldg(px + c + 2);
        }
      }
      ra[i] = v;
      rb[i] = nval[i] ? __ldg(reinterpret_cast<const float4*>(wrow[i] + (size_t)rs * Cp + c))
                      : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  };
  auto sstore = [&](int buf) {
#pragma unroll
    for (int i = 0; i < NL; ++i) {
      const int row = lrow + 64 * i;
      As[buf][lq + 0][row] = ra[i].x;
      As[buf][lq + 1][row] = ra[i].y;
      As[buf][lq + 2][row] = ra[i].z;
      As[buf][lq + 3][row] = ra[i].w;
      Bs[buf][lq + 0][row] = rb[i].x;
      Bs[buf][lq + 1][row] = rb[i].y;
      Bs[buf][lq + 2][row] = rb[i].z;
      Bs[buf][lq + 3][row] = rb[i].w;
    }
  };
  const int nsteps = RS * nch;
  gload(0, 0);
  sstore(0);
  __syncthreads();
  int buf = 0, rs = 0, ch = 0;
  for (int step = 0; step < nsteps; ++step) {
    const bool more = step + 1 < nsteps;
    if (more) {
      if (++ch == nch) { ch = 0; ++rs; }
      gload(rs, ch * 16);
    }
#pragma unroll
    for (int kk = 0; kk < SBK; ++kk) {
      float av[TT], bv[TT];
#pragma unroll
      for (int h = 0; h < TT / 4; ++h) {  // float4 groups at rows h * HALF + ty * 4
        const float4 a4 = *reinterpret_cast<const float4*>(&As[buf][kk][h * HALF + ty * 4]);
        const float4 b4 = *reinterpret_cast<const float4*>(&Bs[buf][kk][h * HALF + tx * 4]);
        av[4 * h] = a4.x; av[4 * h + 1] = a4.y; av[4 * h + 2] = a4.z; av[4 * h + 3] = a4.w;
        bv[4 * h] = b4.x; bv[4 * h + 1] = b4.y; bv[4 * h + 2] = b4.z; bv[4 * h + 3] = b4.w;
      }
#pragma unroll
      for (int i = 0; i < TT; ++i)
#pragma unroll
        for (int j = 0; j < TT; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    if (more) {
      sstore(buf ^ 1);
      __syncthreads();
      buf ^= 1;
    }
  }
  // epilogue: rows (i / 4) * HALF + ty * 4 + i % 4; columns likewise
#pragma unroll
  for (int i = 0; i < TT; ++i) {
    const int m = m0 + (i / 4) * HALF + ty * 4 + (i % 4);
    if (m >= M) continue;
#pragma unroll
    for (int h2 = 0; h2 < TT / 4; ++h2) {
      const int nb = n0 + h2 * HALF + tx * 4;
      float y[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int n = min(nb + j, a.K - 1);
        y[j] = acc[i][h2 * 4 + j] * __ldg(a.scale + n) + __ldg(a.shift + n);
        if (a.relu) y[j] = fmaxf(y[j], 0.f);
      }
      float* o = a.out + (size_t)m * a.ldo;
      if (nb + 4 <= a.K && ((a.ldo | nb) & 3) == 0 && (reinterpret_cast<uintptr_t>(a.out) & 15) == 0) {
        *reinterpret_cast<float4*>(o + nb) = make_float4(y[0], y[1], y[2], y[3]);
      } else {
        for (int j = 0; j < 4 && nb + j < a.K; ++j) o[nb + j] = y[j];
      }
      for (int d_ = 0; d_ < a.out2.n; ++d_) {
        float* o2 = a.out2.p[d_] + (size_t)m * a.out2.ld[d_];
        for (int j = 0; j < 4 && nb + j < a.K; ++j) o2[nb + j] = y[j];
      }
    }
  }
}

void launch_conv_simt(const ConvSimtArgs& a, cudaStream_t st) {
  const int M = a.P * a.Q;
  const long long big = (long long)((M + 127) / 128) * ((a.K + 127) / 128);
  if (big >= 148) {
    dim3 grid((M + 127) / 128, (a.K + 127) / 128);
    launch_pdl(conv_simt_kernel<128>, grid, dim3(256), 0, st, a);
  } else {  // small spatial extent: 64-tiles give 4x the CTAs
    dim3 grid((M + 63) / 64, (a.K + 63) / 64);
    launch_pdl(conv_simt_kernel<64>, grid, dim3(256), 0, st, a);
  }
}

}  // namespace hios
