// misc.cu -- HBM-bound operator kernels: pooling, depthwise
// stage of separable convs, n-ary add, copy (concat fallback and peer pushes),
// GAP, linear head, input/output layout conversion, and the epoch flags used
// for cross-GPU edges (a10/a11).  NHWC with a pixel stride; each thread owns
// one pixel x VEC channels (16-byte vectors: 8 bf16 or 4 fp32) so a warp reads
// contiguous 512-byte runs.
#include <cstdio>
#include <algorithm>
#include <type_traits>

#include "kernels.cuh"

namespace hios {

template <typename T> struct Vec;
template <> struct Vec<float> { static constexpr int N = 4; };
template <> struct Vec<bf16> { static constexpr int N = 8; };

__device__ __forceinline__ float to_f(float x) { return x; }
__device__ __forceinline__ float to_f(bf16 x) { return __bfloat162float(x); }
template <typename T> __device__ __forceinline__ T from_f(float x);
template <> __device__ __forceinline__ float from_f<float>(float x) { return x; }
template <> __device__ __forceinline__ bf16 from_f<bf16>(float x) { return __float2bfloat16_rn(x); }

// load VEC channels starting at c (vector path when fully inside, else scalar)
template <typename T>
__device__ __forceinline__ void load_vec(const T* p, int c, int C, float* v) {
  constexpr int N = Vec<T>::N;
  if (c + N <= C) {
    uint4 raw = *reinterpret_cast<const uint4*>(p);
    const T* e = reinterpret_cast<const T*>(&raw);
#pragma unroll
    for (int j = 0; j < N; ++j) v[j] = to_f(e[j]);
  } else {
#pragma unroll
    for (int j = 0; j < N; ++j) v[j] = (c + j < C) ? to_f(p[j]) : 0.f;
  }
}
template <typename T>
__device__ __forceinline__ void store_vec(T* p, int c, int C, const float* v) {
  constexpr int N = Vec<T>::N;
  if (c + N <= C) {
    uint4 raw;
    T* e = reinterpret_cast<T*>(&raw);
#pragma unroll
    for (int j = 0; j < N; ++j) e[j] = from_f<T>(v[j]);
    *reinterpret_cast<uint4*>(p) = raw;
  } else {
    for (int j = 0; j < N && c + j < C; ++j) p[j] = from_f<T>(v[j]);
  }
}

// 8 channels (one 16-byte bf16 vector, two 16-byte fp32 vectors)
template <typename T>
__device__ __forceinline__ void load8(const T* p, int c, int C, float* v) {
#pragma unroll
  for (int h = 0; h < 8; h += Vec<T>::N) load_vec(p + h, c + h, C, v + h);
}
template <typename T>
__device__ __forceinline__ void store8(T* p, int c, int C, const float* v) {
#pragma unroll
  for (int h = 0; h < 8; h += Vec<T>::N)
    if (c + h < C) store_vec(p + h, c + h, C, v + h);
}

// mixed-precision bf16 x fp32 arithmetic (sm_100: FHFMA.BF16 / FHADD.BF16 read
// either bf16 half of a register directly -- no conversions)
__device__ __forceinline__ float fma_bf16_lo(uint32_t x, uint32_t w, float c) {
  float d;
  asm("{\n.reg .b16 xl, xh, wl, wh;\nmov.b32 {xl, xh}, %1;\nmov.b32 {wl, wh}, %2;\n"
      "fma.rn.f32.bf16 %0, xl, wl, %3;\n}\n" : "=f"(d) : "r"(x), "r"(w), "f"(c));
  return d;
}
__device__ __forceinline__ float fma_bf16_hi(uint32_t x, uint32_t w, float c) {
  float d;
  asm("{\n.reg .b16 xl, xh, wl, wh;\nmov.b32 {xl, xh}, %1;\nmov.b32 {wl, wh}, %2;\n"
      "fma.rn.f32.bf16 %0, xh, wh, %3;\n}\n" : "=f"(d) : "r"(x), "r"(w), "f"(c));
  return d;
}

__device__ __forceinline__ float add_bf16_lo(uint32_t x, float c) {
  float d;
  asm("{\n.reg .b16 xl, xh;\nmov.b32 {xl, xh}, %1;\nadd.rn.f32.bf16 %0, xl, %2;\n}\n" : "=f"(d) : "r"(x), "f"(c));
  return d;
}
__device__ __forceinline__ float add_bf16_hi(uint32_t x, float c) {
  float d;
  asm("{\n.reg .b16 xl, xh;\nmov.b32 {xl, xh}, %1;\nadd.rn.f32.bf16 %0, xh, %2;\n}\n" : "=f"(d) : "r"(x), "f"(c));
  return d;
}

static inline unsigned grid_for(long long n, int block) {
  long long g = (n + block - 1) / block;
  return (unsigned)(g < 1 ? 1 : g);
}

// ---------------------------------------------------------------- pooling
// grid = (ceil(Q * CG / 256), P): one output row per blockIdx.y; KH/KW > 0
// unroll the window (loads hoisted, accumulated immediately).
// (<= 64 registers: four 256-thread CTAs per SM; measured 66 registers
// limited the 3x3 stride-2 max pools at 4096^2 to 37.5 % occupancy)
template <typename T, int KH, int KW>
__global__ void __launch_bounds__(256, 4) pool_kernel(const PoolArgs<T> a) {
  pdl_enter();
  constexpr int N = Vec<T>::N;
  const int kh = KH > 0 ? KH : a.kh, kw = KW > 0 ? KW : a.kw;
  const int CG = (a.C + N - 1) / N;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= a.Q * CG) return;
  const int p = blockIdx.y;
  const int q = idx / CG, cg = idx - q * CG;
  const int c = cg * N;
  const int h0 = p * a.sh - a.ph, w0 = q * a.sw - a.pw;
  if constexpr (std::is_same<T, bf16>::value && KH == 3 && KW == 3) {
    if (a.is_max && c + 8 <= a.C) {
      // bf16 3x3 max, whole vector: all in-bounds taps' loads issued first,
      // then packed __hmax2 (exact in bf16; no conversions)
      uint4 u[9];
      bool ok[9];
#pragma unroll
      for (int t = 0; t < 9; ++t) {
        const int h = h0 + t / 3, w = w0 + t % 3;
        ok[t] = h >= 0 && h < a.H && w >= 0 && w < a.W;
        if (ok[t]) u[t] = __ldg(reinterpret_cast<const uint4*>(a.x + ((size_t)h * a.W + w) * a.ldx + c));
      }
      __nv_bfloat162 m[4];
      const __nv_bfloat162 ninf = __floats2bfloat162_rn(-INFINITY, -INFINITY);
#pragma unroll
      for (int j = 0; j < 4; ++j) m[j] = ninf;
#pragma unroll
      for (int t = 0; t < 9; ++t) {
        if (!ok[t]) continue;
        const __nv_bfloat162* b = reinterpret_cast<const __nv_bfloat162*>(&u[t]);
#pragma unroll
        for (int j = 0; j < 4; ++j) m[j] = __hmax2(m[j], b[j]);
      }
      const size_t pix = (size_t)p * a.Q + q;
      const uint4 o = *reinterpret_cast<const uint4*>(m);
      *reinterpret_cast<uint4*>(a.out + pix * a.ldo + c) = o;
      for (int d_ = 0; d_ < a.out2.n; ++d_) *reinterpret_cast<uint4*>(a.out2.p[d_] + pix * a.out2.ld[d_] + c) = o;
      return;
    }
    if (!a.is_max && c + 8 <= a.C) {
      // bf16 3x3 average: loads first, then FHADD.BF16 into fp32
      uint4 u[9];
      bool ok[9];
#pragma unroll
      for (int t = 0; t < 9; ++t) {
        const int h = h0 + t / 3, w = w0 + t % 3;
        ok[t] = h >= 0 && h < a.H && w >= 0 && w < a.W;
        if (ok[t]) u[t] = __ldg(reinterpret_cast<const uint4*>(a.x + ((size_t)h * a.W + w) * a.ldx + c));
      }
      float acc[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[j] = 0.f;
#pragma unroll
      for (int t = 0; t < 9; ++t) {
        if (!ok[t]) continue;
        acc[0] = add_bf16_lo(u[t].x, acc[0]); acc[1] = add_bf16_hi(u[t].x, acc[1]);
        acc[2] = add_bf16_lo(u[t].y, acc[2]); acc[3] = add_bf16_hi(u[t].y, acc[3]);
        acc[4] = add_bf16_lo(u[t].z, acc[4]); acc[5] = add_bf16_hi(u[t].z, acc[5]);
        acc[6] = add_bf16_lo(u[t].w, acc[6]); acc[7] = add_bf16_hi(u[t].w, acc[7]);
      }
      int div;
      if (a.cip) div = (min(h0 + 3, a.H + a.ph) - h0) * (min(w0 + 3, a.W + a.pw) - w0);
      else div = (min(h0 + 3, a.H) - max(h0, 0)) * (min(w0 + 3, a.W) - max(w0, 0));
      const float inv = 1.f / (float)div;
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[j] *= inv;
      const size_t pix = (size_t)p * a.Q + q;
      store8(a.out + pix * a.ldo + c, c, a.C, acc);
      for (int d_ = 0; d_ < a.out2.n; ++d_) store8(a.out2.p[d_] + pix * a.out2.ld[d_] + c, c, a.C, acc);
      return;
    }
  }
  float acc[N], v[N];
#pragma unroll
  for (int j = 0; j < N; ++j) acc[j] = a.is_max ? -INFINITY : 0.f;
  int cnt = 0;
#pragma unroll
  for (int r = 0; r < (KH > 0 ? KH : 1); ++r) {
    for (int r2 = 0; r2 < (KH > 0 ? 1 : kh); ++r2) {
      const int h = h0 + (KH > 0 ? r : r2);
      if (h < 0 || h >= a.H) continue;
#pragma unroll
      for (int s2 = 0; s2 < (KW > 0 ? KW : 1); ++s2) {
        for (int s3 = 0; s3 < (KW > 0 ? 1 : kw); ++s3) {
          const int w = w0 + (KW > 0 ? s2 : s3);
          if (w < 0 || w >= a.W) continue;
          load_vec(a.x + ((size_t)h * a.W + w) * a.ldx + c, c, a.C, v);
          ++cnt;
#pragma unroll
          for (int j = 0; j < N; ++j) acc[j] = a.is_max ? fmaxf(acc[j], v[j]) : acc[j] + v[j];
        }
      }
    }
  }
  if (!a.is_max) {
    int div = cnt;
    if (a.cip) div = (min(h0 + kh, a.H + a.ph) - h0) * (min(w0 + kw, a.W + a.pw) - w0);
    const float inv = 1.f / (float)div;
#pragma unroll
    for (int j = 0; j < N; ++j) acc[j] *= inv;
  }
  const size_t pix = (size_t)p * a.Q + q;
  store_vec(a.out + pix * a.ldo + c, c, a.C, acc);
  for (int d_ = 0; d_ < a.out2.n; ++d_) store_vec(a.out2.p[d_] + pix * a.out2.ld[d_] + c, c, a.C, acc);
}

// Tiled pooling (same tiling as the depthwise kernel below): a CTA stages
// the input window of 8 output rows x 32 output columns x 16 channels once in
// smem (out-of-bounds = -inf for max, 0 for average; columns de-interleaved by
// parity when sw == 2), then each thread reduces its two output pixels' k x k
// windows from smem.  The average divisor is computed from the window bounds
// (count_include_pad or in-bounds count), as in pool_kernel.
constexpr int kPoolTP = 8, kPoolTQ = 32;

template <typename T, int KS>
__global__ void __launch_bounds__(256) pool_tiled_kernel(const PoolArgs<T> a) {
  extern __shared__ __align__(16) uint8_t psm[];
  constexpr int N = 8;
  constexpr int VB = N * (int)sizeof(T);
  const int kh = KS > 0 ? KS : a.kh, kw = KS > 0 ? KS : a.kw;
  const int IH = (kPoolTP - 1) * a.sh + kh, IW = (kPoolTQ - 1) * a.sw + kw;
  const int half = (IW + 1) / 2;
  // channel slab fastest in the grid: the CTAs of one spatial tile run together
  // and between them read whole pixel rows (DRAM page locality)
  const int q0 = blockIdx.y * kPoolTQ, p0 = blockIdx.z * kPoolTP, c0 = blockIdx.x * 16;
  pdl_enter();
  const int hb = p0 * a.sh - a.ph, wb = q0 * a.sw - a.pw;
  const float pad = a.is_max ? -INFINITY : 0.f;
  const int nel = 2 * IH * IW;
  for (int e = threadIdx.x; e < nel; e += blockDim.x) {
    const int cv = e & 1, pix = e >> 1;
    const int row = pix / IW, col = pix - row * IW;
    const int h = hb + row, w = wb + col, c = c0 + cv * N;
    const int pos = a.sw == 2 ? ((col & 1) * half + (col >> 1)) : col;
    T* d = reinterpret_cast<T*>(psm + ((size_t)(cv * IH + row) * IW + pos) * VB);
    const bool inb = h >= 0 && h < a.H && w >= 0 && w < a.W && c < a.C;
    if (inb && c + N <= a.C) {
      // whole vector in bounds: raw 16-byte copies, no conversions
      const uint4* src = reinterpret_cast<const uint4*>(a.x + ((size_t)h * a.W + w) * a.ldx + c);
#pragma unroll
      for (int u = 0; u < VB / 16; ++u) reinterpret_cast<uint4*>(d)[u] = src[u];
    } else {
      float v[N];
      if (inb) {
        load8(a.x + ((size_t)h * a.W + w) * a.ldx + c, c, a.C, v);
      } else {
#pragma unroll
        for (int j = 0; j < N; ++j) v[j] = pad;
      }
#pragma unroll
      for (int j = 0; j < N; ++j) d[j] = from_f<T>(v[j]);
    }
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int cv = warp & 1, pr0 = warp >> 1;
  const int q = q0 + lane, c = c0 + cv * N;
  if (q >= a.Q || c >= a.C) return;
  const uint8_t* plane = psm + (size_t)cv * IH * IW * VB;
  if constexpr (std::is_same<T, bf16>::value && KS > 0) {
    if (a.is_max) {
      // bf16 max is exact: packed __hmax2 on the staged vectors (no
      // conversions; -inf padding compares like any value)
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        const int pl = pr0 + 4 * k, p = p0 + pl;
        if (p >= a.P) break;
        __nv_bfloat162 m[4];
#pragma unroll
        for (int r = 0; r < KS; ++r) {
          const int row = pl * a.sh + r;
#pragma unroll
          for (int s2 = 0; s2 < KS; ++s2) {
            const int col = lane * a.sw + s2;
            const int pos = a.sw == 2 ? ((col & 1) * half + (col >> 1)) : col;
            const uint4 u = *reinterpret_cast<const uint4*>(plane + ((size_t)row * IW + pos) * VB);
            const __nv_bfloat162* b = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
            for (int j = 0; j < 4; ++j) m[j] = (r == 0 && s2 == 0) ? b[j] : __hmax2(m[j], b[j]);
          }
        }
        const size_t pix = (size_t)p * a.Q + q;
        const uint4 o = *reinterpret_cast<const uint4*>(m);
        if (c + 8 <= a.C) {
          *reinterpret_cast<uint4*>(a.out + pix * a.ldo + c) = o;
          for (int d_ = 0; d_ < a.out2.n; ++d_) *reinterpret_cast<uint4*>(a.out2.p[d_] + pix * a.out2.ld[d_] + c) = o;
        } else {
          const bf16* e = reinterpret_cast<const bf16*>(&o);
          for (int j = 0; j < 8 && c + j < a.C; ++j) {
            a.out[pix * a.ldo + c + j] = e[j];
            for (int d_ = 0; d_ < a.out2.n; ++d_) a.out2.p[d_][pix * a.out2.ld[d_] + c + j] = e[j];
          }
        }
      }
      return;
    }
    {
      // average: FHADD.BF16 straight from the staged bf16 pairs into fp32
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        const int pl = pr0 + 4 * k, p = p0 + pl;
        if (p >= a.P) break;
        float acc[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[j] = 0.f;
#pragma unroll
        for (int r = 0; r < KS; ++r) {
          const int row = pl * a.sh + r;
#pragma unroll
          for (int s2 = 0; s2 < KS; ++s2) {
            const int col = lane * a.sw + s2;
            const int pos = a.sw == 2 ? ((col & 1) * half + (col >> 1)) : col;
            const uint4 u = *reinterpret_cast<const uint4*>(plane + ((size_t)row * IW + pos) * VB);
            acc[0] = add_bf16_lo(u.x, acc[0]); acc[1] = add_bf16_hi(u.x, acc[1]);
            acc[2] = add_bf16_lo(u.y, acc[2]); acc[3] = add_bf16_hi(u.y, acc[3]);
            acc[4] = add_bf16_lo(u.z, acc[4]); acc[5] = add_bf16_hi(u.z, acc[5]);
            acc[6] = add_bf16_lo(u.w, acc[6]); acc[7] = add_bf16_hi(u.w, acc[7]);
          }
        }
        const int h0 = p * a.sh - a.ph, w0 = q * a.sw - a.pw;
        int div;
        if (a.cip) div = (min(h0 + kh, a.H + a.ph) - h0) * (min(w0 + kw, a.W + a.pw) - w0);
        else div = (min(h0 + kh, a.H) - max(h0, 0)) * (min(w0 + kw, a.W) - max(w0, 0));
        const float inv = 1.f / (float)div;
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[j] *= inv;
        const size_t pix = (size_t)p * a.Q + q;
        store8(a.out + pix * a.ldo + c, c, a.C, acc);
        for (int d_ = 0; d_ < a.out2.n; ++d_) store8(a.out2.p[d_] + pix * a.out2.ld[d_] + c, c, a.C, acc);
      }
      return;
    }
  }
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const int pl = pr0 + 4 * k, p = p0 + pl;
    if (p >= a.P) break;
    float acc[N];
#pragma unroll
    for (int j = 0; j < N; ++j) acc[j] = pad;
#pragma unroll
    for (int r = 0; r < (KS > 0 ? KS : 1); ++r) {
      for (int r2 = 0; r2 < (KS > 0 ? 1 : kh); ++r2) {
        const int row = pl * a.sh + (KS > 0 ? r : r2);
#pragma unroll
        for (int s2 = 0; s2 < (KS > 0 ? KS : 1); ++s2) {
          for (int s3 = 0; s3 < (KS > 0 ? 1 : kw); ++s3) {
            const int col = lane * a.sw + (KS > 0 ? s2 : s3);
            const int pos = a.sw == 2 ? ((col & 1) * half + (col >> 1)) : col;
            float v[N];
            load8(reinterpret_cast<const T*>(plane + ((size_t)row * IW + pos) * VB), 0, N, v);
#pragma unroll
            for (int j = 0; j < N; ++j) acc[j] = a.is_max ? fmaxf(acc[j], v[j]) : acc[j] + v[j];
          }
        }
      }
    }
    if (!a.is_max) {
      const int h0 = p * a.sh - a.ph, w0 = q * a.sw - a.pw;
      int div;
      if (a.cip) div = (min(h0 + kh, a.H + a.ph) - h0) * (min(w0 + kw, a.W + a.pw) - w0);
      else div = (min(h0 + kh, a.H) - max(h0, 0)) * (min(w0 + kw, a.W) - max(w0, 0));
      const float inv = 1.f / (float)div;
#pragma unroll
      for (int j = 0; j < N; ++j) acc[j] *= inv;
    }
    const size_t pix = (size_t)p * a.Q + q;
    store8(a.out + pix * a.ldo + c, c, a.C, acc);
    for (int d_ = 0; d_ < a.out2.n; ++d_) store8(a.out2.p[d_] + pix * a.out2.ld[d_] + c, c, a.C, acc);
  }
}

// 3x3 stride-1 average pool (bf16), 64-channel CTAs: a CTA stages the
// 10 x 18 input window of 8 x 16 output pixels x 64 channels (128 contiguous
// bytes per pixel: whole cache lines per load, vs 32-byte pieces in
// pool_tiled_kernel) and each thread reduces four outputs (columns lane/8 +
// 4j of row warp, channel vector lane%8) with FHADD.BF16 from smem.
// (Measured slower: four consecutive columns per thread sharing their vertical
// 3-sums -- avgpool 5d at 4096^2 75.5 -> 81.2 us, more registers.)
constexpr int kP64TP = 8, kP64TQ = 16;
__global__ void __launch_bounds__(256, 6) pool_avg64_kernel(const PoolArgs<bf16> a) {
  __shared__ __align__(16) uint4 tile[(kP64TP + 2) * (kP64TQ + 2) * 8];
  const int c0 = blockIdx.x * 64, q0 = blockIdx.y * kP64TQ, p0 = blockIdx.z * kP64TP;
  pdl_enter();
  const int hb = p0 - a.ph, wb = q0 - a.pw;
  constexpr int NEL = (kP64TP + 2) * (kP64TQ + 2) * 8;
  uint4 raw[6];
#pragma unroll
  for (int b = 0; b < 6; ++b) {
    const int e = threadIdx.x + b * 256;
    raw[b] = make_uint4(0u, 0u, 0u, 0u);
    if (e >= NEL) continue;
    const int cv = e & 7, pix = e >> 3;
    const int row = pix / (kP64TQ + 2), col = pix - row * (kP64TQ + 2);
    const int h = hb + row, w = wb + col, c = c0 + cv * 8;
    if (h >= 0 && h < a.H && w >= 0 && w < a.W && c + 8 <= a.C)
      raw[b] = __ldg(reinterpret_cast<const uint4*>(a.x + ((size_t)h * a.W + w) * a.ldx + c));
  }
#pragma unroll
  for (int b = 0; b < 6; ++b) {
    const int e = threadIdx.x + b * 256;
    if (e < NEL) tile[e] = raw[b];
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int cv = lane & 7, qq = lane >> 3;
  const int p = p0 + warp, c = c0 + cv * 8;
  if (p >= a.P || c >= a.C) return;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int ql = qq + 4 * j, q = q0 + ql;
    if (q >= a.Q) break;
    float acc[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) acc[k] = 0.f;
#pragma unroll
    for (int r = 0; r < 3; ++r)
#pragma unroll
      for (int s2 = 0; s2 < 3; ++s2) {
        const uint4 u = tile[((warp + r) * (kP64TQ + 2) + ql + s2) * 8 + cv];
        acc[0] = add_bf16_lo(u.x, acc[0]); acc[1] = add_bf16_hi(u.x, acc[1]);
        acc[2] = add_bf16_lo(u.y, acc[2]); acc[3] = add_bf16_hi(u.y, acc[3]);
        acc[4] = add_bf16_lo(u.z, acc[4]); acc[5] = add_bf16_hi(u.z, acc[5]);
        acc[6] = add_bf16_lo(u.w, acc[6]); acc[7] = add_bf16_hi(u.w, acc[7]);
      }
    const int h0 = p - a.ph, w0 = q - a.pw;
    int div;
    if (a.cip) div = (min(h0 + 3, a.H + a.ph) - h0) * (min(w0 + 3, a.W + a.pw) - w0);
    else div = (min(h0 + 3, a.H) - max(h0, 0)) * (min(w0 + 3, a.W) - max(w0, 0));
    const float inv = 1.f / (float)div;
#pragma unroll
    for (int k = 0; k < 8; ++k) acc[k] *= inv;
    const size_t pix = (size_t)p * a.Q + q;
    store8(a.out + pix * a.ldo + c, c, a.C, acc);
    for (int d_ = 0; d_ < a.out2.n; ++d_) store8(a.out2.p[d_] + pix * a.out2.ld[d_] + c, c, a.C, acc);
  }
}

template <typename T, int KS>
static void launch_pool_tiled(const PoolArgs<T>& a, size_t smem, cudaStream_t st) {
  static bool attr_set[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && !attr_set[dev]) {
    cudaFuncSetAttribute(pool_tiled_kernel<T, KS>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    attr_set[dev] = true;
  }
  dim3 grid((a.C + 15) / 16, (a.Q + kPoolTQ - 1) / kPoolTQ, (a.P + kPoolTP - 1) / kPoolTP);
  launch_pdl(pool_tiled_kernel<T, KS>, grid, dim3(256), smem, st, a);
}

template <typename T>
void launch_pool(const PoolArgs<T>& a, cudaStream_t st) {
  constexpr int N = Vec<T>::N;
  const size_t smem = (size_t)2 * ((kPoolTP - 1) * a.sh + a.kh) * ((kPoolTQ - 1) * a.sw + a.kw) * 8 * sizeof(T);
  // measured (tools/op_micro.py, B200): tiled 3x3/s1 avgpool 139 us vs 187 us
  // direct; 3x3/s2 maxpool 297 us vs 205 us direct -- stride 1 only
  // bf16 3x3: the direct kernel with all tap loads in flight (measured faster
  // than the smem-tiled kernel); direct wins for stride 2 and for small
  // stride-1 pools (Mixed_6/7 at 1024^2), the tiled kernel for large stride-1
  // average pools.  (A row-streaming kernel measured slower on every shape and
  // was removed, round 2.)
  const bool big_s1 = a.sh == 1 && (long long)a.P * a.Q * a.C >= (4LL << 20);
  if constexpr (std::is_same<T, bf16>::value) {
    // large stride-1 3x3 average pools with whole 8-channel vectors: 64-channel CTAs
    if (big_s1 && !a.is_max && a.kh == 3 && a.kw == 3 && a.sw == 1 && a.C % 8 == 0) {
      dim3 grid((a.C + 63) / 64, (a.Q + kP64TQ - 1) / kP64TQ, (a.P + kP64TP - 1) / kP64TP);
      launch_pdl(pool_avg64_kernel, grid, dim3(256), 0, st, a);
      return;
    }
  }
  if (std::is_same<T, bf16>::value && a.kh == 3 && a.kw == 3 && !big_s1) {
    const int per_row = a.Q * ((a.C + N - 1) / N);
    dim3 grid((per_row + 255) / 256, a.P);
    launch_pdl(pool_kernel<T, 3, 3>, grid, dim3(256), 0, st, a);
    return;
  }
  if (a.sw == 1 && a.sh == 1 && a.kh * a.kw > 1 && smem <= 200 * 1024) {
    if (a.kh == 3 && a.kw == 3) return launch_pool_tiled<T, 3>(a, smem, st);
    return launch_pool_tiled<T, 0>(a, smem, st);
  }
  const int per_row = a.Q * ((a.C + N - 1) / N);
  dim3 grid((per_row + 255) / 256, a.P);
  if (a.kh == 3 && a.kw == 3)
    launch_pdl(pool_kernel<T, 3, 3>, grid, dim3(256), 0, st, a);
  else
    launch_pdl(pool_kernel<T, 0, 0>, grid, dim3(256), 0, st, a);
}

// ------------------------------------------- depthwise (+ aggregation, ReLU)
template <typename T>
__global__ void dw_kernel(const DwArgs<T> a) {
  pdl_enter();
  constexpr int N = Vec<T>::N;
  const int CG = (a.C + N - 1) / N;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= a.P * a.Q * CG) return;
  const int cg = idx % CG;
  const int pix = idx / CG;
  const int q = pix % a.Q, p = pix / a.Q;
  const int c = cg * N;
  float acc[N], v[N], u[N];
#pragma unroll
  for (int j = 0; j < N; ++j) acc[j] = 0.f;
  for (int r = 0; r < a.R; ++r) {
    const int h = p * a.sh - a.ph + r;
    if (h < 0 || h >= a.H) continue;
    for (int s = 0; s < a.S; ++s) {
      const int w = q * a.sw - a.pw + s;
      if (w < 0 || w >= a.W) continue;
      const size_t off = (size_t)h * a.W + w;
#pragma unroll
      for (int j = 0; j < N; ++j) u[j] = 0.f;
      for (int i = 0; i < a.n_in; ++i) {
        load_vec(a.x[i] + off * a.ldx[i] + c, c, a.C, v);
#pragma unroll
        for (int j = 0; j < N; ++j) u[j] += a.agg[i] * v[j];
      }
      const float* wt = a.w + (size_t)(r * a.S + s) * a.C + c;
#pragma unroll
      for (int j = 0; j < N; ++j) {
        float x = a.pre_relu ? fmaxf(u[j], 0.f) : u[j];
        acc[j] += x * ((c + j < a.C) ? __ldg(wt + j) : 0.f);
      }
    }
  }
  store_vec(a.out + (size_t)pix * a.ldo + c, c, a.C, acc);
}

// Tiled depthwise: a CTA owns 8 output rows x 32 output columns x 16
// channels.  The (aggregated, pre-ReLU'd, zero-padded) input window of the
// tile is staged once in smem as [channel vector][row][col] planes (columns
// de-interleaved by parity when sw == 2, so a warp's 32 lanes read 32
// consecutive 16-byte vectors at every tap), the 16 channels' weights as fp32.
// Warp w: channel vector w & 1, output rows (w >> 1) and (w >> 1) + 4; lane:
// output column.  Per kernel row r the thread holds the S weight vectors in
// registers (KS > 0) and reuses them for its two output rows.
constexpr int kDwTP = 8, kDwTQ = 32;
__host__ __device__ inline int dw_tile_rows(int R, int sh) { return (kDwTP - 1) * sh + R; }
__host__ __device__ inline int dw_tile_cols(int S, int sw) { return (kDwTQ - 1) * sw + S; }

template <typename T, int KS>
__global__ void __launch_bounds__(256, 4) dw_tiled_kernel(const DwArgs<T> a) {
  extern __shared__ __align__(16) uint8_t dsm[];
  constexpr int N = 8;                       // channels per vector (16 B bf16, 32 B fp32)
  constexpr int VB = N * (int)sizeof(T);     // bytes per staged vector
  const int R = KS > 0 ? KS : a.R, S = KS > 0 ? KS : a.S;
  const int IH = dw_tile_rows(R, a.sh), IW = dw_tile_cols(S, a.sw);
  const int half = (IW + 1) / 2;
  // channel slab fastest in the grid (see pool_tiled_kernel)
  const int q0 = blockIdx.y * kDwTQ, p0 = blockIdx.z * kDwTP, c0 = blockIdx.x * 16;
  float* sw_ = reinterpret_cast<float*>(dsm);                  // [R*S][16]
  uint8_t* tile = dsm + (size_t)R * S * 16 * sizeof(float);   // [2][IH][IW] vectors
  for (int i = threadIdx.x; i < R * S * 16; i += blockDim.x) {
    const int rs = i >> 4, j = i & 15;
    sw_[i] = (c0 + j < a.C) ? __ldg(a.w + (size_t)rs * a.C + c0 + j) : 0.f;
  }
  pdl_enter();
  const int hb = p0 * a.sh - a.ph, wb = q0 * a.sw - a.pw;
  const int nel = 2 * IH * IW;
  for (int e = threadIdx.x; e < nel; e += blockDim.x) {
    const int cv = e & 1, pix = e >> 1;
    const int row = pix / IW, col = pix - row * IW;
    const int h = hb + row, w = wb + col, c = c0 + cv * N;
    float u[N];
#pragma unroll
    for (int j = 0; j < N; ++j) u[j] = 0.f;
    if (h >= 0 && h < a.H && w >= 0 && w < a.W && c < a.C) {
      const size_t off = (size_t)h * a.W + w;
      for (int i = 0; i < a.n_in; ++i) {
        float v[N];
        load8(a.x[i] + off * a.ldx[i] + c, c, a.C, v);
#pragma unroll
        for (int j = 0; j < N; ++j) u[j] += a.agg[i] * v[j];
      }
      if (a.pre_relu) {
#pragma unroll
        for (int j = 0; j < N; ++j) u[j] = fmaxf(u[j], 0.f);
      }
    }
    const int pos = a.sw == 2 ? ((col & 1) * half + (col >> 1)) : col;
    T* d = reinterpret_cast<T*>(tile + ((size_t)(cv * IH + row) * IW + pos) * VB);
#pragma unroll
    for (int j = 0; j < N; ++j) d[j] = from_f<T>(u[j]);
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int cv = warp & 1, pr0 = warp >> 1;
  const int q = q0 + lane;
  const uint8_t* plane = tile + (size_t)cv * IH * IW * VB;
  const float* wv = sw_ + cv * N;
  float acc[2][N];
#pragma unroll
  for (int k = 0; k < 2; ++k)
#pragma unroll
    for (int j = 0; j < N; ++j) acc[k][j] = 0.f;
  auto tap = [&](float (&ac)[N], int row, int s, const float* wt) {
    const int col = lane * a.sw + s;
    const int pos = a.sw == 2 ? ((col & 1) * half + (col >> 1)) : col;
    const T* src = reinterpret_cast<const T*>(plane + ((size_t)row * IW + pos) * VB);
    float v[N];
    load8(src, 0, N, v);
#pragma unroll
    for (int j = 0; j < N; ++j) ac[j] = fmaf(v[j], wt[j], ac[j]);
  };
  for (int r = 0; r < R; ++r) {
    if (KS > 0) {
      float wr[KS > 0 ? KS : 1][N];
#pragma unroll
      for (int s2 = 0; s2 < (KS > 0 ? KS : 1); ++s2)
#pragma unroll
        for (int j = 0; j < N; ++j) wr[s2][j] = wv[(r * S + s2) * 16 + j];
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        const int row = (pr0 + 4 * k) * a.sh + r;
#pragma unroll
        for (int s2 = 0; s2 < (KS > 0 ? KS : 1); ++s2) tap(acc[k], row, s2, wr[s2]);
      }
    } else {
      for (int s2 = 0; s2 < S; ++s2) {
        float wt[N];
#pragma unroll
        for (int j = 0; j < N; ++j) wt[j] = wv[(r * S + s2) * 16 + j];
#pragma unroll
        for (int k = 0; k < 2; ++k) tap(acc[k], (pr0 + 4 * k) * a.sh + r, s2, wt);
      }
    }
  }
  const int c = c0 + cv * N;
  if (q >= a.Q || c >= a.C) return;
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const int p = p0 + pr0 + 4 * k;
    if (p < a.P) store8(a.out + ((size_t)p * a.Q + q) * a.ldo + c, c, a.C, acc[k]);
  }
}

// Register-blocked depthwise for bf16 (KS x KS, stride SS): the CTA stages
// the same bf16 input window as dw_tiled_kernel (TP = 4 * KR output rows x 32
// columns x 16 channels) plus the weights rounded to bf16; a thread owns KR
// vertically adjacent output rows of one column and 8 channels.  For each
// kernel column s it holds the KS weight vectors of that column in registers
// and walks the (KR - 1) * SS + KS input rows its outputs touch, loading each
// staged vector once and feeding it to every output row that uses it (the
// tiled kernel re-read it per output and per tap: shared-memory bound).
// fma.rn.f32.bf16 (FHFMA.BF16, sm_100) multiplies the bf16 halves directly
// into fp32 accumulators: no conversions in the inner loop.
template <int KS, int SS, int KR>
__global__ void __launch_bounds__(256, 4) dw_reg_kernel(const DwArgs<bf16> a) {
  extern __shared__ __align__(16) uint8_t dsm[];
  constexpr int TP = 4 * KR, N = 8, VB = 16;
  constexpr int IH = (TP - 1) * SS + KS, IW = (kDwTQ - 1) * SS + KS;
  constexpr int HALF = (IW + 1) / 2;
  constexpr int NH = (KR - 1) * SS + KS;  // input rows one thread touches
  const int q0 = blockIdx.y * kDwTQ, p0 = blockIdx.z * TP, c0 = blockIdx.x * 16;
  uint8_t* swb = dsm;                                   // [KS*KS][16] bf16 weights
  uint8_t* tile = dsm + (size_t)KS * KS * 32;           // [2][IH][IW] bf16 vectors
  for (int i = threadIdx.x; i < KS * KS * 16; i += blockDim.x) {
    const int rs = i >> 4, j = i & 15;
    reinterpret_cast<bf16*>(swb)[i] =
        __float2bfloat16_rn((c0 + j < a.C) ? __ldg(a.w + (size_t)rs * a.C + c0 + j) : 0.f);
  }
  pdl_enter();
  const int hb = p0 * SS - a.ph, wb = q0 * SS - a.pw;
  // single input, both 8-channel vectors in bounds: the staging loads of four
  // rounds are issued before any is used (latency overlap), values kept in
  // bf16 (scale 1: exact; ReLU as packed max)
  const bool fast = a.n_in == 1 && c0 + 16 <= a.C && a.agg[0] == 1.f;
  constexpr int NEL = 2 * IH * IW, NB = 4;
  for (int e0 = fast ? (int)threadIdx.x : NEL; e0 < NEL; e0 += NB * 256) {
    uint4 raw[NB];
    int dst[NB];
#pragma unroll
    for (int b = 0; b < NB; ++b) {
      const int e = e0 + b * 256;
      dst[b] = -1;
      raw[b] = make_uint4(0u, 0u, 0u, 0u);
      if (e >= NEL) continue;
      const int cv = e & 1, pix = e >> 1;
      const int row = pix / IW, col = pix - row * IW;
      const int h = hb + row, w = wb + col;
      const int pos = SS == 2 ? ((col & 1) * HALF + (col >> 1)) : col;
      dst[b] = (cv * IH + row) * IW + pos;
      if (h >= 0 && h < a.H && w >= 0 && w < a.W)
        raw[b] = __ldg(reinterpret_cast<const uint4*>(a.x[0] + ((size_t)h * a.W + w) * a.ldx[0] + c0 + cv * N));
    }
#pragma unroll
    for (int b = 0; b < NB; ++b) {
      if (dst[b] < 0) continue;
      uint4 v = raw[b];
      if (a.pre_relu) {
        __nv_bfloat162* p2 = reinterpret_cast<__nv_bfloat162*>(&v);
        const __nv_bfloat162 z = __floats2bfloat162_rn(0.f, 0.f);
#pragma unroll
        for (int j = 0; j < 4; ++j) p2[j] = __hmax2(p2[j], z);
      }
      *reinterpret_cast<uint4*>(tile + (size_t)dst[b] * VB) = v;
    }
  }
  for (int e = fast ? NEL : (int)threadIdx.x; e < NEL; e += blockDim.x) {
    const int cv = e & 1, pix = e >> 1;
    const int row = pix / IW, col = pix - row * IW;
    const int h = hb + row, w = wb + col, c = c0 + cv * N;
    float u[N];
#pragma unroll
    for (int j = 0; j < N; ++j) u[j] = 0.f;
    if (h >= 0 && h < a.H && w >= 0 && w < a.W && c < a.C) {
      const size_t off = (size_t)h * a.W + w;
      for (int i = 0; i < a.n_in; ++i) {
        float v[N];
        load8(a.x[i] + off * a.ldx[i] + c, c, a.C, v);
#pragma unroll
        for (int j = 0; j < N; ++j) u[j] += a.agg[i] * v[j];
      }
      if (a.pre_relu) {
#pragma unroll
        for (int j = 0; j < N; ++j) u[j] = fmaxf(u[j], 0.f);
      }
    }
    const int pos = SS == 2 ? ((col & 1) * HALF + (col >> 1)) : col;
    uint4 pk;
    __nv_bfloat162* b2 = reinterpret_cast<__nv_bfloat162*>(&pk);
#pragma unroll
    for (int j = 0; j < 4; ++j) b2[j] = __floats2bfloat162_rn(u[2 * j], u[2 * j + 1]);
    *reinterpret_cast<uint4*>(tile + ((size_t)(cv * IH + row) * IW + pos) * VB) = pk;
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int cv = warp & 1, pr0 = warp >> 1;
  const uint8_t* plane = tile + (size_t)cv * IH * IW * VB + (size_t)(pr0 * KR * SS) * IW * VB;
  float acc[KR][N];
#pragma unroll
  for (int k = 0; k < KR; ++k)
#pragma unroll
    for (int j = 0; j < N; ++j) acc[k][j] = 0.f;
#pragma unroll 1
  for (int s = 0; s < KS; ++s) {
    uint4 wr[KS];
#pragma unroll
    for (int r = 0; r < KS; ++r) wr[r] = *reinterpret_cast<const uint4*>(swb + (size_t)(r * KS + s) * 32 + cv * 16);
    const int col = lane * SS + s;
    const int pos = SS == 2 ? ((col & 1) * HALF + (col >> 1)) : col;
    const uint8_t* src = plane + (size_t)pos * VB;
#pragma unroll
    for (int hh = 0; hh < NH; ++hh) {
      const uint4 x = *reinterpret_cast<const uint4*>(src + (size_t)hh * IW * VB);
#pragma unroll
      for (int k = 0; k < KR; ++k) {
        const int r = hh - k * SS;
        if (r < 0 || r >= KS) continue;
        acc[k][0] = fma_bf16_lo(x.x, wr[r].x, acc[k][0]); acc[k][1] = fma_bf16_hi(x.x, wr[r].x, acc[k][1]);
        acc[k][2] = fma_bf16_lo(x.y, wr[r].y, acc[k][2]); acc[k][3] = fma_bf16_hi(x.y, wr[r].y, acc[k][3]);
        acc[k][4] = fma_bf16_lo(x.z, wr[r].z, acc[k][4]); acc[k][5] = fma_bf16_hi(x.z, wr[r].z, acc[k][5]);
        acc[k][6] = fma_bf16_lo(x.w, wr[r].w, acc[k][6]); acc[k][7] = fma_bf16_hi(x.w, wr[r].w, acc[k][7]);
      }
    }
  }
  const int q = q0 + lane, c = c0 + cv * N;
  if (q >= a.Q || c >= a.C) return;
#pragma unroll
  for (int k = 0; k < KR; ++k) {
    const int p = p0 + pr0 * KR + k;
    if (p < a.P) store8(a.out + ((size_t)p * a.Q + q) * a.ldo + c, c, a.C, acc[k]);
  }
}

template <int KS, int SS, int KR>
static void launch_dw_reg(const DwArgs<bf16>& a, cudaStream_t st) {
  constexpr int TP = 4 * KR;
  constexpr size_t smem = (size_t)KS * KS * 32 + (size_t)2 * ((TP - 1) * SS + KS) * ((kDwTQ - 1) * SS + KS) * 16;
  static bool attr_set[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && !attr_set[dev]) {
    cudaFuncSetAttribute(dw_reg_kernel<KS, SS, KR>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    attr_set[dev] = true;
  }
  dim3 grid((a.C + 15) / 16, (a.Q + kDwTQ - 1) / kDwTQ, (a.P + TP - 1) / TP);
  launch_pdl(dw_reg_kernel<KS, SS, KR>, grid, dim3(256), smem, st, a);
}

// bf16, square 3/5/7 kernels, stride 1 or 2: the register-blocked kernel
// (4 rows per thread at stride 1, 2 at stride 2)
template <typename T>
static bool try_dw_reg(const DwArgs<T>&, cudaStream_t) { return false; }
template <>
bool try_dw_reg<bf16>(const DwArgs<bf16>& a, cudaStream_t st) {
  if (a.R != a.S || a.sh != a.sw || (a.sh != 1 && a.sh != 2)) return false;
  if (a.sh == 1) {
    if (a.R == 3) { launch_dw_reg<3, 1, 4>(a, st); return true; }
    if (a.R == 5) { launch_dw_reg<5, 1, 4>(a, st); return true; }
    if (a.R == 7) { launch_dw_reg<7, 1, 4>(a, st); return true; }
  } else {
    if (a.R == 3) { launch_dw_reg<3, 2, 2>(a, st); return true; }
    if (a.R == 5) { launch_dw_reg<5, 2, 2>(a, st); return true; }
    if (a.R == 7) { launch_dw_reg<7, 2, 2>(a, st); return true; }
  }
  return false;
}

template <typename T, int KS>
static void launch_dw_tiled(const DwArgs<T>& a, size_t smem, cudaStream_t st) {
  static bool attr_set[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && !attr_set[dev]) {
    cudaFuncSetAttribute(dw_tiled_kernel<T, KS>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    attr_set[dev] = true;
  }
  dim3 grid((a.C + 15) / 16, (a.Q + kDwTQ - 1) / kDwTQ, (a.P + kDwTP - 1) / kDwTP);
  launch_pdl(dw_tiled_kernel<T, KS>, grid, dim3(256), smem, st, a);
}

template <typename T>
void launch_dw(const DwArgs<T>& a, cudaStream_t st) {
  constexpr int N = Vec<T>::N;
  const size_t smem = (size_t)a.R * a.S * 16 * sizeof(float) +
                      (size_t)2 * dw_tile_rows(a.R, a.sh) * dw_tile_cols(a.S, a.sw) * 8 * sizeof(T);
  if (try_dw_reg(a, st)) return;
  if ((a.sw == 1 || a.sw == 2) && smem <= 200 * 1024) {
    if (a.R == 3 && a.S == 3) return launch_dw_tiled<T, 3>(a, smem, st);
    if (a.R == 5 && a.S == 5) return launch_dw_tiled<T, 5>(a, smem, st);
    if (a.R == 7 && a.S == 7) return launch_dw_tiled<T, 7>(a, smem, st);
    return launch_dw_tiled<T, 0>(a, smem, st);
  }
  long long n = (long long)a.P * a.Q * ((a.C + N - 1) / N);
  launch_pdl(dw_kernel<T>, dim3(grid_for(n, 256)), dim3(256), 0, st, a);
}

// ------------------------------------------------------------------- add
template <typename T>
__global__ void add_kernel(const AddArgs<T> a) {
  pdl_enter();
  constexpr int N = Vec<T>::N;
  const int CG = (a.C + N - 1) / N;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= a.HW * CG) return;
  const int c = (idx % CG) * N;
  const size_t pix = idx / CG;
  float acc[N], v[N];
#pragma unroll
  for (int j = 0; j < N; ++j) acc[j] = 0.f;
  if constexpr (std::is_same<T, bf16>::value) {
    if (a.n_in <= 4 && c + 8 <= a.C) {
      // whole vectors, <= 4 inputs: all loads in flight first
      uint4 raw[4];
#pragma unroll
      for (int i = 0; i < 4; ++i)
        if (i < a.n_in) raw[i] = __ldg(reinterpret_cast<const uint4*>(a.x[i] + pix * a.ldx[i] + c));
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        if (i >= a.n_in) break;
        const __nv_bfloat162* p2 = reinterpret_cast<const __nv_bfloat162*>(&raw[i]);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const float2 f = __bfloat1622float2(p2[j]);
          acc[2 * j] += a.agg[i] * f.x;
          acc[2 * j + 1] += a.agg[i] * f.y;
        }
      }
      if (a.relu) {
#pragma unroll
        for (int j = 0; j < N; ++j) acc[j] = fmaxf(acc[j], 0.f);
      }
      store_vec(a.out + pix * a.ldo + c, c, a.C, acc);
      for (int d_ = 0; d_ < a.out2.n; ++d_) store_vec(a.out2.p[d_] + pix * a.out2.ld[d_] + c, c, a.C, acc);
      return;
    }
  }
  for (int i = 0; i < a.n_in; ++i) {
    load_vec(a.x[i] + pix * a.ldx[i] + c, c, a.C, v);
#pragma unroll
    for (int j = 0; j < N; ++j) acc[j] += a.agg[i] * v[j];
  }
  if (a.relu) {
#pragma unroll
    for (int j = 0; j < N; ++j) acc[j] = fmaxf(acc[j], 0.f);
  }
  store_vec(a.out + pix * a.ldo + c, c, a.C, acc);
  for (int d_ = 0; d_ < a.out2.n; ++d_) store_vec(a.out2.p[d_] + pix * a.out2.ld[d_] + c, c, a.C, acc);
}

template <typename T>
void launch_add(const AddArgs<T>& a, cudaStream_t st) {
  constexpr int N = Vec<T>::N;
  long long n = (long long)a.HW * ((a.C + N - 1) / N);
  launch_pdl(add_kernel<T>, dim3(grid_for(n, 256)), dim3(256), 0, st, a);
}

// ------------------------------------------------------------------ copy
template <typename T>
__global__ void copy_kernel(const CopyArgs<T> a) {
  pdl_enter();
  constexpr int N = Vec<T>::N;
  const int CG = (a.C + N - 1) / N;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= a.HW * CG) return;
  const int c = (idx % CG) * N;
  const size_t pix = idx / CG;
  const T* src = a.x + pix * a.ldx + c;
  T* dst = a.out + pix * a.ldo + c;
  // concat slices at channel offsets that are not multiples of 8 are not
  // 16-byte aligned: fall back to element copies there
  const uintptr_t al = reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst);
  if (c + N <= a.C && (al & 15) == 0) {
    *reinterpret_cast<uint4*>(dst) = *reinterpret_cast<const uint4*>(src);
  } else if (c + N <= a.C && (al & 7) == 0) {
    const uint2* s2 = reinterpret_cast<const uint2*>(src);
    uint2* d2 = reinterpret_cast<uint2*>(dst);
    d2[0] = s2[0]; d2[1] = s2[1];
  } else if (c + N <= a.C && (al & 3) == 0) {
    // even channel offsets (e.g. NASNet's 42-channel concat slices): words
    const uint32_t* s4 = reinterpret_cast<const uint32_t*>(src);
    uint32_t* d4 = reinterpret_cast<uint32_t*>(dst);
    const uint32_t w0 = s4[0], w1 = s4[1], w2 = s4[2], w3 = s4[3];
    d4[0] = w0; d4[1] = w1; d4[2] = w2; d4[3] = w3;
  } else {
    for (int j = 0; j < N && c + j < a.C; ++j) dst[j] = src[j];
  }
}

template <typename T>
void launch_copy(const CopyArgs<T>& a, cudaStream_t st) {
  constexpr int N = Vec<T>::N;
  long long n = (long long)a.HW * ((a.C + N - 1) / N);
  launch_pdl(copy_kernel<T>, dim3(grid_for(n, 256)), dim3(256), 0, st, a);
}

// ReLU copy (the input of a pre-ReLU conv, NASNet's ReLU -> conv -> BN): one
// thread per (pixel, N-channel vector), 16-byte vectors when aligned.
template <typename T>
__global__ void relu_copy_kernel(const CopyArgs<T> a) {
  pdl_enter();
  constexpr int N = Vec<T>::N;
  const int CG = (a.C + N - 1) / N;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= a.HW * CG) return;
  const int c = (idx % CG) * N;
  const size_t pix = idx / CG;
  const T* src = a.x + pix * a.ldx + c;
  T* dst = a.out + pix * a.ldo + c;
  const uintptr_t al = reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst);
  if (c + N <= a.C && (al & 15) == 0) {
    uint4 v = *reinterpret_cast<const uint4*>(src);
    if constexpr (sizeof(T) == 2) {
      __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&v);
      const __nv_bfloat162 z = __floats2bfloat162_rn(0.f, 0.f);
#pragma unroll
      for (int j = 0; j < 4; ++j) h[j] = __hmax2(h[j], z);
    } else {
      float* f = reinterpret_cast<float*>(&v);
#pragma unroll
      for (int j = 0; j < 4; ++j) f[j] = fmaxf(f[j], 0.f);
    }
    *reinterpret_cast<uint4*>(dst) = v;
  } else {
    for (int j = 0; j < N && c + j < a.C; ++j) {
      const float f = to_f(src[j]);
      dst[j] = from_f<T>(f > 0.f ? f : 0.f);
    }
  }
}

template <typename T>
void launch_relu_copy(const CopyArgs<T>& a, cudaStream_t st) {
  constexpr int N = Vec<T>::N;
  long long n = (long long)a.HW * ((a.C + N - 1) / N);
  launch_pdl(relu_copy_kernel<T>, dim3(grid_for(n, 256)), dim3(256), 0, st, a);
}

// ------------------------------------------------------------------- GAP
// one block per 8/4-channel group; threads stride over pixels; smem reduce
template <typename T>
__global__ void gap_kernel(const T* x, int HW, int C, int ldx, T* out) {
  pdl_enter();
  constexpr int N = Vec<T>::N;
  const int c = blockIdx.x * N;
  float acc[N], v[N];
#pragma unroll
  for (int j = 0; j < N; ++j) acc[j] = 0.f;
  for (int pix = threadIdx.x; pix < HW; pix += blockDim.x) {
    load_vec(x + (size_t)pix * ldx + c, c, C, v);
#pragma unroll
    for (int j = 0; j < N; ++j) acc[j] += v[j];
  }
  __shared__ float red[N][32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    float s = acc[j];
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) red[j][warp] = s;
  }
  __syncthreads();
  if (warp == 0) {
    const int nw = blockDim.x >> 5;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      float s = lane < nw ? red[j][lane] : 0.f;
      for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      acc[j] = s / (float)HW;
    }
    if (lane == 0) store_vec(out + c, c, C, acc);
  }
}

template <typename T>
void launch_gap(const T* x, int HW, int C, int ldx, T* out, cudaStream_t st) {
  constexpr int N = Vec<T>::N;
  launch_pdl(gap_kernel<T>, dim3((C + N - 1) / N), dim3(512), 0, st, x, HW, C, ldx, out);
}

// ---------------------------------------------------------------- linear
// one warp per output: y[k] = sum_c W[k,c] x[c] + b[k]
template <typename T>
__global__ void linear_kernel(const T* x, int Cin, const T* w, int ldw, const float* b, int K, T* out) {
  pdl_enter();
  const int k = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (k >= K) return;
  constexpr int N = Vec<T>::N;
  float s = 0.f, xv[N], wv[N];
  const T* wr = w + (size_t)k * ldw;
  for (int c = lane * N; c < Cin; c += 32 * N) {
    load_vec(x + c, c, Cin, xv);
    load_vec(wr + c, c, Cin, wv);
#pragma unroll
    for (int j = 0; j < N; ++j) s += xv[j] * wv[j];
  }
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) out[k] = from_f<T>(s + b[k]);
}

template <typename T>
void launch_linear(const T* x, int Cin, const T* w, int ldw, const float* b, int K, T* out, cudaStream_t st) {
  launch_pdl(linear_kernel<T>, dim3((K + 7) / 8), dim3(256), 0, st, x, Cin, w, ldw, b, K, out);
}

// ------------------------------------------------- layout conversion
template <typename T>
__global__ void input_kernel(const float* nchw, int C, int HW, T* out, int ldo) {
  pdl_enter();
  constexpr int N = Vec<T>::N;
  const int pix = blockIdx.x * blockDim.x + threadIdx.x;
  if (pix >= HW) return;
  for (int c0 = 0; c0 < ldo; c0 += N) {
    float v[N];
#pragma unroll
    for (int j = 0; j < N; ++j) v[j] = (c0 + j < C) ? __ldg(nchw + (size_t)(c0 + j) * HW + pix) : 0.f;
    store_vec(out + (size_t)pix * ldo + c0, c0, ldo, v);
  }
}
template <typename T>
void launch_input(const float* nchw, int C, int H, int W, T* out, int ldo, cudaStream_t st) {
  launch_pdl(input_kernel<T>, dim3(grid_for((long long)H * W, 256)), dim3(256), 0, st, nchw, C, H * W, out, ldo);
}

template <typename T>
__global__ void output_kernel(const T* x, int C, int HW, int ldx, float* nchw) {
  pdl_enter();
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= (long long)C * HW) return;
  const int c = (int)(i / HW);
  const long long pix = i % HW;
  nchw[i] = to_f(x[pix * ldx + c]);
}
template <typename T>
void launch_output(const T* x, int C, int H, int W, int ldx, float* nchw, cudaStream_t st) {
  launch_pdl(output_kernel<T>, dim3(grid_for((long long)C * H * W, 256)), dim3(256), 0, st, x, C, H * W, ldx, nchw);
}

// ----------------------------------------------- cross-GPU epoch flags
// epoch: incremented by the first kernel of every per-GPU graph replay.
// signal: after the producer's stores (kernel boundary + system fence), the
// producer GPU writes its epoch into the consumer's flag with a release store.
// wait: the consumer spins (acquire, system scope) until flag >= epoch - lag.
__global__ void epoch_kernel(unsigned* epoch) { *epoch += 1u; }

__global__ void signal_kernel(const unsigned* epoch, unsigned* flag) {
  const unsigned e = *epoch;
  __threadfence_system();
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(flag), "r"(e) : "memory");
}

// a wait that has not seen its flag after kWaitTimeoutNs is a broken schedule
// or a dead peer: report it and trap (the run fails with HIOS_E_CUDA instead
// of hanging the GPU)
constexpr unsigned long long kWaitTimeoutNs = 20ull * 1000 * 1000 * 1000;
__global__ void wait_kernel(const unsigned* epoch, const unsigned* flag, unsigned lag) {
  const unsigned target = *epoch - lag;
  unsigned v;
  unsigned long long t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (unsigned it = 0;; ++it) {
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
    if ((int)(v - target) >= 0) break;
    __nanosleep(64);
    if ((it & 1023) == 1023) {
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      if (t - t0 > kWaitTimeoutNs) {
        printf("hios: flag wait timed out: flag %p = %u, target %u (epoch %u, lag %u)\n", (const void*)flag, v,
               target, *epoch, lag);
        __trap();
      }
    }
  }
}

void launch_epoch(unsigned* epoch, cudaStream_t st) { epoch_kernel<<<1, 1, 0, st>>>(epoch); }
void launch_signal(const unsigned* epoch, unsigned* flag, cudaStream_t st) {
  signal_kernel<<<1, 1, 0, st>>>(epoch, flag);
}
void launch_wait(const unsigned* epoch, const unsigned* flag, unsigned lag, cudaStream_t st) {
  wait_kernel<<<1, 1, 0, st>>>(epoch, flag, lag);
}

__global__ void fill_kernel(uint4* p, size_t n) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = make_uint4(i, i ^ 0x9e3779b9u, 0, 1);
}
void launch_fill(void* p, size_t bytes, cudaStream_t st) {
  fill_kernel<<<148 * 8, 512, 0, st>>>(reinterpret_cast<uint4*>(p), bytes / 16);
}

// ------------------------------------------------- space-to-depth (stems)
// one thread per X' pixel: 4 source pixels (a, b) in {0,1}^2, C <= 4 channels
// each, packed to (a*2+b)*C + c and zero-padded to the pixel stride
template <typename T>
__global__ void s2d_kernel(const S2dArgs<T> a) {
  pdl_enter();
  const long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  // 4 zero pixels of slack past the end (packed-tap windows of the last row)
  if (idx >= (long long)a.P2 * a.Q2 + 4) return;
  const bool tail = idx >= (long long)a.P2 * a.Q2;
  const int i = (int)(idx / a.Q2), j = (int)(idx - (long long)i * a.Q2);
  T v[16];
#pragma unroll
  for (int e = 0; e < 16; ++e) v[e] = from_f<T>(0.f);
#pragma unroll
  for (int ab = 0; ab < 4; ++ab) {
    if (tail) break;
    const int h = 2 * i + (ab >> 1) - a.ph, w = 2 * j + (ab & 1) - a.pw;
    if (h < 0 || h >= a.H || w < 0 || w >= a.W) continue;
    const T* src = a.x + ((size_t)h * a.W + w) * a.ldx;
#pragma unroll
    for (int c = 0; c < 4; ++c)
      if (c < a.C) v[ab * a.C + c] = src[c];
  }
  T* dst = a.out + (size_t)idx * a.ldo;
  // 4C <= 16 channels, ldo is a multiple of 8: 16-byte stores (bf16) / 4 x 16 B (fp32)
  constexpr int N = Vec<T>::N;
  for (int e = 0; e < a.ldo && e < 16; e += N) *reinterpret_cast<uint4*>(dst + e) = *reinterpret_cast<const uint4*>(v + e);
}

template <typename T>
void launch_s2d(const S2dArgs<T>& a, cudaStream_t st) {
  launch_pdl(s2d_kernel<T>, dim3(grid_for((long long)a.P2 * a.Q2 + 4, 256)), dim3(256), 0, st, a);
}

// explicit instantiations
#define HIOS_INST(T)                                                                                   \
  template void launch_pool<T>(const PoolArgs<T>&, cudaStream_t);                                      \
  template void launch_dw<T>(const DwArgs<T>&, cudaStream_t);                                          \
  template void launch_add<T>(const AddArgs<T>&, cudaStream_t);                                        \
  template void launch_copy<T>(const CopyArgs<T>&, cudaStream_t);                                      \
  template void launch_relu_copy<T>(const CopyArgs<T>&, cudaStream_t);                                 \
  template void launch_s2d<T>(const S2dArgs<T>&, cudaStream_t);                                        \
  template void launch_gap<T>(const T*, int, int, int, T*, cudaStream_t);                              \
  template void launch_linear<T>(const T*, int, const T*, int, const float*, int, T*, cudaStream_t);        \
  template void launch_input<T>(const float*, int, int, int, T*, int, cudaStream_t);                   \
  template void launch_output<T>(const T*, int, int, int, int, float*, cudaStream_t);
HIOS_INST(float)
HIOS_INST(bf16)

}  // namespace hios

namespace hios {
// ------------------------------------------------- direct small-C conv
// Stem convolutions with C <= 8 input channels (Inception's 3->32 3x3 s2,
// SqueezeNet's 3->96 7x7 s2): K = C*R*S is tiny, so the tensor-core path
// would waste >90 % of every 64-channel K-step.  One thread computes one
// output pixel x 16 output channels on CUDA cores (fp32 FMA); the C x R x S
// receptive field is read once into registers, weights come from smem.
template <typename T, int CC, int RR, int SS, int KT>
__global__ void __launch_bounds__(128) conv_small_c_kernel(const ConvSmallArgs<T> a) {
  // CC/RR/SS > 0: compile-time receptive field kept in registers; KT output
  // channels x PX=2 neighbouring output pixels (along W) per thread, so each
  // weight read from smem feeds two FMAs
  constexpr int PX = (CC > 0 && CC * RR * SS <= 64) ? 2 : 1;
  extern __shared__ float sw[];  // [K][R*S*C] then scale[K], shift[K]
  const int C = CC > 0 ? CC : a.C, R = RR > 0 ? RR : a.R, S = SS > 0 ? SS : a.S;
  const int RSC = R * S * C;
  for (int i = threadIdx.x; i < a.K * RSC; i += blockDim.x) sw[i] = a.w[i];
  for (int i = threadIdx.x; i < a.K; i += blockDim.x) {
    sw[a.K * RSC + i] = a.scale[i];
    sw[a.K * RSC + a.K + i] = a.shift[i];
  }
  pdl_enter();  // weights staged under the predecessor's tail
  __syncthreads();
  const int KG = (a.K + KT - 1) / KT;
  const int QP = (a.Q + PX - 1) / PX;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= a.P * QP * KG) return;
  const int kg = idx % KG, pq = idx / KG;
  const int qp = pq % QP, p = pq / QP;
  const int q0 = qp * PX;
  constexpr int XN = (CC > 0 && RR > 0 && SS > 0) ? CC * RR * SS : 8 * 49;
  float x[PX][XN];
#pragma unroll
  for (int u = 0; u < PX; ++u) {
    const int h0 = p * a.sh - a.ph, w0 = (q0 + u) * a.sw - a.pw;
    if (CC > 0 && RR > 0 && SS > 0) {
#pragma unroll
      for (int r = 0; r < RR; ++r)
#pragma unroll
        for (int s2 = 0; s2 < SS; ++s2) {
          const int h = h0 + r, w = w0 + s2;
          const bool ok = h >= 0 && h < a.H && w >= 0 && w < a.W && q0 + u < a.Q;
          const T* src = a.x + ((size_t)h * a.W + w) * a.ldx;
          float v8[Vec<T>::N];
          // one 16-byte load per tap (pixel stride >= 8 channels, padding is zero)
          if (ok) load_vec(src, 0, Vec<T>::N, v8);
#pragma unroll
          for (int c = 0; c < CC; ++c) x[u][(r * SS + s2) * CC + c] = ok ? v8[c] : 0.f;
        }
    } else {
      int t = 0;
      for (int r = 0; r < R; ++r)
        for (int s2 = 0; s2 < S; ++s2) {
          const int h = h0 + r, w = w0 + s2;
          const bool ok = h >= 0 && h < a.H && w >= 0 && w < a.W && q0 + u < a.Q;
          const T* src = a.x + ((size_t)h * a.W + w) * a.ldx;
          for (int c = 0; c < C; ++c) x[u][t++] = ok ? to_f(src[c]) : 0.f;
        }
    }
  }
  const int k0 = kg * KT;
  const float* ssc = sw + a.K * RSC;
  const float* ssh = ssc + a.K;
  for (int kb = 0; kb < KT; kb += 16) {
    float acc[PX][16];
#pragma unroll
    for (int u = 0; u < PX; ++u)
#pragma unroll
      for (int j = 0; j < 16; ++j) acc[u][j] = 0.f;
    if (CC > 0 && RR > 0 && SS > 0) {
#pragma unroll
      for (int i = 0; i < XN; ++i) {
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const float wv = sw[min(k0 + kb + j, a.K - 1) * RSC + i];
#pragma unroll
          for (int u = 0; u < PX; ++u) acc[u][j] = fmaf(x[u][i], wv, acc[u][j]);
        }
      }
    } else {
      for (int i = 0; i < RSC; ++i) {
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const float wv = sw[min(k0 + kb + j, a.K - 1) * RSC + i];
#pragma unroll
          for (int u = 0; u < PX; ++u) acc[u][j] = fmaf(x[u][i], wv, acc[u][j]);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < PX; ++u) {
      if (q0 + u >= a.Q) break;
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        const int k = min(k0 + kb + j, a.K - 1);
        float y = acc[u][j] * ssc[k] + ssh[k];
        acc[u][j] = a.relu ? fmaxf(y, 0.f) : y;
      }
      const size_t pix = (size_t)p * a.Q + q0 + u;
      for (int half = 0; half < 16; half += Vec<T>::N) {
        const int k = k0 + kb + half;
        if (k >= a.K) break;
        store_vec(a.out + pix * a.ldo + k, k, a.K, acc[u] + half);
        for (int d_ = 0; d_ < a.out2.n; ++d_) store_vec(a.out2.p[d_] + pix * a.out2.ld[d_] + k, k, a.K, acc[u] + half);
      }
    }
  }
}

template <typename T, int CC, int RR, int SS, int KT>
static void launch_small(const ConvSmallArgs<T>& a, cudaStream_t st) {
  const int KG = (a.K + KT - 1) / KT;
  const size_t smem = ((size_t)a.K * a.R * a.S * a.C + 2 * a.K) * sizeof(float);
  const int px = (CC > 0 && CC * RR * SS <= 64) ? 2 : 1;
  const long long nthreads = (long long)a.P * ((a.Q + px - 1) / px) * KG;
  static bool attr_set[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && !attr_set[dev]) {
    cudaFuncSetAttribute(conv_small_c_kernel<T, CC, RR, SS, KT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         200 * 1024);
    attr_set[dev] = true;
  }
  launch_pdl(conv_small_c_kernel<T, CC, RR, SS, KT>, dim3(grid_for(nthreads, 128)), dim3(128), smem, st, a);
}

template <typename T>
void launch_conv_small_c(const ConvSmallArgs<T>& a, cudaStream_t st) {
  if (a.C == 3 && a.R == 3 && a.S == 3 && a.K % 32 == 0 && a.ldx >= Vec<T>::N)
    launch_small<T, 3, 3, 3, 32>(a, st);           // Inception / RandWire stems
  else if (a.C == 3 && a.R == 7 && a.S == 7 && a.ldx >= Vec<T>::N)
    launch_small<T, 3, 7, 7, 16>(a, st);           // SqueezeNet conv1
  else
    launch_small<T, 0, 0, 0, 16>(a, st);
}
template void launch_conv_small_c<float>(const ConvSmallArgs<float>&, cudaStream_t);
// 3x3 stride-2 stem over 3 channels (kernels.cuh Stem3W): one thread = PX
// horizontally adjacent output pixels x all K channels.  The 3 x (2PX+1)
// input window (one 16-byte load per pixel: pixel pitch >= 8 channels) sits in
// registers; the weights are read from the parameter bank with compile-time
// offsets, i.e. as the constant operand of FFMA.  fp32 accumulation in the
// oracle's (r, s, c) order per output; folded BN + ReLU epilogue.
template <typename T, int PX>
__device__ __forceinline__ void stem3_load(const ConvStem3Args<T>& a, int QP, long long it, float (&x)[3][2 * PX + 1][3]) {
  const int p = (int)(it / QP), q0 = (int)(it - (long long)p * QP) * PX;
  const int h0 = p * 2 - a.ph, w0 = q0 * 2 - a.pw;
#pragma unroll
  for (int r = 0; r < 3; ++r)
#pragma unroll
    for (int s = 0; s < 2 * PX + 1; ++s) {
      const int h = h0 + r, ww = w0 + s;
      float v[Vec<T>::N];
      if (h >= 0 && h < a.H && ww >= 0 && ww < a.W) {
        load_vec(a.x + ((size_t)h * a.W + ww) * a.ldx, 0, Vec<T>::N, v);
      } else {
#pragma unroll
        for (int j = 0; j < Vec<T>::N; ++j) v[j] = 0.f;
      }
#pragma unroll
      for (int c = 0; c < 3; ++c) x[r][s][c] = v[c];
    }
}

// KT < KK: blockIdx.y selects which KT-channel slice of the KK outputs this
// CTA computes (fewer registers per thread, more resident warps)
template <typename T, int KK, int PX, int KT = KK>
__global__ void __launch_bounds__(128) conv_stem3_kernel(const ConvStem3Args<T> a, const Stem3W w) {
  pdl_enter();
  const int QP = (a.Q + PX - 1) / PX;
  const long long it = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (it >= (long long)a.P * QP) return;
  constexpr int XW = 2 * PX + 1;
  float x[3][XW][3];
  stem3_load<T, PX>(a, QP, it, x);
  const int kb = KT < KK ? (int)blockIdx.y * KT : 0;
  static_assert(KT % 2 == 0, "channel pairs");
  // packed fp32x2 FMAs (FFMA2, sm_100): output channels (k, k+1) of one pixel
  // per instruction -- the input value broadcast to both halves, the weight
  // pair {w[i][k], w[i][k+1]} read from the parameter bank; two independent
  // round-to-nearest FMAs, the same arithmetic as fmaf in the same order
  uint64_t acc2[PX][KT / 2];
#pragma unroll
  for (int u = 0; u < PX; ++u)
#pragma unroll
    for (int k = 0; k < KT / 2; ++k) acc2[u][k] = 0ull;
#pragma unroll
  for (int r = 0; r < 3; ++r)
#pragma unroll
    for (int s = 0; s < 3; ++s)
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        const int i = (r * 3 + s) * 3 + c;
        uint64_t xb[PX];
#pragma unroll
        for (int u = 0; u < PX; ++u) {
          const float xv = x[r][2 * u + s][c];
          asm("mov.b64 %0, {%1, %1};" : "=l"(xb[u]) : "f"(xv));
        }
#pragma unroll
        for (int k = 0; k < KT; k += 2) {
          const uint64_t wv = *reinterpret_cast<const uint64_t*>(&w.w[i][kb + k]);  // uniform operand
#pragma unroll
          for (int u = 0; u < PX; ++u)
            asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc2[u][k / 2]) : "l"(xb[u]), "l"(wv));
        }
      }
  float acc[PX][KT];
#pragma unroll
  for (int u = 0; u < PX; ++u)
#pragma unroll
    for (int k = 0; k < KT / 2; ++k) {
      float lo, hi;
      asm("mov.b64 {%0, %1}, %2;" : "=f"(lo), "=f"(hi) : "l"(acc2[u][k]));
      acc[u][2 * k] = lo;
      acc[u][2 * k + 1] = hi;
    }
  const int p = (int)(it / QP), q0 = (int)(it - (long long)p * QP) * PX;
#pragma unroll
  for (int u = 0; u < PX; ++u) {
    if (q0 + u >= a.Q) break;
#pragma unroll
    for (int k = 0; k < KT; ++k) {
      const float y = acc[u][k] * w.scale[kb + k] + w.shift[kb + k];
      acc[u][k] = a.relu ? fmaxf(y, 0.f) : y;
    }
    const size_t pix = (size_t)p * a.Q + q0 + u;
#pragma unroll
    for (int c0 = 0; c0 < KT; c0 += Vec<T>::N) {
      if (kb + c0 >= a.K) break;
      // (pad channels past K, when stored, are exact zeros: zero weights, scale and shift)
      store_vec(a.out + pix * a.ldo + kb + c0, kb + c0, a.kst, acc[u] + c0);
      for (int d_ = 0; d_ < a.out2.n; ++d_) store_vec(a.out2.p[d_] + pix * a.out2.ld[d_] + kb + c0, kb + c0, a.kst, acc[u] + c0);
    }
  }
}

// (measured on B200, Inception Conv2d_1a at 4096^2: one item per thread 226 us;
// a persistent grid-stride variant prefetching the next window 334 us, its
// 216 registers leave 8 warps per SM; 16-channel slices per CTA (blockIdx.y,
// 80 registers, 24 warps per SM) 248 us; pixels per thread PX = 1/3/4:
// 1219/243/287 us -- at PX = 1 the uniform weight loads (LDCU) bound it)
template <typename T, int KK>
static void launch_stem3_k(const ConvStem3Args<T>& a, const Stem3W& w, cudaStream_t st) {
  constexpr int PX = 2;
  const long long n = (long long)a.P * ((a.Q + PX - 1) / PX);
  launch_pdl(conv_stem3_kernel<T, KK, PX>, dim3((unsigned)((n + 127) / 128)), dim3(128), 0, st, a, w);
}

template <typename T>
void launch_conv_stem3(const ConvStem3Args<T>& a, const Stem3W& w, cudaStream_t st) {
  if (a.K <= 32) launch_stem3_k<T, 32>(a, w, st);
  else launch_stem3_k<T, kStem3MaxK>(a, w, st);
}
template void launch_conv_stem3<float>(const ConvStem3Args<float>&, const Stem3W&, cudaStream_t);
template void launch_conv_stem3<bf16>(const ConvStem3Args<bf16>&, const Stem3W&, cudaStream_t);

template void launch_conv_small_c<bf16>(const ConvSmallArgs<bf16>&, cudaStream_t);
}  // namespace hios
