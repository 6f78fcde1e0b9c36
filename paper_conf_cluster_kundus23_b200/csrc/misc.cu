// misc.cu -- HBM-bound operator kernels: pooling, depthwise
// stage of separable convs, n-ary add, copy (concat fallback and peer pushes),
// GAP, linear head, input/output layout conversion, and the epoch flags used
// for cross-GPU edges (a10/a11).  NHWC with a pixel stride; each thread owns
// one pixel x VEC channels (16-byte vectors: 8 bf16 or 4 fp32) so a warp reads
// contiguous 512-byte runs.
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

static inline unsigned grid_for(long long n, int block) {
  long long g = (n + block - 1) / block;
  return (unsigned)(g < 1 ? 1 : g);
}

// ---------------------------------------------------------------- pooling
// grid = (ceil(Q * CG / 256), P): one output row per blockIdx.y; KH/KW > 0
// unroll the window (loads hoisted, accumulated immediately).
template <typename T, int KH, int KW>
__global__ void pool_kernel(const PoolArgs<T> a) {
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
  if (a.out2) store_vec(a.out2 + pix * a.ldo2 + c, c, a.C, acc);
}

template <typename T>
void launch_pool(const PoolArgs<T>& a, cudaStream_t st) {
  constexpr int N = Vec<T>::N;
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

template <typename T>
void launch_dw(const DwArgs<T>& a, cudaStream_t st) {
  constexpr int N = Vec<T>::N;
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
  if (a.out2) store_vec(a.out2 + pix * a.ldo2 + c, c, a.C, acc);
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
  if (c + N <= a.C && ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 15) == 0) {
    *reinterpret_cast<uint4*>(dst) = *reinterpret_cast<const uint4*>(src);
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

__global__ void wait_kernel(const unsigned* epoch, const unsigned* flag, unsigned lag) {
  const unsigned target = *epoch - lag;
  unsigned v;
  while (true) {
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
    if ((int)(v - target) >= 0) break;
    __nanosleep(64);
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

// explicit instantiations
#define HIOS_INST(T)                                                                                   \
  template void launch_pool<T>(const PoolArgs<T>&, cudaStream_t);                                      \
  template void launch_dw<T>(const DwArgs<T>&, cudaStream_t);                                          \
  template void launch_add<T>(const AddArgs<T>&, cudaStream_t);                                        \
  template void launch_copy<T>(const CopyArgs<T>&, cudaStream_t);                                      \
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
        if (a.out2) store_vec(a.out2 + pix * a.ldo2 + k, k, a.K, acc[u] + half);
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
template void launch_conv_small_c<bf16>(const ConvSmallArgs<bf16>&, cudaStream_t);
}  // namespace hios
