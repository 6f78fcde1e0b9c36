// kernels.cuh -- device kernels of the HIOS executor (sm_100a) and their
// host-side launch descriptors.  Activations are NHWC, batch 1, with a pixel
// stride `ldc` (elements, multiple of 8) so producers can write straight into
// a channel slice of a concat buffer (zero-copy concat) or of a peer GPU's
// buffer (fused transfer).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdlib>
#include <utility>

namespace hios {

typedef __nv_bfloat16 bf16;

// Memory-bound kernels are launched WITHOUT programmatic dependent launch:
// measured on Inception-v3 1024 under HIOS w=4, PDL on these kernels LOSES
// ~2.5 % (their early-resident CTAs compete with the concurrent stages); the
// tcgen05 conv keeps PDL (its prologue is long).  pdl_enter() (wait for the
// predecessor grid, then let dependents launch) is a no-op for a normal
// launch, so the kernels stay correct under either launch mode.
__device__ __forceinline__ void pdl_enter() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                              Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 0;  // see above: measured faster without PDL
  return cudaLaunchKernelEx(&cfg, k, std::forward<Args>(args)...);
}

// Remote replicas of an op's output (cross-GPU edges fused into the
// producer's epilogue): one per consumer GPU other than the
// producer's; each store of the output is repeated into every replica (peer
// memory over NVLink, or an aliased logical GPU's buffer).
constexpr int kMaxDst = 7;
template <typename T>
struct Dst {
  T* p[kMaxDst];
  int ld[kMaxDst];  // pixel stride (elements)
  int n;
};

// ------------------------------------------------------------------ conv
// Implicit-GEMM convolution on tcgen05 tensor cores (bf16 in, fp32 TMEM
// accumulate, bf16 out).  GEMM view: M = output pixels (tile = th x tw = 128
// pixels of one spatial block), N = out channels (BLOCK_N <= 256), K = R*S*C
// walked as (r, s, 64-channel chunk).  Both operands arrive by TMA into
// 128B-swizzled K-major smem tiles: A = a 3-D box of the NHWC input at the
// (r, s)-shifted, stride-traversed window (OOB = zero padding), B = a box of
// the [K][R*S][Cp] weights.
struct ConvTcArgs {
  int P, Q, K, C, R, S, sh, sw, ph, pw, dh, dw;
  int th, tw, tiles_q, tiles_m, tiles_n, n_tile, c_chunks, stages, relu;
  int halo, halo_w, a_bufs;  // halo mode: one R x halo_w input box per channel chunk
  int bo_mode;               // descriptor base-offset encoding (debug switch, 0)
  int trace;                 // write a globaltimer timeline (debug)
  int spin;                  // unused (kept for ABI of the debug switches)
  int n_mma;                 // MMA warps splitting the N tile (n_tile % (16 * n_mma) == 0)
  int occ;                   // co-resident CTAs per SM the smem plan allows (1 or 2)
  int dbg;                   // debug switches (timing experiments; 0 in production)
  int ksplit, kpsplit;       // K splits (1) and K-steps (chunk x tap) per split
  int kps;                   // K-steps (64-channel x tap) per pipeline stage
  const float* scale;  // [K] (conv_tc: folded into the weights at upload, unused by the kernel)
  const float* shift;  // [K]
  bf16* out;  int ldo; // primary output (channel offset applied)
  Dst<bf16> out2;      // remote replicas (fused cross-GPU stores)
  int bres;            // halo mode, one N tile: all weights resident in smem (loaded once per CTA)
  int tma_out;         // epilogue leaves smem by TMA bulk-tensor stores (else st.global)
  int out_sw;          // TMA-store slab width in channels (64 / 32 / 16 = 128B/64B/32B swizzle)
  int out_bufs;        // epilogue staging tiles (2: tile i's stores drain while tile i+1 is staged)
  int sres;            // folded-BN scale/shift of all K channels staged once per CTA (K <= kScaleRes)
  int epi;             // epilogue: 0 smem staging + st.global, 1 TMA bulk-tensor stores, 2 direct register stores
  // halo box geometry: hrows rows of halo_w pixels per 64-channel chunk; tap
  // row r starts r * hrow_px pixels into the box (classic halo: hrows = R,
  // hrow_px = halo_w).  vgrid = Wh > 0: "virtual-grid" halo for narrow
  // stride-1 convs -- output (p, q) is virtual position v = p * Wh + q with
  // Wh = Q + (S-1) dw (the padded input row), a tile = 128 consecutive v, the
  // box = whole padded input rows, tap (r, s) = the window at
  // v - v0 + r dh Wh + s dw; virtual columns q >= Q are computed and dropped
  int hrows, hrow_px, vgrid;
  // classic halo, stride 1: hk consecutive output rows per tile (hk > 1: one
  // box of R + hk - 1 input rows feeds hk accumulators, so every input row and
  // every weight stage crosses L2 -> SM once per hk output rows instead of R /
  // once per row; tile_row = output-row group, th = hk)
  int hk;
  int hk_px;  // hk > 1 for a 1x1 conv: the tile is 2 x 128 consecutive pixels of one row (box 256 px)
  int nacc;  // TMEM accumulator sets (2: the epilogue of tile i overlaps the MMAs of tile i+1; 1 when
             // 2 * hk * n_tile > 512 columns)
  int st256;  // direct-store epilogue: every destination 32-byte aligned per pixel (256-bit stores)
};
constexpr int kScaleRes = 512;
constexpr int kMaxABufs = 6;  // halo-mode input boxes in flight

// CUDA-core implicit GEMM (fp32) for the fp32 path (1e-4 parity).
struct ConvSimtArgs {
  const float* x; int H, W, C, ldx;
  const float* w;      // [K][R][S][C]
  int P, Q, K, R, S, sh, sw, ph, pw, dh, dw, relu;
  const float* scale; const float* shift;
  float* out; int ldo;
  Dst<float> out2;
};

// Depthwise stage of a separable conv: a = sum_i agg_i x_i ; relu? ; depthwise.
#define HIOS_MAX_IN 16
template <typename T>
struct DwArgs {
  const T* x[HIOS_MAX_IN]; int ldx[HIOS_MAX_IN]; float agg[HIOS_MAX_IN]; int n_in;
  int H, W, C, P, Q, R, S, sh, sw, ph, pw, pre_relu;
  const float* w;  // [R*S][C]
  T* out; int ldo;
};

template <typename T>
struct PoolArgs {
  const T* x; int H, W, C, ldx;
  int P, Q, kh, kw, sh, sw, ph, pw, is_max, cip;
  T* out; int ldo;
  Dst<T> out2;
};

template <typename T>
struct AddArgs {
  const T* x[HIOS_MAX_IN]; int ldx[HIOS_MAX_IN]; float agg[HIOS_MAX_IN]; int n_in;
  int HW, C, relu;
  T* out; int ldo;
  Dst<T> out2;
};

// direct conv for C <= 8 input channels (stems): fp32 weights [K][R][S][C]
template <typename T>
struct ConvSmallArgs {
  const T* x; int H, W, C, ldx;
  const float* w; const float* scale; const float* shift;
  int P, Q, K, R, S, sh, sw, ph, pw, relu;
  T* out; int ldo; Dst<T> out2;
};

// space-to-depth of a stride-2 small-C stem input (exec.cu: s2d_conv)
template <typename T>
struct S2dArgs {
  const T* x; int H, W, C, ldx, ph, pw;
  T* out; int P2, Q2, ldo;  // X' is P2 x Q2 x 4C (pixel stride ldo)
};

template <typename T>
struct CopyArgs {
  const T* x; int ldx; int HW, C; T* out; int ldo;
};

// launchers (stream-ordered, capture-safe)
void launch_conv_tc(const CUtensorMap& mx, const CUtensorMap& mw, const CUtensorMap& mo, const CUtensorMap& mo2,
                    const ConvTcArgs& a, int grid, size_t smem, cudaStream_t st);
size_t conv_tc_smem_bytes(const ConvTcArgs& a);
// the convs of one stage in one launch (SM ranges per op)
struct ConvTcOp {
  CUtensorMap mx, mw, mo, mo2;
  ConvTcArgs a;
};
constexpr int kMaxGroup = 6;
struct ConvTcGroup {
  ConvTcOp op[kMaxGroup];
  int n;
  int cta0[kMaxGroup + 1];  // op i owns CTAs [cta0[i], cta0[i+1])
};
void launch_conv_tc_group(const ConvTcGroup& G, size_t smem, cudaStream_t st);
__host__ __device__ inline uint32_t halo_bytes_of(int R, int halo_w) {
  return ((uint32_t)R * halo_w * 128u + 1023u) & ~1023u;
}
void launch_conv_simt(const ConvSimtArgs& a, cudaStream_t st);
template <typename T> void launch_conv_small_c(const ConvSmallArgs<T>& a, cudaStream_t st);
// 3x3 stride-2 stems over 3 input channels (Inception-v3 Conv2d_1a, RandWire
// conv1): the 27 x KK folded weights and the BN scale/shift travel in the
// kernel's parameter bank, so every multiply-add is one FFMA with a constant
// operand (no shared-memory weight loads); see misc.cu conv_stem3_kernel
constexpr int kStem3MaxK = 40;
struct __align__(8) Stem3W {
  float w[27][kStem3MaxK];  // [(r*3+s)*3+c][k]  (channel pairs 8-byte aligned: fma.rn.f32x2)
  float scale[kStem3MaxK], shift[kStem3MaxK];
};
template <typename T>
struct ConvStem3Args {
  const T* x; int H, W, ldx;
  int P, Q, K, ph, pw, relu;
  int kst;  // channels stored per pixel: K, or rup(K, 8) when the pad channels are this op's own
  T* out; int ldo; Dst<T> out2;
};
template <typename T> void launch_conv_stem3(const ConvStem3Args<T>& a, const Stem3W& w, cudaStream_t st);

template <typename T> void launch_dw(const DwArgs<T>& a, cudaStream_t st);
template <typename T> void launch_pool(const PoolArgs<T>& a, cudaStream_t st);
template <typename T> void launch_add(const AddArgs<T>& a, cudaStream_t st);
template <typename T> void launch_copy(const CopyArgs<T>& a, cudaStream_t st);
template <typename T> void launch_relu_copy(const CopyArgs<T>& a, cudaStream_t st);
template <typename T> void launch_s2d(const S2dArgs<T>& a, cudaStream_t st);
template <typename T> void launch_gap(const T* x, int HW, int C, int ldx, T* out, cudaStream_t st);
template <typename T> void launch_linear(const T* x, int Cin, const T* w, int ldw, const float* b, int K,
                                         T* out, cudaStream_t st);
template <typename T> void launch_input(const float* nchw, int C, int H, int W, T* out, int ldo,
                                        cudaStream_t st);
template <typename T> void launch_output(const T* x, int C, int H, int W, int ldx, float* nchw,
                                         cudaStream_t st);
void launch_epoch(unsigned* epoch, cudaStream_t st);
void launch_signal(const unsigned* epoch, unsigned* flag, cudaStream_t st);
void launch_wait(const unsigned* epoch, const unsigned* flag, unsigned lag, cudaStream_t st);
void launch_fill(void* p, size_t bytes, cudaStream_t st);

// tensor maps (driver entry point resolved at run time; no -lcuda)
bool make_tmap_3d(CUtensorMap* m, const void* base, uint64_t d0, uint64_t d1, uint64_t d2,
                  uint64_t stride1_bytes, uint64_t stride2_bytes, uint32_t b0, uint32_t b1, uint32_t b2,
                  uint32_t e1, uint32_t e2, int swizzle_bytes = 128);

}  // namespace hios
