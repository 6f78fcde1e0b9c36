// conv_tc.cu -- implicit-GEMM convolution on Blackwell 5th-gen tensor cores
// ("convolution ... operators" of G).
//
// GEMM view: M = output pixels, N = output channels, K = R*S*C.  bf16
// operands, fp32 accumulation in TMEM, folded-BN scale/shift + ReLU + bf16
// epilogue.  Persistent, warp-specialised CTA (384 threads):
//   warps 0-3   TMA producers (one lane each, K-steps round-robin)
//   warps 4-7   MMA issuers (one lane each, one N sub-tile each): 4 x
//               tcgen05.mma.kind::f16 (M=128, N=n_tile/n_mma, K=16) per K-step;
//               warp 4 allocates TMEM
//   warps 8-11  epilogue: tcgen05.ld -> scale/shift/ReLU -> bf16 -> smem
//               staging -> coalesced stores
//               to the local buffer / concat slice and, optionally, a peer
//               GPU's replica (cross-GPU edge fused into the epilogue)
// Two TMEM accumulators (2 x n_tile columns) let the epilogue of tile i run
// under the main loop of tile i+1.  Tiles are walked N-fastest so CTAs that
// share an input tile run together (L2 reuse).
//
// Operand staging (both 128B-swizzled, K-major, by TMA):
//   halo mode  (stride 1 along W, one output row of 128 pixels per tile):
//              per 64-channel chunk ONE box of R input rows x (128+(S-1)dw)
//              pixels; the A operand of tap (r, s) is the row window starting
//              at pixel r*Wh + s*dw of that box (descriptor start + base
//              offset), so every input pixel crosses L2->SM once per tile
//              instead of R*S times; B (weights of one tap) streams through
//              a ring.
//   tap mode   (generic: strides, narrow outputs): per K-step (r, s, chunk)
//              one box of th x tw output positions of the (r,s)-shifted input
//              with the conv stride as TMA traversal stride, plus B.
// Out-of-bounds TMA reads return zero = the convolution's zero padding.
#include <cstdio>
#include <cstdlib>

#include "kernels.cuh"

namespace hios {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
// try_wait suspends in hardware for a bounded time per probe; a barrier that
// never completes (a producer / consumer mismatch) traps after 2^26 failed
// probes (seconds) instead of hanging the GPU (the run then fails with a CUDA
// error).  Kept as one tight asm loop: the wait sits in the MMA issue path.
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p, q;\n"
      ".reg .u32 n;\n"
      "mov.u32 n, 0;\n"
      "HIOS_WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@p bra HIOS_DONE_%=;\n"
      "add.u32 n, n, 1;\n"
      "setp.lt.u32 q, n, 67108864;\n"
      "@q bra HIOS_WAIT_%=;\n"
      "trap;\n"
      "HIOS_DONE_%=:\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void sts128(uint32_t addr, uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3) {
  asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(a0), "r"(a1), "r"(a2), "r"(a3)
               : "memory");
}
__device__ __forceinline__ uint4 lds128(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr)
               : "memory");
  return v;
}
// folded-BN epilogue of two accumulator columns: + shift (the scale is folded
// into the weights at upload, exec.cu conv_layout), optional ReLU, rounded to
// bf16x2; lo -> bits [0,16)
__device__ __forceinline__ uint32_t bias_relu_pack(uint32_t lo, uint32_t hi, float b_lo, float b_hi, int relu) {
  float y0 = __uint_as_float(lo) + b_lo, y1 = __uint_as_float(hi) + b_hi;
  if (relu) { y0 = fmaxf(y0, 0.f); y1 = fmaxf(y1, 0.f); }
  __nv_bfloat162 b2 = __floats2bfloat162_rn(y0, y1);
  return *reinterpret_cast<uint32_t*>(&b2);
}
__device__ __forceinline__ void st_global_256(void* p, const uint32_t (&v)[8]) {
  asm volatile("st.global.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(p), "r"(v[0]), "r"(v[1]), "r"(v[2]),
               "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
               : "memory");
}
__device__ __forceinline__ uint16_t lds16(uint32_t addr) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(addr) : "memory");
  return v;
}

// non-blocking probe loop (no HW suspend between probes)
__device__ __forceinline__ void mbar_spin(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "HIOS_SPIN_%=:\n"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra HIOS_SPIN_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_3d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1,
                                            int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], "
      "[%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* map, uint32_t src, int c0, int c1, int c2) {
  asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(src), "r"(c0), "r"(c1), "r"(c2)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// one lane of a converged warp (the others skip the guarded issue but keep
// running the warp-uniform loop, so operands stay in uniform registers)
__device__ __forceinline__ bool elect_one() {
  uint32_t pred = 0;
  asm volatile(
      "{\n"
      ".reg .pred P;\n"
      "elect.sync _|P, 0xffffffff;\n"
      "selp.b32 %0, 1, 0, P;\n"
      "}\n"
      : "=r"(pred));
  return pred != 0;
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// UMMA shared-memory descriptor: K-major, 128B swizzle, 8-row atoms 1024 B
// apart.  The swizzle phase follows the absolute smem address bits [7,10), so
// a window starting at any 128-byte row of a TMA-written (same-swizzle) box is
// addressed with base offset 0 (measured on B200: a non-zero base offset
// breaks the shifted halo windows).
__device__ __forceinline__ uint64_t umma_desc_sw128(uint32_t saddr, int bo_mode = 0) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);        // start address  [0,14)
  d |= (uint64_t)1 << 16;                          // LBO (unused for swizzled K-major)
  d |= (uint64_t)(1024 >> 4) << 32;                // SBO = 1024 B
  d |= (uint64_t)1 << 46;                          // descriptor version (sm_100)
  if (bo_mode) d |= (uint64_t)((saddr >> 7) & 7u) << 49;  // (measured: must stay 0)
  d |= (uint64_t)2 << 61;                          // SWIZZLE_128B
  return d;
}

__device__ __forceinline__ void mma_bf16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
// the same, issued only where `on` != 0 (elected lane) -- predicated instead
// of branched, so the issuing warp's loop stays convergent and its operands
// stay in uniform registers
__device__ __forceinline__ void mma_bf16_on(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc,
                                            uint32_t on) {
  asm volatile(
      "{\n"
      ".reg .pred p, q;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "setp.ne.b32 q, %5, 0;\n"
      "@q tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc), "r"(on));
}
__device__ __forceinline__ void mma_commit_on(uint32_t bar, uint32_t on) {
  asm volatile(
      "{\n"
      ".reg .pred q;\n"
      "setp.ne.b32 q, %1, 0;\n"
      "@q tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n"
      "}\n" ::"r"(bar),
      "r"(on)
      : "memory");
}
__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar)
               : "memory");
}

// halo mode, B ring: one chunk's R_ x S_ taps, KPS_ taps per ring stage;
// HK_ output rows per tile: each weight stage feeds HK_ accumulators (TMEM
// columns dstride apart), output row j reading the window one box row lower
template <int R_, int S_, int KPS_, int HK_>
__device__ __forceinline__ void halo_taps_ring(uint32_t d, uint64_t a0, uint64_t bD0, uint64_t bst16, uint64_t b16,
                                               uint32_t idesc, int kv, uint32_t on, uint64_t row_r16,
                                               uint64_t row_s16, uint32_t accum, uint32_t& st, uint32_t& ph,
                                               uint32_t ST, uint32_t full0, uint32_t empty0, uint32_t dstride) {
  uint64_t b0 = 0;
#pragma unroll
  for (int t = 0; t < R_ * S_; ++t) {
    if (t % KPS_ == 0) {
      mbar_wait(full0 + 8 * st, ph);
      tc_fence_after();
      b0 = bD0 + (uint64_t)st * bst16;
    }
    const uint64_t bd = b0 + (uint64_t)(t % KPS_) * b16;
#pragma unroll
    for (int j = 0; j < HK_; ++j) {
      const uint64_t ad = a0 + (uint64_t)(t / S_ + j) * row_r16 + (uint64_t)(t % S_) * row_s16;
      const uint32_t dj = d + (uint32_t)j * dstride;
      mma_bf16_on(dj, ad, bd, idesc, t == 0 ? accum : 1u, on);
      if (kv > 1) mma_bf16_on(dj, ad + 2, bd + 2, idesc, 1u, on);
      if (kv > 2) mma_bf16_on(dj, ad + 4, bd + 4, idesc, 1u, on);
      if (kv > 3) mma_bf16_on(dj, ad + 6, bd + 6, idesc, 1u, on);
    }
    if (t % KPS_ == KPS_ - 1 || t == R_ * S_ - 1) {
      mma_commit_on(empty0 + 8 * st, on);
      if (++st == ST) { st = 0; ph ^= 1u; }
    }
  }
}

// halo mode, resident weights: one chunk's R_ x S_ taps (kv K=16 slices
// each) with compile-time window offsets r * row_r16 + s * row_s16; HK_ rows
template <int R_, int S_, int HK_>
__device__ __forceinline__ void halo_taps_bres(uint32_t d, uint64_t a0, uint64_t b0, uint32_t idesc, int kv,
                                               uint32_t on, uint64_t row_r16, uint64_t row_s16, uint64_t b16,
                                               uint32_t accum, uint32_t dstride) {
#pragma unroll
  for (int t = 0; t < R_ * S_; ++t) {
    const uint64_t bd = b0 + (uint64_t)t * b16;
#pragma unroll
    for (int j = 0; j < HK_; ++j) {
      const uint64_t ad = a0 + (uint64_t)(t / S_ + j) * row_r16 + (uint64_t)(t % S_) * row_s16;
      const uint32_t dj = d + (uint32_t)j * dstride;
      mma_bf16_on(dj, ad, bd, idesc, t == 0 ? accum : 1u, on);
      if (kv > 1) mma_bf16_on(dj, ad + 2, bd + 2, idesc, 1u, on);
      if (kv > 2) mma_bf16_on(dj, ad + 4, bd + 4, idesc, 1u, on);
      if (kv > 3) mma_bf16_on(dj, ad + 6, bd + 6, idesc, 1u, on);
    }
  }
}

// the same for ONE elected lane (the caller branches on elect_one()): plain,
// unpredicated tcgen05.mma with a compile-time K=16 slice count KV_.  With a
// single active thread ptxas keeps the descriptors in uniform registers and
// issues the MMAs back to back; issued lane-predicated from the converged warp
// every descriptor went through R2UR (~150 cycles per MMA in the kernel).
// Measured: Conv2d_2a-4096 298 -> 192 us, Conv2d_2b 291 -> 262 us, Conv2d_2a
// at 1024^2 21.9 -> 16.0 us.  (The whole issue loop on one lane -- ring and
// tap modes too -- measured slower for the weight-ring convs: Conv2d_4a-4096
// 367 -> 379 us, NASNet-2048 10.78 -> 11.10 ms.)
template <int R_, int S_, int HK_, int KV_>
__device__ __forceinline__ void halo_taps_bres_lane(uint32_t d, uint64_t a0, uint64_t b0, uint32_t idesc,
                                                    uint64_t row_r16, uint64_t row_s16, uint64_t b16, uint32_t accum,
                                                    uint32_t dstride) {
#pragma unroll
  for (int t = 0; t < R_ * S_; ++t) {
    const uint64_t bd = b0 + (uint64_t)t * b16;
#pragma unroll
    for (int j = 0; j < HK_; ++j) {
      const uint64_t ad = a0 + (uint64_t)(t / S_ + j) * row_r16 + (uint64_t)(t % S_) * row_s16;
      const uint32_t dj = d + (uint32_t)j * dstride;
#pragma unroll
      for (int q = 0; q < KV_; ++q) mma_bf16(dj, ad + 2 * q, bd + 2 * q, idesc, (t == 0 && q == 0) ? accum : 1u);
    }
  }
}
// dispatch on the chunk's K=16 slice count (1, 2 or 4; 3 -> false: the caller
// issues the lane-predicated loop)
template <int R_, int S_, int HK_, int KVMIN>
__device__ __forceinline__ void halo_taps_bres_lane_kv(int kv, uint32_t d, uint64_t a0, uint64_t b0, uint32_t idesc,
                                                       uint64_t row_r16, uint64_t row_s16, uint64_t b16, uint32_t accum,
                                                       uint32_t dstride) {
  if (kv == 4) halo_taps_bres_lane<R_, S_, HK_, 4>(d, a0, b0, idesc, row_r16, row_s16, b16, accum, dstride);
  else if (KVMIN <= 3 && kv == 3) halo_taps_bres_lane<R_, S_, HK_, 3>(d, a0, b0, idesc, row_r16, row_s16, b16, accum, dstride);
  else if (KVMIN <= 2 && kv == 2) halo_taps_bres_lane<R_, S_, HK_, 2>(d, a0, b0, idesc, row_r16, row_s16, b16, accum, dstride);
  else if (KVMIN <= 1) halo_taps_bres_lane<R_, S_, HK_, 1>(d, a0, b0, idesc, row_r16, row_s16, b16, accum, dstride);
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// tcgen05.ld without the wait: the destination registers are only valid after
// tmem_wait_pin() (which names them as in/out operands, so no use of them can
// be scheduled ahead of the wait)
__device__ __forceinline__ void tmem_ld16_nw(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_pin(uint32_t (&r)[16]) {
  asm volatile("tcgen05.wait::ld.sync.aligned;"
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]), "+r"(r[6]), "+r"(r[7]),
                 "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]), "+r"(r[12]), "+r"(r[13]), "+r"(r[14]),
                 "+r"(r[15])::"memory");
}
__device__ __forceinline__ void pin16(uint32_t (&r)[16]) {
  asm volatile(""
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]), "+r"(r[6]), "+r"(r[7]),
                 "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]), "+r"(r[12]), "+r"(r[13]), "+r"(r[14]),
                 "+r"(r[15])::"memory");
}

// optional timeline instrumentation (HIOS_TRACE): globaltimer at checkpoints
__device__ unsigned long long g_conv_trace[256 * 8];
__device__ unsigned long long g_conv_trace2[32 * 48];  // per CTA: issue[16], full[16], empty_ok[16]
__device__ unsigned long long g_conv_trace3[32 * 8];   // per CTA: epilogue checkpoints
__device__ unsigned long long g_conv_trace4[32 * 16];  // per CTA: first-tile epilogue, fine-grained
__device__ unsigned long long g_conv_trace5[32 * 48];  // per CTA: epilogue tfull[16], stores issued[16]
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define TRACE2(slot, k)                                                   \
  do {                                                                    \
    if (a.trace && blockIdx.x < 32 && (k) < 16) g_conv_trace2[blockIdx.x * 48 + (slot) * 16 + (k)] = gtimer(); \
  } while (0)
#define TRACE3(k)                                                         \
  do {                                                                    \
    if (a.trace && blockIdx.x < 32) g_conv_trace3[blockIdx.x * 8 + (k)] = gtimer(); \
  } while (0)
#define TRACE4(k)                                                         \
  do {                                                                    \
    if (a.trace && blockIdx.x < 32 && tcount == 0 && et == 0) g_conv_trace4[blockIdx.x * 16 + (k)] = gtimer(); \
  } while (0)
#define TRACE5(slot, k)                                                   \
  do {                                                                    \
    if (a.trace && blockIdx.x < 32 && (k) < 16 && et == 0) g_conv_trace5[blockIdx.x * 48 + (slot) * 16 + (k)] = gtimer(); \
  } while (0)
#define TRACE(k)                                                          \
  do {                                                                    \
    if (a.trace && blockIdx.x < 256) g_conv_trace[blockIdx.x * 8 + (k)] = gtimer(); \
  } while (0)

// split and output-tile index of persistent tile number `tile`
__device__ __forceinline__ void split_of(const ConvTcArgs& a, int tile, int tiles_mn, int& split, int& tmn) {
  split = tile / tiles_mn;
  tmn = tile - split * tiles_mn;
}

static __host__ __device__ inline uint32_t tmem_cols(int n) {
  uint32_t c = 32;
  while ((int)c < n) c <<= 1;
  return c;
}


constexpr int kProducers = 4;  // TMA issuing warps
constexpr int kMma = 4;        // MMA issuing warps (one N sub-tile each)
constexpr int kEpi = 4;        // epilogue warps (one TMEM lane quarter each)
constexpr int kThreads = 32 * (kProducers + kMma + kEpi);
constexpr int kEpiWarp0 = kProducers + kMma;

// output pixel of accumulator row m of M-tile m_blk (tile origin p0, q0)
__device__ __forceinline__ void tile_pixel(const ConvTcArgs& a, int m_blk, int p0, int q0, int m, int& p, int& q) {
  if (a.vgrid) {
    const int v = m_blk * 128 + m;
    p = v / a.vgrid;
    q = v - p * a.vgrid;  // q >= Q: a virtual column, dropped by the caller
  } else {
    const int hh = m / a.tw;
    p = p0 + hh;
    q = q0 + (m - hh * a.tw);
  }
}

__host__ __device__ inline uint32_t stage_pitch(int n_tile) { return (uint32_t)n_tile * 2u + 16u; }

// One conv's persistent tile loop on CTAs cta = 0..ncta-1 of its SM range
// (conv_tc_kernel: the whole grid; conv_tc_group_kernel: the op's partition).
__device__ __forceinline__ void conv_tc_body(const CUtensorMap* pmx, const CUtensorMap* pmw,
                                             const CUtensorMap* pmo, const CUtensorMap* pmo2, const ConvTcArgs& a,
                                             const int cta, const int ncta) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int ST = a.stages;
  const uint32_t A_BYTES = 128 * 128;
  const uint32_t B_BYTES = (uint32_t)a.n_tile * 128;
  const uint32_t H_BYTES = a.halo ? halo_bytes_of(a.hrows, a.halo_w) : 0u;
  const uint32_t PITCH = stage_pitch(a.n_tile);
  uint8_t* sA = smem;  // halo: a_bufs x H_BYTES ; tap: ST x kps x A_BYTES
  uint8_t* sB = smem + (a.halo ? a.a_bufs * H_BYTES : ST * a.kps * A_BYTES);
  // B: a ring of ST stages x kps K-steps, or (bres) every K-step's weights resident
  uint8_t* sOut = sB + (a.bres ? (uint32_t)(a.c_chunks * a.R * a.S) : (uint32_t)(ST * a.kps)) * B_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sOut + (uint32_t)a.out_bufs * 128u * PITCH);
  // barriers: full[ST] empty[ST] afull[2] aempty[2] tfull[2] tempty[2]
  const uint32_t full0 = smem_u32(bars), empty0 = full0 + 8 * ST;
  const uint32_t afull0 = empty0 + 8 * ST, aempty0 = afull0 + 8 * kMaxABufs, tfull0 = aempty0 + 8 * kMaxABufs,
                 tempty0 = tfull0 + 16;
  constexpr int kBarX = 2 * kMaxABufs + 4;  // afull/aempty[kMaxABufs], tfull/tempty[2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * ST + kBarX);
  const uint32_t bres_bar = smem_u32(bars + 2 * ST + kBarX + 1);  // resident weights landed
  float* s_scale = reinterpret_cast<float*>(bars + 2 * ST + kBarX + 2);  // [kScaleRes]
  float* s_shift = s_scale + kScaleRes;                            // [kScaleRes]

  // warp index via a shuffle from lane 0: provably warp-uniform for ptxas, so
  // role-derived values (MMA sub-tile, TMEM column, B descriptor) stay in
  // uniform registers (CUTLASS canonical_warp_idx_sync)
  const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
  // the whole TMEM (512 columns): one conv CTA per SM (164 registers x 384
  // threads), so the allocation is always column 0 -- a compile-time TMEM
  // base keeps the MMA issue loop's accumulator address in uniform registers
  // (measured: a loaded base was re-broadcast with R2UR per MMA)
  const uint32_t ncols = 512;
  const int RS = a.R * a.S;
  const int tiles_mn = a.tiles_m * a.tiles_n;
  const int tiles = tiles_mn * a.ksplit;  // split-K: each split owns a chunk range
  const int nmma = a.n_mma;  // active MMA warps; N sub-tile = n_tile / nmma
  const int n_sub = a.n_tile / nmma;
  if (threadIdx.x == 0) TRACE(0);

  if (threadIdx.x == 0) {
    for (int i = 0; i < ST; ++i) {
      mbar_init(full0 + 8 * i, 1);
      mbar_init(empty0 + 8 * i, nmma);
    }
    mbar_init(bres_bar, 1);
    for (int i = 0; i < kMaxABufs; ++i) {
      mbar_init(afull0 + 8 * i, 1);
      mbar_init(aempty0 + 8 * i, nmma);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(tfull0 + 8 * i, nmma);
      mbar_init(tempty0 + 8 * i, 32 * kEpi);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(pmx)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(pmw)) : "memory");
    if (a.tma_out) {
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(pmo)) : "memory");
      if (a.out2.n) asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(pmo2)) : "memory");
    }
  }
  if (warp == kProducers) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(ncols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (*tmem_slot != 0u) __trap();  // cannot happen with one CTA per SM
  const uint32_t tmem = 0u;
  if (threadIdx.x == 0) TRACE(1);
  // Programmatic dependent launch: the set-up above (barriers, TMEM,
  // descriptor prefetch) overlapped the previous kernel's tail; inputs are
  // read only after the predecessor grid has completed and flushed.
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  asm volatile("griddepcontrol.wait;" ::: "memory");

  // Each stage is owned by one producer warp (st = w mod n_prod, n_prod | ST),
  // so a stage's empty barrier is never waited on two phases ahead (parity
  // waits cannot tell phase u from u-2).  A stage carries up to `kps`
  // consecutive K-steps: one full/empty handshake (~0.3 us of fixed latency,
  // measured) is amortised over kps x 4 MMAs.
  const int n_prod = (ST % 4 == 0) ? 4 : ((ST % 2 == 0) ? 2 : 1);
  const int KPS = a.kps;
  const uint32_t A_STAGE = a.halo ? 0u : (uint32_t)KPS * A_BYTES;
  const uint32_t B_STAGE = (uint32_t)KPS * B_BYTES;
  if (warp < kProducers) {
    if (warp < n_prod || (a.halo && warp == 0)) {
      // ------------------------------------------------------ TMA producers
      uint32_t st = 0, ph = 0, ab = 0, aph = 0, ks = 0;
      int hcount = 0;  // halo loads issued (trace only)
      int mine = warp < n_prod ? warp : 1 << 30;
      const uint32_t sA0 = smem_u32(sA), sB0 = smem_u32(sB);
      if (a.bres && warp == 0) {
        // the CTA's whole B (tiles_n == 1): every (chunk, tap) box once
        if (elect_one()) {
          const int nb = a.c_chunks * RS;
          mbar_expect_tx(bres_bar, (uint32_t)nb * B_BYTES);
          for (int i = 0; i < nb; ++i) {
            const int c2 = i / RS;
            tma_load_3d(sB0 + (uint32_t)i * B_BYTES, pmw, bres_bar, c2 * 64, i - c2 * RS, 0);
          }
        }
        __syncwarp();
      }
      if (a.bres) mine = 1 << 30;  // no B ring
      for (int tile = cta; tile < tiles; tile += ncta) {
        int split, tmn;
        split_of(a, tile, tiles_mn, split, tmn);
        const int m_blk = tmn / a.tiles_n, n_blk = tmn - m_blk * a.tiles_n;
        const int tp = m_blk / a.tiles_q, tq = m_blk - tp * a.tiles_q;
        const int p0 = tp * a.th, q0 = tq * a.tw, n0 = n_blk * a.n_tile;
        // vgrid: the box = whole padded input rows from the tile's first row
        const int x0 = a.vgrid ? -a.pw : q0 * a.sw - a.pw;
        const int y0 = a.vgrid ? (m_blk * 128) / a.vgrid - a.ph : p0 * a.sh - a.ph;
        // split-K: this split's K-steps [k_lo, k_hi) (any (chunk, tap) boundary)
        const int k_lo = split * a.kpsplit, k_hi = min(a.c_chunks * RS, k_lo + a.kpsplit);
        int cc = k_lo / RS, rs = k_lo - (k_lo / RS) * RS;
        int r = rs / a.S, s = rs - (rs / a.S) * a.S;
        int k = k_lo;
        while (k < k_hi) {
          if (a.halo && rs == 0 && warp == 0) {
            mbar_wait(aempty0 + 8 * ab, aph ^ 1u);
            if (elect_one()) {
              if (a.bres) TRACE2(0, hcount);
              if (a.dbg & 4) {  // timing experiment: no halo loads (stale smem)
                mbar_arrive(afull0 + 8 * ab);
              } else {
                mbar_expect_tx(afull0 + 8 * ab, (uint32_t)a.hrows * a.halo_w * 128u);
                tma_load_3d(sA0 + ab * H_BYTES, pmx, afull0 + 8 * ab, cc * 64, x0, y0);
              }
            }
            __syncwarp();
          }
          if (a.halo && rs == 0) {
            if (++ab == (uint32_t)a.a_bufs) { ab = 0; aph ^= 1u; }
            ++hcount;
          }
          // K-steps of this stage: up to KPS, never crossing a chunk in halo mode
          int nk = KPS;
          if (a.halo) nk = min(nk, RS - rs);
          nk = min(nk, k_hi - k);
          if (mine == 0) {
            mbar_wait(empty0 + 8 * st, ph ^ 1u);
            if (elect_one()) {
              TRACE2(2, ks);
              int c2, rs2, r2, s2;
              const int cnt = nk;  // this stage's K-steps (tap mode may cross chunks)
              if (a.dbg & 2) {
                mbar_arrive(full0 + 8 * st);
              } else {
                mbar_expect_tx(full0 + 8 * st, (uint32_t)cnt * ((a.halo ? 0u : A_BYTES) + B_BYTES));
                c2 = cc; rs2 = rs; r2 = r; s2 = s;
                for (int j = 0; j < cnt; ++j) {
                  if (!a.halo)
                    tma_load_3d(sA0 + st * A_STAGE + j * A_BYTES, pmx, full0 + 8 * st, c2 * 64, x0 + s2 * a.dw,
                                y0 + r2 * a.dh);
                  tma_load_3d(sB0 + st * B_STAGE + j * B_BYTES, pmw, full0 + 8 * st, c2 * 64, rs2, n0);
                  if (++s2 == a.S) { s2 = 0; ++r2; }
                  if (++rs2 == RS) { rs2 = 0; r2 = 0; s2 = 0; ++c2; }
                }
              }
              if (ks == 0) TRACE(2);
              TRACE2(0, ks);
            }
            __syncwarp();
            mine = n_prod;
          }
          --mine;
          if (++st == (uint32_t)ST) { st = 0; ph ^= 1u; }
          // advance by nk K-steps
          for (int j = 0; j < nk; ++j, ++ks) {
            if (++s == a.S) { s = 0; ++r; }
            if (++rs == RS) { rs = 0; r = 0; s = 0; ++cc; }
          }
          k += nk;
        }
      }
    }
    __syncwarp();
  } else if (warp < kProducers + kMma) {
    const int j = warp - kProducers;  // N sub-tile of this MMA warp
    if (j < nmma) {
      // ------------------------------------------------------ MMA issuers
      const uint32_t idesc = (1u << 4)                          // D f32
                             | (1u << 7)                        // A bf16
                             | (1u << 10)                       // B bf16
                             | ((uint32_t)(n_sub >> 3) << 17)   // N
                             | ((uint32_t)(128 >> 4) << 24);    // M = 128
      uint32_t st = 0, ph = 0, ab = 0, aph = 0, ks = 0, acc = 0, tph = 0;
      const uint32_t sA0 = smem_u32(sA), sB0 = smem_u32(sB) + (uint32_t)(j * n_sub) * 128u;
      const uint32_t row_r = (uint32_t)a.hrow_px * 128u, row_s = (uint32_t)a.dw * 128u;
      int tcount = 0;
      if (a.bres) {
        mbar_wait(bres_bar, 0);
        tc_fence_after();
      }
      if (a.halo) {
        // halo mode, lean issue loop: per tap two 64-bit descriptor adds and
        // up to 4 predicated MMAs (no branches on the elected lane, no
        // per-K-step parameter reloads)
        const int C = a.C, nchunks = a.c_chunks, S_ = a.S, kps = KPS, bres = a.bres, abufs = a.a_bufs;
        const uint32_t on = elect_one() ? 1u : 0u;
        const uint32_t ST_ = (uint32_t)ST;
        const uint64_t row_r16 = row_r >> 4, row_s16 = row_s >> 4, b16 = B_BYTES >> 4, bst16 = B_STAGE >> 4;
        const uint64_t bres0 = umma_desc_sw128(sB0), bD0h = bres0;
        const bool fixed_ring = !(a.dbg & 32) && ((a.R == 3 && a.S == 3 && KPS >= 2 && KPS <= 4) ||
                                                  (a.R == 5 && a.S == 5 && KPS == 4) ||
                                                  (a.R == 1 && a.S == 1 && KPS == 1) ||
                                                  (a.R * a.S == 7 && (a.R == 1 || a.S == 1) && KPS == 4) ||
                                                  (a.R * a.S == 3 && (a.R == 1 || a.S == 1) && KPS == 3));
        const bool hk2 = a.hk == 2;  // (plan_conv_tc: hk > 1 only for fixed-loop shapes, hk <= 2)
        const bool fixed_rs = !(a.dbg & 32) && ((a.R == 3 && a.S == 3) || (a.R == 1 && a.S == 1) ||
                                                (a.R == 2 && a.S == 1) || (a.R == 4 && a.S == 1) ||
                                                (a.R == 5 && a.S == 5));
        for (int tile = cta; tile < tiles; tile += ncta, ++tcount) {
          mbar_wait(tempty0 + 8 * acc, tph ^ 1u);
          tc_fence_after();
          const uint32_t d = tmem + acc * (uint32_t)(a.hk * a.n_tile) + (uint32_t)(j * n_sub);
          uint32_t accum = 0;
          // vgrid: the tile's window starts v0 mod Wh pixels into the box
          uint32_t xoff = 0;
          int split_, tmn_;
          split_of(a, tile, tiles_mn, split_, tmn_);
          if (a.vgrid) {
            const int m0 = (tmn_ / a.tiles_n) * 128;
            xoff = (uint32_t)(m0 - (m0 / a.vgrid) * a.vgrid) * 128u;
          }
          // the tile's channel chunks [c_lo, c_hi) (a K split of whole chunks;
          // kpsplit = R * S * c_chunks without split-K)
          const int c_lo = split_ * a.kpsplit / RS, c_hi = min(nchunks, c_lo + a.kpsplit / RS);
          for (int cc = c_lo; cc < c_hi; ++cc) {
            mbar_wait(afull0 + 8 * ab, aph);
            tc_fence_after();
            if (bres && lane == 0 && j == 0) TRACE2(1, tcount);
            const uint64_t a0 = umma_desc_sw128(sA0 + ab * H_BYTES + xoff);
            const int kv = min(4, (C - cc * 64 + 15) >> 4);
            if (bres && fixed_rs) {
              // resident weights, common kernel shapes: the chunk's taps fully
              // unrolled with compile-time window offsets, issued by the
              // elected lane alone (halo_taps_bres_lane)
              const uint64_t bc = bres0 + (uint64_t)(cc * RS) * b16;
              const uint32_t dsx = (uint32_t)a.n_tile;
              // (3x3 with 2 or 4 K=16 slices, 1x1 with any: the lane-issued
              // instantiations; other shapes / slice counts the predicated loop)
              const bool lane_ok = (a.R == 3 && S_ == 3 && (kv == 2 || kv == 4)) || (a.R == 1 && S_ == 1);
              bool done = false;
              if (lane_ok) {
                if (on) {
                  if (a.R == 3) {
                    if (hk2) halo_taps_bres_lane_kv<3, 3, 2, 2>(kv, d, a0, bc, idesc, row_r16, row_s16, b16, accum, dsx);
                    else halo_taps_bres_lane_kv<3, 3, 1, 2>(kv, d, a0, bc, idesc, row_r16, row_s16, b16, accum, dsx);
                  } else {
                    if (hk2) halo_taps_bres_lane_kv<1, 1, 2, 1>(kv, d, a0, bc, idesc, row_r16, row_s16, b16, accum, dsx);
                    else halo_taps_bres_lane_kv<1, 1, 1, 1>(kv, d, a0, bc, idesc, row_r16, row_s16, b16, accum, dsx);
                  }
                }
                __syncwarp();
                done = true;
              }
              if (done) {
              } else if (a.R == 3 && S_ == 3) {
                if (hk2) halo_taps_bres<3, 3, 2>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
                else halo_taps_bres<3, 3, 1>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
              }
              else if (a.R == 1 && S_ == 1) {
                if (hk2) halo_taps_bres<1, 1, 2>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
                else halo_taps_bres<1, 1, 1>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
              }
              else if (a.R == 2 && S_ == 1) {
                if (hk2) halo_taps_bres<2, 1, 2>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
                else halo_taps_bres<2, 1, 1>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
              }
              else if (a.R == 4 && S_ == 1) {
                if (hk2) halo_taps_bres<4, 1, 2>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
                else halo_taps_bres<4, 1, 1>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
              }
              else if (a.R == 5 && S_ == 5) {
                if (hk2) halo_taps_bres<5, 5, 2>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
                else halo_taps_bres<5, 5, 1>(d, a0, bc, idesc, kv, on, row_r16, row_s16, b16, accum, dsx);
              }
              else __trap();  // unreachable: fixed_rs lists exactly these shapes
              accum = 1;
              mma_commit_on(aempty0 + 8 * ab, on);
              if (++ab == (uint32_t)abufs) { ab = 0; aph ^= 1u; }
              continue;
            }
            if (!bres && fixed_ring) {
              // B ring, common shapes: the chunk's taps unrolled with
              // compile-time window offsets; stage waits / releases at
              // compile-time tap boundaries (kps taps per stage)
              // (dispatch on R, S and kps together: each template's stage
              // boundaries must match the producer's)
              const uint32_t dsr = (uint32_t)a.n_tile;
              if (a.R == 3 && S_ == 3 && kps == 3) {
                if (hk2) halo_taps_ring<3, 3, 3, 2>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
                else halo_taps_ring<3, 3, 3, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              }
              else if (a.R == 3 && S_ == 3 && kps == 2) {
                if (hk2) halo_taps_ring<3, 3, 2, 2>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
                else halo_taps_ring<3, 3, 2, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              }
              else if (a.R == 3 && S_ == 3 && kps == 4) {
                if (hk2) halo_taps_ring<3, 3, 4, 2>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
                else halo_taps_ring<3, 3, 4, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              }
              else if (a.R == 5 && S_ == 5 && kps == 4) {
                if (hk2) halo_taps_ring<5, 5, 4, 2>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
                else halo_taps_ring<5, 5, 4, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              }
              else if (a.R == 1 && S_ == 7 && kps == 4) halo_taps_ring<1, 7, 4, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              else if (a.R == 7 && S_ == 1 && kps == 4) {
                if (hk2) halo_taps_ring<7, 1, 4, 2>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
                else halo_taps_ring<7, 1, 4, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              }
              else if (a.R == 1 && S_ == 3 && kps == 3) halo_taps_ring<1, 3, 3, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              else if (a.R == 3 && S_ == 1 && kps == 3) {
                if (hk2) halo_taps_ring<3, 1, 3, 2>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
                else halo_taps_ring<3, 1, 3, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              }
              else if (a.R == 1 && S_ == 1 && kps == 1) {
                if (hk2) halo_taps_ring<1, 1, 1, 2>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
                else halo_taps_ring<1, 1, 1, 1>(d, a0, bD0h, bst16, b16, idesc, kv, on, row_r16, row_s16, accum, st, ph, ST_, full0, empty0, dsr);
              }
              else __trap();  // unreachable: fixed_ring lists exactly these shapes
              accum = 1;
              mma_commit_on(aempty0 + 8 * ab, on);
              if (++ab == (uint32_t)abufs) { ab = 0; aph ^= 1u; }
              continue;
            }
            if (a.hk != 1) __trap();  // plan_conv_tc: row groups only for the unrolled shapes
            uint64_t aoff_r = 0, aoff = 0;
            int s_ = 0;
            for (int t = 0; t < RS;) {
              const int nk = min(kps, RS - t);
              uint64_t b0;
              if (!bres) {
                mbar_wait(full0 + 8 * st, ph);
                tc_fence_after();
                b0 = bD0h + (uint64_t)st * bst16;
              } else {
                b0 = bres0 + (uint64_t)(cc * RS + t) * b16;
              }
              for (int jj = 0; jj < nk; ++jj) {
                const uint64_t ad = a0 + aoff, bd = b0 + (uint64_t)jj * b16;
                mma_bf16_on(d, ad, bd, idesc, accum, on);
                if (kv > 1) mma_bf16_on(d, ad + 2, bd + 2, idesc, 1u, on);
                if (kv > 2) mma_bf16_on(d, ad + 4, bd + 4, idesc, 1u, on);
                if (kv > 3) mma_bf16_on(d, ad + 6, bd + 6, idesc, 1u, on);
                accum = 1;
                if (++s_ == S_) { s_ = 0; aoff_r += row_r16; aoff = aoff_r; } else { aoff += row_s16; }
              }
              t += nk;
              if (!bres) {
                mma_commit_on(empty0 + 8 * st, on);
                if (++st == ST_) { st = 0; ph ^= 1u; }
              }
            }
            mma_commit_on(aempty0 + 8 * ab, on);
            if (++ab == (uint32_t)abufs) { ab = 0; aph ^= 1u; }
          }
          if (bres && lane == 0 && j == 0) TRACE2(2, tcount);
          mma_commit_on(tfull0 + 8 * acc, on);
          __syncwarp();
          if (lane == 0 && tcount == 0 && j == 0) TRACE(4);
          if (a.nacc == 2) acc ^= 1u;
          if (acc == 0) tph ^= 1u;
        }
      } else {
        // tap mode, lean issue loop: a stage carries up to kps K-steps (may
        // cross a 64-channel chunk); descriptors are stage bases + strides
        // (the whole loop on the elected lane: waits, MMAs, commits -- the
        // descriptors stay in uniform registers, see halo_taps_bres_lane)
        const int C = a.C, kps = KPS;
        const uint32_t on = 1u;
        const uint32_t ST_ = (uint32_t)ST;
        const uint64_t aD0 = umma_desc_sw128(sA0), bD0 = umma_desc_sw128(sB0);
        const uint64_t ast16 = A_STAGE >> 4, bst16 = B_STAGE >> 4, a16 = A_BYTES >> 4, b16 = B_BYTES >> 4;
        if (elect_one())
        for (int tile = cta; tile < tiles; tile += ncta, ++tcount) {
          mbar_wait(tempty0 + 8 * acc, tph ^ 1u);
          tc_fence_after();
          const uint32_t d = tmem + acc * (uint32_t)a.n_tile + (uint32_t)(j * n_sub);
          uint32_t accum = 0;
          int split, tmn_;
          split_of(a, tile, tiles_mn, split, tmn_);
          const int k_lo = split * a.kpsplit, k_hi = min(a.c_chunks * RS, k_lo + a.kpsplit);
          int cc = k_lo / RS, rs = k_lo - (k_lo / RS) * RS;
          int kv = min(4, (C - cc * 64 + 15) >> 4);
          const int ktot = k_hi - k_lo;
          for (int k = 0; k < ktot;) {
            const int nk = min(kps, ktot - k);
            mbar_wait(full0 + 8 * st, ph);
            tc_fence_after();
            if (lane == 0 && k == 0 && j == 0 && tcount == 0) TRACE(3);
            if (lane == 0 && j == 0) TRACE2(1, k);
            const uint64_t a0 = aD0 + st * ast16, b0 = bD0 + st * bst16;
            for (int jj = 0; jj < nk; ++jj) {
              const uint64_t ad = a0 + (uint64_t)jj * a16, bd = b0 + (uint64_t)jj * b16;
              // 4 x K=16 inside the 128-byte swizzle row; K=16 slices past
              // the last real input channel are all zero and skipped
              mma_bf16_on(d, ad, bd, idesc, accum, on);
              if (kv > 1) mma_bf16_on(d, ad + 2, bd + 2, idesc, 1u, on);
              if (kv > 2) mma_bf16_on(d, ad + 4, bd + 4, idesc, 1u, on);
              if (kv > 3) mma_bf16_on(d, ad + 6, bd + 6, idesc, 1u, on);
              accum = 1;
              if (++rs == RS) { rs = 0; ++cc; kv = min(4, (C - cc * 64 + 15) >> 4); }
            }
            k += nk;
            mma_commit_on(empty0 + 8 * st, on);
            if (++st == ST_) { st = 0; ph ^= 1u; }
          }
          mma_commit_on(tfull0 + 8 * acc, on);
          if (tcount == 0 && j == 0) TRACE(4);
          if (a.nacc == 2) acc ^= 1u;
          if (acc == 0) tph ^= 1u;
        }
        __syncwarp();
      }
    }
    __syncwarp();
  } else {
    // -------------------------------------------------------- epilogue
    // TMEM -> registers -> folded BN + ReLU -> bf16 -> smem staging tile;
    // the accumulator is released to the MMA warps as soon as it is read,
    // then the tile leaves smem in coalesced 16-byte row segments (to the
    // local destination and, fused, to the peer GPU's replica).
    const int ew = warp - kEpiWarp0;
    const int lw = warp & 3;  // TMEM lane quarter this warp may access
    const int m = lw * 32 + lane;
    const int et = threadIdx.x - 32 * kEpiWarp0;  // 0..127
    uint32_t tcount = 0, acc = 0, tph = 0;
    if (a.sres) {
      // all K channels' BN shift once per CTA (rounded up to the N tile;
      // channels past K read the last one and are clipped at the store)
      const int kr = a.tiles_n * a.n_tile;
      for (int jj = et; jj < kr; jj += 128) {
        const int nj = min(jj, a.K - 1);
        asm volatile("st.shared.f32 [%0], %1;" ::"r"(smem_u32(s_shift + jj)), "f"(__ldg(a.shift + nj)) : "memory");
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
    }
    for (int tile = cta; tile < tiles; tile += ncta, ++tcount) {
      int split, tmn;
      split_of(a, tile, tiles_mn, split, tmn);
      const int m_blk = tmn / a.tiles_n, n_blk = tmn - m_blk * a.tiles_n;
      const int tp = m_blk / a.tiles_q, tq = m_blk - tp * a.tiles_q;
      const int p0 = tp * a.th, q0 = tq * a.tw, n0 = n_blk * a.n_tile;
      const int n_valid = min(a.n_tile, a.K - n0);
      // staging tile of this tile (two alternate when out_bufs == 2, so the
      // bulk stores of tile i drain while tile i+1 is staged)
      const uint32_t ob = a.out_bufs == 2 ? (tcount & 1u) : 0u;
      const uint32_t sOut_t = smem_u32(sOut) + ob * 128u * PITCH;
      TRACE4(0);
      if (a.sres && (a.tma_out || a.epi == 2)) {
        // scale/shift resident; each warp stages and ships only its own 32
        // rows, so it only waits for its own earlier stores out of this buffer
        // (direct-store mode: no staging at all)
        if (a.tma_out) {
          if (lane == 0) {
            if (a.out_bufs == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
            else bulk_wait_read0();
          }
          __syncwarp();
        }
      } else {
        // previous tile fully copied out of sOut / s_shift (all 128 threads;
        // TMA-store mode: the bulk stores have finished reading sOut)
        if (a.tma_out && lane == 0) bulk_wait_read0();
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (!a.sres) {
          for (int jj = et; jj < a.n_tile; jj += 128) {
            const int nj = min(n0 + jj, a.K - 1);
            asm volatile("st.shared.f32 [%0], %1;" ::"r"(smem_u32(s_shift + jj)), "f"(__ldg(a.shift + nj)) : "memory");
          }
          asm volatile("bar.sync 1, 128;" ::: "memory");
        }
      }
      TRACE4(1);
      mbar_wait(tfull0 + 8 * acc, tph);
      __syncwarp();
      tc_fence_after();
      TRACE4(2);
      TRACE5(0, tcount);
      if (tcount == 0 && warp == kEpiWarp0 && lane == 0) TRACE(5);
      const uint32_t tbase = tmem + ((uint32_t)(lw * 32) << 16) + acc * (uint32_t)(a.hk * a.n_tile);
      if (a.dbg & 16) {  // timing experiment: accumulator released unread
        tc_fence_before();
        mbar_arrive(tempty0 + 8 * acc);
        TRACE5(1, tcount);
        if (a.nacc == 2) acc ^= 1u;
        if (acc == 0) tph ^= 1u;
        continue;
      }
      if (a.epi == 2) {
        // direct stores: each thread owns one output pixel (its TMEM lane)
        // and writes its n_valid channels as 16-byte vectors straight from
        // registers -- no staging, no proxy fence, no bulk-group waits
        // (measured slower: warp-staged coalesced copy-out, Inception-1024
        // HIOS-LP 0.86 -> 1.00 ms)
        const float* shs = s_shift + (a.sres ? n0 : 0);
        for (int jr = 0; jr < a.hk; ++jr) {  // output row jr of the tile's row group
        const uint32_t tbj = tbase + (uint32_t)(jr * a.n_tile);
        int p, q;
        tile_pixel(a, m_blk, p0, q0, m, p, q);
        if (a.hk_px) q += jr * 128;  // pixel pairs (1x1): the second 128 pixels of the row segment
        else p += jr;                 // row groups: the next output row
        const bool valid = p < a.P && q < a.Q;
        const size_t pix = (size_t)p * a.Q + q;
        bf16* o1 = a.out + pix * a.ldo + n0;
        for (int col = 0; col < a.n_tile; col += 32) {
          const bool two = col + 16 < a.n_tile;  // warp-uniform
          uint32_t r0[16], r1[16];
          tmem_ld16_nw(tbj + (uint32_t)col, r0);
          if (two) tmem_ld16_nw(tbj + (uint32_t)col + 16u, r1);
          float sf[32];
#pragma unroll
          for (int q4 = 0; q4 < 8; ++q4) {
            const uint4 w = lds128(smem_u32(shs + col + 4 * q4));
            sf[4 * q4] = __uint_as_float(w.x); sf[4 * q4 + 1] = __uint_as_float(w.y);
            sf[4 * q4 + 2] = __uint_as_float(w.z); sf[4 * q4 + 3] = __uint_as_float(w.w);
          }
          if (jr == 0 && col < 64) TRACE4(3 + 2 * (col >> 5));
          tmem_wait_pin(r0);
          pin16(r1);
          if (jr == 0 && col < 64) TRACE4(4 + 2 * (col >> 5));
#pragma unroll
          for (int hlf = 0; hlf < 2; ++hlf) {
            const int c16 = col + 16 * hlf;
            if (hlf == 1 && !two) break;
            const uint32_t* r = hlf ? r1 : r0;
            uint32_t pk[8];
#pragma unroll
            for (int e = 0; e < 8; ++e)
              pk[e] = bias_relu_pack(r[2 * e], r[2 * e + 1], sf[16 * hlf + 2 * e], sf[16 * hlf + 2 * e + 1], a.relu);
            if (!valid) continue;
            if (a.st256 && c16 + 16 <= n_valid) {
              // 32-byte stores (one full sector per thread and instruction:
              // half the L1 store requests of 16-byte vectors)
              st_global_256(o1 + c16, pk);
              for (int d_ = 0; d_ < a.out2.n; ++d_) st_global_256(a.out2.p[d_] + pix * a.out2.ld[d_] + n0 + c16, pk);
              continue;
            }
#pragma unroll
            for (int v8 = 0; v8 < 2; ++v8) {
              const int c8 = c16 + 8 * v8;
              if (c8 + 8 <= n_valid) {
                const uint4 v = make_uint4(pk[4 * v8], pk[4 * v8 + 1], pk[4 * v8 + 2], pk[4 * v8 + 3]);
                *reinterpret_cast<uint4*>(o1 + c8) = v;
                for (int d_ = 0; d_ < a.out2.n; ++d_)
                  *reinterpret_cast<uint4*>(a.out2.p[d_] + pix * a.out2.ld[d_] + n0 + c8) = v;
              } else {
                for (int e = 0; e < 8 && c8 + e < n_valid; ++e) {
                  const uint16_t hv = (uint16_t)(pk[4 * v8 + (e >> 1)] >> (16 * (e & 1)));
                  reinterpret_cast<uint16_t*>(o1)[c8 + e] = hv;
                  for (int d_ = 0; d_ < a.out2.n; ++d_)
                    reinterpret_cast<uint16_t*>(a.out2.p[d_] + pix * a.out2.ld[d_] + n0)[c8 + e] = hv;
                }
              }
            }
          }
          if (jr == 0 && col < 64) TRACE4(7 + (col >> 5));
        }
        }  // jr
        TRACE4(9);
        tc_fence_before();
        mbar_arrive(tempty0 + 8 * acc);
        TRACE5(1, tcount);
        if (a.nacc == 2) acc ^= 1u;
        if (acc == 0) tph ^= 1u;
        continue;
      }
      const uint32_t srow = sOut_t + (uint32_t)m * PITCH;
      // TMA-store staging: slabs of out_sw channels, [128 rows][out_sw*2 B],
      // 16-byte chunks XOR-swizzled like the tensor map (bits 4.. ^= bits 7..)
      const uint32_t SWB = (uint32_t)a.out_sw * 2u, swm = SWB / 16u - 1u;
      const uint32_t sw_log = a.out_sw == 64 ? 6u : (a.out_sw == 32 ? 5u : 4u);
      // resident shifts are indexed by absolute channel (n0 + col)
      const uint32_t s_sh = smem_u32(s_shift) + (a.sres ? (uint32_t)n0 * 4u : 0u);
      // one 16-column group: folded BN + ReLU -> bf16 -> staging tile
      auto emit16 = [&](int col, const uint32_t (&r)[16], const float* sf) {
        uint32_t pk[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) pk[q] = bias_relu_pack(r[2 * q], r[2 * q + 1], sf[2 * q], sf[2 * q + 1], a.relu);
        if (a.tma_out) {
          const uint32_t slab = (uint32_t)col >> sw_log;
          const uint32_t cb = ((uint32_t)col - (slab << sw_log)) * 2u;  // byte in the slab row
          const uint32_t base = sOut_t + slab * 128u * SWB;
          const uint32_t o0 = (uint32_t)m * SWB + cb, o1 = o0 + 16u;
          sts128(base + (o0 ^ (((o0 >> 7) & swm) << 4)), pk[0], pk[1], pk[2], pk[3]);
          sts128(base + (o1 ^ (((o1 >> 7) & swm) << 4)), pk[4], pk[5], pk[6], pk[7]);
        } else {
          sts128(srow + col * 2, pk[0], pk[1], pk[2], pk[3]);
          sts128(srow + col * 2 + 16, pk[4], pk[5], pk[6], pk[7]);
        }
      };
      // 32 columns per round: two TMEM loads in flight, the BN parameters
      // (broadcast ld.shared.v4; a generic pointer would compile to slow
      // generic LD.E) fetched under their latency, one wait
      for (int col = 0; col < a.n_tile; col += 32) {
        const bool two = col + 16 < a.n_tile;  // warp-uniform
        uint32_t r0[16], r1[16];
        tmem_ld16_nw(tbase + (uint32_t)col, r0);
        if (two) tmem_ld16_nw(tbase + (uint32_t)col + 16u, r1);
        float sf[32];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const uint4 w = lds128(s_sh + (uint32_t)(col + 4 * q) * 4u);
          sf[4 * q] = __uint_as_float(w.x); sf[4 * q + 1] = __uint_as_float(w.y);
          sf[4 * q + 2] = __uint_as_float(w.z); sf[4 * q + 3] = __uint_as_float(w.w);
        }
        tmem_wait_pin(r0);
        pin16(r1);
        if (col < 16 * 6) TRACE4(3 + col / 32);
        emit16(col, r0, sf);
        if (two) emit16(col + 16, r1, sf + 16);
      }
      tc_fence_before();
      mbar_arrive(tempty0 + 8 * acc);  // TMEM accumulator free for the next tile
      if (tcount == 0 && warp == kEpiWarp0 && lane == 0) TRACE(6);
      if (a.nacc == 2) acc ^= 1u;
      if (acc == 0) tph ^= 1u;
      TRACE4(9);
      if (a.tma_out) {
        // each warp ships its own 32 rows as soon as they are staged (the
        // four warps' bulk-tensor stores issue in parallel; the tensor map
        // clips pixels beyond P x Q and channels beyond K)
        fence_proxy_async_smem();  // generic-proxy smem writes -> async proxy
        __syncwarp();
        TRACE4(10);
        if (lane == 0) {
          const int bw = a.tw < 32 ? a.tw : 32;
          const int mr = lw * 32, hh0 = mr / a.tw, ww0 = mr - hh0 * a.tw;
          (void)bw;
          const uint32_t nslab = (uint32_t)a.n_tile >> sw_log;
          for (uint32_t sl = 0; sl < nslab; ++sl) {
            const int c0 = n0 + (int)(sl << sw_log);
            if (c0 >= a.K) break;
            const uint32_t src = sOut_t + sl * 128u * SWB + (uint32_t)mr * SWB;
            tma_store_3d(pmo, src, c0, q0 + ww0, p0 + hh0);
            if (a.out2.n) tma_store_3d(pmo2, src, c0, q0 + ww0, p0 + hh0);
          }
          bulk_commit();
        }
        __syncwarp();
        TRACE4(12);
        TRACE5(1, tcount);
        if (tcount == 0 && et == 0) TRACE3(1);
        continue;
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
      TRACE4(11);
      if (tcount == 0 && et == 0) TRACE3(0);
      // coalesced copy-out: the 128 epilogue threads walk (row, 16-byte
      // chunk) pairs row-major, so consecutive lanes store consecutive 16 B of
      // one output pixel row (loads issued ahead of the dependent stores)
      const int row_bytes = n_valid * 2;
      const int chunks = row_bytes >> 4;
      const uint32_t sbase = sOut_t;
      const int total = 128 * chunks;
      for (int i0 = et; i0 < total; i0 += 128 * 4) {
        uint4 v[4];
        int rr[4], cc4[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int i = i0 + u * 128;
          rr[u] = i / chunks;
          cc4[u] = i - rr[u] * chunks;
          if (i < total) v[u] = lds128(sbase + (uint32_t)rr[u] * PITCH + (uint32_t)cc4[u] * 16u);
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int i = i0 + u * 128;
          if (i >= total) break;
          int p, q;
          tile_pixel(a, m_blk, p0, q0, rr[u], p, q);
          if (p >= a.P || q >= a.Q) continue;
          const size_t pix = (size_t)p * a.Q + q;
          *reinterpret_cast<uint4*>(a.out + pix * a.ldo + n0 + cc4[u] * 8) = v[u];
          for (int d_ = 0; d_ < a.out2.n; ++d_) *reinterpret_cast<uint4*>(a.out2.p[d_] + pix * a.out2.ld[d_] + n0 + cc4[u] * 8) = v[u];
        }
      }
      if (n_valid & 7) {  // channel tail (K % 8 != 0): element copies
        const int tail0 = chunks * 8, nt = n_valid - tail0;
        for (int i = et; i < 128 * nt; i += 128) {
          const int rr1 = i / nt, e = tail0 + (i - rr1 * nt);
          int p, q;
          tile_pixel(a, m_blk, p0, q0, rr1, p, q);
          if (p >= a.P || q >= a.Q) continue;
          const size_t pix = (size_t)p * a.Q + q;
          const uint16_t v = lds16(sbase + (uint32_t)rr1 * PITCH + (uint32_t)e * 2u);
          reinterpret_cast<uint16_t*>(a.out + pix * a.ldo + n0)[e] = v;
          for (int d_ = 0; d_ < a.out2.n; ++d_) reinterpret_cast<uint16_t*>(a.out2.p[d_] + pix * a.out2.ld[d_] + n0)[e] = v;
        }
      }
      if (tcount == 0 && et == 0) TRACE3(1);
    }
    if (a.tma_out && lane == 0) bulk_wait0();  // stores complete before the CTA retires
    tcount = 0;
    TRACE4(13);
    if (et == 0) TRACE3(2);
  }
  if (lane == 0 && warp < 8) TRACE3(3 + (warp >> 1));
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) TRACE(7);
  if (warp == kProducers) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(ncols));
  }
}

__global__ void __launch_bounds__(kThreads, 1)
    conv_tc_kernel(const __grid_constant__ CUtensorMap mx, const __grid_constant__ CUtensorMap mw,
                   const __grid_constant__ CUtensorMap mo, const __grid_constant__ CUtensorMap mo2,
                   const ConvTcArgs a) {
  conv_tc_body(&mx, &mw, &mo, &mo2, a, blockIdx.x, gridDim.x);
}

// A stage's convolutions in ONE launch (the stage's
// concurrent group as one kernel partitioning the SMs across its operators,
// P:84-86): CTAs [cta0[i], cta0[i+1]) run op i's persistent tile loop.  The
// partition is explicit (sized by each op's work, exec.cu plan_group), so no op
// of the stage can occupy SMs its peers need, and the stage costs one launch.
// Each op index is a compile-time constant in its own case, so the op's
// arguments stay constant-bank operands exactly as in conv_tc_kernel (measured:
// one runtime-indexed body made every conv ~24 % slower: Inception-1024
// sequential 0.96 -> 1.19 ms).
template <int I>
__device__ __forceinline__ void conv_tc_group_op(const ConvTcGroup& G) {
  conv_tc_body(&G.op[I].mx, &G.op[I].mw, &G.op[I].mo, &G.op[I].mo2, G.op[I].a, (int)blockIdx.x - G.cta0[I],
               G.cta0[I + 1] - G.cta0[I]);
}
__global__ void __launch_bounds__(kThreads, 1) conv_tc_group_kernel(const __grid_constant__ ConvTcGroup G) {
  int i = 0;
  while (i + 1 < G.n && (int)blockIdx.x >= G.cta0[i + 1]) ++i;
  static_assert(kMaxGroup == 6, "one case per group slot");
  switch (i) {
    case 0: conv_tc_group_op<0>(G); break;
    case 1: conv_tc_group_op<1>(G); break;
    case 2: conv_tc_group_op<2>(G); break;
    case 3: conv_tc_group_op<3>(G); break;
    case 4: conv_tc_group_op<4>(G); break;
    default: conv_tc_group_op<5>(G); break;
  }
}

size_t conv_tc_smem_bytes(const ConvTcArgs& a) {
  const size_t B = a.bres ? (size_t)a.n_tile * 128 * a.c_chunks * a.R * a.S : (size_t)a.n_tile * 128 * a.kps * a.stages;
  const size_t A = a.halo ? (size_t)a.a_bufs * halo_bytes_of(a.hrows, a.halo_w) : (size_t)a.stages * a.kps * 128 * 128;
  return 1024 + A + B + (size_t)a.out_bufs * 128 * (size_t)stage_pitch(a.n_tile) +
         (2 * a.stages + 2 * kMaxABufs + 6) * 8 +
         2 * kScaleRes * 4;
}

void launch_conv_tc_group(const ConvTcGroup& G, size_t smem, cudaStream_t st) {
  static bool attr_set[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && !attr_set[dev]) {
    cudaFuncSetAttribute(conv_tc_group_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr_set[dev] = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(G.cta0[G.n]);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, conv_tc_group_kernel, G);
}

void launch_conv_tc(const CUtensorMap& mx, const CUtensorMap& mw, const CUtensorMap& mo, const CUtensorMap& mo2,
                    const ConvTcArgs& a, int grid, size_t smem, cudaStream_t st) {
  static bool attr_set[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && !attr_set[dev]) {
    cudaFuncSetAttribute(conv_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr_set[dev] = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, conv_tc_kernel, mx, mw, mo, mo2, a);
}

}  // namespace hios

extern "C" int hios_debug_conv_trace_reset(void) {
  static unsigned long long zero[2048];
  return (int)cudaMemcpyToSymbol(hios::g_conv_trace, zero, sizeof(zero));
}

extern "C" int hios_debug_conv_trace4(unsigned long long* out) {
  return (int)cudaMemcpyFromSymbol(out, hios::g_conv_trace4, sizeof(unsigned long long) * 32 * 16);
}

extern "C" int hios_debug_conv_trace3(unsigned long long* out) {
  return (int)cudaMemcpyFromSymbol(out, hios::g_conv_trace3, sizeof(unsigned long long) * 32 * 8);
}

extern "C" int hios_debug_conv_trace5(unsigned long long* out) {
  return (int)cudaMemcpyFromSymbol(out, hios::g_conv_trace5, sizeof(unsigned long long) * 32 * 48);
}
extern "C" int hios_debug_conv_trace2(unsigned long long* out) {
  return (int)cudaMemcpyFromSymbol(out, hios::g_conv_trace2, sizeof(unsigned long long) * 32 * 48);
}

extern "C" int hios_debug_conv_trace(unsigned long long* out, int n) {
  return (int)cudaMemcpyFromSymbol(out, hios::g_conv_trace, sizeof(unsigned long long) * (n < 2048 ? n : 2048));
}

namespace hios {
// ------------------------------------------------------------ tensor maps
typedef CUresult (*PFN_encodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                     const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                     CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static PFN_encodeTiled get_encode() {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  return fn;
}

bool make_tmap_3d(CUtensorMap* m, const void* base, uint64_t d0, uint64_t d1, uint64_t d2, uint64_t stride1_bytes,
                  uint64_t stride2_bytes, uint32_t b0, uint32_t b1, uint32_t b2, uint32_t e1, uint32_t e2,
                  int swizzle_bytes) {
  PFN_encodeTiled enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[3] = {d0, d1, d2};
  cuuint64_t strides[2] = {stride1_bytes, stride2_bytes};
  cuuint32_t box[3] = {b0, b1, b2};
  cuuint32_t es[3] = {1, e1, e2};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE,
                   swizzle_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                   : swizzle_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                         : CU_TENSOR_MAP_SWIZZLE_32B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS && getenv("HIOS_TMAP_VERBOSE")) {
    fprintf(stderr, "hios: cuTensorMapEncodeTiled failed (%d): dims %llu %llu %llu box %u %u %u es %u %u\n", (int)r,
            (unsigned long long)d0, (unsigned long long)d1, (unsigned long long)d2, b0, b1, b2, e1, e2);
  }
  return r == CUDA_SUCCESS;
}

}  // namespace hios
