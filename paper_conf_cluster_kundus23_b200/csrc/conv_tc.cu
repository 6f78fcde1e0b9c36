// conv_tc.cu -- implicit-GEMM convolution on Blackwell 5th-gen tensor cores.
//
// One CTA = one 128-pixel x BLOCK_N output tile.  Warp roles (128 threads):
//   warp 0 lane 0  TMA producer: per K-step (r, s, 64-channel chunk) one 3-D
//                  box of the NHWC input at the (r,s)-shifted window with the
//                  conv stride as the TMA traversal stride (OOB -> zero, i.e.
//                  the conv padding) and one box of the [K][R*S][Cp] weights,
//                  both 128B-swizzled K-major, into a `stages`-deep ring
//   warp 1 lane 0  MMA issuer: 4 x tcgen05.mma.kind::f16 (M=128, N=BLOCK_N,
//                  K=16) per K-step into the TMEM accumulator; tcgen05.commit
//                  frees the smem slot
//   warp 2         TMEM allocator (BLOCK_N fp32 columns)
//   warps 0-3      epilogue: tcgen05.ld 32 lanes x 16 columns -> folded-BN
//                  scale/shift -> ReLU -> bf16 -> 16-byte stores into the
//                  destination (local buffer, concat slice, and optionally a
//                  peer GPU's replica: the transfer fused into the epilogue)
// SURVEY §8(a) a8; PAPER.md P:80 (conv operators of G).
#include <cstdio>

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
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "HIOS_WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra HIOS_WAIT_%=;\n"
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
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// UMMA shared-memory descriptor: K-major, 128B swizzle, 8-row atoms 1024 B apart.
__device__ __forceinline__ uint64_t umma_desc_sw128(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);  // start address  [0,14)
  d |= (uint64_t)1 << 16;                    // LBO (unused for swizzled K-major) [16,30)
  d |= (uint64_t)(1024 >> 4) << 32;          // SBO = 1024 B   [32,46)
  d |= (uint64_t)1 << 46;                    // descriptor version (sm_100)
  d |= (uint64_t)2 << 61;                    // SWIZZLE_128B
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
__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar)
               : "memory");
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

static __host__ __device__ inline uint32_t tmem_cols(int n) {
  uint32_t c = 32;
  while ((int)c < n) c <<= 1;
  return c;
}

__global__ void __launch_bounds__(128, 1)
    conv_tc_kernel(const __grid_constant__ CUtensorMap mx, const __grid_constant__ CUtensorMap mw,
                   const ConvTcArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int ST = a.stages;
  const uint32_t A_BYTES = 128 * 128;
  const uint32_t B_BYTES = (uint32_t)a.n_tile * 128;
  uint8_t* sA = smem;
  uint8_t* sB = smem + ST * A_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sB + ST * B_BYTES);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * ST + 1);
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + ST), accum = smem_u32(bars + 2 * ST);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int tp = blockIdx.x / a.tiles_q, tq = blockIdx.x % a.tiles_q;
  const int p0 = tp * a.th, q0 = tq * a.tw, n0 = blockIdx.y * a.n_tile;
  const uint32_t ncols = tmem_cols(a.n_tile);

  if (threadIdx.x == 0) {
    for (int i = 0; i < ST; ++i) {
      mbar_init(full0 + 8 * i, 1);
      mbar_init(empty0 + 8 * i, 1);
    }
    mbar_init(accum, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mx)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mw)) : "memory");
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(ncols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  const int KI = a.R * a.S * a.c_chunks;
  if (warp == 0 && lane == 0) {
    // ---------------- TMA producer
    for (int ki = 0; ki < KI; ++ki) {
      const int st = ki % ST;
      const uint32_t ph = (uint32_t)(ki / ST) & 1u;
      mbar_wait(empty0 + 8 * st, ph ^ 1u);
      mbar_expect_tx(full0 + 8 * st, A_BYTES + B_BYTES);
      const int rs = ki / a.c_chunks, cc = ki - rs * a.c_chunks;
      const int r = rs / a.S, s = rs - r * a.S;
      tma_load_3d(smem_u32(sA + st * A_BYTES), &mx, full0 + 8 * st, cc * 64, q0 * a.sw - a.pw + s * a.dw,
                  p0 * a.sh - a.ph + r * a.dh);
      tma_load_3d(smem_u32(sB + st * B_BYTES), &mw, full0 + 8 * st, cc * 64, rs, n0);
    }
  } else if (warp == 1 && lane == 0) {
    // ---------------- MMA issuer (single thread)
    const uint32_t idesc = (1u << 4)                             // D format f32
                           | (1u << 7)                           // A bf16
                           | (1u << 10)                          // B bf16
                           | ((uint32_t)(a.n_tile >> 3) << 17)   // N
                           | ((uint32_t)(128 >> 4) << 24);       // M = 128
    for (int ki = 0; ki < KI; ++ki) {
      const int st = ki % ST;
      const uint32_t ph = (uint32_t)(ki / ST) & 1u;
      mbar_wait(full0 + 8 * st, ph);
      tc_fence_after();
      const uint64_t ad = umma_desc_sw128(smem_u32(sA + st * A_BYTES));
      const uint64_t bd = umma_desc_sw128(smem_u32(sB + st * B_BYTES));
#pragma unroll
      for (int k = 0; k < 4; ++k)  // 4 x K=16 inside the 128-byte swizzle row
        mma_bf16(tmem, ad + 2 * k, bd + 2 * k, idesc, (ki | k) != 0);
      mma_commit(empty0 + 8 * st);
    }
    mma_commit(accum);
  }
  // ---------------- epilogue (all 4 warps; warp w owns TMEM lanes 32w..32w+31)
  mbar_wait(accum, 0);
  __syncwarp();
  tc_fence_after();
  const int m = warp * 32 + lane;
  const int hh = m / a.tw, ww = m - hh * a.tw;
  const int p = p0 + hh, q = q0 + ww;
  const bool valid = p < a.P && q < a.Q;
  const size_t pix = (size_t)p * a.Q + q;
  for (int col = 0; col < a.n_tile; col += 16) {
    uint32_t r[16];
    tmem_ld16(tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)col, r);
    const int n = n0 + col;
    if (!valid || n >= a.K) continue;
    float v[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      const int nj = min(n + j, a.K - 1);
      float y = __uint_as_float(r[j]) * __ldg(a.scale + nj) + __ldg(a.shift + nj);
      v[j] = a.relu ? fmaxf(y, 0.f) : y;
    }
    if (n + 16 <= a.K) {
      uint32_t pk[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        __nv_bfloat162 b2 = __floats2bfloat162_rn(v[2 * j], v[2 * j + 1]);
        pk[j] = *reinterpret_cast<uint32_t*>(&b2);
      }
      uint4* d = reinterpret_cast<uint4*>(a.out + pix * a.ldo + n);
      d[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      d[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
      if (a.out2) {
        uint4* d2 = reinterpret_cast<uint4*>(a.out2 + pix * a.ldo2 + n);
        d2[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
        d2[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
      }
    } else {
      for (int j = 0; j < 16 && n + j < a.K; ++j) {
        a.out[pix * a.ldo + n + j] = __float2bfloat16_rn(v[j]);
        if (a.out2) a.out2[pix * a.ldo2 + n + j] = __float2bfloat16_rn(v[j]);
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(ncols));
  }
}

size_t conv_tc_smem_bytes(int n_tile, int stages) {
  return 1024 + (size_t)stages * (128 * 128 + (size_t)n_tile * 128) + (2 * stages + 1) * 8 + 16;
}

void launch_conv_tc(const CUtensorMap& mx, const CUtensorMap& mw, const ConvTcArgs& a, int n_tiles_m,
                    int n_tiles_n, size_t smem, cudaStream_t st) {
  static bool attr_set[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && !attr_set[dev]) {
    cudaFuncSetAttribute(conv_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr_set[dev] = true;
  }
  conv_tc_kernel<<<dim3(n_tiles_m, n_tiles_n), 128, smem, st>>>(mx, mw, a);
}

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
                  uint64_t stride2_bytes, uint32_t b0, uint32_t b1, uint32_t b2, uint32_t e1, uint32_t e2) {
  PFN_encodeTiled enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[3] = {d0, d1, d2};
  cuuint64_t strides[2] = {stride1_bytes, stride2_bytes};
  cuuint32_t box[3] = {b0, b1, b2};
  cuuint32_t es[3] = {1, e1, e2};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    fprintf(stderr, "hios: cuTensorMapEncodeTiled failed (%d): dims %llu %llu %llu box %u %u %u es %u %u\n", (int)r,
            (unsigned long long)d0, (unsigned long long)d1, (unsigned long long)d2, b0, b1, b2, e1, e2);
    return false;
  }
  return true;
}

}  // namespace hios
