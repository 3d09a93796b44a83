// Persistent, warp-specialised tcgen05 GEMM for sm_100a:  y[M,N] = A[M,K] * W[N,K]^T (+bias) -> epilogue.
//
// S:§8(a) a1, a3, a8, a9, a11 (+a12 Euler in the epilogue) and the a0 conditioning / modulation
// GEMMs all run through this kernel.  Design (B200-native, not the paper's: the paper ships no
// kernels):
//   * one CTA per SM (persistent, static tile striding), 128 x BN output tiles, BK = 64;
//   * warp 0 = TMA producer (128B-swizzled K-major tiles, mbarrier complete_tx), warp 1 = single-
//     thread tcgen05.mma issuer (M=128, N=BN, K=16 per instruction), warp 2 = TMEM allocator,
//     warps 4-7 = epilogue (tcgen05.ld 32x32b -> registers -> fused epilogue -> global);
//   * two TMEM accumulators (2 x BN fp32 columns) so the epilogue of tile i overlaps the MMAs of
//     tile i+1;  4-8 smem stages depending on BN.
// Tile order walks M fastest so consecutive CTAs share the same weight tile (weights stream from
// HBM once per N-column while the activations stay L2-resident).
#include <cstdio>
#include <cudaTypedefs.h>

#include "kernels.h"
#include "ptx.cuh"

namespace tsv {

static constexpr int BM = 128;
static constexpr int BK = 64;
static constexpr int GEMM_THREADS = 256;

template <int BN>
struct GemmCfg {
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = (BN == 256) ? 4 : (BN == 128 ? 6 : 8);
  static constexpr int TMEM_COLS = 2 * BN;  // power of two >= 32
  static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/;
};

struct GemmArgs {
  int M, N, K;
  int num_m, num_n, num_tiles;
  GemmEpi epi;
};

template <int BN>
__device__ __forceinline__ void epilogue_chunk(const GemmArgs& a, int row, int n0, const uint32_t (&r)[32]) {
  const GemmEpi& e = a.epi;
  float v[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
  if (e.bias) {
    const uint4* bp = reinterpret_cast<const uint4*>(e.bias + n0);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint4 u = __ldg(bp + q);
      float2 f0 = unpack_bf16x2(u.x), f1 = unpack_bf16x2(u.y), f2 = unpack_bf16x2(u.z), f3 = unpack_bf16x2(u.w);
      v[q * 8 + 0] += f0.x; v[q * 8 + 1] += f0.y; v[q * 8 + 2] += f1.x; v[q * 8 + 3] += f1.y;
      v[q * 8 + 4] += f2.x; v[q * 8 + 5] += f2.y; v[q * 8 + 6] += f3.x; v[q * 8 + 7] += f3.y;
    }
  }
  if (row >= a.M) return;
  int mode = e.mode;
  bf16* ob = nullptr;
  if (mode == EPI_SPLIT_GELU) {
    if (n0 >= e.n_split) {
      mode = EPI_GELU_BF16;
      ob = reinterpret_cast<bf16*>(e.out1) + (long long)row * e.ld1 + (n0 - e.n_split);
    } else {
      mode = EPI_STORE_BF16;
      ob = reinterpret_cast<bf16*>(e.out0) + (long long)row * e.ld0 + n0;
    }
  } else if (mode <= EPI_SILU_BF16) {
    ob = reinterpret_cast<bf16*>(e.out0) + (long long)row * e.ld0 + n0;
  }
  if (mode <= EPI_SILU_BF16) {
    if (mode == EPI_GELU_BF16) {
#pragma unroll
      for (int i = 0; i < 32; ++i) v[i] = gelu_tanh(v[i]);
    } else if (mode == EPI_SILU_BF16) {
#pragma unroll
      for (int i = 0; i < 32; ++i) v[i] = silu(v[i]);
    }
    uint4* dst = reinterpret_cast<uint4*>(ob);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint4 u;
      u.x = pack_bf16x2(v[q * 8 + 0], v[q * 8 + 1]);
      u.y = pack_bf16x2(v[q * 8 + 2], v[q * 8 + 3]);
      u.z = pack_bf16x2(v[q * 8 + 4], v[q * 8 + 5]);
      u.w = pack_bf16x2(v[q * 8 + 6], v[q * 8 + 7]);
      dst[q] = u;
    }
    return;
  }
  float* of = reinterpret_cast<float*>(e.out0) + (long long)row * e.ld0 + n0;
  float4* d4 = reinterpret_cast<float4*>(of);
  if (mode == EPI_STORE_F32) {
#pragma unroll
    for (int q = 0; q < 8; ++q) d4[q] = make_float4(v[q * 4], v[q * 4 + 1], v[q * 4 + 2], v[q * 4 + 3]);
  } else if (mode == EPI_ACCUM_F32) {
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      float4 x = d4[q];
      d4[q] = make_float4(x.x + v[q * 4], x.y + v[q * 4 + 1], x.z + v[q * 4 + 2], x.w + v[q * 4 + 3]);
    }
  } else if (mode == EPI_RESID_GATE) {
    const float4* g4 = reinterpret_cast<const float4*>(e.gate + n0);
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      float4 x = d4[q];
      float4 g = __ldg(g4 + q);
      x.x += g.x * v[q * 4 + 0];
      x.y += g.y * v[q * 4 + 1];
      x.z += g.z * v[q * 4 + 2];
      x.w += g.w * v[q * 4 + 3];
      d4[q] = x;
    }
  } else if (mode == EPI_EULER) {
    const float dt = *e.scalar;
    if (e.out1) {
      float4* v4 = reinterpret_cast<float4*>(reinterpret_cast<float*>(e.out1) + (long long)row * e.ld1 + n0);
#pragma unroll
      for (int q = 0; q < 8; ++q) v4[q] = make_float4(v[q * 4], v[q * 4 + 1], v[q * 4 + 2], v[q * 4 + 3]);
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      float4 x = d4[q];
      x.x += dt * v[q * 4 + 0];
      x.y += dt * v[q * 4 + 1];
      x.z += dt * v[q * 4 + 2];
      x.w += dt * v[q * 4 + 3];
      d4[q] = x;
    }
  }
}

template <int BN>
__global__ void __launch_bounds__(GEMM_THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ GemmArgs args) {
  using C = GemmCfg<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
  uint64_t* full = bars;
  uint64_t* empty = bars + C::STAGES;
  uint64_t* tfull = bars + 2 * C::STAGES;
  uint64_t* tempty = bars + 2 * C::STAGES + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * C::STAGES + 4);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int num_k = args.K / BK;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&tfull[i], 1);
      mbar_init(&tempty[i], 128);
    }
    fence_mbar_init();
  }
  if (warp == 2) tmem_alloc<C::TMEM_COLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ---------------- TMA producer
      int stage = 0;
      uint32_t phase = 0;
      for (int t = blockIdx.x; t < args.num_tiles; t += gridDim.x) {
        const int m_blk = t % args.num_m, n_blk = t / args.num_m;
        for (int kb = 0; kb < num_k; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          mbar_arrive_expect_tx(&full[stage], C::STAGE_BYTES);
          tma_load_2d(&tmA, &full[stage], sA + stage * C::A_BYTES, kb * BK, m_blk * BM);
          tma_load_2d(&tmB, &full[stage], sB + stage * C::B_BYTES, kb * BK, n_blk * BN);
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ---------------- MMA issuer
      constexpr uint32_t idesc = make_idesc_bf16(BM, BN);
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int t = blockIdx.x; t < args.num_tiles; t += gridDim.x, ++it) {
        const int acc = it & 1;
        const uint32_t acc_phase = (it >> 1) & 1;
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = 0; kb < num_k; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t a_addr = smem_u32(sA + stage * C::A_BYTES);
          const uint32_t b_addr = smem_u32(sB + stage * C::B_BYTES);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            umma_bf16_ss(d_tmem, make_sw128_desc(a_addr + k * 32), make_sw128_desc(b_addr + k * 32), idesc,
                         (kb | k) != 0);
          }
          umma_commit(&empty[stage]);
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
        umma_commit(&tfull[acc]);
      }
    }
  } else if (warp >= 4) {
    // ---------------- epilogue: warp (4..7) owns TMEM lanes [32*(warp-4), +32)
    const int wq = warp - 4;
    int it = 0;
    for (int t = blockIdx.x; t < args.num_tiles; t += gridDim.x, ++it) {
      const int m_blk = t % args.num_m, n_blk = t / args.num_m;
      const int acc = it & 1;
      const uint32_t acc_phase = (it >> 1) & 1;
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int row = m_blk * BM + wq * 32 + lane;
      const uint32_t tbase = tmem_base + ((uint32_t)(wq * 32) << 16) + acc * BN;
#pragma unroll 1
      for (int c = 0; c < BN / 32; ++c) {
        uint32_t r[32];
        tmem_ld32(tbase + c * 32, r);
        tmem_ld_wait();
        epilogue_chunk<BN>(args, row, n_blk * BN + c * 32, r);
      }
      tc_fence_before();
      mbar_arrive(&tempty[acc]);
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc<C::TMEM_COLS>(tmem_base);
}

// ------------------------------------------------------------------ host side
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

static int make_tmap_2d(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer, uint64_t row_bytes,
                        uint32_t box_inner, uint32_t box_outer) {
  auto enc = get_encode();
  if (!enc) return -1;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {row_bytes};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? 0 : -2;
}

int gemm_plan(GemmPlan* p, const bf16* A, long long lda, const bf16* W, long long ldw, int M, int N, int K,
              const GemmEpi& epi, int num_sms, const char** err, int force_bn) {
  *err = nullptr;
  if (M <= 0 || N <= 0 || K <= 0) { *err = "gemm: empty shape"; return -1; }
  if (K % BK) { *err = "gemm: K must be a multiple of 64"; return -1; }
  if (N % 64) { *err = "gemm: N must be a multiple of 64"; return -1; }
  if ((lda * 2) % 16 || (ldw * 2) % 16) { *err = "gemm: row strides must be 16-byte multiples"; return -1; }
  if ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(W)) & 15) {
    *err = "gemm: operands must be 16-byte aligned"; return -1;
  }
  int bn = force_bn;
  if (!bn) {
    const int nm = (M + BM - 1) / BM;
    if (N % 256 == 0 && (long long)nm * (N / 256) >= num_sms * 3 / 4) bn = 256;
    else if (N % 128 == 0 && (long long)nm * (N / 128) >= num_sms * 3 / 4) bn = 128;
    else if (N % 256 == 0 && N >= 4096) bn = 256;
    else bn = (N % 128 == 0 && nm * (N / 128) >= num_sms / 2) ? 128 : 64;
  }
  if (N % bn) { *err = "gemm: N not a multiple of the tile width"; return -1; }
  p->M = M; p->N = N; p->K = K; p->BN = bn; p->epi = epi;
  if (make_tmap_2d(&p->tmA, A, K, M, lda * 2, BK, BM)) { *err = "gemm: cuTensorMapEncodeTiled(A) failed"; return -1; }
  if (make_tmap_2d(&p->tmB, W, K, N, ldw * 2, BK, bn)) { *err = "gemm: cuTensorMapEncodeTiled(W) failed"; return -1; }
  const int tiles = ((M + BM - 1) / BM) * (N / bn);
  p->grid = tiles < num_sms ? tiles : num_sms;
  return 0;
}

template <int BN>
static void launch_bn(const GemmPlan& p, cudaStream_t s) {
  using C = GemmCfg<BN>;
  static unsigned long long attr_done = 0;  // one bit per device
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(attr_done >> dev & 1ull)) {
    cudaFuncSetAttribute(gemm_tc_kernel<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM_BYTES);
    attr_done |= 1ull << dev;
  }
  GemmArgs a;
  a.M = p.M; a.N = p.N; a.K = p.K;
  a.num_m = (p.M + BM - 1) / BM;
  a.num_n = p.N / BN;
  a.num_tiles = a.num_m * a.num_n;
  a.epi = p.epi;
  gemm_tc_kernel<BN><<<p.grid, GEMM_THREADS, C::SMEM_BYTES, s>>>(p.tmA, p.tmB, a);
}

void gemm_launch(const GemmPlan& p, cudaStream_t s) {
  switch (p.BN) {
    case 256: launch_bn<256>(p, s); break;
    case 128: launch_bn<128>(p, s); break;
    default: launch_bn<64>(p, s); break;
  }
}

}  // namespace tsv
