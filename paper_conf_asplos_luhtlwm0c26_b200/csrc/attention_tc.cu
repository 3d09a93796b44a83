// Joint text+image attention on the 5th-gen tensor cores (S:§8(a) a6):
//   O = softmax(q k^T / sqrt(D)) v, non-causal, per head, fp32 online softmax, bf16 operands.
//
// One CTA = one (head, 128-query tile).  Warp roles:
//   warp 0      TMA producer: Q once, then K/V tiles of 128 keys into a 2-stage ring
//               (3-D tensor maps [rows][heads][D] -> one map serves every head and layout);
//   warp 1      single-thread tcgen05.mma issuer:  S_j = Q K_j^T into one of two TMEM S buffers
//               (issued one tile ahead), then O += P_j V_j (V consumed MN-major straight from the
//               TMA tile, no transpose);
//   warps 4-7   softmax: thread i owns query row i (TMEM lane i): tcgen05.ld of its 128 scores,
//               row max / exp2 / row sum in registers, P_j as bf16 into a 128B-swizzled K-major
//               smem tile (double-buffered), conditional O rescale (only when the running max grows
//               by more than 2^8, so P stays <= 256 and rescales are rare), final 1/l and store.
// TMEM: S0 | S1 | O  (128 + 128 + D fp32 columns).
#include <cfloat>
#include <cstdlib>
#include <cudaTypedefs.h>

#include "kernels.h"
#include "ptx.cuh"

namespace tsv {

namespace {

constexpr int AT_BM = 128;     // queries per CTA
constexpr int AT_BN = 128;     // keys per tile
constexpr int AT_THREADS = 256;
constexpr float RESCALE_THRESHOLD = 8.0f;  // log2 domain

template <int D>
struct AttnCfg {
  static constexpr int NSUB = D / 64;                  // 64-wide sub-tiles of the head dim
  static constexpr int Q_BYTES = AT_BM * D * 2;
  static constexpr int KV_TILE = AT_BN * D * 2;         // one K (or V) tile
  static constexpr int P_BYTES = AT_BM * AT_BN * 2;     // 2 sub-tiles of 64 keys
  static constexpr int OFF_Q = 0;
  static constexpr int OFF_K = OFF_Q + Q_BYTES;              // 2 stages
  static constexpr int OFF_V = OFF_K + 2 * KV_TILE;          // 2 stages
  static constexpr int OFF_P = OFF_V + 2 * KV_TILE;          // 2 buffers
  static constexpr int OFF_BAR = OFF_P + 2 * P_BYTES;
  static constexpr int SMEM = OFF_BAR + 256 + 1024;
  static constexpr int TMEM_COLS = 512;
  static constexpr int O_COL = 256;
};

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]),
      "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]),
      "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]),
      "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31]));
}
__device__ __forceinline__ float fast_exp2(float x) {  // MUFU.EX2; ex2(-inf) = +0
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// 2^x without the MUFU: x = n + f (n = round(x), |f| <= 1/2), 2^f by a cubic (Taylor of e^(f ln2),
// rel. error <= 7e-4 on |f| <= 1/2), 2^n added to the exponent field.  x is clamped at -126 so the
// exponent add cannot wrap (the true value is < 2^-126 there).  Finite x only.
__device__ __forceinline__ float poly_exp2(float x) {
  x = fmaxf(x, -126.0f);
  const float t = x + 12582912.0f;          // 1.5 * 2^23: round(x) lands in the low mantissa bits
  const float n = t - 12582912.0f;
  const float f = x - n;
  float p = fmaf(0.0555041086648216f, f, 0.2402265069591007f);
  p = fmaf(p, f, 0.6931471805599453f);
  p = fmaf(p, f, 1.0f);
  return __int_as_float(__float_as_int(p) + (__float_as_int(t) << 23));
}
// The same on a pair, with the sm_100 paired FP32 ops (FADD2 / FFMA2: two lanes per instruction).
__device__ __forceinline__ float2 poly_exp2_x2(float2 x) {
  x.x = fmaxf(x.x, -126.0f);
  x.y = fmaxf(x.y, -126.0f);
  const float2 magic = make_float2(12582912.0f, 12582912.0f);
  const float2 t = __fadd2_rn(x, magic);
  const float2 n = __fadd2_rn(t, make_float2(-12582912.0f, -12582912.0f));
  const float2 f = __ffma2_rn(n, make_float2(-1.0f, -1.0f), x);
  float2 p = __ffma2_rn(make_float2(0.0555041086648216f, 0.0555041086648216f), f,
                        make_float2(0.2402265069591007f, 0.2402265069591007f));
  p = __ffma2_rn(p, f, make_float2(0.6931471805599453f, 0.6931471805599453f));
  p = __ffma2_rn(p, f, make_float2(1.0f, 1.0f));
  return make_float2(__int_as_float(__float_as_int(p.x) + (__float_as_int(t.x) << 23)),
                     __int_as_float(__float_as_int(p.y) + (__float_as_int(t.y) << 23)));
}
__device__ __forceinline__ void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// MN-major, 128B-swizzled B operand (rows = K, 64 N-elements per 128-byte row):
// SBO = 1024 B between 8-row K atoms, LBO = byte distance between 64-wide N blocks.
__device__ __forceinline__ uint64_t make_sw128_mn_desc(uint32_t smem_addr, uint32_t lbo_bytes) {
  uint64_t lo = ((smem_addr & 0x3FFFFu) >> 4) | ((uint64_t)((lbo_bytes >> 4) & 0x3FFFu) << 16);
  uint64_t hi = (1024u >> 4) | (1u << 14) | (2u << 29);
  return lo | (hi << 32);
}

__host__ __device__ constexpr uint32_t make_idesc_bf16_bmn(int M, int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

}  // namespace

template <int D>
__global__ void __launch_bounds__(AT_THREADS, 1)
    attention_tc_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                        const __grid_constant__ CUtensorMap tmV, bf16* __restrict__ o, long long ldo, int L,
                        float scale_log2) {
  using C = AttnCfg<D>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + C::OFF_BAR);
  uint64_t* q_full = bars + 0;
  uint64_t* kv_full = bars + 1;    // [2]
  uint64_t* kv_empty = bars + 3;   // [2]
  uint64_t* s_full = bars + 5;     // [2]
  uint64_t* s_free = bars + 7;     // [2]
  uint64_t* p_full = bars + 9;     // [2]
  uint64_t* pv_done = bars + 11;   // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 14);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int head = blockIdx.y;
  const int q0 = blockIdx.x * AT_BM;
  const int n_tiles = (L + AT_BN - 1) / AT_BN;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmQ);
    tma_prefetch_desc(&tmK);
    tma_prefetch_desc(&tmV);
    mbar_init(q_full, 1);
    for (int i = 0; i < 2; ++i) {
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
      mbar_init(&s_full[i], 1);
      mbar_init(&s_free[i], 128);
      mbar_init(&p_full[i], 128);
      mbar_init(&pv_done[i], 1);
    }
    fence_mbar_init();
  }
  if (warp == 2) tmem_alloc<C::TMEM_COLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  grid_dep_wait();

  if (warp == 0) {
    if (lane == 0) {
      // ---------------------------------------------------------------- producer
      mbar_arrive_expect_tx(q_full, C::Q_BYTES);
      for (int s = 0; s < C::NSUB; ++s)
        tma_load_3d(&tmQ, q_full, sm + C::OFF_Q + s * (AT_BM * 128), s * 64, head, q0);
      for (int j = 0; j < n_tiles; ++j) {
        const int st = j & 1;
        if (j >= 2) mbar_wait(&kv_empty[st], ((j - 2) >> 1) & 1);
        mbar_arrive_expect_tx(&kv_full[st], 2 * C::KV_TILE);
        for (int s = 0; s < C::NSUB; ++s) {
          tma_load_3d(&tmK, &kv_full[st], sm + C::OFF_K + st * C::KV_TILE + s * (AT_BN * 128), s * 64, head,
                      j * AT_BN);
          tma_load_3d(&tmV, &kv_full[st], sm + C::OFF_V + st * C::KV_TILE + s * (AT_BN * 128), s * 64, head,
                      j * AT_BN);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ---------------------------------------------------------------- MMA issuer
      constexpr uint32_t idesc_s = make_idesc_bf16(AT_BM, AT_BN);
      constexpr uint32_t idesc_o = make_idesc_bf16_bmn(AT_BM, D);
      const uint32_t sQ = smem_u32(sm + C::OFF_Q);
      mbar_wait(q_full, 0);
      auto issue_s = [&](int j) {
        const int st = j & 1;
        mbar_wait(&kv_full[st], (j >> 1) & 1);
        if (j >= 2) mbar_wait(&s_free[st], ((j - 2) >> 1) & 1);
        tc_fence_after();
        const uint32_t sK = smem_u32(sm + C::OFF_K + st * C::KV_TILE);
#pragma unroll
        for (int kk = 0; kk < D / 16; ++kk) {
          const uint32_t off = (kk >> 2) * (AT_BM * 128) + (kk & 3) * 32;
          const uint32_t offk = (kk >> 2) * (AT_BN * 128) + (kk & 3) * 32;
          umma_bf16_ss(tmem + st * 128, make_sw128_desc(sQ + off), make_sw128_desc(sK + offk), idesc_s, kk > 0);
        }
        umma_commit(&s_full[st]);
      };
      issue_s(0);
      for (int j = 0; j < n_tiles; ++j) {
        if (j + 1 < n_tiles) issue_s(j + 1);
        const int st = j & 1;
        mbar_wait(&p_full[st], (j >> 1) & 1);
        tc_fence_after();
        const uint32_t sP = smem_u32(sm + C::OFF_P + st * C::P_BYTES);
        const uint32_t sV = smem_u32(sm + C::OFF_V + st * C::KV_TILE);
#pragma unroll
        for (int kk = 0; kk < AT_BN / 16; ++kk) {
          const uint32_t offp = (kk >> 2) * (AT_BM * 128) + (kk & 3) * 32;
          umma_bf16_ss(tmem + C::O_COL, make_sw128_desc(sP + offp),
                       make_sw128_mn_desc(sV + kk * 2048, AT_BN * 128), idesc_o, (j | kk) != 0);
        }
        umma_commit(&pv_done[st]);
        umma_commit(&kv_empty[st]);
      }
    }
  } else if (warp >= 4) {
    // ---------------------------------------------------------------- softmax (thread = query row)
    const int wq = warp - 4;
    const int row = wq * 32 + lane;
    const uint32_t lane_base = (uint32_t)(wq * 32) << 16;
    float m_ref = -FLT_MAX, l_sum = 0.f;
    for (int j = 0; j < n_tiles; ++j) {
      const int st = j & 1;
      mbar_wait(&s_full[st], (j >> 1) & 1);
      tc_fence_after();
      uint32_t sr[4][32];
#pragma unroll
      for (int c = 0; c < 4; ++c) tmem_ld32(tmem + lane_base + st * 128 + c * 32, sr[c]);
      tmem_ld_wait();
      tc_fence_before();
      mbar_arrive(&s_free[st]);
      const int kbase = j * AT_BN;
      // row max on the raw scores (scale > 0); keys >= L only exist in the last tile
      // row max with 8 independent accumulators (a single chain would be 128 dependent FMNMX)
      float mx[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) mx[q] = -FLT_MAX;
      if (kbase + AT_BN > L) {
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (kbase + c * 32 + i >= L) sr[c][i] = __float_as_uint(-INFINITY);
      }
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int i = 0; i < 32; ++i) mx[i & 7] = fmaxf(mx[i & 7], __uint_as_float(sr[c][i]));
      const float mt = fmaxf(fmaxf(fmaxf(mx[0], mx[1]), fmaxf(mx[2], mx[3])),
                             fmaxf(fmaxf(mx[4], mx[5]), fmaxf(mx[6], mx[7]))) * scale_log2;
      bool rescale = false;
      float alpha = 1.f;
      if (j == 0) {
        m_ref = mt;
      } else if (mt > m_ref + RESCALE_THRESHOLD) {
        rescale = true;
        alpha = exp2f(m_ref - mt);
        m_ref = mt;
      }
      l_sum *= alpha;
      // P = exp2(x - m_ref) -> bf16, packed in pairs
      // P = 2^(s * scale_log2 - m_ref): one FFMA + one MUFU.EX2 per score
      uint32_t pk[64];
      float ls0 = 0.f, ls1 = 0.f;
      const float neg_m = -m_ref;
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int i = 0; i < 32; i += 2) {
          const float p0 = fast_exp2(fmaf(__uint_as_float(sr[c][i]), scale_log2, neg_m));
          const float p1 = fast_exp2(fmaf(__uint_as_float(sr[c][i + 1]), scale_log2, neg_m));
          ls0 += p0;
          ls1 += p1;
          pk[c * 16 + i / 2] = pack_bf16x2(p0, p1);
        }
      l_sum += ls0 + ls1;
      if (j >= 2) mbar_wait(&pv_done[st], ((j - 2) >> 1) & 1);  // P buffer st free
      // tcgen05.ld/st are warp-collective (.sync.aligned): rescale the whole warp's rows together
      // (alpha = 1 for rows that did not need it).
      if (__any_sync(0xffffffffu, rescale)) {
        mbar_wait(&pv_done[st ^ 1], ((j - 1) >> 1) & 1);         // O holds tiles < j
        tc_fence_after();
#pragma unroll
        for (int c = 0; c < D / 32; ++c) {
          uint32_t ov[32];
          tmem_ld32(tmem + lane_base + C::O_COL + c * 32, ov);
          tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 32; ++i) ov[i] = __float_as_uint(__uint_as_float(ov[i]) * alpha);
          tmem_st32(tmem + lane_base + C::O_COL + c * 32, ov);
        }
        tmem_st_wait();
      }
      // write P row into the K-major SW128 tile: sub-tile t (keys 64t..), atom row/8, chunk ^ (row & 7)
      uint8_t* pbase = sm + C::OFF_P + st * C::P_BYTES + (row >> 3) * 1024 + (row & 7) * 128;
#pragma unroll
      for (int t = 0; t < 2; ++t)
#pragma unroll
        for (int ch = 0; ch < 8; ++ch) {
          const int q = t * 32 + ch * 4;  // index into pk (pairs)
          uint4 v = make_uint4(pk[q], pk[q + 1], pk[q + 2], pk[q + 3]);
          *reinterpret_cast<uint4*>(pbase + t * (AT_BM * 128) + ((ch ^ (row & 7)) << 4)) = v;
        }
      fence_proxy_async();
      tc_fence_before();
      mbar_arrive(&p_full[st]);
    }
    // epilogue: O / l -> bf16
    const int jl = n_tiles - 1;
    mbar_wait(&pv_done[jl & 1], (jl >> 1) & 1);
    tc_fence_after();
    const float inv = 1.f / l_sum;
    const int grow = q0 + row;
#pragma unroll
    for (int c = 0; c < D / 32; ++c) {
      uint32_t ov[32];
      tmem_ld32(tmem + lane_base + C::O_COL + c * 32, ov);
      tmem_ld_wait();
      if (grow < L) {
        uint4* dst = reinterpret_cast<uint4*>(o + (long long)grow * ldo + head * D + c * 32);
#pragma unroll
        for (int qd = 0; qd < 4; ++qd) {
          uint4 v;
          v.x = pack_bf16x2(__uint_as_float(ov[qd * 8 + 0]) * inv, __uint_as_float(ov[qd * 8 + 1]) * inv);
          v.y = pack_bf16x2(__uint_as_float(ov[qd * 8 + 2]) * inv, __uint_as_float(ov[qd * 8 + 3]) * inv);
          v.z = pack_bf16x2(__uint_as_float(ov[qd * 8 + 4]) * inv, __uint_as_float(ov[qd * 8 + 5]) * inv);
          v.w = pack_bf16x2(__uint_as_float(ov[qd * 8 + 6]) * inv, __uint_as_float(ov[qd * 8 + 7]) * inv);
          dst[qd] = v;
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc<C::TMEM_COLS>(tmem);
}

// ------------------------------------------------------------------ v3: two query tiles per CTA
// One CTA = one head x 256 queries as two 128-query tiles t = 0, 1 that share every K/V tile
// (half the K/V traffic per query).  Two softmax warpgroups (warps 4-7: tile 0, 8-11: tile 1)
// ping-pong with the tensor core: while WG0 turns S0_j into P0_j, the single MMA thread runs
// PV1_{j-1} and S1_j, and vice versa.  P_j is written back into the S_t TMEM columns as bf16
// (tcgen05.st) and consumed from TMEM by the PV MMA (A operand in TMEM), so no shared-memory P.
// Because S_t{j+1} overwrites P_t{j} in TMEM, the MMA thread issues PV_t{j} before S_t{j+1}; the
// in-order tcgen05 pipe makes "S_t{j} complete" imply "O_t holds tiles < j", so a rare rescale
// of O (running max grew by > 2^8) needs no extra wait.
// TMEM: S0 | S1 | O0 | O1 (128 + 128 + D + D fp32 columns).  Smem: Q0, Q1, 2 K/V stages.
#ifndef TSV_FA_NST64
#define TSV_FA_NST64 4
#endif
template <int D>
struct FaCfg {
  static constexpr int NSUB = D / 64;
  static constexpr int Q_TILE = AT_BM * D * 2;
  static constexpr int KV_TILE = AT_BN * D * 2;
  // K/V ring depth: D = 128 fills shared memory with 2 stages; D = 64 has room for 4
  static constexpr int NST = TSV_FA_NST64 > 0 && D == 64 ? TSV_FA_NST64 : 2;
  static constexpr int OFF_Q = 0;                        // 2 tiles
  static constexpr int OFF_K = OFF_Q + 2 * Q_TILE;       // NST stages
  static constexpr int OFF_V = OFF_K + NST * KV_TILE;    // NST stages
  static constexpr int OFF_BAR = OFF_V + NST * KV_TILE;
  static constexpr int SMEM = OFF_BAR + 256 + 1024;
  static constexpr int O_COL = 256;
};
constexpr int FA_THREADS = 384;

// NPOLY of every 8 exp2 pairs are evaluated on the FMA/ALU pipes (poly_exp2_x2), the rest on MUFU.
// SPLIT: P_t{j} is handed to the MMA thread in two halves (keys 0-63, then 64-127), each with its
// own barrier, so PV over the first 64 keys runs on the tensor core while the softmax warps still
// evaluate the second half's exponentials.
// LAZY: the row max is not recomputed per tile.  P = 2^(s*scale - m_ref) is evaluated with the
// running reference directly; the tile's row sum bounds every p in it (p <= sum), so a row whose
// sum stays <= 2^LAZY_LOG2 has no p > 2^LAZY_LOG2 and needs no rescale (m_ref is only a
// stabiliser: softmax is exact for any reference that keeps p finite).  Otherwise (the max grew
// a lot: early tiles) the warp reloads S from TMEM and takes the exact path (row max, rescale).
// Saves the 128 FMNMX per row per tile and the max-before-exp dependency on the softmax chain.
constexpr float LAZY_LIMIT = 65536.0f;   // 2^16
// KV split (blockIdx.z = split): see AttnSplitWs.  nsplit = 1: the whole key range, no workspace.
struct AttnSplitArgs {
  int nsplit = 1, tps = 0;   // splits, key tiles per split
  int* cnt = nullptr;
  float* ws = nullptr;
};

template <int D, int NPOLY, bool SPLIT, bool LAZY = false>
__global__ void __launch_bounds__(FA_THREADS, 1)
    attention_fa_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                        const __grid_constant__ CUtensorMap tmV, bf16* __restrict__ o, long long ldo, int L,
                        float scale_log2, const __grid_constant__ AttnScatter sc,
                        const __grid_constant__ AttnSplitArgs sa) {
  using C = FaCfg<D>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + C::OFF_BAR);
  constexpr int NST = C::NST;
  uint64_t* q_full = bars + 0;
  uint64_t* kv_full = bars + 1;              // [NST stages]
  uint64_t* kv_empty = bars + 1 + NST;       // [NST stages]
  uint64_t* s_full = bars + 1 + 2 * NST;     // [2 q-tiles]
  uint64_t* p_full = bars + 3 + 2 * NST;     // [2 q-tiles]  (SPLIT: first half of P)
  uint64_t* o_done = bars + 5 + 2 * NST;     // [2 q-tiles]
  uint64_t* p_full2 = bars + 7 + 2 * NST;    // [2 q-tiles]  SPLIT: second half of P
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 10 + 2 * NST);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int head = blockIdx.y;
  const int q0 = blockIdx.x * 2 * AT_BM;
  // this CTA's key tiles: [j0, j0 + n_tiles) (all of them unless the launch splits the keys)
  const int n_all = (L + AT_BN - 1) / AT_BN;
  const int j0 = sa.nsplit > 1 ? (int)blockIdx.z * sa.tps : 0;
  const int n_tiles = sa.nsplit > 1 ? min(n_all - j0, sa.tps) : n_all;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmQ);
    tma_prefetch_desc(&tmK);
    tma_prefetch_desc(&tmV);
    mbar_init(q_full, 1);
    for (int i = 0; i < NST; ++i) {
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&s_full[i], 1);
      mbar_init(&p_full[i], 128);
      mbar_init(&p_full2[i], 128);
      mbar_init(&o_done[i], 1);
    }
    fence_mbar_init();
  }
  if (warp == 2) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  // registers: the producer / MMA warpgroup needs few, the softmax warpgroups hold a 128-score row
  // each (80 * 128 + 208 * 256 <= 168 * 384, the launch allocation: inc blocks until the pool has them)
  grid_dep_wait();
  if (warp < 4) {
   regs_dec<80>();
   if (warp == 0) {
    if (lane == 0) {
      // ---------------------------------------------------------------- producer
      mbar_arrive_expect_tx(q_full, 2 * C::Q_TILE);
      for (int t = 0; t < 2; ++t)
        for (int s = 0; s < C::NSUB; ++s)
          tma_load_3d(&tmQ, q_full, sm + C::OFF_Q + t * C::Q_TILE + s * (AT_BM * 128), s * 64, head,
                      q0 + t * AT_BM);
      for (int j = 0; j < n_tiles; ++j) {
        const int st = j % NST;
        if (j >= NST) mbar_wait(&kv_empty[st], ((j / NST) - 1) & 1);
        mbar_arrive_expect_tx(&kv_full[st], 2 * C::KV_TILE);
        for (int s = 0; s < C::NSUB; ++s) {
          tma_load_3d(&tmK, &kv_full[st], sm + C::OFF_K + st * C::KV_TILE + s * (AT_BN * 128), s * 64, head,
                      (j0 + j) * AT_BN);
          tma_load_3d(&tmV, &kv_full[st], sm + C::OFF_V + st * C::KV_TILE + s * (AT_BN * 128), s * 64, head,
                      (j0 + j) * AT_BN);
        }
      }
    }
   } else if (warp == 1) {
    // ---------------------------------------------------------------- MMA issuer
    // The whole warp runs the loop (warp-uniform control flow keeps descriptors in uniform
    // registers); one elected lane issues each batch of MMAs back to back.  Descriptors are bases +
    // compile-time offsets (the 14-bit address field cannot carry: smem < 256 KB).
    constexpr uint32_t idesc_s = make_idesc_bf16(AT_BM, AT_BN);
    constexpr uint32_t idesc_o = make_idesc_bf16_bmn(AT_BM, D);
    const uint64_t dq0 = make_sw128_desc(smem_u32(sm + C::OFF_Q));
    const uint64_t dk0 = make_sw128_desc(smem_u32(sm + C::OFF_K));
    const uint64_t dv0 = make_sw128_mn_desc(smem_u32(sm + C::OFF_V), AT_BN * 128);
    mbar_wait(q_full, 0);
    auto issue_s = [&](int t, int j) {
      const uint64_t dq = dq0 + (uint64_t)((t * C::Q_TILE) >> 4);
      const uint64_t dk = dk0 + (uint64_t)(((j % NST) * C::KV_TILE) >> 4);
      if (elect_one()) {
#pragma unroll
        for (int kk = 0; kk < D / 16; ++kk) {
          const uint32_t off = ((kk >> 2) * (AT_BM * 128) + (kk & 3) * 32) >> 4;
          umma_bf16_ss(tmem + t * 128, dq + off, dk + off, idesc_s, kk > 0);
        }
        umma_commit(&s_full[t]);
      }
      __syncwarp();
    };
    auto issue_pv = [&](int t, int j, bool release) {
      const uint64_t dv = dv0 + (uint64_t)(((j % NST) * C::KV_TILE) >> 4);
      mbar_wait(&p_full[t], j & 1);
      tc_fence_after();
      if (elect_one()) {
#pragma unroll
        for (int kk = 0; kk < AT_BN / 16; ++kk) {
          if (SPLIT && kk == AT_BN / 32) {
            mbar_wait(&p_full2[t], j & 1);
            tc_fence_after();
          }
          umma_bf16_ts(tmem + C::O_COL + t * D, tmem + t * 128 + kk * 8, dv + (uint64_t)(kk * (2048 >> 4)), idesc_o,
                       (j | kk) != 0);
        }
        if (release) umma_commit(&kv_empty[j % NST]);
      }
      __syncwarp();
    };
    for (int j = 0; j < n_tiles; ++j) {
      mbar_wait(&kv_full[j % NST], (j / NST) & 1);
      tc_fence_after();
      for (int t = 0; t < 2; ++t) {
        if (j > 0) issue_pv(t, j - 1, t == 1);
        issue_s(t, j);
      }
    }
    for (int t = 0; t < 2; ++t) {
      issue_pv(t, n_tiles - 1, false);
      if (elect_one()) umma_commit(&o_done[t]);
      __syncwarp();
    }
   }
  } else {
    regs_inc<208>();
    // ---------------------------------------------------------------- softmax WG t (thread = query row)
    const int t = (warp - 4) >> 2;
    const int wq = (warp - 4) & 3;
    const int row = wq * 32 + lane;
    const uint32_t lane_base = (uint32_t)(wq * 32) << 16;
    const uint32_t s_col = tmem + lane_base + t * 128;
    const uint32_t o_col = tmem + lane_base + C::O_COL + t * D;
    float m_ref = -FLT_MAX, l_sum = 0.f;
    for (int j = 0; j < n_tiles; ++j) {
      mbar_wait(&s_full[t], j & 1);
      tc_fence_after();
      uint32_t sr[4][32];
      const int kbase = (j0 + j) * AT_BN;
      const bool full = kbase + AT_BN <= L;
      const bool lazy = LAZY && !SPLIT && j > 0 && full;
      if (!lazy) {
#pragma unroll
        for (int c = 0; c < 4; ++c) tmem_ld32(s_col + c * 32, sr[c]);
        tmem_ld_wait();
      }
      if (lazy) {
        const float2 sc2 = make_float2(scale_log2, scale_log2), nm2 = make_float2(-m_ref, -m_ref);
        float2 lz[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
        // no max before the exponentials: the TMEM loads are pipelined with the arithmetic (chunk
        // c + 1 is in flight while chunk c is exponentiated)
        tmem_ld32(s_col, sr[0]);
        tmem_ld_wait_dep(sr[0]);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          if (c < 3) tmem_ld32(s_col + (c + 1) * 32, sr[c + 1]);
#pragma unroll
          for (int i = 0; i < 32; i += 2) {
            float2 x = __ffma2_rn(make_float2(__uint_as_float(sr[c][i]), __uint_as_float(sr[c][i + 1])), sc2, nm2);
            float2 p;
            if (((i >> 1) & 7) >= 8 - NPOLY) {
              // the polynomial path wraps the exponent field outside [-126, 127]: clamp both sides
              // (a clamped x > 64 still makes the sum exceed the limit)
              x.x = fminf(x.x, 64.f);
              x.y = fminf(x.y, 64.f);
              p = poly_exp2_x2(x);
            } else {
              p = make_float2(fast_exp2(x.x), fast_exp2(x.y));
            }
            lz[(i >> 1) & 3] = __fadd2_rn(lz[(i >> 1) & 3], p);
            sr[c >> 1][(c & 1) * 16 + i / 2] = pack_bf16x2(p.x, p.y);
          }
          if (c < 3) tmem_ld_wait_dep(sr[c + 1]);
        }
        const float2 l01 = __fadd2_rn(lz[0], lz[1]), l23 = __fadd2_rn(lz[2], lz[3]);
        const float2 l4 = __fadd2_rn(l01, l23);
        const float ts = l4.x + l4.y;
        if (!__any_sync(0xffffffffu, !(ts <= LAZY_LIMIT))) {   // also catches inf / NaN
          l_sum += ts;
          tmem_st32(s_col, sr[0]);
          tmem_st32(s_col + 32, sr[1]);
          tmem_st_wait();
          tc_fence_before();
          mbar_arrive(&p_full[t]);
          continue;
        }
        // rare: reload the untouched S columns and take the exact path below
#pragma unroll
        for (int c = 0; c < 4; ++c) tmem_ld32(s_col + c * 32, sr[c]);
        tmem_ld_wait();
      }
      // row max with 8 independent accumulators (a single chain would be 128 dependent FMNMX)
      float mx[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) mx[q] = -FLT_MAX;
      if (!full) {
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (kbase + c * 32 + i >= L) sr[c][i] = __float_as_uint(-INFINITY);
      }
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int i = 0; i < 32; ++i) mx[i & 7] = fmaxf(mx[i & 7], __uint_as_float(sr[c][i]));
      const float mt = fmaxf(fmaxf(fmaxf(mx[0], mx[1]), fmaxf(mx[2], mx[3])),
                             fmaxf(fmaxf(mx[4], mx[5]), fmaxf(mx[6], mx[7]))) * scale_log2;
      bool rescale = false;
      float alpha = 1.f;
      if (j == 0) {
        m_ref = mt;
      } else if (mt > m_ref + RESCALE_THRESHOLD) {
        rescale = true;
        alpha = exp2f(m_ref - mt);
        m_ref = mt;
      }
      l_sum *= alpha;
      // P = 2^(s * scale_log2 - m_ref) as packed bf16 pairs, in place of S (columns 0..63 of S_t):
      // keys [64h, 64h + 64) land in sr[h] and TMEM columns [32h, 32h + 32)
      const float neg_m = -m_ref;
      float2 lsum[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        if (full) {
          // Per tile each softmax warpgroup must finish inside the ~1024-cycle window in which the
          // tensor core works on the other query tile.  MUFU.EX2 alone needs 1024 cycles per tile
          // (16/clk/SM), so NPOLY pairs in 8 are evaluated on the FMA/ALU pipes (Cody-Waite split +
          // cubic, rel. error < 1e-3 << bf16 ulp of P), and the arithmetic uses paired FP32 ops.
          const float2 sc2 = make_float2(scale_log2, scale_log2), nm2 = make_float2(neg_m, neg_m);
#pragma unroll
          for (int c = 2 * h; c < 2 * h + 2; ++c)
#pragma unroll
            for (int i = 0; i < 32; i += 2) {
              const float2 x = __ffma2_rn(make_float2(__uint_as_float(sr[c][i]), __uint_as_float(sr[c][i + 1])),
                                          sc2, nm2);
              float2 p;
              if (((i >> 1) & 7) >= 8 - NPOLY) p = poly_exp2_x2(x);
              else p = make_float2(fast_exp2(x.x), fast_exp2(x.y));
              lsum[(i >> 1) & 3] = __fadd2_rn(lsum[(i >> 1) & 3], p);     // 8 independent partial sums
              sr[h][(c & 1) * 16 + i / 2] = pack_bf16x2(p.x, p.y);        // packed P overwrites consumed S
            }
        } else {
#pragma unroll
          for (int c = 2 * h; c < 2 * h + 2; ++c)
#pragma unroll
            for (int i = 0; i < 32; i += 2) {
              const float p0 = fast_exp2(fmaf(__uint_as_float(sr[c][i]), scale_log2, neg_m));
              const float p1 = fast_exp2(fmaf(__uint_as_float(sr[c][i + 1]), scale_log2, neg_m));
              lsum[(i >> 1) & 3] = __fadd2_rn(lsum[(i >> 1) & 3], make_float2(p0, p1));
              sr[h][(c & 1) * 16 + i / 2] = pack_bf16x2(p0, p1);
            }
        }
        if (h == 0 && __any_sync(0xffffffffu, rescale)) {
          // S_t{j} complete => PV_t{j-1} complete (in-order pipe): O_t can be rescaled now, before any
          // part of P_t{j} is handed over (here S columns 64-127 are consumed: registers are free)
#pragma unroll
          for (int c = 0; c < D / 32; ++c) {
            uint32_t ov[32];
            tmem_ld32(o_col + c * 32, ov);
            tmem_ld_wait();
#pragma unroll
            for (int i = 0; i < 32; ++i) ov[i] = __float_as_uint(__uint_as_float(ov[i]) * alpha);
            tmem_st32(o_col + c * 32, ov);
          }
        }
        if (SPLIT || h == 1) {
          if (SPLIT) {
            tmem_st32(s_col + 32 * h, sr[h]);
          } else {
            tmem_st32(s_col, sr[0]);
            tmem_st32(s_col + 32, sr[1]);
          }
          tmem_st_wait();
          tc_fence_before();
          mbar_arrive(h == 0 ? &p_full[t] : (SPLIT ? &p_full2[t] : &p_full[t]));
        }
      }
      const float2 l01 = __fadd2_rn(lsum[0], lsum[1]), l23 = __fadd2_rn(lsum[2], lsum[3]);
      const float2 l4 = __fadd2_rn(l01, l23);
      l_sum += l4.x + l4.y;
    }
    // epilogue: O_t / l -> bf16
    mbar_wait(&o_done[t], 0);
    tc_fence_after();
    float inv = 1.f / l_sum;
    const int grow = q0 + t * AT_BM + row;
    // output row: local (plain) or, fused a7, the owning rank's row of its stream-concatenated input
    bf16* orow = o + (long long)grow * ldo + head * D;
    if (sc.k > 0 && grow < L) {
      int p = 0, lr;
      if (grow < sc.Lt) {
        while (p + 1 < sc.k && grow >= sc.t_off[p + 1]) ++p;
        lr = grow - sc.t_off[p];
      } else {
        const int gi = grow - sc.Lt;
        while (p + 1 < sc.k && gi >= sc.i_off[p + 1]) ++p;
        lr = sc.nt[p] + gi - sc.i_off[p];
      }
      orow = sc.dst[p] + (long long)lr * sc.ld + sc.col0 + head * D;
    }
    if (sa.nsplit > 1) {
      // KV split: unnormalised O_t (layout [D][128]: coalesced across the warp's rows), reference m
      // and sum l of this split -> ws; the last split of these 32 rows merges in split order:
      // O = sum_s 2^(m_s - M) O_s / sum_s 2^(m_s - M) l_s, M = max_s m_s
      const size_t slab = (size_t)AT_BM * (D + 2);
      const int nqb = gridDim.x;
      const size_t qt = ((size_t)head * nqb + blockIdx.x) * 2 + t;   // query tile
      auto ws_at = [&](int s2) { return sa.ws + (qt * sa.nsplit + s2) * slab; };
      float* mine = ws_at(blockIdx.z);
#pragma unroll
      for (int c = 0; c < D / 32; ++c) {
        uint32_t ov[32];
        tmem_ld32(o_col + c * 32, ov);
        tmem_ld_wait();
#pragma unroll
        for (int i = 0; i < 32; ++i) __stcg(mine + (size_t)(c * 32 + i) * AT_BM + row, __uint_as_float(ov[i]));
      }
      __stcg(mine + (size_t)D * AT_BM + row, m_ref);
      __stcg(mine + (size_t)(D + 1) * AT_BM + row, l_sum);
      __threadfence();
      __syncwarp();
      int* cnt = sa.cnt + qt * 4 + wq;
      int done = 0;
      if (lane == 0) done = atomicAdd(cnt, 1);
      done = __shfl_sync(0xffffffffu, done, 0);
      if (done == sa.nsplit - 1) {
        __threadfence();
        float mmax = -FLT_MAX;
        float ms[8], wsum = 0.f;
#pragma unroll
        for (int s2 = 0; s2 < 8; ++s2)
          if (s2 < sa.nsplit) {
            ms[s2] = __ldcg(ws_at(s2) + (size_t)D * AT_BM + row);
            mmax = fmaxf(mmax, ms[s2]);
          }
#pragma unroll
        for (int s2 = 0; s2 < 8; ++s2)
          if (s2 < sa.nsplit) {
            ms[s2] = exp2f(ms[s2] - mmax);   // now the merge weight of split s2
            wsum += ms[s2] * __ldcg(ws_at(s2) + (size_t)(D + 1) * AT_BM + row);
          }
        inv = 1.f / wsum;
        // the whole row (D values) accumulates in registers, one split at a time: each split's D
        // loads are independent, so the merge costs nsplit L2 round trips (not nsplit x D/32)
        float acc[D];
#pragma unroll
        for (int i = 0; i < D; ++i) acc[i] = 0.f;
#pragma unroll
        for (int s2 = 0; s2 < 8; ++s2)
          if (s2 < sa.nsplit) {
            const float* src = ws_at(s2) + row;
            const float w = ms[s2];
#pragma unroll
            for (int i = 0; i < D; ++i) acc[i] = fmaf(w, __ldcg(src + (size_t)i * AT_BM), acc[i]);
          }
        if (grow < L) {
#pragma unroll
          for (int c = 0; c < D / 32; ++c) {
            uint4* dst = reinterpret_cast<uint4*>(orow + c * 32);
#pragma unroll
            for (int qd = 0; qd < 4; ++qd) {
              const float* a8 = acc + c * 32 + qd * 8;
              uint4 v;
              v.x = pack_bf16x2(a8[0] * inv, a8[1] * inv);
              v.y = pack_bf16x2(a8[2] * inv, a8[3] * inv);
              v.z = pack_bf16x2(a8[4] * inv, a8[5] * inv);
              v.w = pack_bf16x2(a8[6] * inv, a8[7] * inv);
              dst[qd] = v;
            }
          }
        }
        if (lane == 0) *cnt = 0;   // re-armed for the next launch
      }
    } else
#pragma unroll
    for (int c = 0; c < D / 32; ++c) {
      uint32_t ov[32];
      tmem_ld32(o_col + c * 32, ov);
      tmem_ld_wait();
      if (grow < L) {
        uint4* dst = reinterpret_cast<uint4*>(orow + c * 32);
#pragma unroll
        for (int qd = 0; qd < 4; ++qd) {
          uint4 v;
          v.x = pack_bf16x2(__uint_as_float(ov[qd * 8 + 0]) * inv, __uint_as_float(ov[qd * 8 + 1]) * inv);
          v.y = pack_bf16x2(__uint_as_float(ov[qd * 8 + 2]) * inv, __uint_as_float(ov[qd * 8 + 3]) * inv);
          v.z = pack_bf16x2(__uint_as_float(ov[qd * 8 + 4]) * inv, __uint_as_float(ov[qd * 8 + 5]) * inv);
          v.w = pack_bf16x2(__uint_as_float(ov[qd * 8 + 6]) * inv, __uint_as_float(ov[qd * 8 + 7]) * inv);
          dst[qd] = v;
        }
      }
    }
  }
  grid_dep_launch();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc<512>(tmem);
}

// ------------------------------------------------------------------ v5: 64-key tiles, S double-buffered
// v3's chain S_t(j) -> softmax -> PV_t(j) -> S_t(j+1) serialises the softmax with the tensor core
// (P_t(j) aliases the only S_t buffer).  v5 uses 64-key K/V tiles so that each query tile owns two
// 64-column S buffers (TMEM: S_t,b at 128 t + 64 b, O_t at 256 + D t; 512 columns for D = 128):
// the MMA thread issues S_t(j+1) into the other buffer BEFORE PV_t(j), so the tensor core computes
// the next scores while the softmax warps exponentiate the current ones.  Per iteration the MMA
// thread issues PV_0(j), S_0(j+2), PV_1(j), S_1(j+2): S_t(j+2) reuses buffer j & 1 right behind
// PV_t(j) in the same in-order tcgen05 pipe, so each softmax warpgroup has two tiles of look-ahead.  Because S_t(j) no longer implies "PV_t(j-1) complete", a rare
// O rescale first waits on pv_done[t] (committed after every PV_t).
template <int D>
struct Fa5Cfg {
  static constexpr int BN = 64;                          // keys per K/V tile
  static constexpr int NSUB = D / 64;
  static constexpr int Q_TILE = AT_BM * D * 2;
  static constexpr int KV_TILE = BN * D * 2;             // one K (or V) tile
  static constexpr int NST = D == 128 ? 4 : 6;           // K/V stages
  static constexpr int OFF_Q = 0;                        // 2 tiles
  static constexpr int OFF_K = OFF_Q + 2 * Q_TILE;
  static constexpr int OFF_V = OFF_K + NST * KV_TILE;
  static constexpr int OFF_BAR = OFF_V + NST * KV_TILE;
  static constexpr int SMEM = OFF_BAR + 256 + 1024;
  static constexpr int O_COL = 256;
};

template <int D, int NPOLY>
__global__ void __launch_bounds__(FA_THREADS, 1)
    attention_fa5_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                         const __grid_constant__ CUtensorMap tmV, bf16* __restrict__ o, long long ldo, int L,
                         float scale_log2, const __grid_constant__ AttnScatter sc) {
  using C = Fa5Cfg<D>;
  constexpr int BN = C::BN, NST = C::NST;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + C::OFF_BAR);
  uint64_t* q_full = bars + 0;
  uint64_t* kv_full = bars + 1;            // [NST]
  uint64_t* kv_empty = bars + 1 + NST;     // [NST]
  uint64_t* s_full = bars + 1 + 2 * NST;   // [2 t][2 buffers]
  uint64_t* p_full = bars + 5 + 2 * NST;   // [2 t][2 buffers]
  uint64_t* pv_done = bars + 9 + 2 * NST;  // [2 t], every PV_t
  uint64_t* o_done = bars + 11 + 2 * NST;  // [2 t], the last PV_t
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 14 + 2 * NST);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int head = blockIdx.y;
  const int q0 = blockIdx.x * 2 * AT_BM;
  const int n_tiles = (L + BN - 1) / BN;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmQ);
    tma_prefetch_desc(&tmK);
    tma_prefetch_desc(&tmV);
    mbar_init(q_full, 1);
    for (int i = 0; i < NST; ++i) {
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
    }
    for (int i = 0; i < 4; ++i) {
      mbar_init(&s_full[i], 1);
      mbar_init(&p_full[i], 128);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&pv_done[i], 1);
      mbar_init(&o_done[i], 1);
    }
    fence_mbar_init();
  }
  if (warp == 2) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  grid_dep_wait();
  if (warp < 4) {
    regs_dec<80>();
    if (warp == 0) {
      if (lane == 0) {
        // -------------------------------------------------------------- producer
        mbar_arrive_expect_tx(q_full, 2 * C::Q_TILE);
        for (int t = 0; t < 2; ++t)
          for (int s = 0; s < C::NSUB; ++s)
            tma_load_3d(&tmQ, q_full, sm + C::OFF_Q + t * C::Q_TILE + s * (AT_BM * 128), s * 64, head,
                        q0 + t * AT_BM);
        for (int j = 0; j < n_tiles; ++j) {
          const int st = j % NST;
          if (j >= NST) mbar_wait(&kv_empty[st], ((j / NST) - 1) & 1);
          mbar_arrive_expect_tx(&kv_full[st], 2 * C::KV_TILE);
          for (int s = 0; s < C::NSUB; ++s) {
            tma_load_3d(&tmK, &kv_full[st], sm + C::OFF_K + st * C::KV_TILE + s * (BN * 128), s * 64, head, j * BN);
            tma_load_3d(&tmV, &kv_full[st], sm + C::OFF_V + st * C::KV_TILE + s * (BN * 128), s * 64, head, j * BN);
          }
        }
      }
    } else if (warp == 1) {
      // -------------------------------------------------------------- MMA issuer (whole warp,
      // one elected lane per MMA batch; descriptors = bases + compile-time offsets, see v3)
      constexpr uint32_t idesc_s = make_idesc_bf16(AT_BM, BN);
      constexpr uint32_t idesc_o = make_idesc_bf16_bmn(AT_BM, D);
      const uint64_t dq0 = make_sw128_desc(smem_u32(sm + C::OFF_Q));
      const uint64_t dk0 = make_sw128_desc(smem_u32(sm + C::OFF_K));
      const uint64_t dv0 = make_sw128_mn_desc(smem_u32(sm + C::OFF_V), BN * 128);
      mbar_wait(q_full, 0);
      auto issue_s = [&](int t, int j) {   // S_t(j) into buffer j & 1 (K tile already resident)
        const uint64_t dq = dq0 + (uint64_t)((t * C::Q_TILE) >> 4);
        const uint64_t dk = dk0 + (uint64_t)(((j % NST) * C::KV_TILE) >> 4);
        if (elect_one()) {
#pragma unroll
          for (int kk = 0; kk < D / 16; ++kk) {
            const uint32_t offq = ((kk >> 2) * (AT_BM * 128) + (kk & 3) * 32) >> 4;
            const uint32_t offk = ((kk >> 2) * (BN * 128) + (kk & 3) * 32) >> 4;
            umma_bf16_ss(tmem + t * 128 + (j & 1) * 64, dq + offq, dk + offk, idesc_s, kk > 0);
          }
          umma_commit(&s_full[t * 2 + (j & 1)]);
        }
        __syncwarp();
      };
      auto issue_pv = [&](int t, int j) {  // O_t += P_t(j) V(j); P_t(j) in TMEM buffer j & 1
        const uint64_t dv = dv0 + (uint64_t)(((j % NST) * C::KV_TILE) >> 4);
        mbar_wait(&p_full[t * 2 + (j & 1)], (j >> 1) & 1);
        tc_fence_after();
        if (elect_one()) {
#pragma unroll
          for (int kk = 0; kk < BN / 16; ++kk)
            umma_bf16_ts(tmem + C::O_COL + t * D, tmem + t * 128 + (j & 1) * 64 + kk * 8,
                         dv + (uint64_t)(kk * (2048 >> 4)), idesc_o, (j | kk) != 0);
          umma_commit(&pv_done[t]);
          if (j == n_tiles - 1) umma_commit(&o_done[t]);
        }
        __syncwarp();
      };
      // two tiles of look-ahead per query tile: S_t(j+2) (into buffer j & 1) right behind PV_t(j)
      for (int j = 0; j < 2 && j < n_tiles; ++j) {
        mbar_wait(&kv_full[j], 0);
        tc_fence_after();
        issue_s(0, j);
        issue_s(1, j);
      }
      for (int j = 0; j < n_tiles; ++j) {
        const bool ahead = j + 2 < n_tiles;
        for (int t = 0; t < 2; ++t) {
          issue_pv(t, j);
          if (ahead) {
            if (t == 0) {
              mbar_wait(&kv_full[(j + 2) % NST], ((j + 2) / NST) & 1);
              tc_fence_after();
            }
            issue_s(t, j + 2);
          }
        }
        if (elect_one()) umma_commit(&kv_empty[j % NST]);
        __syncwarp();
      }
    }
  } else {
    regs_inc<208>();
    // ---------------------------------------------------------------- softmax WG t (thread = query row)
    const int t = (warp - 4) >> 2;
    const int wq = (warp - 4) & 3;
    const int row = wq * 32 + lane;
    const uint32_t lane_base = (uint32_t)(wq * 32) << 16;
    const uint32_t o_col = tmem + lane_base + C::O_COL + t * D;
    float m_ref = -FLT_MAX, l_sum = 0.f;
    for (int j = 0; j < n_tiles; ++j) {
      const uint32_t s_col = tmem + lane_base + t * 128 + (j & 1) * 64;
      mbar_wait(&s_full[t * 2 + (j & 1)], (j >> 1) & 1);
      tc_fence_after();
      uint32_t sr[2][32];
      tmem_ld32(s_col, sr[0]);
      tmem_ld32(s_col + 32, sr[1]);
      tmem_ld_wait();
      const int kbase = j * BN;
      const bool full = kbase + BN <= L;
      if (!full) {
#pragma unroll
        for (int c = 0; c < 2; ++c)
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (kbase + c * 32 + i >= L) sr[c][i] = __float_as_uint(-INFINITY);
      }
      float mx[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) mx[q] = -FLT_MAX;
#pragma unroll
      for (int c = 0; c < 2; ++c)
#pragma unroll
        for (int i = 0; i < 32; ++i) mx[i & 7] = fmaxf(mx[i & 7], __uint_as_float(sr[c][i]));
      const float mt = fmaxf(fmaxf(fmaxf(mx[0], mx[1]), fmaxf(mx[2], mx[3])),
                             fmaxf(fmaxf(mx[4], mx[5]), fmaxf(mx[6], mx[7]))) * scale_log2;
      bool rescale = false;
      float alpha = 1.f;
      if (j == 0) {
        m_ref = mt;
      } else if (mt > m_ref + RESCALE_THRESHOLD) {
        rescale = true;
        alpha = exp2f(m_ref - mt);
        m_ref = mt;
      }
      l_sum *= alpha;
      const float neg_m = -m_ref;
      float2 lsum[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
      if (full) {
        const float2 sc2 = make_float2(scale_log2, scale_log2), nm2 = make_float2(neg_m, neg_m);
#pragma unroll
        for (int c = 0; c < 2; ++c)
#pragma unroll
          for (int i = 0; i < 32; i += 2) {
            const float2 x = __ffma2_rn(make_float2(__uint_as_float(sr[c][i]), __uint_as_float(sr[c][i + 1])), sc2,
                                        nm2);
            float2 p;
            if (((i >> 1) & 7) >= 8 - NPOLY) p = poly_exp2_x2(x);
            else p = make_float2(fast_exp2(x.x), fast_exp2(x.y));
            lsum[(i >> 1) & 3] = __fadd2_rn(lsum[(i >> 1) & 3], p);
            sr[0][c * 16 + i / 2] = pack_bf16x2(p.x, p.y);      // packed P overwrites consumed S
          }
      } else {
#pragma unroll
        for (int c = 0; c < 2; ++c)
#pragma unroll
          for (int i = 0; i < 32; i += 2) {
            const float p0 = fast_exp2(fmaf(__uint_as_float(sr[c][i]), scale_log2, neg_m));
            const float p1 = fast_exp2(fmaf(__uint_as_float(sr[c][i + 1]), scale_log2, neg_m));
            lsum[(i >> 1) & 3] = __fadd2_rn(lsum[(i >> 1) & 3], make_float2(p0, p1));
            sr[0][c * 16 + i / 2] = pack_bf16x2(p0, p1);
          }
      }
      if (__any_sync(0xffffffffu, rescale)) {
        // O_t must hold exactly tiles < j: wait for PV_t(j-1) (S_t(j) was issued before it)
        mbar_wait(&pv_done[t], (j - 1) & 1);
        tc_fence_after();
#pragma unroll
        for (int c = 0; c < D / 32; ++c) {
          uint32_t ov[32];
          tmem_ld32(o_col + c * 32, ov);
          tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 32; ++i) ov[i] = __float_as_uint(__uint_as_float(ov[i]) * alpha);
          tmem_st32(o_col + c * 32, ov);
        }
      }
      tmem_st32(s_col, sr[0]);
      tmem_st_wait();
      tc_fence_before();
      mbar_arrive(&p_full[t * 2 + (j & 1)]);
      const float2 l01 = __fadd2_rn(lsum[0], lsum[1]), l23 = __fadd2_rn(lsum[2], lsum[3]);
      const float2 l4 = __fadd2_rn(l01, l23);
      l_sum += l4.x + l4.y;
    }
    // epilogue: O_t / l -> bf16 once the last PV_t is complete (pv_done may be two phases behind
    // here: S_t(n-1) complete only implies PV_t(n-3) complete)
    mbar_wait(&o_done[t], 0);
    tc_fence_after();
    const float inv = 1.f / l_sum;
    const int grow = q0 + t * AT_BM + row;
    bf16* orow = o + (long long)grow * ldo + head * D;
    if (sc.k > 0 && grow < L) {
      int p = 0, lr;
      if (grow < sc.Lt) {
        while (p + 1 < sc.k && grow >= sc.t_off[p + 1]) ++p;
        lr = grow - sc.t_off[p];
      } else {
        const int gi = grow - sc.Lt;
        while (p + 1 < sc.k && gi >= sc.i_off[p + 1]) ++p;
        lr = sc.nt[p] + gi - sc.i_off[p];
      }
      orow = sc.dst[p] + (long long)lr * sc.ld + sc.col0 + head * D;
    }
#pragma unroll
    for (int c = 0; c < D / 32; ++c) {
      uint32_t ov[32];
      tmem_ld32(o_col + c * 32, ov);
      tmem_ld_wait();
      if (grow < L) {
        uint4* dst = reinterpret_cast<uint4*>(orow + c * 32);
#pragma unroll
        for (int qd = 0; qd < 4; ++qd) {
          uint4 v;
          v.x = pack_bf16x2(__uint_as_float(ov[qd * 8 + 0]) * inv, __uint_as_float(ov[qd * 8 + 1]) * inv);
          v.y = pack_bf16x2(__uint_as_float(ov[qd * 8 + 2]) * inv, __uint_as_float(ov[qd * 8 + 3]) * inv);
          v.z = pack_bf16x2(__uint_as_float(ov[qd * 8 + 4]) * inv, __uint_as_float(ov[qd * 8 + 5]) * inv);
          v.w = pack_bf16x2(__uint_as_float(ov[qd * 8 + 6]) * inv, __uint_as_float(ov[qd * 8 + 7]) * inv);
          dst[qd] = v;
        }
      }
    }
  }
  grid_dep_launch();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc<512>(tmem);
}

// ------------------------------------------------------------------ v6: CTA pair (cta_group::2)
// A cluster of 2 CTAs computes 512 queries of one head as two pair tiles t = 0, 1 of 256 queries:
// CTA r holds rows [256 t + 128 r, +128) of pair tile t (its Q tiles, its S/P/O rows in its TMEM).
// The even CTA issues tcgen05.mma.cta_group::2 with M = 256: S_t = Q_t K^T (N = 128 keys, each CTA
// holds 64 of the keys) and O_t += P_t V (N = D, each CTA holds D/2 columns of V).  Per SM the
// S MMA reads 96 B/clk of shared memory instead of 128 (the 1-CTA kernel's S MMA sits at the
// shared-memory port limit, like a 128x128 GEMM tile) and K/V tiles cost half the TMA bytes.
// Softmax: v3's lazy-max body per CTA; P hand-over is one arrive per softmax warp on the even
// CTA's barrier (8 warps per pair tile).
template <int D>
struct Fa2Cfg {
  static constexpr int NSUB = D / 64;
  static constexpr int Q_TILE = AT_BM * D * 2;          // 128 rows
  static constexpr int K_HALF = (AT_BN / 2) * D * 2;    // 64 keys x D
  static constexpr int V_HALF = AT_BN * (D / 2) * 2;    // 128 keys x D/2 (one 128-byte swizzle column)
  static constexpr int STAGE = K_HALF + V_HALF;
  static constexpr int NST = 4;
  static constexpr int OFF_Q = 0;                        // 2 tiles
  static constexpr int OFF_KV = OFF_Q + 2 * Q_TILE;      // NST stages of [K half | V half]
  static constexpr int OFF_BAR = OFF_KV + NST * STAGE;
  static constexpr int SMEM = OFF_BAR + 256 + 1024;
  static constexpr int O_COL = 256;
};
static_assert(Fa2Cfg<128>::SMEM <= 227 * 1024, "pair attention smem");

template <int D, int NPOLY>
__global__ void __launch_bounds__(FA_THREADS, 1)
    attention_fa2_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                         const __grid_constant__ CUtensorMap tmV, bf16* __restrict__ o, long long ldo, int L,
                         float scale_log2, const __grid_constant__ AttnScatter sc) {
  static_assert(D == 128, "pair kernel: D = 128 (V halves are one 64-column swizzle block)");
  using C = Fa2Cfg<D>;
  constexpr int NST = C::NST;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + C::OFF_BAR);
  uint64_t* q_full = bars + 0;             // even CTA: both CTAs' Q bytes
  uint64_t* kv_full = bars + 1;            // [NST] even CTA: both halves
  uint64_t* kv_empty = bars + 1 + NST;     // [NST] both CTAs (multicast commit)
  uint64_t* s_full = bars + 1 + 2 * NST;   // [2 t] both CTAs (multicast commit)
  uint64_t* p_full = bars + 3 + 2 * NST;   // [2 t] even CTA: 8 softmax warps
  uint64_t* o_done = bars + 5 + 2 * NST;   // [2 t] both CTAs
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 8 + 2 * NST);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;
  const int head = blockIdx.y;
  const int qc = (blockIdx.x >> 1) * 4 * AT_BM;   // the pair's first query
  const int n_tiles = (L + AT_BN - 1) / AT_BN;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmQ);
    tma_prefetch_desc(&tmK);
    tma_prefetch_desc(&tmV);
    mbar_init(q_full, 1);
    for (int i = 0; i < NST; ++i) {
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&s_full[i], 1);
      mbar_init(&p_full[i], 8);
      mbar_init(&o_done[i], 1);
    }
    fence_mbar_init();
  }
  if (warp == 2) tmem_alloc_pair<512>(tmem_slot);
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  grid_dep_wait();
  if (warp < 4) {
    regs_dec<80>();
    if (warp == 0) {
      if (lane == 0) {
        // -------------------------------------------------------------- producer (both CTAs)
        if (leader) mbar_arrive_expect_tx(q_full, 2 * 2 * C::Q_TILE);
        for (int t = 0; t < 2; ++t)
          for (int s = 0; s < C::NSUB; ++s)
            tma_load_3d_pair(&tmQ, q_full, sm + C::OFF_Q + t * C::Q_TILE + s * (AT_BM * 128), s * 64, head,
                             qc + t * 2 * AT_BM + (int)rank * AT_BM);
        for (int j = 0; j < n_tiles; ++j) {
          const int st = j % NST;
          if (j >= NST) mbar_wait(&kv_empty[st], ((j / NST) - 1) & 1);
          if (leader) mbar_arrive_expect_tx(&kv_full[st], 2 * C::STAGE);
          uint8_t* sk = sm + C::OFF_KV + st * C::STAGE;
          for (int s = 0; s < C::NSUB; ++s)   // keys [128 j + 64 r, +64), all D
            tma_load_3d_pair(&tmK, &kv_full[st], sk + s * ((AT_BN / 2) * 128), s * 64, head,
                             j * AT_BN + (int)rank * (AT_BN / 2));
          // keys [128 j, +128), columns [64 r, +64)
          tma_load_3d_pair(&tmV, &kv_full[st], sk + C::K_HALF, (int)rank * 64, head, j * AT_BN);
        }
      }
    } else if (warp == 1 && leader) {
      // -------------------------------------------------------------- MMA issuer (even CTA, whole warp)
      constexpr uint32_t idesc_s = make_idesc_bf16(2 * AT_BM, AT_BN);
      constexpr uint32_t idesc_o = make_idesc_bf16_bmn(2 * AT_BM, D);
      const uint64_t dq0 = make_sw128_desc(smem_u32(sm + C::OFF_Q));
      const uint64_t dk0 = make_sw128_desc(smem_u32(sm + C::OFF_KV));
      const uint64_t dv0 = make_sw128_mn_desc(smem_u32(sm + C::OFF_KV + C::K_HALF), AT_BN * 128);
      mbar_wait(q_full, 0);
      auto issue_s = [&](int t, int j) {
        const uint64_t dq = dq0 + (uint64_t)((t * C::Q_TILE) >> 4);
        const uint64_t dk = dk0 + (uint64_t)(((j % NST) * C::STAGE) >> 4);
        if (elect_one()) {
#pragma unroll
          for (int kk = 0; kk < D / 16; ++kk) {
            const uint32_t offq = ((kk >> 2) * (AT_BM * 128) + (kk & 3) * 32) >> 4;
            const uint32_t offk = ((kk >> 2) * ((AT_BN / 2) * 128) + (kk & 3) * 32) >> 4;
            umma_bf16_ss_pair(tmem + t * 128, dq + offq, dk + offk, idesc_s, kk > 0);
          }
          umma_commit_pair(&s_full[t]);
        }
        __syncwarp();
      };
      auto issue_pv = [&](int t, int j, bool release) {
        const uint64_t dv = dv0 + (uint64_t)(((j % NST) * C::STAGE) >> 4);
        mbar_wait(&p_full[t], j & 1);
        tc_fence_after();
        if (elect_one()) {
#pragma unroll
          for (int kk = 0; kk < AT_BN / 16; ++kk)
            umma_bf16_ts_pair(tmem + C::O_COL + t * D, tmem + t * 128 + kk * 8, dv + (uint64_t)(kk * (2048 >> 4)),
                              idesc_o, (j | kk) != 0);
          if (release) umma_commit_pair(&kv_empty[j % NST]);
        }
        __syncwarp();
      };
      for (int j = 0; j < n_tiles; ++j) {
        mbar_wait(&kv_full[j % NST], (j / NST) & 1);
        tc_fence_after();
        for (int t = 0; t < 2; ++t) {
          if (j > 0) issue_pv(t, j - 1, t == 1);
          issue_s(t, j);
        }
      }
      for (int t = 0; t < 2; ++t) {
        issue_pv(t, n_tiles - 1, false);
        if (elect_one()) umma_commit_pair(&o_done[t]);
        __syncwarp();
      }
    }
  } else {
    regs_inc<208>();
    // ---------------------------------------------------------------- softmax WG t (thread = query row)
    const int t = (warp - 4) >> 2;
    const int wq = (warp - 4) & 3;
    const int row = wq * 32 + lane;
    const uint32_t lane_base = (uint32_t)(wq * 32) << 16;
    const uint32_t s_col = tmem + lane_base + t * 128;
    const uint32_t o_col = tmem + lane_base + C::O_COL + t * D;
    float m_ref = -FLT_MAX, l_sum = 0.f;
    auto hand_over = [&]() {   // P_t(j) stored: one arrive per warp on the even CTA's barrier
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive_remote(&p_full[t], 0);
    };
    for (int j = 0; j < n_tiles; ++j) {
      mbar_wait(&s_full[t], j & 1);
      tc_fence_after();
      uint32_t sr[4][32];
#pragma unroll
      for (int c = 0; c < 4; ++c) tmem_ld32(s_col + c * 32, sr[c]);
      tmem_ld_wait();
      const int kbase = j * AT_BN;
      const bool full = kbase + AT_BN <= L;
      if (j > 0 && full) {
        // lazy max (see attention_fa_kernel): P with the running reference, exact path if any row's
        // tile sum exceeds the bound
        const float2 sc2 = make_float2(scale_log2, scale_log2), nm2 = make_float2(-m_ref, -m_ref);
        float2 lz[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
          for (int i = 0; i < 32; i += 2) {
            float2 x = __ffma2_rn(make_float2(__uint_as_float(sr[c][i]), __uint_as_float(sr[c][i + 1])), sc2, nm2);
            float2 p;
            if (((i >> 1) & 7) >= 8 - NPOLY) {
              x.x = fminf(x.x, 64.f);
              x.y = fminf(x.y, 64.f);
              p = poly_exp2_x2(x);
            } else {
              p = make_float2(fast_exp2(x.x), fast_exp2(x.y));
            }
            lz[(i >> 1) & 3] = __fadd2_rn(lz[(i >> 1) & 3], p);
            sr[c >> 1][(c & 1) * 16 + i / 2] = pack_bf16x2(p.x, p.y);
          }
        const float2 l01 = __fadd2_rn(lz[0], lz[1]), l23 = __fadd2_rn(lz[2], lz[3]);
        const float2 l4 = __fadd2_rn(l01, l23);
        const float ts = l4.x + l4.y;
        if (!__any_sync(0xffffffffu, !(ts <= LAZY_LIMIT))) {
          l_sum += ts;
          tmem_st32(s_col, sr[0]);
          tmem_st32(s_col + 32, sr[1]);
          hand_over();
          continue;
        }
#pragma unroll
        for (int c = 0; c < 4; ++c) tmem_ld32(s_col + c * 32, sr[c]);
        tmem_ld_wait();
      }
      // exact path: first tile, the masked last tile, and lazy overflows
      float mx[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) mx[q] = -FLT_MAX;
      if (!full) {
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (kbase + c * 32 + i >= L) sr[c][i] = __float_as_uint(-INFINITY);
      }
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int i = 0; i < 32; ++i) mx[i & 7] = fmaxf(mx[i & 7], __uint_as_float(sr[c][i]));
      const float mt = fmaxf(fmaxf(fmaxf(mx[0], mx[1]), fmaxf(mx[2], mx[3])),
                             fmaxf(fmaxf(mx[4], mx[5]), fmaxf(mx[6], mx[7]))) * scale_log2;
      bool rescale = false;
      float alpha = 1.f;
      if (j == 0) {
        m_ref = mt;
      } else if (mt > m_ref + RESCALE_THRESHOLD) {
        rescale = true;
        alpha = exp2f(m_ref - mt);
        m_ref = mt;
      }
      l_sum *= alpha;
      const float neg_m = -m_ref;
      float2 lsum[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int i = 0; i < 32; i += 2) {
          const float p0 = fast_exp2(fmaf(__uint_as_float(sr[c][i]), scale_log2, neg_m));
          const float p1 = fast_exp2(fmaf(__uint_as_float(sr[c][i + 1]), scale_log2, neg_m));
          lsum[(i >> 1) & 3] = __fadd2_rn(lsum[(i >> 1) & 3], make_float2(p0, p1));
          sr[c >> 1][(c & 1) * 16 + i / 2] = pack_bf16x2(p0, p1);
        }
      if (__any_sync(0xffffffffu, rescale)) {
        // S_t(j) complete => PV_t(j-1) complete (in-order pipe of the pair): O_t holds tiles < j
#pragma unroll
        for (int c = 0; c < D / 32; ++c) {
          uint32_t ov[32];
          tmem_ld32(o_col + c * 32, ov);
          tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 32; ++i) ov[i] = __float_as_uint(__uint_as_float(ov[i]) * alpha);
          tmem_st32(o_col + c * 32, ov);
        }
      }
      tmem_st32(s_col, sr[0]);
      tmem_st32(s_col + 32, sr[1]);
      hand_over();
      const float2 l01 = __fadd2_rn(lsum[0], lsum[1]), l23 = __fadd2_rn(lsum[2], lsum[3]);
      const float2 l4 = __fadd2_rn(l01, l23);
      l_sum += l4.x + l4.y;
    }
    // epilogue: O_t / l -> bf16
    mbar_wait(&o_done[t], 0);
    tc_fence_after();
    const float inv = 1.f / l_sum;
    const int grow = qc + t * 2 * AT_BM + (int)rank * AT_BM + row;
    bf16* orow = o + (long long)grow * ldo + head * D;
    if (sc.k > 0 && grow < L) {
      int p = 0, lr;
      if (grow < sc.Lt) {
        while (p + 1 < sc.k && grow >= sc.t_off[p + 1]) ++p;
        lr = grow - sc.t_off[p];
      } else {
        const int gi = grow - sc.Lt;
        while (p + 1 < sc.k && gi >= sc.i_off[p + 1]) ++p;
        lr = sc.nt[p] + gi - sc.i_off[p];
      }
      orow = sc.dst[p] + (long long)lr * sc.ld + sc.col0 + head * D;
    }
#pragma unroll
    for (int c = 0; c < D / 32; ++c) {
      uint32_t ov[32];
      tmem_ld32(o_col + c * 32, ov);
      tmem_ld_wait();
      if (grow < L) {
        uint4* dst = reinterpret_cast<uint4*>(orow + c * 32);
#pragma unroll
        for (int qd = 0; qd < 4; ++qd) {
          uint4 v;
          v.x = pack_bf16x2(__uint_as_float(ov[qd * 8 + 0]) * inv, __uint_as_float(ov[qd * 8 + 1]) * inv);
          v.y = pack_bf16x2(__uint_as_float(ov[qd * 8 + 2]) * inv, __uint_as_float(ov[qd * 8 + 3]) * inv);
          v.z = pack_bf16x2(__uint_as_float(ov[qd * 8 + 4]) * inv, __uint_as_float(ov[qd * 8 + 5]) * inv);
          v.w = pack_bf16x2(__uint_as_float(ov[qd * 8 + 6]) * inv, __uint_as_float(ov[qd * 8 + 7]) * inv);
          dst[qd] = v;
        }
      }
    }
  }
  grid_dep_launch();
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  if (warp == 2) tmem_dealloc_pair<512>(tmem);
}

// ------------------------------------------------------------------ host
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
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

// [rows][heads][D] view of a strided activation: element (r, h, d) at base + r*ld + h*D + d
static int make_tmap_heads(CUtensorMap* m, const void* base, int D, int H, int L, long long ld, int box_rows = 128) {
  auto enc = encode_fn();
  if (!enc) return -1;
  cuuint64_t dims[3] = {(cuuint64_t)D, (cuuint64_t)H, (cuuint64_t)L};
  cuuint64_t strides[2] = {(cuuint64_t)D * 2, (cuuint64_t)ld * 2};
  cuuint32_t box[3] = {64, 1, (cuuint32_t)box_rows};
  cuuint32_t es[3] = {1, 1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? 0 : -2;
}

// default share of exp2 evaluated by polynomial, per head dim (tools/microbench.py sweep)
template <int D>
constexpr int default_npoly() { return D == 64 ? 2 : 1; }   // measured (profiles/README.md)

template <int D, int NP, bool SPLIT = false, bool LAZY = false>
static void launch_fa(const CUtensorMap& tq, const CUtensorMap& tk, const CUtensorMap& tv, bf16* o, long long ldo,
                      int L, int H, float scale_log2, const AttnScatter& sc, cudaStream_t s,
                      const AttnSplitArgs& sa = AttnSplitArgs()) {
  static unsigned long long done = 0;
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(done >> dev & 1ull)) {
    cudaFuncSetAttribute(attention_fa_kernel<D, NP, SPLIT, LAZY>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         FaCfg<D>::SMEM);
    done |= 1ull << dev;
  }
  dim3 grid((L + 2 * AT_BM - 1) / (2 * AT_BM), H, sa.nsplit);
  launch_pdl(attention_fa_kernel<D, NP, SPLIT, LAZY>, grid, dim3(FA_THREADS), FaCfg<D>::SMEM, s, tq, tk, tv, o, ldo, L, scale_log2,
             sc, sa);
}

template <int D, int NP>
static void launch_fa5(const CUtensorMap& tq, const CUtensorMap& tk, const CUtensorMap& tv, bf16* o, long long ldo,
                       int L, int H, float scale_log2, const AttnScatter& sc, cudaStream_t s) {
  static unsigned long long done = 0;
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(done >> dev & 1ull)) {
    cudaFuncSetAttribute(attention_fa5_kernel<D, NP>, cudaFuncAttributeMaxDynamicSharedMemorySize, Fa5Cfg<D>::SMEM);
    done |= 1ull << dev;
  }
  dim3 grid((L + 2 * AT_BM - 1) / (2 * AT_BM), H);
  launch_pdl(attention_fa5_kernel<D, NP>, grid, dim3(FA_THREADS), Fa5Cfg<D>::SMEM, s, tq, tk, tv, o, ldo, L,
             scale_log2, sc);
}

template <int NP>
static void launch_fa2(const CUtensorMap& tq, const CUtensorMap& tk, const CUtensorMap& tv, bf16* o, long long ldo,
                       int L, int H, float scale_log2, const AttnScatter& sc, cudaStream_t s) {
  static unsigned long long done = 0;
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(done >> dev & 1ull)) {
    cudaFuncSetAttribute(attention_fa2_kernel<128, NP>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         Fa2Cfg<128>::SMEM);
    done |= 1ull << dev;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(2 * ((L + 4 * AT_BM - 1) / (4 * AT_BM)), H);
  cfg.blockDim = dim3(FA_THREADS);
  cfg.dynamicSmemBytes = Fa2Cfg<128>::SMEM;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  attr[1].id = cudaLaunchAttributeClusterDimension;
  attr[1].val.clusterDim.x = 2;
  attr[1].val.clusterDim.y = 1;
  attr[1].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  cudaLaunchKernelEx(&cfg, attention_fa2_kernel<128, NP>, tq, tk, tv, o, ldo, L, scale_log2, sc);
}

// KV-split factor for a launch of C = ceil(L/256) x H CTAs: the S in 1..8 minimising the estimated
// makespan (below), each split >= 4 key tiles.
static int KV_MIN_TILES = 4, KV_SPLIT_COST = 6;   // TSV_KV_MIN / TSV_KV_COST override (tuning)
static AttnSplitArgs plan_kv_split(int L, int H, int D, const AttnSplitWs* w) {
  static bool env_read = false;
  if (!env_read) {
    if (const char* v = getenv("TSV_KV_MIN")) KV_MIN_TILES = atoi(v);
    if (const char* v = getenv("TSV_KV_COST")) KV_SPLIT_COST = atoi(v);
    env_read = true;
  }
  AttnSplitArgs a;
  if (!w || !w->cnt || !w->ws) return a;
  static int sms_of[64] = {0};
  int dev = 0;
  cudaGetDevice(&dev);
  if (!sms_of[dev & 63]) cudaDeviceGetAttribute(&sms_of[dev & 63], cudaDevAttrMultiProcessorCount, dev);
  const int sms = sms_of[dev & 63] ? sms_of[dev & 63] : 148;
  const int n_all = (L + AT_BN - 1) / AT_BN;
  const long long C = (long long)((L + 2 * AT_BM - 1) / (2 * AT_BM)) * H;
  int best = 1;
  if (w->force > 0) {
    best = w->force < n_all ? w->force : n_all;
  } else {
    // makespan in key-tile units: waves x (tiles per split + fixed cost), the fixed cost (prologue,
    // pipeline fill, epilogue; + the merge when split) fitted to tools/microbench.py attnsplit
    double bestc = (double)((C + sms - 1) / sms) * (n_all + 2);
    for (int S = 2; S <= 8; ++S) {
      const int tps = (n_all + S - 1) / S;
      if (tps < KV_MIN_TILES) break;
      const double cost = (double)((C * S + sms - 1) / sms) * (tps + KV_SPLIT_COST);
      if (cost < bestc * 0.95) { bestc = cost; best = S; }
    }
  }
  if (best < 2) return a;
  const int tps = (n_all + best - 1) / best;
  best = (n_all + tps - 1) / tps;   // no empty split
  if (best < 2 || best > 8) return a;
  if ((long long)C * 2 * best * AT_BM * (D + 2) * 4 > w->ws_bytes || C * 2 * 4 > w->cnt_ints) return a;
  a.nsplit = best;
  a.tps = tps;
  a.cnt = w->cnt;
  a.ws = w->ws;
  return a;
}

template <int D>
static int launch_tc(const bf16* q, long long ldq, const bf16* k, long long ldk, const bf16* v, long long ldv, bf16* o,
                     long long ldo, int L, int H, int version, const AttnScatter& sc, cudaStream_t s,
                     const AttnSplitWs* spw) {
  CUtensorMap tq, tk, tv;
  if (make_tmap_heads(&tq, q, D, H, L, ldq) || make_tmap_heads(&tk, k, D, H, L, ldk) ||
      make_tmap_heads(&tv, v, D, H, L, ldv))
    return -1;
  static unsigned long long done = 0;
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(done >> dev & 1ull)) {
    cudaFuncSetAttribute(attention_tc_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, AttnCfg<D>::SMEM);
    done |= 1ull << dev;
  }
  const float scale_log2 = (1.0f / sqrtf((float)D)) * 1.4426950408889634f;
  if (version >= 40 && version < 50) {   // v5: 64-key K/V tiles, double-buffered S; 40 + n: n of 8 exp2 pairs by polynomial
    CUtensorMap tk64, tv64;
    if (make_tmap_heads(&tk64, k, D, H, L, ldk, 64) || make_tmap_heads(&tv64, v, D, H, L, ldv, 64)) return -1;
    switch (version - 40) {
      case 0: launch_fa5<D, 0>(tq, tk64, tv64, o, ldo, L, H, scale_log2, sc, s); break;
      case 1: launch_fa5<D, 1>(tq, tk64, tv64, o, ldo, L, H, scale_log2, sc, s); break;
      case 2: launch_fa5<D, 2>(tq, tk64, tv64, o, ldo, L, H, scale_log2, sc, s); break;
      case 3: launch_fa5<D, 3>(tq, tk64, tv64, o, ldo, L, H, scale_log2, sc, s); break;
      case 4: launch_fa5<D, 4>(tq, tk64, tv64, o, ldo, L, H, scale_log2, sc, s); break;
      default: return -3;
    }
    return 0;
  }
  if (version >= 60) {   // 60 + n: CTA-pair kernel (D = 128 only), lazy max, n of 8 exp2 pairs by polynomial
    if (D != 128) return -3;
    CUtensorMap tk64, tv64;   // K halves: 64-key boxes; V halves: 128 keys x 64 columns (the default box)
    if (make_tmap_heads(&tk64, k, D, H, L, ldk, 64)) return -1;
    switch (version - 60) {
      case 0: launch_fa2<0>(tq, tk64, tv, o, ldo, L, H, scale_log2, sc, s); break;
      case 1: launch_fa2<1>(tq, tk64, tv, o, ldo, L, H, scale_log2, sc, s); break;
      case 2: launch_fa2<2>(tq, tk64, tv, o, ldo, L, H, scale_log2, sc, s); break;
      case 3: launch_fa2<3>(tq, tk64, tv, o, ldo, L, H, scale_log2, sc, s); break;
      default: return -3;
    }
    return 0;
  }
  if (version >= 50) {   // 50 + n: lazy row max (see attention_fa_kernel), n of 8 exp2 pairs by polynomial
    const AttnSplitArgs sa = plan_kv_split(L, H, D, spw);
    switch (version - 50) {
      case 0: launch_fa<D, 0, false, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
      case 1: launch_fa<D, 1, false, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
      case 2: launch_fa<D, 2, false, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
      case 3: launch_fa<D, 3, false, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
      case 4: launch_fa<D, 4, false, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
      default: return -3;
    }
    return 0;
  }
  if (version == 2) {
    dim3 grid((L + AT_BM - 1) / AT_BM, H);
    attention_tc_kernel<D><<<grid, AT_THREADS, AttnCfg<D>::SMEM, s>>>(tq, tk, tv, o, ldo, L, scale_log2);
  } else {
    // version 3: the default poly share; 10 + n: n of 8 exp2 pairs by polynomial (tuning sweeps);
    // 20 + n: the same with P handed over in two halves (SPLIT)
    const int np = version >= 10 ? version % 10 : default_npoly<D>();
    if (version >= 20) {
      switch (np) {
        case 1: launch_fa<D, 1, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
        case 2: launch_fa<D, 2, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
        case 3: launch_fa<D, 3, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
        case 4: launch_fa<D, 4, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
        default: return -3;
      }
      return 0;
    }
    switch (np) {
      case 1: launch_fa<D, 1>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
      case 2: launch_fa<D, 2>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
      case 3: launch_fa<D, 3>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
      case 4: launch_fa<D, 4>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
      case 5: launch_fa<D, 5>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s); break;
      default: return -3;
    }
  }
  return 0;
}

// The step's variant per head dim (profiles/README.md, attention table); TSV_ATTN_D128 / TSV_ATTN_D64
// override it with any tsv_op_attention impl number >= 3 (same-box A/B of whole steps).
static int default_version(int D) {
  static int v[2] = {-1, -1};
  int& r = v[D == 128];
  if (r < 0) {
    const char* e = getenv(D == 128 ? "TSV_ATTN_D128" : "TSV_ATTN_D64");
    r = e ? atoi(e) : (D == 128 ? 51 : 52);   // lazy max; 1 (D = 128) / 2 (D = 64) of 8 exp2 pairs by polynomial (in-step A/B)
    if (r < 3) r = 3;
  }
  return r;
}

// returns 0 if the tensor-core path was launched, nonzero if the layout is unsupported by TMA.
// version 3: two query tiles per CTA, P in TMEM (the step's kernel); version 2: one query tile,
// P in shared memory (kept for comparison).
int attention_launch(const bf16* q, long long ldq, const bf16* k, long long ldk, const bf16* v, long long ldv,
                     bf16* o, long long ldo, int L, int H, int D, cudaStream_t s, int version,
                     const AttnScatter* scatter, const AttnSplitWs* split) {
  if (L <= 0 || H <= 0) return 0;
  AttnScatter sc;
  if (scatter) {
    sc = *scatter;
    if (sc.k < 1 || sc.k > 8 || version == 2) return -4;
  }
  if (((ldq | ldk | ldv) * 2) % 16 || ((reinterpret_cast<uintptr_t>(q) | reinterpret_cast<uintptr_t>(k) |
                                        reinterpret_cast<uintptr_t>(v)) & 15))
    return -1;
  if (version == 3) version = default_version(D);
  if (D == 128) return launch_tc<128>(q, ldq, k, ldk, v, ldv, o, ldo, L, H, version, sc, s, split);
  if (D == 64) return launch_tc<64>(q, ldq, k, ldk, v, ldv, o, ldo, L, H, version, sc, s, split);
  return -1;
}

}  // namespace tsv
