// Joint text+image attention on the 5th-gen tensor cores (S:§8(a) a6):
//   O = softmax(q k^T / sqrt(D)) v, non-causal, per head, fp32 softmax, bf16 operands.
//
// One CTA = one head x 256 queries as two 128-query tiles t = 0, 1 that share every K/V tile
// (half the K/V traffic per query).  Warp roles:
//   warps 0, 3  TMA producers: Q0, Q1 once, then K tiles of 128 keys into an NK-stage ring (warp 0)
//               and V tiles into an NV-stage ring (warp 3) (3-D tensor maps [rows][heads][D] -> one
//               map serves every head and layout);
//   warp 1      tcgen05.mma issuer (the whole warp runs the loop, one elected lane issues):
//               S_t(j) = Q_t K_j^T into TMEM, O_t += P_t(j) V_j with P read from TMEM and V
//               consumed MN-major straight from the TMA tile (no transpose, no smem P);
//   warps 4-11  two softmax warpgroups (4-7: tile 0, 8-11: tile 1), thread = query row = TMEM lane.
// The two warpgroups ping-pong with the tensor core: while WG0 turns S_0(j) into P_0(j), the MMA
// warp runs PV_1(j-1) and S_1(j), and vice versa.  P_t(j) is written back into the S_t columns as
// bf16 (tcgen05.st), so S_t(j+1) must follow PV_t(j): the MMA warp issues PV_t(j) before S_t(j+1),
// and the in-order tcgen05 pipe makes "S_t(j) complete" imply "O_t holds tiles < j" (a rare O
// rescale needs no extra wait).
// TMEM: S0 | S1 | O0 | O1 (128 + 128 + D + D fp32 columns).  Smem: Q0, Q1, NK K and NV V stages.
//
// Softmax (lazy row max): P = 2^(s * scale_log2 - m_ref) is evaluated with the running reference
// m_ref directly, without a per-tile max: the tile's row sum bounds every p in it (p <= sum), so a
// row whose sum stays <= 2^16 needs no rescale (m_ref only stabilises: softmax is exact for any
// reference that keeps p finite).  Otherwise (the max grew a lot: early tiles) the warp reloads S
// from TMEM and takes the exact path (row max, conditional O rescale when the max grows by > 2^8).
// Without the max the four TMEM loads of S are pipelined under the exponentials.  NPOLY of every 8
// exp2 pairs are evaluated on the FMA pipe (Cody-Waite split + cubic) to relieve MUFU.EX2.
//
// KV split (AttnSplitArgs): the last work items of a launch (or all of them: SP = 4/8 head shards) are
// split into key ranges, and the last range of a 32-row warp merges the (O, m, l) partials in range order.
//
// Measured dead ends (profiles/README.md): one query tile per CTA with P in shared
// memory; 64-key tiles with double-buffered S (the N = 64 S MMA re-reads Q from shared memory at
// 192 B/clk); P handed over in two halves; CTA-pair (cta_group::2) tiles (-17 %: the pair couples
// both CTAs' softmax chains); two softmax warps per row; packed ex2 (two MUFU ops per instruction).
#include <algorithm>
#include <cfloat>
#include <map>
#include <mutex>
#include <tuple>
#include <vector>
#include <cstdio>
#include <cstdlib>
#include <cudaTypedefs.h>

#include "kernels.h"
#include "ptx.cuh"

namespace tsv {

namespace {

constexpr int AT_BM = 128;     // queries per tile
constexpr int AT_BN = 128;     // keys per tile
constexpr float RESCALE_THRESHOLD = 8.0f;  // log2 domain
constexpr float LAZY_LIMIT = 65536.0f;     // 2^16

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
// 2^x without the MUFU on a pair, with the sm_100 paired FP32 ops (FADD2 / FFMA2): x = n + f
// (n = round(x), |f| <= 1/2), 2^f by a cubic (Taylor of e^(f ln2), rel. error <= 7e-4 on
// |f| <= 1/2, below the bf16 rounding P gets anyway), 2^n added to the exponent field.  x is
// clamped at -126 so the exponent add cannot wrap (the true value is < 2^-126 there).
__device__ __forceinline__ float2 poly_exp2_x2(float2 x) {
  x.x = fmaxf(x.x, -126.0f);
  x.y = fmaxf(x.y, -126.0f);
  const float2 magic = make_float2(12582912.0f, 12582912.0f);   // 1.5 * 2^23: round(x) in the low bits
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
// The same 2^x for a pair of raw scores s (x = s * scale - m), with the clamp to [-126, 64] done by
// the saturating FFMA: y = sat(s * ca + cb) in [0, 1] (ca = scale / 190, cb = (126 - m) / 190), so
// x' = 190 y - 126 in [-126, 64] -- two FFMA.SAT instead of the scale FFMA2 and four FMNMX.  The
// rounding to n and the remainder f = x' - n come straight from y: t = 190 y + (magic - 126) holds
// n = round(x') in its low bits, f = 190 y - (t - (magic - 126)).  |x' - x| <= ~2e-5 (two fp32
// roundings at |x| <= 190): a relative error of ~1.4e-5 in p, far below P's bf16 rounding.
__device__ __forceinline__ float sat_fma(float a, float b, float c) {
  float d;
  asm("fma.rn.sat.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
  return d;
}
// DEG = 3: the cubic above; DEG = 2: the minimax quadratic for the relative error on |f| <= 1/2
// (Remez: max 1.72e-3, P's bf16 rounding is 1.95e-3) -- one FFMA2 less per pair.
template <int DEG = 3>
__device__ __forceinline__ float2 poly_exp2_sat_x2(float s0, float s1, float ca, float cb) {
  const float2 y = make_float2(sat_fma(s0, ca, cb), sat_fma(s1, ca, cb));
  const float2 k190 = make_float2(190.0f, 190.0f);
  const float2 t = __ffma2_rn(y, k190, make_float2(12582786.0f, 12582786.0f));      // magic - 126
  const float2 nn = __ffma2_rn(t, make_float2(-1.0f, -1.0f), make_float2(12582786.0f, 12582786.0f));  // -(n + 126)
  const float2 f = __ffma2_rn(y, k190, nn);
  float2 p;
  if constexpr (DEG == 2) {
    p = __ffma2_rn(make_float2(0.23842894f, 0.23842894f), f, make_float2(0.703448f, 0.703448f));
    p = __ffma2_rn(p, f, make_float2(1.0004431f, 1.0004431f));
  } else {
    p = __ffma2_rn(make_float2(0.0555041086648216f, 0.0555041086648216f), f,
                   make_float2(0.2402265069591007f, 0.2402265069591007f));
    p = __ffma2_rn(p, f, make_float2(0.6931471805599453f, 0.6931471805599453f));
    p = __ffma2_rn(p, f, make_float2(1.0f, 1.0f));
  }
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

// K and V tiles flow through separate rings (NK and NV stages) filled by two producer warps: a K
// stage is free as soon as both S MMAs of its tile completed, a V stage only after both PV MMAs, so
// the next K load starts ~one tile of tensor time earlier than with one joint K/V stage (r02: the
// MMA warp spent most of its stall samples waiting for K/V data with the joint 2-stage ring).
// KV = 0: NK = NV = 2 (D = 128) / 4 (D = 64) (3 + 2 stages fill the 227 KB at D = 128 and measured
// slower); KV = 3: one joint K+V ring (NK = NV stages, one producer, a stage freed after both PV MMAs:
// round 1's design, kept at D = 64 where it measured better).
// RS (rotating S buffers, D = 64 only): three 128-column S buffers shared by the two query tiles
// (S index n = 2 j + t lives in buffer n % 3) instead of one per tile, so the MMA warp runs one S
// ahead -- S_t(j+1) is computed while P_t(j) still waits for its PV MMA -- and a softmax warpgroup
// finds its next scores ready instead of waiting for PV_t(j) + S_t(j+1) (at D = 64 the tensor work
// of a tile, 512 cycles, is shorter than its softmax).  TMEM: 3 x 128 (S) + 2 x 64 (O) = 512.
template <int D, int KV = 0, bool RS = false>
struct FaCfg {
  static constexpr int NSUB = D / 64;
  static constexpr int Q_TILE = AT_BM * D * 2;
  static constexpr int KV_TILE = AT_BN * D * 2;
  static_assert(KV == 0 || KV == 3, "K/V ring layout");
  static constexpr int NK = D == 64 ? 4 : 2;
  static constexpr int NV = D == 64 ? 4 : 2;
  static constexpr int OFF_Q = 0;                        // 2 tiles
  static constexpr int OFF_K = OFF_Q + 2 * Q_TILE;       // NK stages
  static constexpr int OFF_V = OFF_K + NK * KV_TILE;     // NV stages
  static constexpr int OFF_BAR = OFF_V + NV * KV_TILE;
  static constexpr int NBAR = 1 + 2 * NK + 2 * NV + 3 + 6 + 2 + 6 + 1;   // mbarriers + the TMEM address slot
  static_assert(NBAR * 8 <= 512, "barrier region");
  static constexpr int SMEM = OFF_BAR + 512 + 1024;      // barriers + 1 KB alignment slack
  static constexpr int NSB = RS ? 3 : 2;                 // S buffers
  static constexpr int O_COL = NSB * 128;
  static_assert(O_COL + 2 * D <= 512, "TMEM columns (RS needs D = 64)");
};
// setmaxnreg: the producer / MMA warpgroup drops to 80 registers, the two softmax warpgroups take
// 208.  The CTA's pool is what the launch allocated -- 384 threads x the count ptxas fits under
// __launch_bounds__(384, 1) (64K / 384 rounded down to 8 = 168) -- and an .inc blocks until the pool
// has the registers, so the split must fit that pool (a 4-tile variant that over-asked hung).
static_assert(80 * 128 + 208 * 256 <= ((65536 / 384) & ~7) * 384, "setmaxnreg split exceeds the pool");
static_assert(FaCfg<128>::SMEM <= 232448 && FaCfg<64>::SMEM <= 232448 && FaCfg<64, 3, true>::SMEM <= 232448,
              "attention shared memory > 227 KB");
constexpr int FA_THREADS = 384;

// The launch is 1-D over work items i = query block + nqb * head: CTAs [0, n_plain) are items 0..n_plain-1
// over all their keys; the remaining n_tail items ("the tail", dispatched last) are split into nsplit
// key ranges, CTA n_plain + z * n_tail + u covering range z of item n_plain + u, z-major (every tail
// item's first range before any second range).  n_plain = 0: every item split (the uniform KV split).
struct AttnSplitArgs {
  int nsplit = 1, tps = 0;   // key ranges per tail item, tiles of the largest
  int n_plain = 0, n_tail = 0, nqb = 1;
  int bound[9] = {0};        // range z covers key tiles [bound[z], bound[z + 1])
  int* cnt = nullptr;
  float* ws = nullptr;
};

template <int D, int NPOLY, int KV, bool RS = false, int PSAT = 0>
__global__ void __launch_bounds__(FA_THREADS, 1)
    attention_fa_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                        const __grid_constant__ CUtensorMap tmV, bf16* __restrict__ o, long long ldo, int L,
                        float scale_log2, const __grid_constant__ AttnScatter sc,
                        const __grid_constant__ AttnSplitArgs sa) {
  using C = FaCfg<D, KV, RS>;
  constexpr bool JOINT = KV == 3;   // K and V of a tile share one stage and one barrier pair
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1 KB alignment by pointer arithmetic on the shared array (an integer round trip would make the
  // derived pointers generic: the epilogue's staging accesses compiled to LD.E / ST.E instead of LDS / STS)
  uint8_t* sm = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + C::OFF_BAR);
  constexpr int NK = C::NK, NV = C::NV;
  uint64_t* q_full = bars + 0;
  uint64_t* k_full = bars + 1;                    // [NK stages]
  uint64_t* k_empty = k_full + NK;                // [NK stages]
  uint64_t* v_full = k_empty + NK;                // [NV stages]
  uint64_t* v_empty = v_full + NV;                // [NV stages]
  // RS lets the warps of one softmax warpgroup drift up to two tiles apart (S_t(j+1), S_t(j+2) can be
  // ready before PV_t(j) consumed P_t(j)), so the per-tile barriers that see arrivals or waits from
  // several of a warpgroup's tiles at once come in three copies, tile j using copy j % 3 (phase
  // (j / 3) & 1): one barrier would mix a fast warp's arrival for tile j+1 into tile j's phase.
  uint64_t* s_full = v_empty + NV;                // [3: per S buffer (RS) / per q-tile]
  uint64_t* p_full = s_full + 3;                  // [2 q-tiles][3]
  uint64_t* o_done = p_full + 6;                  // [2 q-tiles]
  uint64_t* pv_done = o_done + 2;                 // [2 q-tiles][3] RS: PV_t(j) complete (a rescale's wait)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(pv_done + 6);

  // tile j's copy of a per-tile barrier of q-tile t, and the phase parity to wait for
  auto tb = [](uint64_t* base, int t, int j) { return base + t * 3 + (RS ? j % 3 : 0); };
  auto tpar = [](int j) { return (uint32_t)((RS ? j / 3 : j) & 1); };
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // work item and key range of this CTA (see AttnSplitArgs)
  const int bid = blockIdx.x;
  const bool split = bid >= sa.n_plain && sa.nsplit > 1;
  const int tail_u = split ? (bid - sa.n_plain) % sa.n_tail : 0;
  const int zr = split ? (bid - sa.n_plain) / sa.n_tail : 0;
  const int item = split ? sa.n_plain + tail_u : bid;
  const int head = item / sa.nqb;
  const int q0 = (item - head * sa.nqb) * 2 * AT_BM;
  // this CTA's key tiles: [j0, j0 + n_tiles) (all of them unless the launch splits the keys)
  const int n_all = (L + AT_BN - 1) / AT_BN;
  const int j0 = split ? sa.bound[zr] : 0;
  const int n_tiles = split ? sa.bound[zr + 1] - j0 : n_all;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmQ);
    tma_prefetch_desc(&tmK);
    tma_prefetch_desc(&tmV);
    mbar_init(q_full, 1);
    for (int i = 0; i < NK; ++i) {
      mbar_init(&k_full[i], 1);
      mbar_init(&k_empty[i], 1);
    }
    for (int i = 0; i < NV; ++i) {
      mbar_init(&v_full[i], 1);
      mbar_init(&v_empty[i], 1);
    }
    for (int i = 0; i < 3; ++i) mbar_init(&s_full[i], 1);
    for (int i = 0; i < 6; ++i) {
      mbar_init(&p_full[i], 128);
      mbar_init(&pv_done[i], 1);
    }
    for (int i = 0; i < 2; ++i) mbar_init(&o_done[i], 1);
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
      // ---------------------------------------------------------------- producer: Q, then the K ring
      mbar_arrive_expect_tx(q_full, 2 * C::Q_TILE);
      for (int t = 0; t < 2; ++t)
        for (int s = 0; s < C::NSUB; ++s)
          tma_load_3d(&tmQ, q_full, sm + C::OFF_Q + t * C::Q_TILE + s * (AT_BM * 128), s * 64, head,
                      q0 + t * AT_BM);
      for (int j = 0; j < n_tiles; ++j) {
        const int st = j % NK;
        if (j >= NK) mbar_wait(&k_empty[st], ((j / NK) - 1) & 1);
        mbar_arrive_expect_tx(&k_full[st], (JOINT ? 2 : 1) * C::KV_TILE);
        for (int s = 0; s < C::NSUB; ++s) {
          tma_load_3d(&tmK, &k_full[st], sm + C::OFF_K + st * C::KV_TILE + s * (AT_BN * 128), s * 64, head,
                      (j0 + j) * AT_BN);
          if (JOINT)
            tma_load_3d(&tmV, &k_full[st], sm + C::OFF_V + st * C::KV_TILE + s * (AT_BN * 128), s * 64, head,
                        (j0 + j) * AT_BN);
        }
      }
    }
   } else if (warp == 3 && !JOINT) {
    if (lane == 0) {
      // ---------------------------------------------------------------- producer: the V ring
      // V(0) is needed only after S(0): start once Q has landed (K(0) was issued right behind it), so
      // the first S MMAs do not share the start-up bandwidth with V traffic (short key loops: small
      // images, KV splits).  q_full completes exactly once, so this wait cannot miss its phase.
      mbar_wait(q_full, 0);
      for (int j = 0; j < n_tiles; ++j) {
        const int st = j % NV;
        if (j >= NV) mbar_wait(&v_empty[st], ((j / NV) - 1) & 1);
        mbar_arrive_expect_tx(&v_full[st], C::KV_TILE);
        for (int s = 0; s < C::NSUB; ++s)
          tma_load_3d(&tmV, &v_full[st], sm + C::OFF_V + st * C::KV_TILE + s * (AT_BN * 128), s * 64, head,
                      (j0 + j) * AT_BN);
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
    // S buffer of S index n = 2 j + t: the tile's own (t) or, RS, the rotating n % 3
    auto sbuf = [](int t, int j) { return RS ? (2 * j + t) % 3 : t; };
    auto issue_s = [&](int t, int j) {   // t == 1 releases the K stage (both S MMAs of tile j issued)
      const uint64_t dq = dq0 + (uint64_t)((t * C::Q_TILE) >> 4);
      const uint64_t dk = dk0 + (uint64_t)(((j % NK) * C::KV_TILE) >> 4);
      const int b = sbuf(t, j);
      if (elect_one()) {
#pragma unroll
        for (int kk = 0; kk < D / 16; ++kk) {
          const uint32_t off = ((kk >> 2) * (AT_BM * 128) + (kk & 3) * 32) >> 4;
          umma_bf16_ss(tmem + b * 128, dq + off, dk + off, idesc_s, kk > 0);
        }
        umma_commit(&s_full[b]);
        if (t == 1 && !JOINT) umma_commit(&k_empty[j % NK]);
      }
      __syncwarp();
    };
    auto issue_pv = [&](int t, int j) {   // t == 0 waits for the V tile, t == 1 releases it
      const uint64_t dv = dv0 + (uint64_t)(((j % NV) * C::KV_TILE) >> 4);
      if (t == 0 && !JOINT) mbar_wait(&v_full[j % NV], (j / NV) & 1);
#ifdef TSV_ATTN_DEBUG
      if (!mbar_wait_bounded(tb(p_full, t, j), tpar(j), 1 << 22)) {
        if (lane == 0) printf("p_full hang: blk %d head %d t %d j %d\n", bid, head, t, j);
        __trap();
      }
#else
      mbar_wait(tb(p_full, t, j), tpar(j));
#endif
      tc_fence_after();
      if (elect_one()) {
        const int b = sbuf(t, j);
#pragma unroll
        for (int kk = 0; kk < AT_BN / 16; ++kk)
          umma_bf16_ts(tmem + C::O_COL + t * D, tmem + b * 128 + kk * 8, dv + (uint64_t)(kk * (2048 >> 4)), idesc_o,
                       (j | kk) != 0);
        if (RS) umma_commit(tb(pv_done, t, j));
        if (t == 1) umma_commit(JOINT ? &k_empty[j % NK] : &v_empty[j % NV]);
      }
      __syncwarp();
    };
    if constexpr (RS) {
      // S indices 0, 1, 2 up front; then each PV (S index m) is followed by S index m + 3, which
      // reuses the buffer that PV just read (the in-order tcgen05 pipe orders the two)
      auto s_at = [&](int m) {
        const int jj = m >> 1, tt = m & 1;
        if (jj >= n_tiles) return;
        if (tt == 0) {
          mbar_wait(&k_full[jj % NK], (jj / NK) & 1);
          tc_fence_after();
        }
        issue_s(tt, jj);
      };
      for (int m = 0; m < 3; ++m) s_at(m);
      for (int j = 0; j < n_tiles; ++j)
        for (int t = 0; t < 2; ++t) {
          issue_pv(t, j);
          if (j == n_tiles - 1) {
            if (elect_one()) umma_commit(&o_done[t]);
            __syncwarp();
          }
          s_at(2 * j + t + 3);
        }
    } else {
      for (int j = 0; j < n_tiles; ++j) {
        mbar_wait(&k_full[j % NK], (j / NK) & 1);
        tc_fence_after();
        for (int t = 0; t < 2; ++t) {
          if (j > 0) issue_pv(t, j - 1);
          issue_s(t, j);
        }
      }
      for (int t = 0; t < 2; ++t) {
        issue_pv(t, n_tiles - 1);
        if (elect_one()) umma_commit(&o_done[t]);
        __syncwarp();
      }
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
    auto hand_over = [&](int j) {   // P_t(j) is in TMEM: release it to the MMA warp
      tmem_st_wait();
      tc_fence_before();
      mbar_arrive(tb(p_full, t, j));   // (one arrival per warp after __syncwarp measured no faster)
    };
    for (int j = 0; j < n_tiles; ++j) {
      // this tile's S (and then P) buffer: its own, or (RS) buffer (2 j + t) % 3, used for the
      // ((2 j + t) / 3)-th time
      const int sb = RS ? (2 * j + t) % 3 : t;
      const uint32_t s_col = tmem + lane_base + sb * 128;
#ifdef TSV_ATTN_DEBUG
      if (!mbar_wait_bounded(&s_full[sb], (RS ? (2 * j + t) / 3 : j) & 1, 1 << 22)) {
        if (lane == 0) printf("s_full hang: blk %d head %d t %d j %d sb %d\n", bid, head, t, j, sb);
        __trap();
      }
#else
      mbar_wait(&s_full[sb], (RS ? (2 * j + t) / 3 : j) & 1);
#endif
      tc_fence_after();
      uint32_t sr[4][32];
      const int kbase = (j0 + j) * AT_BN;
      const bool full = kbase + AT_BN <= L;
      if (j > 0 && full) {
        // lazy path: no max before the exponentials, so the TMEM loads are pipelined with the
        // arithmetic (chunk c + 1 is in flight while chunk c is exponentiated)
        const float2 sc2 = make_float2(scale_log2, scale_log2), nm2 = make_float2(-m_ref, -m_ref);
        const float sat_a = scale_log2 * (1.0f / 190.0f), sat_b = (126.0f - m_ref) * (1.0f / 190.0f);
        float2 lz[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
        tmem_ld32(s_col, sr[0]);
        tmem_ld_wait_dep(sr[0]);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          if (c < 3) tmem_ld32(s_col + (c + 1) * 32, sr[c + 1]);
#pragma unroll
          for (int i = 0; i < 32; i += 2) {
            float2 p;
            if (PSAT && NPOLY != 9 && ((i >> 1) & 7) >= 8 - NPOLY) {
              p = poly_exp2_sat_x2<PSAT == 2 ? 2 : 3>(__uint_as_float(sr[c][i]), __uint_as_float(sr[c][i + 1]), sat_a,
                                                      sat_b);
              lz[(i >> 1) & 3] = __fadd2_rn(lz[(i >> 1) & 3], p);
              sr[c >> 1][(c & 1) * 16 + i / 2] = pack_bf16x2(p.x, p.y);
              continue;
            }
            float2 x = __ffma2_rn(make_float2(__uint_as_float(sr[c][i]), __uint_as_float(sr[c][i + 1])), sc2, nm2);
            if (NPOLY == 9) {
              p = x;   // diagnostic (impl 59): no exponential -- the pipeline's ceiling without softmax math
            } else if (((i >> 1) & 7) >= 8 - NPOLY) {
              // the polynomial path wraps the exponent field outside [-126, 127]: clamp both sides
              // (a clamped x > 64 still makes the sum exceed the limit)
              x.x = fminf(x.x, 64.f);
              x.y = fminf(x.y, 64.f);
              p = poly_exp2_x2(x);
            } else {
              p = make_float2(fast_exp2(x.x), fast_exp2(x.y));
            }
            lz[(i >> 1) & 3] = __fadd2_rn(lz[(i >> 1) & 3], p);
            // packed P overwrites consumed S: keys [64h, 64h + 64) land in sr[h]
            sr[c >> 1][(c & 1) * 16 + i / 2] = pack_bf16x2(p.x, p.y);
          }
          if (c < 3) tmem_ld_wait_dep(sr[c + 1]);
        }
        const float2 l01 = __fadd2_rn(lz[0], lz[1]), l23 = __fadd2_rn(lz[2], lz[3]);
        const float2 l4 = __fadd2_rn(l01, l23);
        const float ts = l4.x + l4.y;
        if (NPOLY == 9 || !__any_sync(0xffffffffu, !(ts <= LAZY_LIMIT))) {   // also catches inf / NaN
          l_sum += ts;
          tmem_st32(s_col, sr[0]);
          tmem_st32(s_col + 32, sr[1]);
          hand_over(j);
          continue;
        }
      }
      // exact path (first tile, the ragged last tile, or a lazy tile whose sum overflowed): reload
      // S, row max with 8 independent accumulators (one chain would be 128 dependent FMNMX)
#pragma unroll
      for (int c = 0; c < 4; ++c) tmem_ld32(s_col + c * 32, sr[c]);
      tmem_ld_wait();
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
        for (int i = 0; i < 32; i += 2) {   // all MUFU here (masked keys give ex2(-inf) = 0)
          const float p0 = fast_exp2(fmaf(__uint_as_float(sr[c][i]), scale_log2, neg_m));
          const float p1 = fast_exp2(fmaf(__uint_as_float(sr[c][i + 1]), scale_log2, neg_m));
          lsum[(i >> 1) & 3] = __fadd2_rn(lsum[(i >> 1) & 3], make_float2(p0, p1));
          sr[c >> 1][(c & 1) * 16 + i / 2] = pack_bf16x2(p0, p1);
        }
      if (__any_sync(0xffffffffu, rescale)) {
        // S_t(j) complete => PV_t(j-1) complete (in-order pipe): O_t can be rescaled now, before
        // P_t(j) is handed over.  RS issues S_t(j) ahead of PV_t(j-1), so it waits for PV_t(j-1)
        // explicitly (pv_done copy (j - 1) % 3; PV_t(j+2) cannot complete before P_t(j+2)).
        // tcgen05.ld/st are warp-collective: the whole warp's rows are rescaled together (alpha = 1
        // for rows that did not need it).
        if (RS) {
#ifdef TSV_ATTN_DEBUG
          if (!mbar_wait_bounded(tb(pv_done, t, j - 1), tpar(j - 1), 1 << 22)) {
            if (lane == 0) printf("RS pv_done hang: blk %d head %d t %d j %d\n", bid, head, t, j);
            __trap();
          }
#else
          mbar_wait(tb(pv_done, t, j - 1), tpar(j - 1));
#endif
          tc_fence_after();
        }
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
      hand_over(j);
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
    if (split) {
      // KV split: unnormalised O_t (layout [D][128]: coalesced across the warp's rows), reference m
      // and sum l of this split -> ws; the last split of these 32 rows merges in split order:
      // O = sum_s 2^(m_s - M) O_s / sum_s 2^(m_s - M) l_s, M = max_s m_s
      const size_t slab = (size_t)AT_BM * (D + 2);
      const size_t qt = (size_t)tail_u * 2 + t;   // query tile among the tail items'
      auto ws_at = [&](int s2) { return sa.ws + (qt * sa.nsplit + s2) * slab; };
      float* mine = ws_at(zr);
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

template <int D, int NP, int KV = 0, bool RS = false, int PS = 0>
static cudaError_t launch_fa(const CUtensorMap& tq, const CUtensorMap& tk, const CUtensorMap& tv, bf16* o,
                             long long ldo, int L, int H, float scale_log2, const AttnScatter& sc, cudaStream_t s,
                             const AttnSplitArgs& sa) {
  static unsigned long long done = 0;
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(done >> dev & 1ull)) {
    cudaError_t e = cudaFuncSetAttribute(attention_fa_kernel<D, NP, KV, RS, PS>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, FaCfg<D, KV, RS>::SMEM);
    if (e != cudaSuccess) return e;
    done |= 1ull << dev;
  }
  dim3 grid(sa.n_plain + sa.n_tail * (sa.nsplit > 1 ? sa.nsplit : 0));
  return launch_pdl(attention_fa_kernel<D, NP, KV, RS, PS>, grid, dim3(FA_THREADS), FaCfg<D, KV, RS>::SMEM, s, tq, tk, tv,
                    o, ldo, L, scale_log2, sc, sa);
}

// KV split for a launch of C = ceil(L/256) x H work items (one per head and 256 queries, one CTA per
// SM): the last T items (the tail) are split into S key ranges each, chosen by a list-scheduling
// model of the launch.  CTAs are dispatched in block order to the first free SM; a CTA costs its key
// tiles + a fixed cost (prologue, pipeline fill, epilogue: 2 tiles; + the merge when split: 6, fitted
// to tools/microbench.py attnsplit).  The whole items come first in equal waves (closed form), then
// the tail's S x T short CTAs fill the last wave's gaps.  T = C is the uniform split of round 1.
// E.g. FLUX 2048^2 at SP = 8 (198 items of 132 tiles on 148 SMs): all items halved costs 218 tiles of
// time, 148 whole + the last 50 in 5 ranges 200 (ideal 179).  TSV_KV_TAIL=0: uniform splits only.
static int KV_MIN_TILES = 4, KV_SPLIT_COST = 6, KV_TAIL = 1;   // TSV_KV_MIN / _COST / _TAIL (tuning)
static double KV_GAIN = 0.97;   // a split plan must beat the unsplit launch's modeled makespan by 3 % (TSV_KV_GAIN)
static double kv_makespan(long long n_plain, int plain_cost, long long T, const int* sz, int S, int sms, int fixed) {
  // n_plain equal CTAs first: q full rounds, r SMs one more; then the tail list-scheduled
  std::vector<double> h(sms);
  const long long q = n_plain / sms, r = n_plain % sms;
  for (int i = 0; i < sms; ++i) h[i] = (double)(q + (i < r ? 1 : 0)) * plain_cost;
  auto cmp = [](double x, double y) { return x > y; };
  std::make_heap(h.begin(), h.end(), cmp);
  for (int z = 0; z < S; ++z)
    for (long long c = 0; c < T; ++c) {
      std::pop_heap(h.begin(), h.end(), cmp);
      h.back() += sz[z] + fixed;
      std::push_heap(h.begin(), h.end(), cmp);
    }
  return *std::max_element(h.begin(), h.end());
}
static AttnSplitArgs plan_kv_split(int L, int H, int D, const AttnSplitWs* w, int sms_override = 0) {
  static bool env_read = false;
  if (!env_read) {
    if (const char* v = getenv("TSV_KV_MIN")) KV_MIN_TILES = atoi(v);
    if (const char* v = getenv("TSV_KV_COST")) KV_SPLIT_COST = atoi(v);
    if (const char* v = getenv("TSV_KV_TAIL")) KV_TAIL = atoi(v);
    if (const char* v = getenv("TSV_KV_GAIN")) KV_GAIN = atof(v);
    env_read = true;
  }
  const int n_all = (L + AT_BN - 1) / AT_BN;
  const int nqb = (L + 2 * AT_BM - 1) / (2 * AT_BM);
  const long long C = (long long)nqb * H;
  AttnSplitArgs a;
  a.n_plain = (int)C;
  a.nqb = nqb;
  if (!w || !w->cnt || !w->ws) return a;
  static int sms_of[64] = {0};
  int dev = 0;
  if (sms_override <= 0) {
    cudaGetDevice(&dev);
    if (!sms_of[dev & 63]) cudaDeviceGetAttribute(&sms_of[dev & 63], cudaDevAttrMultiProcessorCount, dev);
  }
  const int sms = sms_override > 0 ? sms_override : (sms_of[dev & 63] ? sms_of[dev & 63] : 148);
  // the workspace bounds the tail: T items x 2 query tiles x S ranges x (O, m, l) slabs; 4 counters each
  const long long slab = (long long)AT_BM * (D + 2) * 4;
  auto fits = [&](long long T, int S) { return T * 2 * S * slab <= w->ws_bytes && T * 2 * 4 <= w->cnt_ints; };
  long long bestT = 0;
  std::vector<int> sz;   // tiles per range (empty: no split)
  if (w->force > 0) {
    const int f = w->force < n_all ? w->force : n_all;
    const int tps = (n_all + f - 1) / f;
    for (int j = 0; j < n_all; j += tps) sz.push_back(std::min(tps, n_all - j));
    bestT = C;
  } else {
    // plans depend on (L, H, SMs, knobs) only: cached (each step graph captures a shape once anyway)
    static std::map<std::tuple<int, int, int, int, int, int, int>, std::pair<long long, std::vector<int>>> cache;
    static std::mutex cache_mu;   // launches may come from several host threads (one per engine / device)
    std::lock_guard<std::mutex> lock(cache_mu);
    const auto key = std::make_tuple(L, H, sms, KV_MIN_TILES, KV_SPLIT_COST, KV_TAIL, (int)(KV_GAIN * 1000));
    auto it = cache.find(key);
    if (it != cache.end()) {
      bestT = it->second.first;
      sz = it->second.second;
    } else {
      const double base = kv_makespan(C, n_all + 2, 0, nullptr, 0, sms, 0);
      double bestc = base;
      for (int S = 2; S <= 8; ++S) {
        const int eq = (n_all + S - 1) / S;
        if (eq < KV_MIN_TILES) break;
        int t[8];
        int left = n_all;
        for (int z = 0; z < S; ++z) { t[z] = std::min(eq, left); left -= t[z]; }
        if (t[S - 1] < 1) continue;
        // tails: every item (the uniform split), or up to three waves' worth of the last items
        const long long t_hi = KV_TAIL ? std::min<long long>(C, 3LL * sms) : 0;
        for (long long T = t_hi; T >= 0; --T) {
          const long long TT = T == 0 ? C : T;   // T = 0 encodes the uniform split (all C items)
          if (T == 0 && t_hi == C) break;        // already evaluated
          if (!fits(TT, S)) continue;
          const double c = kv_makespan(C - TT, n_all + 2, TT, t, S, sms, KV_SPLIT_COST);
          if (c < bestc && c < base * KV_GAIN) {
            bestc = c;
            bestT = TT;
            sz.assign(t, t + S);
          }
        }
      }
      cache[key] = std::make_pair(bestT, sz);
    }
  }
  const int best = (int)sz.size();
  if (best < 2 || best > 8 || bestT < 1 || !fits(bestT, best)) return a;
  a.nsplit = best;
  a.tps = *std::max_element(sz.begin(), sz.end());
  a.n_plain = (int)(C - bestT);
  a.n_tail = (int)bestT;
  a.bound[0] = 0;
  for (int z = 0; z < best; ++z) a.bound[z + 1] = a.bound[z] + sz[z];
  a.cnt = w->cnt;
  a.ws = w->ws;
  return a;
}

// host-only view of the planner (tsv_attention_split_plan): the plan a launch of (L, H, D) would use
int attention_split_plan(int L, int H, int D, long long ws_bytes, int cnt_ints, int force, int sms, int* n_plain,
                         int* n_tail, int* nsplit, int* bounds) {
  static float dummy_ws;
  static int dummy_cnt;
  AttnSplitWs w;
  w.cnt = &dummy_cnt;   // never dereferenced by the planner
  w.cnt_ints = cnt_ints;
  w.ws = &dummy_ws;
  w.ws_bytes = ws_bytes;
  w.force = force;
  const AttnSplitArgs a = plan_kv_split(L, H, D, &w, sms > 0 ? sms : 148);
  *n_plain = a.n_plain;
  *n_tail = a.n_tail;
  *nsplit = a.nsplit;
  for (int z = 0; z < 9; ++z) bounds[z] = a.bound[z];
  return 0;
}

// The step's variant per head dim (profiles/README.md, attention table); TSV_ATTN_D128 / TSV_ATTN_D64
// override it with any tsv_op_attention impl number (same-box A/B of whole steps).
static int default_version(int D) {
  static int v[2] = {-1, -1};
  int& r = v[D == 128];
  if (r < 0) {
    const char* e = getenv(D == 128 ? "TSV_ATTN_D128" : "TSV_ATTN_D64");
    // D = 128: separate K / V rings, 2 of 8 exp2 pairs by the saturating-FFMA cubic (impl 56); D = 64: the
    // joint ring (the split rings measured -2 % on the SD3 1024^2 step) with rotating S buffers, 3 of 8 by
    // the saturating-FFMA quadratic (impl 103).  Same-box step A/B (profiles/r02/ab_psat_l2hint.txt,
    // ab_l2last_d128psat.txt, ab_quad.txt): FLUX 2048^2 333.0 -> 330.4 ms vs impl 51 (the quadratic, 64:
    // -0.15 %, noise), SD3 2048^2 143.9 -> 140.6 ms (96) vs 92, 140.1 -> 137.7 ms (103) vs 96
    r = e ? atoi(e) : (D == 128 ? 56 : 103);
    if (r < 50 || r > 109) r = D == 128 ? 56 : 103;
  }
  return r;
}

template <int D>
static int launch_tc(const bf16* q, long long ldq, const bf16* k, long long ldk, const bf16* v, long long ldv, bf16* o,
                     long long ldo, int L, int H, int version, const AttnScatter& sc, cudaStream_t s,
                     const AttnSplitWs* spw) {
  CUtensorMap tq, tk, tv;
  if (make_tmap_heads(&tq, q, D, H, L, ldq) || make_tmap_heads(&tk, k, D, H, L, ldk) ||
      make_tmap_heads(&tv, v, D, H, L, ldv))
    return -1;
  const float scale_log2 = (1.0f / sqrtf((float)D)) * 1.4426950408889634f;
  const AttnSplitArgs sa = plan_kv_split(L, H, D, spw);
  cudaError_t e;
  // Kept variants (the step's defaults, their round-2 predecessors, diagnostics); the other sweep points
  // were removed after their measurements (profiles/README.md, profiles/r02/ab_*, mb_*).
  if constexpr (D == 64) {
    // rotating S buffers (RS) on the joint K+V ring: 92 = 2 of 8 exp2 pairs by the clamped cubic (round 2),
    // 96 = 3 of 8 by the saturating-FFMA cubic, 103 = 3 of 8 by the saturating-FFMA quadratic (default),
    // 99 = diagnostic without exponentials (wrong results: the pipeline's ceiling)
    switch (version) {
      case 92: return launch_fa<D, 2, 3, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa) == cudaSuccess ? 0 : -5;
      case 96: return launch_fa<D, 3, 3, true, 1>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa) == cudaSuccess ? 0 : -5;
      case 103: return launch_fa<D, 3, 3, true, 2>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa) == cudaSuccess ? 0 : -5;
      case 99: return launch_fa<D, 9, 3, true>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa) == cudaSuccess ? 0 : -5;
      default: break;
    }
  }
  // both head dims, one S buffer per query tile: 50 = all exp2 on MUFU, 51 = 1 of 8 pairs by the clamped
  // cubic (round 2's D = 128 default), 56 = 2 of 8 by the saturating-FFMA cubic (D = 128 default), 59 =
  // diagnostic without exponentials; 81 / 83 = the joint K+V ring (round 1's producer), 1 / 3 of 8
  switch (version) {
    case 50: e = launch_fa<D, 0>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
    case 51: e = launch_fa<D, 1>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
    case 56: e = launch_fa<D, 2, 0, false, 1>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
    case 59: e = launch_fa<D, 9>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
    case 81: e = launch_fa<D, 1, 3>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
    case 83: e = launch_fa<D, 3, 3>(tq, tk, tv, o, ldo, L, H, scale_log2, sc, s, sa); break;
    default: return -3;
  }
  return e == cudaSuccess ? 0 : -5;
}

// returns 0 if the kernel was launched; -1: layout unsupported by TMA (alignment), -3: unknown
// version, -4: bad scatter, -5: launch error (cudaGetLastError has it)
int attention_launch(const bf16* q, long long ldq, const bf16* k, long long ldk, const bf16* v, long long ldv,
                     bf16* o, long long ldo, int L, int H, int D, cudaStream_t s, int version,
                     const AttnScatter* scatter, const AttnSplitWs* split) {
  if (L <= 0 || H <= 0) return 0;
  AttnScatter sc;
  if (scatter) {
    sc = *scatter;
    if (sc.k < 1 || sc.k > 8) return -4;
  }
  if (((ldq | ldk | ldv) * 2) % 16 || ((reinterpret_cast<uintptr_t>(q) | reinterpret_cast<uintptr_t>(k) |
                                        reinterpret_cast<uintptr_t>(v)) & 15))
    return -1;
  if (version <= 3) version = default_version(D);
  if (D == 128) return launch_tc<128>(q, ldq, k, ldk, v, ldv, o, ldo, L, H, version, sc, s, split);
  if (D == 64) return launch_tc<64>(q, ldq, k, ldk, v, ldv, o, ldo, L, H, version, sc, s, split);
  return -1;
}

}  // namespace tsv
