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
#include <cstdlib>
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
  static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/ + 4 * 32 * 36 * 4;
};

// Up to GEMM_MAX_PROBLEMS problems with the same N and K (e.g. the img and txt streams of a double
// block, times the two CFG branches for SD3) share one persistent launch: tiles
// [tile0[q], tile0[q+1]) belong to problem q.
struct GemmArgs {
  int N, K, num_n, num_tiles, nprob;
  // split-K (1-CTA tiles only): tile t = split s * tiles_per_split + t0 covers k-blocks
  // [s * kps, min(num_k, (s + 1) * kps)).  Each split stores its fp32 partial (per epilogue warp:
  // 32 rows x BN) into ws and counts itself in sem[4 t0 + warp]; the last to arrive sums the
  // partials in split order 0..splits-1 (deterministic whoever arrives last) and runs the epilogue.
  int splits, kps, tiles_per_split;
  int* sem;
  float* ws;
  int group_n, serpentine;   // rasterisation (decode_tile)
  int M[GEMM_MAX_PROBLEMS], num_m[GEMM_MAX_PROBLEMS], tile0[GEMM_MAX_PROBLEMS];
  GemmEpi epi[GEMM_MAX_PROBLEMS];
};
struct GemmMaps {
  CUtensorMap A[GEMM_MAX_PROBLEMS];
  CUtensorMap B[GEMM_MAX_PROBLEMS];
};
// > 4 KB of kernel parameters (CUDA 12.1+, up to 32 764 bytes)
static_assert(sizeof(GemmArgs) + sizeof(GemmMaps) <= 32764, "GEMM kernel parameters too large");

// Rasterisation: groups of group_n weight-column tiles; inside a group the n index varies fastest,
// then m.  A wave of 148 concurrent tiles therefore touches <= group_n weight tiles and
// ~148/group_n activation row-blocks, both L2-resident, so activations are streamed from HBM about
// num_n / group_n times instead of num_n times (measured: 2.8 GB -> algorithmic for 2048^2 fc1).
// serpentine: odd groups walk m backwards, so a group starts on the activation rows the previous
// group used last (still in L2) instead of on the evicted first rows.
__device__ __forceinline__ void decode_tile(const GemmArgs& a, int t, int& p, int& m_blk, int& n_blk) {
  p = 0;
#pragma unroll
  for (int q = 1; q < GEMM_MAX_PROBLEMS; ++q)
    if (q < a.nprob && t >= a.tile0[q]) p = q;
  const int lt = t - a.tile0[p];
  const int nm = a.num_m[p];
  const int G = a.group_n;
  const int group = lt / (G * nm);
  const int first_n = group * G;
  const int gsize = min(G, a.num_n - first_n);
  const int r = lt - group * G * nm;
  m_blk = r / gsize;
  if (a.serpentine && (group & 1)) m_blk = nm - 1 - m_blk;
  n_blk = first_n + r % gsize;
}

__device__ __forceinline__ void add_bias32(const bf16* bias, int n0, float (&v)[32]) {
  const uint4* bp = reinterpret_cast<const uint4*>(bias + n0);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    uint4 u = __ldg(bp + q);
    float2 f0 = unpack_bf16x2(u.x), f1 = unpack_bf16x2(u.y), f2 = unpack_bf16x2(u.z), f3 = unpack_bf16x2(u.w);
    v[q * 8 + 0] += f0.x; v[q * 8 + 1] += f0.y; v[q * 8 + 2] += f1.x; v[q * 8 + 3] += f1.y;
    v[q * 8 + 4] += f2.x; v[q * 8 + 5] += f2.y; v[q * 8 + 6] += f3.x; v[q * 8 + 7] += f3.y;
  }
}

__device__ __forceinline__ void store_bf16x32(bf16* ob, const float (&v)[32]) {
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
}

// Destination of one head block (columns [col0, col0 + D), head-aligned) of the QKV output:
// element (row, d) goes to base + rowmap(row) * stride + d.  Plain [M, ld0]; Ulysses pack
// [k][pack_rows][3][H/k][D]; or (fused a5) the owner's [L][3][H/k][D] at the row's global position.
// Computed once per head so the store loop has no integer divisions.
struct QkvDst {
  bf16* base;
  long long stride;
  int nt;             // rows < nt map to r0 + row, the rest to r1 + row - nt
  long long r0, r1;
  __device__ __forceinline__ bf16* at(int row) const {
    return base + (row < nt ? r0 + row : r1 + (row - nt)) * stride;
  }
};
__device__ __forceinline__ QkvDst qkv_head_dst(const GemmEpi& e, int col0) {
  QkvDst q;
  if (e.k_sp <= 1) {
    q.base = reinterpret_cast<bf16*>(e.out0) + col0;
    q.stride = e.ld0; q.nt = 1 << 30; q.r0 = 0; q.r1 = 0;
    return q;
  }
  const int h = e.qk_h, D = e.qk_D;
  const int part = col0 / h, hd = (col0 - part * h) / D;
  const int hk = h / D / e.k_sp;
  const int dst = hd / hk, hl = hd - dst * hk;
  q.stride = 3LL * hk * D;
  if (e.peer[0]) {
    q.base = e.peer[dst] + ((long long)part * hk + hl) * D;
    q.nt = e.peer_nt; q.r0 = e.peer_row0; q.r1 = e.peer_row1;
  } else {
    q.base = e.pack + ((long long)dst * e.pack_rows + e.pack_row0) * q.stride + ((long long)part * hk + hl) * D;
    q.nt = 1 << 30; q.r0 = 0; q.r1 = 0;
  }
  return q;
}

// ------------------------------------------------------------------ epilogue (coalesced via smem)
// A tcgen05.ld 32x32b chunk gives thread i the 32 columns of row i.  Writing those straight to
// global memory makes every warp store touch 32 rows (one 16-byte piece per row).  Instead each
// epilogue warp stages its 32 x 32 fp32 block in shared memory and re-reads it so that 8 lanes
// cover one row: every global load/store of the epilogue is a full 128-byte (fp32) or 64-byte
// (bf16) row segment.
constexpr int STG_PITCH = 36;                  // floats per staged row (16-byte aligned, spreads banks)
constexpr int STG_FLOATS = 32 * STG_PITCH;     // per epilogue warp
constexpr int STG_BYTES = 4 * STG_FLOATS * 4;  // 4 epilogue warps

__device__ __forceinline__ void stage_write(float* stg, int lane, const float (&v)[32]) {
  float4* rowp = reinterpret_cast<float4*>(stg + lane * STG_PITCH);
#pragma unroll
  for (int q = 0; q < 8; ++q) rowp[q] = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
}
__device__ __forceinline__ float4 stage_read(const float* stg, int rr, int c4) {
  return *reinterpret_cast<const float4*>(stg + rr * STG_PITCH + c4 * 4);
}
__device__ __forceinline__ uint2 pack4_bf16(float4 a) {
  return make_uint2(pack_bf16x2(a.x, a.y), pack_bf16x2(a.z, a.w));
}

// Fused a3 + a4: one thread = one row; a head of D columns is D/32 TMEM chunks.  Pass 1 sums the
// squares of y = acc + b over the head, pass 2 re-reads TMEM, computes RoPE(y * rsqrt(ms + eps) * g)
// per row and stores through the staging tile.  row0 = tile row of lane 0 of this warp.
__device__ __forceinline__ void epilogue_qk_head(const GemmEpi& e, int M, int row0, int col0, uint32_t tcol,
                                                 float* stg, int lane) {
  const int D = e.qk_D;
  const int row = row0 + lane;
  const bool norm = col0 < 2 * e.qk_h && e.gq != nullptr;
  float rn = 1.f;
  if (norm) {
    float ss = 0.f;
    for (int c = 0; c < D / 32; ++c) {
      uint32_t r[32];
      tmem_ld32(tcol + c * 32, r);
      tmem_ld_wait();
      float v[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
      if (e.bias) add_bias32(e.bias, col0 + c * 32, v);
#pragma unroll
      for (int i = 0; i < 32; ++i) ss += v[i] * v[i];
    }
    rn = rsqrtf(ss / (float)D + 1e-6f);
  }
  const bf16* g = col0 < e.qk_h ? e.gq : e.gk;
  const QkvDst qd = qkv_head_dst(e, col0);
  for (int c = 0; c < D / 32; ++c) {
    uint32_t r[32];
    tmem_ld32(tcol + c * 32, r);
    tmem_ld_wait();
    float v[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
    if (e.bias) add_bias32(e.bias, col0 + c * 32, v);
    if (norm && row < M) {
      const uint4* gp = reinterpret_cast<const uint4*>(g + c * 32);
      const float4* cp = reinterpret_cast<const float4*>(e.cosb + (long long)row * (D / 2) + c * 16);
      const float4* sp = reinterpret_cast<const float4*>(e.sinb + (long long)row * (D / 2) + c * 16);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint4 gu = __ldg(gp + q);
        float2 g0 = unpack_bf16x2(gu.x), g1 = unpack_bf16x2(gu.y), g2 = unpack_bf16x2(gu.z), g3 = unpack_bf16x2(gu.w);
        float gg[8] = {g0.x, g0.y, g1.x, g1.y, g2.x, g2.y, g3.x, g3.y};
        const float4 c4 = __ldg(cp + q), s4 = __ldg(sp + q);  // pairs 4q..4q+3 of this chunk
        const float cs[4] = {c4.x, c4.y, c4.z, c4.w}, sn[4] = {s4.x, s4.y, s4.z, s4.w};
#pragma unroll
        for (int p = 0; p < 4; ++p) {
          const float cc = cs[p], ss_ = sn[p];
          const float y0 = v[q * 8 + 2 * p] * rn * gg[2 * p], y1 = v[q * 8 + 2 * p + 1] * rn * gg[2 * p + 1];
          v[q * 8 + 2 * p] = cc * y0 - ss_ * y1;
          v[q * 8 + 2 * p + 1] = ss_ * y0 + cc * y1;
        }
      }
    }
    stage_write(stg, lane, v);
    __syncwarp();
    const int c4 = lane & 7;
#pragma unroll
    for (int it = 0; it < 8; ++it) {
      const int rr = it * 4 + (lane >> 3);
      if (row0 + rr < M)
        *reinterpret_cast<uint2*>(qd.at(row0 + rr) + c * 32 + c4 * 4) = pack4_bf16(stage_read(stg, rr, c4));
    }
    __syncwarp();
  }
}

// TMEM chunk (thread = row, 32 columns) -> row-coalesced layout through the warp's staging tile:
// a[it] = columns [4 c4, 4 c4 + 4) of row it * 4 + (lane >> 3), c4 = lane & 7.
__device__ __forceinline__ void stage_chunk(const uint32_t (&r)[32], float* stg, int lane, float4 (&a)[8]) {
  float v[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
  stage_write(stg, lane, v);
  __syncwarp();
#pragma unroll
  for (int it = 0; it < 8; ++it) a[it] = stage_read(stg, it * 4 + (lane >> 3), lane & 7);
  __syncwarp();  // the staging tile may be overwritten by the next chunk from here on
}

// epilogue of one 32 x 32 chunk in the staged layout (bias, activation / fp32-stream update, stores)
// this lane's 4 bias values of the chunk at column n0 (bf16 pairs; zero when the GEMM has no bias)
__device__ __forceinline__ uint2 load_bias4(const GemmEpi& e, int n0, int lane) {
  return e.bias ? __ldg(reinterpret_cast<const uint2*>(e.bias + n0 + (lane & 7) * 4)) : make_uint2(0u, 0u);
}
// bpre: the chunk's bias values when the caller prefetched them (load_bias4), else read here
__device__ __forceinline__ void finish_chunk(const GemmEpi& e, int M, int row0, int n0, float4 (&a)[8], int lane,
                                             const uint2* bpre = nullptr) {
  const int c4 = lane & 7;
  const int col = n0 + c4 * 4;  // this lane's 4 columns for all 8 row groups
  float4 b = make_float4(0.f, 0.f, 0.f, 0.f);
  if (e.bias) {
    const uint2 bu = bpre ? *bpre : __ldg(reinterpret_cast<const uint2*>(e.bias + col));
    const float2 b0 = unpack_bf16x2(bu.x), b1 = unpack_bf16x2(bu.y);
    b = make_float4(b0.x, b0.y, b1.x, b1.y);
  }
#pragma unroll
  for (int it = 0; it < 8; ++it) {
    a[it].x += b.x; a[it].y += b.y; a[it].z += b.z; a[it].w += b.w;
  }
  int mode = e.mode;
  bf16* ob = nullptr;
  long long ldb = e.ld0;
  if (mode == EPI_SPLIT_GELU) {  // n0 (and the whole 32-column chunk) is on one side of the split
    if (n0 >= e.n_split) {
      mode = EPI_GELU_BF16;
      ob = reinterpret_cast<bf16*>(e.out1) + (col - e.n_split);
      ldb = e.ld1;
    } else {
      mode = EPI_STORE_BF16;
      ob = reinterpret_cast<bf16*>(e.out0) + col;
    }
  } else if (mode <= EPI_SILU_BF16) {
    ob = reinterpret_cast<bf16*>(e.out0) + col;
  }
  const int rbase = row0 + (lane >> 3);
  if (mode <= EPI_SILU_BF16) {
#pragma unroll
    for (int it = 0; it < 8; ++it) {
      float4 y = a[it];
      if (mode == EPI_GELU_BF16) { y.x = gelu_tanh(y.x); y.y = gelu_tanh(y.y); y.z = gelu_tanh(y.z); y.w = gelu_tanh(y.w); }
      else if (mode == EPI_SILU_BF16) { y.x = silu(y.x); y.y = silu(y.y); y.z = silu(y.z); y.w = silu(y.w); }
      if (rbase + it * 4 < M) *reinterpret_cast<uint2*>(ob + (long long)(rbase + it * 4) * ldb) = pack4_bf16(y);
    }
    return;
  }
  float* out = reinterpret_cast<float*>(e.out0) + col;
  if (mode == EPI_STORE_F32) {
#pragma unroll
    for (int it = 0; it < 8; ++it)
      if (rbase + it * 4 < M) *reinterpret_cast<float4*>(out + (long long)(rbase + it * 4) * e.ld0) = a[it];
    return;
  }
  // read-modify-write of the fp32 stream: issue all 8 loads before any store (independent rows)
  float4 x[8];
#pragma unroll
  for (int it = 0; it < 8; ++it)
    x[it] = rbase + it * 4 < M ? __ldcg(reinterpret_cast<const float4*>(out + (long long)(rbase + it * 4) * e.ld0))
                               : make_float4(0.f, 0.f, 0.f, 0.f);   // L2: split-K partners write from other SMs
  float4 g = make_float4(1.f, 1.f, 1.f, 1.f);
  if (mode == EPI_RESID_GATE) g = __ldg(reinterpret_cast<const float4*>(e.gate + col));
  if (mode == EPI_CFG_EULER) {  // a = v_c; out1 holds v_u: a <- v_u + alpha (v_c - v_u)
    const float* vu = reinterpret_cast<const float*>(e.out1) + col;
#pragma unroll
    for (int it = 0; it < 8; ++it) {
      if (rbase + it * 4 >= M) continue;
      const float4 u = *reinterpret_cast<const float4*>(vu + (long long)(rbase + it * 4) * e.ld1);
      a[it] = make_float4(u.x + e.alpha * (a[it].x - u.x), u.y + e.alpha * (a[it].y - u.y),
                          u.z + e.alpha * (a[it].z - u.z), u.w + e.alpha * (a[it].w - u.w));
    }
  }
  if (mode == EPI_EULER || mode == EPI_CFG_EULER) {
    const float dt = *e.scalar;
    g = make_float4(dt, dt, dt, dt);
    if (e.out1) {
      float* vout = reinterpret_cast<float*>(e.out1) + col;
#pragma unroll
      for (int it = 0; it < 8; ++it)
        if (rbase + it * 4 < M) *reinterpret_cast<float4*>(vout + (long long)(rbase + it * 4) * e.ld1) = a[it];
    }
  }
#pragma unroll
  for (int it = 0; it < 8; ++it) {
    const float4 y = make_float4(x[it].x + g.x * a[it].x, x[it].y + g.y * a[it].y, x[it].z + g.z * a[it].z,
                                 x[it].w + g.w * a[it].w);
    if (rbase + it * 4 < M) *reinterpret_cast<float4*>(out + (long long)(rbase + it * 4) * e.ld0) = y;
  }
}

__device__ __forceinline__ void epilogue_chunk(const GemmEpi& e, int M, int row0, int n0, const uint32_t (&r)[32],
                                               float* stg, int lane) {
  float4 a[8];
  stage_chunk(r, stg, lane, a);
  finish_chunk(e, M, row0, n0, a, lane);
}

// split-K epilogue of one epilogue warp (32 rows x BN of one output tile): store the fp32 partial
// (row-coalesced) into its workspace slot; the last of the args.splits partials to arrive (counter
// per slot) sums them in split order 0..splits-1 and runs the tile's epilogue.  `slot` indexes the
// warp's rows inside the tile (nslot per tile); the counter is re-armed to 0 for the next launch.
template <int BN>
__device__ __forceinline__ void split_epilogue(const GemmArgs& args, const GemmEpi& epi, int Mp, int row0, int n_blk,
                                               uint32_t tbase, float* stg, int lane, int t0, int sp, int slot,
                                               int nslot) {
  const size_t part = (size_t)32 * BN;
  auto ws_at = [&](int s) { return args.ws + ((size_t)(s * args.tiles_per_split + t0) * nslot + slot) * part; };
  const int c4 = lane & 7;
  float* mine = ws_at(sp) + (size_t)(lane >> 3) * BN + c4 * 4;
#pragma unroll 1
  for (int c = 0; c < BN / 32; ++c) {
    uint32_t r[32];
    tmem_ld32(tbase + c * 32, r);
    tmem_ld_wait();
    float4 a[8];
    stage_chunk(r, stg, lane, a);
#pragma unroll
    for (int it = 0; it < 8; ++it) __stcg(reinterpret_cast<float4*>(mine + (size_t)it * 4 * BN + c * 32), a[it]);
  }
  __threadfence();
  __syncwarp();
  int* cnt = args.sem + t0 * nslot + slot;
  int done = 0;
  if (lane == 0) done = atomicAdd(cnt, 1);
  done = __shfl_sync(0xffffffffu, done, 0);
  if (done != args.splits - 1) return;
  __threadfence();
#pragma unroll 1
  for (int c = 0; c < BN / 32; c += 2) {   // two chunks per round: 16 independent L2 loads in flight
    float4 a[2][8];
#pragma unroll
    for (int h = 0; h < 2; ++h)
#pragma unroll
      for (int it = 0; it < 8; ++it) a[h][it] = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll 1
    for (int s2 = 0; s2 < args.splits; ++s2) {   // fixed order: deterministic whoever arrives last
      const float* src = ws_at(s2) + (size_t)(lane >> 3) * BN + c4 * 4 + c * 32;
      float4 u[2][8];
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int it = 0; it < 8; ++it) u[h][it] = __ldcg(reinterpret_cast<const float4*>(src + (size_t)it * 4 * BN + h * 32));
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int it = 0; it < 8; ++it) {
          a[h][it].x += u[h][it].x; a[h][it].y += u[h][it].y; a[h][it].z += u[h][it].z; a[h][it].w += u[h][it].w;
        }
    }
    finish_chunk(epi, Mp, row0, n_blk * BN + c * 32, a[0], lane);
    finish_chunk(epi, Mp, row0, n_blk * BN + (c + 1) * 32, a[1], lane);
  }
  if (lane == 0) *cnt = 0;   // re-armed for the next launch (the kernel boundary orders it)
}

// SPLITK: the split-K instantiation (args.splits > 1); the plain one compiles without any of it
template <int BN, bool SPLITK = false>
__global__ void __launch_bounds__(GEMM_THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ GemmMaps maps, const __grid_constant__ GemmArgs args) {
  using C = GemmCfg<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1 KB alignment by pointer arithmetic on the shared array (an integer round trip would make the
  // derived pointers generic: the epilogue's staging accesses compiled to LD.E / ST.E instead of LDS / STS)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
  uint64_t* full = bars;
  uint64_t* empty = bars + C::STAGES;
  uint64_t* tfull = bars + 2 * C::STAGES;
  uint64_t* tempty = bars + 2 * C::STAGES + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * C::STAGES + 4);
  float* stg_all = reinterpret_cast<float*>(smem + C::STAGES * C::STAGE_BYTES + 256);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int num_k = args.K / BK;

  if (warp == 0 && lane == 0) {
    for (int q = 0; q < args.nprob; ++q) {
      tma_prefetch_desc(&maps.A[q]);
      tma_prefetch_desc(&maps.B[q]);
    }
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
  // The weights (B) do not depend on the previous kernel: the first stages of the first tile are
  // requested before the programmatic-dependency wait, so their HBM latency overlaps the previous
  // kernel's tail.  A (and the fp32 stream) come from the previous kernel: after the wait.
  // split-K range of tile t
  auto krange = [&](int t, int& t0, int& s, int& kb0, int& kb1) {
    if (SPLITK) {
      s = t / args.tiles_per_split;
      t0 = t - s * args.tiles_per_split;
      kb0 = s * args.kps;
      kb1 = min(num_k, kb0 + args.kps);
    } else {
      s = 0; t0 = t; kb0 = 0; kb1 = num_k;
    }
  };
  int npre = 0;
  if (warp == 0 && lane == 0 && (int)blockIdx.x < args.num_tiles) {
    int pr, m_blk, n_blk, t0, sp, kb0, kb1;
    krange(blockIdx.x, t0, sp, kb0, kb1);
    decode_tile(args, t0, pr, m_blk, n_blk);
    npre = kb1 - kb0 < C::STAGES ? kb1 - kb0 : C::STAGES;
    for (int i = 0; i < npre; ++i) {
      mbar_arrive_expect_tx(&full[i], C::STAGE_BYTES);
      tma_load_2d(&maps.B[pr], &full[i], sB + i * C::B_BYTES, (kb0 + i) * BK, n_blk * BN);
    }
  }
  grid_dep_wait();

  if (warp == 0) {
    if (lane == 0) {
      // ---------------- TMA producer
      int stage = 0;
      uint32_t phase = 0;
      for (int t = blockIdx.x; t < args.num_tiles; t += gridDim.x) {
        int pr, m_blk, n_blk, t0, sp, kb0, kb1;
        krange(t, t0, sp, kb0, kb1);
        decode_tile(args, t0, pr, m_blk, n_blk);
        const CUtensorMap* tA = &maps.A[pr];
        const CUtensorMap* tB = &maps.B[pr];
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          const bool pre = t == (int)blockIdx.x && kb - kb0 < npre;   // B already requested
          if (!pre) mbar_arrive_expect_tx(&full[stage], C::STAGE_BYTES);
          tma_load_2d(tA, &full[stage], sA + stage * C::A_BYTES, kb * BK, m_blk * BM);
          if (!pre) tma_load_2d(tB, &full[stage], sB + stage * C::B_BYTES, kb * BK, n_blk * BN);
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issuer: the whole warp runs the loop (uniform registers), one elected
    // lane issues each k-step's MMAs back to back; descriptors = stage bases + constant offsets
    constexpr uint32_t idesc = make_idesc_bf16(BM, BN);
    const uint64_t da0 = make_sw128_desc(smem_u32(sA)), db0 = make_sw128_desc(smem_u32(sB));
    int stage = 0;
    uint32_t phase = 0;
    int it = 0;
    for (int t = blockIdx.x; t < args.num_tiles; t += gridDim.x, ++it) {
      int t0, sp, kb0, kb1;
      krange(t, t0, sp, kb0, kb1);
      const int acc = it & 1;
      const uint32_t acc_phase = (it >> 1) & 1;
      mbar_wait(&tempty[acc], acc_phase ^ 1);
      tc_fence_after();
      const uint32_t d_tmem = tmem_base + acc * BN;
      for (int kb = kb0; kb < kb1; ++kb) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        const uint64_t da = da0 + (uint64_t)((stage * C::A_BYTES) >> 4);
        const uint64_t db = db0 + (uint64_t)((stage * C::B_BYTES) >> 4);
        if (elect_one()) {
#pragma unroll
          for (int k = 0; k < BK / 16; ++k)
            umma_bf16_ss(d_tmem, da + 2 * k, db + 2 * k, idesc, (kb != kb0 || k != 0) ? 1u : 0u);
          umma_commit(&empty[stage]);
          if (kb == kb1 - 1) umma_commit(&tfull[acc]);
        }
        __syncwarp();
        if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
      }
    }
  } else if (warp >= 4) {
    // ---------------- epilogue: warp (4..7) owns TMEM lanes [32*(warp-4), +32)
    const int wq = warp - 4;
    float* stg = stg_all + wq * STG_FLOATS;
    int it = 0;
    for (int t = blockIdx.x; t < args.num_tiles; t += gridDim.x, ++it) {
      int pr, m_blk, n_blk, t0, sp, kb0, kb1;
      krange(t, t0, sp, kb0, kb1);
      decode_tile(args, t0, pr, m_blk, n_blk);
      const GemmEpi& epi = args.epi[pr];
      const int Mp = args.M[pr];
      const int acc = it & 1;
      const uint32_t acc_phase = (it >> 1) & 1;
      // plain epilogues: the first chunk's bias is loaded while the MMAs still run, each next chunk's
      // while the current one is finished (the load latency sat in front of every chunk)
      uint2 bnext = make_uint2(0u, 0u);
      if (!SPLITK) bnext = load_bias4(epi, n_blk * BN, lane);
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int row0 = m_blk * BM + wq * 32;
      const uint32_t tbase = tmem_base + ((uint32_t)(wq * 32) << 16) + acc * BN;
      if (SPLITK) {
        split_epilogue<BN>(args, epi, Mp, row0, n_blk, tbase, stg, lane, t0, sp, wq, 4);
      } else if (epi.qk_h > 0 && n_blk * BN < 3 * epi.qk_h) {
#pragma unroll 1
        for (int hd = 0; hd < BN / epi.qk_D; ++hd)
          epilogue_qk_head(epi, Mp, row0, n_blk * BN + hd * epi.qk_D, tbase + hd * epi.qk_D, stg, lane);
      } else {
#pragma unroll 1
        for (int c = 0; c < BN / 32; ++c) {
          uint32_t r[32];
          tmem_ld32(tbase + c * 32, r);
          const uint2 bcur = bnext;
          if (c + 1 < BN / 32) bnext = load_bias4(epi, n_blk * BN + (c + 1) * 32, lane);
          tmem_ld_wait();
          float4 a[8];
          stage_chunk(r, stg, lane, a);
          finish_chunk(epi, Mp, row0, n_blk * BN + c * 32, a, lane, &bcur);
        }
      }
      tc_fence_before();
      mbar_arrive(&tempty[acc]);
    }
  }
  grid_dep_launch();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc<C::TMEM_COLS>(tmem_base);
}

// ------------------------------------------------------------------ CTA-pair (cta_group::2) variant
// A cluster of 2 CTAs on one TPC computes a 256 x 256 tile: CTA r loads rows [128r, 128r+128) of the
// A tile and rows [128r, 128r+128) of the B (weight) tile; the even CTA issues
// tcgen05.mma.cta_group::2 (M = 256, N = 256), which reads A and B from both CTAs' shared memory
// at the same offsets and leaves CTA r's 128 output rows in CTA r's TMEM.  Per SM this halves the
// operand bytes read from shared memory per MMA compared with the 1-CTA 128 x 256 tile.
template <int BN_>
struct Gemm2Cfg {
  static constexpr int BN = BN_;
  static constexpr int A_BYTES = 128 * BK * 2;
  static constexpr int B_BYTES = (BN / 2) * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = BN == 256 ? 6 : 8;
  static constexpr int TMEM_COLS = 2 * BN;
  static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 + 256 + 4 * 32 * 36 * 4;
};

template <int BN_, bool SPLITK = false>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(GEMM_THREADS, 1)
    gemm_tc2_kernel(const __grid_constant__ GemmMaps maps, const __grid_constant__ GemmArgs args) {
  using C = Gemm2Cfg<BN_>;
  constexpr int BN = C::BN;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1 KB alignment by pointer arithmetic on the shared array (an integer round trip would make the
  // derived pointers generic: the epilogue's staging accesses compiled to LD.E / ST.E instead of LDS / STS)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
  uint64_t* full = bars;
  uint64_t* empty = bars + C::STAGES;
  uint64_t* tfull = bars + 2 * C::STAGES;
  uint64_t* tempty = bars + 2 * C::STAGES + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * C::STAGES + 4);
  float* stg_all = reinterpret_cast<float*>(smem + C::STAGES * C::STAGE_BYTES + 256);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;
  const int cid = blockIdx.x >> 1, ncl = gridDim.x >> 1;
  const int num_k = args.K / BK;

  if (warp == 0 && lane == 0) {
    for (int q = 0; q < args.nprob; ++q) {
      tma_prefetch_desc(&maps.A[q]);
      tma_prefetch_desc(&maps.B[q]);
    }
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&tfull[i], 1);
      mbar_init(&tempty[i], 2 * 128);  // both CTAs' epilogue threads drain before reuse
    }
    fence_mbar_init();
  }
  if (warp == 2) tmem_alloc_pair<C::TMEM_COLS>(tmem_slot);
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  // weights of the first stages before the programmatic-dependency wait (see gemm_tc_kernel)
  auto krange = [&](int t, int& t0, int& s, int& kb0, int& kb1) {   // split-K range (see GemmArgs)
    if (SPLITK) {
      s = t / args.tiles_per_split;
      t0 = t - s * args.tiles_per_split;
      kb0 = s * args.kps;
      kb1 = min(num_k, kb0 + args.kps);
    } else {
      s = 0; t0 = t; kb0 = 0; kb1 = num_k;
    }
  };
  int npre = 0;
  if (warp == 0 && lane == 0 && cid < args.num_tiles) {
    int pr, m_blk, n_blk, t0, sp, kb0, kb1;
    krange(cid, t0, sp, kb0, kb1);
    decode_tile(args, t0, pr, m_blk, n_blk);
    npre = kb1 - kb0 < C::STAGES ? kb1 - kb0 : C::STAGES;
    for (int i = 0; i < npre; ++i) {
      if (leader) mbar_arrive_expect_tx(&full[i], 2 * C::STAGE_BYTES);
      tma_load_2d_pair(&maps.B[pr], &full[i], sB + i * C::B_BYTES, (kb0 + i) * BK, n_blk * BN + (int)rank * (BN / 2));
    }
  }
  grid_dep_wait();  // A (and the fp32 stream) come from the previous kernel

  if (warp == 0) {
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      for (int t = cid; t < args.num_tiles; t += ncl) {
        int pr, m_blk, n_blk, t0, sp, kb0, kb1;
        krange(t, t0, sp, kb0, kb1);
        decode_tile(args, t0, pr, m_blk, n_blk);
        const CUtensorMap* tA = &maps.A[pr];
        const CUtensorMap* tB = &maps.B[pr];
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          const bool pre = t == cid && kb - kb0 < npre;   // B already requested
          if (leader && !pre) mbar_arrive_expect_tx(&full[stage], 2 * C::STAGE_BYTES);
          tma_load_2d_pair(tA, &full[stage], sA + stage * C::A_BYTES, kb * BK, m_blk * 256 + (int)rank * 128);
          if (!pre)
            tma_load_2d_pair(tB, &full[stage], sB + stage * C::B_BYTES, kb * BK, n_blk * BN + (int)rank * (BN / 2));
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (leader) {
      // MMA issuer of the pair (even CTA): whole warp in the loop, one elected lane issues
      constexpr uint32_t idesc = make_idesc_bf16(256, BN);
      const uint64_t da0 = make_sw128_desc(smem_u32(sA)), db0 = make_sw128_desc(smem_u32(sB));
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int t = cid; t < args.num_tiles; t += ncl, ++it) {
        int t0, sp, kb0, kb1;
        krange(t, t0, sp, kb0, kb1);
        const int acc = it & 1;
        const uint32_t acc_phase = (it >> 1) & 1;
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint64_t da = da0 + (uint64_t)((stage * C::A_BYTES) >> 4);
          const uint64_t db = db0 + (uint64_t)((stage * C::B_BYTES) >> 4);
          if (elect_one()) {
#pragma unroll
            for (int k = 0; k < BK / 16; ++k)
              umma_bf16_ss_pair(d_tmem, da + 2 * k, db + 2 * k, idesc, (kb != kb0 || k != 0) ? 1u : 0u);
            umma_commit_pair(&empty[stage]);
            if (kb == kb1 - 1) umma_commit_pair(&tfull[acc]);
          }
          __syncwarp();
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp >= 4) {
    const int wq = warp - 4;
    float* stg = stg_all + wq * STG_FLOATS;
    int it = 0;
    for (int t = cid; t < args.num_tiles; t += ncl, ++it) {
      int pr, m_blk, n_blk, t0, sp, kb0, kb1;
      krange(t, t0, sp, kb0, kb1);
      decode_tile(args, t0, pr, m_blk, n_blk);
      const GemmEpi& epi = args.epi[pr];
      const int Mp = args.M[pr];
      const int acc = it & 1;
      const uint32_t acc_phase = (it >> 1) & 1;
      // plain epilogues: bias prefetched one chunk ahead (see gemm_tc_kernel)
      uint2 bnext = make_uint2(0u, 0u);
      if (!SPLITK) bnext = load_bias4(epi, n_blk * BN, lane);
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int row0 = m_blk * 256 + (int)rank * 128 + wq * 32;
      const uint32_t tbase = tmem_base + ((uint32_t)(wq * 32) << 16) + acc * BN;
      if (SPLITK) {
        split_epilogue<BN>(args, epi, Mp, row0, n_blk, tbase, stg, lane, t0, sp, (int)rank * 4 + wq, 8);
      } else if (epi.qk_h > 0 && n_blk * BN < 3 * epi.qk_h) {
#pragma unroll 1
        for (int hd = 0; hd < BN / epi.qk_D; ++hd)
          epilogue_qk_head(epi, Mp, row0, n_blk * BN + hd * epi.qk_D, tbase + hd * epi.qk_D, stg, lane);
      } else {
#pragma unroll 1
        for (int c = 0; c < BN / 32; ++c) {
          uint32_t r[32];
          tmem_ld32(tbase + c * 32, r);
          const uint2 bcur = bnext;
          if (c + 1 < BN / 32) bnext = load_bias4(epi, n_blk * BN + (c + 1) * 32, lane);
          tmem_ld_wait();
          float4 a[8];
          stage_chunk(r, stg, lane, a);
          finish_chunk(epi, Mp, row0, n_blk * BN + c * 32, a, lane, &bcur);
        }
      }
      tc_fence_before();
      mbar_arrive_remote(&tempty[acc], 0);
    }
  }
  grid_dep_launch();
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  if (warp == 2) tmem_dealloc_pair<C::TMEM_COLS>(tmem_base);
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

static const char* check_epi(const GemmEpi& epi, int bn) {
  if (epi.mode == EPI_CFG_EULER && (!epi.out1 || !epi.scalar)) return "gemm: CFG Euler needs v_u (out1) and dt";
  if (!epi.qk_h) return nullptr;
  if (epi.qk_D != 64 && epi.qk_D != 128) return "gemm: fused QK-norm needs D in {64, 128}";
  if (bn % epi.qk_D || epi.qk_h % epi.qk_D || (epi.qk_h / epi.qk_D) % epi.k_sp)
    return "gemm: fused QK-norm needs D | BN, D | h and k_sp | heads";
  if (epi.mode != EPI_STORE_BF16 && epi.mode != EPI_SPLIT_GELU) return "gemm: fused QK-norm needs a bf16 store";
  if (epi.mode == EPI_SPLIT_GELU && epi.n_split != 3 * epi.qk_h) return "gemm: split must be at 3h";
  if (epi.gq && (!epi.gk || !epi.cosb || !epi.sinb)) return "gemm: fused QK-norm needs both gains and RoPE tables";
  if (!epi.gq && epi.k_sp <= 1) return "gemm: a QKV epilogue without norm needs k_sp > 1 (else a plain store)";
  if (epi.k_sp > 1 && !epi.pack && !epi.peer[0]) return "gemm: the Ulysses pack needs the pack buffer or peer buffers";
  if (epi.peer[0]) {
    if (epi.k_sp > 8) return "gemm: at most 8 peers";
    for (int d = 0; d < epi.k_sp; ++d)
      if (!epi.peer[d]) return "gemm: missing peer buffer";
  }
  return nullptr;
}

int gemm_plan_multi(GemmPlan* p, const GemmProblem* probs, int nprob, int N, int K, int num_sms, const char** err,
                    int force_bn, int force_pair, const GemmSplitWs* sws, int force_splits) {
  *err = nullptr;
  p->splits = 1; p->kps = K / BK; p->sem = nullptr; p->ws = nullptr;
  // Split-K for launches too small to fill the GPU (small M: the text stream, SP = 4/8 shards,
  // 256^2 / 512^2 at k >= 2): the splits' fp32 partials are summed by the last split, which then
  // runs the ordinary epilogue, so any epilogue but the fused QK-norm / RoPE / pack one qualifies.
  // Few tiles otherwise leave most SMs idle while the weights stream through a handful of them
  // (each SM pulls ~64 B/clk from L2: a weight-streaming GEMM needs most of the 148 SMs).
  bool split_ok = sws != nullptr && sws->sem && sws->ws;
  for (int q = 0; q < nprob && split_ok; ++q)
    split_ok = !probs[q].epi.qk_h;   // the last split runs the tile's ordinary epilogue (any mode but the
                                     // fused QK-norm / RoPE / pack one) on the summed partials
  if (N <= 0 || K <= 0) { *err = "gemm: empty shape"; return -1; }
  if (K % BK) { *err = "gemm: K must be a multiple of 64"; return -1; }
  if (N % 64) { *err = "gemm: N must be a multiple of 64"; return -1; }
  long long nm_total = 0;
  int qk_D = 0;
  for (int q = 0; q < nprob; ++q) {
    const GemmProblem& g = probs[q];
    if (g.M <= 0) { *err = "gemm: empty problem"; return -1; }
    if ((g.lda * 2) % 16 || (g.ldw * 2) % 16) { *err = "gemm: row strides must be 16-byte multiples"; return -1; }
    if ((reinterpret_cast<uintptr_t>(g.A) | reinterpret_cast<uintptr_t>(g.W)) & 15) {
      *err = "gemm: operands must be 16-byte aligned"; return -1;
    }
    nm_total += (g.M + BM - 1) / BM;
    if (g.epi.qk_h) qk_D = g.epi.qk_D > qk_D ? g.epi.qk_D : qk_D;
  }
  int bn = force_bn;
  if (!bn) {
    // Widest tile: measured on B200 (tools/microbench.py), 128x256 beats 128x128 even at 0.65
    // waves (e.g. 1024x3072x12288: 968 vs 768 TFLOP/s) — narrower tiles are smem-bandwidth bound.
    (void)nm_total;
    bn = (N % 256 == 0) ? 256 : (N % 128 == 0 ? 128 : 64);
    if (bn < qk_D) bn = qk_D;  // a head must sit inside one tile
  }
  if (N % bn) { *err = "gemm: N not a multiple of the tile width"; return -1; }
  int maxM = 0;
  for (int q = 0; q < nprob; ++q) maxM = probs[q].M > maxM ? probs[q].M : maxM;
  // CTA pairs (256 x 256 tiles, cta_group::2): faster per tile (half the smem operand traffic per
  // SM) but half as many tiles.  Measured (tools/microbench.py): pairs win for long K (>= 8192) or
  // when the pair tiles still fill ~half the SM pairs; e.g. 1024x3072x3072 (48 pair tiles) is
  // faster as 96 single-CTA tiles.
  long long pair_tiles = 0;
  for (int q = 0; q < nprob; ++q) pair_tiles += (long long)((probs[q].M + 255) / 256) * (N / 256);
  const bool pair_auto = bn == 256 && maxM > 128 && (K >= 8192 || pair_tiles * 2 >= (long long)num_sms * 9 / 10);
  bool pair = force_pair >= 0 ? (force_pair > 0 && bn >= 128) : pair_auto;
  if (force_pair < 0 && !force_bn && bn == 256 && maxM > 128 && qk_D <= 128) {
    // 256 x 128 pair tiles vs the choice above.  Per-SM time ~ waves * K * BN * e + E (one epilogue
    // and pipeline fill not overlapped), fitted to tools/microbench.py after the warp-wide MMA
    // issue: e = 1 (256-wide tiles) / 1.2 (128-wide), E = 420k / 210k.  E.g. 1536x3072x3072
    // 836 vs 745 TFLOP/s and 576x3072x3072 644 vs 453 (128 wins: two tiles per pair overlap the
    // epilogue), 1536x3072x15360 1537 vs 1399 (256 wins: one full wave, long K).
    long long single_tiles = 0;
    for (int q = 0; q < nprob; ++q) single_tiles += (long long)((probs[q].M + BM - 1) / BM) * (N / 256);
    const long long pairs = num_sms / 2;
    const double c_pair256 = (double)((pair_tiles + pairs - 1) / pairs) * K * 256.0 + 420e3;
    const double c_single = (double)((single_tiles + num_sms - 1) / num_sms) * K * 256.0 + 420e3;
    const double c_pair128 = (double)((2 * pair_tiles + pairs - 1) / pairs) * K * 128.0 * 1.2 + 210e3;
    if (c_pair128 < (pair ? c_pair256 : c_single)) {
      bn = 128;
      pair = true;
    }
  }
  const int bm = pair ? 256 : BM;
  p->nprob = nprob; p->N = N; p->K = K; p->BN = bn; p->pair = pair;
  // TSV_GEMM_GROUP / TSV_GEMM_SERP (read once): rasterisation A/B (tools/ab_*.sh)
  static int env_group = -1, env_serp = -1;
  if (env_group < 0) {
    const char* g = getenv("TSV_GEMM_GROUP");
    const char* sp = getenv("TSV_GEMM_SERP");
    env_group = g ? atoi(g) : 0;
    env_serp = sp ? atoi(sp) : 1;
  }
  p->group_n = env_group > 0 ? env_group : 16;   // r02 sweep (profiles/r02): 16 + serpentine, -17 % DRAM bytes at 2048^2
  p->serpentine = env_serp;
  int tiles = 0;
  for (int q = 0; q < nprob; ++q) {
    const GemmProblem& g = probs[q];
    if ((*err = check_epi(g.epi, bn))) return -1;
    p->Mq[q] = g.M;
    p->epiq[q] = g.epi;
    p->tile0[q] = tiles;
    tiles += ((g.M + bm - 1) / bm) * (N / bn);
    if (make_tmap_2d(&p->tmAq[q], g.A, K, g.M, g.lda * 2, BK, BM)) { *err = "gemm: cuTensorMapEncodeTiled(A) failed"; return -1; }
    if (make_tmap_2d(&p->tmBq[q], g.W, K, N, g.ldw * 2, BK, pair ? bn / 2 : bn)) {
      *err = "gemm: cuTensorMapEncodeTiled(W) failed"; return -1;
    }
  }
  p->tiles = tiles;
  if (pair) {
    const int clusters = tiles < num_sms / 2 ? tiles : num_sms / 2;
    p->grid = 2 * clusters;
  } else {
    p->grid = tiles < num_sms ? tiles : num_sms;
  }
  p->M = probs[0].M;
  p->epi = probs[0].epi;
  int want_splits = 1;
  if (split_ok) {
    const int num_k = K / BK;
    const long long units = pair ? num_sms / 2 : num_sms;   // clusters or CTAs
    if (force_splits > 0) {
      want_splits = force_splits;
    } else if (tiles * 2 <= units) {
      // measured (tools/microbench.py split, SPLIT_SWEEP): CTA pairs are best filling the SM pairs
      // once (S = 3 for 24 pair tiles), 1-CTA tiles at about half the SMs (S = 6 for 12 tiles):
      // beyond that the partial-sum traffic and the in-order reduction cost more than they give
      want_splits = (int)(pair ? units / tiles : units / (2 * tiles));
      if (want_splits > num_k / 4) want_splits = num_k / 4;   // >= 256 of K per split
      if (want_splits > 6) want_splits = 6;
    }
    const long long per_split = (long long)tiles * bm * bn * 4;   // fp32 partials
    if (want_splits * per_split > sws->ws_bytes) want_splits = (int)(sws->ws_bytes / per_split);
    if ((long long)tiles * (pair ? 8 : 4) > sws->sem_ints) want_splits = 1;
  }
  if (want_splits > 1) {
    const int num_k = K / BK;
    int kps = (num_k + want_splits - 1) / want_splits;
    if (kps < 1) kps = 1;
    p->splits = (num_k + kps - 1) / kps;
    p->kps = kps;
    if (p->splits > 1) {
      p->sem = sws->sem;
      p->ws = sws->ws;
      p->tiles = tiles * p->splits;
      if (pair) {
        const int clusters = p->tiles < num_sms / 2 ? p->tiles : num_sms / 2;
        p->grid = 2 * clusters;
      } else {
        p->grid = p->tiles < num_sms ? p->tiles : num_sms;
      }
    } else {
      p->splits = 1;
      p->kps = num_k;
    }
  }
  return 0;
}

int gemm_plan(GemmPlan* p, const bf16* A, long long lda, const bf16* W, long long ldw, int M, int N, int K,
              const GemmEpi& epi, int num_sms, const char** err, int force_bn, int force_pair, const GemmSplitWs* sws,
              int force_splits) {
  GemmProblem g{A, lda, W, ldw, M, epi};
  return gemm_plan_multi(p, &g, 1, N, K, num_sms, err, force_bn, force_pair, sws, force_splits);
}

template <int BN>
static void launch_bn(const GemmPlan& p, cudaStream_t s) {
  using C = GemmCfg<BN>;
  static unsigned long long attr_done = 0;  // one bit per device
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(attr_done >> dev & 1ull)) {
    cudaFuncSetAttribute(gemm_tc_kernel<BN, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM_BYTES);
    cudaFuncSetAttribute(gemm_tc_kernel<BN, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM_BYTES);
    attr_done |= 1ull << dev;
  }
  const bool sk = p.splits > 1;
  GemmArgs a;
  GemmMaps maps;
  const int bm = p.pair ? 256 : BM;
  a.N = p.N; a.K = p.K; a.num_n = p.N / BN; a.num_tiles = p.tiles; a.nprob = p.nprob;
  a.splits = p.splits; a.kps = p.kps; a.tiles_per_split = p.tiles / p.splits; a.sem = p.sem; a.ws = p.ws;
  a.group_n = p.group_n; a.serpentine = p.serpentine;
  for (int q = 0; q < GEMM_MAX_PROBLEMS; ++q) {
    const int qq = q < p.nprob ? q : 0;
    a.M[q] = p.Mq[qq];
    a.num_m[q] = (p.Mq[qq] + bm - 1) / bm;
    a.tile0[q] = p.tile0[qq];
    a.epi[q] = p.epiq[qq];
    maps.A[q] = p.tmAq[qq];
    maps.B[q] = p.tmBq[qq];
  }
  if constexpr (BN >= 128) {
    if (p.pair) {
      static unsigned long long attr2 = 0;
      if (!(attr2 >> dev & 1ull)) {
        cudaFuncSetAttribute(gemm_tc2_kernel<BN, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             Gemm2Cfg<BN>::SMEM_BYTES);
        cudaFuncSetAttribute(gemm_tc2_kernel<BN, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             Gemm2Cfg<BN>::SMEM_BYTES);
        attr2 |= 1ull << dev;
      }
      if (sk) launch_pdl(gemm_tc2_kernel<BN, true>, dim3(p.grid), dim3(GEMM_THREADS), Gemm2Cfg<BN>::SMEM_BYTES, s, maps, a);
      else launch_pdl(gemm_tc2_kernel<BN, false>, dim3(p.grid), dim3(GEMM_THREADS), Gemm2Cfg<BN>::SMEM_BYTES, s, maps, a);
      return;
    }
  }
  // 1-CTA tiles (the only variant for 64-wide tiles: gemm_plan never pairs them)
  if (sk) launch_pdl(gemm_tc_kernel<BN, true>, dim3(p.grid), dim3(GEMM_THREADS), C::SMEM_BYTES, s, maps, a);
  else launch_pdl(gemm_tc_kernel<BN, false>, dim3(p.grid), dim3(GEMM_THREADS), C::SMEM_BYTES, s, maps, a);
}

void gemm_launch(const GemmPlan& p, cudaStream_t s) {
  switch (p.BN) {
    case 256: launch_bn<256>(p, s); break;
    case 128: launch_bn<128>(p, s); break;
    default: launch_bn<64>(p, s); break;
  }
}

}  // namespace tsv
