// Joint text+image attention (S:§8(a) a6): O = softmax(q k^T / sqrt(D)) v, non-causal, exact
// max-subtracted online softmax (flash-attention recurrence) in fp32, bf16 operands.
//
// v1: warp-level mma.sync (m16n8k16) tiles, 64 queries per CTA (4 warps x 16 rows), 64-key
// K/V tiles double-buffered with cp.async into XOR-swizzled shared memory.  This is the first
// correct path; the tcgen05/TMEM attention is the planned replacement ("next").
#include <cfloat>

#include "kernels.h"
#include "ptx.cuh"

namespace tsv {

namespace {

constexpr int ATT_BQ = 64;   // queries per CTA
constexpr int ATT_BK = 64;   // keys per tile
constexpr int ATT_WARPS = 4;

__device__ __forceinline__ void cp_async16(uint32_t smem, const void* g, bool pred) {
  const int sz = pred ? 16 : 0;
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem), "l"(g), "r"(sz));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N)); }

__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void mma16816(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                         uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// row r, 16-byte chunk c of a tile whose rows hold NCH chunks; XOR swizzle by (r & 7)
template <int NCH>
__device__ __forceinline__ uint32_t swz(int r, int c) {
  return (uint32_t)(r * NCH * 16 + ((c ^ (r & 7)) * 16));
}

template <int D>
__device__ __forceinline__ void load_tile(uint32_t sbase, const bf16* g, long long ld, int row0, int L, int tid) {
  constexpr int NCH = D / 8;
  constexpr int TOTAL = ATT_BK * NCH;
#pragma unroll
  for (int i = tid; i < TOTAL; i += ATT_WARPS * 32) {
    const int r = i / NCH, c = i % NCH;
    const int gr = row0 + r;
    const bool ok = gr < L;
    const bf16* src = g + (long long)(ok ? gr : 0) * ld + c * 8;
    cp_async16(sbase + swz<NCH>(r, c), src, ok);
  }
}

}  // namespace

template <int D>
__global__ void __launch_bounds__(ATT_WARPS * 32) attention_mma_kernel(const bf16* __restrict__ q, long long ldq,
                                                                        const bf16* __restrict__ k, long long ldk,
                                                                        const bf16* __restrict__ v, long long ldv,
                                                                        bf16* __restrict__ o, long long ldo, int L,
                                                                        float scale_log2) {
  constexpr int NCH = D / 8;
  constexpr int TILE_BYTES = ATT_BK * D * 2;
  extern __shared__ __align__(128) uint8_t sm[];
  const uint32_t sQ = smem_u32(sm);
  const uint32_t sK = sQ + ATT_BQ * D * 2;           // 2 stages
  const uint32_t sV = sK + 2 * TILE_BYTES;           // 2 stages

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int head = blockIdx.y;
  const int q0 = blockIdx.x * ATT_BQ;
  const bf16* qh = q + head * D;
  const bf16* kh = k + head * D;
  const bf16* vh = v + head * D;

  // Q tile + first K/V tile
  load_tile<D>(sQ, qh, ldq, q0, L, tid);
  load_tile<D>(sK, kh, ldk, 0, L, tid);
  load_tile<D>(sV, vh, ldv, 0, L, tid);
  cp_async_commit();

  const int n_tiles = (L + ATT_BK - 1) / ATT_BK;
  uint32_t qf[D / 16][4];
  float acc[D / 8][4];
#pragma unroll
  for (int i = 0; i < D / 8; ++i) acc[i][0] = acc[i][1] = acc[i][2] = acc[i][3] = 0.f;
  float m_r[2] = {-FLT_MAX, -FLT_MAX}, l_r[2] = {0.f, 0.f};

  for (int t = 0; t < n_tiles; ++t) {
    const int st = t & 1;
    if (t + 1 < n_tiles) {
      load_tile<D>(sK + (st ^ 1) * TILE_BYTES, kh, ldk, (t + 1) * ATT_BK, L, tid);
      load_tile<D>(sV + (st ^ 1) * TILE_BYTES, vh, ldv, (t + 1) * ATT_BK, L, tid);
    }
    cp_async_commit();
    cp_async_wait<1>();
    __syncthreads();
    if (t == 0) {
#pragma unroll
      for (int kk = 0; kk < D / 16; ++kk) {
        const int r = warp * 16 + (lane & 15);
        const int c = 2 * kk + (lane >> 4);
        ldsm_x4(sQ + swz<NCH>(r, c), qf[kk][0], qf[kk][1], qf[kk][2], qf[kk][3]);
      }
    }
    const uint32_t kb = sK + st * TILE_BYTES, vb = sV + st * TILE_BYTES;
    // S = Q K^T  (16 x 64 per warp)
    float s[ATT_BK / 8][4];
#pragma unroll
    for (int j = 0; j < ATT_BK / 8; ++j) s[j][0] = s[j][1] = s[j][2] = s[j][3] = 0.f;
#pragma unroll
    for (int kk = 0; kk < D / 16; ++kk) {
#pragma unroll
      for (int jj = 0; jj < ATT_BK / 16; ++jj) {
        const int r = jj * 16 + (lane & 7) + ((lane >> 4) << 3);
        const int c = 2 * kk + ((lane >> 3) & 1);
        uint32_t b0, b1, b2, b3;
        ldsm_x4(kb + swz<NCH>(r, c), b0, b1, b2, b3);
        mma16816(s[2 * jj], qf[kk][0], qf[kk][1], qf[kk][2], qf[kk][3], b0, b1);
        mma16816(s[2 * jj + 1], qf[kk][0], qf[kk][1], qf[kk][2], qf[kk][3], b2, b3);
      }
    }
    // mask keys >= L, scale into log2 domain, online softmax
    const int key0 = t * ATT_BK;
    float mx[2] = {m_r[0], m_r[1]};
#pragma unroll
    for (int j = 0; j < ATT_BK / 8; ++j) {
      const int kc = key0 + j * 8 + 2 * (lane & 3);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int key = kc + (e & 1);
        float x = s[j][e] * scale_log2;
        if (key >= L) x = -INFINITY;
        s[j][e] = x;
        mx[e >> 1] = fmaxf(mx[e >> 1], x);
      }
    }
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      mx[i] = fmaxf(mx[i], __shfl_xor_sync(0xffffffffu, mx[i], 1));
      mx[i] = fmaxf(mx[i], __shfl_xor_sync(0xffffffffu, mx[i], 2));
    }
    float alpha[2], rs[2] = {0.f, 0.f};
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      alpha[i] = exp2f(m_r[i] - mx[i]);
      m_r[i] = mx[i];
    }
#pragma unroll
    for (int j = 0; j < ATT_BK / 8; ++j) {
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float p = exp2f(s[j][e] - mx[e >> 1]);
        s[j][e] = p;
        rs[e >> 1] += p;
      }
    }
#pragma unroll
    for (int i = 0; i < 2; ++i) l_r[i] = l_r[i] * alpha[i] + rs[i];
#pragma unroll
    for (int n = 0; n < D / 8; ++n) {
      acc[n][0] *= alpha[0]; acc[n][1] *= alpha[0];
      acc[n][2] *= alpha[1]; acc[n][3] *= alpha[1];
    }
    // O += P V
#pragma unroll
    for (int kk = 0; kk < ATT_BK / 16; ++kk) {
      const uint32_t a0 = pack_bf16x2(s[2 * kk][0], s[2 * kk][1]);
      const uint32_t a1 = pack_bf16x2(s[2 * kk][2], s[2 * kk][3]);
      const uint32_t a2 = pack_bf16x2(s[2 * kk + 1][0], s[2 * kk + 1][1]);
      const uint32_t a3 = pack_bf16x2(s[2 * kk + 1][2], s[2 * kk + 1][3]);
#pragma unroll
      for (int dd = 0; dd < D / 16; ++dd) {
        const int r = kk * 16 + (lane & 7) + (((lane >> 3) & 1) << 3);
        const int c = 2 * dd + (lane >> 4);
        uint32_t b0, b1, b2, b3;
        ldsm_x4_t(vb + swz<NCH>(r, c), b0, b1, b2, b3);
        mma16816(acc[2 * dd], a0, a1, a2, a3, b0, b1);
        mma16816(acc[2 * dd + 1], a0, a1, a2, a3, b2, b3);
      }
    }
    __syncthreads();
  }
  // finalize: quad-reduce row sums, normalise, store
#pragma unroll
  for (int i = 0; i < 2; ++i) {
    l_r[i] += __shfl_xor_sync(0xffffffffu, l_r[i], 1);
    l_r[i] += __shfl_xor_sync(0xffffffffu, l_r[i], 2);
    l_r[i] = 1.f / l_r[i];
  }
  const int r0 = q0 + warp * 16 + (lane >> 2);
#pragma unroll
  for (int n = 0; n < D / 8; ++n) {
    const int col = head * D + n * 8 + 2 * (lane & 3);
    if (r0 < L)
      *reinterpret_cast<uint32_t*>(o + (long long)r0 * ldo + col) = pack_bf16x2(acc[n][0] * l_r[0], acc[n][1] * l_r[0]);
    if (r0 + 8 < L)
      *reinterpret_cast<uint32_t*>(o + (long long)(r0 + 8) * ldo + col) =
          pack_bf16x2(acc[n][2] * l_r[1], acc[n][3] * l_r[1]);
  }
}

void attention_mma_launch(const bf16* q, long long ldq, const bf16* k, long long ldk, const bf16* v, long long ldv,
                      bf16* o, long long ldo, int L, int H, int D, cudaStream_t s) {
  if (L <= 0 || H <= 0) return;
  dim3 grid((L + ATT_BQ - 1) / ATT_BQ, H);
  const float scale_log2 = (1.0f / sqrtf((float)D)) * 1.4426950408889634f;
  if (D == 128) {
    const int smem = ATT_BQ * 128 * 2 + 4 * ATT_BK * 128 * 2;
    static unsigned long long done = 0;
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(done >> dev & 1ull)) {
      cudaFuncSetAttribute(attention_mma_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      done |= 1ull << dev;
    }
    attention_mma_kernel<128><<<grid, ATT_WARPS * 32, smem, s>>>(q, ldq, k, ldk, v, ldv, o, ldo, L, scale_log2);
  } else {
    const int smem = ATT_BQ * 64 * 2 + 4 * ATT_BK * 64 * 2;
    attention_mma_kernel<64><<<grid, ATT_WARPS * 32, smem, s>>>(q, ldq, k, ldk, v, ldv, o, ldo, L, scale_log2);
  }
}

}  // namespace tsv
