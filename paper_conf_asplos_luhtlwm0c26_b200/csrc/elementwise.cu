// HBM-bound kernels of the step (S:§8(a) a2, a4, Ulysses pack/unpack) plus the SYNTH-1 generator.
// Vectorised 16-byte accesses, one warp per row (LN) or per (row, head) (QK-norm + RoPE).
#include "kernels.h"
#include "ptx.cuh"

namespace tsv {

// ------------------------------------------------------------------ a2: LN-modulate
// u = LN(x) (no affine, biased variance, eps 1e-6) * (1 + scale) + shift   -> bf16
// One CTA of T threads per row, NV float4 per thread (h = 4 * T * NV): the row stays in registers,
// two block reductions (mean, then centred sum of squares), ~10 CTAs resident per SM.
template <int T>
__device__ __forceinline__ float block_sum(float v, float* red) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (T == 32) return v;
  const int w = threadIdx.x >> 5;
  __syncthreads();  // red[] reuse
  if ((threadIdx.x & 31) == 0) red[w] = v;
  __syncthreads();
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < T / 32; ++i) s += red[i];
  return s;
}

template <int T, int NV>
__global__ void __launch_bounds__(T) ln_mod_kernel(const float* __restrict__ x, long long ldx, bf16* __restrict__ u,
                                                   long long ldu, const float* __restrict__ shift0,
                                                   const float* __restrict__ scale0, const float* __restrict__ shift1,
                                                   const float* __restrict__ scale1, int n_first, int rows_b,
                                                   long long mstride) {
  __shared__ float red[T / 32];
  const int row = blockIdx.x;
  const int t = threadIdx.x;
  grid_dep_wait();
  // rows are B blocks of rows_b (SD3's CFG pair; B = 1 for FLUX); block b's modulation vectors sit
  // b * mstride floats further.  Inside a block rows [0, n_first) take (shift0, scale0), the others
  // (shift1, scale1): both streams of a double block in one launch
  const int b = row / rows_b, r = row - b * rows_b;
  const float* shift = (r < n_first ? shift0 : shift1) + b * mstride;
  const float* scale = (r < n_first ? scale0 : scale1) + b * mstride;
  constexpr int h = 4 * T * NV;
  const float4* xr = reinterpret_cast<const float4*>(x + (long long)row * ldx);
  float4 v[NV], shv[NV], scv[NV];
#pragma unroll
  for (int i = 0; i < NV; ++i) v[i] = xr[i * T + t];
  // the modulation vectors are independent of the row statistics: issue their loads up front
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    shv[i] = __ldg(reinterpret_cast<const float4*>(shift) + i * T + t);
    scv[i] = __ldg(reinterpret_cast<const float4*>(scale) + i * T + t);
  }
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < NV; ++i) s += (v[i].x + v[i].y) + (v[i].z + v[i].w);
  const float mean = block_sum<T>(s, red) * (1.0f / h);
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    float a = v[i].x - mean, b = v[i].y - mean, c = v[i].z - mean, d = v[i].w - mean;
    q += (a * a + b * b) + (c * c + d * d);
  }
  const float rstd = rsqrtf(block_sum<T>(q, red) * (1.0f / h) + 1e-6f);
  uint2* ur = reinterpret_cast<uint2*>(u + (long long)row * ldu);
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = i * T + t;
    const float4 sh = shv[i], sc = scv[i];
    float a = (v[i].x - mean) * rstd * (1.f + sc.x) + sh.x;
    float b = (v[i].y - mean) * rstd * (1.f + sc.y) + sh.y;
    float cc = (v[i].z - mean) * rstd * (1.f + sc.z) + sh.z;
    float d = (v[i].w - mean) * rstd * (1.f + sc.w) + sh.w;
    ur[c] = make_uint2(pack_bf16x2(a, b), pack_bf16x2(cc, d));
  }
  grid_dep_launch();   // the next kernel (a GEMM) may start its prologue / weight prefetch
}

// Persistent-row variant: CTA b handles rows b, b + grid, ... (grid ~ 4 CTAs per SM), keeps the
// modulation vectors in registers while consecutive rows share them (one reload at the txt/img
// boundary), and prefetches the next row's x while the current row is reduced and written.
template <int T, int NV>
__global__ void __launch_bounds__(T) ln_mod_rows_kernel(const float* __restrict__ x, long long ldx,
                                                        bf16* __restrict__ u, long long ldu,
                                                        const float* __restrict__ shift0,
                                                        const float* __restrict__ scale0,
                                                        const float* __restrict__ shift1,
                                                        const float* __restrict__ scale1, int n_first, int rows_b,
                                                        long long mstride, int M) {
  __shared__ float red[T / 32];
  const int t = threadIdx.x;
  constexpr int h = 4 * T * NV;
  grid_dep_wait();
  int row = blockIdx.x;
  float4 v[NV], shv[NV], scv[NV];
  const float* cur = nullptr;
  if (row < M) {
    const float4* xr = reinterpret_cast<const float4*>(x + (long long)row * ldx);
#pragma unroll
    for (int i = 0; i < NV; ++i) v[i] = __ldcs(xr + i * T + t);
  }
  for (; row < M; row += gridDim.x) {
    const int b = row / rows_b, r = row - b * rows_b;
    const float* shift = (r < n_first ? shift0 : shift1) + b * mstride;
    if (shift != cur) {   // uniform across the CTA
      const float* scale = (r < n_first ? scale0 : scale1) + b * mstride;
#pragma unroll
      for (int i = 0; i < NV; ++i) {
        shv[i] = __ldg(reinterpret_cast<const float4*>(shift) + i * T + t);
        scv[i] = __ldg(reinterpret_cast<const float4*>(scale) + i * T + t);
      }
      cur = shift;
    }
    const int nrow = row + gridDim.x;
    float4 vn[NV];
    if (nrow < M) {   // prefetch the next row under this row's reductions
      const float4* xn = reinterpret_cast<const float4*>(x + (long long)nrow * ldx);
#pragma unroll
      for (int i = 0; i < NV; ++i) vn[i] = __ldcs(xn + i * T + t);
    }
    float sm = 0.f;
#pragma unroll
    for (int i = 0; i < NV; ++i) sm += (v[i].x + v[i].y) + (v[i].z + v[i].w);
    const float mean = block_sum<T>(sm, red) * (1.0f / h);
    float q = 0.f;
#pragma unroll
    for (int i = 0; i < NV; ++i) {
      float a = v[i].x - mean, bb = v[i].y - mean, c = v[i].z - mean, d = v[i].w - mean;
      q += (a * a + bb * bb) + (c * c + d * d);
    }
    const float rstd = rsqrtf(block_sum<T>(q, red) * (1.0f / h) + 1e-6f);
    uint2* ur = reinterpret_cast<uint2*>(u + (long long)row * ldu);
#pragma unroll
    for (int i = 0; i < NV; ++i) {
      const int c = i * T + t;
      const float4 sh = shv[i], sc = scv[i];
      const float a = (v[i].x - mean) * rstd * (1.f + sc.x) + sh.x;
      const float bb = (v[i].y - mean) * rstd * (1.f + sc.y) + sh.y;
      const float cc = (v[i].z - mean) * rstd * (1.f + sc.z) + sh.z;
      const float d = (v[i].w - mean) * rstd * (1.f + sc.w) + sh.w;
      ur[c] = make_uint2(pack_bf16x2(a, bb), pack_bf16x2(cc, d));
    }
    if (nrow < M) {
#pragma unroll
      for (int i = 0; i < NV; ++i) v[i] = vn[i];
    }
  }
  grid_dep_launch();
}

// Warp per row (8 rows per 256-thread CTA): the row stays in registers (NV float4 per lane), both
// reductions are warp shuffles (no block barriers), the modulation vectors come through L1 (shared
// by every row of a stream).  Rows [0, n_first) of each block of rows_b take (shift0, scale0).
template <int NV>
__global__ void __launch_bounds__(256) ln_mod_warp_kernel(const float* __restrict__ x, long long ldx,
                                                          bf16* __restrict__ u, long long ldu,
                                                          const float* __restrict__ shift0,
                                                          const float* __restrict__ scale0,
                                                          const float* __restrict__ shift1,
                                                          const float* __restrict__ scale1, int n_first, int rows_b,
                                                          long long mstride, int M) {
  const int row = blockIdx.x * 8 + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  grid_dep_wait();
  if (row >= M) return;
  const int b = row / rows_b, r = row - b * rows_b;
  const float* shift = (r < n_first ? shift0 : shift1) + b * mstride;
  const float* scale = (r < n_first ? scale0 : scale1) + b * mstride;
  constexpr int h = 128 * NV;
  const float4* xr = reinterpret_cast<const float4*>(x + (long long)row * ldx);
  float4 v[NV];
#pragma unroll
  for (int i = 0; i < NV; ++i) v[i] = xr[i * 32 + lane];
  float sm = 0.f;
#pragma unroll
  for (int i = 0; i < NV; ++i) sm += (v[i].x + v[i].y) + (v[i].z + v[i].w);
#pragma unroll
  for (int o = 16; o; o >>= 1) sm += __shfl_xor_sync(0xffffffffu, sm, o);
  const float mean = sm * (1.0f / h);
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const float a = v[i].x - mean, bb = v[i].y - mean, c = v[i].z - mean, d = v[i].w - mean;
    q += (a * a + bb * bb) + (c * c + d * d);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
  const float rstd = rsqrtf(q * (1.0f / h) + 1e-6f);
  uint2* ur = reinterpret_cast<uint2*>(u + (long long)row * ldu);
  const float4* shp = reinterpret_cast<const float4*>(shift);
  const float4* scp = reinterpret_cast<const float4*>(scale);
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = i * 32 + lane;
    const float4 sh = __ldg(shp + c), sc = __ldg(scp + c);
    const float a = (v[i].x - mean) * rstd * (1.f + sc.x) + sh.x;
    const float bb = (v[i].y - mean) * rstd * (1.f + sc.y) + sh.y;
    const float cc = (v[i].z - mean) * rstd * (1.f + sc.z) + sh.z;
    const float d = (v[i].w - mean) * rstd * (1.f + sc.w) + sh.w;
    ur[c] = make_uint2(pack_bf16x2(a, bb), pack_bf16x2(cc, d));
  }
  grid_dep_launch();
}

// generic fallback (h multiple of 128): two passes over global memory
__global__ void __launch_bounds__(256) ln_mod_generic(const float* __restrict__ x, long long ldx, bf16* __restrict__ u,
                                                      long long ldu, const float* __restrict__ shift0,
                                                      const float* __restrict__ scale0,
                                                      const float* __restrict__ shift1,
                                                      const float* __restrict__ scale1, int n_first, int M, int h,
                                                      int rows_b, long long mstride) {
  const int row = blockIdx.x * 8 + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  grid_dep_wait();
  grid_dep_launch();
  if (row >= M) return;
  const int b = row / rows_b, r = row - b * rows_b;
  const float* shift = (r < n_first ? shift0 : shift1) + b * mstride;
  const float* scale = (r < n_first ? scale0 : scale1) + b * mstride;
  const float* xr = x + (long long)row * ldx;
  float s = 0.f;
  for (int c = lane; c < h; c += 32) s += xr[c];
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float mean = s / h;
  float q = 0.f;
  for (int c = lane; c < h; c += 32) { float a = xr[c] - mean; q += a * a; }
  for (int o = 16; o; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
  const float rstd = rsqrtf(q / h + 1e-6f);
  for (int c = lane; c < h; c += 32)
    u[(long long)row * ldu + c] = __float2bfloat16_rn((xr[c] - mean) * rstd * (1.f + scale[c]) + shift[c]);
}

// LN-modulate kernel choice (tsv_op_ln_mod impl; TSV_LN_IMPL): 0 CTA per row, 1 warp per row,
// 2 persistent rows (the default: same-box FLUX 512^2 step A/B -0.5 %)
int g_ln_impl = 2;

void ln_mod2b_launch(const float* x, long long ldx, bf16* u, long long ldu, const float* shift0,
                     const float* scale0, const float* shift1, const float* scale1, int n_first, int rows_b, int B,
                     long long mstride, int h, cudaStream_t s) {
  const int M = rows_b * B;
  if (M <= 0) return;
  if (g_ln_impl == 1 && (h == 3072 || h == 1536)) {
    const dim3 grid((M + 7) / 8);
    if (h == 3072)
      launch_pdl(ln_mod_warp_kernel<24>, grid, dim3(256), 0, s, x, ldx, u, ldu, shift0, scale0, shift1, scale1, n_first,
                 rows_b, mstride, M);
    else
      launch_pdl(ln_mod_warp_kernel<12>, grid, dim3(256), 0, s, x, ldx, u, ldu, shift0, scale0, shift1, scale1, n_first,
                 rows_b, mstride, M);
    return;
  }
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  // persistent rows only pay off while the launch is about one wave of row-CTAs (512^2: -0.5 % step);
  // at 2048^2 (16 896 rows) the CTA-per-row kernel streams faster (measured, profiles/README.md)
  if (g_ln_impl == 2 && (h == 3072 || h == 1536 || h == 256) && M <= 16 * sms) {
    const int grid = M < 4 * sms ? M : 4 * sms;
    if (h == 3072)
      launch_pdl(ln_mod_rows_kernel<256, 3>, dim3(grid), dim3(256), 0, s, x, ldx, u, ldu, shift0, scale0, shift1,
                 scale1, n_first, rows_b, mstride, M);
    else if (h == 1536)
      launch_pdl(ln_mod_rows_kernel<128, 3>, dim3(grid), dim3(128), 0, s, x, ldx, u, ldu, shift0, scale0, shift1,
                 scale1, n_first, rows_b, mstride, M);
    else
      launch_pdl(ln_mod_rows_kernel<32, 2>, dim3(grid), dim3(32), 0, s, x, ldx, u, ldu, shift0, scale0, shift1,
                 scale1, n_first, rows_b, mstride, M);
    return;
  }
  switch (h) {
    case 3072:
      launch_pdl(ln_mod_kernel<256, 3>, dim3(M), dim3(256), 0, s, x, ldx, u, ldu, shift0, scale0, shift1, scale1, n_first,
                 rows_b, mstride);
      break;
    case 1536:
      launch_pdl(ln_mod_kernel<128, 3>, dim3(M), dim3(128), 0, s, x, ldx, u, ldu, shift0, scale0, shift1, scale1, n_first,
                 rows_b, mstride);
      break;
    case 256:
      launch_pdl(ln_mod_kernel<32, 2>, dim3(M), dim3(32), 0, s, x, ldx, u, ldu, shift0, scale0, shift1, scale1, n_first,
                 rows_b, mstride);
      break;
    default:
      launch_pdl(ln_mod_generic, dim3((M + 7) / 8), dim3(256), 0, s, x, ldx, u, ldu, shift0, scale0, shift1, scale1,
                 n_first, M, h, rows_b, mstride);
      break;
  }
}

void ln_mod2_launch(const float* x, long long ldx, bf16* u, long long ldu, const float* shift0,
                    const float* scale0, const float* shift1, const float* scale1, int n_first, int M, int h,
                    cudaStream_t s) {
  ln_mod2b_launch(x, ldx, u, ldu, shift0, scale0, shift1, scale1, n_first, M, 1, 0, h, s);
}

void ln_mod_launch(const float* x, long long ldx, bf16* u, long long ldu, const float* shift, const float* scale,
                   int M, int h, cudaStream_t s) {
  ln_mod2_launch(x, ldx, u, ldu, shift, scale, shift, scale, M, M, h, s);
}

// ------------------------------------------------------------------ a4: QK-RMSNorm + RoPE (+ Ulysses pack)
// One warp per (row, head).  Lane l holds D/32 consecutive elements (pairs 2 per 4 elements).
template <int D>
__global__ void __launch_bounds__(256) qk_norm_rope_kernel(bf16* __restrict__ qkv, long long ld, int rows, int n_first,
                                                           int H, const bf16* __restrict__ gq0,
                                                           const bf16* __restrict__ gk0, const bf16* __restrict__ gq1,
                                                           const bf16* __restrict__ gk1, const float* __restrict__ cosb,
                                                           const float* __restrict__ sinb, bf16* __restrict__ pack,
                                                           int k_sp) {
  constexpr int E = D / 32;  // elements per lane (4 for D=128, 2 for D=64)
  const long long gw = (long long)blockIdx.x * 8 + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (gw >= (long long)rows * H) return;
  const int row = (int)(gw / H), head = (int)(gw % H);
  const bool first = row < n_first;
  const bf16* gq = first ? gq0 : gq1;
  const bf16* gk = first ? gk0 : gk1;
  const int hD = H * D;
  bf16* base = qkv + (long long)row * ld;
  const float* cr = cosb + (long long)row * (D / 2);
  const float* sr = sinb + (long long)row * (D / 2);
  const int d0 = lane * E;
  float cs[E / 2], sn[E / 2];
#pragma unroll
  for (int p = 0; p < E / 2; ++p) {
    cs[p] = __ldg(cr + d0 / 2 + p);
    sn[p] = __ldg(sr + d0 / 2 + p);
  }
  bf16* dst_base = nullptr;
  int hk = H / k_sp;
  if (pack) {
    const int dst = head / hk, hl = head % hk;
    dst_base = pack + (((long long)dst * rows + row) * 3) * hk * D + (long long)hl * D;
  }
#pragma unroll
  for (int part = 0; part < 2; ++part) {
    bf16* src = base + part * hD + head * D + d0;
    float x[E];
    if constexpr (E == 4) {
      uint2 u = *reinterpret_cast<const uint2*>(src);
      float2 a = unpack_bf16x2(u.x), b = unpack_bf16x2(u.y);
      x[0] = a.x; x[1] = a.y; x[2] = b.x; x[3] = b.y;
    } else {
      uint32_t u = *reinterpret_cast<const uint32_t*>(src);
      float2 a = unpack_bf16x2(u);
      x[0] = a.x; x[1] = a.y;
    }
    float ss = 0.f;
#pragma unroll
    for (int e = 0; e < E; ++e) ss += x[e] * x[e];
#pragma unroll
    for (int o = 16; o; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
    const float r = rsqrtf(ss * (1.0f / D) + 1e-6f);
    const bf16* g = part == 0 ? gq : gk;
    float y[E];
#pragma unroll
    for (int e = 0; e < E; ++e) y[e] = x[e] * r * __bfloat162float(g[d0 + e]);
    float z[E];
#pragma unroll
    for (int p = 0; p < E / 2; ++p) {
      z[2 * p] = cs[p] * y[2 * p] - sn[p] * y[2 * p + 1];
      z[2 * p + 1] = sn[p] * y[2 * p] + cs[p] * y[2 * p + 1];
    }
    bf16* dst = pack ? dst_base + part * hk * D + d0 : src;
    if constexpr (E == 4) {
      *reinterpret_cast<uint2*>(dst) = make_uint2(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]));
    } else {
      *reinterpret_cast<uint32_t*>(dst) = pack_bf16x2(z[0], z[1]);
    }
  }
  if (pack) {  // v: plain copy into the send layout
    const bf16* src = base + 2 * hD + head * D + d0;
    bf16* dst = dst_base + 2 * hk * D + d0;
    if constexpr (E == 4) *reinterpret_cast<uint2*>(dst) = *reinterpret_cast<const uint2*>(src);
    else *reinterpret_cast<uint32_t*>(dst) = *reinterpret_cast<const uint32_t*>(src);
  }
}

void qk_norm_rope_launch(bf16* qkv, long long ld, int rows, int n_first, int H, int D, const bf16* gq0,
                         const bf16* gk0, const bf16* gq1, const bf16* gk1, const float* cosb, const float* sinb,
                         bf16* pack_out, int k_sp, cudaStream_t s) {
  if (rows <= 0) return;
  const long long warps = (long long)rows * H;
  dim3 grid((unsigned)((warps + 7) / 8));
  if (D == 128)
    qk_norm_rope_kernel<128><<<grid, 256, 0, s>>>(qkv, ld, rows, n_first, H, gq0, gk0, gq1, gk1, cosb, sinb,
                                                  pack_out, k_sp);
  else
    qk_norm_rope_kernel<64><<<grid, 256, 0, s>>>(qkv, ld, rows, n_first, H, gq0, gk0, gq1, gk1, cosb, sinb,
                                                 pack_out, k_sp);
}

// ------------------------------------------------------------------ small conversions
__global__ void f32_to_bf16_kernel(const float* __restrict__ src, long long lds, bf16* __restrict__ dst,
                                   long long ldd, int M, int C, int act) {
  grid_dep_wait();
  grid_dep_launch();
  long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  long long n = (long long)M * C;
  for (; i < n; i += (long long)gridDim.x * blockDim.x) {
    int m = (int)(i / C), c = (int)(i % C);
    float v = src[(long long)m * lds + c];
    if (act == 1) v = silu(v);
    dst[(long long)m * ldd + c] = __float2bfloat16_rn(v);
  }
}
void f32_to_bf16_launch(const float* src, long long lds, bf16* dst, long long ldd, int M, int C, cudaStream_t s) {
  if (M <= 0 || C <= 0) return;
  long long n = (long long)M * C;
  int blocks = (int)((n + 255) / 256);
  if (blocks > 4096) blocks = 4096;
  launch_pdl(f32_to_bf16_kernel, dim3(blocks), dim3(256), 0, s, src, lds, dst, ldd, M, C, 0);
}
void silu_bf16_launch(const float* src, long long lds, bf16* dst, long long ldd, int M, int C, cudaStream_t s) {
  if (M <= 0 || C <= 0) return;
  long long n = (long long)M * C;
  int blocks = (int)((n + 255) / 256);
  if (blocks > 4096) blocks = 4096;
  launch_pdl(f32_to_bf16_kernel, dim3(blocks), dim3(256), 0, s, src, lds, dst, ldd, M, C, 1);
}

// rows x cols bf16, cols multiple of 8, strides multiple of 8 elements
__global__ void copy2d_bf16_kernel(const uint4* __restrict__ src, long long lds8, uint4* __restrict__ dst,
                                   long long ldd8, int rows, int cols8) {
  grid_dep_wait();
  grid_dep_launch();
  long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  long long n = (long long)rows * cols8;
  for (; i < n; i += (long long)gridDim.x * blockDim.x) {
    int r = (int)(i / cols8), c = (int)(i % cols8);
    dst[r * ldd8 + c] = src[r * lds8 + c];
  }
}
void copy2d_bf16_launch(const bf16* src, long long lds, bf16* dst, long long ldd, int rows, int cols, cudaStream_t s) {
  if (rows <= 0 || cols <= 0) return;
  long long n = (long long)rows * (cols / 8);
  int blocks = (int)((n + 255) / 256);
  if (blocks > 8192) blocks = 8192;
  launch_pdl(copy2d_bf16_kernel, dim3(blocks), dim3(256), 0, s, reinterpret_cast<const uint4*>(src), lds / 8,
             reinterpret_cast<uint4*>(dst), ldd / 8, rows, cols / 8);
}

__global__ void select_row_kernel(const float* __restrict__ src, long long stride, const int* __restrict__ idx,
                                  float* __restrict__ dst, long long n) {
  grid_dep_wait();
  grid_dep_launch();
  const float* s = src + (long long)(*idx) * stride;
  long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long n4 = n / 4;
  for (; i < n4; i += (long long)gridDim.x * blockDim.x)
    reinterpret_cast<float4*>(dst)[i] = reinterpret_cast<const float4*>(s)[i];
  if (blockIdx.x == 0 && threadIdx.x < (n & 3)) dst[n4 * 4 + threadIdx.x] = s[n4 * 4 + threadIdx.x];
}
void select_row_launch(const float* src, long long stride, const int* idx_dev, float* dst, long long n,
                       cudaStream_t s) {
  if (n <= 0) return;
  int blocks = (int)((n / 4 + 255) / 256);
  if (blocks < 1) blocks = 1;
  if (blocks > 2048) blocks = 2048;
  launch_pdl(select_row_kernel, dim3(blocks), dim3(256), 0, s, src, stride, idx_dev, dst, n);
}

// ------------------------------------------------------------------ SYNTH-1 (see include/tsv.h)
__device__ __forceinline__ uint64_t splitmix64_mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__global__ void synth_kernel(void* dst, uint64_t seed, uint32_t tid, uint64_t idx0, long long n, int kind, float c) {
  const uint64_t key = seed ^ ((uint64_t)tid << 48);
  long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i < n; i += (long long)gridDim.x * blockDim.x) {
    const uint64_t h = splitmix64_mix(((idx0 + (uint64_t)i) ^ key) + 0x9E3779B97F4A7C15ull);
    const int u = (int)(h >> 40);
    const float r = (float)(u - (1 << 23)) * 1.1920928955078125e-07f;  // exact: 24-bit int * 2^-23
    float v = __fmul_rn(r, c);
    if (kind == 2) {
      reinterpret_cast<float*>(dst)[i] = v;
    } else {
      if (kind == 1) v = __fadd_rn(1.0f, v);
      reinterpret_cast<bf16*>(dst)[i] = __float2bfloat16_rn(v);
    }
  }
}
void synth_launch(void* dst, uint64_t seed, uint32_t tensor_id, uint64_t idx0, long long n, int kind, float c,
                  cudaStream_t s) {
  if (n <= 0) return;
  long long blocks = (n + 255) / 256;
  if (blocks > 148 * 64) blocks = 148 * 64;
  synth_kernel<<<(unsigned)blocks, 256, 0, s>>>(dst, seed, tensor_id, idx0, n, kind, c);
}

// ------------------------------------------------------------------ per-shard position tables
__global__ void rope_table_kernel(float* cosb, float* sinb, int nt, long long i0, int ni, long long wp, int half,
                                  int d0, int d1, int d2, double theta) {
  const long long n = (long long)(nt + ni) * half;
  for (long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x; idx < n;
       idx += (long long)gridDim.x * blockDim.x) {
    const long long row = idx / half;
    const int pair = (int)(idx % half);
    float c = 1.f, s = 0.f;
    if (row >= nt) {
      const long long p = i0 + (row - nt);
      int a, j, da;
      if (pair < d0 / 2) { a = 0; j = pair; da = d0; }
      else if (pair < (d0 + d1) / 2) { a = 1; j = pair - d0 / 2; da = d1; }
      else { a = 2; j = pair - (d0 + d1) / 2; da = d2; }
      const double id = a == 0 ? 0.0 : (a == 1 ? (double)(p / wp) : (double)(p % wp));
      const double ang = id * (1.0 / pow(theta, (2.0 * j) / da));
      c = (float)cos(ang);
      s = (float)sin(ang);
    }
    cosb[idx] = c;
    sinb[idx] = s;
  }
}
void rope_table_launch(float* cosb, float* sinb, int nt, long long i0, int ni, long long wp, int D,
                       const int axes_dim[3], double theta, cudaStream_t s) {
  const long long n = (long long)(nt + ni) * (D / 2);
  if (n <= 0) return;
  const long long blocks = std::min<long long>((n + 255) / 256, 148 * 16);
  rope_table_kernel<<<(unsigned)blocks, 256, 0, s>>>(cosb, sinb, nt, i0, ni, wp, D / 2, axes_dim[0], axes_dim[1],
                                                      axes_dim[2], theta);
}

__global__ void sincos_pe_kernel(float* pe, long long i0, int ni, long long n_c, long long top, long long left,
                                 double q, int h) {
  const int quarter = h / 4;
  const long long n = (long long)ni * quarter;
  for (long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x; idx < n;
       idx += (long long)gridDim.x * blockDim.x) {
    const long long r = idx / quarter;
    const int j = (int)(idx % quarter);
    const long long p = i0 + r;
    const double pr = (double)(p / n_c + top) / q, pc = (double)(p % n_c + left) / q;
    const double w = 1.0 / pow(10000.0, (double)j / quarter);
    float* o = pe + r * h;
    o[j] = (float)sin(pc * w);
    o[quarter + j] = (float)cos(pc * w);
    o[2 * quarter + j] = (float)sin(pr * w);
    o[3 * quarter + j] = (float)cos(pr * w);
  }
}
void sincos_pe_launch(float* pe, long long i0, int ni, long long n_c, long long top, long long left, double q, int h,
                      cudaStream_t s) {
  const long long n = (long long)ni * (h / 4);
  if (n <= 0) return;
  const long long blocks = std::min<long long>((n + 255) / 256, 148 * 16);
  sincos_pe_kernel<<<(unsigned)blocks, 256, 0, s>>>(pe, i0, ni, n_c, top, left, q, h);
}

// ------------------------------------------------------------------ cross-process barrier
__global__ void ipc_barrier_kernel(const __grid_constant__ IpcBarrier b) {
  grid_dep_wait();
  int* own = b.flags[b.rank];
  const int epoch = own[63] + 1;   // this member's barrier count (every member calls the same sequence)
  own[63] = epoch;
  __threadfence_system();          // this GPU's earlier peer stores are visible before the flag
  for (int p = 0; p < b.k; ++p)
    if (p != b.rank) asm volatile("st.release.sys.global.s32 [%0], %1;" ::"l"(b.flags[p] + b.rank), "r"(epoch) : "memory");
  for (int p = 0; p < b.k; ++p) {
    if (p == b.rank) continue;
    long long spins = 0;
    for (;;) {
      int v;
      asm volatile("ld.acquire.sys.global.s32 %0, [%1];" : "=r"(v) : "l"(own + p) : "memory");
      if (v >= epoch) break;
      __nanosleep(200);
      if (++spins > (1ll << 25)) { own[62] = 1; break; }   // ~10 s: give up rather than hang
    }
  }
  __threadfence_system();
  grid_dep_launch();
}

void ipc_barrier_launch(const IpcBarrier& b, cudaStream_t s) {
  launch_pdl(ipc_barrier_kernel, dim3(1), dim3(1), 0, s, b);
}

}  // namespace tsv
