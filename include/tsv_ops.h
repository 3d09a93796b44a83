/*
 * tsv_ops.h — kernel-level C-ABI of libtsv.so (device pointers), used by the parity tests and
 * the kernel micro-benchmarks.  Each entry launches exactly the kernel the step uses for that
 * operation; no host computation.  All pointers are device pointers owned by the caller;
 * `stream` is a cudaStream_t (NULL = legacy default stream).  Asynchronous; errors are launch
 * errors (TSV_E_CUDA) or argument errors (TSV_E_INVAL) with tsv_last_error() set.
 *
 * Citations: S:§8(a) rows of SURVEY.md (the hot-path scope table); TT = public FLUX.1 code
 * (architecture facts; the paper cites FLUX.1-dev without equations).
 */
#ifndef TSV_OPS_H_
#define TSV_OPS_H_

#include <stdint.h>
#include "tsv.h"

#ifdef __cplusplus
extern "C" {
#endif

/* GEMM epilogue modes (y = A W^T + bias, fp32 accumulate, S:§8(a) a1/a3/a8/a9/a11/a12) */
enum {
  TSV_EPI_STORE_BF16 = 0, /* out0 bf16 [M, ld0] = y */
  TSV_EPI_GELU_BF16 = 1,  /* out0 = gelu_tanh(y) */
  TSV_EPI_SILU_BF16 = 2,  /* out0 = silu(y) */
  TSV_EPI_SPLIT_GELU = 3, /* n < n_split: out0[m, n] = y; else out1[m, n - n_split] = gelu_tanh(y) */
  TSV_EPI_RESID_GATE = 4, /* out0 fp32 [m, n] += gate[n] * y */
  TSV_EPI_STORE_F32 = 5,  /* out0 fp32 = y */
  TSV_EPI_ACCUM_F32 = 6,  /* out0 fp32 += y */
  TSV_EPI_EULER = 7       /* out1 fp32 (optional) = y; out0 fp32 += (*scalar) * y */
};

/* A [M, K] bf16 (row stride lda elements), W [N, K] bf16 (nn.Linear layout, row stride ldw),
 * bias [N] bf16 or NULL, gate [N] fp32, scalar: device fp32.  K % 64 == 0, N % 64 == 0, 16-byte
 * aligned operands and row strides.  force_bn in {0 (auto), 64, 128, 256}; force_pair: -1 auto,
 * 0 single-CTA tiles, 1 CTA-pair (cta_group::2) 256 x 256 tiles (needs BN = 256).
 * Launched with programmatic dependent launch: W is treated as a constant (its first tiles are
 * requested before the wait on the previous kernel), so W must not be written by the kernel
 * launched immediately before on the same stream if that kernel is one of this library's. */
tsv_status tsv_op_gemm(const void* A, int64_t lda, const void* W, int64_t ldw, int M, int N, int K, int mode,
                       void* out0, int64_t ld0, void* out1, int64_t ld1, int n_split, const void* bias,
                       const float* gate, const float* scalar, int force_bn, int force_pair, void* stream);

/* The same GEMM with split-K (a8 / a9 on small row counts): K is cut into `splits` ranges
 * (0: the engine's automatic choice, which may be 1); each range's fp32 partial goes to ws and the
 * last range to finish an output tile sums the partials in range order 0..splits-1 and applies the
 * epilogue once, so the result is deterministic.  Modes: TSV_EPI_STORE_BF16 / GELU_BF16 /
 * SILU_BF16 / STORE_F32 (out0 = f(A W^T + bias)), TSV_EPI_RESID_GATE (out0 += gate * (A W^T +
 * bias)), TSV_EPI_ACCUM_F32 (out0 += A W^T + bias).  sem: device int buffer of
 * sem_ints >= 4 * output tiles entries, zero on entry and left zero; ws: device buffer of ws_bytes
 * (splits * tiles * 128 * tile width * 4 bytes are used; the split factor is capped to fit).  One
 * (sem, ws) pair per concurrently running launch.  TSV_E_INVAL for other modes. */
tsv_status tsv_op_gemm_split(const void* A, int64_t lda, const void* W, int64_t ldw, int M, int N, int K, int mode,
                             void* out0, int64_t ld0, const void* bias, const float* gate, int splits, int* sem,
                             int sem_ints, float* ws, int64_t ws_bytes, void* stream);

/* a3 + a4 fused (the step's QKV / linear1 GEMM): y = A W^T + bias with columns "(K H D)" =
 * [q | k | v] over [0, 3h) (+ GELU columns >= 3h into out1 when mode = TSV_EPI_SPLIT_GELU,
 * n_split = 3h).  q and k heads become RoPE(RMSNorm(y) * g) (eps 1e-6; gq/gk bf16 [D]; cos/sin fp32
 * [M][D/2] indexed by GEMM row); v passes through.  k_sp = 1: written to out0 [M, ld0];
 * k_sp > 1: written to pack laid out [k_sp][pack_rows][3][H/k_sp][D] at row pack_row0 + m. */
tsv_status tsv_op_gemm_qkv(const void* A, int64_t lda, const void* W, int64_t ldw, int M, int N, int K, int mode,
                           void* out0, int64_t ld0, void* out1, int64_t ld1, const void* bias, int h, int D,
                           const void* gq, const void* gk, const float* cosb, const float* sinb, int k_sp,
                           void* pack, int pack_rows, int pack_row0, void* stream);

/* a2: u[m, :] = bf16(LN(x[m, :]) * (1 + scale) + shift); x fp32, LN without affine, eps 1e-6.
 * impl 0: one CTA per row (block reductions); impl 1: one warp per row; impl 2: persistent CTAs
 * (~4 per SM) looping over rows with the modulation vectors kept in registers and the next row
 * prefetched, used for launches of <= 16 rows per SM (else impl 0).  impl 1: h in {1536, 3072};
 * impl 2: h in {256, 1536, 3072}; other h fall back to impl 0.  The engine's step uses impl 2
 * (TSV_LN_IMPL at engine creation selects another).
 * Errors: TSV_E_INVAL (h % 128, impl). */
tsv_status tsv_op_ln_mod(const float* x, int64_t ldx, void* u, int64_t ldu, const float* shift,
                         const float* scale, int M, int h, int impl, void* stream);

/* a4: on qkv bf16 [rows, 3*H*D] (columns "(K H D)"), q and k of every head become
 * RoPE(RMSNorm(x) * g) (eps 1e-6; pair (2j, 2j+1) rotated by the per-row table angle j).
 * Rows < n_first use gains gq0/gk0, the others gq1/gk1 (bf16 [D]).  cos/sin: fp32 [rows, D/2].
 * pack == NULL: in place.  Otherwise q, k, v are written to pack laid out
 * [k_sp][rows][3][H/k_sp][D] (the Ulysses send buffer) and qkv is not modified. */
tsv_status tsv_op_qk_norm_rope(void* qkv, int64_t ld, int rows, int n_first, int H, int D, const void* gq0,
                               const void* gk0, const void* gq1, const void* gk1, const float* cosb,
                               const float* sinb, void* pack, int k_sp, void* stream);

/* a6: O = softmax(q k^T / sqrt(D)) v, non-causal, per head h < H; q(l, h) at q + l*ldq + h*D
 * (bf16, same for k, v, o).  D in {64, 128}.  Operands and row strides 16-byte aligned.
 * impl 0: the tcgen05/TMEM kernel the step uses (= impl 56 for D = 128, 103 for D = 64; the
 * environment variables TSV_ATTN_D128 / TSV_ATTN_D64 select another impl for the step);
 * 50 / 51 / 56: separate K and V TMA rings (2 + 2 stages at D = 128, 4 + 4 at D = 64) with 0 / 1 / 2
 * of every 8 exp2 pairs evaluated by a polynomial on the FMA pipe instead of MUFU.EX2 (51: cubic with
 * clamps, 56: cubic with the clamp folded into saturating FFMAs); 81 / 83: one joint K+V ring, 1 / 3
 * polynomial pairs; D = 64 only, the joint ring with three rotating S buffers shared by the two query
 * tiles (S computed one ahead): 92 (2 pairs, clamped cubic), 96 (3, saturating cubic), 103 (3,
 * saturating minimax quadratic); 59, 99: DIAGNOSTIC ONLY, wrong results -- P = the scaled score without
 * any exponential (the pipeline's ceiling without the softmax arithmetic).
 * Other values: TSV_E_INVAL. */
tsv_status tsv_op_attention(const void* q, int64_t ldq, const void* k, int64_t ldk, const void* v, int64_t ldv,
                            void* o, int64_t ldo, int L, int H, int D, int impl, void* stream);

/* a6 with the key range split (flash-decoding style) for launches with too few CTAs (SP = 4/8 head
 * shards, small images): nsplit key ranges (0: the engine's automatic choice -- whole work items
 * first, the launch's last items split into key ranges by a list-scheduling model, possibly none;
 * > 0: every item in nsplit equal ranges; capped at 8 and by the workspace), each range's
 * unnormalised O, reference and sum go to ws and the last range to finish a query tile merges them
 * in range order (deterministic).  The step's attention kernel (impl 0).  cnt: zeroed device ints
 * (>= 8 per split 256-query block and head), left zero; ws: fp32 device workspace (nsplit x 2 x 128
 * x (D + 2) floats per split 256-query block and head).
 * Same operand rules as tsv_op_attention. */
/* Host only (no GPU needed): the KV-split plan tsv_op_attention_split(nsplit = 0 or the forced
 * nsplit) and the step would use for (L, H, D) with a workspace of ws_bytes / cnt_ints on a GPU with
 * `sms` SMs (<= 0: 148).  Work items = ceil(L / 256) x H; the first *n_plain run over all keys, the
 * last *n_tail in *nsplit key ranges, range z = key tiles (of 128) [bounds[z], bounds[z + 1])
 * (bounds: 9 ints, caller-owned).  *nsplit = 1: no split.  The same list-scheduling model as the
 * launch.  Errors: TSV_E_INVAL. */
tsv_status tsv_attention_split_plan(int L, int H, int D, int64_t ws_bytes, int cnt_ints, int nsplit, int sms,
                                    int* n_plain, int* n_tail, int* nsplit_out, int* bounds);

tsv_status tsv_op_attention_split(const void* q, int64_t ldq, const void* k, int64_t ldk, const void* v, int64_t ldv,
                                  void* o, int64_t ldo, int L, int H, int D, int nsplit, int* cnt, int cnt_ints,
                                  float* ws, int64_t ws_bytes, void* stream);

/* SYNTH-1 on device: n values of (seed, tensor_id) starting at element idx0.
 * kind 0: bf16 rne(r*c); 1: bf16 rne(1 + r*c); 2: fp32 r*c. */
tsv_status tsv_op_synth(void* dst, uint64_t seed, uint32_t tensor_id, uint64_t idx0, int64_t n, int kind, float c,
                        void* stream);

#ifdef __cplusplus
}
#endif
#endif /* TSV_OPS_H_ */
