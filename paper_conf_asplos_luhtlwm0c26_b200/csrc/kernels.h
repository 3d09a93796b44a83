// Host-side launchers of the sm_100a kernels (internal to libtsv.so; the public C-ABI is in
// include/tsv.h and include/tsv_ops.h).
#pragma once
#include <cstddef>
#include <cstdint>
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

namespace tsv {

using bf16 = __nv_bfloat16;

// Launch with programmatic stream serialisation (PDL): inside a captured step graph the next
// kernel's prologue overlaps this kernel's tail; kernels call grid_dep_wait() before reading
// their inputs (ptx.cuh).
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

// ------------------------------------------------------------------ GEMM  y = A W^T (+ bias) -> epilogue
enum EpiMode : int {
  EPI_STORE_BF16 = 0,   // out0[m,n] = bf16(acc + b)
  EPI_GELU_BF16 = 1,    // out0[m,n] = bf16(gelu_tanh(acc + b))
  EPI_SILU_BF16 = 2,    // out0[m,n] = bf16(silu(acc + b))
  EPI_SPLIT_GELU = 3,   // n < n_split: out0[m,n] = bf16(acc+b); else out1[m,n-n_split] = bf16(gelu(acc+b))
  EPI_RESID_GATE = 4,   // out0 (fp32) [m,n] += gate[n] * (acc + b)
  EPI_STORE_F32 = 5,    // out0 (fp32) [m,n] = acc + b
  EPI_ACCUM_F32 = 6,    // out0 (fp32) [m,n] += acc + b
  EPI_EULER = 7,        // v = acc + b; out1 (fp32, optional) [m,n] = v; out0 (fp32) [m,n] += (*scalar) * v
  EPI_CFG_EULER = 8,    // v_c = acc + b; v = out1 + alpha (v_c - out1) (out1 holds v_u on entry);
                        // out1 (fp32) [m,n] = v; out0 (fp32) [m,n] += (*scalar) * v   (SD3 CFG, S23)
};
constexpr int GEMM_MAX_PROBLEMS = 16;  // 2 streams x up to 8 evaluations (requests x CFG branches)

struct GemmEpi {
  int mode = EPI_STORE_BF16;
  void* out0 = nullptr;
  long long ld0 = 0;  // elements
  void* out1 = nullptr;
  long long ld1 = 0;
  int n_split = 0;
  const bf16* bias = nullptr;   // [N]
  const float* gate = nullptr;  // [N]
  const float* scalar = nullptr;
  float alpha = 0.f;            // EPI_CFG_EULER guidance scale
  // Fused a4 (QK-RMSNorm + RoPE, Ulysses pack) for a QKV-producing GEMM (modes STORE_BF16 /
  // SPLIT_GELU): columns [0, 3*qk_h) are "(K H D)" q|k|v; q and k heads get
  // RoPE(RMSNorm(y) * g), v passes through.  qk_h = 0 disables; gq = gk = null keeps the
  // Ulysses pack but skips norm and RoPE (SD3: no QK-norm, no RoPE).
  int qk_h = 0;
  int qk_D = 0;
  const bf16* gq = nullptr;
  const bf16* gk = nullptr;
  const float* cosb = nullptr;  // [M][qk_D/2], indexed by GEMM row
  const float* sinb = nullptr;
  // k_sp > 1: q|k|v columns are written to pack[dst][pack_rows][3][H/k_sp][D] at row pack_row0 + m
  int k_sp = 1;
  bf16* pack = nullptr;
  int pack_rows = 0;
  int pack_row0 = 0;
  // Fused a5 (k_sp > 1 and peer[0] != null): the q|k|v columns of head block dst go straight into
  // rank dst's attention input peer[dst] = [L][3][H/k_sp][D] at the row's global position (the
  // all-to-all #1 becomes the epilogue's stores: local, or peer memory over NVLink).  A problem
  // covers at most two contiguous global ranges (a single block's [txt_r; img_r] rows).
  bf16* peer[8] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
  int peer_row0 = 0;   // GEMM rows [0, peer_nt) -> global rows peer_row0 + m
  int peer_nt = 1 << 30;
  int peer_row1 = 0;   // GEMM rows [peer_nt, M) -> global rows peer_row1 + m - peer_nt
};

// Fused a7 for the attention epilogue: output row g (global order [txt_0..txt_{k-1};
// img_0..img_{k-1}], Lt text rows) of local head hl goes to the rank p owning g, at its local row
// (txt: g - t_off[p]; img: nt[p] + g - Lt - i_off[p]) and column col0 + hl*D of dst[p] (row stride
// ld).  k = 0: plain output o[g*ldo + hl*D].
struct AttnScatter {
  int k = 0;
  int Lt = 0;
  int col0 = 0;
  long long ld = 0;
  bf16* dst[8];
  int t_off[9], i_off[9], nt[8];
};

struct GemmProblem {
  const bf16* A;
  long long lda;
  const bf16* W;
  long long ldw;
  int M;
  GemmEpi epi;
};

struct GemmPlan {
  int nprob = 1;
  CUtensorMap tmAq[GEMM_MAX_PROBLEMS], tmBq[GEMM_MAX_PROBLEMS];
  int Mq[GEMM_MAX_PROBLEMS] = {}, tile0[GEMM_MAX_PROBLEMS] = {};
  GemmEpi epiq[GEMM_MAX_PROBLEMS];
  int M = 0, N = 0, K = 0;
  int BN = 256;
  int tiles = 0, grid = 0;
  bool pair = false;  // CTA-pair (cta_group::2) 256 x 256 tiles
  int splits = 1;     // split-K factor (1-CTA tiles, fp32-accumulating epilogues only)
  int kps = 0;        // k-blocks (of 64) per split
  int* sem = nullptr; // split-K arrival counters, 4 per output tile, zero between launches
  float* ws = nullptr; // split-K partials
  int group_n = 16;    // rasterisation: weight-column tiles per group
  int serpentine = 1;  // odd groups walk the row blocks backwards (activation reuse across groups)
  GemmEpi epi;
};
// split-K workspace of one stream: counters (zeroed once, left zero by every launch) + partials
struct GemmSplitWs {
  int* sem = nullptr;
  int sem_ints = 0;
  float* ws = nullptr;
  long long ws_bytes = 0;
};

// A: [M, K] bf16 row stride lda (elements); W: [N, K] bf16 row stride ldw. K % 64 == 0, N % 64 == 0.
// Returns 0 on success, nonzero (and sets *err) on invalid arguments.
// sws: a split-K workspace (per stream: concurrent launches need their own) enables split-K for
// small launches with fp32-accumulating epilogues; force_splits > 0 requests that factor (tests).
// Null: no split-K.
int gemm_plan(GemmPlan* p, const bf16* A, long long lda, const bf16* W, long long ldw, int M, int N, int K,
              const GemmEpi& epi, int num_sms, const char** err, int force_bn = 0, int force_pair = -1,
              const GemmSplitWs* sws = nullptr, int force_splits = 0);
// One launch for up to GEMM_MAX_PROBLEMS problems sharing N and K (persistent tile loop over all;
// each problem has its own A, W and epilogue).
int gemm_plan_multi(GemmPlan* p, const GemmProblem* probs, int nprob, int N, int K, int num_sms, const char** err,
                    int force_bn = 0, int force_pair = -1, const GemmSplitWs* sws = nullptr,
                    int force_splits = 0);
void gemm_launch(const GemmPlan& p, cudaStream_t s);

// ------------------------------------------------------------------ elementwise / norm kernels
// u[m, :] = bf16( LN(x[m, :]) * (1 + scale) + shift ), x fp32 row stride ldx, u row stride ldu
void ln_mod_launch(const float* x, long long ldx, bf16* u, long long ldu, const float* shift, const float* scale,
                   int M, int h, cudaStream_t s);
// same, rows [0, n_first) modulated by (shift0, scale0), rows [n_first, M) by (shift1, scale1)
void ln_mod2_launch(const float* x, long long ldx, bf16* u, long long ldu, const float* shift0,
                    const float* scale0, const float* shift1, const float* scale1, int n_first, int M, int h,
                    cudaStream_t s);

extern int g_ln_impl;  // LN-modulate kernel choice: 0 CTA per row, 1 warp per row
// B blocks of rows_b rows (block b = rows [b*rows_b, (b+1)*rows_b)); inside a block rows [0, n_first)
// use (shift0, scale0), the rest (shift1, scale1); block b's vectors are offset by b * mstride floats.
void ln_mod2b_launch(const float* x, long long ldx, bf16* u, long long ldu, const float* shift0,
                     const float* scale0, const float* shift1, const float* scale1, int n_first, int rows_b, int B,
                     long long mstride, int h, cudaStream_t s);

// In-place on a qkv buffer [rows, 3*H*D] (row stride ld): q,k <- RoPE(RMSNorm(.) * g).
// Rows [0, n_first) use gains (gq0, gk0), rows [n_first, rows) use (gq1, gk1).
// cos/sin tables: [rows, D/2] fp32.
// If pack_out != null the result for all of q, k, v is instead written to the Ulysses send
// buffer pack_out laid out [k_sp][rows][3][H/k_sp][D] (bf16), and qkv is left unchanged.
void qk_norm_rope_launch(bf16* qkv, long long ld, int rows, int n_first, int H, int D, const bf16* gq0,
                         const bf16* gk0, const bf16* gq1, const bf16* gk1, const float* cosb, const float* sinb,
                         bf16* pack_out, int k_sp, cudaStream_t s);

// Joint attention, non-causal: O[l, h*D + d] = softmax(q k^T / sqrt(D)) v for heads h in [0, H).
// attention_launch: tcgen05/TMEM kernel (returns nonzero if the layout is not TMA-compatible, the
// version is unknown or the launch failed).  version <= 3: the default per head dim; 50 + n: n of 8
// exp2 pairs by polynomial (attention_tc.cu).
// q(l, h) at q + l*ldq + h*D (same for k, v, o). L rows.
// KV-split (flash-decoding style) for launches with too few CTAs to fill the GPU (SP = 4/8 head
// shards, small images): split s of a (query block, head) covers key tiles [s tps, (s+1) tps);
// each split stores its unnormalised O (fp32, [D][128] per query tile), reference m and sum l to ws
// and the last split of a query-tile warp (counter in cnt) merges them in split order.
struct AttnSplitWs {
  int* cnt = nullptr;   // zero on entry, left zero
  int cnt_ints = 0;
  float* ws = nullptr;
  long long ws_bytes = 0;
  int force = 0;        // > 0: this split factor (tests); 0: automatic
};
// the KV-split plan a launch would use (host only; sms <= 0: 148)
int attention_split_plan(int L, int H, int D, long long ws_bytes, int cnt_ints, int force, int sms, int* n_plain,
                         int* n_tail, int* nsplit, int* bounds);
int attention_launch(const bf16* q, long long ldq, const bf16* k, long long ldk, const bf16* v, long long ldv,
                     bf16* o, long long ldo, int L, int H, int D, cudaStream_t s, int version = 3,
                     const AttnScatter* scatter = nullptr, const AttnSplitWs* split = nullptr);

// dst[m, c] = bf16(src[m, c]) (fp32 -> bf16), row strides in elements
void f32_to_bf16_launch(const float* src, long long lds, bf16* dst, long long ldd, int M, int C, cudaStream_t s);
// dst[m, c] = bf16(silu(src[m, c]))
void silu_bf16_launch(const float* src, long long lds, bf16* dst, long long ldd, int M, int C, cudaStream_t s);
// dst[r, :] = src[r, :] copies of rows, 2D strided bf16 (used by Ulysses unpack)
void copy2d_bf16_launch(const bf16* src, long long lds, bf16* dst, long long ldd, int rows, int cols, cudaStream_t s);
// dst[m] = src[*idx_dev * stride + m] for m < n (fp32): per-step row selection inside a graph
void select_row_launch(const float* src, long long stride, const int* idx_dev, float* dst, long long n,
                       cudaStream_t s);

// Cross-process group barrier over CUDA-IPC flag windows (fused transport, one rank per process):
// member r bumps its epoch, stores it into every peer's flags[r] (release, system scope) and waits
// until every peer's epoch has arrived in its own flags (acquire).  Bounded wait: after ~10 s it
// records an error flag (flags[rank][62]) and returns instead of hanging.
struct IpcBarrier {
  int* flags[8];
  int k = 0;
  int rank = 0;
};
void ipc_barrier_launch(const IpcBarrier& b, cudaStream_t s);

// ------------------------------------------------------------------ per-shard position tables
// FLUX RoPE tables (S22: angles in fp64, stored fp32) of one shard's rows [txt (nt) ; img (ni)]:
// cos/sin [nt + ni, D/2]; text rows are position 0 (cos 1, sin 0); image row r is token
// p = i0 + r at (row p / wp, col p % wp) of the patch grid; pair i belongs to axis a (axes_dim
// split of D/2 pairs), theta_{p,i} = id_a(p) * theta^(-2j/d_a) with j the pair's index in its axis.
void rope_table_launch(float* cosb, float* sinb, int nt, long long i0, int ni, long long wp, int D,
                       const int axes_dim[3], double theta, cudaStream_t s);
// SD3 2-D sin-cos position embedding (fp64 -> fp32) of image rows [i0, i0 + ni): pe [ni, h], patch
// p at (pr, pc) = ((p / n_c + top) / q, (p % n_c + left) / q); channels [sin(pc w), cos(pc w),
// sin(pr w), cos(pr w)], w_j = 10000^(-j / (h/4)).
void sincos_pe_launch(float* pe, long long i0, int ni, long long n_c, long long top, long long left, double q, int h,
                      cudaStream_t s);

// ------------------------------------------------------------------ SYNTH-1 generator
// kind: 0 'w'/'b'/'x' (bf16 = rne(r*c)), 1 'g' (bf16 = rne(1 + r*c)), 2 'f' (fp32 = r*c)
void synth_launch(void* dst, uint64_t seed, uint32_t tensor_id, uint64_t idx0, long long n, int kind, float c,
                  cudaStream_t s);

}  // namespace tsv
