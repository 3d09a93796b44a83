/*
 * tsv.h — C-ABI of libtsv.so: one denoising step of a FLUX.1-dev-shaped MMDiT on one request's
 * latent, under step-level Ulysses sequence parallelism of degree k in {1, 2, 4, 8}.
 *
 * This is the computation TetriServe's scheduler allocates GPUs to (paper: "TetriServe:
 * Efficiently Serving Mixed DiT Workloads", ASPLOS '26; cited P:<line of PAPER.md>).  The calls
 * follow the paper's problem statement (§4.1):
 *   - a request has S_i dependent denoising steps; a step can start only after the
 *     previous one completed (step dependency);
 *   - each step runs on k GPUs, k a power of two, chosen per step (step-level SP, P:73,
 *     P:114), on a named GPU group (process groups pre-created);
 *   - between steps the latent is handed off between GPU groups through a Future-like handle
 *      -> tsv_request_reshard + tsv_event;
 *   - the scheduler consumes an offline-profiled step-latency table T(res, k)
 *     -> tsv_latency_table.
 * The DiT math itself is public FLUX.1-dev (the paper gives no equations); see
 * DESIGN.md for every reading taken where the paper is silent.
 *
 * Conventions
 *   - Every call returns tsv_status; no C++ exception crosses the ABI.  On failure the call sets
 *     a thread-local message readable with tsv_last_error() (valid until the next call on the
 *     same thread).
 *   - The engine owns all device memory (weights, latent shards, workspaces, communicators).
 *     The caller owns every host buffer it passes; host pointers are only read/written during
 *     the call (copies are synchronous with respect to the caller).
 *   - Handles are plain integers.  Requests are destroyed explicitly, events may be released
 *     (tsv_event_release); groups live as long as the engine.
 *   - Ranks.  An engine hosts "slots" = global SP ranks [rank_base, rank_base + n_local) on the
 *     listed CUDA devices (a device may repeat: virtual ranks on one GPU, used by the
 *     single-GPU SP tests).  world_size is the total number of ranks over all processes.  One
 *     process per GPU (torchrun) uses n_local = 1, rank_base = RANK, world_size = WORLD_SIZE.
 *   - Thread safety: one control thread per engine.
 *
 * SYNTH-1 (seeded synthetic weights and inputs; restated independently in synth/__init__.py)
 *   key = seed ^ (tensor_id << 48) ^ idx;  h = splitmix64_mix(key + 0x9E3779B97F4A7C15);
 *   u = h >> 40;  r = float32((u - 2^23) * 2^-23) in [-1, 1)
 *   bf16 kinds: val = bf16_rne(float32(r * c)), c = float32(sqrt(3) * sigma):
 *       weights sigma = 1/sqrt(fan_in), biases sigma = 0.02, inputs T, y sigma = 1;
 *   RMSNorm gains: val = bf16_rne(float32(1 + float32(r * float32(sqrt(3) * 0.1))));
 *   latent x_T (fp32): val = float32(r * float32(sqrt(3))).
 *   Weight seed: the engine's weight_seed; input seed: the request's seed.
 *
 * Tensor ids (SYNTH-1 tensor_id; h = hidden, D = head_dim, F = mlp_hidden, in = in_ch):
 *   global   0 img_in.w [h,in]  1 img_in.b [h]  2 txt_in.w [h,ctx]  3 txt_in.b [h]
 *            4 time_in.in.w [h,256] 5 .b  6 time_in.out.w [h,h] 7 .b
 *            8 guidance_in.in.w [h,256] 9 .b  10 guidance_in.out.w [h,h] 11 .b
 *            12 vector_in.in.w [h,vec] 13 .b  14 vector_in.out.w [h,h] 15 .b
 *            16 final.mod.w [2h,h] 17 final.mod.b [2h]  18 final.lin.w [in,h] 19 final.lin.b [in]
 *   double block j, stream s (0 = img, 1 = txt): base = 64 + 32 j + 16 s
 *            +0 mod.w [6h,h] +1 mod.b [6h] +2 qkv.w [3h,h] +3 qkv.b [3h] +4 q_norm.g [D]
 *            +5 k_norm.g [D] +6 proj.w [h,h] +7 proj.b [h] +8 fc1.w [F,h] +9 fc1.b [F]
 *            +10 fc2.w [h,F] +11 fc2.b [h]
 *   single block j: base = 4096 + 16 j
 *            +0 mod.w [3h,h] +1 mod.b [3h] +2 lin1.w [3h+F,h] +3 lin1.b [3h+F] +4 q_norm.g [D]
 *            +5 k_norm.g [D] +6 lin2.w [h,h+F] +7 lin2.b [h]
 *   request inputs: 1 x_T [L_i,in] (fp32)  2 T [L_t,ctx] (bf16)  3 y [vec] (bf16)
 *
 * SD3 family (family = TSV_FAMILY_SD3): the same ids where the tensor exists.  Globals 0-7 and
 * 12-19 (no guidance embedder; img_in = the 2x2 patch-embed conv flattened in (c, ph, pw) order;
 * final.mod rows are (scale, shift)).  Joint block j, stream s: the double-block ids without the
 * QK-norm gains (+4, +5); qkv.w stacks to_q; to_k; to_v (img) or add_q; add_k; add_v (txt).  The
 * txt stream of the last block is context_pre_only: +0 mod.w [2h,h] (scale, shift), +1 mod.b
 * [2h], +2 qkv.w, +3 qkv.b only.  Request inputs: 1 x_T, 2 T_c, 3 y_c (conditional branch),
 * 4 T_u [L_t,ctx], 5 y_u [vec] (unconditional branch of the CFG pair).
 */
#ifndef TSV_H_
#define TSV_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  TSV_OK = 0,
  TSV_E_INVAL = -1,       /* bad argument (shape, k not a power of two, rank outside the engine...) */
  TSV_E_STATE = -2,       /* violates step dependency or handle in the wrong state */
  TSV_E_OOM = -3,         /* device allocation failed */
  TSV_E_CUDA = -4,        /* CUDA runtime / launch error */
  TSV_E_NCCL = -5,        /* NCCL error */
  TSV_E_UNSUPPORTED = -6  /* valid but not supported (e.g. k does not divide the head count) */
} tsv_status;

typedef struct tsv_engine tsv_engine; /* opaque */
typedef int64_t tsv_request;
typedef int32_t tsv_group;
typedef int64_t tsv_event;

/* Caller-supplied device allocator (tsv_engine_set_allocator).  alloc returns `bytes` of device
 * memory on `device` usable in stream order on `stream` (a cudaStream_t), or NULL on failure;
 * free returns a pointer obtained from alloc with the same device and stream.  The engine calls
 * free only once every use of the buffer is ordered before `stream`'s current position (same
 * contract as cudaFreeAsync / PyTorch's caching allocator).  Both are called from the thread
 * that makes the engine call. */
typedef void* (*tsv_alloc_fn)(void* ctx, size_t bytes, int device, void* stream);
typedef void (*tsv_free_fn)(void* ctx, void* ptr, int device, void* stream);

typedef struct {
  int hidden;        /* h: 3072 for FLUX.1-dev */
  int heads;         /* H: 24 */
  int head_dim;      /* D: 128 (64 or 128 supported) */
  int mlp_hidden;    /* F: 12288 */
  int n_double;      /* 19 double-stream blocks */
  int n_single;      /* 38 single-stream blocks */
  int in_ch;         /* 64: packed 16-channel latent with 2x2 patches */
  int ctx_dim;       /* 4096: T5 context width */
  int vec_dim;       /* 768: pooled CLIP width */
  int text_tokens;   /* L_t: 512 */
  int axes_dim[3];   /* RoPE axes split of D: (16, 56, 56) */
  float theta;       /* RoPE base: 10000 */
  int guidance_embed;/* 1: FLUX-dev guidance embedder present */
  int family;        /* TSV_FAMILY_FLUX (double + single blocks, QK-RMSNorm, 3-axis RoPE) or
                        TSV_FAMILY_SD3 (SD3-medium MMDiT: joint blocks only, no QK-norm, no RoPE,
                        2-D sin-cos position embedding, context_pre_only last block, CFG pair;
                        DESIGN.md O-SD3).  axes_dim / theta / guidance_embed are ignored for SD3. */
  float cfg_scale;   /* SD3: classifier-free guidance scale s (7.0): v = v_u + s (v_c - v_u) */
  float shift;       /* SD3: flow-matching schedule shift (3.0): t_j = s u / (1 + (s - 1) u), u = 1 - j/S */
  int pe_max;        /* SD3: pos_embed_max_size (192) */
  int pe_base;       /* SD3: base_size (64); patch (r, c) sits at ((r + top) pe_base / pe_max, ...) */
} tsv_model_desc;

#define TSV_FAMILY_FLUX 0
#define TSV_FAMILY_SD3 1

/* Named presets: "flux" (FLUX.1-dev shapes), "tiny" (config 1: h=256, H=4, D=64, F=1024,
 * 1 double block, L_t=64), "tiny_s" (tiny + 1 single block), "tiny2" (2 double + 2 single),
 * "sd3" (SD3-medium shapes, config 5: h=1536, H=24, D=64, F=6144, 24 joint blocks, L_t=333,
 * ctx 4096, pooled 2048, CFG 7, shift 3) and "tiny_sd3" (h=256, H=4, 2 joint blocks, L_t=77). */
tsv_status tsv_model_preset(const char* name, tsv_model_desc* out);

/* Create an engine hosting global ranks [rank_base, rank_base + n_local) on devices[0..n_local).
 * Device state is set up lazily, on the first call that needs it (tsv_group_create,
 * tsv_debug_read_weight): streams, then all weights on every distinct device with SYNTH-1
 * (weight_seed), so that tsv_engine_set_allocator / tsv_engine_set_stream can come first.
 * Errors: TSV_E_INVAL (bad desc / ranks / device), TSV_E_CUDA. */
tsv_status tsv_engine_create(const tsv_model_desc* model, const int* devices, int n_local, int rank_base,
                             int world_size, uint64_t weight_seed, tsv_engine** out);
void tsv_engine_destroy(tsv_engine* eng);

/* Optional PyTorch hooks (north_star: "PyTorch is used only for device memory, streams and process
 * groups"; S:§8(b) conventions).  Both must be called before the engine's device state exists (before
 * the first tsv_group_create), else TSV_E_STATE.
 * tsv_engine_set_allocator: every device buffer of the engine except CUDA-IPC windows (weights,
 * workspaces, per-request latents / modulation tables / tables) comes from alloc_fn and goes back
 * through free_fn (see tsv_alloc_fn for the ordering contract); the engine never calls cudaMalloc
 * for them.  Per-request buffers are allocated on the stream of the rank that uses them and
 * released stream-ordered on that stream.  Without a caller allocator the engine uses cudaMalloc
 * for engine-lifetime buffers and cudaMallocAsync / cudaFreeAsync for per-request ones.
 * Errors: TSV_E_INVAL (NULL function), TSV_E_STATE.
 * tsv_engine_set_stream: every rank hosted on `device` issues its kernels, copies and collectives
 * on `cuda_stream` (a cudaStream_t the caller owns and keeps alive while the engine exists),
 * instead of an engine-created non-blocking stream; virtual ranks on that device then share it
 * (they run serialised).  Errors: TSV_E_INVAL (device not in the engine), TSV_E_STATE. */
tsv_status tsv_engine_set_allocator(tsv_engine* eng, void* ctx, tsv_alloc_fn alloc_fn, tsv_free_fn free_fn);
tsv_status tsv_engine_set_stream(tsv_engine* eng, int device, void* cuda_stream);

/* Multi-process only: NCCL unique id (128 bytes) to be broadcast by the caller (e.g. with
 * torch.distributed) to every member of a group, and the world communicator used by reshard
 * between processes.  tsv_engine_init_world is collective over all world_size ranks. */
tsv_status tsv_nccl_unique_id(uint8_t out[128]);
tsv_status tsv_engine_init_world(tsv_engine* eng, const uint8_t nccl_id[128]);

/* Create a GPU group of k ranks (k in {1,2,4,8}, k a power of two); group rank = position
 * in `ranks`.  Arbitrary subsets of the engine's world are allowed (S14).  If every rank is
 * local, nccl_id may be NULL (in-process transport: peer copies); otherwise nccl_id is the
 * group's unique id and the call is collective over the group's processes.  The communicator is
 * created and warmed once here.  Errors: TSV_E_INVAL (k not a power of two, duplicate or
 * out-of-range rank), TSV_E_UNSUPPORTED (k does not divide the head count, S24), TSV_E_NCCL. */
tsv_status tsv_group_create(tsv_engine* eng, const int* ranks, int k, const uint8_t* nccl_id, tsv_group* out);

/* Create a request: height/width in pixels (multiples of 16, L_i = (H/16)(W/16)),
 * num_steps S >= 1, guidance g (FLUX guidance embedding; ignored for SD3, whose guidance is the
 * model's cfg_scale).  Inputs x_T, T, y are SYNTH-1 from `seed` (tensor ids 1-3; SD3 also 4-5)
 * and held in host memory until the first step lands on a group.  Errors: TSV_E_INVAL. */
tsv_status tsv_request_create(tsv_engine* eng, int height_px, int width_px, int num_steps, uint64_t seed,
                              float guidance, tsv_request* out);

/* Replace the request's inputs before its first step: x [L_i*in] fp32 row-major, T [L_t*ctx]
 * bf16 bits, y [vec] bf16 bits.  SD3: T is [2][L_t*ctx] = (T_c, T_u) and y is [2][vec] =
 * (y_c, y_u).  Any pointer may be NULL (keeps the current value).
 * Errors: TSV_E_STATE if a step already ran. */
tsv_status tsv_request_set_inputs(tsv_engine* eng, tsv_request req, const float* x, const uint16_t* T,
                                  const uint16_t* y);

/* Run denoising step `step` of `req` on `group`:  v = DiT(x_s, t_s, T, y, g),
 * x_{s+1} = x_s + (t_{s+1} - t_s) v  (flow-matching Euler; schedule t_j = sigma(1 - j/S),
 * DESIGN.md).  SD3: v = v_u + s (v_c - v_u) over the CFG pair, both branches in the same
 * launches (batch 2, S23).  `step` must equal the request's next step else TSV_E_STATE; if the
 * group differs from the request's current group, the latent is resharded first (timed
 * separately).  Asynchronous: `done` (may be NULL) completes when every rank of the group
 * finished.  Multi-process: every process hosting a rank of the group makes the call; processes
 * with no rank in the group return TSV_OK without work (done = -1).  Errors: TSV_E_INVAL,
 * TSV_E_STATE, TSV_E_CUDA, TSV_E_NCCL. */
tsv_status tsv_request_step(tsv_engine* eng, tsv_request req, int step, tsv_group group, tsv_event* done);

/* Selective batching (S:§8(f) NEXT #3): run the NEXT step of each of the n requests
 * (each at its own step index, schedule and inputs) as ONE batched step on `group` — every GEMM,
 * LN and all-to-all launch covers all of them (per-request modulation, latents and Euler), attention
 * runs per request.  The requests must share the resolution; they are moved (resharded) onto the
 * group first if needed.  n <= 8 for FLUX, <= 4 for SD3 (whose requests are CFG pairs).  Results
 * equal n separate tsv_request_step calls (same arithmetic per row).  Errors: TSV_E_INVAL (unknown
 * or repeated request, mixed resolutions, n out of range), TSV_E_STATE (a request has no step left),
 * TSV_E_CUDA, TSV_E_NCCL. */
tsv_status tsv_request_step_batch(tsv_engine* eng, const tsv_request* reqs, int n, tsv_group group, tsv_event* done);

/* Move the latent of `req` to `group` without running a step: bit-exact row moves given by the
 * reshard map (tsv_reshard_plan).  Asynchronous and non-blocking (P:409's "asynchronous,
 * non-blocking" hand-off): the row copies are ordered after the request's last step on the old
 * ranks, the new ranks' streams wait for them, and the old shards are released stream-ordered; the
 * host does not wait for the device.  On a GPU the request never ran on, its per-request state is
 * set up too: the text rows (pinned host -> device) and their embedding, the RoPE / position
 * tables (computed on the device), and the modulation table of all steps — copied from another
 * local rank that already holds it, else computed (one M = S GEMM). */
tsv_status tsv_request_reshard(tsv_engine* eng, tsv_request req, tsv_group group, tsv_event* done);

/* Events (the latent "future").  For a group using CUDA-IPC windows, wait / query /
 * elapsed also check the group's device barrier: a member that stalled for ~10 s made the barrier
 * give up, and the call then returns TSV_E_STATE (the step's results are invalid; the group must
 * be recreated). */
tsv_status tsv_event_wait(tsv_engine* eng, tsv_event ev);
/* Release an event handle (a serving loop releases each step's event once it is done with it); the
 * handle may be returned again by a later call.  Waiting on a released handle: TSV_E_INVAL. */
tsv_status tsv_event_release(tsv_engine* eng, tsv_event ev);
tsv_status tsv_event_query(tsv_engine* eng, tsv_event ev, int* done);
/* Device time between two events of the same group, max over the group's local ranks (ms). */
tsv_status tsv_event_elapsed_ms(tsv_engine* eng, tsv_event start, tsv_event end, float* ms);
tsv_status tsv_group_record(tsv_engine* eng, tsv_group group, tsv_event* out);

/* Latent rows [row0, row0 + nrows) of x_s ([L_i, in] fp32, row-major; in multi-process mode only
 * rows held by local ranks).  Before the first step these are the host inputs.  read waits for
 * the request's pending work.  Errors: TSV_E_INVAL (rows not local / out of range). */
tsv_status tsv_request_read_latent(tsv_engine* eng, tsv_request req, int64_t row0, int64_t nrows, float* host);
tsv_status tsv_request_write_latent(tsv_engine* eng, tsv_request req, int64_t row0, int64_t nrows,
                                    const float* host);
/* Velocity v of the last completed step, same row convention. */
tsv_status tsv_request_read_velocity(tsv_engine* eng, tsv_request req, int64_t row0, int64_t nrows, float* host);
/* Next step index, current group (-1 before the first step), and L_i. */
tsv_status tsv_request_info(tsv_engine* eng, tsv_request req, int* next_step, tsv_group* group, int64_t* image_tokens);
tsv_status tsv_request_destroy(tsv_engine* eng, tsv_request req);

/* Offline step-latency table: for each (res_px[i], ks[j]) runs `warmup` untimed and `iters`
 * timed steps of a square res x res request on the group of the first ks[j] engine ranks and
 * writes the median step latency (ms, max over ranks) to ms_out[i*n_k + j] and its coefficient
 * of variation (stddev/mean) to cv_out[i*n_k + j].  Collective in multi-process
 * mode (requires tsv_engine_init_world).  Entries with k > world_size are set to -1. */
tsv_status tsv_latency_table(tsv_engine* eng, const int* res_px, int n_res, const int* ks, int n_k, int warmup,
                             int iters, double* ms_out, double* cv_out);

/* Index maps, exported for tests (S:§8(c) O-SP): rank r of k owns rows [begin, end) with
 * begin = r*floor(n/k) + min(r, n mod k).  Reshard plan k_src -> k_dst: up to max_copies
 * entries of 5 int64 (src_rank, src_row0, dst_rank, dst_row0, rows); *n_copies <= k_src+k_dst-1. */
tsv_status tsv_shard_range(int64_t n_rows, int k, int rank, int64_t* begin, int64_t* end);
tsv_status tsv_reshard_plan(int64_t n_rows, int k_src, int k_dst, int64_t* out, int max_copies, int* n_copies);

/* Ulysses all-to-all plan of rank `rank` in a group of k (S:§8(a) a5/a7), as the step
 * executes it: up to max_ops entries of 4 int64 (peer, is_send, row0, rows).  which = 1 (seq ->
 * head): sends read the pack buffer [k][rows_rank] rows, receives write the [L] rows of the
 * attention input in global order [txt_0..txt_{k-1}; img_0..img_{k-1}]; which = 2 (head -> seq):
 * sends read the [L] attention-output rows, receives write [k][rows_rank].  Sends and receives
 * between two ranks match in plan order.  Row widths: 3h/k (which = 1), h/k (which = 2). */
tsv_status tsv_a2a_plan(int which, int64_t text_rows, int64_t image_rows, int k, int rank, int64_t* out, int max_ops,
                        int* n_ops);

/* Debug / parity: copy weight tensor `tensor_id` (bf16 bits) from the device of local slot 0. */
tsv_status tsv_debug_read_weight(tsv_engine* eng, int tensor_id, uint16_t* host, size_t n);
/* Per-kernel-class device-time profiling: when enabled, every launch is bracketed by CUDA events
 * on its launching stream.  Classes (TSV_PROF_CLASSES = 6): 0 GEMM, 1 attention, 2 LN-modulate,
 * 3 QK-norm+RoPE(+pack), 4 all-to-all / transfers, 5 other (casts, unpack).  enable != 0 also
 * resets the counters.  profile_read synchronises and writes 6 entries to each non-NULL array:
 * summed device ms, launches, algorithmic FLOPs and algorithmic HBM bytes per class. */
#define TSV_PROF_CLASSES 6
tsv_status tsv_engine_profile(tsv_engine* eng, int enable);
/* When a group has exactly one rank in this process, each step is captured once as a CUDA graph
 * (per request, group and buffer set) and replayed for later steps; the step index is read from
 * device memory, so one graph serves every step.  enable = 0 launches kernels directly.  Default
 * on; with profiling on, the profiled graph carries an event pair around every launch. */
tsv_status tsv_engine_set_graphs(tsv_engine* eng, int enable);

/* Ulysses transport of groups whose ranks all live in this process (S:§8(f) NEXT #2):
 *   TSV_TRANSPORT_FUSED (default): the all-to-alls are fused into the producers' epilogues —
 *     the QKV GEMM stores each head block's q|k|v straight into the owning rank's attention input
 *     ([L][3][H/k][D], global row order) and the attention kernel stores each output row straight
 *     into the owning rank's [txt_r; img_r] activation rows; a stream barrier (events) per exchange
 *     point is all that is left of the collective.  Stores go to peer memory over NVLink when the
 *     ranks are on different GPUs (peer access is enabled at engine creation).
 *   TSV_TRANSPORT_EXCHANGE: pack buffer + explicit exchange (peer copies in-process; NCCL
 *     send/recv across processes) + unpack — the baseline, bit-identical results.
 * Groups spanning processes use NCCL (exchange) unless their members exchanged CUDA-IPC windows
 * (tsv_group_ipc_export / _import below), then the fused stores go straight into the other
 * processes' windows and a device-side flag barrier replaces each all-to-all.  Errors: TSV_E_INVAL. */
#define TSV_TRANSPORT_EXCHANGE 0
#define TSV_TRANSPORT_FUSED 1
tsv_status tsv_engine_set_transport(tsv_engine* eng, int mode);

/* Fused transport across processes (one rank per process; S:§8(f) NEXT #2).  Collective over the
 * group's members, in this order:
 *   1. every member calls tsv_group_ipc_export: allocates its windows — the attention input
 *      [max_evals][max_tokens][3][H/k][D] bf16, the activation rows [max_evals][max_tokens/k + 2]
 *      [h + F] bf16 and 256 barrier flags — and writes an opaque blob (out = NULL: *len = blob
 *      size); max_tokens >= L_t + L_i of every request the group will run, max_evals >= requests
 *      per batch x CFG branches (<= 8);
 *   2. the caller all-gathers the k blobs (e.g. torch.distributed), concatenated in group-rank order;
 *   3. every member calls tsv_group_ipc_import, which maps the peers' windows (cudaIpcOpenMemHandle).
 * Afterwards steps on the group (with TSV_TRANSPORT_FUSED) need no NCCL communicator: the QKV and
 * attention epilogues store into the owners' windows and a device barrier orders the members (a
 * stalled peer makes the barrier give up after ~10 s instead of hanging; the next tsv_event_wait /
 * _query / _elapsed_ms on the group then returns TSV_E_STATE).  Groups may then be
 * created without nccl_id or a world communicator.  Errors: TSV_E_INVAL (sizes, foreign blob),
 * TSV_E_STATE (import before export), TSV_E_UNSUPPORTED (group not spanning processes), TSV_E_CUDA. */
tsv_status tsv_group_ipc_export(tsv_engine* eng, tsv_group group, int64_t max_tokens, int max_evals, uint8_t* out,
                                size_t* len);
tsv_status tsv_group_ipc_import(tsv_engine* eng, tsv_group group, const uint8_t* blobs, size_t blob_len);
tsv_status tsv_engine_profile_read(tsv_engine* eng, double* ms, int64_t* launches, double* flops, double* bytes);
/* Number of kernels this engine launched so far (all slots). */
tsv_status tsv_engine_kernel_count(tsv_engine* eng, int64_t* count);

const char* tsv_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* TSV_H_ */
