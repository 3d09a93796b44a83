// libtsv.so engine: weights, GPU groups, requests, the denoising step under Ulysses SP, reshard,
// events and the step-latency table.  Implements include/tsv.h.
//
// Step (S:§8(a), per rank r of a group of k; rows of rank r = [txt_r ; img_r]):
//   a1 embed      img = x_s W_img^T + b (latent cast to bf16), txt = T W_txt^T + b    -> x fp32
//   double j      per stream: a2 LN-mod -> a3 QKV GEMM -> a4 QK-RMSNorm+RoPE(+pack) ->
//                 a5 a2a #1 -> a6 attention -> a7 a2a #2 -> (unpack) -> a8 proj + gated residual
//                 -> a9 LN-mod -> fc1+GELU -> fc2 + gated residual
//   single j      a2 LN-mod -> linear1 (qkv | GELU(mlp)) -> a4 -> a5 -> a6 -> a7 -> linear2 + gated residual
//   final         a2 LN-mod(img rows) -> a11 linear -> a12 Euler x += dt v (GEMM epilogue)
// Conditioning (a0) runs once per (request, GPU): vec_s for all steps, then the modulation table
// mod[s] = W_mod SiLU(vec_s) + b as one [S, n_mod] GEMM.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <tuple>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include <cuda_runtime.h>
#include <nccl.h>

#include "../../include/tsv.h"
#include "../../include/tsv_ops.h"
#include "kernels.h"
#include "model.h"

namespace tsv {

// ------------------------------------------------------------------ errors
static thread_local std::string g_err;
static tsv_status fail(tsv_status s, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}
#define CK(call)                                                                                  \
  do {                                                                                            \
    cudaError_t e_ = (call);                                                                      \
    if (e_ != cudaSuccess)                                                                        \
      return fail(e_ == cudaErrorMemoryAllocation ? TSV_E_OOM : TSV_E_CUDA, "%s:%d %s: %s", __FILE__, \
                  __LINE__, #call, cudaGetErrorString(e_));                                       \
  } while (0)
#define NK(call)                                                                                   \
  do {                                                                                             \
    ncclResult_t r_ = (call);                                                                      \
    if (r_ != ncclSuccess)                                                                         \
      return fail(TSV_E_NCCL, "%s:%d %s: %s", __FILE__, __LINE__, #call, ncclGetErrorString(r_)); \
  } while (0)
#define TRY(expr)                 \
  do {                            \
    tsv_status s_ = (expr);       \
    if (s_ != TSV_OK) return s_;  \
  } while (0)

// TSV_TRACE=1: host-side timestamps of the landing / reshard phases on stderr (diagnostics)
static void trace(const char* what) {
  static const bool on = getenv("TSV_TRACE") && atoi(getenv("TSV_TRACE"));
  if (!on) return;
  static auto t0 = std::chrono::steady_clock::now();
  const auto t = std::chrono::steady_clock::now();
  fprintf(stderr, "[tsv trace] %10.3f ms  %s\n", std::chrono::duration<double, std::milli>(t - t0).count(), what);
}

static int64_t shard_begin(int64_t n, int k, int r) { return (int64_t)r * (n / k) + std::min<int64_t>(r, n % k); }

// ------------------------------------------------------------------ SYNTH-1 on the host (request inputs)
static inline uint64_t sm64_mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static inline float synth_r(uint64_t seed, uint32_t tid, uint64_t idx) {
  const uint64_t h = sm64_mix((idx ^ (seed ^ ((uint64_t)tid << 48))) + 0x9E3779B97F4A7C15ull);
  return (float)((int)(h >> 40) - (1 << 23)) * (1.0f / 8388608.0f);
}
static inline uint16_t f32_to_bf16_bits(float f) {
  uint32_t b;
  memcpy(&b, &f, 4);
  b = (b + 0x7FFFu + ((b >> 16) & 1u)) >> 16;
  return (uint16_t)b;
}
static inline float bf16_bits_to_f32(uint16_t u) {
  uint32_t b = (uint32_t)u << 16;
  float f;
  memcpy(&f, &b, 4);
  return f;
}

// ------------------------------------------------------------------ device buffers
// Where device memory comes from (tsv_engine_set_allocator): the caller's allocator (e.g. PyTorch's
// caching allocator), or CUDA.  Buffers are allocated and released *stream-ordered* on the stream
// that uses them (kind STREAM: cudaMallocAsync / cudaFreeAsync, or the caller's allocator with that
// stream), so landing and resharding a request never block the host; engine-lifetime buffers
// (weights, workspaces) are plain allocations (kind STATIC).  IPC windows always use cudaMalloc
// (kind RAW: cudaIpcGetMemHandle needs an allocation of its own).
struct Allocator {
  void* ctx = nullptr;
  tsv_alloc_fn alloc = nullptr;
  tsv_free_fn free = nullptr;
};
enum AllocKind { AK_STATIC = 0, AK_STREAM = 1, AK_RAW = 2 };
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  int device = -1;
  int kind = AK_STATIC;
  const Allocator* al = nullptr;   // the caller's allocator (nullptr: CUDA)
  cudaStream_t stream = nullptr;   // the stream it was allocated on (ordering of the release)
  // release on the allocation stream; the caller guarantees every use of the buffer is ordered
  // before the stream's current position (stream-ordered kinds) or has completed (STATIC / RAW)
  void release() {
    if (p) {
      int cur;
      cudaGetDevice(&cur);
      cudaSetDevice(device);
      if (al && kind != AK_RAW) al->free(al->ctx, p, device, stream);
      else if (kind == AK_STREAM) cudaFreeAsync(p, stream);
      else cudaFree(p);
      cudaSetDevice(cur);
    }
    p = nullptr;
    bytes = 0;
  }
};
static tsv_status dev_alloc(DevBuf& b, int device, size_t bytes, const Allocator* al = nullptr, int kind = AK_RAW,
                            cudaStream_t stream = nullptr) {
  if (b.p && b.bytes >= bytes && b.device == device) return TSV_OK;
  b.release();
  if (bytes == 0) return TSV_OK;
  CK(cudaSetDevice(device));
  void* p = nullptr;
  if (al && kind != AK_RAW) {
    p = al->alloc(al->ctx, bytes, device, stream);
    if (!p) return fail(TSV_E_OOM, "caller allocator returned NULL for %zu bytes on device %d", bytes, device);
  } else {
    cudaError_t e = kind == AK_STREAM ? cudaMallocAsync(&p, bytes, stream) : cudaMalloc(&p, bytes);
    if (e != cudaSuccess)
      return fail(TSV_E_OOM, "cudaMalloc%s(%zu) on device %d: %s", kind == AK_STREAM ? "Async" : "", bytes, device,
                  cudaGetErrorString(e));
  }
  b.p = p;
  b.bytes = bytes;
  b.device = device;
  b.kind = kind;
  b.al = al && kind != AK_RAW ? al : nullptr;
  b.stream = stream;
  return TSV_OK;
}

struct DeviceState {
  int device = -1;
  int num_sms = 148;
  DevBuf weights;  // bf16 blob
};

struct Workspace {
  DevBuf x, u, qkv, cat, hbuf, latb, pack, recv, obuf, orecv;
  DevBuf bmod;  // fp32 [B][n_mod] this step's modulation rows of every evaluation, then B dt values
};

// A captured step graph (per slot; keyed by every buffer pointer, group, batch and profiling flag)
struct ProfRec {
  int cls;
  int device;
  cudaEvent_t a, b;
};
struct StepGraph {
  cudaGraphExec_t exec = nullptr;
  int64_t kernels = 0;
  std::vector<int64_t> reqs;          // requests whose buffers the graph references
  std::vector<ProfRec> prof;          // profiled graphs: the event pairs recorded at every replay
  double flops[8] = {0}, bytes[8] = {0};
  int64_t launch[8] = {0};
  uint64_t last_use = 0;
};

struct Slot {
  int rank = -1;
  int device = -1;
  DeviceState* ds = nullptr;
  cudaStream_t stream = nullptr;
  bool own_stream = true;  // false: shares another slot's stream (TSV_VIRTUAL_SERIAL)
  Workspace ws;
  DevBuf scratch;  // conditioning temporaries
  DevBuf sem;      // split-K arrival counters of this slot's GEMM launches (zero between launches)
  DevBuf splitws;  // split-K partials
  AttnSplitWs aws() const {   // the attention's KV split reuses the GEMM split-K buffers (same stream)
    AttnSplitWs w;
    w.cnt = reinterpret_cast<int*>(sem.p);
    w.cnt_ints = (int)(sem.bytes / sizeof(int));
    w.ws = reinterpret_cast<float*>(splitws.p);
    w.ws_bytes = (long long)splitws.bytes;
    return w;
  }
  GemmSplitWs sws() const {
    GemmSplitWs w;
    w.sem = reinterpret_cast<int*>(sem.p);
    w.sem_ints = (int)(sem.bytes / sizeof(int));
    w.ws = reinterpret_cast<float*>(splitws.p);
    w.ws_bytes = (long long)splitws.bytes;
    return w;
  }
  std::map<uint64_t, StepGraph> graphs;
};
constexpr int SEM_INTS = 4096;
constexpr size_t SPLIT_WS_BYTES = 128u << 20;
// TSV_GEMM_BN / TSV_GEMM_PAIR (read at engine creation): force the step GEMMs' tile width / CTA
// pairing (planner A/B measurements only; 0 / -1 = the planner's choice)
static int gemm_force_env(const char* name, int dflt) {
  const char* v = getenv(name);
  return v ? atoi(v) : dflt;
}
// TSV_SPLITK=0 (read at engine creation) disables split-K for small GEMM launches (A/B measurements)
static bool splitk_env() {
  const char* v = getenv("TSV_SPLITK");
  return v ? atoi(v) != 0 : true;
}

// per (request, slot): state that depends only on the request
// Page-locked host memory (inputs and staging of host-computed values): host->device copies from
// it are truly asynchronous (a pageable source makes cudaMemcpyAsync wait for the stream's prior
// work before staging).
template <class T>
struct Pinned {
  T* p = nullptr;
  size_t n = 0;
  Pinned() = default;
  Pinned(const Pinned&) = delete;
  Pinned& operator=(const Pinned&) = delete;
  Pinned(Pinned&& o) noexcept : p(o.p), n(o.n) { o.p = nullptr; o.n = 0; }
  Pinned& operator=(Pinned&& o) noexcept {
    if (this != &o) { reset(); p = o.p; n = o.n; o.p = nullptr; o.n = 0; }
    return *this;
  }
  ~Pinned() { reset(); }
  void reset() {
    if (p) cudaFreeHost(p);
    p = nullptr;
    n = 0;
  }
  tsv_status alloc(size_t count) {
    reset();
    if (!count) return TSV_OK;
    void* q = nullptr;
    cudaError_t e = cudaHostAlloc(&q, count * sizeof(T), cudaHostAllocPortable);
    if (e != cudaSuccess) return fail(TSV_E_OOM, "cudaHostAlloc(%zu): %s", count * sizeof(T), cudaGetErrorString(e));
    p = static_cast<T*>(q);
    n = count;
    return TSV_OK;
  }
  T* data() { return p; }
  const T* data() const { return p; }
  size_t size() const { return n; }
};

struct ReqDev {
  DevBuf mod;       // fp32 [S * B_model, n_mod]
  DevBuf dt;        // fp32 [S]
  DevBuf step;      // int: the step index the next launch runs
  Pinned<uint8_t> stage;          // host-computed conditioning inputs until their copies complete
  cudaEvent_t ready_ev = nullptr; // mod / dt complete (recorded on the slot's stream)
  bool ready = false;
};
// per (request, slot, shard layout): the constant, position-dependent state of a shard -- kept for
// the request's lifetime, so a request returning to a rank in the same position (k, rank) reuses it
// and a reshard then moves only the latent rows (P:409's latent hand-off)
struct ShardAux {
  DevBuf T, cosb, sinb;
  DevBuf pe;   // SD3: fp32 [ni, h] sin-cos position embedding of this shard's image rows
  DevBuf txt;  // fp32 [branches][nt, h]: a1 text embedding T W^T + b (constant per request,
               // computed when the layout first lands, copied into the residual stream every step)
  void release() { T.release(); cosb.release(); sinb.release(); pe.release(); txt.release(); }
};
// per (request, slot, shard): the latent state of the current group position
struct ReqShard {
  int rank_in_group = 0, k = 1;
  int64_t t0 = 0, nt = 0, i0 = 0, ni = 0;  // txt rows [t0, t0+nt), img rows [i0, i0+ni)
  DevBuf lat, vel;
  ShardAux* ax = nullptr;                  // owned by Request::aux
  void release() {
    lat.release(); vel.release();
  }
};

struct Group {
  std::vector<int> ranks;  // global ranks, position = group rank
  int k = 1;
  bool all_local = true;
  std::vector<int> local_slots;      // slot index per local member (same order as ranks filtered)
  std::vector<int> local_positions;  // group rank of each local member
  ncclComm_t comm = nullptr;         // multi-process transport (one local rank)
  std::vector<cudaEvent_t> ev_a, ev_b;  // per local member, for in-process all-to-all ordering
  // cross-process fused transport (CUDA IPC windows; tsv_group_ipc_export / _import): this rank's
  // attention-input and activation windows, mapped into every member, and barrier flags
  bool ipc = false;
  int64_t win_tokens = 0;
  int win_evals = 0;
  DevBuf win_recv, win_cat, win_flags;
  bool ipc_failed = false;  // the device barrier gave up on a stalled member (check_ipc_barrier)
  // multi-stream step graphs (several local ranks on their own streams): fork / join events per
  // local member, and a switch-off if capturing this group's step ever failed
  std::vector<cudaEvent_t> ev_pre, ev_join;
  cudaEvent_t ev_fork = nullptr, ev_post = nullptr;
  bool no_graph = false;
  std::vector<void*> peer_recv, peer_cat, peer_flags;  // by group rank (own entry = own window)
  std::vector<void*> opened;                           // IPC mappings to close
};

struct Request {
  int64_t id = 0;
  int height = 0, width = 0, S = 0;
  uint64_t seed = 0;
  float guidance = 3.5f;
  int64_t Li = 0, Lt = 0;
  int next_step = 0;
  int group = -1;
  Pinned<float> x_host;      // [Li, in] until the first landing
  Pinned<uint16_t> T_host;   // [B][Lt, ctx] bf16 bits (SD3: branch 0 = T_c, 1 = T_u)
  Pinned<uint16_t> y_host;   // [B][vec] bf16 bits
  std::vector<double> ts;         // t_0..t_S
  std::map<int, ReqDev> dev;      // by slot
  std::map<int, ReqShard> shard;  // by slot (current group)
  std::map<std::tuple<int, int, int>, ShardAux> aux;   // by (slot, k, rank in group)
  std::map<int, cudaEvent_t> last;  // by slot: completion of the last submitted work
  bool has_velocity = false;
};

struct EventRec {
  std::vector<std::pair<int, cudaEvent_t>> evs;  // (slot, event)
  int group = -1;                                // the group whose work it marks (-1: none)
};

}  // namespace tsv

using namespace tsv;

struct tsv_engine {
  Model model;
  uint64_t weight_seed = 0;
  bool inited = false;                       // device state (streams, weights) exists
  Allocator al;                              // tsv_engine_set_allocator (al.alloc == nullptr: CUDA)
  std::map<int, cudaStream_t> user_stream;   // tsv_engine_set_stream, by device
  std::vector<std::pair<cudaGraphExec_t, cudaEvent_t>> dead_graphs;   // dropped, maybe still running
  const Allocator* alp() const { return al.alloc ? &al : nullptr; }
  bool splitk = true;      // split-K for small fp32-stream GEMM launches (TSV_SPLITK at creation)
  int force_bn = 0, force_pair = -1;   // TSV_GEMM_BN / TSV_GEMM_PAIR (A/B only)
  int rank_base = 0, n_local = 0, world = 0;
  std::vector<Slot> slots;
  std::map<int, std::unique_ptr<DeviceState>> devs;
  std::vector<Group> groups;
  std::map<int64_t, Request> requests;
  int64_t next_req = 1;
  std::vector<EventRec> events;
  std::vector<int64_t> free_events;   // released handles (tsv_event_release), reused by new_event
  ncclComm_t world_comm = nullptr;
  int64_t kernel_count = 0;
  // per-kernel-class profiling (tsv_engine_profile)
  bool prof = false;
  bool graphs = true;  // replay each step as a CUDA graph when a group has one local rank
  int transport = TSV_TRANSPORT_FUSED;  // in-process groups: all-to-alls as epilogue peer stores
  uint64_t graph_clock = 0;
  std::vector<ProfRec> prof_recs;
  std::map<int, std::vector<cudaEvent_t>> ev_pool;  // by device
  double prof_flops[8] = {0}, prof_bytes[8] = {0};
  int64_t prof_launch[8] = {0};

  int slot_of_rank(int rank) const {
    int i = rank - rank_base;
    return (i >= 0 && i < n_local) ? i : -1;
  }
  const bf16* W(const Slot& s, int id) const {
    return reinterpret_cast<const bf16*>(s.ds->weights.p) + model.find(id)->offset;
  }
};

namespace tsv {

// ------------------------------------------------------------------ launch helpers (count + profile kernels)
enum KClass { KC_GEMM = 0, KC_ATTN = 1, KC_LNMOD = 2, KC_QKROPE = 3, KC_A2A = 4, KC_OTHER = 5, KC_N = 6 };

static cudaEvent_t pool_event(tsv_engine* e, int device) {
  auto& v = e->ev_pool[device];
  if (!v.empty()) { cudaEvent_t ev = v.back(); v.pop_back(); return ev; }
  cudaEvent_t ev = nullptr;
  cudaEventCreate(&ev);
  return ev;
}

// Buffers of slot s: engine-lifetime (weights, workspaces) and per-request (stream-ordered on the
// slot's stream; see DevBuf).
static tsv_status salloc(tsv_engine* e, DevBuf& b, const Slot& s, size_t bytes) {
  return dev_alloc(b, s.device, bytes, e->alp(), AK_STATIC, s.stream);
}
static tsv_status qalloc(tsv_engine* e, DevBuf& b, const Slot& s, size_t bytes) {
  return dev_alloc(b, s.device, bytes, e->alp(), AK_STREAM, s.stream);
}

// Counts one launch of class `cls` (kernels = number of CUDA kernels it launches) and, when
// profiling is on, brackets it with CUDA events on the launching stream.
struct ProfScope {
  tsv_engine* e;
  Slot* s;
  int cls;
  cudaEvent_t a = nullptr;
  ProfScope(tsv_engine* e_, Slot& s_, int cls_, double flops, double bytes, int kernels = 1)
      : e(e_), s(&s_), cls(cls_) {
    e->kernel_count += kernels;
    if (!e->prof) return;
    e->prof_flops[cls] += flops;
    e->prof_bytes[cls] += bytes;
    e->prof_launch[cls] += 1;
    a = pool_event(e, s->device);
    // External: inside a step-graph capture this becomes an event-record node replayed with
    // the graph (a plain record would only add an intra-graph dependency).  Outside a capture
    // (direct launches: k > 1 with several local ranks) the flag is invalid: plain record.
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(s->stream, &cs);
    flags = cs == cudaStreamCaptureStatusActive ? cudaEventRecordExternal : cudaEventRecordDefault;
    cudaEventRecordWithFlags(a, s->stream, flags);
  }
  ~ProfScope() {
    if (!a) return;
    cudaEvent_t b = pool_event(e, s->device);
    cudaEventRecordWithFlags(b, s->stream, flags);
    e->prof_recs.push_back({cls, s->device, a, b});
  }
  unsigned flags = cudaEventRecordDefault;
};

static tsv_status gemm(tsv_engine* e, Slot& s, const bf16* A, long long lda, const bf16* Wt, long long ldw, int M,
                       int N, int K, const GemmEpi& epi) {
  if (M <= 0) return TSV_OK;
  GemmPlan p;
  const char* err = nullptr;
  const GemmSplitWs w = s.sws();
  int fbn = e->force_bn;
  if (fbn && (N % fbn || (epi.qk_h && fbn < epi.qk_D))) fbn = 0;   // keep the planner's where illegal
  if (gemm_plan(&p, A, lda, Wt, ldw, M, N, K, epi, s.ds->num_sms, &err, fbn, fbn ? e->force_pair : -1,
                e->splitk ? &w : nullptr))
    return fail(TSV_E_INVAL, "%s (M=%d N=%d K=%d)", err, M, N, K);
  const double out_b = (epi.mode <= EPI_SPLIT_GELU) ? 2.0
                       : (epi.mode == EPI_STORE_F32 ? 4.0 : (epi.mode == EPI_CFG_EULER ? 16.0 : 8.0));
  ProfScope ps(e, s, KC_GEMM, 2.0 * M * N * (double)K,
               2.0 * ((double)M * K + (double)N * K) + out_b * (double)M * N);
  gemm_launch(p, s.stream);
  return TSV_OK;
}
// Up to four problems with the same N, K in one persistent launch (the img and txt streams of a
// double block; x2 for SD3's CFG pair): better wave quantization than one launch per problem.
static tsv_status gemm_multi(tsv_engine* e, Slot& s, const GemmProblem* probs, int np, int N, int K) {
  if (np > GEMM_MAX_PROBLEMS) return fail(TSV_E_INVAL, "gemm_multi: %d problems", np);
  GemmProblem nz[GEMM_MAX_PROBLEMS];
  int n = 0;
  for (int i = 0; i < np; ++i)
    if (probs[i].M > 0) nz[n++] = probs[i];
  if (!n) return TSV_OK;
  GemmPlan p;
  const char* err = nullptr;
  const GemmSplitWs w = s.sws();
  int fbn = e->force_bn;
  if (fbn && (N % fbn || (nz[0].epi.qk_h && fbn < nz[0].epi.qk_D))) fbn = 0;   // keep the planner's where illegal
  if (gemm_plan_multi(&p, nz, n, N, K, s.ds->num_sms, &err, fbn, fbn ? e->force_pair : -1, e->splitk ? &w : nullptr))
    return fail(TSV_E_INVAL, "%s (N=%d K=%d)", err, N, K);
  double fl = 0, by = 2.0 * N * K * n;
  for (int i = 0; i < n; ++i) {
    const double out_b = (nz[i].epi.mode <= EPI_SPLIT_GELU) ? 2.0
                         : (nz[i].epi.mode == EPI_STORE_F32 ? 4.0 : (nz[i].epi.mode == EPI_CFG_EULER ? 16.0 : 8.0));
    fl += 2.0 * nz[i].M * N * (double)K;
    by += 2.0 * nz[i].M * K + out_b * nz[i].M * N;
  }
  ProfScope ps(e, s, KC_GEMM, fl, by);
  gemm_launch(p, s.stream);
  return TSV_OK;
}


static GemmEpi epi_of(int mode, void* out0, long long ld0, const bf16* bias, const float* gate = nullptr,
                      void* out1 = nullptr, long long ld1 = 0, int n_split = 0, const float* scalar = nullptr) {
  GemmEpi g;
  g.mode = mode; g.out0 = out0; g.ld0 = ld0; g.bias = bias; g.gate = gate; g.out1 = out1; g.ld1 = ld1;
  g.n_split = n_split; g.scalar = scalar;
  return g;
}

// ------------------------------------------------------------------ weights
static tsv_status init_weights(tsv_engine* e, DeviceState& ds, const Slot& s) {
  const Model& m = e->model;
  TRY(salloc(e, ds.weights, s, m.total * 2));
  CK(cudaSetDevice(ds.device));
  CK(cudaMemsetAsync(ds.weights.p, 0, m.total * 2, s.stream));
  for (const auto& t : m.tensors) {
    synth_launch(reinterpret_cast<bf16*>(ds.weights.p) + t.offset, e->weight_seed, (uint32_t)t.id, 0, t.numel(),
                 t.kind, t.c, s.stream);
    e->kernel_count++;  // init-time (not a step kernel)
  }
  CK(cudaGetLastError());
  CK(cudaStreamSynchronize(s.stream));
  return TSV_OK;
}

// ------------------------------------------------------------------ per-request state on a slot
static tsv_status ensure_reqdev(tsv_engine* e, Request& R, int si) {
  ReqDev& rd = R.dev[si];
  if (rd.ready) return TSV_OK;
  Slot& s = e->slots[si];
  const Model& m = e->model;
  const int h = m.h, S = R.S, B = m.B;
  CK(cudaSetDevice(s.device));
  const size_t mod_bytes = (size_t)S * B * m.n_mod * 4;
  TRY(qalloc(e, rd.mod, s, mod_bytes));
  TRY(qalloc(e, rd.dt, s, (size_t)S * 4));
  TRY(qalloc(e, rd.step, s, 16));
  if (!rd.ready_ev) CK(cudaEventCreateWithFlags(&rd.ready_ev, cudaEventDisableTiming));
  // another rank of this engine already holds the request's table (in-process reshard onto a new
  // GPU): copy it (85 MB for FLUX at S = 20, a peer copy over NVLink) instead of recomputing it
  // (which reads the 6.5 GB of modulation weights)
  for (auto& kv : R.dev) {
    if (kv.first == si || !kv.second.ready) continue;
    const Slot& src = e->slots[kv.first];
    CK(cudaStreamWaitEvent(s.stream, kv.second.ready_ev, 0));
    CK(cudaMemcpyPeerAsync(rd.mod.p, s.device, kv.second.mod.p, src.device, mod_bytes, s.stream));
    CK(cudaMemcpyPeerAsync(rd.dt.p, s.device, kv.second.dt.p, src.device, (size_t)S * 4, s.stream));
    CK(cudaEventRecord(rd.ready_ev, s.stream));
    rd.ready = true;   // (a ReqDev is only released with its request, after all its copies)
    return TSV_OK;
  }
  // host-side: sinusoidal embeddings e(t_s), e(g) (fp64 -> bf16), y (bf16), dt, staged in pinned
  // memory owned by rd (the copies stay asynchronous).  Row i*B + b is step i of CFG branch b
  // (SD3: b = 0 conditional, 1 unconditional).
  const int Sp = S * B;
  const size_t n_et = (size_t)Sp * 256, n_ey = (size_t)Sp * m.vec;
  TRY(rd.stage.alloc(2 * (2 * n_et + n_ey) + 4 * (size_t)S));
  uint16_t* et = reinterpret_cast<uint16_t*>(rd.stage.data());
  uint16_t* eg = et + n_et;
  uint16_t* ey = eg + n_et;
  float* dt = reinterpret_cast<float*>(ey + n_ey);
  auto emb = [](double t, uint16_t* out) {
    for (int j = 0; j < 128; ++j) {
      double f = std::exp(-std::log(10000.0) * j / 128.0);
      double a = 1000.0 * t * f;
      out[j] = f32_to_bf16_bits((float)std::cos(a));
      out[128 + j] = f32_to_bf16_bits((float)std::sin(a));
    }
  };
  for (int i = 0; i < S; ++i) {
    for (int b = 0; b < B; ++b) {
      emb(R.ts[i], &et[(size_t)(i * B + b) * 256]);
      emb((double)R.guidance, &eg[(size_t)(i * B + b) * 256]);
      memcpy(&ey[(size_t)(i * B + b) * m.vec], R.y_host.data() + (size_t)b * m.vec, m.vec * 2);
    }
    dt[i] = (float)(R.ts[i + 1] - R.ts[i]);
  }
  // scratch: et, eg, ey (bf16 [Sp,256],[Sp,256],[Sp,vec]); hid bf16 [Sp,h]; vec f32 [Sp,h]; asilu bf16 [Sp,h]
  const size_t o_et = 0, o_eg = o_et + (size_t)Sp * 256 * 2, o_ey = o_eg + (size_t)Sp * 256 * 2;
  const size_t o_hid = (o_ey + (size_t)Sp * m.vec * 2 + 255) & ~size_t(255);
  const size_t o_vec = (o_hid + (size_t)Sp * h * 2 + 255) & ~size_t(255);
  const size_t o_as = (o_vec + (size_t)Sp * h * 4 + 255) & ~size_t(255);
  const size_t total = o_as + (size_t)Sp * h * 2;
  TRY(salloc(e, s.scratch, s, total));
  uint8_t* sc = reinterpret_cast<uint8_t*>(s.scratch.p);
  CK(cudaMemcpyAsync(sc + o_et, et, n_et * 2, cudaMemcpyHostToDevice, s.stream));
  CK(cudaMemcpyAsync(sc + o_eg, eg, n_et * 2, cudaMemcpyHostToDevice, s.stream));
  CK(cudaMemcpyAsync(sc + o_ey, ey, n_ey * 2, cudaMemcpyHostToDevice, s.stream));
  CK(cudaMemcpyAsync(rd.dt.p, dt, S * 4, cudaMemcpyHostToDevice, s.stream));
  bf16* hid = reinterpret_cast<bf16*>(sc + o_hid);
  float* vec = reinterpret_cast<float*>(sc + o_vec);
  bf16* as = reinterpret_cast<bf16*>(sc + o_as);
  // vec = MLP_t(e(t)) + MLP_g(e(g)) + MLP_y(y)   (TT:model.py:119-120 + FLUX-dev guidance_in)
  struct MlpIds { size_t off; int K; int w1, b1, w2, b2; bool on; };
  MlpIds mlps[3] = {{o_et, 256, 4, 5, 6, 7, true}, {o_eg, 256, 8, 9, 10, 11, m.d.guidance_embed != 0},
                    {o_ey, m.vec, 12, 13, 14, 15, true}};
  bool first = true;
  for (auto& ml : mlps) {
    if (!ml.on) continue;
    TRY(gemm(e, s, reinterpret_cast<bf16*>(sc + ml.off), ml.K, e->W(s, ml.w1), ml.K, Sp, h, ml.K,
             epi_of(EPI_SILU_BF16, hid, h, e->W(s, ml.b1))));
    TRY(gemm(e, s, hid, h, e->W(s, ml.w2), h, Sp, h, h,
             epi_of(first ? EPI_STORE_F32 : EPI_ACCUM_F32, vec, h, e->W(s, ml.b2))));
    first = false;
  }
  {
    ProfScope ps(e, s, KC_OTHER, 0.0, (double)Sp * h * 6.0);
    silu_bf16_launch(vec, h, as, h, Sp, h, s.stream);
  }
  // modulation table for all steps: [S*B, n_mod] = SiLU(vec) W_mod^T + b   (TT:layers.py:142)
  const bf16* wb = reinterpret_cast<const bf16*>(s.ds->weights.p);
  TRY(gemm(e, s, as, h, wb + m.modw_off, h, Sp, (int)m.n_mod, h,
           epi_of(EPI_STORE_F32, rd.mod.p, m.n_mod, wb + m.modb_off)));
  CK(cudaGetLastError());
  CK(cudaEventRecord(rd.ready_ev, s.stream));
  rd.ready = true;
  return TSV_OK;
}

// Per-request state of one shard on its slot, all enqueued on the slot's stream (no host wait):
// buffers (stream-ordered), the text rows T (pinned host -> device), the RoPE cos/sin tables
// (FLUX; fp64 angles -> fp32, S22) or the SD3 sin-cos position embedding (S13) computed on the
// device, and the a1 text embedding txt = T W_txt^T + b of the shard's text rows (constant per
// request: computed here once, copied into the residual stream by every step).
static tsv_status setup_shard(tsv_engine* e, Request& R, int si, int rank_in_group, int k, ReqShard& sh) {
  Slot& s = e->slots[si];
  const Model& m = e->model;
  sh.rank_in_group = rank_in_group;
  sh.k = k;
  sh.t0 = shard_begin(R.Lt, k, rank_in_group);
  sh.nt = shard_begin(R.Lt, k, rank_in_group + 1) - sh.t0;
  sh.i0 = shard_begin(R.Li, k, rank_in_group);
  sh.ni = shard_begin(R.Li, k, rank_in_group + 1) - sh.i0;
  CK(cudaSetDevice(s.device));
  TRY(qalloc(e, sh.lat, s, std::max<size_t>(1, sh.ni) * m.in * 4));
  TRY(qalloc(e, sh.vel, s, std::max<size_t>(1, sh.ni) * m.in * 4));
  const auto key = std::make_tuple(si, k, rank_in_group);
  auto found = R.aux.find(key);
  if (found != R.aux.end()) {   // this layout was set up on this rank before: nothing to recompute
    sh.ax = &found->second;
    return TSV_OK;
  }
  ShardAux& ax = R.aux[key];
  sh.ax = &ax;
  TRY(qalloc(e, ax.T, s, std::max<size_t>(1, sh.nt) * m.B * m.ctx * 2));
  TRY(qalloc(e, ax.txt, s, std::max<size_t>(1, sh.nt) * m.B * m.h * 4));
  const size_t rows = sh.nt + sh.ni;
  if (sh.nt)
    for (int b = 0; b < m.B; ++b)
      CK(cudaMemcpyAsync(reinterpret_cast<uint16_t*>(ax.T.p) + (size_t)b * sh.nt * m.ctx,
                         R.T_host.data() + ((size_t)b * R.Lt + sh.t0) * m.ctx, sh.nt * m.ctx * 2,
                         cudaMemcpyHostToDevice, s.stream));
  if (m.sd3) {
    TRY(qalloc(e, ax.pe, s, std::max<size_t>(1, sh.ni) * m.h * 4));
    // patch (r, c) of the n_r x n_c grid sits at ((r + top) / q, (c + left) / q), q = pe_max / pe_base,
    // top = floor((pe_max - n_r) / 2) (floor toward -inf, S13)
    const int64_t n_r = R.height / 16, n_c = R.width / 16;
    auto floordiv2 = [](int64_t a) { return a >= 0 ? a / 2 : -((-a + 1) / 2); };
    ProfScope ps(e, s, KC_OTHER, 0.0, (double)sh.ni * m.h * 4.0);
    sincos_pe_launch(reinterpret_cast<float*>(ax.pe.p), sh.i0, (int)sh.ni, n_c, floordiv2(m.d.pe_max - n_r),
                     floordiv2(m.d.pe_max - n_c), (double)m.d.pe_max / m.d.pe_base, m.h, s.stream);
  } else {
    TRY(qalloc(e, ax.cosb, s, std::max<size_t>(1, rows) * (m.D / 2) * 4));
    TRY(qalloc(e, ax.sinb, s, std::max<size_t>(1, rows) * (m.D / 2) * 4));
    ProfScope ps(e, s, KC_OTHER, 0.0, (double)rows * m.D * 4.0);
    rope_table_launch(reinterpret_cast<float*>(ax.cosb.p), reinterpret_cast<float*>(ax.sinb.p), (int)sh.nt, sh.i0,
                      (int)sh.ni, R.width / 16, m.D, m.d.axes_dim, (double)m.d.theta, s.stream);
  }
  if (sh.nt) {
    GemmProblem pt[GEMM_MAX_PROBLEMS];
    for (int b = 0; b < m.B; ++b)
      pt[b] = {reinterpret_cast<bf16*>(ax.T.p) + b * sh.nt * m.ctx, m.ctx, e->W(s, 2), m.ctx, (int)sh.nt,
               epi_of(EPI_STORE_F32, reinterpret_cast<float*>(ax.txt.p) + b * sh.nt * m.h, m.h, e->W(s, 3))};
    TRY(gemm_multi(e, s, pt, m.B, m.h, m.ctx));
  }
  CK(cudaGetLastError());
  return TSV_OK;
}

// B = evaluations per step (requests in the batch x CFG branches)
static tsv_status ensure_workspace(tsv_engine* e, Slot& s, int64_t rows, int64_t L, int k, int B) {
  const Model& m = e->model;
  const int64_t h = m.h, F = m.F;
  Workspace& w = s.ws;
  const int64_t r1 = std::max<int64_t>(rows, 1);
  const int64_t r = r1 * B;  // every activation buffer holds the B evaluations back to back
  TRY(salloc(e, w.x, s, r * h * 4));
  TRY(salloc(e, w.u, s, r * h * 2));
  TRY(salloc(e, w.qkv, s, r * 3 * h * 2));
  TRY(salloc(e, w.cat, s, r * (h + F) * 2));
  TRY(salloc(e, w.hbuf, s, r * F * 2));
  TRY(salloc(e, w.latb, s, r * m.in * 2));
  TRY(salloc(e, w.bmod, s, ((size_t)B * m.n_mod + 64) * 4));
  if (k > 1) {
    TRY(salloc(e, w.pack, s, r * 3 * h * 2));
    TRY(salloc(e, w.recv, s, B * L * 3 * (h / k) * 2));
    TRY(salloc(e, w.obuf, s, B * L * (h / k) * 2));
    TRY(salloc(e, w.orecv, s, r * h * 2));
  }
  return TSV_OK;
}

// ------------------------------------------------------------------ the step
struct RankCtx {
  int si;                 // slot index
  Slot* s;
  ReqShard* sh;           // request 0's shard (the batch shares resolution and group: same rows)
  std::vector<ReqShard*> shq;  // per request of the batch
  std::vector<ReqDev*> rdq;
  int64_t nt, ni, rows;   // local rows per evaluation: [txt (nt) ; img (ni)]
  float* x;
  bf16 *u, *qkv, *cat, *hbuf, *latb, *pack, *recv, *obuf, *orecv;
  float* mod;             // this step's modulation rows: evaluation b at mod + b * n_mod; dt of
                          // request q at mod + B * n_mod + q
};

struct StepEnv {
  tsv_engine* e;
  Request* R;             // request 0 of the batch (shared L_t, L_i)
  std::vector<Request*> Rq;
  int B = 1;              // evaluations: requests x CFG branches; evaluation b = q * B_model + branch
  Group* g;
  bool fused = false;     // all-to-alls fused into the QKV-GEMM / attention epilogues (peer stores)
  std::vector<RankCtx> rc;
  // global layout for the all-to-alls
  std::vector<int64_t> t_off, t_cnt, i_off, i_cnt;  // per group rank
  // fused transport: every member's attention input and activation buffer, by group rank
  std::vector<bf16*> recv_of, cat_of;
  bool ipc = false;       // members in other processes (CUDA IPC windows, device barrier)
};

// ------------------------------------------------------------------ Ulysses all-to-alls (a5, a7)
// A plan entry is one contiguous block of `rows` rows (of the all-to-all's row width) exchanged
// with `peer`: sent from / received into the caller's buffer at row `row0`.  Sends and receives
// between a pair of ranks are matched in plan order (NCCL point-to-point semantics); the same plan
// drives the NCCL path and the in-process peer-copy path (and is exported as tsv_a2a_plan).
struct A2AOp {
  int peer, send;
  int64_t row0, rows;
};

// which = 1 (seq -> head): send buffer = pack [k][rows_r] rows (chunk p = peer p's heads),
//                          recv buffer = recv [L] rows in global order [txt_0..txt_k-1; img_0..img_k-1].
// which = 2 (head -> seq): send buffer = obuf [L] rows, recv buffer = orecv [k][rows_r] rows.
static void a2a_plan(int which, int64_t Lt, int64_t Li, int k, int r, std::vector<A2AOp>& ops) {
  ops.clear();
  auto tb = [&](int q) { return shard_begin(Lt, k, q); };
  auto tc = [&](int q) { return shard_begin(Lt, k, q + 1) - shard_begin(Lt, k, q); };
  auto ib = [&](int q) { return shard_begin(Li, k, q); };
  auto ic = [&](int q) { return shard_begin(Li, k, q + 1) - shard_begin(Li, k, q); };
  const int64_t rows_r = tc(r) + ic(r);
  for (int p = 0; p < k; ++p) {
    if (which == 1) {
      if (tc(r)) ops.push_back({p, 1, p * rows_r, tc(r)});
      if (ic(r)) ops.push_back({p, 1, p * rows_r + tc(r), ic(r)});
      if (tc(p)) ops.push_back({p, 0, tb(p), tc(p)});
      if (ic(p)) ops.push_back({p, 0, Lt + ib(p), ic(p)});
    } else {
      if (tc(p)) ops.push_back({p, 1, tb(p), tc(p)});
      if (ic(p)) ops.push_back({p, 1, Lt + ib(p), ic(p)});
      if (tc(r)) ops.push_back({p, 0, p * rows_r, tc(r)});
      if (ic(r)) ops.push_back({p, 0, p * rows_r + tc(r), ic(r)});
    }
  }
}

static tsv_status a2a_exec(StepEnv& E, int which) {
  tsv_engine* e = E.e;
  const Model& m = e->model;
  Group& g = *E.g;
  const int k = g.k;
  const int64_t w = (which == 1 ? 3 : 1) * (int64_t)m.h / k;  // bf16 per row
  const int64_t L = E.R->Lt + E.R->Li;
  // B evaluations (SD3's CFG pair) exchange back to back: the [k][rows_r] buffer of branch b
  // starts at b * k * rows_r * w, the [L] buffer at b * L * w.
  const int B = E.B;
  auto sendbuf = [&](RankCtx& c, int b) {
    return which == 1 ? c.pack + b * k * c.rows * w : c.obuf + b * L * w;
  };
  auto recvbuf = [&](RankCtx& c, int b) {
    return which == 1 ? c.recv + b * L * w : c.orecv + b * k * c.rows * w;
  };
  std::vector<A2AOp> ops;
  if (g.comm) {
    RankCtx& c = E.rc[0];
    const int r = g.local_positions[0];
    CK(cudaSetDevice(c.s->device));
    ProfScope ps(e, *c.s, KC_A2A, 0.0, 2.0 * B * c.rows * w * (k - 1));
    a2a_plan(which, E.R->Lt, E.R->Li, k, r, ops);
    NK(ncclGroupStart());
    for (int b = 0; b < B; ++b)
      for (const A2AOp& o : ops) {
        if (o.send) NK(ncclSend(sendbuf(c, b) + o.row0 * w, o.rows * w, ncclBfloat16, o.peer, g.comm, c.s->stream));
        else NK(ncclRecv(recvbuf(c, b) + o.row0 * w, o.rows * w, ncclBfloat16, o.peer, g.comm, c.s->stream));
      }
    NK(ncclGroupEnd());
    return TSV_OK;
  }
  // in-process: all k ranks are local (rc indexed by group rank); receiver streams pull.
  std::vector<std::vector<A2AOp>> plans(k);
  for (int r = 0; r < k; ++r) a2a_plan(which, E.R->Lt, E.R->Li, k, r, plans[r]);
  for (int r = 0; r < k; ++r) CK(cudaEventRecord(g.ev_a[r], E.rc[r].s->stream));
  for (int d = 0; d < k; ++d) {
    RankCtx& dst = E.rc[d];
    CK(cudaSetDevice(dst.s->device));
    ProfScope ps(e, *dst.s, KC_A2A, 0.0, 2.0 * B * dst.rows * w * (k - 1), 0);
    for (int r = 0; r < k; ++r) CK(cudaStreamWaitEvent(dst.s->stream, g.ev_a[r], 0));
    std::vector<int> nth_recv(k, 0);
    for (const A2AOp& o : plans[d]) {
      if (o.send) continue;
      const int p = o.peer;
      int idx = nth_recv[p]++, seen = 0;
      const A2AOp* match = nullptr;
      for (const A2AOp& so : plans[p])
        if (so.send && so.peer == d && seen++ == idx) { match = &so; break; }
      if (!match || match->rows != o.rows) return fail(TSV_E_STATE, "all-to-all plan mismatch");
      RankCtx& src = E.rc[p];
      // UVA copy (cudaMemcpyDefault): peer or same-device, and capturable into a step graph
      // (cudaMemcpyPeerAsync is not)
      for (int b = 0; b < B; ++b)
        CK(cudaMemcpyAsync(recvbuf(dst, b) + o.row0 * w, sendbuf(src, b) + match->row0 * w, o.rows * w * 2,
                           cudaMemcpyDefault, dst.s->stream));
    }
    CK(cudaEventRecord(g.ev_b[d], dst.s->stream));
  }
  for (int r = 0; r < k; ++r)
    for (int d = 0; d < k; ++d) CK(cudaStreamWaitEvent(E.rc[r].s->stream, g.ev_b[d], 0));
  return TSV_OK;
}

// In-process group barrier: every member's stream waits for every member's work so far.  With the
// fused transport this is the whole all-to-all: the data already moved in the producers' epilogues.
static tsv_status group_sync(StepEnv& E) {
  Group& g = *E.g;
  const int k = g.k;
  if (E.ipc) {
    // members in other processes: a device-side barrier over the IPC flag windows
    ProfScope ps(E.e, *E.rc[0].s, KC_A2A, 0.0, 0.0, 1);
    IpcBarrier b;
    b.k = k;
    b.rank = g.local_positions[0];
    for (int d = 0; d < k; ++d) b.flags[d] = reinterpret_cast<int*>(g.peer_flags[d]);
    ipc_barrier_launch(b, E.rc[0].s->stream);
    return TSV_OK;
  }
  ProfScope ps(E.e, *E.rc[0].s, KC_A2A, 0.0, 0.0, 0);
  for (int r = 0; r < k; ++r) {
    CK(cudaSetDevice(E.rc[r].s->device));
    CK(cudaEventRecord(g.ev_a[r], E.rc[r].s->stream));
  }
  for (int r = 0; r < k; ++r) {
    CK(cudaSetDevice(E.rc[r].s->device));
    for (int d = 0; d < k; ++d)
      if (d != r) CK(cudaStreamWaitEvent(E.rc[r].s->stream, g.ev_a[d], 0));
  }
  return TSV_OK;
}

static tsv_status a2a_qkv(StepEnv& E) { return E.fused ? group_sync(E) : a2a_exec(E, 1); }

// Fused a5 destinations for one QKV-GEMM problem of rank c, evaluation b: kind 0 = its txt rows,
// 1 = its img rows, 2 = its [txt_r; img_r] rows (single blocks).
static void peer_epi(StepEnv& E, RankCtx& c, GemmEpi& epi, int b, int kind) {
  const Model& m = E.e->model;
  const int k = E.g->k;
  const int64_t L = E.R->Lt + E.R->Li, w = 3 * (int64_t)m.h / k;
  const int r = c.sh->rank_in_group;
  for (int d = 0; d < k; ++d) epi.peer[d] = E.recv_of[d] + b * L * w;
  const int tg = (int)E.t_off[r], ig = (int)(E.R->Lt + E.i_off[r]);
  epi.peer_nt = 1 << 30;
  if (kind == 0) epi.peer_row0 = tg;
  else if (kind == 1) epi.peer_row0 = ig;
  else { epi.peer_row0 = tg; epi.peer_nt = (int)c.nt; epi.peer_row1 = ig; }
}

// all-to-all #2 then unpack: cat[i, d*h/k + c] = orecv[d][i][c]
static tsv_status a2a_o(StepEnv& E) {
  if (E.fused) return group_sync(E);   // the attention epilogues stored into every owner's cat
  tsv_engine* e = E.e;
  const Model& m = e->model;
  const int k = E.g->k;
  const int64_t w = (int64_t)m.h / k;
  TRY(a2a_exec(E, 2));
  for (auto& c : E.rc) {
    CK(cudaSetDevice(c.s->device));
    for (int b = 0; b < E.B; ++b)
      for (int d = 0; d < k; ++d) {
        ProfScope ps(e, *c.s, KC_OTHER, 0.0, 4.0 * c.rows * w);
        copy2d_bf16_launch(c.orecv + ((int64_t)b * k + d) * c.rows * w, w, c.cat + b * c.rows * (m.h + m.F) + d * w,
                           m.h + m.F, (int)c.rows, (int)w, c.s->stream);
      }
  }
  return TSV_OK;
}

// attention for all local ranks (after a2a #1); output into cat[:, :h] (k = 1) or obuf (k > 1)
static tsv_status attention_all(StepEnv& E) {
  tsv_engine* e = E.e;
  const Model& m = e->model;
  const int k = E.g->k;
  const int64_t L = E.R->Lt + E.R->Li;
  for (auto& c : E.rc) {
    CK(cudaSetDevice(c.s->device));
    const double Lq = k == 1 ? (double)c.rows : (double)L;
    for (int b = 0; b < E.B; ++b) {  // one launch per evaluation (request x CFG branch)
      ProfScope ps(e, *c.s, KC_ATTN, 4.0 * Lq * Lq * m.D * (m.H / k), 8.0 * Lq * m.D * (m.H / k));
      const AttnSplitWs kvw = c.s->aws();
      const AttnSplitWs* kvs = e->splitk ? &kvw : nullptr;
      int rc;
      if (k == 1) {
        const bf16* q = c.qkv + b * c.rows * 3 * m.h;
        rc = attention_launch(q, 3 * m.h, q + m.h, 3 * m.h, q + 2 * m.h, 3 * m.h, c.cat + b * c.rows * (m.h + m.F),
                              m.h + m.F, (int)c.rows, m.H, m.D, c.s->stream, 3, nullptr, kvs);
      } else if (E.fused) {
        // fused a7: each output row goes straight to its owner's cat[:, r*h/k + ...]
        const int64_t w = 3 * (int64_t)m.h / k;
        const bf16* q = c.recv + b * L * w;
        AttnScatter sc;
        sc.k = k;
        sc.Lt = (int)E.R->Lt;
        sc.col0 = c.sh->rank_in_group * (m.h / k);
        sc.ld = m.h + m.F;
        for (int p = 0; p < k; ++p) {
          sc.dst[p] = E.cat_of[p] + b * (E.t_cnt[p] + E.i_cnt[p]) * (m.h + m.F);
          sc.t_off[p] = (int)E.t_off[p];
          sc.i_off[p] = (int)E.i_off[p];
          sc.nt[p] = (int)E.t_cnt[p];
        }
        sc.t_off[k] = (int)E.R->Lt;
        sc.i_off[k] = (int)E.R->Li;
        rc = attention_launch(q, w, q + m.h / k, w, q + 2 * m.h / k, w, nullptr, 0, (int)L, m.H / k, m.D, c.s->stream,
                              3, &sc, kvs);
      } else {
        const int64_t w = 3 * (int64_t)m.h / k;
        const bf16* q = c.recv + b * L * w;
        rc = attention_launch(q, w, q + m.h / k, w, q + 2 * m.h / k, w, c.obuf + b * L * (m.h / k), m.h / k, (int)L,
                              m.H / k, m.D, c.s->stream, 3, nullptr, kvs);
      }
      if (rc == -5) CK(cudaGetLastError());
      if (rc) return fail(TSV_E_CUDA, "attention launch failed (%d)", rc);
    }
  }
  return TSV_OK;
}

// a4 fused into the QKV GEMM epilogue: QK-RMSNorm + RoPE on rows [r0, r0 + n) of this rank, written
// in place (k = 1) or straight into the Ulysses send buffer (k > 1).
static GemmEpi qk_fused(StepEnv& E, RankCtx& c, GemmEpi epi, int64_t r0, const bf16* gq, const bf16* gk, int kind,
                        int b) {
  const Model& m = E.e->model;
  epi.qk_h = m.h;
  epi.qk_D = m.D;
  epi.gq = gq;
  epi.gk = gk;
  epi.cosb = reinterpret_cast<const float*>(c.sh->ax->cosb.p) + r0 * (m.D / 2);
  epi.sinb = reinterpret_cast<const float*>(c.sh->ax->sinb.p) + r0 * (m.D / 2);
  epi.k_sp = E.g->k;
  epi.pack = E.g->k > 1 ? c.pack + b * c.rows * 3 * m.h : nullptr;
  epi.pack_rows = (int)c.rows;
  epi.pack_row0 = (int)r0;
  if (E.fused) peer_epi(E, c, epi, b, kind);
  return epi;
}


static tsv_status run_step_sd3(StepEnv& E);

// this step's modulation rows and dt of every request of the batch, selected on the device from
// each request's step index (so one captured graph serves every step)
static void select_rows(StepEnv& E, RankCtx& c) {
  tsv_engine* e = E.e;
  const Model& m = e->model;
  Slot& s = *c.s;
  const int64_t nm = m.B * m.n_mod;
  for (size_t q = 0; q < E.Rq.size(); ++q) {
    ProfScope ps(e, s, KC_OTHER, 0.0, 8.0 * nm, 2);
    const int* step_dev = reinterpret_cast<const int*>(c.rdq[q]->step.p);
    select_row_launch(reinterpret_cast<const float*>(c.rdq[q]->mod.p), nm, step_dev, c.mod + q * nm, nm, s.stream);
    select_row_launch(reinterpret_cast<const float*>(c.rdq[q]->dt.p), 1, step_dev, c.mod + E.B * m.n_mod + q, 1,
                      s.stream);
  }
}


// a1 text embedding: the shard's txt = T W_txt^T + b was computed when it landed (setup_shard); every
// step copies it into the residual stream rows [b R, b R + nt) of evaluation b (a 4 x ctx/h smaller
// copy instead of an M = nt, K = 4096 weight-streaming GEMM).  per_req = evaluations per request
// (1 FLUX, 2 SD3 CFG branches; branch br uses txt rows br * nt).
static tsv_status txt_embed(tsv_engine* e, Slot& s, const std::vector<ReqShard*>& shq, float* x, int64_t R, int64_t nt,
                            int B, int per_req) {
  if (!nt) return TSV_OK;
  const int h = e->model.h;
  for (int b = 0; b < B; ++b) {
    ReqShard* sh = shq[b / per_req];
    CK(cudaMemcpyAsync(x + b * R * h, reinterpret_cast<float*>(sh->ax->txt.p) + (b % per_req) * nt * h,
                       nt * h * sizeof(float), cudaMemcpyDeviceToDevice, s.stream));
  }
  return TSV_OK;
}

static tsv_status run_step(StepEnv& E) {
  tsv_engine* e = E.e;
  const Model& m = e->model;
  const int h = m.h, F = m.F, B = E.B;
  const int64_t ldc = h + F, nm = m.n_mod;
  for (auto& c : E.rc) {
    CK(cudaSetDevice(c.s->device));
    select_rows(E, c);
  }
  if (m.sd3) return run_step_sd3(E);
  // FLUX: evaluation b = request b of the batch; its rows are [b*R, (b+1)*R) of every buffer.
  // a1: embeddings
  for (auto& c : E.rc) {
    Slot& s = *c.s;
    CK(cudaSetDevice(s.device));
    const int64_t R = c.rows;
    GemmProblem pi[GEMM_MAX_PROBLEMS];
    for (int b = 0; b < B; ++b) {
      if (c.ni) {
        ProfScope ps(e, s, KC_OTHER, 0.0, 6.0 * c.ni * m.in);
        f32_to_bf16_launch(reinterpret_cast<float*>(c.shq[b]->lat.p), m.in, c.latb + b * c.ni * m.in, m.in, (int)c.ni,
                           m.in, s.stream);
      }
      pi[b] = {c.latb + b * c.ni * m.in, m.in, e->W(s, 0), m.in, (int)c.ni,
               epi_of(EPI_STORE_F32, c.x + (b * R + c.nt) * h, h, e->W(s, 1))};
    }
    TRY(gemm_multi(e, s, pi, B, h, m.in));
    TRY(txt_embed(e, s, c.shq, c.x, R, c.nt, B, 1));
  }
  // double-stream blocks
  for (int j = 0; j < m.d.n_double; ++j) {
    for (auto& c : E.rc) {
      Slot& s = *c.s;
      CK(cudaSetDevice(s.device));
      const int64_t R = c.rows;
      {  // a2 for both streams of every evaluation: rows [txt; img] per evaluation
        const float* mt = c.mod + m.mod_double(j, 1);
        const float* mi = c.mod + m.mod_double(j, 0);
        ProfScope ps(e, s, KC_LNMOD, 0.0, (double)B * R * h * 6.0 + 16.0 * B * h);
        ln_mod2b_launch(c.x, h, c.u, h, mt, mt + h, mi, mi + h, (int)c.nt, (int)R, B, nm, h, s.stream);
      }
      GemmProblem pq[GEMM_MAX_PROBLEMS];
      int n = 0;
      for (int b = 0; b < B; ++b)
        for (int st = 0; st < 2; ++st) {  // 0 = img, 1 = txt
          const int base = double_base(j, st);
          const int64_t r0 = st == 0 ? c.nt : 0, nr = st == 0 ? c.ni : c.nt;
          pq[n++] = {c.u + (b * R + r0) * h, h, e->W(s, base + 2), h, (int)nr,
                     qk_fused(E, c, epi_of(EPI_STORE_BF16, c.qkv + (b * R + r0) * 3 * h, 3 * h, e->W(s, base + 3)), r0,
                              e->W(s, base + 4), e->W(s, base + 5), st == 0 ? 1 : 0, b)};
        }
      TRY(gemm_multi(e, s, pq, n, 3 * h, h));   // a3 + a4 for both streams in one launch
    }
    if (E.g->k > 1) TRY(a2a_qkv(E));
    TRY(attention_all(E));
    if (E.g->k > 1) TRY(a2a_o(E));
    for (auto& c : E.rc) {
      Slot& s = *c.s;
      CK(cudaSetDevice(s.device));
      const int64_t R = c.rows;
      GemmProblem pp[GEMM_MAX_PROBLEMS], p1[GEMM_MAX_PROBLEMS], p2[GEMM_MAX_PROBLEMS];
      int n = 0;
      for (int b = 0; b < B; ++b)
        for (int st = 0; st < 2; ++st) {
          const int base = double_base(j, st);
          const int64_t r0 = st == 0 ? c.nt : 0, nr = st == 0 ? c.ni : c.nt;
          const float* md = c.mod + b * nm + m.mod_double(j, st);
          float* x = c.x + (b * R + r0) * h;
          pp[n] = {c.cat + (b * R + r0) * ldc, ldc, e->W(s, base + 6), h, (int)nr,
                   epi_of(EPI_RESID_GATE, x, h, e->W(s, base + 7), md + 2 * h)};
          p1[n] = {c.u + (b * R + r0) * h, h, e->W(s, base + 8), h, (int)nr,
                   epi_of(EPI_GELU_BF16, c.hbuf + (b * R + r0) * F, F, e->W(s, base + 9))};
          p2[n] = {c.hbuf + (b * R + r0) * F, F, e->W(s, base + 10), F, (int)nr,
                   epi_of(EPI_RESID_GATE, x, h, e->W(s, base + 11), md + 5 * h)};
          ++n;
        }
      TRY(gemm_multi(e, s, pp, n, h, h));        // a8: out-proj + gated residual, both streams
      {                                          // a9: LN-modulate both streams
        const float* mt = c.mod + m.mod_double(j, 1);
        const float* mi = c.mod + m.mod_double(j, 0);
        ProfScope ps(e, s, KC_LNMOD, 0.0, (double)B * R * h * 6.0 + 16.0 * B * h);
        ln_mod2b_launch(c.x, h, c.u, h, mt + 3 * h, mt + 4 * h, mi + 3 * h, mi + 4 * h, (int)c.nt, (int)R, B, nm, h,
                        s.stream);
      }
      TRY(gemm_multi(e, s, p1, n, F, h));        // fc1 + GELU
      TRY(gemm_multi(e, s, p2, n, h, F));        // fc2 + gated residual
    }
  }
  // single-stream blocks on x = [txt; img] (zero-copy join, a10)
  for (int j = 0; j < m.d.n_single; ++j) {
    const int base = single_base(j);
    for (auto& c : E.rc) {
      Slot& s = *c.s;
      CK(cudaSetDevice(s.device));
      const int64_t R = c.rows;
      if (!R) continue;
      {
        const float* md = c.mod + m.mod_single(j);
        ProfScope ps(e, s, KC_LNMOD, 0.0, (double)B * R * h * 6.0 + 16.0 * B * h);
        ln_mod2b_launch(c.x, h, c.u, h, md, md + h, md, md + h, (int)R, (int)R, B, nm, h, s.stream);
      }
      GemmProblem p1[GEMM_MAX_PROBLEMS];
      for (int b = 0; b < B; ++b)
        p1[b] = {c.u + b * R * h, h, e->W(s, base + 2), h, (int)R,
                 qk_fused(E, c, epi_of(EPI_SPLIT_GELU, c.qkv + b * R * 3 * h, 3 * h, e->W(s, base + 3), nullptr,
                                       c.cat + b * R * ldc + h, ldc, 3 * h),
                          0, e->W(s, base + 4), e->W(s, base + 5), 2, b)};
      TRY(gemm_multi(e, s, p1, B, 3 * h + F, h));
    }
    if (E.g->k > 1) TRY(a2a_qkv(E));
    TRY(attention_all(E));
    if (E.g->k > 1) TRY(a2a_o(E));
    for (auto& c : E.rc) {
      Slot& s = *c.s;
      CK(cudaSetDevice(s.device));
      const int64_t R = c.rows;
      if (!R) continue;
      GemmProblem p2[GEMM_MAX_PROBLEMS];
      for (int b = 0; b < B; ++b) {
        const float* md = c.mod + b * nm + m.mod_single(j);
        p2[b] = {c.cat + b * R * ldc, ldc, e->W(s, base + 6), ldc, (int)R,
                 epi_of(EPI_RESID_GATE, c.x + b * R * h, h, e->W(s, base + 7), md + 2 * h)};
      }
      TRY(gemm_multi(e, s, p2, B, h, h + F));
    }
  }
  // final layer + Euler (a11, a12), every request of the batch in one launch
  for (auto& c : E.rc) {
    Slot& s = *c.s;
    CK(cudaSetDevice(s.device));
    if (!c.ni) continue;
    const int64_t R = c.rows;
    {
      const float* md = c.mod + m.mod_final();
      ProfScope ps(e, s, KC_LNMOD, 0.0, (double)B * R * h * 6.0 + 16.0 * B * h);
      ln_mod2b_launch(c.x, h, c.u, h, md, md + h, md, md + h, (int)c.nt, (int)R, B, nm, h, s.stream);
    }
    GemmProblem pf[GEMM_MAX_PROBLEMS];
    for (int b = 0; b < B; ++b)
      pf[b] = {c.u + (b * R + c.nt) * h, h, e->W(s, 18), h, (int)c.ni,
               epi_of(EPI_EULER, c.shq[b]->lat.p, m.in, e->W(s, 19), nullptr, c.shq[b]->vel.p, m.in, 0,
                      c.mod + B * nm + b)};
    TRY(gemm_multi(e, s, pf, B, m.in, h));
  }
  for (auto& c : E.rc) CK(cudaGetLastError());
  return TSV_OK;
}

// SD3-medium step (DESIGN.md O-SD3).  Every request contributes B_model = 2 evaluations (branch 0
// conditional, 1 unconditional, S23); evaluation b = q*2 + branch owns rows [b*rows, (b+1)*rows) of
// each activation buffer, laid out [txt_r ; img_r] like FLUX, and all evaluations share every
// launch.  Joint blocks are double blocks without QK-norm and RoPE, so the QKV epilogue is a plain
// store (k = 1) or a pure Ulysses pack / peer store (k > 1); joint attention over [txt; img] equals
// diffusers' [img; txt] (no position-dependent term, the softmax is permutation-equivariant).  The
// last block's txt stream is context_pre_only (AdaLayerNormContinuous (scale, shift), QKV only).
// The CFG combine is fused into the Euler epilogue of the final linear.
static tsv_status run_step_sd3(StepEnv& E) {
  tsv_engine* e = E.e;
  const Model& m = e->model;
  const int h = m.h, F = m.F, B = E.B, nq = (int)E.Rq.size();
  const int64_t ldc = h + F, nm = m.n_mod;
  const int k = E.g->k;
  const int nd = m.d.n_double;
  // a1: img = x W^T + b + PE (identical for both branches of a request), txt_b = T_b W^T + b
  for (auto& c : E.rc) {
    Slot& s = *c.s;
    CK(cudaSetDevice(s.device));
    const int64_t R = c.rows;
    if (c.ni) {
      GemmProblem pi[GEMM_MAX_PROBLEMS];
      for (int q = 0; q < nq; ++q) {
        float* xi = c.x + (2 * q * R + c.nt) * h;
        {
          ProfScope ps(e, s, KC_OTHER, 0.0, 6.0 * c.ni * m.in);
          f32_to_bf16_launch(reinterpret_cast<float*>(c.shq[q]->lat.p), m.in, c.latb + q * c.ni * m.in, m.in,
                             (int)c.ni, m.in, s.stream);
        }
        CK(cudaMemcpyAsync(xi, c.shq[q]->ax->pe.p, c.ni * h * 4, cudaMemcpyDeviceToDevice, s.stream));
        pi[q] = {c.latb + q * c.ni * m.in, m.in, e->W(s, 0), m.in, (int)c.ni, epi_of(EPI_ACCUM_F32, xi, h, e->W(s, 1))};
      }
      TRY(gemm_multi(e, s, pi, nq, h, m.in));
      for (int q = 0; q < nq; ++q) {
        float* xi = c.x + (2 * q * R + c.nt) * h;
        CK(cudaMemcpyAsync(xi + R * h, xi, c.ni * h * 4, cudaMemcpyDeviceToDevice, s.stream));
      }
    }
    TRY(txt_embed(e, s, c.shq, c.x, R, c.nt, B, 2));
  }
  for (int j = 0; j < nd; ++j) {
    const bool last = j == nd - 1;  // context_pre_only
    for (auto& c : E.rc) {
      Slot& s = *c.s;
      CK(cudaSetDevice(s.device));
      const int64_t R = c.rows;
      if (!R) continue;
      // a2: LN-modulate both streams of every evaluation in one launch
      {
        const float* mi = c.mod + m.mod_double(j, 0);
        const float* mt = c.mod + m.mod_double(j, 1);
        ProfScope ps(e, s, KC_LNMOD, 0.0, (double)B * R * h * 6.0 + 16.0 * B * h);
        ln_mod2b_launch(c.x, h, c.u, h, last ? mt + h : mt, last ? mt : mt + h, mi, mi + h, (int)c.nt, (int)R, B, nm,
                        h, s.stream);
      }
      // a3 (+ Ulysses pack / peer stores for k > 1): 2 streams x B evaluations in one launch
      GemmProblem pq[GEMM_MAX_PROBLEMS];
      int n = 0;
      for (int b = 0; b < B; ++b)
        for (int st = 0; st < 2; ++st) {
          const int base = double_base(j, st);
          const int64_t r0 = st == 0 ? c.nt : 0, nr = st == 0 ? c.ni : c.nt;
          GemmEpi ep = epi_of(EPI_STORE_BF16, c.qkv + (b * R + r0) * 3 * h, 3 * h, e->W(s, base + 3));
          if (k > 1) {
            ep.qk_h = h; ep.qk_D = m.D; ep.k_sp = k;
            ep.pack = c.pack + b * R * 3 * h; ep.pack_rows = (int)R; ep.pack_row0 = (int)r0;
            if (E.fused) peer_epi(E, c, ep, b, st == 0 ? 1 : 0);
          }
          pq[n++] = {c.u + (b * R + r0) * h, h, e->W(s, base + 2), h, (int)nr, ep};
        }
      TRY(gemm_multi(e, s, pq, n, 3 * h, h));
    }
    if (k > 1) TRY(a2a_qkv(E));
    TRY(attention_all(E));
    if (k > 1) TRY(a2a_o(E));
    for (auto& c : E.rc) {
      Slot& s = *c.s;
      CK(cudaSetDevice(s.device));
      const int64_t R = c.rows;
      if (!R) continue;
      GemmProblem pp[GEMM_MAX_PROBLEMS], p1[GEMM_MAX_PROBLEMS], p2[GEMM_MAX_PROBLEMS];
      int n = 0;
      for (int b = 0; b < B; ++b)
        for (int st = 0; st < 2; ++st) {
          if (last && st == 1) continue;  // the context_pre_only txt stream ends at its QKV
          const int base = double_base(j, st);
          const int64_t r0 = st == 0 ? c.nt : 0, nr = st == 0 ? c.ni : c.nt;
          const float* md = c.mod + b * nm + m.mod_double(j, st);
          float* x = c.x + (b * R + r0) * h;
          pp[n] = {c.cat + (b * R + r0) * ldc, ldc, e->W(s, base + 6), h, (int)nr,
                   epi_of(EPI_RESID_GATE, x, h, e->W(s, base + 7), md + 2 * h)};
          p1[n] = {c.u + (b * R + r0) * h, h, e->W(s, base + 8), h, (int)nr,
                   epi_of(EPI_GELU_BF16, c.hbuf + (b * R + r0) * F, F, e->W(s, base + 9))};
          p2[n] = {c.hbuf + (b * R + r0) * F, F, e->W(s, base + 10), F, (int)nr,
                   epi_of(EPI_RESID_GATE, x, h, e->W(s, base + 11), md + 5 * h)};
          ++n;
        }
      TRY(gemm_multi(e, s, pp, n, h, h));  // a8: out-proj + gated residual
      {                                     // a9: LN-modulate (every evaluation, one launch)
        const float* mi = c.mod + m.mod_double(j, 0);
        // context_pre_only: the txt rows are dead after the attention; they are normalised with
        // the img vectors (in bounds, result unused) so all evaluations stay one launch
        const float* mt = last ? mi : c.mod + m.mod_double(j, 1);
        ProfScope ps(e, s, KC_LNMOD, 0.0, (double)B * R * h * 6.0 + 16.0 * B * h);
        ln_mod2b_launch(c.x, h, c.u, h, mt + 3 * h, mt + 4 * h, mi + 3 * h, mi + 4 * h, (int)c.nt, (int)R, B, nm, h,
                        s.stream);
      }
      TRY(gemm_multi(e, s, p1, n, F, h));  // fc1 + GELU
      TRY(gemm_multi(e, s, p2, n, h, F));  // fc2 + gated residual
    }
  }
  // final: AdaLayerNormContinuous (scale, shift) per evaluation, linear; v_u stored, then the
  // conditional GEMM's epilogue forms v = v_u + s (v_c - v_u) and x += dt v
  for (auto& c : E.rc) {
    Slot& s = *c.s;
    CK(cudaSetDevice(s.device));
    if (!c.ni) continue;
    const int64_t R = c.rows;
    {
      const float* md = c.mod + m.mod_final();
      ProfScope ps(e, s, KC_LNMOD, 0.0, (double)B * R * h * 6.0 + 16.0 * B * h);
      ln_mod2b_launch(c.x, h, c.u, h, md + h, md, md + h, md, (int)c.nt, (int)R, B, nm, h, s.stream);
    }
    GemmProblem pu[GEMM_MAX_PROBLEMS], pc[GEMM_MAX_PROBLEMS];
    for (int q = 0; q < nq; ++q) {
      pu[q] = {c.u + ((2 * q + 1) * R + c.nt) * h, h, e->W(s, 18), h, (int)c.ni,
               epi_of(EPI_STORE_F32, c.shq[q]->vel.p, m.in, e->W(s, 19))};
      GemmEpi ep = epi_of(EPI_CFG_EULER, c.shq[q]->lat.p, m.in, e->W(s, 19), nullptr, c.shq[q]->vel.p, m.in, 0,
                          c.mod + B * nm + q);
      ep.alpha = m.d.cfg_scale;
      pc[q] = {c.u + (2 * q * R + c.nt) * h, h, e->W(s, 18), h, (int)c.ni, ep};
    }
    TRY(gemm_multi(e, s, pu, nq, m.in, h));
    TRY(gemm_multi(e, s, pc, nq, m.in, h));
  }
  for (auto& c : E.rc) CK(cudaGetLastError());
  return TSV_OK;
}

// ------------------------------------------------------------------ landing / reshard
static tsv_status record_last(tsv_engine* e, Request& R, int si) {
  Slot& s = e->slots[si];
  CK(cudaSetDevice(s.device));
  auto it = R.last.find(si);
  if (it == R.last.end()) {
    cudaEvent_t ev;
    CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    it = R.last.emplace(si, ev).first;
  }
  CK(cudaEventRecord(it->second, s.stream));
  return TSV_OK;
}

static void drop_request_graphs(tsv_engine* e, int64_t id);

// Move the request to group gi (a13).  First landing: latent rows come from the pinned
// host inputs.  Otherwise bit-exact row moves old shard -> new shard by the reshard map, each copy
// ordered after the request's last work on its source rank.  Nothing here waits on the host: the
// new shards' state is enqueued on their streams (setup_shard, ensure_reqdev), and the old shards
// are released stream-ordered on their own streams after every copy that reads them.
static tsv_status move_request(tsv_engine* e, Request& R, int gi) {
  Group& g = e->groups[gi];
  const Model& m = e->model;
  std::map<int, ReqShard> next;
  for (size_t q = 0; q < g.local_slots.size(); ++q) {
    const int si = g.local_slots[q];
    Slot& s = e->slots[si];
    CK(cudaSetDevice(s.device));
    // the new rank's stream follows the request's previous work there (its shard buffers may reuse
    // memory the old shard on this slot still reads)
    auto it = R.last.find(si);
    if (it != R.last.end()) CK(cudaStreamWaitEvent(s.stream, it->second, 0));
    trace("move: setup_shard");
    TRY(setup_shard(e, R, si, g.local_positions[q], g.k, next[si]));
    trace("move: ensure_reqdev");
    TRY(ensure_reqdev(e, R, si));
    trace("move: slot done");
  }
  if (R.group < 0) {
    for (auto& kv : next) {
      Slot& s = e->slots[kv.first];
      ReqShard& sh = kv.second;
      CK(cudaSetDevice(s.device));
      if (sh.ni)
        CK(cudaMemcpyAsync(sh.lat.p, R.x_host.data() + sh.i0 * m.in, sh.ni * m.in * 4, cudaMemcpyHostToDevice,
                           s.stream));
    }
  } else {
    Group& og = e->groups[R.group];
    const int ks = og.k, kd = g.k;
    if (!og.all_local || !g.all_local) {
      // multi-process: exchange rows over the world communicator
      if (!e->world_comm) return fail(TSV_E_STATE, "reshard across processes needs tsv_engine_init_world");
      NK(ncclGroupStart());
      for (int sr = 0; sr < ks; ++sr) {
        const int64_t a0 = shard_begin(R.Li, ks, sr), a1 = shard_begin(R.Li, ks, sr + 1);
        for (int dr = 0; dr < kd; ++dr) {
          const int64_t b0 = shard_begin(R.Li, kd, dr), b1 = shard_begin(R.Li, kd, dr + 1);
          const int64_t lo = std::max(a0, b0), hi = std::min(a1, b1);
          if (hi <= lo) continue;
          const int src_rank = og.ranks[sr], dst_rank = g.ranks[dr];
          const int ss = e->slot_of_rank(src_rank), ds = e->slot_of_rank(dst_rank);
          if (ss >= 0 && ds >= 0) {
            CK(cudaStreamWaitEvent(e->slots[ds].stream, R.last[ss], 0));
            CK(cudaMemcpyPeerAsync(reinterpret_cast<float*>(next[ds].lat.p) + (lo - b0) * m.in, e->slots[ds].device,
                                   reinterpret_cast<float*>(R.shard[ss].lat.p) + (lo - a0) * m.in,
                                   e->slots[ss].device, (hi - lo) * m.in * 4, e->slots[ds].stream));
          } else if (ss >= 0) {
            NK(ncclSend(reinterpret_cast<float*>(R.shard[ss].lat.p) + (lo - a0) * m.in, (hi - lo) * m.in, ncclFloat32,
                        dst_rank, e->world_comm, e->slots[ss].stream));
          } else if (ds >= 0) {
            NK(ncclRecv(reinterpret_cast<float*>(next[ds].lat.p) + (lo - b0) * m.in, (hi - lo) * m.in, ncclFloat32,
                        src_rank, e->world_comm, e->slots[ds].stream));
          }
        }
      }
      NK(ncclGroupEnd());
    } else {
      for (int sr = 0; sr < ks; ++sr) {
        const int64_t a0 = shard_begin(R.Li, ks, sr), a1 = shard_begin(R.Li, ks, sr + 1);
        const int ss = e->slot_of_rank(og.ranks[sr]);
        for (int dr = 0; dr < kd; ++dr) {
          const int64_t b0 = shard_begin(R.Li, kd, dr), b1 = shard_begin(R.Li, kd, dr + 1);
          const int64_t lo = std::max(a0, b0), hi = std::min(a1, b1);
          if (hi <= lo) continue;
          const int ds = e->slot_of_rank(g.ranks[dr]);
          Slot& dslot = e->slots[ds];
          CK(cudaSetDevice(dslot.device));
          CK(cudaStreamWaitEvent(dslot.stream, R.last[ss], 0));
          CK(cudaMemcpyPeerAsync(reinterpret_cast<float*>(next[ds].lat.p) + (lo - b0) * m.in, dslot.device,
                                 reinterpret_cast<float*>(R.shard[ss].lat.p) + (lo - a0) * m.in, e->slots[ss].device,
                                 (hi - lo) * m.in * 4, dslot.stream));
        }
      }
    }
    trace("move: copies enqueued");
    // the old shards' buffers: released on their own streams once every new rank's copies (which
    // read them) are done -- stream-ordered, the host never waits
    for (auto& kv : next) TRY(record_last(e, R, kv.first));
    for (auto& kv : R.shard) {
      Slot& os = e->slots[kv.first];
      CK(cudaSetDevice(os.device));
      for (auto& nk : next)
        if (nk.first != kv.first) CK(cudaStreamWaitEvent(os.stream, R.last[nk.first], 0));
      kv.second.release();
    }
    trace("move: old shards released");
    drop_request_graphs(e, R.id);   // cached step graphs reference the old shards' buffers
    trace("move: graphs dropped");
  }
  R.shard.swap(next);
  R.group = gi;
  R.has_velocity = false;
  for (auto& kv : R.shard) TRY(record_last(e, R, kv.first));
  return TSV_OK;
}

// Event handles index e->events; released handles (tsv_event_release) are reused, so a serving
// loop that releases its step events keeps a bounded set of CUDA events.
static tsv_status new_event(tsv_engine* e, const std::vector<int>& slots_, tsv_event* out, int gi = -1) {
  EventRec rec;
  rec.group = gi;
  for (int si : slots_) {
    Slot& s = e->slots[si];
    CK(cudaSetDevice(s.device));
    cudaEvent_t ev;
    CK(cudaEventCreate(&ev));
    CK(cudaEventRecord(ev, s.stream));
    rec.evs.push_back({si, ev});
  }
  int64_t id;
  if (!e->free_events.empty()) {
    id = e->free_events.back();
    e->free_events.pop_back();
    e->events[id] = std::move(rec);
  } else {
    e->events.push_back(std::move(rec));
    id = (int64_t)e->events.size() - 1;
  }
  if (out) *out = (tsv_event)id;
  return TSV_OK;
}

// A dropped step graph may still be executing (its last replay is in flight on the slot's stream):
// it is destroyed once an event recorded behind that replay has completed (sweep_graphs), so that
// dropping never waits on the device.
static void drop_graph(tsv_engine* e, Slot& s, StepGraph& gr) {
  if (!gr.exec) return;
  cudaEvent_t ev = nullptr;
  cudaSetDevice(s.device);
  if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) == cudaSuccess &&
      cudaEventRecord(ev, s.stream) == cudaSuccess) {
    e->dead_graphs.push_back({gr.exec, ev});
  } else {   // cannot defer: wait for the slot's work, then destroy
    if (ev) cudaEventDestroy(ev);
    cudaStreamSynchronize(s.stream);
    cudaGraphExecDestroy(gr.exec);
  }
  gr.exec = nullptr;
}
static void sweep_graphs(tsv_engine* e, bool all) {
  for (size_t i = 0; i < e->dead_graphs.size();) {
    auto& d = e->dead_graphs[i];
    if (all || cudaEventQuery(d.second) == cudaSuccess) {
      if (all) cudaEventSynchronize(d.second);
      cudaGraphExecDestroy(d.first);
      cudaEventDestroy(d.second);
      d = e->dead_graphs.back();
      e->dead_graphs.pop_back();
    } else {
      cudaGetLastError();   // clear cudaErrorNotReady
      ++i;
    }
  }
}

// One step of every request in Rs (each at its own next step) as one batched step on group gi.
// The requests share the resolution (checked by the caller); their shards land on the group first.
static tsv_status do_step(tsv_engine* e, const std::vector<Request*>& Rs, int gi, tsv_event* done) {
  Group& g = e->groups[gi];
  if (g.local_slots.empty()) {
    if (done) *done = -1;
    for (Request* R : Rs) R->next_step++;
    return TSV_OK;
  }
  sweep_graphs(e, false);
  for (Request* R : Rs)
    if (R->group != gi) TRY(move_request(e, *R, gi));
  const Model& m = e->model;
  Request& R0 = *Rs[0];
  StepEnv E;
  E.e = e; E.R = &R0; E.Rq = Rs; E.g = &g;
  E.B = (int)Rs.size() * m.B;
  E.fused = e->transport == TSV_TRANSPORT_FUSED && (g.all_local || g.ipc) && g.k > 1;
  E.ipc = E.fused && !g.all_local;
  if (!g.all_local && !g.comm && !E.ipc)
    return fail(TSV_E_STATE, "group spans processes without NCCL: exchange IPC windows first (tsv_group_ipc_export/import)");
  if (E.ipc && (R0.Lt + R0.Li > g.win_tokens || E.B > g.win_evals))
    return fail(TSV_E_INVAL, "step (L = %lld, %d evaluations) exceeds the group's IPC windows (%lld, %d)",
                (long long)(R0.Lt + R0.Li), E.B, (long long)g.win_tokens, g.win_evals);
  const int k = g.k;
  E.t_off.resize(k); E.t_cnt.resize(k); E.i_off.resize(k); E.i_cnt.resize(k);
  for (int r = 0; r < k; ++r) {
    E.t_off[r] = shard_begin(R0.Lt, k, r);
    E.t_cnt[r] = shard_begin(R0.Lt, k, r + 1) - E.t_off[r];
    E.i_off[r] = shard_begin(R0.Li, k, r);
    E.i_cnt[r] = shard_begin(R0.Li, k, r + 1) - E.i_off[r];
  }
  const int64_t L = R0.Lt + R0.Li;
  for (size_t q = 0; q < g.local_slots.size(); ++q) {
    const int si = g.local_slots[q];
    Slot& s = e->slots[si];
    ReqShard& sh = R0.shard[si];
    TRY(ensure_workspace(e, s, sh.nt + sh.ni, L, k, E.B));
    RankCtx c;
    c.si = si; c.s = &s; c.sh = &sh;
    for (Request* R : Rs) { c.shq.push_back(&R->shard[si]); c.rdq.push_back(&R->dev[si]); }
    c.nt = sh.nt; c.ni = sh.ni; c.rows = sh.nt + sh.ni;
    c.x = reinterpret_cast<float*>(s.ws.x.p);
    c.u = reinterpret_cast<bf16*>(s.ws.u.p);
    c.qkv = reinterpret_cast<bf16*>(s.ws.qkv.p);
    c.cat = reinterpret_cast<bf16*>(s.ws.cat.p);
    c.hbuf = reinterpret_cast<bf16*>(s.ws.hbuf.p);
    c.latb = reinterpret_cast<bf16*>(s.ws.latb.p);
    c.pack = reinterpret_cast<bf16*>(s.ws.pack.p);
    c.recv = reinterpret_cast<bf16*>(s.ws.recv.p);
    c.obuf = reinterpret_cast<bf16*>(s.ws.obuf.p);
    c.orecv = reinterpret_cast<bf16*>(s.ws.orecv.p);
    c.mod = reinterpret_cast<float*>(s.ws.bmod.p);
    if (E.ipc) {  // the attention input and activation rows live in the group's shared windows
      c.recv = reinterpret_cast<bf16*>(g.win_recv.p);
      c.cat = reinterpret_cast<bf16*>(g.win_cat.p);
    }
    E.rc.push_back(c);
  }
  if (E.fused) {
    for (int d = 0; d < k; ++d) {
      E.recv_of.push_back(E.ipc ? reinterpret_cast<bf16*>(g.peer_recv[d]) : E.rc[d].recv);
      E.cat_of.push_back(E.ipc ? reinterpret_cast<bf16*>(g.peer_cat[d]) : E.rc[d].cat);
    }
  }
  // each slot's stream must follow every request's previous work on that slot; then publish the
  // step indices (pageable source: staged at call time, so the host value can change right after)
  for (auto& c : E.rc) {
    CK(cudaSetDevice(c.s->device));
    for (size_t q = 0; q < Rs.size(); ++q) {
      auto it = Rs[q]->last.find(c.si);
      if (it != Rs[q]->last.end()) CK(cudaStreamWaitEvent(c.s->stream, it->second, 0));
      int st = Rs[q]->next_step;
      CK(cudaMemcpyAsync(c.rdq[q]->step.p, &st, sizeof(int), cudaMemcpyHostToDevice, c.s->stream));
    }
  }
  // Replay (or capture once) the whole step as one CUDA graph launched on the first local rank's
  // stream ("origin").  Local ranks on other streams (several ranks in this process: virtual ranks
  // on one GPU, or GPUs of one process) are forked from and joined back to the origin inside the
  // capture, so their kernels and the cross-rank event edges of the transports become one
  // multi-stream (multi-device) graph; around the launch the other streams hand their order to the
  // origin and take it back.
  cudaStream_t origin = E.rc[0].s->stream;
  std::vector<int> others;   // indices into E.rc of the ranks on streams other than the origin
  for (size_t i = 0; i < E.rc.size(); ++i) {
    bool seen = E.rc[i].s->stream == origin;
    for (int o : others) seen = seen || E.rc[o].s->stream == E.rc[i].s->stream;
    if (!seen) others.push_back((int)i);
  }
  const bool multi = !others.empty();
  if (multi && g.ev_pre.empty()) {
    g.ev_pre.assign(E.rc.size(), nullptr);
    g.ev_join.assign(E.rc.size(), nullptr);
    for (int o : others) {
      CK(cudaSetDevice(E.rc[o].s->device));
      CK(cudaEventCreateWithFlags(&g.ev_pre[o], cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&g.ev_join[o], cudaEventDisableTiming));
    }
    CK(cudaSetDevice(E.rc[0].s->device));
    CK(cudaEventCreateWithFlags(&g.ev_fork, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&g.ev_post, cudaEventDisableTiming));
  }
  if (e->graphs && !g.no_graph) {
    // cached per (first) slot by every buffer the step references
    Slot& slot = *E.rc[0].s;
    uint64_t key = 1469598103934665603ull;
    auto mix = [&](uint64_t v) { key = (key ^ v) * 1099511628211ull; };
    for (const RankCtx& c : E.rc) {
      const void* ptrs[] = {c.x, c.u, c.qkv, c.cat, c.hbuf, c.latb, c.pack, c.recv, c.obuf, c.orecv, c.mod};
      for (const void* p : ptrs) mix(reinterpret_cast<uintptr_t>(p));
      for (size_t q = 0; q < Rs.size(); ++q) {
        const ReqShard* sh = c.shq[q];
        const ReqDev* rd = c.rdq[q];
        const void* rp[] = {sh->lat.p, sh->vel.p, sh->ax->T.p, sh->ax->cosb.p, sh->ax->sinb.p, sh->ax->pe.p, rd->mod.p, rd->dt.p,
                            rd->step.p};
        for (const void* p : rp) mix(reinterpret_cast<uintptr_t>(p));
        mix((uint64_t)Rs[q]->id);
      }
      mix((uint64_t)c.rows);
      mix((uint64_t)c.si);
    }
    mix((uint64_t)E.rc.size());
    mix((uint64_t)gi);
    mix((uint64_t)Rs.size());
    mix((uint64_t)e->prof);   // a profiled graph carries event-record nodes around every launch
    mix((uint64_t)E.fused * 2 + (uint64_t)E.ipc);   // the transport changes the epilogues and exchanges
    auto it = slot.graphs.find(key);
    if (it == slot.graphs.end()) {
      // bounded cache: evict the least recently used graph
      if (slot.graphs.size() >= 64) {
        auto lru = slot.graphs.begin();
        for (auto jt = slot.graphs.begin(); jt != slot.graphs.end(); ++jt)
          if (jt->second.last_use < lru->second.last_use) lru = jt;
        drop_graph(e, slot, lru->second);
        slot.graphs.erase(lru);
      }
      CK(cudaSetDevice(slot.device));
      StepGraph gr;
      for (Request* R : Rs) gr.reqs.push_back(R->id);
      const int64_t k0 = e->kernel_count;
      const size_t r0 = e->prof_recs.size();
      double f0[8], b0[8];
      int64_t l0[8];
      for (int i = 0; i < 8; ++i) { f0[i] = e->prof_flops[i]; b0[i] = e->prof_bytes[i]; l0[i] = e->prof_launch[i]; }
      CK(cudaStreamBeginCapture(slot.stream, cudaStreamCaptureModeThreadLocal));
      tsv_status st = TSV_OK;
      cudaError_t fe = cudaSuccess;
      if (multi) {   // fork the other ranks' streams into the capture
        if ((fe = cudaEventRecord(g.ev_fork, origin)) == cudaSuccess)
          for (int o : others)
            if (fe == cudaSuccess) {
              cudaSetDevice(E.rc[o].s->device);
              fe = cudaStreamWaitEvent(E.rc[o].s->stream, g.ev_fork, 0);
            }
      }
      if (fe == cudaSuccess) st = run_step(E);
      if (multi && fe == cudaSuccess && st == TSV_OK) {   // join them back
        for (int o : others)
          if (fe == cudaSuccess) {
            cudaSetDevice(E.rc[o].s->device);
            if ((fe = cudaEventRecord(g.ev_join[o], E.rc[o].s->stream)) == cudaSuccess) {
              cudaSetDevice(slot.device);
              fe = cudaStreamWaitEvent(origin, g.ev_join[o], 0);
            }
          }
      }
      cudaSetDevice(slot.device);
      cudaGraph_t graph = nullptr;
      cudaError_t ce = cudaStreamEndCapture(slot.stream, &graph);
      if (multi && (fe != cudaSuccess || ce != cudaSuccess)) {
        // this group's step cannot be captured across its streams (e.g. a driver without
        // multi-device capture): launch it directly from now on
        if (graph) cudaGraphDestroy(graph);
        cudaGetLastError();
        e->prof_recs.resize(r0);
        for (int i = 0; i < 8; ++i) { e->prof_flops[i] = f0[i]; e->prof_bytes[i] = b0[i]; e->prof_launch[i] = l0[i]; }
        e->kernel_count = k0;
        g.no_graph = true;
        TRY(run_step(E));
        goto stepped;
      }
      // what ProfScope recorded during capture belongs to the graph: re-added at every replay
      gr.prof.assign(e->prof_recs.begin() + r0, e->prof_recs.end());
      e->prof_recs.resize(r0);
      for (int i = 0; i < 8; ++i) {
        gr.flops[i] = e->prof_flops[i] - f0[i];
        gr.bytes[i] = e->prof_bytes[i] - b0[i];
        gr.launch[i] = e->prof_launch[i] - l0[i];
        e->prof_flops[i] = f0[i]; e->prof_bytes[i] = b0[i]; e->prof_launch[i] = l0[i];
      }
      if (st != TSV_OK) { if (graph) cudaGraphDestroy(graph); return st; }
      if (ce != cudaSuccess) return fail(TSV_E_CUDA, "step capture: %s", cudaGetErrorString(ce));
      ce = cudaGraphInstantiate(&gr.exec, graph, 0);
      cudaGraphDestroy(graph);
      if (ce != cudaSuccess) return fail(TSV_E_CUDA, "graph instantiate: %s", cudaGetErrorString(ce));
      gr.kernels = e->kernel_count - k0;
      e->kernel_count = k0;
      it = slot.graphs.emplace(key, std::move(gr)).first;
    }
    StepGraph& gr = it->second;
    gr.last_use = ++e->graph_clock;
    if (multi)   // the origin follows the other ranks' work so far (their step-index copies included)
      for (int o : others) {
        CK(cudaSetDevice(E.rc[o].s->device));
        CK(cudaEventRecord(g.ev_pre[o], E.rc[o].s->stream));
        CK(cudaSetDevice(slot.device));
        CK(cudaStreamWaitEvent(origin, g.ev_pre[o], 0));
      }
    CK(cudaSetDevice(slot.device));
    CK(cudaGraphLaunch(gr.exec, slot.stream));
    if (multi) {   // and the other ranks' streams follow the graph
      CK(cudaEventRecord(g.ev_post, origin));
      for (int o : others) {
        CK(cudaSetDevice(E.rc[o].s->device));
        CK(cudaStreamWaitEvent(E.rc[o].s->stream, g.ev_post, 0));
      }
    }
    e->kernel_count += gr.kernels;
    if (e->prof) {
      // the graph's event pairs now hold this replay's timestamps
      e->prof_recs.insert(e->prof_recs.end(), gr.prof.begin(), gr.prof.end());
      for (int i = 0; i < 8; ++i) {
        e->prof_flops[i] += gr.flops[i];
        e->prof_bytes[i] += gr.bytes[i];
        e->prof_launch[i] += gr.launch[i];
      }
    }
  } else {
    TRY(run_step(E));
  }
stepped:
  for (Request* R : Rs) {
    for (auto& c : E.rc) TRY(record_last(e, *R, c.si));
    R->next_step++;
    R->has_velocity = true;
  }
  if (done) TRY(new_event(e, g.local_slots, done, gi));
  return TSV_OK;
}

static void release_reqdev(ReqDev& d) {
  d.mod.release();
  d.dt.release();
  d.step.release();
  if (d.ready_ev) cudaEventDestroy(d.ready_ev);
  d.ready_ev = nullptr;
  d.stage.reset();
  d.ready = false;
}

// drop every cached step graph that references request `id` (its buffers are about to be freed)
static void drop_request_graphs(tsv_engine* e, int64_t id) {
  for (auto& s : e->slots)
    for (auto it = s.graphs.begin(); it != s.graphs.end();) {
      const auto& r = it->second.reqs;
      if (std::find(r.begin(), r.end(), id) != r.end()) {
        drop_graph(e, s, it->second);
        it = s.graphs.erase(it);
      } else {
        ++it;
      }
    }
}

}  // namespace tsv

// ================================================================== C ABI
extern "C" {

const char* tsv_last_error(void) { return g_err.c_str(); }

tsv_status tsv_model_preset(const char* name, tsv_model_desc* out) {
  if (!name || !out) return fail(TSV_E_INVAL, "null argument");
  tsv_model_desc d{};
  std::string n(name);
  if (n == "flux") {
    d = {3072, 24, 128, 12288, 19, 38, 64, 4096, 768, 512, {16, 56, 56}, 10000.f, 1};
  } else if (n == "tiny" || n == "tiny_s" || n == "tiny2") {
    d = {256, 4, 64, 1024, 1, 0, 64, 512, 256, 64, {8, 28, 28}, 10000.f, 1};
    if (n == "tiny_s") d.n_single = 1;
    if (n == "tiny2") { d.n_double = 2; d.n_single = 2; }
  } else if (n == "sd3" || n == "tiny_sd3") {
    // SD3-medium (config 5): h 1536, 24 heads of 64, F 6144, 24 joint blocks, L_t = 333 (77 CLIP +
    // 256 T5), ctx 4096, pooled 2048; "tiny_sd3": h 256, 4 heads, 2 joint blocks, L_t = 77
    d = {1536, 24, 64, 6144, 24, 0, 64, 4096, 2048, 333, {0, 0, 0}, 10000.f, 0};
    if (n == "tiny_sd3") { d.hidden = 256; d.heads = 4; d.mlp_hidden = 1024; d.n_double = 2; d.ctx_dim = 512;
                           d.vec_dim = 256; d.text_tokens = 77; }
    d.family = TSV_FAMILY_SD3; d.cfg_scale = 7.0f; d.shift = 3.0f; d.pe_max = 192; d.pe_base = 64;
  } else {
    return fail(TSV_E_INVAL, "unknown preset '%s'", name);
  }
  *out = d;
  return TSV_OK;
}

tsv_status tsv_engine_create(const tsv_model_desc* model, const int* devices, int n_local, int rank_base,
                             int world_size, uint64_t weight_seed, tsv_engine** out) {
  if (!model || !devices || !out || n_local <= 0 || rank_base < 0 || world_size < rank_base + n_local)
    return fail(TSV_E_INVAL, "tsv_engine_create: bad arguments");
  int ndev = 0;
  CK(cudaGetDeviceCount(&ndev));
  for (int i = 0; i < n_local; ++i)
    if (devices[i] < 0 || devices[i] >= ndev) return fail(TSV_E_INVAL, "device %d out of range (%d)", devices[i], ndev);
  auto e = std::make_unique<tsv_engine>();
  std::string err;
  if (!build_model(*model, &e->model, &err)) return fail(TSV_E_INVAL, "%s", err.c_str());
  e->weight_seed = weight_seed;
  e->splitk = splitk_env();
  e->force_bn = gemm_force_env("TSV_GEMM_BN", 0);
  e->force_pair = gemm_force_env("TSV_GEMM_PAIR", -1);
  if (const char* li = getenv("TSV_LN_IMPL")) g_ln_impl = atoi(li);   // LN-modulate variant (A/B)
  e->rank_base = rank_base;
  e->n_local = n_local;
  e->world = world_size;
  e->slots.resize(n_local);
  for (int i = 0; i < n_local; ++i) {
    e->slots[i].rank = rank_base + i;
    e->slots[i].device = devices[i];
  }
  *out = e.release();
  return TSV_OK;
}

// Device state, created on first use (after the optional allocator / stream hooks): per slot a
// stream (the caller's for its device, else an engine-owned non-blocking one), the device's weights,
// split-K counters and workspace; peer access (and memory-pool access for the stream-ordered
// per-request buffers) between the engine's distinct devices.
static tsv_status ensure_init(tsv_engine* e) {
  if (e->inited) return TSV_OK;
  for (int i = 0; i < e->n_local; ++i) {
    Slot& s = e->slots[i];
    CK(cudaSetDevice(s.device));
    // TSV_VIRTUAL_SERIAL=1: virtual ranks on one device share one stream, so every kernel runs alone
    // on the GPU as it would on a rank's own GPU (per-rank timing of k > 1 on one device); default:
    // one stream per rank (the ranks' kernels overlap)
    const char* vs = getenv("TSV_VIRTUAL_SERIAL");
    Slot* first = nullptr;
    for (int j = 0; j < i; ++j)
      if (e->slots[j].device == s.device) { first = &e->slots[j]; break; }
    auto us = e->user_stream.find(s.device);
    if (us != e->user_stream.end()) {
      s.stream = us->second;
      s.own_stream = false;
    } else if (vs && atoi(vs) && first) {
      s.stream = first->stream;
      s.own_stream = false;
    } else {
      CK(cudaStreamCreateWithFlags(&s.stream, cudaStreamNonBlocking));
      s.own_stream = true;
    }
    auto it = e->devs.find(s.device);
    if (it == e->devs.end()) {
      auto ds = std::make_unique<DeviceState>();
      ds->device = s.device;
      CK(cudaDeviceGetAttribute(&ds->num_sms, cudaDevAttrMultiProcessorCount, s.device));
      // stream-ordered pool of the per-request buffers: keep freed memory cached (no release to
      // the OS at synchronisation points)
      cudaMemPool_t pool;
      CK(cudaDeviceGetDefaultMemPool(&pool, s.device));
      uint64_t keep = UINT64_MAX;
      CK(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep));
      TRY(init_weights(e, *ds, s));
      if (!e->alp()) {
        // pre-grow the pool (TSV_POOL_RESERVE_MB, default 2 GiB: the per-request state of ~18 FLUX
        // 2048^2 requests on a rank): growing it on a request's first landing maps new memory
        // (tens of ms of host time) inside what should be an enqueue-only reshard call
        const char* rv = getenv("TSV_POOL_RESERVE_MB");
        const size_t mb = rv ? (size_t)atoll(rv) : 2048;
        if (mb) {
          void* p = nullptr;
          CK(cudaMallocAsync(&p, mb << 20, s.stream));
          CK(cudaFreeAsync(p, s.stream));
          CK(cudaStreamSynchronize(s.stream));
        }
      }
      it = e->devs.emplace(s.device, std::move(ds)).first;
    }
    s.ds = it->second.get();
    TRY(salloc(e, s.sem, s, SEM_INTS * sizeof(int)));
    CK(cudaMemsetAsync(s.sem.p, 0, SEM_INTS * sizeof(int), s.stream));
    TRY(salloc(e, s.splitws, s, SPLIT_WS_BYTES));
  }
  // peer access between distinct local devices (in-process all-to-all and reshard), also for the
  // stream-ordered pools
  for (auto& a : e->devs)
    for (auto& b : e->devs) {
      if (a.first == b.first) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, a.first, b.first);
      if (can) {
        cudaSetDevice(a.first);
        cudaError_t r = cudaDeviceEnablePeerAccess(b.first, 0);
        if (r != cudaSuccess && r != cudaErrorPeerAccessAlreadyEnabled) return fail(TSV_E_CUDA, "peer access");
        cudaGetLastError();
        cudaMemPool_t pool;
        CK(cudaDeviceGetDefaultMemPool(&pool, b.first));
        cudaMemAccessDesc d{};
        d.location.type = cudaMemLocationTypeDevice;
        d.location.id = a.first;
        d.flags = cudaMemAccessFlagsProtReadWrite;
        CK(cudaMemPoolSetAccess(pool, &d, 1));   // device a may access b's pool allocations
      }
    }
  for (auto& s : e->slots) {
    CK(cudaSetDevice(s.device));
    CK(cudaStreamSynchronize(s.stream));
  }
  e->inited = true;
  return TSV_OK;
}

tsv_status tsv_engine_set_allocator(tsv_engine* e, void* ctx, tsv_alloc_fn alloc_fn, tsv_free_fn free_fn) {
  if (!e || !alloc_fn || !free_fn) return fail(TSV_E_INVAL, "null argument");
  if (e->inited) return fail(TSV_E_STATE, "the allocator must be set before the engine's first group");
  e->al.ctx = ctx;
  e->al.alloc = alloc_fn;
  e->al.free = free_fn;
  return TSV_OK;
}

tsv_status tsv_engine_set_stream(tsv_engine* e, int device, void* cuda_stream) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  if (e->inited) return fail(TSV_E_STATE, "streams must be set before the engine's first group");
  bool found = false;
  for (auto& s : e->slots) found = found || s.device == device;
  if (!found) return fail(TSV_E_INVAL, "device %d hosts no rank of this engine", device);
  e->user_stream[device] = reinterpret_cast<cudaStream_t>(cuda_stream);
  return TSV_OK;
}

void tsv_engine_destroy(tsv_engine* e) {
  if (!e) return;
  if (!e->inited) {   // no device state: requests hold only pinned host memory
    delete e;
    return;
  }
  for (auto& s : e->slots) {
    cudaSetDevice(s.device);
    cudaStreamSynchronize(s.stream);
  }
  for (auto& s : e->slots)
    for (auto& kv : s.graphs) drop_graph(e, s, kv.second);
  sweep_graphs(e, true);
  for (auto& kv : e->requests) {
    for (auto& d : kv.second.dev) release_reqdev(d.second);
    for (auto& sh : kv.second.shard) sh.second.release();
    for (auto& ax : kv.second.aux) ax.second.release();
    for (auto& l : kv.second.last) cudaEventDestroy(l.second);
  }
  for (auto& g : e->groups) {
    for (void* p : g.opened) cudaIpcCloseMemHandle(p);
    g.win_recv.release(); g.win_cat.release(); g.win_flags.release();
    if (g.comm) ncclCommDestroy(g.comm);
    for (auto ev : g.ev_a) cudaEventDestroy(ev);
    for (auto ev : g.ev_b) cudaEventDestroy(ev);
    for (auto ev : g.ev_pre) if (ev) cudaEventDestroy(ev);
    for (auto ev : g.ev_join) if (ev) cudaEventDestroy(ev);
    if (g.ev_fork) cudaEventDestroy(g.ev_fork);
    if (g.ev_post) cudaEventDestroy(g.ev_post);
  }
  if (e->world_comm) ncclCommDestroy(e->world_comm);
  for (auto& rec : e->events)
    for (auto& p : rec.evs) cudaEventDestroy(p.second);
  for (auto& s : e->slots) {
    Workspace& w = s.ws;
    for (DevBuf* b : {&w.x, &w.u, &w.qkv, &w.cat, &w.hbuf, &w.latb, &w.pack, &w.recv, &w.obuf, &w.orecv, &w.bmod,
                      &s.scratch, &s.sem, &s.splitws})
      b->release();
    cudaSetDevice(s.device);
    if (s.own_stream) cudaStreamDestroy(s.stream);
  }
  for (auto& d : e->devs) d.second->weights.release();
  delete e;
}

tsv_status tsv_nccl_unique_id(uint8_t out[128]) {
  if (!out) return fail(TSV_E_INVAL, "null argument");
  ncclUniqueId id;
  NK(ncclGetUniqueId(&id));
  static_assert(sizeof(id) == 128, "ncclUniqueId size");
  memcpy(out, &id, 128);
  return TSV_OK;
}

tsv_status tsv_engine_init_world(tsv_engine* e, const uint8_t nccl_id[128]) {
  if (!e || !nccl_id) return fail(TSV_E_INVAL, "null argument");
  if (e->n_local != 1) return fail(TSV_E_UNSUPPORTED, "world communicator needs one local rank per process");
  if (e->world_comm) return TSV_OK;
  ncclUniqueId id;
  memcpy(&id, nccl_id, 128);
  CK(cudaSetDevice(e->slots[0].device));
  NK(ncclCommInitRank(&e->world_comm, e->world, id, e->rank_base));
  return TSV_OK;
}

tsv_status tsv_group_create(tsv_engine* e, const int* ranks, int k, const uint8_t* nccl_id, tsv_group* out) {
  if (!e || !ranks || !out) return fail(TSV_E_INVAL, "null argument");
  if (k < 1 || (k & (k - 1))) return fail(TSV_E_INVAL, "k = %d is not a power of two (P:225)", k);
  if (k > e->world) return fail(TSV_E_INVAL, "k = %d exceeds the world size %d", k, e->world);
  for (int i = 0; i < k; ++i) {
    if (ranks[i] < 0 || ranks[i] >= e->world) return fail(TSV_E_INVAL, "rank %d outside the world", ranks[i]);
    for (int j = 0; j < i; ++j)
      if (ranks[j] == ranks[i]) return fail(TSV_E_INVAL, "duplicate rank %d", ranks[i]);
  }
  if (e->model.H % k) return fail(TSV_E_UNSUPPORTED, "k = %d does not divide the head count %d (S24)", k, e->model.H);
  if ((e->model.h / k) % 64) return fail(TSV_E_UNSUPPORTED, "hidden/k must be a multiple of 64");
  TRY(ensure_init(e));
  Group g;
  g.ranks.assign(ranks, ranks + k);
  g.k = k;
  for (int i = 0; i < k; ++i) {
    const int si = e->slot_of_rank(ranks[i]);
    if (si >= 0) { g.local_slots.push_back(si); g.local_positions.push_back(i); }
    else g.all_local = false;
  }
  if (!g.all_local && !g.local_slots.empty()) {
    if (g.local_slots.size() != 1) return fail(TSV_E_UNSUPPORTED, "mixed local/remote groups need one local rank");
    Slot& s = e->slots[g.local_slots[0]];
    CK(cudaSetDevice(s.device));
    if (nccl_id) {
      ncclUniqueId id;
      memcpy(&id, nccl_id, 128);
      NK(ncclCommInitRank(&g.comm, k, id, g.local_positions[0]));
    } else if (e->world_comm) {
      NK(ncclCommSplit(e->world_comm, 1, g.local_positions[0], &g.comm, nullptr));
    }
  }
  if (!g.all_local && g.comm) {
    Slot& s = e->slots[g.local_slots[0]];
    // warm the communicator once
    DevBuf tmp;
    TRY(dev_alloc(tmp, s.device, 256 * k));
    NK(ncclGroupStart());
    for (int p = 0; p < k; ++p) {
      NK(ncclSend(reinterpret_cast<uint8_t*>(tmp.p) + 0, 64, ncclUint8, p, g.comm, s.stream));
      NK(ncclRecv(reinterpret_cast<uint8_t*>(tmp.p) + 128 + 0, 64, ncclUint8, p, g.comm, s.stream));
    }
    NK(ncclGroupEnd());
    CK(cudaStreamSynchronize(s.stream));
    tmp.release();
  } else if (!g.all_local && g.local_slots.empty() && !nccl_id && e->world_comm) {
    ncclComm_t none = nullptr;
    NK(ncclCommSplit(e->world_comm, NCCL_SPLIT_NOCOLOR, 0, &none, nullptr));
  }
  if (g.all_local) {
    // order local_slots by group rank (already in group order); events for the in-process a2a
    for (int i = 0; i < k; ++i) {
      Slot& s = e->slots[g.local_slots[i]];
      CK(cudaSetDevice(s.device));
      cudaEvent_t a, b;
      CK(cudaEventCreateWithFlags(&a, cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&b, cudaEventDisableTiming));
      g.ev_a.push_back(a);
      g.ev_b.push_back(b);
    }
  }
  e->groups.push_back(std::move(g));
  *out = (tsv_group)e->groups.size() - 1;
  return TSV_OK;
}

// ------------------------------------------------------------------ cross-process fused transport
namespace {
struct IpcBlob {
  uint32_t magic;
  int32_t rank;
  int64_t tokens;
  int32_t evals;
  int32_t pad;
  cudaIpcMemHandle_t recv, cat, flags;
};
}  // namespace

tsv_status tsv_group_ipc_export(tsv_engine* e, tsv_group gi, int64_t max_tokens, int max_evals, uint8_t* out,
                                size_t* len) {
  if (!e || !len) return fail(TSV_E_INVAL, "null argument");
  if (gi < 0 || gi >= (int)e->groups.size()) return fail(TSV_E_INVAL, "unknown group %d", gi);
  Group& g = e->groups[gi];
  if (g.all_local || g.local_slots.size() != 1) return fail(TSV_E_UNSUPPORTED, "IPC windows are for groups spanning processes with one local rank");
  if (max_tokens <= 0 || max_evals < 1 || max_evals > GEMM_MAX_PROBLEMS / 2) return fail(TSV_E_INVAL, "bad window size");
  if (!out) { *len = sizeof(IpcBlob); return TSV_OK; }
  if (*len < sizeof(IpcBlob)) return fail(TSV_E_INVAL, "blob buffer too small (%zu bytes)", sizeof(IpcBlob));
  const Model& m = e->model;
  const int k = g.k;
  Slot& s = e->slots[g.local_slots[0]];
  const int64_t rows_max = max_tokens / k + 2;
  TRY(dev_alloc(g.win_recv, s.device, (size_t)max_evals * max_tokens * 3 * (m.h / k) * 2));
  TRY(dev_alloc(g.win_cat, s.device, (size_t)max_evals * rows_max * (m.h + m.F) * 2));
  TRY(dev_alloc(g.win_flags, s.device, 256 * sizeof(int)));
  CK(cudaSetDevice(s.device));
  CK(cudaMemset(g.win_flags.p, 0, 256 * sizeof(int)));
  CK(cudaDeviceSynchronize());
  IpcBlob b{};
  b.magic = 0x7E7151C0u;
  b.rank = g.local_positions[0];
  b.tokens = max_tokens;
  b.evals = max_evals;
  CK(cudaIpcGetMemHandle(&b.recv, g.win_recv.p));
  CK(cudaIpcGetMemHandle(&b.cat, g.win_cat.p));
  CK(cudaIpcGetMemHandle(&b.flags, g.win_flags.p));
  memcpy(out, &b, sizeof b);
  *len = sizeof b;
  g.win_tokens = max_tokens;
  g.win_evals = max_evals;
  return TSV_OK;
}

tsv_status tsv_group_ipc_import(tsv_engine* e, tsv_group gi, const uint8_t* blobs, size_t blob_len) {
  if (!e || !blobs) return fail(TSV_E_INVAL, "null argument");
  if (gi < 0 || gi >= (int)e->groups.size()) return fail(TSV_E_INVAL, "unknown group %d", gi);
  Group& g = e->groups[gi];
  if (!g.win_recv.p) return fail(TSV_E_STATE, "export this rank's windows first");
  if (blob_len != sizeof(IpcBlob)) return fail(TSV_E_INVAL, "blob length %zu, expected %zu", blob_len, sizeof(IpcBlob));
  const int k = g.k, me = g.local_positions[0];
  Slot& s = e->slots[g.local_slots[0]];
  CK(cudaSetDevice(s.device));
  g.peer_recv.assign(k, nullptr);
  g.peer_cat.assign(k, nullptr);
  g.peer_flags.assign(k, nullptr);
  for (int d = 0; d < k; ++d) {
    IpcBlob b;
    memcpy(&b, blobs + (size_t)d * sizeof(IpcBlob), sizeof b);
    if (b.magic != 0x7E7151C0u || b.rank != d) return fail(TSV_E_INVAL, "blob %d is not group rank %d's", d, d);
    if (b.tokens != g.win_tokens || b.evals != g.win_evals) return fail(TSV_E_INVAL, "members exported different window sizes");
    if (d == me) {
      g.peer_recv[d] = g.win_recv.p;
      g.peer_cat[d] = g.win_cat.p;
      g.peer_flags[d] = g.win_flags.p;
      continue;
    }
    void* pr = nullptr;
    void* pc = nullptr;
    void* pf = nullptr;
    CK(cudaIpcOpenMemHandle(&pr, b.recv, cudaIpcMemLazyEnablePeerAccess));
    CK(cudaIpcOpenMemHandle(&pc, b.cat, cudaIpcMemLazyEnablePeerAccess));
    CK(cudaIpcOpenMemHandle(&pf, b.flags, cudaIpcMemLazyEnablePeerAccess));
    g.opened.insert(g.opened.end(), {pr, pc, pf});
    g.peer_recv[d] = pr;
    g.peer_cat[d] = pc;
    g.peer_flags[d] = pf;
  }
  g.ipc = true;
  return TSV_OK;
}

tsv_status tsv_request_create(tsv_engine* e, int height, int width, int num_steps, uint64_t seed, float guidance,
                              tsv_request* out) {
  if (!e || !out) return fail(TSV_E_INVAL, "null argument");
  if (height <= 0 || width <= 0 || height % 16 || width % 16)
    return fail(TSV_E_INVAL, "height and width must be positive multiples of 16 (P:442)");
  if (num_steps < 1) return fail(TSV_E_INVAL, "num_steps must be >= 1");
  const Model& m = e->model;
  Request R;
  R.height = height; R.width = width; R.S = num_steps; R.seed = seed; R.guidance = guidance;
  R.Li = (int64_t)(height / 16) * (width / 16);
  R.Lt = m.Lt;
  // inputs live in pinned host memory: the first landing's copies do not wait on the device
  TRY(R.x_host.alloc((size_t)R.Li * m.in));
  for (size_t i = 0; i < R.x_host.size(); ++i) R.x_host.p[i] = synth_r(seed, 1, i) * synth_scale(1.0);
  // T, y of evaluation b: SYNTH-1 ids (2, 3) for b = 0 and (4, 5) for SD3's unconditional b = 1
  const size_t nT = (size_t)R.Lt * m.ctx;
  const float c1 = synth_scale(1.0);
  TRY(R.T_host.alloc(nT * m.B));
  TRY(R.y_host.alloc((size_t)m.vec * m.B));
  for (int b = 0; b < m.B; ++b) {
    for (size_t i = 0; i < nT; ++i) R.T_host.p[b * nT + i] = f32_to_bf16_bits(synth_r(seed, 2 + 2 * b, i) * c1);
    for (int i = 0; i < m.vec; ++i) R.y_host.p[(size_t)b * m.vec + i] = f32_to_bf16_bits(synth_r(seed, 3 + 2 * b, i) * c1);
  }
  R.ts.resize(num_steps + 1);
  if (m.sd3) {
    // SD3: t_j = s u / (1 + (s - 1) u), u = 1 - j/S (shift s = 3; S20)
    const double sh = m.d.shift;
    for (int j = 0; j <= num_steps; ++j) {
      const double u = 1.0 - (double)j / num_steps;
      R.ts[j] = sh * u / (1.0 + (sh - 1.0) * u);
    }
  } else {
    // schedule t_j = sigma(1 - j/S), sigma(u) = e^mu / (e^mu + (1/u - 1)), mu linear in L_i
    const double mu = 0.5 + (1.15 - 0.5) / (4096.0 - 256.0) * ((double)R.Li - 256.0);
    for (int j = 0; j <= num_steps; ++j) {
      const double u = 1.0 - (double)j / num_steps;
      R.ts[j] = u > 0 ? std::exp(mu) / (std::exp(mu) + (1.0 / u - 1.0)) : 0.0;
    }
  }
  R.ts[0] = 1.0;
  R.ts[num_steps] = 0.0;
  const int64_t id = e->next_req++;
  R.id = id;
  e->requests.emplace(id, std::move(R));
  *out = id;
  return TSV_OK;
}

static Request* get_req(tsv_engine* e, tsv_request r) {
  auto it = e->requests.find(r);
  return it == e->requests.end() ? nullptr : &it->second;
}

tsv_status tsv_request_set_inputs(tsv_engine* e, tsv_request r, const float* x, const uint16_t* T, const uint16_t* y) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  Request* R = get_req(e, r);
  if (!R) return fail(TSV_E_INVAL, "unknown request %lld", (long long)r);
  if (R->group >= 0 || R->next_step > 0) return fail(TSV_E_STATE, "inputs can only be set before the first step");
  if (x) memcpy(R->x_host.data(), x, R->x_host.size() * 4);
  if (T) memcpy(R->T_host.data(), T, R->T_host.size() * 2);
  if (y) memcpy(R->y_host.data(), y, R->y_host.size() * 2);
  return TSV_OK;
}

tsv_status tsv_request_step(tsv_engine* e, tsv_request r, int step, tsv_group gi, tsv_event* done) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  Request* R = get_req(e, r);
  if (!R) return fail(TSV_E_INVAL, "unknown request %lld", (long long)r);
  if (gi < 0 || gi >= (int)e->groups.size()) return fail(TSV_E_INVAL, "unknown group %d", gi);
  if (step != R->next_step)
    return fail(TSV_E_STATE, "step %d requested but the next step is %d (step dependency, P:235-239)", step,
                R->next_step);
  if (step >= R->S) return fail(TSV_E_STATE, "request has only %d steps", R->S);
  return do_step(e, std::vector<Request*>{R}, gi, done);
}

tsv_status tsv_request_step_batch(tsv_engine* e, const tsv_request* reqs, int n, tsv_group gi, tsv_event* done) {
  if (!e || !reqs) return fail(TSV_E_INVAL, "null argument");
  if (gi < 0 || gi >= (int)e->groups.size()) return fail(TSV_E_INVAL, "unknown group %d", gi);
  const int max_req = GEMM_MAX_PROBLEMS / (2 * e->model.B);
  if (n < 1 || n > max_req) return fail(TSV_E_INVAL, "batch of %d requests (1..%d for this model)", n, max_req);
  std::vector<Request*> Rs;
  for (int i = 0; i < n; ++i) {
    Request* R = get_req(e, reqs[i]);
    if (!R) return fail(TSV_E_INVAL, "unknown request %lld", (long long)reqs[i]);
    for (Request* o : Rs)
      if (o == R) return fail(TSV_E_INVAL, "request %lld appears twice", (long long)reqs[i]);
    if (R->next_step >= R->S) return fail(TSV_E_STATE, "request %lld has no step left", (long long)reqs[i]);
    if (!Rs.empty() && (R->height != Rs[0]->height || R->width != Rs[0]->width))
      return fail(TSV_E_INVAL, "a batch needs one resolution (P:411)");
    Rs.push_back(R);
  }
  return do_step(e, Rs, gi, done);
}

tsv_status tsv_request_reshard(tsv_engine* e, tsv_request r, tsv_group gi, tsv_event* done) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  Request* R = get_req(e, r);
  if (!R) return fail(TSV_E_INVAL, "unknown request %lld", (long long)r);
  if (gi < 0 || gi >= (int)e->groups.size()) return fail(TSV_E_INVAL, "unknown group %d", gi);
  if (R->group != gi) TRY(move_request(e, *R, gi));
  if (done) TRY(new_event(e, e->groups[gi].local_slots, done, gi));
  return TSV_OK;
}

tsv_status tsv_group_record(tsv_engine* e, tsv_group gi, tsv_event* out) {
  if (!e || !out) return fail(TSV_E_INVAL, "null argument");
  if (gi < 0 || gi >= (int)e->groups.size()) return fail(TSV_E_INVAL, "unknown group %d", gi);
  return new_event(e, e->groups[gi].local_slots, out, gi);
}

// A group over CUDA-IPC windows: did its device barrier give up on a stalled member (flag 62 of this
// rank's window, set by ipc_barrier_kernel)?  Called once the event's work completed.
static tsv_status check_ipc_barrier(tsv_engine* e, int gi) {
  if (gi < 0 || gi >= (int)e->groups.size()) return TSV_OK;
  Group& g = e->groups[gi];
  if (!g.ipc || !g.win_flags.p) return TSV_OK;
  if (!g.ipc_failed) {
    int flag = 0;
    CK(cudaSetDevice(g.win_flags.device));
    CK(cudaMemcpy(&flag, reinterpret_cast<int*>(g.win_flags.p) + 62, sizeof(int), cudaMemcpyDeviceToHost));
    g.ipc_failed = flag != 0;
  }
  if (g.ipc_failed)
    return fail(TSV_E_STATE, "group %d: the cross-process barrier timed out waiting for a member (~10 s); the "
                "step's results are invalid and the group must be recreated", gi);
  return TSV_OK;
}

tsv_status tsv_event_release(tsv_engine* e, tsv_event ev) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  if (ev == -1) return TSV_OK;
  if (ev < 0 || ev >= (int64_t)e->events.size() || e->events[ev].evs.empty()) return fail(TSV_E_INVAL, "unknown event");
  for (auto& p : e->events[ev].evs) cudaEventDestroy(p.second);   // legal while pending (released when done)
  e->events[ev].evs.clear();
  e->free_events.push_back(ev);
  return TSV_OK;
}

tsv_status tsv_event_wait(tsv_engine* e, tsv_event ev) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  if (ev == -1) return TSV_OK;
  if (ev < 0 || ev >= (int64_t)e->events.size() || e->events[ev].evs.empty()) return fail(TSV_E_INVAL, "unknown event");
  for (auto& p : e->events[ev].evs) CK(cudaEventSynchronize(p.second));
  return check_ipc_barrier(e, e->events[ev].group);
}

tsv_status tsv_event_query(tsv_engine* e, tsv_event ev, int* done) {
  if (!e || !done) return fail(TSV_E_INVAL, "null argument");
  if (ev == -1) { *done = 1; return TSV_OK; }
  if (ev < 0 || ev >= (int64_t)e->events.size() || e->events[ev].evs.empty()) return fail(TSV_E_INVAL, "unknown event");
  *done = 1;
  for (auto& p : e->events[ev].evs) {
    cudaError_t q = cudaEventQuery(p.second);
    if (q == cudaErrorNotReady) { *done = 0; cudaGetLastError(); }
    else if (q != cudaSuccess) return fail(TSV_E_CUDA, "event query: %s", cudaGetErrorString(q));
  }
  return *done ? check_ipc_barrier(e, e->events[ev].group) : TSV_OK;
}

tsv_status tsv_event_elapsed_ms(tsv_engine* e, tsv_event a, tsv_event b, float* ms) {
  if (!e || !ms) return fail(TSV_E_INVAL, "null argument");
  if (a < 0 || b < 0 || a >= (int64_t)e->events.size() || b >= (int64_t)e->events.size() || e->events[a].evs.empty() ||
      e->events[b].evs.empty())
    return fail(TSV_E_INVAL, "unknown event");
  auto& ea = e->events[a].evs;
  auto& eb = e->events[b].evs;
  if (ea.size() != eb.size()) return fail(TSV_E_INVAL, "events of different groups");
  float mx = 0.f;
  for (size_t i = 0; i < ea.size(); ++i) {
    if (ea[i].first != eb[i].first) return fail(TSV_E_INVAL, "events of different groups");
    CK(cudaEventSynchronize(eb[i].second));
    float t = 0.f;
    CK(cudaEventElapsedTime(&t, ea[i].second, eb[i].second));
    mx = std::max(mx, t);
  }
  *ms = mx;
  TRY(check_ipc_barrier(e, e->events[a].group));
  return check_ipc_barrier(e, e->events[b].group);
}

static tsv_status latent_io(tsv_engine* e, tsv_request r, int64_t row0, int64_t nrows, float* host, bool write,
                            bool velocity) {
  if (!e || !host) return fail(TSV_E_INVAL, "null argument");
  Request* R = get_req(e, r);
  if (!R) return fail(TSV_E_INVAL, "unknown request %lld", (long long)r);
  const int in = e->model.in;
  if (row0 < 0 || nrows < 0 || row0 + nrows > R->Li) return fail(TSV_E_INVAL, "rows out of range");
  if (velocity && !R->has_velocity) return fail(TSV_E_STATE, "no completed step");
  if (R->group < 0) {
    if (velocity) return fail(TSV_E_STATE, "no completed step");
    if (write) memcpy(R->x_host.data() + row0 * in, host, nrows * in * 4);
    else memcpy(host, R->x_host.data() + row0 * in, nrows * in * 4);
    return TSV_OK;
  }
  // rows must be covered by local shards
  int64_t covered = 0;
  for (auto& kv : R->shard) {
    ReqShard& sh = kv.second;
    const int64_t lo = std::max(row0, sh.i0), hi = std::min(row0 + nrows, sh.i0 + sh.ni);
    if (hi <= lo) continue;
    covered += hi - lo;
    Slot& s = e->slots[kv.first];
    CK(cudaSetDevice(s.device));
    float* dev = reinterpret_cast<float*>(velocity ? sh.vel.p : sh.lat.p) + (lo - sh.i0) * in;
    float* hp = host + (lo - row0) * in;
    CK(cudaStreamWaitEvent(s.stream, R->last[kv.first], 0));
    if (write) CK(cudaMemcpyAsync(dev, hp, (hi - lo) * in * 4, cudaMemcpyHostToDevice, s.stream));
    else CK(cudaMemcpyAsync(hp, dev, (hi - lo) * in * 4, cudaMemcpyDeviceToHost, s.stream));
    CK(cudaStreamSynchronize(s.stream));
    TRY(record_last(e, *R, kv.first));
  }
  if (covered != nrows) return fail(TSV_E_INVAL, "rows [%lld, %lld) are not all held by local ranks", (long long)row0,
                                    (long long)(row0 + nrows));
  return TSV_OK;
}

tsv_status tsv_request_read_latent(tsv_engine* e, tsv_request r, int64_t row0, int64_t nrows, float* host) {
  return latent_io(e, r, row0, nrows, host, false, false);
}
tsv_status tsv_request_write_latent(tsv_engine* e, tsv_request r, int64_t row0, int64_t nrows, const float* host) {
  return latent_io(e, r, row0, nrows, const_cast<float*>(host), true, false);
}
tsv_status tsv_request_read_velocity(tsv_engine* e, tsv_request r, int64_t row0, int64_t nrows, float* host) {
  return latent_io(e, r, row0, nrows, host, false, true);
}

tsv_status tsv_request_info(tsv_engine* e, tsv_request r, int* next_step, tsv_group* group, int64_t* li) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  Request* R = get_req(e, r);
  if (!R) return fail(TSV_E_INVAL, "unknown request %lld", (long long)r);
  if (next_step) *next_step = R->next_step;
  if (group) *group = R->group;
  if (li) *li = R->Li;
  return TSV_OK;
}

tsv_status tsv_request_destroy(tsv_engine* e, tsv_request r) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  auto it = e->requests.find(r);
  if (it == e->requests.end()) return fail(TSV_E_INVAL, "unknown request %lld", (long long)r);
  Request& R = it->second;
  for (auto& l : R.last) { cudaEventSynchronize(l.second); cudaEventDestroy(l.second); }
  drop_request_graphs(e, r);
  for (auto& d : R.dev) release_reqdev(d.second);
  for (auto& sh : R.shard) sh.second.release();
  for (auto& ax : R.aux) ax.second.release();
  e->requests.erase(it);
  return TSV_OK;
}

tsv_status tsv_latency_table(tsv_engine* e, const int* res_px, int n_res, const int* ks, int n_k, int warmup,
                             int iters, double* ms_out, double* cv_out) {
  if (!e || !res_px || !ks || !ms_out || n_res <= 0 || n_k <= 0 || iters < 1 || warmup < 0)
    return fail(TSV_E_INVAL, "bad arguments");
  const bool multi = e->n_local < e->world;
  if (multi && !e->world_comm) return fail(TSV_E_STATE, "multi-process latency table needs tsv_engine_init_world");
  for (int i = 0; i < n_res; ++i)
    for (int j = 0; j < n_k; ++j) {
      const int k = ks[j];
      double& out_ms = ms_out[i * n_k + j];
      double* out_cv = cv_out ? &cv_out[i * n_k + j] : nullptr;
      if (k > e->world || k < 1 || (k & (k - 1)) || e->model.H % k) {
        out_ms = -1;
        if (out_cv) *out_cv = -1;
        continue;
      }
      std::vector<int> ranks(k);
      for (int q = 0; q < k; ++q) ranks[q] = q;
      tsv_group g;
      TRY(tsv_group_create(e, ranks.data(), k, nullptr, &g));
      tsv_request rq;
      TRY(tsv_request_create(e, res_px[i], res_px[i], warmup + iters, 1000 + i, 3.5f, &rq));
      std::vector<double> times;
      for (int st = 0; st < warmup + iters; ++st) {
        tsv_event a = -1, b = -1;
        if (st == 0) TRY(tsv_request_reshard(e, rq, g, nullptr));
        if (!e->groups[g].local_slots.empty()) TRY(tsv_group_record(e, g, &a));
        TRY(tsv_request_step(e, rq, st, g, &b));
        float ms = 0.f;
        if (b >= 0) TRY(tsv_event_elapsed_ms(e, a, b, &ms));
        if (multi) {
          // max over ranks
          Slot& s = e->slots[0];
          DevBuf tb;
          TRY(dev_alloc(tb, s.device, 4));
          CK(cudaMemcpyAsync(tb.p, &ms, 4, cudaMemcpyHostToDevice, s.stream));
          NK(ncclAllReduce(tb.p, tb.p, 1, ncclFloat32, ncclMax, e->world_comm, s.stream));
          CK(cudaMemcpyAsync(&ms, tb.p, 4, cudaMemcpyDeviceToHost, s.stream));
          CK(cudaStreamSynchronize(s.stream));
          tb.release();
        }
        if (st >= warmup) times.push_back(ms);
      }
      TRY(tsv_request_destroy(e, rq));
      std::vector<double> sorted = times;
      std::sort(sorted.begin(), sorted.end());
      const size_t n = sorted.size();
      out_ms = n % 2 ? sorted[n / 2] : 0.5 * (sorted[n / 2 - 1] + sorted[n / 2]);
      double mean = 0, var = 0;
      for (double t : times) mean += t;
      mean /= n;
      for (double t : times) var += (t - mean) * (t - mean);
      var = n > 1 ? var / (n - 1) : 0.0;
      if (out_cv) *out_cv = mean > 0 ? std::sqrt(var) / mean : 0.0;
    }
  return TSV_OK;
}

tsv_status tsv_shard_range(int64_t n, int k, int r, int64_t* b, int64_t* en) {
  if (!b || !en || n < 0 || k < 1 || r < 0 || r >= k) return fail(TSV_E_INVAL, "bad shard arguments");
  *b = shard_begin(n, k, r);
  *en = shard_begin(n, k, r + 1);
  return TSV_OK;
}

tsv_status tsv_reshard_plan(int64_t n, int ks, int kd, int64_t* out, int max_copies, int* n_copies) {
  if (!n_copies || n < 0 || ks < 1 || kd < 1 || (max_copies > 0 && !out)) return fail(TSV_E_INVAL, "bad arguments");
  int c = 0;
  for (int s = 0; s < ks; ++s) {
    const int64_t a0 = shard_begin(n, ks, s), a1 = shard_begin(n, ks, s + 1);
    for (int d = 0; d < kd; ++d) {
      const int64_t b0 = shard_begin(n, kd, d), b1 = shard_begin(n, kd, d + 1);
      const int64_t lo = std::max(a0, b0), hi = std::min(a1, b1);
      if (hi <= lo) continue;
      if (c < max_copies) {
        int64_t* o = out + 5 * c;
        o[0] = s; o[1] = lo - a0; o[2] = d; o[3] = lo - b0; o[4] = hi - lo;
      }
      ++c;
    }
  }
  *n_copies = c;
  if (c > max_copies) return fail(TSV_E_INVAL, "plan has %d copies, buffer holds %d", c, max_copies);
  return TSV_OK;
}

tsv_status tsv_a2a_plan(int which, int64_t Lt, int64_t Li, int k, int rank, int64_t* out, int max_ops, int* n_ops) {
  if (!n_ops || (which != 1 && which != 2) || Lt < 0 || Li < 0 || k < 1 || rank < 0 || rank >= k ||
      (max_ops > 0 && !out))
    return fail(TSV_E_INVAL, "bad arguments");
  std::vector<A2AOp> ops;
  a2a_plan(which, Lt, Li, k, rank, ops);
  *n_ops = (int)ops.size();
  if ((int)ops.size() > max_ops) return fail(TSV_E_INVAL, "plan has %d ops, buffer holds %d", (int)ops.size(), max_ops);
  for (size_t i = 0; i < ops.size(); ++i) {
    out[4 * i + 0] = ops[i].peer;
    out[4 * i + 1] = ops[i].send;
    out[4 * i + 2] = ops[i].row0;
    out[4 * i + 3] = ops[i].rows;
  }
  return TSV_OK;
}

tsv_status tsv_debug_read_weight(tsv_engine* e, int id, uint16_t* host, size_t n) {
  if (!e || !host) return fail(TSV_E_INVAL, "null argument");
  const TensorInfo* t = e->model.find(id);
  if (!t) return fail(TSV_E_INVAL, "unknown tensor id %d", id);
  if (n != (size_t)t->numel()) return fail(TSV_E_INVAL, "tensor %d has %lld elements", id, (long long)t->numel());
  TRY(ensure_init(e));
  Slot& s = e->slots[0];
  CK(cudaSetDevice(s.device));
  CK(cudaMemcpy(host, reinterpret_cast<const bf16*>(s.ds->weights.p) + t->offset, n * 2, cudaMemcpyDeviceToHost));
  return TSV_OK;
}

tsv_status tsv_engine_set_transport(tsv_engine* e, int mode) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  if (mode != TSV_TRANSPORT_EXCHANGE && mode != TSV_TRANSPORT_FUSED) return fail(TSV_E_INVAL, "bad transport %d", mode);
  e->transport = mode;
  return TSV_OK;
}

tsv_status tsv_engine_set_graphs(tsv_engine* e, int enable) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  e->graphs = enable != 0;
  return TSV_OK;
}

tsv_status tsv_engine_profile(tsv_engine* e, int enable) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  // events are not recycled: profiled step graphs keep re-recording theirs
  e->prof_recs.clear();
  for (int i = 0; i < 8; ++i) { e->prof_flops[i] = 0; e->prof_bytes[i] = 0; e->prof_launch[i] = 0; }
  e->prof = enable != 0;
  return TSV_OK;
}

tsv_status tsv_engine_profile_read(tsv_engine* e, double* ms, int64_t* launches, double* flops, double* bytes) {
  if (!e) return fail(TSV_E_INVAL, "null engine");
  double acc[8] = {0};
  for (auto& r : e->prof_recs) {
    CK(cudaSetDevice(r.device));
    CK(cudaEventSynchronize(r.b));
    float t = 0.f;
    CK(cudaEventElapsedTime(&t, r.a, r.b));
    acc[r.cls] += t;
  }
  for (int i = 0; i < KC_N; ++i) {
    if (ms) ms[i] = acc[i];
    if (launches) launches[i] = e->prof_launch[i];
    if (flops) flops[i] = e->prof_flops[i];
    if (bytes) bytes[i] = e->prof_bytes[i];
  }
  return TSV_OK;
}

tsv_status tsv_engine_kernel_count(tsv_engine* e, int64_t* count) {
  if (!e || !count) return fail(TSV_E_INVAL, "null argument");
  *count = e->kernel_count;
  return TSV_OK;
}

// ------------------------------------------------------------------ kernel-level ops (tsv_ops.h)
tsv_status tsv_op_gemm(const void* A, int64_t lda, const void* Wt, int64_t ldw, int M, int N, int K, int mode,
                       void* out0, int64_t ld0, void* out1, int64_t ld1, int n_split, const void* bias,
                       const float* gate, const float* scalar, int force_bn, int force_pair, void* stream) {
  if (mode < 0 || mode > EPI_EULER) return fail(TSV_E_INVAL, "bad epilogue mode %d", mode);
  if (force_bn && force_bn != 64 && force_bn != 128 && force_bn != 256) return fail(TSV_E_INVAL, "bad force_bn");
  int dev = 0, sms = 148;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  GemmPlan p;
  const char* err = nullptr;
  GemmEpi epi = epi_of(mode, out0, ld0, reinterpret_cast<const bf16*>(bias), gate, out1, ld1, n_split, scalar);
  if (gemm_plan(&p, reinterpret_cast<const bf16*>(A), lda, reinterpret_cast<const bf16*>(Wt), ldw, M, N, K, epi, sms,
                &err, force_bn, force_pair))
    return fail(TSV_E_INVAL, "%s", err);
  gemm_launch(p, reinterpret_cast<cudaStream_t>(stream));
  CK(cudaGetLastError());
  return TSV_OK;
}

tsv_status tsv_op_gemm_split(const void* A, int64_t lda, const void* Wt, int64_t ldw, int M, int N, int K, int mode,
                             void* out0, int64_t ld0, const void* bias, const float* gate, int splits, int* sem,
                             int sem_ints, float* ws, int64_t ws_bytes, void* stream) {
  if (mode != EPI_RESID_GATE && mode != EPI_ACCUM_F32 && mode != EPI_STORE_F32 && mode != EPI_STORE_BF16 &&
      mode != EPI_GELU_BF16 && mode != EPI_SILU_BF16)
    return fail(TSV_E_INVAL, "split-K op: mode must be STORE_BF16, GELU_BF16, SILU_BF16, STORE_F32, RESID_GATE or ACCUM_F32");
  if (!sem || !ws || splits < 0) return fail(TSV_E_INVAL, "split-K needs counters, a workspace and splits >= 0");
  GemmSplitWs w;
  w.sem = sem;
  w.sem_ints = sem_ints;
  w.ws = ws;
  w.ws_bytes = ws_bytes;
  int dev = 0, sms = 148;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  GemmPlan p;
  const char* err = nullptr;
  GemmEpi epi = epi_of(mode, out0, ld0, reinterpret_cast<const bf16*>(bias), gate, nullptr, 0, 0, nullptr);
  if (gemm_plan(&p, reinterpret_cast<const bf16*>(A), lda, reinterpret_cast<const bf16*>(Wt), ldw, M, N, K, epi, sms,
                &err, 0, -1, &w, splits))
    return fail(TSV_E_INVAL, "%s", err);
  gemm_launch(p, reinterpret_cast<cudaStream_t>(stream));
  CK(cudaGetLastError());
  return TSV_OK;
}

tsv_status tsv_op_gemm_qkv(const void* A, int64_t lda, const void* Wt, int64_t ldw, int M, int N, int K, int mode,
                           void* out0, int64_t ld0, void* out1, int64_t ld1, const void* bias, int h, int D,
                           const void* gq, const void* gk, const float* cosb, const float* sinb, int k_sp,
                           void* pack, int pack_rows, int pack_row0, void* stream) {
  if (mode != EPI_STORE_BF16 && mode != EPI_SPLIT_GELU) return fail(TSV_E_INVAL, "mode must be STORE_BF16 or SPLIT_GELU");
  int dev = 0, sms = 148;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  GemmEpi epi = epi_of(mode, out0, ld0, reinterpret_cast<const bf16*>(bias), nullptr, out1, ld1,
                       mode == EPI_SPLIT_GELU ? 3 * h : 0, nullptr);
  epi.qk_h = h;
  epi.qk_D = D;
  epi.gq = reinterpret_cast<const bf16*>(gq);
  epi.gk = reinterpret_cast<const bf16*>(gk);
  epi.cosb = cosb;
  epi.sinb = sinb;
  epi.k_sp = k_sp;
  epi.pack = reinterpret_cast<bf16*>(pack);
  epi.pack_rows = pack_rows;
  epi.pack_row0 = pack_row0;
  GemmPlan p;
  const char* err = nullptr;
  if (gemm_plan(&p, reinterpret_cast<const bf16*>(A), lda, reinterpret_cast<const bf16*>(Wt), ldw, M, N, K, epi, sms,
                &err, 0))
    return fail(TSV_E_INVAL, "%s", err);
  gemm_launch(p, reinterpret_cast<cudaStream_t>(stream));
  CK(cudaGetLastError());
  return TSV_OK;
}

tsv_status tsv_op_ln_mod(const float* x, int64_t ldx, void* u, int64_t ldu, const float* shift, const float* scale,
                         int M, int h, int impl, void* stream) {
  if (h % 128) return fail(TSV_E_INVAL, "h must be a multiple of 128");
  if (impl < 0 || impl > 2) return fail(TSV_E_INVAL, "bad impl %d", impl);
  const int keep = g_ln_impl;
  g_ln_impl = impl;
  ln_mod_launch(x, ldx, reinterpret_cast<bf16*>(u), ldu, shift, scale, M, h, reinterpret_cast<cudaStream_t>(stream));
  g_ln_impl = keep;
  CK(cudaGetLastError());
  return TSV_OK;
}

tsv_status tsv_op_qk_norm_rope(void* qkv, int64_t ld, int rows, int n_first, int H, int D, const void* gq0,
                               const void* gk0, const void* gq1, const void* gk1, const float* cosb,
                               const float* sinb, void* pack, int k_sp, void* stream) {
  if (D != 64 && D != 128) return fail(TSV_E_INVAL, "D must be 64 or 128");
  if (k_sp < 1 || H % k_sp) return fail(TSV_E_INVAL, "k_sp must divide H");
  qk_norm_rope_launch(reinterpret_cast<bf16*>(qkv), ld, rows, n_first, H, D, reinterpret_cast<const bf16*>(gq0),
                      reinterpret_cast<const bf16*>(gk0), reinterpret_cast<const bf16*>(gq1),
                      reinterpret_cast<const bf16*>(gk1), cosb, sinb, reinterpret_cast<bf16*>(pack), k_sp,
                      reinterpret_cast<cudaStream_t>(stream));
  CK(cudaGetLastError());
  return TSV_OK;
}

tsv_status tsv_op_attention(const void* q, int64_t ldq, const void* k, int64_t ldk, const void* v, int64_t ldv,
                            void* o, int64_t ldo, int L, int H, int D, int impl, void* stream) {
  if (D != 64 && D != 128) return fail(TSV_E_INVAL, "D must be 64 or 128");
  if (impl < 0) return fail(TSV_E_INVAL, "bad attention impl %d", impl);
  const int rc = attention_launch(reinterpret_cast<const bf16*>(q), ldq, reinterpret_cast<const bf16*>(k), ldk,
                                  reinterpret_cast<const bf16*>(v), ldv, reinterpret_cast<bf16*>(o), ldo, L, H, D,
                                  reinterpret_cast<cudaStream_t>(stream), impl == 0 ? 3 : impl);
  if (rc == -3) return fail(TSV_E_INVAL, "bad attention impl %d", impl);
  if (rc == -5) CK(cudaGetLastError());
  if (rc) return fail(TSV_E_INVAL, "attention: operands must be 16-byte aligned with 16-byte row strides");
  CK(cudaGetLastError());
  return TSV_OK;
}

tsv_status tsv_attention_split_plan(int L, int H, int D, int64_t ws_bytes, int cnt_ints, int nsplit, int sms,
                                    int* n_plain, int* n_tail, int* nsplit_out, int* bounds) {
  if (L <= 0 || H <= 0 || (D != 64 && D != 128)) return fail(TSV_E_INVAL, "split plan: L, H > 0 and D in {64, 128}");
  if (nsplit < 0 || !n_plain || !n_tail || !nsplit_out || !bounds) return fail(TSV_E_INVAL, "split plan: bad arguments");
  attention_split_plan(L, H, D, ws_bytes, cnt_ints, nsplit, sms, n_plain, n_tail, nsplit_out, bounds);
  return TSV_OK;
}

tsv_status tsv_op_attention_split(const void* q, int64_t ldq, const void* k, int64_t ldk, const void* v, int64_t ldv,
                                  void* o, int64_t ldo, int L, int H, int D, int nsplit, int* cnt, int cnt_ints,
                                  float* ws, int64_t ws_bytes, void* stream) {
  if (D != 64 && D != 128) return fail(TSV_E_INVAL, "D must be 64 or 128");
  if (!cnt || !ws || nsplit < 0) return fail(TSV_E_INVAL, "KV split needs counters, a workspace and nsplit >= 0");
  AttnSplitWs w;
  w.cnt = cnt;
  w.cnt_ints = cnt_ints;
  w.ws = ws;
  w.ws_bytes = ws_bytes;
  w.force = nsplit;
  if (attention_launch(reinterpret_cast<const bf16*>(q), ldq, reinterpret_cast<const bf16*>(k), ldk,
                       reinterpret_cast<const bf16*>(v), ldv, reinterpret_cast<bf16*>(o), ldo, L, H, D,
                       reinterpret_cast<cudaStream_t>(stream), 3, nullptr, &w))
    return fail(TSV_E_INVAL, "attention: operands must be 16-byte aligned with 16-byte row strides");
  CK(cudaGetLastError());
  return TSV_OK;
}

tsv_status tsv_op_synth(void* dst, uint64_t seed, uint32_t tid, uint64_t idx0, int64_t n, int kind, float c,
                        void* stream) {
  if (kind < 0 || kind > 2) return fail(TSV_E_INVAL, "bad kind");
  synth_launch(dst, seed, tid, idx0, n, kind, c, reinterpret_cast<cudaStream_t>(stream));
  CK(cudaGetLastError());
  return TSV_OK;
}

}  // extern "C"
