"""B200-native step-level-SP DiT step (TetriServe's hot path): Python binding of libtsv.so.

The functions below keep the C-ABI's names (without the ``tsv_`` prefix) and only marshal
arguments; every step runs in libtsv.so's sm_100a kernels.  ``Engine`` is a thin owner of an
engine handle with the same methods.
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _lib
from ._lib import EPI, EXPORTED, LIB_PATH, ModelDesc, TsvError, check, last_error, lib  # noqa: F401

__all__ = ["Engine", "ModelDesc", "TsvError", "model_preset", "shard_range", "reshard_plan", "nccl_unique_id",
           "op_gemm", "op_ln_mod", "op_qk_norm_rope", "op_attention", "op_synth", "EPI", "LIB_PATH"]


def model_preset(name: str) -> ModelDesc:
    d = ModelDesc()
    check(lib.tsv_model_preset(name.encode(), C.byref(d)))
    return d


def shard_range(n_rows: int, k: int, rank: int) -> tuple[int, int]:
    b, e = C.c_int64(), C.c_int64()
    check(lib.tsv_shard_range(n_rows, k, rank, C.byref(b), C.byref(e)))
    return b.value, e.value


def reshard_plan(n_rows: int, k_src: int, k_dst: int):
    buf = (C.c_int64 * (5 * (k_src + k_dst)))()
    n = C.c_int()
    check(lib.tsv_reshard_plan(n_rows, k_src, k_dst, buf, k_src + k_dst, C.byref(n)))
    return [tuple(buf[5 * i:5 * i + 5]) for i in range(n.value)]


def a2a_plan(which: int, text_rows: int, image_rows: int, k: int, rank: int):
    """[(peer, is_send, row0, rows)] of the step's Ulysses all-to-all #which for `rank` (tsv_a2a_plan)."""
    cap = 4 * k
    buf = (C.c_int64 * (4 * cap))()
    n = C.c_int()
    check(lib.tsv_a2a_plan(which, text_rows, image_rows, k, rank, buf, cap, C.byref(n)))
    return [tuple(buf[4 * i:4 * i + 4]) for i in range(n.value)]


def nccl_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    check(lib.tsv_nccl_unique_id(buf))
    return bytes(buf)


def _f32p(a: np.ndarray):
    assert a.dtype == np.float32 and a.flags.c_contiguous
    return a.ctypes.data_as(C.POINTER(C.c_float))


def _u16p(a: np.ndarray):
    assert a.dtype == np.uint16 and a.flags.c_contiguous
    return a.ctypes.data_as(C.POINTER(C.c_uint16))


class Engine:
    """Owns a tsv_engine*.  ``devices[i]`` hosts global rank ``rank_base + i``."""

    def __init__(self, model: str | ModelDesc = "flux", devices=(0,), rank_base: int = 0,
                 world_size: int | None = None, weight_seed: int = 0x7E7125E7):
        desc = model_preset(model) if isinstance(model, str) else model
        self.desc = desc
        devs = (C.c_int * len(devices))(*devices)
        self.n_local = len(devices)
        self.world_size = world_size if world_size is not None else rank_base + len(devices)
        h = C.c_void_p()
        check(lib.tsv_engine_create(C.byref(desc), devs, len(devices), rank_base, self.world_size, weight_seed,
                                    C.byref(h)))
        self.h = h
        self._groups: dict[tuple, int] = {}

    def close(self):
        if self.h:
            lib.tsv_engine_destroy(self.h)
            self.h = None

    # --------------------------------------------------------------- PyTorch hooks (before the first group)
    def use_torch_allocator(self):
        """Back every engine buffer (except CUDA-IPC windows) with PyTorch's caching allocator
        (tsv_engine_set_allocator); the callbacks only forward to torch.cuda.caching_allocator_*."""
        import torch

        def _alloc(ctx, nbytes, device, stream):
            try:
                return torch.cuda.caching_allocator_alloc(int(nbytes), device, stream or 0)
            except Exception:   # OOM: the engine reports TSV_E_OOM
                return None

        def _free(ctx, ptr, device, stream):
            torch.cuda.caching_allocator_delete(ptr)

        self._alloc_cb = _lib.ALLOC_FN(_alloc)   # kept alive as long as the engine
        self._free_cb = _lib.FREE_FN(_free)
        check(lib.tsv_engine_set_allocator(self.h, None, self._alloc_cb, self._free_cb))

    def set_stream(self, device: int, stream):
        """Issue every rank on `device` on `stream` (a torch.cuda.Stream or a raw cudaStream_t)."""
        handle = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
        self._streams = getattr(self, "_streams", []) + [stream]   # keep the caller's stream alive
        check(lib.tsv_engine_set_stream(self.h, device, C.c_void_p(handle)))

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # --------------------------------------------------------------- groups
    def init_world(self, nccl_id: bytes):
        check(lib.tsv_engine_init_world(self.h, (C.c_uint8 * 128).from_buffer_copy(nccl_id)))

    def group_create(self, ranks, nccl_id: bytes | None = None) -> int:
        ranks = tuple(int(r) for r in ranks)
        if ranks in self._groups and nccl_id is None:
            return self._groups[ranks]
        arr = (C.c_int * len(ranks))(*ranks)
        g = C.c_int32()
        idp = (C.c_uint8 * 128).from_buffer_copy(nccl_id) if nccl_id is not None else None
        check(lib.tsv_group_create(self.h, arr, len(ranks), idp, C.byref(g)))
        self._groups[ranks] = g.value
        return g.value

    def group_ipc_export(self, group: int, max_tokens: int, max_evals: int = 2) -> bytes:
        """Step 1 of the cross-process fused transport: this rank's window handles (a blob)."""
        n = C.c_size_t(0)
        check(lib.tsv_group_ipc_export(self.h, group, max_tokens, max_evals, None, C.byref(n)))
        buf = (C.c_uint8 * n.value)()
        check(lib.tsv_group_ipc_export(self.h, group, max_tokens, max_evals, buf, C.byref(n)))
        return bytes(buf)

    def group_ipc_import(self, group: int, blobs) -> None:
        """Step 3: every member's blob, in group-rank order."""
        joined = b"".join(blobs)
        arr = (C.c_uint8 * len(joined)).from_buffer_copy(joined)
        check(lib.tsv_group_ipc_import(self.h, group, arr, len(blobs[0])))

    # --------------------------------------------------------------- requests
    def request_create(self, height: int, width: int, num_steps: int = 20, seed: int = 1000,
                       guidance: float = 3.5) -> int:
        r = C.c_int64()
        check(lib.tsv_request_create(self.h, height, width, num_steps, seed, guidance, C.byref(r)))
        return r.value

    def request_set_inputs(self, req: int, x=None, T_bits=None, y_bits=None):
        check(lib.tsv_request_set_inputs(self.h, req, _f32p(x) if x is not None else None,
                                         _u16p(T_bits) if T_bits is not None else None,
                                         _u16p(y_bits) if y_bits is not None else None))

    def request_step(self, req: int, step: int, group: int) -> int:
        ev = C.c_int64(-1)
        check(lib.tsv_request_step(self.h, req, step, group, C.byref(ev)))
        return ev.value

    def request_step_batch(self, reqs, group: int) -> int:
        """The next step of every request in `reqs` (same resolution) as one batched step."""
        arr = (C.c_int64 * len(reqs))(*reqs)
        ev = C.c_int64(-1)
        check(lib.tsv_request_step_batch(self.h, arr, len(reqs), group, C.byref(ev)))
        return ev.value

    def request_reshard(self, req: int, group: int) -> int:
        ev = C.c_int64(-1)
        check(lib.tsv_request_reshard(self.h, req, group, C.byref(ev)))
        return ev.value

    def event_wait(self, ev: int):
        check(lib.tsv_event_wait(self.h, ev))

    def event_release(self, ev: int):
        check(lib.tsv_event_release(self.h, ev))

    def event_query(self, ev: int) -> bool:
        d = C.c_int()
        check(lib.tsv_event_query(self.h, ev, C.byref(d)))
        return bool(d.value)

    def group_record(self, group: int) -> int:
        ev = C.c_int64()
        check(lib.tsv_group_record(self.h, group, C.byref(ev)))
        return ev.value

    def event_elapsed_ms(self, a: int, b: int) -> float:
        ms = C.c_float()
        check(lib.tsv_event_elapsed_ms(self.h, a, b, C.byref(ms)))
        return ms.value

    def request_info(self, req: int):
        ns, g, li = C.c_int(), C.c_int32(), C.c_int64()
        check(lib.tsv_request_info(self.h, req, C.byref(ns), C.byref(g), C.byref(li)))
        return ns.value, g.value, li.value

    def read_latent(self, req: int, row0: int = 0, nrows: int | None = None, out: np.ndarray | None = None):
        li = self.request_info(req)[2]
        nrows = li - row0 if nrows is None else nrows
        out = np.empty((nrows, self.desc.in_ch), np.float32) if out is None else out
        check(lib.tsv_request_read_latent(self.h, req, row0, nrows, _f32p(out)))
        return out

    def write_latent(self, req: int, x: np.ndarray, row0: int = 0):
        x = np.ascontiguousarray(x, dtype=np.float32)
        check(lib.tsv_request_write_latent(self.h, req, row0, x.shape[0], _f32p(x)))

    def read_velocity(self, req: int, row0: int = 0, nrows: int | None = None):
        li = self.request_info(req)[2]
        nrows = li - row0 if nrows is None else nrows
        out = np.empty((nrows, self.desc.in_ch), np.float32)
        check(lib.tsv_request_read_velocity(self.h, req, row0, nrows, _f32p(out)))
        return out

    def request_destroy(self, req: int):
        check(lib.tsv_request_destroy(self.h, req))

    def latency_table(self, res_px, ks, warmup: int = 3, iters: int = 20):
        res_px, ks = list(res_px), list(ks)
        ms = (C.c_double * (len(res_px) * len(ks)))()
        cv = (C.c_double * (len(res_px) * len(ks)))()
        check(lib.tsv_latency_table(self.h, (C.c_int * len(res_px))(*res_px), len(res_px),
                                    (C.c_int * len(ks))(*ks), len(ks), warmup, iters, ms, cv))
        return (np.array(ms[:]).reshape(len(res_px), len(ks)), np.array(cv[:]).reshape(len(res_px), len(ks)))

    def debug_read_weight(self, tensor_id: int, n: int) -> np.ndarray:
        out = np.empty(n, np.uint16)
        check(lib.tsv_debug_read_weight(self.h, tensor_id, _u16p(out), n))
        return out

    PROF_CLASSES = ("gemm", "attention", "ln_mod", "qk_norm_rope", "a2a", "other")

    def set_transport(self, fused: bool = True):
        """Ulysses all-to-alls of in-process groups: fused into the epilogues (default) or the
        pack / exchange / unpack baseline."""
        check(lib.tsv_engine_set_transport(self.h, 1 if fused else 0))

    def set_graphs(self, enable: bool = True):
        check(lib.tsv_engine_set_graphs(self.h, int(enable)))

    def profile(self, enable: bool = True):
        check(lib.tsv_engine_profile(self.h, int(enable)))

    def profile_read(self) -> dict:
        n = len(self.PROF_CLASSES)
        ms, fl, by = (C.c_double * n)(), (C.c_double * n)(), (C.c_double * n)()
        la = (C.c_int64 * n)()
        check(lib.tsv_engine_profile_read(self.h, ms, la, fl, by))
        return {c: dict(ms=ms[i], launches=la[i], flops=fl[i], bytes=by[i]) for i, c in enumerate(self.PROF_CLASSES)}

    def kernel_count(self) -> int:
        c = C.c_int64()
        check(lib.tsv_engine_kernel_count(self.h, C.byref(c)))
        return c.value


# ------------------------------------------------------------------- kernel-level ops (device pointers)
def _ptr(t):
    if t is None:
        return None
    return C.c_void_p(t.data_ptr() if hasattr(t, "data_ptr") else int(t))


def _stream(stream):
    if stream is None:
        import torch
        return C.c_void_p(torch.cuda.current_stream().cuda_stream)
    return C.c_void_p(int(stream))


def op_gemm(A, W, mode, out0, out1=None, bias=None, gate=None, scalar=None, n_split=0, M=None, N=None, K=None,
            lda=None, ldw=None, ld0=None, ld1=None, force_bn=0, force_pair=-1, stream=None):
    M = A.shape[0] if M is None else M
    K = A.shape[1] if K is None else K
    N = W.shape[0] if N is None else N
    lda = A.stride(0) if lda is None else lda
    ldw = W.stride(0) if ldw is None else ldw
    ld0 = out0.stride(0) if ld0 is None else ld0
    ld1 = (out1.stride(0) if out1 is not None else 0) if ld1 is None else ld1
    check(lib.tsv_op_gemm(_ptr(A), lda, _ptr(W), ldw, M, N, K, EPI[mode] if isinstance(mode, str) else mode,
                          _ptr(out0), ld0, _ptr(out1), ld1, n_split, _ptr(bias), _ptr(gate), _ptr(scalar), force_bn, force_pair,
                          _stream(stream)))


def op_gemm_split(A, W, mode, out0, sem, ws, splits=0, bias=None, gate=None, stream=None):
    """Split-K GEMM into the fp32 stream (mode RESID_GATE / ACCUM_F32); sem: zeroed int32 device
    buffer; ws: fp32 device workspace for the partials."""
    M, K = A.shape
    N = W.shape[0]
    check(lib.tsv_op_gemm_split(_ptr(A), A.stride(0), _ptr(W), W.stride(0), M, N, K,
                                EPI[mode] if isinstance(mode, str) else mode, _ptr(out0), out0.stride(0), _ptr(bias),
                                _ptr(gate), splits, _ptr(sem), sem.numel(), _ptr(ws), ws.numel() * 4,
                                _stream(stream)))


def op_gemm_qkv(A, W, out0, h, D, gq, gk, cosb, sinb, bias=None, mode="STORE_BF16", out1=None, ld1=None,
                k_sp=1, pack=None, pack_rows=0, pack_row0=0, stream=None):
    M, K = A.shape
    N = W.shape[0]
    check(lib.tsv_op_gemm_qkv(_ptr(A), A.stride(0), _ptr(W), W.stride(0), M, N, K, EPI[mode], _ptr(out0),
                              out0.stride(0), _ptr(out1), (ld1 or (out1.stride(0) if out1 is not None else 0)),
                              _ptr(bias), h, D, _ptr(gq), _ptr(gk), _ptr(cosb), _ptr(sinb), k_sp, _ptr(pack),
                              pack_rows, pack_row0, _stream(stream)))


def op_ln_mod(x, u, shift, scale, impl=0, stream=None):
    M, h = x.shape
    check(lib.tsv_op_ln_mod(_ptr(x), x.stride(0), _ptr(u), u.stride(0), _ptr(shift), _ptr(scale), M, h, impl,
                            _stream(stream)))


def op_qk_norm_rope(qkv, n_first, H, D, gq0, gk0, gq1, gk1, cosb, sinb, pack=None, k_sp=1, stream=None):
    rows = qkv.shape[0]
    check(lib.tsv_op_qk_norm_rope(_ptr(qkv), qkv.stride(0), rows, n_first, H, D, _ptr(gq0), _ptr(gk0), _ptr(gq1),
                                  _ptr(gk1), _ptr(cosb), _ptr(sinb), _ptr(pack), k_sp, _stream(stream)))


def op_attention_split(q, k, v, o, L, H, D, cnt, ws, nsplit=0, ldq=None, ldk=None, ldv=None, ldo=None, stream=None):
    """The step's attention with the key range split nsplit ways (0: automatic); cnt: zeroed int32
    device buffer, ws: fp32 device workspace."""
    check(lib.tsv_op_attention_split(_ptr(q), ldq or q.stride(0), _ptr(k), ldk or k.stride(0), _ptr(v),
                                     ldv or v.stride(0), _ptr(o), ldo or o.stride(0), L, H, D, nsplit, _ptr(cnt),
                                     cnt.numel(), _ptr(ws), ws.numel() * 4, _stream(stream)))


def attention_split_plan(L, H, D, ws_bytes, cnt_ints, nsplit=0, sms=148):
    """The KV-split plan of an attention launch (host only): dict(n_plain, n_tail, nsplit, bounds)."""
    n_plain, n_tail, ns = C.c_int(), C.c_int(), C.c_int()
    b = (C.c_int * 9)()
    check(lib.tsv_attention_split_plan(L, H, D, ws_bytes, cnt_ints, nsplit, sms, C.byref(n_plain), C.byref(n_tail),
                                       C.byref(ns), b))
    return {"n_plain": n_plain.value, "n_tail": n_tail.value, "nsplit": ns.value, "bounds": list(b)[:ns.value + 1]}


def op_attention(q, k, v, o, L, H, D, ldq=None, ldk=None, ldv=None, ldo=None, impl=0, stream=None):
    """impl 0: the step's tcgen05 kernel; other impl numbers: the kept variants (include/tsv_ops.h)."""
    check(lib.tsv_op_attention(_ptr(q), ldq or q.stride(0), _ptr(k), ldk or k.stride(0), _ptr(v), ldv or v.stride(0),
                               _ptr(o), ldo or o.stride(0), L, H, D, impl, _stream(stream)))


def op_synth(dst, seed, tensor_id, n, kind, c, idx0=0, stream=None):
    check(lib.tsv_op_synth(_ptr(dst), seed, tensor_id, idx0, n, kind, float(c), _stream(stream)))
