"""ctypes binding of libtsv.so (include/tsv.h, include/tsv_ops.h): argument marshalling only.

Every step of the hot path runs in libtsv.so's CUDA kernels.  There is no CPU fallback: if the
library is missing or cannot be loaded this module raises at import time.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TSV_LIB") or os.path.join(_HERE, "libtsv.so")   # TSV_LIB: A/B builds (tools/ab_bench.sh)

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libtsv.so not built ({LIB_PATH}); run `python -c 'import __graft_entry__ as g; g.build()'`")

# libnccl.so.2 is resolved through the rpath baked in at link time (pip nvidia-nccl-cu12 2.28.9).
lib = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)

TSV_OK, TSV_E_INVAL, TSV_E_STATE, TSV_E_OOM, TSV_E_CUDA, TSV_E_NCCL, TSV_E_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
STATUS_NAMES = {0: "TSV_OK", -1: "TSV_E_INVAL", -2: "TSV_E_STATE", -3: "TSV_E_OOM", -4: "TSV_E_CUDA",
                -5: "TSV_E_NCCL", -6: "TSV_E_UNSUPPORTED"}

EPI = dict(STORE_BF16=0, GELU_BF16=1, SILU_BF16=2, SPLIT_GELU=3, RESID_GATE=4, STORE_F32=5, ACCUM_F32=6, EULER=7)


class TsvError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class ModelDesc(C.Structure):
    _fields_ = [("hidden", C.c_int), ("heads", C.c_int), ("head_dim", C.c_int), ("mlp_hidden", C.c_int),
                ("n_double", C.c_int), ("n_single", C.c_int), ("in_ch", C.c_int), ("ctx_dim", C.c_int),
                ("vec_dim", C.c_int), ("text_tokens", C.c_int), ("axes_dim", C.c_int * 3), ("theta", C.c_float),
                ("guidance_embed", C.c_int), ("family", C.c_int), ("cfg_scale", C.c_float), ("shift", C.c_float),
                ("pe_max", C.c_int), ("pe_base", C.c_int)]


FAMILY_FLUX, FAMILY_SD3 = 0, 1


class SchedRequest(C.Structure):
    _fields_ = [("deadline", C.c_double), ("remaining_steps", C.c_int), ("table_row", C.c_int)]


_i32, _i64, _u64, _p, _f32 = C.c_int, C.c_int64, C.c_uint64, C.c_void_p, C.c_float
_P = C.POINTER

# tsv_alloc_fn / tsv_free_fn (include/tsv.h)
ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_void_p, C.c_size_t, C.c_int, C.c_void_p)
FREE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_void_p, C.c_int, C.c_void_p)

_SIGS = {
    "tsv_last_error": (C.c_char_p, []),
    "tsv_model_preset": (_i32, [C.c_char_p, _P(ModelDesc)]),
    "tsv_engine_create": (_i32, [_P(ModelDesc), _P(_i32), _i32, _i32, _i32, _u64, _P(_p)]),
    "tsv_engine_destroy": (None, [_p]),
    "tsv_engine_set_allocator": (_i32, [_p, _p, ALLOC_FN, FREE_FN]),
    "tsv_engine_set_stream": (_i32, [_p, _i32, _p]),
    "tsv_nccl_unique_id": (_i32, [_P(C.c_uint8)]),
    "tsv_engine_init_world": (_i32, [_p, _P(C.c_uint8)]),
    "tsv_group_create": (_i32, [_p, _P(_i32), _i32, _P(C.c_uint8), _P(C.c_int32)]),
    "tsv_group_ipc_export": (_i32, [_p, C.c_int32, _i64, _i32, _P(C.c_uint8), _P(C.c_size_t)]),
    "tsv_group_ipc_import": (_i32, [_p, C.c_int32, _P(C.c_uint8), C.c_size_t]),
    "tsv_request_create": (_i32, [_p, _i32, _i32, _i32, _u64, _f32, _P(_i64)]),
    "tsv_request_set_inputs": (_i32, [_p, _i64, _P(_f32), _P(C.c_uint16), _P(C.c_uint16)]),
    "tsv_request_step": (_i32, [_p, _i64, _i32, C.c_int32, _P(_i64)]),
    "tsv_request_step_batch": (_i32, [_p, _P(_i64), _i32, C.c_int32, _P(_i64)]),
    "tsv_request_reshard": (_i32, [_p, _i64, C.c_int32, _P(_i64)]),
    "tsv_event_wait": (_i32, [_p, _i64]),
    "tsv_event_release": (_i32, [_p, _i64]),
    "tsv_event_query": (_i32, [_p, _i64, _P(_i32)]),
    "tsv_event_elapsed_ms": (_i32, [_p, _i64, _i64, _P(_f32)]),
    "tsv_group_record": (_i32, [_p, C.c_int32, _P(_i64)]),
    "tsv_request_read_latent": (_i32, [_p, _i64, _i64, _i64, _P(_f32)]),
    "tsv_request_write_latent": (_i32, [_p, _i64, _i64, _i64, _P(_f32)]),
    "tsv_request_read_velocity": (_i32, [_p, _i64, _i64, _i64, _P(_f32)]),
    "tsv_request_info": (_i32, [_p, _i64, _P(_i32), _P(C.c_int32), _P(_i64)]),
    "tsv_request_destroy": (_i32, [_p, _i64]),
    "tsv_latency_table": (_i32, [_p, _P(_i32), _i32, _P(_i32), _i32, _i32, _i32, _P(C.c_double), _P(C.c_double)]),
    "tsv_shard_range": (_i32, [_i64, _i32, _i32, _P(_i64), _P(_i64)]),
    "tsv_reshard_plan": (_i32, [_i64, _i32, _i32, _P(_i64), _i32, _P(_i32)]),
    "tsv_a2a_plan": (_i32, [_i32, _i64, _i64, _i32, _i32, _P(_i64), _i32, _P(_i32)]),
    "tsv_debug_read_weight":(_i32, [_p, _i32, _P(C.c_uint16), C.c_size_t]),
    "tsv_engine_kernel_count": (_i32, [_p, _P(_i64)]),
    "tsv_engine_profile": (_i32, [_p, _i32]),
    "tsv_engine_set_graphs": (_i32, [_p, _i32]),
    "tsv_engine_set_transport": (_i32, [_p, _i32]),
    "tsv_engine_profile_read": (_i32, [_p, _P(C.c_double), _P(_i64), _P(C.c_double), _P(C.c_double)]),
    "tsv_op_gemm": (_i32, [_p, _i64, _p, _i64, _i32, _i32, _i32, _i32, _p, _i64, _p, _i64, _i32, _p, _p, _p, _i32, _i32,
                            _p]),
    "tsv_op_gemm_split": (_i32, [_p, _i64, _p, _i64, _i32, _i32, _i32, _i32, _p, _i64, _p, _p, _i32, _p, _i32, _p,
                                  _i64, _p]),
    "tsv_attention_split_plan": (_i32, [_i32, _i32, _i32, _i64, _i32, _i32, _i32, _p, _p, _p, _p]),
    "tsv_op_attention_split": (_i32, [_p, _i64, _p, _i64, _p, _i64, _p, _i64, _i32, _i32, _i32, _i32, _p, _i32, _p,
                                       _i64, _p]),
    "tsv_op_gemm_qkv": (_i32, [_p, _i64, _p, _i64, _i32, _i32, _i32, _i32, _p, _i64, _p, _i64, _p, _i32, _i32,
                               _p, _p, _p, _p, _i32, _p, _i32, _i32, _p]),
    "tsv_op_ln_mod": (_i32, [_p, _i64, _p, _i64, _p, _p, _i32, _i32, _i32, _p]),
    "tsv_op_qk_norm_rope": (_i32, [_p, _i64, _i32, _i32, _i32, _i32, _p, _p, _p, _p, _p, _p, _p, _i32, _p]),
    "tsv_op_attention": (_i32, [_p, _i64, _p, _i64, _p, _i64, _p, _i64, _i32, _i32, _i32, _i32, _p]),
    "tsv_op_synth": (_i32, [_p, _u64, C.c_uint32, _u64, _i64, _i32, _f32, _p]),
    "tsv_sched_allocate": (_i32, [_P(C.c_double), _i32, _P(_i32), _i32, _P(SchedRequest), C.c_double, _i32, _P(_i32),
                                  _P(_i32)]),
    "tsv_sched_round": (_i32, [_P(C.c_double), _i32, _P(_i32), _i32, _P(SchedRequest), _i32, C.c_double, C.c_double,
                               _i32, _P(_i32), _P(_i32), _P(_i32)]),
    "tsv_sched_round_ex": (_i32, [_P(C.c_double), _i32, _P(_i32), _i32, _P(SchedRequest), _i32, C.c_double,
                                  C.c_double, _i32, _i32, _P(_i32), _P(_i32), _P(_i32)]),
    "tsv_sched_place": (_i32, [_P(C.c_double), _i32, _P(_i32), _i32, _P(_i32), _P(_i32), _P(C.c_uint64), _i32, _i32,
                               _i32, _P(C.c_uint64)]),
    "tsv_sched_last_error": (C.c_char_p, []),
}

EXPORTED = sorted(_SIGS)

for _name, (_res, _args) in _SIGS.items():
    _fn = getattr(lib, _name)
    _fn.restype = _res
    _fn.argtypes = _args


def last_error() -> str:
    return lib.tsv_last_error().decode(errors="replace")


def check(status: int) -> None:
    if status != TSV_OK:
        raise TsvError(status, last_error())


def check_sched(status: int) -> None:
    if status != TSV_OK:
        raise TsvError(status, lib.tsv_sched_last_error().decode(errors="replace"))
