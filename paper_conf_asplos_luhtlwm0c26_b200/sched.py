"""Binding of libtsv.so's round-based scheduler (include/tsv_sched.h): argument marshalling only."""
from __future__ import annotations

import ctypes as C

import numpy as np

from ._lib import SchedRequest, check_sched, lib


def _table(T, ks):
    T = np.ascontiguousarray(T, dtype=np.float64)
    ks = list(ks)
    return T, (C.c_int * len(ks))(*ks), T.shape[0], len(ks)


def _reqs(requests):
    arr = (SchedRequest * max(len(requests), 1))()
    for i, (deadline, steps, row) in enumerate(requests):
        arr[i].deadline = deadline
        arr[i].remaining_steps = steps
        arr[i].table_row = row
    return arr


def allocate(T, ks, deadline: float, steps: int, row: int, now: float, N: int):
    """-> (steps per degree (list aligned with ks), late flag)."""
    T, kk, n_res, n_k = _table(T, ks)
    r = _reqs([(deadline, steps, row)])
    out = (C.c_int * n_k)()
    late = C.c_int()
    check_sched(lib.tsv_sched_allocate(T.ctypes.data_as(C.POINTER(C.c_double)), n_res, kk, n_k, r, now, N, out,
                                       C.byref(late)))
    return list(out), bool(late.value)


def schedule_round(T, ks, requests, now: float, tau: float, N: int, work_conserving: bool = False):
    """requests: [(deadline, remaining_steps, table_row)] -> (survivors, [(gpus, steps)]).
    work_conserving: Alg. 1's argmax tie goes to the largest capacity (S31b) instead of the smallest."""
    T, kk, n_res, n_k = _table(T, ks)
    R = len(requests)
    arr = _reqs(requests)
    g = (C.c_int * max(R, 1))()
    s = (C.c_int * max(R, 1))()
    sv = C.c_int()
    check_sched(lib.tsv_sched_round_ex(T.ctypes.data_as(C.POINTER(C.c_double)), n_res, kk, n_k, arr, R, now, tau, N,
                                       1 if work_conserving else 0, g, s, C.byref(sv)))
    return sv.value, [(g[i], s[i]) for i in range(R)]


def place(T, ks, rows, gpus, prev, N: int, scale_up: bool = True):
    """-> [set of GPU ids] per request.  prev: [set of GPU ids held last round] per request."""
    T, kk, n_res, n_k = _table(T, ks)
    R = len(gpus)
    rr = (C.c_int * max(R, 1))(*rows)
    gg = (C.c_int * max(R, 1))(*gpus)
    pm = (C.c_uint64 * max(R, 1))(*[sum(1 << g for g in p) for p in prev])
    out = (C.c_uint64 * max(R, 1))()
    check_sched(lib.tsv_sched_place(T.ctypes.data_as(C.POINTER(C.c_double)), n_res, kk, n_k, rr, gg, pm, R, N,
                                    1 if scale_up else 0, out))
    return [{b for b in range(N) if out[i] >> b & 1} for i in range(R)]
