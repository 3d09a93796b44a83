"""SYNTH-1 counter-hash generator in numpy (see synth/__init__.py for the spec)."""
from __future__ import annotations

import math
import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

GOLDEN_GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64_mix(z: np.ndarray) -> np.ndarray:
    """The splitmix64 output function (Steele, Lea, Flood 2014) on uint64 arrays."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def hash_u64(seed: int, tensor_id: int, idx: np.ndarray) -> np.ndarray:
    key = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) ^ (np.uint64(tensor_id) << np.uint64(48))
    with np.errstate(over="ignore"):
        return splitmix64_mix((np.asarray(idx, dtype=np.uint64) ^ key) + GOLDEN_GAMMA)


def uniform_pm1(seed: int, tensor_id: int, idx: np.ndarray) -> np.ndarray:
    """r in [-1, 1) as float32; exact (24-bit numerator, power-of-two scale)."""
    u = (hash_u64(seed, tensor_id, idx) >> np.uint64(40)).astype(np.int64)
    return ((u - (1 << 23)).astype(np.float32) * np.float32(2.0 ** -23)).astype(np.float32)


def bf16_rne_bits(x: np.ndarray) -> np.ndarray:
    """Round float32 -> bfloat16 (round to nearest even); returns uint16 bits.
    Inputs are finite by construction."""
    b = np.asarray(x, dtype=np.float32).view(np.uint32)
    lsb = (b >> np.uint32(16)) & np.uint32(1)
    with np.errstate(over="ignore"):
        r = (b + np.uint32(0x7FFF) + lsb) >> np.uint32(16)
    return r.astype(np.uint16)


def bf16_bits_to_f32(bits: np.ndarray) -> np.ndarray:
    return (np.asarray(bits, dtype=np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32)


def scale_for(kind: str, fan_in: int | None = None) -> np.float32:
    if kind == "w":
        sigma = 1.0 / math.sqrt(fan_in)
    elif kind == "b":
        sigma = 0.02
    elif kind in ("x", "f"):
        sigma = 1.0
    elif kind == "g":
        sigma = 0.1
    else:
        raise ValueError(kind)
    return np.float32(math.sqrt(3.0) * sigma)


def _gen_chunk(seed, tensor_id, kind, c, lo, hi):
    idx = np.arange(lo, hi, dtype=np.uint64)
    r = uniform_pm1(seed, tensor_id, idx)
    v = (r * c).astype(np.float32)  # one IEEE float32 multiply, RNE
    if kind == "f":
        return v
    if kind == "g":
        v = (np.float32(1.0) + v).astype(np.float32)
    return bf16_rne_bits(v)


_CHUNK = 1 << 22


def gen_tensor_bits(seed: int, tensor_id: int, n: int, kind: str, fan_in: int | None = None,
                    threads: int | None = None) -> np.ndarray:
    """Raw result: uint16 bf16 bits for kinds w/b/x/g, float32 for kind f."""
    c = scale_for(kind, fan_in)
    chunks = [(lo, min(n, lo + _CHUNK)) for lo in range(0, n, _CHUNK)]
    if len(chunks) <= 1:
        return _gen_chunk(seed, tensor_id, kind, c, 0, n)
    threads = threads or min(len(chunks), len(os.sched_getaffinity(0)))
    with ThreadPoolExecutor(threads) as ex:
        parts = list(ex.map(lambda lh: _gen_chunk(seed, tensor_id, kind, c, *lh), chunks))
    return np.concatenate(parts)


def gen_tensor(seed: int, tensor_id: int, shape, kind: str, fan_in: int | None = None,
               dtype=np.float64) -> np.ndarray:
    """Generated tensor as float values (default float64) of the given shape."""
    n = int(np.prod(shape))
    raw = gen_tensor_bits(seed, tensor_id, n, kind, fan_in)
    vals = raw if kind == "f" else bf16_bits_to_f32(raw)
    return vals.astype(dtype).reshape(shape)
