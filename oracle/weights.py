"""Lazy float64 access to the synthetic bf16-valued parameters (SYNTH-1)."""
from __future__ import annotations

import numpy as np

import synth
from .config import ModelCfg, WEIGHT_SEED, tensor_table


class Weights:
    """Generates tensors on demand; caches up to ``cache_bytes`` of float64."""

    def __init__(self, cfg: ModelCfg, seed: int = WEIGHT_SEED, cache_bytes: int = 2 << 30,
                 overrides: dict | None = None):
        self.cfg = cfg
        self.seed = seed
        self.table = {name: (tid, shape, kind, fan) for tid, name, shape, kind, fan in tensor_table(cfg)}
        self.cache: dict[str, np.ndarray] = {}
        self.cache_bytes = cache_bytes
        self.overrides = dict(overrides or {})

    def __getitem__(self, name: str) -> np.ndarray:
        if name in self.overrides:
            return self.overrides[name]
        if name in self.cache:
            return self.cache[name]
        tid, shape, kind, fan = self.table[name]
        a = synth.gen_tensor(self.seed, tid, shape, kind, fan)
        if a.nbytes + sum(v.nbytes for v in self.cache.values()) <= self.cache_bytes:
            self.cache[name] = a
        return a

    def drop(self, prefix: str) -> None:
        for k in [k for k in self.cache if k.startswith(prefix)]:
            del self.cache[k]


def request_inputs(cfg: ModelCfg, height: int, width: int, seed: int):
    """x_T [L_i, in] (fp32 values), T [L_t, ctx] and y [vec] (bf16 values), as float64."""
    L_i = (height // 16) * (width // 16)
    x = synth.gen_tensor(seed, 1, (L_i, cfg.in_ch), "f")
    T = synth.gen_tensor(seed, 2, (cfg.text_tokens, cfg.ctx_dim), "x")
    y = synth.gen_tensor(seed, 3, (cfg.vec_dim,), "x")
    return x, T, y


def sd3_request_inputs(cfg: ModelCfg, height: int, width: int, seed: int):
    """SD3 CFG pair: x_T, (T_c, y_c) conditional, (T_u, y_u) unconditional (tensor ids 1-5)."""
    x, T_c, y_c = request_inputs(cfg, height, width, seed)
    T_u = synth.gen_tensor(seed, 4, (cfg.text_tokens, cfg.ctx_dim), "x")
    y_u = synth.gen_tensor(seed, 5, (cfg.vec_dim,), "x")
    return x, T_c, y_c, T_u, y_u
