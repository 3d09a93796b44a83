"""Float64 oracle of one FLUX.1-dev-shaped denoising step (S:§8(a) a0-a12, §8(c) O-FLUX).

Every function is the plain definition, in the order the public model states
it (TT = torchtitan's mirror of BFL's FLUX code, cited for architecture facts
only; the paper cites FLUX.1-dev [21] and SD3 [3] without equations, P:100,
P:426).  No blocking, fusion or reordering; attention is the naive
max-subtracted softmax, chunked over queries only to bound memory.

Test infrastructure only — see oracle/__init__.py.
"""
from __future__ import annotations

import math

import numpy as np

from .config import ModelCfg
from .weights import Weights

EPS = 1e-6  # LayerNorm eps (TT:layers.py:170) and RMSNorm eps (BFL; S:§8(c) S6)


# ----------------------------------------------------------------------------- schedule (a0)
def time_shift(mu: float, t: np.ndarray) -> np.ndarray:
    """sigma(t) = e^mu / (e^mu + (1/t - 1)), sigma(0) := 0 (BFL get_schedule; S:§8(c) 1)."""
    t = np.asarray(t, dtype=np.float64)
    out = np.zeros_like(t)
    nz = t > 0
    out[nz] = math.exp(mu) / (math.exp(mu) + (1.0 / t[nz] - 1.0))
    return out


def schedule_mu(L_i: int) -> float:
    """mu = 0.5 + (1.15 - 0.5)(L_i - 256)/(4096 - 256), linear in the image-token count."""
    m = (1.15 - 0.5) / (4096 - 256)
    return 0.5 + m * (L_i - 256)


def schedule(num_steps: int, L_i: int) -> np.ndarray:
    """t_j = sigma(1 - j/S), j = 0..S (t_0 = 1, t_S = 0)."""
    t = np.linspace(1.0, 0.0, num_steps + 1)
    return time_shift(schedule_mu(L_i), t)


# ----------------------------------------------------------------------------- elementwise
def silu(x):
    return x / (1.0 + np.exp(-x))


def gelu_tanh(x):
    """GELU, tanh approximation (nn.GELU(approximate="tanh"), TT:layers.py:185)."""
    return 0.5 * x * (1.0 + np.tanh(math.sqrt(2.0 / math.pi) * (x + 0.044715 * x ** 3)))


def timestep_embedding(t: float, dim: int = 256, max_period: float = 10000.0, factor: float = 1000.0):
    """e(t) = [cos(1000 t f_j), sin(1000 t f_j)], f_j = exp(-ln(max_period) j / (dim/2)) (TT:layers.py:35-54)."""
    half = dim // 2
    f = np.exp(-math.log(max_period) * np.arange(half, dtype=np.float64) / half)
    a = factor * float(t) * f
    return np.concatenate([np.cos(a), np.sin(a)])


def linear(x, w, b=None):
    """y = x W^T + b (nn.Linear)."""
    y = x @ w.T
    return y if b is None else y + b


def mlp_embed(z, w1, b1, w2, b2):
    """MLPEmbedder: W2 SiLU(W1 z + b1) + b2 (TT:layers.py:62-76)."""
    return linear(silu(linear(z, w1, b1)), w2, b2)


def layer_norm(x):
    """LayerNorm without affine, biased variance, eps 1e-6 (TT:layers.py:170)."""
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + EPS)


def modulate(xn, shift, scale):
    """(1 + scale) * xn + shift (TT:layers.py:215-216)."""
    return (1.0 + scale) * xn + shift


def ln_modulate(x, shift, scale):
    """a2: u = LN(x)(1 + scale) + shift."""
    return modulate(layer_norm(x), shift, scale)


def rms_norm(x, g):
    """x * rsqrt(mean(x^2) + eps) * g over the last axis (BFL RMSNorm; eps 1e-6, S:§8(c) S6)."""
    return x / np.sqrt((x ** 2).mean(axis=-1, keepdims=True) + EPS) * g


# ----------------------------------------------------------------------------- RoPE (a4)
def position_ids(L_t: int, height: int, width: int) -> np.ndarray:
    """[L_t + L_i, 3]: text (0,0,0); image token p = r (W/16) + c -> (0, r, c) (S:§8(c) 4)."""
    hp, wp = height // 16, width // 16
    img = np.zeros((hp * wp, 3), dtype=np.float64)
    img[:, 1] = np.repeat(np.arange(hp), wp)
    img[:, 2] = np.tile(np.arange(wp), hp)
    return np.concatenate([np.zeros((L_t, 3)), img], axis=0)


def rope_angles(ids: np.ndarray, axes_dim, theta: float) -> np.ndarray:
    """theta_{p,i}: pair i of axis a (local j) -> id_a * theta^(-2j/d_a) (TT:math.py:21-30). [L, D/2]."""
    cols = []
    for a, d in enumerate(axes_dim):
        j = np.arange(0, d, 2, dtype=np.float64) / d
        omega = 1.0 / (theta ** j)
        cols.append(ids[:, a:a + 1] * omega[None, :])
    return np.concatenate(cols, axis=1)


def apply_rope(x: np.ndarray, ang: np.ndarray) -> np.ndarray:
    """Rotate adjacent pairs: (x0, x1) -> (cos x0 - sin x1, sin x0 + cos x1) (TT:math.py:33-38).
    x [L, H, D], ang [L, D/2]."""
    c = np.cos(ang)[:, None, :]
    s = np.sin(ang)[:, None, :]
    x0 = x[..., 0::2]
    x1 = x[..., 1::2]
    out = np.empty_like(x)
    out[..., 0::2] = c * x0 - s * x1
    out[..., 1::2] = s * x0 + c * x1
    return out


# ----------------------------------------------------------------------------- attention (a6)
def attention(q, k, v, q_chunk: int = 1024):
    """softmax(q k^T / sqrt(D)) v per head, exact max-subtracted softmax (TT:math.py:12-18).
    q, k, v: [L, H, D] -> [L, H, D]."""
    L, H, D = q.shape
    out = np.empty((L, H, D), dtype=np.float64)
    scale = 1.0 / math.sqrt(D)
    for h in range(H):
        kh = k[:, h, :]
        vh = v[:, h, :]
        for s0 in range(0, L, q_chunk):
            s = (q[s0:s0 + q_chunk, h, :] @ kh.T) * scale
            s = s - s.max(axis=1, keepdims=True)
            p = np.exp(s)
            p /= p.sum(axis=1, keepdims=True)
            out[s0:s0 + q_chunk, h, :] = p @ vh
    return out


def split_qkv(qkv, H, D):
    """Columns ordered "(K H D)": [q | k | v] (TT:layers.py:113)."""
    L = qkv.shape[0]
    t = qkv.reshape(L, 3, H, D)
    return t[:, 0], t[:, 1], t[:, 2]


# ----------------------------------------------------------------------------- conditioning (a0)
def conditioning_vec(cfg: ModelCfg, W: Weights, t: float, y, guidance: float):
    """vec = MLP_t(e(t)) + MLP_g(e(g)) + MLP_y(y) (TT:model.py:119-120; FLUX-dev guidance_in, S:§8(c) 2)."""
    vec = mlp_embed(timestep_embedding(t), W["time_in.in.w"], W["time_in.in.b"],
                    W["time_in.out.w"], W["time_in.out.b"])
    if cfg.guidance_embed:
        vec = vec + mlp_embed(timestep_embedding(guidance), W["guidance_in.in.w"], W["guidance_in.in.b"],
                              W["guidance_in.out.w"], W["guidance_in.out.b"])
    vec = vec + mlp_embed(y, W["vector_in.in.w"], W["vector_in.in.b"],
                          W["vector_in.out.w"], W["vector_in.out.b"])
    return vec


def modulation(W: Weights, prefix: str, vec, n_chunks: int):
    """mod = W SiLU(vec) + b, split into n_chunks of h (TT:layers.py:127-146)."""
    m = linear(silu(vec), W[prefix + "mod.w"], W[prefix + "mod.b"])
    return np.split(m, n_chunks)


# ----------------------------------------------------------------------------- blocks
def double_block(cfg: ModelCfg, W: Weights, j: int, img, txt, vec, ang, taps=None):
    """DoubleStreamBlock (TT:layers.py:203-246): separate weights per stream, joint attention
    over [txt; img]."""
    H, D = cfg.heads, cfg.head_dim
    streams = {}
    for sn, x in (("img", img), ("txt", txt)):
        p = f"double{j}.{sn}."
        sh1, sc1, g1, sh2, sc2, g2 = modulation(W, p, vec, 6)
        u = ln_modulate(x, sh1, sc1)
        q, k, v = split_qkv(linear(u, W[p + "qkv.w"], W[p + "qkv.b"]), H, D)
        q = rms_norm(q, W[p + "q_norm.g"])
        k = rms_norm(k, W[p + "k_norm.g"])
        streams[sn] = dict(x=x, q=q, k=k, v=v, g1=g1, sh2=sh2, sc2=sc2, g2=g2)
    L_t = txt.shape[0]
    q = np.concatenate([streams["txt"]["q"], streams["img"]["q"]])
    k = np.concatenate([streams["txt"]["k"], streams["img"]["k"]])
    v = np.concatenate([streams["txt"]["v"], streams["img"]["v"]])
    q = apply_rope(q, ang)
    k = apply_rope(k, ang)
    o = attention(q, k, v).reshape(q.shape[0], H * D)
    outs = {"txt": o[:L_t], "img": o[L_t:]}
    res = {}
    for sn in ("img", "txt"):
        p = f"double{j}.{sn}."
        st = streams[sn]
        x = st["x"] + st["g1"] * linear(outs[sn], W[p + "proj.w"], W[p + "proj.b"])
        u2 = ln_modulate(x, st["sh2"], st["sc2"])
        hdn = gelu_tanh(linear(u2, W[p + "fc1.w"], W[p + "fc1.b"]))
        x = x + st["g2"] * linear(hdn, W[p + "fc2.w"], W[p + "fc2.b"])
        res[sn] = x
    if taps is not None:
        taps[f"double{j}"] = (res["img"].copy(), res["txt"].copy())
    return res["img"], res["txt"]


def single_block(cfg: ModelCfg, W: Weights, j: int, x, vec, ang, taps=None):
    """SingleStreamBlock (TT:layers.py:250-304): parallel linear1 -> [qkv | mlp], linear2 over
    [attn, GELU(mlp)]."""
    h, H, D = cfg.hidden, cfg.heads, cfg.head_dim
    p = f"single{j}."
    sh, sc, g = modulation(W, p, vec, 3)
    u = ln_modulate(x, sh, sc)
    y1 = linear(u, W[p + "lin1.w"], W[p + "lin1.b"])
    qkv, mlp = y1[:, :3 * h], y1[:, 3 * h:]
    q, k, v = split_qkv(qkv, H, D)
    q = apply_rope(rms_norm(q, W[p + "q_norm.g"]), ang)
    k = apply_rope(rms_norm(k, W[p + "k_norm.g"]), ang)
    o = attention(q, k, v).reshape(x.shape[0], h)
    out = linear(np.concatenate([o, gelu_tanh(mlp)], axis=1), W[p + "lin2.w"], W[p + "lin2.b"])
    x = x + g * out
    if taps is not None:
        taps[f"single{j}"] = x.copy()
    return x


def final_layer(W: Weights, img, vec):
    """LastLayer (TT:layers.py:325-329): chunk order (shift, scale)."""
    m = linear(silu(vec), W["final.mod.w"], W["final.mod.b"])
    shift, scale = np.split(m, 2)
    return linear(ln_modulate(img, shift, scale), W["final.lin.w"], W["final.lin.b"])


# ----------------------------------------------------------------------------- one step
def flux_step(cfg: ModelCfg, W: Weights, x_lat, T, y, t: float, t_next: float, guidance: float,
              height: int, width: int, taps=None, drop_weights: bool = True):
    """One denoising step: v = DiT(x_s, t_s, T, y, g);  x_{s+1} = x_s + (t_{s+1} - t_s) v
    (flow-matching Euler, S:§8(a) a12).  Returns (v, x_next)."""
    L_t = T.shape[0]
    vec = conditioning_vec(cfg, W, t, y, guidance)
    img = linear(x_lat, W["img_in.w"], W["img_in.b"])      # a1 (TT:model.py:118)
    txt = linear(T, W["txt_in.w"], W["txt_in.b"])          # a1 (TT:model.py:121)
    ang = rope_angles(position_ids(L_t, height, width), cfg.axes_dim, cfg.theta)
    for j in range(cfg.n_double):
        img, txt = double_block(cfg, W, j, img, txt, vec, ang, taps)
        if drop_weights:
            W.drop(f"double{j}.")
    x = np.concatenate([txt, img])                         # a10 (TT:model.py:129)
    for j in range(cfg.n_single):
        x = single_block(cfg, W, j, x, vec, ang, taps)
        if drop_weights:
            W.drop(f"single{j}.")
    img = x[L_t:]                                          # a10 (TT:model.py:132)
    v = final_layer(W, img, vec)                           # a11
    return v, x_lat + (t_next - t) * v                     # a12


def request_step(cfg: ModelCfg, W: Weights, x_lat, T, y, step: int, num_steps: int, guidance: float,
                 height: int, width: int, **kw):
    ts = schedule(num_steps, x_lat.shape[0])
    return flux_step(cfg, W, x_lat, T, y, ts[step], ts[step + 1], guidance, height, width, **kw)
