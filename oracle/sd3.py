"""Float64 oracle of one SD3-medium-shaped denoising step with classifier-free guidance
(BASELINE.json config 5; S:§8(c) O-SD3).

The paper serves SD3 next to FLUX (P:426 cites [3]) and gives no equations, so the
definitions are the public SD3-medium ones (diffusers SD3Transformer2DModel, which is
not installed on this image): MMDiT joint blocks with separate per-stream weights,
adaLN-Zero modulation, no QK-norm, no RoPE, a 2-D sin-cos position embedding added
after the 2x2 patch embedding, a context_pre_only last block, an AdaLayerNormContinuous
output (chunk order scale, shift, S7), shift-3 flow-matching schedule and CFG batch 2
(v = v_u + s (v_c - v_u), s = 7).  Readings: DESIGN.md S13, S20, S21, S23, S25-S27.

Joint attention runs over [img; txt] (diffusers' concatenation order).  Plain
definitions only; no blocking or fusion.

Test infrastructure only — see oracle/__init__.py.
"""
from __future__ import annotations

import numpy as np

from . import flux as F
from .config import ModelCfg
from .weights import Weights


# ----------------------------------------------------------------------------- schedule
def schedule(cfg: ModelCfg, num_steps: int) -> np.ndarray:
    """sigma_j = s u / (1 + (s - 1) u), u = 1 - j/S, j = 0..S (shift s = 3; S20)."""
    u = np.linspace(1.0, 0.0, num_steps + 1)
    return cfg.shift * u / (1.0 + (cfg.shift - 1.0) * u)


# ----------------------------------------------------------------------------- position embedding
def sincos_1d(dim: int, pos: np.ndarray) -> np.ndarray:
    """[sin(pos w_j), cos(pos w_j)], w_j = 10000^(-j/(dim/2)), j < dim/2.  [n, dim]."""
    half = dim // 2
    omega = 1.0 / 10000.0 ** (np.arange(half, dtype=np.float64) / half)
    a = np.asarray(pos, dtype=np.float64)[:, None] * omega[None, :]
    return np.concatenate([np.sin(a), np.cos(a)], axis=1)


def sincos_2d(h: int, pos_r: np.ndarray, pos_c: np.ndarray) -> np.ndarray:
    """First h/2 channels encode the column coordinate, the last h/2 the row coordinate
    (meshgrid(w, h) puts w first)."""
    return np.concatenate([sincos_1d(h // 2, pos_c), sincos_1d(h // 2, pos_r)], axis=1)


def pos_embed(cfg: ModelCfg, n_r: int, n_c: int) -> np.ndarray:
    """Centre crop of the pe_max x pe_max table whose grid is scaled by pe_base / pe_max:
    patch (r, c), token p = r n_c + c, sits at ((r + top) / 3, (c + left) / 3) with
    top = floor((pe_max - n_r) / 2), left = floor((pe_max - n_c) / 2).  Grids larger than
    pe_max extend the same formula (floor toward -inf, S13).  [n_r n_c, h]."""
    top = (cfg.pe_max - n_r) // 2
    left = (cfg.pe_max - n_c) // 2
    den = cfg.pe_max / cfg.pe_base
    r = np.repeat(np.arange(n_r), n_c)
    c = np.tile(np.arange(n_c), n_r)
    return sincos_2d(cfg.hidden, (r + top) / den, (c + left) / den)


# ----------------------------------------------------------------------------- blocks
def joint_block(cfg: ModelCfg, W: Weights, j: int, img, txt, vec, taps=None):
    """JointTransformerBlock: per-stream AdaLayerNormZero (shift, scale, gate) x 2, separate
    q/k/v linears, joint attention over [img; txt], per-stream out projection and GELU(tanh)
    MLP.  The last block is context_pre_only: its txt stream uses AdaLayerNormContinuous
    (scale, shift), contributes q/k/v only and is dropped (returns txt = None)."""
    H, D = cfg.heads, cfg.head_dim
    last = j == cfg.n_double - 1
    pi, pt = f"joint{j}.img.", f"joint{j}.txt."
    sh1, sc1, g1, sh2, sc2, g2 = F.modulation(W, pi, vec, 6)
    q_i, k_i, v_i = F.split_qkv(F.linear(F.ln_modulate(img, sh1, sc1), W[pi + "qkv.w"], W[pi + "qkv.b"]), H, D)
    if last:
        c_sc, c_sh = F.modulation(W, pt, vec, 2)
        u_t = F.ln_modulate(txt, c_sh, c_sc)
    else:
        c_sh1, c_sc1, c_g1, c_sh2, c_sc2, c_g2 = F.modulation(W, pt, vec, 6)
        u_t = F.ln_modulate(txt, c_sh1, c_sc1)
    q_t, k_t, v_t = F.split_qkv(F.linear(u_t, W[pt + "qkv.w"], W[pt + "qkv.b"]), H, D)
    L_i = img.shape[0]
    o = F.attention(np.concatenate([q_i, q_t]), np.concatenate([k_i, k_t]), np.concatenate([v_i, v_t]))
    o = o.reshape(o.shape[0], H * D)
    o_i, o_t = o[:L_i], o[L_i:]
    img = img + g1 * F.linear(o_i, W[pi + "proj.w"], W[pi + "proj.b"])
    hdn = F.gelu_tanh(F.linear(F.ln_modulate(img, sh2, sc2), W[pi + "fc1.w"], W[pi + "fc1.b"]))
    img = img + g2 * F.linear(hdn, W[pi + "fc2.w"], W[pi + "fc2.b"])
    if last:
        txt = None
    else:
        txt = txt + c_g1 * F.linear(o_t, W[pt + "proj.w"], W[pt + "proj.b"])
        hdn = F.gelu_tanh(F.linear(F.ln_modulate(txt, c_sh2, c_sc2), W[pt + "fc1.w"], W[pt + "fc1.b"]))
        txt = txt + c_g2 * F.linear(hdn, W[pt + "fc2.w"], W[pt + "fc2.b"])
    if taps is not None:
        taps[f"joint{j}"] = (img.copy(), None if txt is None else txt.copy())
    return img, txt


def final_layer(W: Weights, img, vec):
    """norm_out (AdaLayerNormContinuous, chunk order (scale, shift), S7) then proj_out."""
    m = F.linear(F.silu(vec), W["final.mod.w"], W["final.mod.b"])
    scale, shift = np.split(m, 2)
    return F.linear(F.ln_modulate(img, shift, scale), W["final.lin.w"], W["final.lin.b"])


def conditioning_vec(cfg: ModelCfg, W: Weights, t: float, y):
    """temb = TimestepEmbedding(sinusoid(1000 t), [cos, sin]) + PixArt text projection of the
    pooled embedding y (both Linear-SiLU-Linear; the same MLP form as FLUX, no guidance)."""
    return F.conditioning_vec(cfg, W, t, y, 0.0)


def forward(cfg: ModelCfg, W: Weights, x_lat, T, y, t: float, height: int, width: int, taps=None):
    """One transformer evaluation: velocity v [L_i, in] for one branch of the CFG pair."""
    vec = conditioning_vec(cfg, W, t, y)
    img = F.linear(x_lat, W["img_in.w"], W["img_in.b"]) + pos_embed(cfg, height // 16, width // 16)
    txt = F.linear(T, W["txt_in.w"], W["txt_in.b"])
    for j in range(cfg.n_double):
        img, txt = joint_block(cfg, W, j, img, txt, vec, taps)
    return final_layer(W, img, vec)


def sd3_step(cfg: ModelCfg, W: Weights, x_lat, T_c, y_c, T_u, y_u, t: float, t_next: float,
             height: int, width: int, taps=None):
    """CFG step: v = v_u + s (v_c - v_u) over the batch-2 pair [uncond; cond] (S23);
    x_{s+1} = x_s + (t_{s+1} - t_s) v.  Returns (v, x_next)."""
    tu = {} if taps is not None else None
    v_u = forward(cfg, W, x_lat, T_u, y_u, t, height, width, tu)
    v_c = forward(cfg, W, x_lat, T_c, y_c, t, height, width, taps)
    if taps is not None:
        taps.update({k + ".u": v for k, v in tu.items()})
    v = v_u + cfg.cfg_scale * (v_c - v_u)
    return v, x_lat + (t_next - t) * v


def request_step(cfg: ModelCfg, W: Weights, x_lat, T_c, y_c, T_u, y_u, step: int, num_steps: int,
                 height: int, width: int, **kw):
    ts = schedule(cfg, num_steps)
    return sd3_step(cfg, W, x_lat, T_c, y_c, T_u, y_u, ts[step], ts[step + 1], height, width, **kw)
