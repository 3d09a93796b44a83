"""Simulated Ulysses sequence parallelism with k virtual ranks (S:§8(c) O-SP), float64.

Ulysses (cites [18]): tokens are sharded across k ranks; around each
attention an all-to-all transposes tokens<->heads so every rank runs exact
attention over the full joint sequence for H/k heads, and a second
all-to-all returns the output to the token shards.  Step-level SP (P:73,
P:114) re-chooses k per step; the latent moves between groups by
a reshard, which is pure index arithmetic.

Readings: text rows are sharded with the same rule as image rows
(S3); rank r owns contiguous rows [start(n,k,r), start(n,k,r+1)) with
start(n,k,r) = r*floor(n/k) + min(r, n mod k) (S4); heads are contiguous H/k
slices; after the first all-to-all the rows are in the global order
[txt_0..txt_{k-1}; img_0..img_{k-1}] (= the k = 1 order).

Test infrastructure only — see oracle/__init__.py.
"""
from __future__ import annotations

import numpy as np

from . import flux as F
from .config import ModelCfg
from .weights import Weights


def shard_start(n: int, k: int, r: int) -> int:
    return r * (n // k) + min(r, n % k)


def shard_range(n: int, k: int, r: int) -> tuple[int, int]:
    if not (k >= 1 and 0 <= r < k and n >= 0):
        raise ValueError("bad shard")
    return shard_start(n, k, r), shard_start(n, k, r + 1)


def shard(x: np.ndarray, k: int) -> list[np.ndarray]:
    """Row-shard x into k contiguous pieces (copy)."""
    n = x.shape[0]
    return [x[slice(*shard_range(n, k, r))].copy() for r in range(k)]


def gather(parts: list[np.ndarray]) -> np.ndarray:
    return np.concatenate(parts, axis=0)


def reshard_plan(n: int, k_src: int, k_dst: int):
    """Copies (src_rank, src_row0, dst_rank, dst_row0, rows) for reshard k_src -> k_dst:
    the overlaps of the two contiguous partitions of [0, n)."""
    plan = []
    for s in range(k_src):
        a0, a1 = shard_range(n, k_src, s)
        for d in range(k_dst):
            b0, b1 = shard_range(n, k_dst, d)
            lo, hi = max(a0, b0), min(a1, b1)
            if hi > lo:
                plan.append((s, lo - a0, d, lo - b0, hi - lo))
    return plan


def reshard(parts: list[np.ndarray], k_dst: int) -> list[np.ndarray]:
    """Apply reshard_plan element by element (no float ops)."""
    n = sum(p.shape[0] for p in parts)
    out = [np.empty((b - a,) + parts[0].shape[1:], dtype=parts[0].dtype)
           for a, b in (shard_range(n, k_dst, d) for d in range(k_dst))]
    for s, s0, d, d0, m in reshard_plan(n, len(parts), k_dst):
        out[d][d0:d0 + m] = parts[s][s0:s0 + m]
    return out


# ----------------------------------------------------------------------------- simulated SP step
def _a2a_seq_to_head(parts_txt, parts_img, k, H):
    """[rows_r, H, D] per rank (txt and img separately) -> per rank d: [L, H/k, D] with rows in
    the global order [txt_0..txt_{k-1}; img_0..img_{k-1}]."""
    hk = H // k
    out = []
    for d in range(k):
        rows = [p[:, d * hk:(d + 1) * hk] for p in parts_txt] + [p[:, d * hk:(d + 1) * hk] for p in parts_img]
        out.append(np.concatenate(rows))
    return out


def _a2a_head_to_seq(o_parts, k, H, D, L_t, L_i):
    """Inverse of _a2a_seq_to_head: per rank d [L, H/k, D] -> per rank r (txt [t_r, H*D], img [i_r, H*D])."""
    hk = H // k
    txt, img = [], []
    for r in range(k):
        t0, t1 = shard_range(L_t, k, r)
        i0, i1 = shard_range(L_i, k, r)
        t = np.concatenate([o_parts[d][t0:t1] for d in range(k)], axis=1)           # heads d*hk..
        i = np.concatenate([o_parts[d][L_t + i0:L_t + i1] for d in range(k)], axis=1)
        txt.append(t.reshape(t1 - t0, H * D))
        img.append(i.reshape(i1 - i0, H * D))
    return txt, img


def flux_step_sp(cfg: ModelCfg, W: Weights, x_lat, T, y, t: float, t_next: float, guidance: float,
                 height: int, width: int, k: int):
    """The same step as flux.flux_step, computed by k simulated Ulysses ranks.  Row-local work
    (a1-a4, a8-a12) runs per rank on its rows; a6 runs per rank on its head slice over all rows."""
    h, H, D = cfg.hidden, cfg.heads, cfg.head_dim
    if H % k:
        raise ValueError("k must divide the head count (S24)")
    L_t, L_i = T.shape[0], x_lat.shape[0]
    vec = F.conditioning_vec(cfg, W, t, y, guidance)  # replicated per rank (scalars only)
    ang = F.rope_angles(F.position_ids(L_t, height, width), cfg.axes_dim, cfg.theta)
    ang_t = shard(ang[:L_t], k)
    ang_i = shard(ang[L_t:], k)
    img = [F.linear(p, W["img_in.w"], W["img_in.b"]) for p in shard(x_lat, k)]
    txt = [F.linear(p, W["txt_in.w"], W["txt_in.b"]) for p in shard(T, k)]

    def attn_sp(qkv_t, qkv_i, gq, gk):
        # per rank: RMSNorm + RoPE on own rows (global positions, S5), then a2a #1.
        q_t, k_t, v_t, q_i, k_i, v_i = [], [], [], [], [], []
        for r in range(k):
            for (qkv, ang_r, gqs, gks, qs, ks, vs) in ((qkv_t[r], ang_t[r], gq[0], gk[0], q_t, k_t, v_t),
                                                        (qkv_i[r], ang_i[r], gq[1], gk[1], q_i, k_i, v_i)):
                q, kk, v = F.split_qkv(qkv, H, D)
                qs.append(F.apply_rope(F.rms_norm(q, gqs), ang_r))
                ks.append(F.apply_rope(F.rms_norm(kk, gks), ang_r))
                vs.append(v)
        Q = _a2a_seq_to_head(q_t, q_i, k, H)
        K = _a2a_seq_to_head(k_t, k_i, k, H)
        V = _a2a_seq_to_head(v_t, v_i, k, H)
        O = [F.attention(Q[d], K[d], V[d]) for d in range(k)]
        return _a2a_head_to_seq(O, k, H, D, L_t, L_i)                      # a2a #2

    for j in range(cfg.n_double):
        mods = {sn: F.modulation(W, f"double{j}.{sn}.", vec, 6) for sn in ("img", "txt")}
        qkv = {}
        for sn, xs in (("img", img), ("txt", txt)):
            p = f"double{j}.{sn}."
            sh1, sc1 = mods[sn][0], mods[sn][1]
            qkv[sn] = [F.linear(F.ln_modulate(x, sh1, sc1), W[p + "qkv.w"], W[p + "qkv.b"]) for x in xs]
        pt, pi = f"double{j}.txt.", f"double{j}.img."
        o_t, o_i = attn_sp(qkv["txt"], qkv["img"], (W[pt + "q_norm.g"], W[pi + "q_norm.g"]),
                           (W[pt + "k_norm.g"], W[pi + "k_norm.g"]))
        for sn, xs, os_ in (("img", img, o_i), ("txt", txt, o_t)):
            p = f"double{j}.{sn}."
            _, _, g1, sh2, sc2, g2 = mods[sn]
            for r in range(k):
                x = xs[r] + g1 * F.linear(os_[r], W[p + "proj.w"], W[p + "proj.b"])
                hdn = F.gelu_tanh(F.linear(F.ln_modulate(x, sh2, sc2), W[p + "fc1.w"], W[p + "fc1.b"]))
                xs[r] = x + g2 * F.linear(hdn, W[p + "fc2.w"], W[p + "fc2.b"])
        W.drop(f"double{j}.")
    # single blocks: each rank keeps [txt_r; img_r] (a10, zero-copy on the GPU)
    for j in range(cfg.n_single):
        p = f"single{j}."
        sh, sc, g = F.modulation(W, p, vec, 3)
        q_t, q_i, mlp_t, mlp_i = [], [], [], []
        for r in range(k):
            for x, qs, ms in ((txt[r], q_t, mlp_t), (img[r], q_i, mlp_i)):
                y1 = F.linear(F.ln_modulate(x, sh, sc), W[p + "lin1.w"], W[p + "lin1.b"])
                qs.append(y1[:, :3 * h])
                ms.append(y1[:, 3 * h:])
        g_q, g_k = W[p + "q_norm.g"], W[p + "k_norm.g"]
        o_t, o_i = attn_sp(q_t, q_i, (g_q, g_q), (g_k, g_k))
        for r in range(k):
            for xs, os_, ms in ((txt, o_t, mlp_t), (img, o_i, mlp_i)):
                out = F.linear(np.concatenate([os_[r], F.gelu_tanh(ms[r])], axis=1), W[p + "lin2.w"], W[p + "lin2.b"])
                xs[r] = xs[r] + g * out
        W.drop(p)
    v = [F.final_layer(W, img[r], vec) for r in range(k)]
    xs = shard(x_lat, k)
    return gather(v), gather([xs[r] + (t_next - t) * v[r] for r in range(k)])


def sd3_step_sp(cfg: ModelCfg, W: Weights, x_lat, T_c, y_c, T_u, y_u, t: float, t_next: float,
                height: int, width: int, k: int):
    """sd3.sd3_step computed by k simulated Ulysses ranks (both CFG branches).  Rows after
    the first all-to-all follow diffusers' joint order [img_0..img_{k-1}; txt_0..txt_{k-1}]."""
    from . import sd3 as S3
    H, D = cfg.heads, cfg.head_dim
    if H % k:
        raise ValueError("k must divide the head count (S24)")
    L_i = x_lat.shape[0]
    pe = shard(S3.pos_embed(cfg, height // 16, width // 16), k)

    def branch(T, y):
        L_t = T.shape[0]
        vec = S3.conditioning_vec(cfg, W, t, y)
        img = [F.linear(p, W["img_in.w"], W["img_in.b"]) + pe[r] for r, p in enumerate(shard(x_lat, k))]
        txt = [F.linear(p, W["txt_in.w"], W["txt_in.b"]) for p in shard(T, k)]
        for j in range(cfg.n_double):
            last = j == cfg.n_double - 1
            pi, pt = f"joint{j}.img.", f"joint{j}.txt."
            mi = F.modulation(W, pi, vec, 6)
            mt = F.modulation(W, pt, vec, 2 if last else 6)
            t_sh, t_sc = (mt[1], mt[0]) if last else (mt[0], mt[1])
            qi = [F.split_qkv(F.linear(F.ln_modulate(x, mi[0], mi[1]), W[pi + "qkv.w"], W[pi + "qkv.b"]), H, D)
                  for x in img]
            qt = [F.split_qkv(F.linear(F.ln_modulate(x, t_sh, t_sc), W[pt + "qkv.w"], W[pt + "qkv.b"]), H, D)
                  for x in txt]
            Q, K, V = (_a2a_seq_to_head([a[c] for a in qi], [a[c] for a in qt], k, H) for c in range(3))
            O = [F.attention(Q[d], K[d], V[d]) for d in range(k)]
            o_i, o_t = _a2a_head_to_seq(O, k, H, D, L_i, L_t)      # (first stream, second stream)
            for r in range(k):
                x = img[r] + mi[2] * F.linear(o_i[r], W[pi + "proj.w"], W[pi + "proj.b"])
                hdn = F.gelu_tanh(F.linear(F.ln_modulate(x, mi[3], mi[4]), W[pi + "fc1.w"], W[pi + "fc1.b"]))
                img[r] = x + mi[5] * F.linear(hdn, W[pi + "fc2.w"], W[pi + "fc2.b"])
                if not last:
                    x = txt[r] + mt[2] * F.linear(o_t[r], W[pt + "proj.w"], W[pt + "proj.b"])
                    hdn = F.gelu_tanh(F.linear(F.ln_modulate(x, mt[3], mt[4]), W[pt + "fc1.w"], W[pt + "fc1.b"]))
                    txt[r] = x + mt[5] * F.linear(hdn, W[pt + "fc2.w"], W[pt + "fc2.b"])
        return [S3.final_layer(W, img[r], vec) for r in range(k)]

    v_u = branch(T_u, y_u)
    v_c = branch(T_c, y_c)
    v = [v_u[r] + cfg.cfg_scale * (v_c[r] - v_u[r]) for r in range(k)]
    xs = shard(x_lat, k)
    return gather(v), gather([xs[r] + (t_next - t) * v[r] for r in range(k)])
