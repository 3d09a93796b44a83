"""Pins of the SD3-medium oracle (oracle/sd3.py; config 5) against things other than itself:
MAE's library sin-cos table, translation invariance of the embedding's inner product, the
torchtitan FLUX double block (the MMDiT joint block with QK-norm and RoPE switched off), the
AdaLayerNormContinuous chunk order, adaLN-Zero, CFG special cases, the FLUX time-shift form
of the schedule, and simulated SP invariance with an uneven (77-token) text stream."""
import math

import numpy as np
import pytest

from oracle import flux as F
from oracle import sd3 as S3
from oracle import sp as SP
from oracle.config import SD3, TINY_SD3, ModelCfg, tensor_table
from oracle.weights import Weights, sd3_request_inputs

torch = pytest.importorskip("torch")


# ----------------------------------------------------------------------------- position embedding
def test_sincos_matches_mae_library():
    from transformers.models.vit_mae import modeling_vit_mae as mae
    h = 64
    ref = mae.get_2d_sincos_pos_embed(h, 12)
    grid = np.arange(12)
    got = S3.sincos_2d(h, np.repeat(grid, 12), np.tile(grid, 12))
    assert np.allclose(got, ref, rtol=0, atol=1e-6)          # MAE builds its grid in float32
    # the 1-D encoder on fractional positions equals MAE's (which takes arbitrary positions)
    pos = np.arange(192) / 3.0
    assert np.allclose(S3.sincos_1d(768, pos), mae.get_1d_sincos_pos_embed_from_grid(768, pos), rtol=0, atol=1e-12)


def test_pos_embed_crop_and_scale():
    cfg = SD3
    full = S3.pos_embed(cfg, 192, 192).reshape(192, 192, cfg.hidden)
    assert np.allclose(full[0, 0], np.r_[np.zeros(384), np.ones(384), np.zeros(384), np.ones(384)])
    for n_r, n_c in ((32, 32), (64, 128), (33, 17)):
        top, left = (192 - n_r) // 2, (192 - n_c) // 2
        got = S3.pos_embed(cfg, n_r, n_c)
        assert np.array_equal(got, full[top:top + n_r, left:left + n_c].reshape(-1, cfg.hidden))
    # <PE(p), PE(p')> = sum_j cos(w_j dc / 3) + cos(w_j dr / 3): the grid spacing is 1/3
    pe = S3.pos_embed(cfg, 64, 64)
    w = 1.0 / 10000.0 ** (np.arange(384) / 384)
    rng = np.random.default_rng(0)
    for _ in range(20):
        a, b = rng.integers(0, 4096, 2)
        dr, dc = a // 64 - b // 64, a % 64 - b % 64
        assert math.isclose(pe[a] @ pe[b], np.cos(w * dc / 3).sum() + np.cos(w * dr / 3).sum(), rel_tol=1e-10)
    # 4096^2: 256 > 192 patches, the analytic extension (S13): centred, symmetric offsets
    big = S3.pos_embed(cfg, 256, 256).reshape(256, 256, cfg.hidden)
    assert np.allclose(big[32, 32], full[0, 0])          # top = floor(-64/2) = -32


# ----------------------------------------------------------------------------- blocks vs library
def _load(t, a):
    t.data.copy_(torch.from_numpy(np.ascontiguousarray(a)))


class _NoQKNorm(torch.nn.Module):
    def forward(self, q, k, v):
        return q, k


def _tt_joint(tt_layers, cfg, W, j, txt_mod=None):
    """The MMDiT joint block as torchtitan's FLUX DoubleStreamBlock with QK-norm replaced by
    the identity and zero RoPE angles."""
    blk = tt_layers.DoubleStreamBlock(cfg.hidden, cfg.heads, cfg.mlp_hidden / cfg.hidden, qkv_bias=True).double()
    for sn in ("img", "txt"):
        p = f"joint{j}.{sn}."
        mod = getattr(blk, f"{sn}_mod").lin
        if sn == "txt" and txt_mod is not None:
            _load(mod.weight, txt_mod[0]); _load(mod.bias, txt_mod[1])
        else:
            _load(mod.weight, W[p + "mod.w"]); _load(mod.bias, W[p + "mod.b"])
        at = getattr(blk, f"{sn}_attn")
        _load(at.qkv.weight, W[p + "qkv.w"]); _load(at.qkv.bias, W[p + "qkv.b"])
        at.norm = _NoQKNorm()
        if txt_mod is None or sn == "img":
            _load(at.proj.weight, W[p + "proj.w"]); _load(at.proj.bias, W[p + "proj.b"])
            mlp = getattr(blk, f"{sn}_mlp")
            _load(mlp[0].weight, W[p + "fc1.w"]); _load(mlp[0].bias, W[p + "fc1.b"])
            _load(mlp[2].weight, W[p + "fc2.w"]); _load(mlp[2].bias, W[p + "fc2.b"])
    return blk


def test_joint_blocks_and_final_vs_torchtitan(tt_layers):
    cfg = TINY_SD3
    W = Weights(cfg)
    rng = np.random.default_rng(1)
    L_t, L_i = 7, 24
    img = rng.standard_normal((L_i, cfg.hidden))
    txt = rng.standard_normal((L_t, cfg.hidden))
    vec = rng.standard_normal(cfg.hidden)
    ids = np.zeros((L_t + L_i, 3))
    pe = tt_layers.EmbedND(cfg.head_dim, 10000, [8, 28, 28])(torch.from_numpy(ids)[None])  # zero angles
    tv = torch.from_numpy(vec)[None]
    ti, tt = torch.from_numpy(img)[None], torch.from_numpy(txt)[None]

    # block 0: a full joint block (torchtitan concatenates [txt; img], diffusers [img; txt])
    with torch.no_grad():
        ri, rt = _tt_joint(tt_layers, cfg, W, 0)(img=ti, txt=tt, vec=tv, pe=pe)
    oi, ot = S3.joint_block(cfg, W, 0, img, txt, vec)
    # the library applies even a zero rotation in float32 (TT:math.py:30-38): ~1e-7 relative
    assert np.allclose(oi, ri[0].numpy(), rtol=1e-6, atol=1e-6)
    assert np.allclose(ot, rt[0].numpy(), rtol=1e-6, atol=1e-6)

    # block 1 (last): context_pre_only; txt AdaLayerNormContinuous rows are (scale, shift) ->
    # the library block's 6-chunk (shift1, scale1, ...) with the other chunks zero
    h = cfg.hidden
    w2, b2 = W["joint1.txt.mod.w"], W["joint1.txt.mod.b"]
    w6, b6 = np.zeros((6 * h, h)), np.zeros(6 * h)
    w6[:h], w6[h:2 * h] = w2[h:], w2[:h]
    b6[:h], b6[h:2 * h] = b2[h:], b2[:h]
    with torch.no_grad():
        ri, _ = _tt_joint(tt_layers, cfg, W, 1, txt_mod=(w6, b6))(img=ti, txt=tt, vec=tv, pe=pe)
    oi, ot = S3.joint_block(cfg, W, 1, img, txt, vec)
    assert ot is None
    assert np.allclose(oi, ri[0].numpy(), rtol=1e-6, atol=1e-6)

    # final layer: (scale, shift) = the library LastLayer's (shift, scale) with halves swapped
    ll = tt_layers.LastLayer(cfg.hidden, 1, cfg.in_ch).double()
    fw, fb = W["final.mod.w"], W["final.mod.b"]
    _load(ll.adaLN_modulation[1].weight, np.concatenate([fw[h:], fw[:h]]))
    _load(ll.adaLN_modulation[1].bias, np.concatenate([fb[h:], fb[:h]]))
    _load(ll.linear.weight, W["final.lin.w"]); _load(ll.linear.bias, W["final.lin.b"])
    with torch.no_grad():
        rf = ll(ti, tv)
    assert np.allclose(S3.final_layer(W, img, vec), rf[0].numpy(), rtol=1e-10, atol=1e-10)


def test_conditioning_vec_vs_torchtitan(tt_layers):
    cfg = TINY_SD3
    W = Weights(cfg)
    _, _, y, _, _ = sd3_request_inputs(cfg, 64, 64, 7)
    ref = 0
    for name, z in (("time_in", F.timestep_embedding(0.6)), ("vector_in", y)):
        m = tt_layers.MLPEmbedder(z.shape[0], cfg.hidden).double()
        _load(m.in_layer.weight, W[name + ".in.w"]); _load(m.in_layer.bias, W[name + ".in.b"])
        _load(m.out_layer.weight, W[name + ".out.w"]); _load(m.out_layer.bias, W[name + ".out.b"])
        with torch.no_grad():
            ref = ref + m(torch.from_numpy(z)[None])[0].numpy()
    assert np.allclose(S3.conditioning_vec(cfg, W, 0.6, y), ref, rtol=1e-11, atol=1e-12)


# ----------------------------------------------------------------------------- schedule, CFG, adaLN-Zero
def test_schedule_is_flux_time_shift_with_mu_ln3():
    ts = S3.schedule(SD3, 20)
    assert ts[0] == 1.0 and ts[-1] == 0.0 and np.all(np.diff(ts) < 0)
    assert np.allclose(ts, F.time_shift(math.log(3.0), np.linspace(1, 0, 21)), rtol=1e-14, atol=0)


def test_cfg_special_cases():
    cfg = TINY_SD3
    W = Weights(cfg)
    x, Tc, yc, Tu, yu = sd3_request_inputs(cfg, 64, 48, 11)
    v_c = S3.forward(cfg, W, x, Tc, yc, 0.7, 64, 48)
    # equal branches: the guidance term vanishes
    v, xn = S3.sd3_step(cfg, W, x, Tc, yc, Tc, yc, 0.7, 0.6, 64, 48)
    assert np.allclose(v, v_c, rtol=1e-12, atol=1e-12)
    # scale 1: the conditional branch alone
    c1 = ModelCfg(**{**cfg.__dict__, "cfg_scale": 1.0})
    v1, _ = S3.sd3_step(c1, W, x, Tc, yc, Tu, yu, 0.7, 0.6, 64, 48)
    assert np.allclose(v1, v_c, rtol=1e-12, atol=1e-12)
    # scale 0: the unconditional branch alone
    c0 = ModelCfg(**{**cfg.__dict__, "cfg_scale": 0.0})
    v0, _ = S3.sd3_step(c0, W, x, Tc, yc, Tu, yu, 0.7, 0.6, 64, 48)
    assert np.allclose(v0, S3.forward(cfg, W, x, Tu, yu, 0.7, 64, 48), rtol=1e-12, atol=1e-12)


def test_adaln_zero_closed_form():
    cfg = TINY_SD3
    W = Weights(cfg)
    zero = {name: np.zeros(shape) for _, name, shape, _, _ in tensor_table(cfg) if "mod." in name}
    Wz = Weights(cfg, overrides=zero)
    x, Tc, yc, Tu, yu = sd3_request_inputs(cfg, 64, 64, 12)
    v, xn = S3.sd3_step(cfg, Wz, x, Tc, yc, Tu, yu, 0.7, 0.6, 64, 64)
    img = x @ W["img_in.w"].T + W["img_in.b"] + S3.pos_embed(cfg, 4, 4)
    v_ref = F.layer_norm(img) @ W["final.lin.w"].T + W["final.lin.b"]   # both branches equal
    assert np.allclose(v, v_ref, rtol=1e-12, atol=1e-12)
    assert np.allclose(xn, x - 0.1 * v_ref, rtol=1e-12, atol=1e-12)


def test_tensor_table_shapes():
    t = {name: shape for _, name, shape, _, _ in tensor_table(SD3)}
    ids = [tid for tid, *_ in tensor_table(SD3)]
    assert len(ids) == len(set(ids))
    assert t["img_in.w"] == (1536, 64) and t["vector_in.in.w"] == (1536, 2048)
    assert t["joint23.txt.mod.w"] == (3072, 1536) and "joint23.txt.proj.w" not in t
    assert t["joint22.txt.fc1.w"] == (6144, 1536)
    n = sum(int(np.prod(s)) for s in t.values())
    assert 2.0e9 < n < 2.1e9    # SD3-medium's ~2B transformer parameters (minus pos-embed table)


@pytest.mark.parametrize("k", [2, 4])
def test_sp_invariance(k):
    cfg = TINY_SD3     # 77 text tokens: uneven shards (k = 4 -> 20, 19, 19, 19)
    W = Weights(cfg)
    x, Tc, yc, Tu, yu = sd3_request_inputs(cfg, 80, 96, 13)
    v1, x1 = S3.sd3_step(cfg, W, x, Tc, yc, Tu, yu, 0.8, 0.7, 80, 96)
    vk, xk = SP.sd3_step_sp(cfg, W, x, Tc, yc, Tu, yu, 0.8, 0.7, 80, 96, k)
    assert np.max(np.abs(vk - v1)) <= 1e-12 * np.max(np.abs(v1))
    assert np.max(np.abs(xk - x1)) <= 1e-12 * np.max(np.abs(x1))
