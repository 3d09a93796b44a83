"""Pins for the oracle (CPU only): closed forms, special cases, brute force, library routines,
and an independent implementation of the public FLUX blocks (torchtitan's mirror of BFL code).

Each test names the plausible oracle mistake it would catch.
"""
import math

import numpy as np
import pytest

import synth
from oracle import flux as F
from oracle import sp as SP
from oracle.config import FLUX, TINY, TINY2, ModelCfg, image_tokens
from oracle.weights import Weights, request_inputs

torch = pytest.importorskip("torch")


# ----------------------------------------------------------------------------- SYNTH-1
def test_splitmix64_reference_vectors():
    # splitmix64 seeded with 0 yields these first three outputs (Steele et al. 2014 reference
    # sequence); our counter hash at key = j*gamma reproduces output j+1.
    G = int(synth.GOLDEN_GAMMA)
    idx = np.array([0, G, (2 * G) & (2 ** 64 - 1)], dtype=np.uint64)
    got = [int(v) for v in synth.hash_u64(0, 0, idx)]
    assert got == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]


def test_bf16_rounding_matches_torch():
    rng = np.random.default_rng(0)
    x = (rng.standard_normal(100000) * 10 ** rng.uniform(-5, 5, 100000)).astype(np.float32)
    x = np.concatenate([x, np.float32([1.0, 1 + 2 ** -8, 1 + 3 * 2 ** -8, -1 - 2 ** -8])])
    ours = synth.bf16_rne_bits(x)
    ref = torch.from_numpy(x).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(ours, ref)
    assert list(ours[-4:]) == [0x3F80, 0x3F80, 0x3F82, 0xBF80]  # ties to even


def test_uniform_range_and_moments():
    r = synth.uniform_pm1(7, 3, np.arange(1 << 20, dtype=np.uint64))
    assert r.min() >= -1.0 and r.max() < 1.0
    assert abs(r.mean()) < 3e-3 and abs(r.var() - 1 / 3) < 3e-3
    w = synth.gen_tensor(7, 3, (1024, 1024), "w", 1024)
    assert abs(w.std() - 1 / 32) < 2e-4


# ----------------------------------------------------------------------------- shapes (P1)
@pytest.mark.parametrize("res,tokens", [(256, 256), (512, 1024), (1024, 4096), (2048, 16384)])
def test_token_counts_table1(res, tokens):
    # Table 1 and L_i = H*W/16^2
    assert image_tokens(res, res) == tokens


def test_bad_resolution():
    with pytest.raises(ValueError):
        image_tokens(500, 512)


# ----------------------------------------------------------------------------- schedule (P8)
def test_schedule_closed_form():
    assert F.schedule_mu(256) == pytest.approx(0.5)
    assert F.schedule_mu(4096) == pytest.approx(1.15)
    ts = F.schedule(20, 1024)
    assert ts[0] == 1.0 and ts[-1] == 0.0 and np.all(np.diff(ts) < 0)
    # mu = 0 -> identity time shift
    assert F.time_shift(0.0, np.array([0.25, 0.5, 0.75])) == pytest.approx([0.25, 0.5, 0.75])
    # shifted schedule at L_i = 4096, t = 0.5: e^1.15 / (e^1.15 + 1)
    assert F.time_shift(1.15, np.array([0.5]))[0] == pytest.approx(math.exp(1.15) / (math.exp(1.15) + 1))


# ----------------------------------------------------------------------------- elementwise (P5, P6)
def test_timestep_embedding(tt_layers):
    e0 = F.timestep_embedding(0.0)
    assert np.array_equal(e0, np.concatenate([np.ones(128), np.zeros(128)]))
    for t in (0.0, 0.37, 1.0, 3.5):
        ref = tt_layers.timestep_embedding(torch.tensor([t], dtype=torch.float64), 256)[0]
        # TT builds freqs in float32 (TT:layers.py:47); agree to float32 argument rounding
        assert np.allclose(F.timestep_embedding(t), ref.numpy(), atol=5e-4)


def test_gelu_silu_library():
    x = np.linspace(-8, 8, 1001)
    xt = torch.from_numpy(x)
    assert np.allclose(F.gelu_tanh(x), torch.nn.functional.gelu(xt, approximate="tanh").numpy(), rtol=1e-13, atol=1e-15)
    assert np.allclose(F.silu(x), torch.nn.functional.silu(xt).numpy(), rtol=1e-13, atol=1e-15)
    assert F.gelu_tanh(np.array([0.0]))[0] == 0.0


def test_layernorm_library_and_invariants():
    rng = np.random.default_rng(1)
    x = rng.standard_normal((7, 96)) * 3 + 1
    ref = torch.nn.functional.layer_norm(torch.from_numpy(x), (96,), eps=1e-6).numpy()
    assert np.allclose(F.layer_norm(x), ref, rtol=1e-12, atol=1e-12)
    assert np.allclose(F.layer_norm(x + 5.0), F.layer_norm(x), atol=1e-12)   # shift invariance
    c = np.full((1, 96), 2.5)
    sh, sc = rng.standard_normal(96), rng.standard_normal(96)
    assert np.allclose(F.ln_modulate(c, sh, sc), sh)                        # constant row -> shift


def test_rmsnorm_closed_form():
    g = np.linspace(0.5, 1.5, 64)
    for c in (-3.0, 0.01, 7.0):
        got = F.rms_norm(np.full((1, 64), c), g)[0]
        assert np.allclose(got, np.sign(c) * g * abs(c) / math.sqrt(c * c + 1e-6), rtol=1e-14)


# ----------------------------------------------------------------------------- RoPE (P4)
def test_rope_properties_and_library(tt_layers):
    from torchtitan.experiments.flux.model.math import apply_rope as tt_apply_rope
    rng = np.random.default_rng(2)
    ids = F.position_ids(3, 64, 80)                     # 3 text + 4x5 image tokens
    assert ids.shape == (23, 3) and np.all(ids[:3] == 0)
    assert list(ids[3 + 7]) == [0, 1, 2]                # token 7 = row 1, col 2 of a 5-wide grid
    ang = F.rope_angles(ids, (16, 56, 56), 10000.0)
    x = rng.standard_normal((23, 2, 128))
    y = F.apply_rope(x, ang)
    # norm of each pair preserved; text (position 0) unchanged
    assert np.allclose(x[..., 0::2] ** 2 + x[..., 1::2] ** 2, y[..., 0::2] ** 2 + y[..., 1::2] ** 2)
    assert np.allclose(y[:3], x[:3])
    # library: TT's EmbedND + apply_rope on [B, H, L, D]
    emb = tt_layers.EmbedND(128, 10000, [16, 56, 56])(torch.from_numpy(ids)[None])
    xt = torch.from_numpy(x).permute(1, 0, 2)[None]
    ref, _ = tt_apply_rope(xt, xt, emb)
    assert np.allclose(y, ref[0].permute(1, 0, 2).numpy(), rtol=1e-6, atol=1e-6)


def test_rope_relative_property():
    rng = np.random.default_rng(3)
    q, k = rng.standard_normal((1, 1, 64)), rng.standard_normal((1, 1, 64))
    axes = (8, 28, 28)
    pm, pn = np.array([[0, 3.0, 5.0]]), np.array([[0, 7.0, 2.0]])
    lhs = np.sum(F.apply_rope(q, F.rope_angles(pm, axes, 1e4)) * F.apply_rope(k, F.rope_angles(pn, axes, 1e4)))
    rhs = np.sum(q * F.apply_rope(k, F.rope_angles(pn - pm, axes, 1e4)))
    assert lhs == pytest.approx(rhs, rel=1e-12)


# ----------------------------------------------------------------------------- attention (P3)
def _attention_bruteforce(q, k, v):
    L, H, D = q.shape
    out = np.zeros_like(q)
    for h in range(H):
        for i in range(L):
            s = [sum(q[i, h, d] * k[j, h, d] for d in range(D)) / math.sqrt(D) for j in range(L)]
            m = max(s)
            e = [math.exp(x - m) for x in s]
            z = sum(e)
            for d in range(D):
                out[i, h, d] = sum(e[j] * v[j, h, d] for j in range(L)) / z
    return out


def test_attention_bruteforce_and_special_cases():
    rng = np.random.default_rng(4)
    q, k, v = (rng.standard_normal((6, 2, 4)) for _ in range(3))
    assert np.allclose(F.attention(q, k, v, q_chunk=4), _attention_bruteforce(q, k, v), rtol=1e-12)
    # L = 1 -> V
    assert np.allclose(F.attention(q[:1], k[:1], v[:1]), v[:1])
    # identical keys -> mean(V)
    kk = np.repeat(k[:1], 6, axis=0)
    assert np.allclose(F.attention(q, kk, v), np.repeat(v.mean(axis=0, keepdims=True), 6, axis=0))
    # a dominant key -> its V row
    kd = k.copy()
    kd[2] = 1e3 * q[0]
    assert np.allclose(F.attention(q[:1], kd, v)[0], v[2])
    # permutation of KV rows leaves the output unchanged
    p = rng.permutation(6)
    assert np.allclose(F.attention(q, k[p], v[p]), F.attention(q, k, v), rtol=1e-12)


def test_attention_sdpa_library():
    rng = np.random.default_rng(5)
    q, k, v = (rng.standard_normal((300, 3, 64)) for _ in range(3))
    t = [torch.from_numpy(a).permute(1, 0, 2)[None] for a in (q, k, v)]
    ref = torch.nn.functional.scaled_dot_product_attention(*t)[0].permute(1, 0, 2).numpy()
    assert np.allclose(F.attention(q, k, v, q_chunk=128), ref, rtol=1e-10, atol=1e-12)


# ----------------------------------------------------------------------------- blocks vs library
def _load(mod, W, name):
    mod.data.copy_(torch.from_numpy(W[name]))


def _tt_double(tt_layers, cfg, W, j):
    blk = tt_layers.DoubleStreamBlock(cfg.hidden, cfg.heads, cfg.mlp_hidden / cfg.hidden, qkv_bias=True).double()
    for sn in ("img", "txt"):
        p = f"double{j}.{sn}."
        _load(getattr(blk, f"{sn}_mod").lin.weight, W, p + "mod.w")
        _load(getattr(blk, f"{sn}_mod").lin.bias, W, p + "mod.b")
        at = getattr(blk, f"{sn}_attn")
        _load(at.qkv.weight, W, p + "qkv.w"); _load(at.qkv.bias, W, p + "qkv.b")
        _load(at.proj.weight, W, p + "proj.w"); _load(at.proj.bias, W, p + "proj.b")
        _load(at.norm.query_norm.weight, W, p + "q_norm.g"); _load(at.norm.key_norm.weight, W, p + "k_norm.g")
        at.norm.query_norm.eps = 1e-6
        at.norm.key_norm.eps = 1e-6   # BFL eps (S6); TT leaves nn.RMSNorm's default
        mlp = getattr(blk, f"{sn}_mlp")
        _load(mlp[0].weight, W, p + "fc1.w"); _load(mlp[0].bias, W, p + "fc1.b")
        _load(mlp[2].weight, W, p + "fc2.w"); _load(mlp[2].bias, W, p + "fc2.b")
    return blk


def test_double_single_final_vs_torchtitan(tt_layers):
    cfg = TINY2
    W = Weights(cfg)
    rng = np.random.default_rng(6)
    L_t, hgt, wid = 5, 48, 64
    L_i = image_tokens(hgt, wid)
    img = rng.standard_normal((L_i, cfg.hidden))
    txt = rng.standard_normal((L_t, cfg.hidden))
    vec = rng.standard_normal(cfg.hidden)
    ids = F.position_ids(L_t, hgt, wid)
    ang = F.rope_angles(ids, cfg.axes_dim, cfg.theta)
    pe = tt_layers.EmbedND(cfg.head_dim, int(cfg.theta), list(cfg.axes_dim))(torch.from_numpy(ids)[None])
    tv = torch.from_numpy(vec)[None]

    # double block
    blk = _tt_double(tt_layers, cfg, W, 0)
    with torch.no_grad():
        ri, rt = blk(img=torch.from_numpy(img)[None], txt=torch.from_numpy(txt)[None], vec=tv, pe=pe)
    oi, ot = F.double_block(cfg, W, 0, img, txt, vec, ang)
    # TT casts the RoPE table to float32 (TT:math.py:30): agree to ~1e-7 relative
    assert np.allclose(oi, ri[0].numpy(), rtol=1e-6, atol=1e-6)
    assert np.allclose(ot, rt[0].numpy(), rtol=1e-6, atol=1e-6)

    # single block
    sb = tt_layers.SingleStreamBlock(cfg.hidden, cfg.heads, cfg.mlp_hidden / cfg.hidden).double()
    p = "single0."
    _load(sb.modulation.lin.weight, W, p + "mod.w"); _load(sb.modulation.lin.bias, W, p + "mod.b")
    _load(sb.linear1.weight, W, p + "lin1.w"); _load(sb.linear1.bias, W, p + "lin1.b")
    _load(sb.linear2.weight, W, p + "lin2.w"); _load(sb.linear2.bias, W, p + "lin2.b")
    _load(sb.norm.query_norm.weight, W, p + "q_norm.g"); _load(sb.norm.key_norm.weight, W, p + "k_norm.g")
    sb.norm.query_norm.eps = 1e-6
    sb.norm.key_norm.eps = 1e-6
    x = np.concatenate([txt, img])
    with torch.no_grad():
        rs = sb(torch.from_numpy(x)[None], vec=tv, pe=pe)
    assert np.allclose(F.single_block(cfg, W, 0, x, vec, ang), rs[0].numpy(), rtol=1e-6, atol=1e-6)

    # final layer
    ll = tt_layers.LastLayer(cfg.hidden, 1, cfg.in_ch).double()
    _load(ll.adaLN_modulation[1].weight, W, "final.mod.w"); _load(ll.adaLN_modulation[1].bias, W, "final.mod.b")
    _load(ll.linear.weight, W, "final.lin.w"); _load(ll.linear.bias, W, "final.lin.b")
    with torch.no_grad():
        rf = ll(torch.from_numpy(img)[None], tv)
    assert np.allclose(F.final_layer(W, img, vec), rf[0].numpy(), rtol=1e-10, atol=1e-10)


def test_flux_step_vs_torchtitan_model(tt_layers):
    """The whole oracle step (a0 conditioning, a1 img_in AND txt_in embeddings, the [txt; img] join
    and split, every block, the final layer, a12 Euler) against torchtitan's independent FluxModel
    forward with the same weights -- the pin of the txt_in leg, which the block-level pins (random
    txt) and adaLN-Zero (txt irrelevant) leave open.  FluxModel has no guidance embedder (S:§8(c)
    "Where TT differs" i), so guidance_in is zeroed on the oracle side: MLP_g(e(g)) = 0."""
    model_mod = pytest.importorskip("torchtitan.experiments.flux.model.model")
    args_mod = pytest.importorskip("torchtitan.experiments.flux.model.args")
    cfg = TINY2
    zero = {n: np.zeros_like(Weights(cfg)[n]) for n in ("guidance_in.in.w", "guidance_in.in.b",
                                                        "guidance_in.out.w", "guidance_in.out.b")}
    W = Weights(cfg, overrides=zero)
    hgt, wid, steps, step = 48, 64, 20, 3
    x, T, y = request_inputs(cfg, hgt, wid, 1234)
    v_o, xn_o = F.request_step(cfg, W, x, T, y, step, steps, 3.5, hgt, wid, drop_weights=False)

    a = args_mod.FluxModelArgs(in_channels=cfg.in_ch, out_channels=cfg.in_ch, vec_in_dim=cfg.vec_dim,
                               context_in_dim=cfg.ctx_dim, hidden_size=cfg.hidden,
                               mlp_ratio=cfg.mlp_hidden / cfg.hidden, num_heads=cfg.heads, depth=cfg.n_double,
                               depth_single_blocks=cfg.n_single, axes_dim=tuple(cfg.axes_dim), theta=int(cfg.theta),
                               qkv_bias=True)
    m = model_mod.FluxModel(a).double()
    _load(m.img_in.weight, W, "img_in.w"); _load(m.img_in.bias, W, "img_in.b")
    _load(m.txt_in.weight, W, "txt_in.w"); _load(m.txt_in.bias, W, "txt_in.b")
    for nme, mod in (("time_in", m.time_in), ("vector_in", m.vector_in)):
        _load(mod.in_layer.weight, W, nme + ".in.w"); _load(mod.in_layer.bias, W, nme + ".in.b")
        _load(mod.out_layer.weight, W, nme + ".out.w"); _load(mod.out_layer.bias, W, nme + ".out.b")
    for j in range(cfg.n_double):
        m.double_blocks[j] = _tt_double(tt_layers, cfg, W, j)
    for j, sb in enumerate(m.single_blocks):
        p = f"single{j}."
        _load(sb.modulation.lin.weight, W, p + "mod.w"); _load(sb.modulation.lin.bias, W, p + "mod.b")
        _load(sb.linear1.weight, W, p + "lin1.w"); _load(sb.linear1.bias, W, p + "lin1.b")
        _load(sb.linear2.weight, W, p + "lin2.w"); _load(sb.linear2.bias, W, p + "lin2.b")
        _load(sb.norm.query_norm.weight, W, p + "q_norm.g"); _load(sb.norm.key_norm.weight, W, p + "k_norm.g")
        sb.norm.query_norm.eps = 1e-6
        sb.norm.key_norm.eps = 1e-6
    ll = m.final_layer
    _load(ll.adaLN_modulation[1].weight, W, "final.mod.w"); _load(ll.adaLN_modulation[1].bias, W, "final.mod.b")
    _load(ll.linear.weight, W, "final.lin.w"); _load(ll.linear.bias, W, "final.lin.b")
    ids = F.position_ids(T.shape[0], hgt, wid)
    ts = F.schedule(steps, x.shape[0])
    with torch.no_grad():
        v_t = m(img=torch.from_numpy(x)[None], img_ids=torch.from_numpy(ids[T.shape[0]:])[None],
                txt=torch.from_numpy(T)[None], txt_ids=torch.from_numpy(ids[:T.shape[0]])[None],
                timesteps=torch.tensor([ts[step]], dtype=torch.float64), y=torch.from_numpy(y)[None])[0].numpy()
    # TT rotates q, k in float32 (its RoPE table and apply_rope cast to float, TT:math.py:30-36):
    # ~1e-7 per rotation, 1e-5 normwise after 2 + 2 blocks; every other op is float64 on both sides
    vmax = np.abs(v_t).max()
    assert np.max(np.abs(v_o - v_t)) <= 5e-5 * vmax
    assert np.max(np.abs(xn_o - (x + (ts[step + 1] - ts[step]) * v_t))) <= 5e-5 * vmax
    # the pin sees the text embedding: a dropped txt_in bias, or a perturbed txt_in weight, moves v far
    # outside that bound (perturbations must vary across channels: LayerNorm ignores a constant shift)
    rng = np.random.default_rng(3)
    for nme, new in (("txt_in.b", np.zeros_like(W["txt_in.b"])),
                     ("txt_in.w", W["txt_in.w"] + 0.01 * rng.standard_normal(W["txt_in.w"].shape))):
        W2 = Weights(cfg, overrides=dict(zero, **{nme: new}))
        v_2, _ = F.request_step(cfg, W2, x, T, y, step, steps, 3.5, hgt, wid, drop_weights=False)
        assert np.max(np.abs(v_2 - v_t)) > 2e-3 * vmax, nme


def test_conditioning_vec_vs_torchtitan(tt_layers):
    cfg = TINY
    W = Weights(cfg)
    y = W["vector_in.in.b"][:0]  # placeholder to warm cache
    x, T, y = request_inputs(cfg, 64, 64, 1000)
    got = F.conditioning_vec(cfg, W, 0.6, y, 3.5)
    ref = 0
    for name, z in (("time_in", F.timestep_embedding(0.6)), ("guidance_in", F.timestep_embedding(3.5)),
                    ("vector_in", y)):
        m = tt_layers.MLPEmbedder(z.shape[0], cfg.hidden).double()
        _load(m.in_layer.weight, W, name + ".in.w"); _load(m.in_layer.bias, W, name + ".in.b")
        _load(m.out_layer.weight, W, name + ".out.w"); _load(m.out_layer.bias, W, name + ".out.b")
        with torch.no_grad():
            ref = ref + m(torch.from_numpy(z)[None])[0].numpy()
    assert np.allclose(got, ref, rtol=1e-11, atol=1e-12)


# ----------------------------------------------------------------------------- adaLN-Zero (P7), Euler (P8)
def test_adaln_zero_closed_form():
    cfg = TINY2
    W = Weights(cfg)
    zero = {}
    for tid, name, shape, kind, fan in __import__("oracle.config", fromlist=["x"]).tensor_table(cfg):
        if "mod." in name:
            zero[name] = np.zeros(shape)
    Wz = Weights(cfg, overrides=zero)
    x, T, y = request_inputs(cfg, 64, 64, 1001)
    v, xn = F.flux_step(cfg, Wz, x, T, y, 0.7, 0.6, 3.5, 64, 64)
    # every gate is 0 -> blocks are the identity; final shift = scale = 0
    img = x @ W["img_in.w"].T + W["img_in.b"]
    v_ref = F.layer_norm(img) @ W["final.lin.w"].T + W["final.lin.b"]
    assert np.allclose(v, v_ref, rtol=1e-12, atol=1e-12)
    assert np.allclose(xn, x - 0.1 * v_ref, rtol=1e-12, atol=1e-12)


def test_euler_zero_velocity():
    cfg = TINY
    Wz = Weights(cfg, overrides={"final.lin.w": np.zeros((cfg.in_ch, cfg.hidden)),
                                 "final.lin.b": np.zeros(cfg.in_ch)})
    x, T, y = request_inputs(cfg, 64, 64, 1002)
    v, xn = F.flux_step(cfg, Wz, x, T, y, 0.7, 0.6, 3.5, 64, 64)
    assert np.all(v == 0) and np.array_equal(xn, x)


# ----------------------------------------------------------------------------- SP (P9), index maps (P10)
@pytest.mark.parametrize("k", [1, 2, 4])
def test_sp_invariance(k):
    cfg = ModelCfg("tiny2_t66", 256, 4, 64, 1024, 2, 2, ctx_dim=512, vec_dim=256, text_tokens=66,
                   axes_dim=(8, 28, 28))   # 66 text tokens: uneven shards at k = 4
    W = Weights(cfg)
    x, T, y = request_inputs(cfg, 96, 80, 1003)
    v1, x1 = F.flux_step(cfg, W, x, T, y, 0.8, 0.7, 3.5, 96, 80)
    vk, xk = SP.flux_step_sp(cfg, W, x, T, y, 0.8, 0.7, 3.5, 96, 80, k)
    assert np.max(np.abs(vk - v1)) <= 1e-12 * np.max(np.abs(v1))
    assert np.max(np.abs(xk - x1)) <= 1e-12 * np.max(np.abs(x1))


def test_shard_ranges():
    assert [SP.shard_range(10, 4, r) for r in range(4)] == [(0, 3), (3, 6), (6, 8), (8, 10)]
    assert [SP.shard_range(333, 8, r)[1] - SP.shard_range(333, 8, r)[0] for r in range(8)] == [42] * 5 + [41] * 3
    for n in (0, 1, 7, 1024, 16384, 333):
        for k in (1, 2, 4, 8):
            rs = [SP.shard_range(n, k, r) for r in range(k)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(k - 1))
            assert max(b - a for a, b in rs) - min(b - a for a, b in rs) <= 1


def test_reshard_bitwise():
    rng = np.random.default_rng(7)
    x = rng.standard_normal((1037, 64)).astype(np.float32)
    for k in (1, 2, 4, 8):
        assert np.array_equal(SP.gather(SP.shard(x, k)), x)
        for k2 in (1, 2, 4, 8):
            y = SP.reshard(SP.shard(x, k), k2)
            assert all(np.array_equal(a, b) for a, b in zip(y, SP.shard(x, k2)))
            back = SP.reshard(y, k)
            assert all(np.array_equal(a, b) for a, b in zip(back, SP.shard(x, k)))
    # number of copies is at most k + k' - 1
    for k in (1, 2, 4, 8):
        for k2 in (1, 2, 4, 8):
            assert len(SP.reshard_plan(16384, k, k2)) <= k + k2 - 1
