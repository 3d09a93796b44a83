"""Kernel-level parity (GPU): each kernel of the hot path against the float64 oracle / exact
integer arithmetic, through the kernel-level C-ABI (include/tsv_ops.h)."""
import math

import numpy as np
import pytest

import synth
from oracle import flux as F
from oracle.config import TINY, tensor_table

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def tsv():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_luhtlwm0c26_b200 as m
    return m


def _bf16(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(torch.bfloat16).cuda()


def _f32(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).cuda()


def _np(t):
    return t.float().cpu().numpy().astype(np.float64)


def _rel(g, o):
    return float(np.max(np.abs(g - o)) / max(np.max(np.abs(o)), 1e-30))


# ----------------------------------------------------------------------------- SYNTH-1
def test_synth_kernel_bitwise(tsv):
    for kind, sk, fan in ((0, "w", 3072), (0, "b", None), (1, "g", None), (2, "f", None)):
        n = 100_003
        c = synth.scale_for(sk, fan)
        ref = synth.gen_tensor_bits(0x7E7125E7, 77, n, sk, fan)
        if kind == 2:
            out = torch.empty(n, dtype=torch.float32, device="cuda")
            tsv.op_synth(out, 0x7E7125E7, 77, n, kind, c)
            torch.cuda.synchronize()
            assert np.array_equal(out.cpu().numpy().view(np.uint32), ref.view(np.uint32))
        else:
            out = torch.empty(n, dtype=torch.bfloat16, device="cuda")
            tsv.op_synth(out, 0x7E7125E7, 77, n, kind, c)
            torch.cuda.synchronize()
            assert np.array_equal(out.view(torch.int16).cpu().numpy().view(np.uint16), ref)


def test_engine_weights_bitwise(tsv):
    eng = tsv.Engine("tiny", devices=[0])
    for tid, name, shape, kind, fan in tensor_table(TINY):
        n = int(np.prod(shape))
        got = eng.debug_read_weight(tid, n)
        ref = synth.gen_tensor_bits(0x7E7125E7, tid, n, kind, fan)
        assert np.array_equal(got, ref), name
    eng.close()


# ----------------------------------------------------------------------------- GEMM
GEMM_SHAPES = [(1, 64, 64), (100, 256, 128), (128, 768, 256), (300, 1024, 256), (333, 3072, 3072),
               (1536, 3072, 3072), (20, 3584, 256), (513, 64, 3072)]


@pytest.mark.parametrize("M,N,K", GEMM_SHAPES)
@pytest.mark.parametrize("bn,pair", [(0, -1), (64, 0), (128, 0), (128, 1), (256, 0), (256, 1)])
def test_gemm_integer_exact(tsv, M, N, K, bn, pair):
    if bn and N % bn:
        pytest.skip("N not a multiple of the tile")
    rng = np.random.default_rng(M * 7 + N + K + bn)
    A = rng.integers(-4, 5, (M, K)).astype(np.float32)
    W = rng.integers(-4, 5, (N, K)).astype(np.float32)
    b = rng.integers(-4, 5, N).astype(np.float32)
    exact = A.astype(np.float64) @ W.astype(np.float64).T + b   # |sums| < 2^24: exact in fp32
    out = torch.zeros(M, N, dtype=torch.float32, device="cuda")
    tsv.op_gemm(_bf16(A), _bf16(W), "STORE_F32", out, bias=_bf16(b), force_bn=bn, force_pair=pair)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().astype(np.float64), exact)
    outb = torch.zeros(M, N, dtype=torch.bfloat16, device="cuda")
    tsv.op_gemm(_bf16(A), _bf16(W), "STORE_BF16", outb, bias=_bf16(b), force_bn=bn, force_pair=pair)
    torch.cuda.synchronize()
    ref_b = torch.from_numpy(exact.astype(np.float32)).to(torch.bfloat16)
    assert torch.equal(outb.cpu(), ref_b)


@pytest.mark.parametrize("M,N,K", [(1, 3072, 3072), (192, 3072, 12288), (300, 1536, 6144), (576, 3072, 15360),
                                   (1024, 3072, 3072), (70, 128, 1024)])
@pytest.mark.parametrize("splits", [0, 2, 5, 16])
def test_gemm_split_k_integer_exact(tsv, M, N, K, splits):
    """Split-K into the fp32 stream: integer operands make every partial sum exact, so any split
    factor (incl. more tiles than SMs: persistent CTAs) must reproduce x0 + A W^T + b bit for bit,
    and the semaphores must be left re-armed (all zero)."""
    rng = np.random.default_rng(M + N + K + splits)
    A = rng.integers(-2, 3, (M, K)).astype(np.float32)
    W = rng.integers(-2, 3, (N, K)).astype(np.float32)
    b = rng.integers(-4, 5, N).astype(np.float32)
    x0 = rng.integers(-100, 101, (M, N)).astype(np.float32)
    exact = x0.astype(np.float64) + A.astype(np.float64) @ W.astype(np.float64).T + b   # |.| < 2^24
    x = _f32(x0)
    sem = torch.zeros(4096, dtype=torch.int32, device="cuda")
    ws = torch.empty(64 << 18, dtype=torch.float32, device="cuda")
    tsv.op_gemm_split(_bf16(A), _bf16(W), "ACCUM_F32", x, sem, ws, splits=splits, bias=_bf16(b))
    torch.cuda.synchronize()
    assert np.array_equal(x.cpu().numpy().astype(np.float64), exact)
    assert torch.count_nonzero(sem) == 0


@pytest.mark.parametrize("M,N,K", [(64, 3072, 4096), (192, 12288, 3072), (100, 1536, 1536)])
def test_gemm_split_k_store_modes(tsv, M, N, K):
    """Split-K with the non-accumulating epilogues (the last split applies them to the summed
    partials): fp32 store bit-exact on integer operands, bf16 / GELU equal to the unsplit launch
    after rounding (same fp32 sum up to order) within one bf16 ulp."""
    rng = np.random.default_rng(M + N + K)
    A = rng.integers(-2, 3, (M, K)).astype(np.float32)
    W = rng.integers(-2, 3, (N, K)).astype(np.float32)
    b = rng.integers(-4, 5, N).astype(np.float32)
    exact = A.astype(np.float64) @ W.astype(np.float64).T + b
    sem = torch.zeros(4096, dtype=torch.int32, device="cuda")
    ws = torch.empty(64 << 18, dtype=torch.float32, device="cuda")
    o = torch.zeros(M, N, device="cuda")
    tsv.op_gemm_split(_bf16(A), _bf16(W), "STORE_F32", o, sem, ws, splits=3, bias=_bf16(b))
    torch.cuda.synchronize()
    assert np.array_equal(o.cpu().numpy().astype(np.float64), exact)
    Af = synth.bf16_bits_to_f32(synth.bf16_rne_bits(rng.standard_normal((M, K)).astype(np.float32)))
    Wf = synth.bf16_bits_to_f32(synth.bf16_rne_bits((rng.standard_normal((N, K)) / math.sqrt(K)).astype(np.float32)))
    y = Af.astype(np.float64) @ Wf.astype(np.float64).T + b
    for mode, fn in (("STORE_BF16", lambda v: v), ("GELU_BF16", F.gelu_tanh)):
        o1 = torch.zeros(M, N, dtype=torch.bfloat16, device="cuda")
        o2 = torch.zeros(M, N, dtype=torch.bfloat16, device="cuda")
        tsv.op_gemm_split(_bf16(Af), _bf16(Wf), mode, o1, sem, ws, splits=4, bias=_bf16(b))
        tsv.op_gemm(_bf16(Af), _bf16(Wf), mode, o2, bias=_bf16(b))
        torch.cuda.synchronize()
        assert _rel(_np(o1), fn(y)) < 1e-2
        assert _rel(_np(o1), _np(o2)) < 1e-2
    assert torch.count_nonzero(sem) == 0


def test_gemm_split_k_resid_gate_deterministic(tsv):
    rng = np.random.default_rng(21)
    M, N, K = 192, 3072, 12288
    A = synth.bf16_bits_to_f32(synth.bf16_rne_bits(rng.standard_normal((M, K)).astype(np.float32)))
    W = synth.bf16_bits_to_f32(synth.bf16_rne_bits((rng.standard_normal((N, K)) / math.sqrt(K)).astype(np.float32)))
    b = synth.bf16_bits_to_f32(synth.bf16_rne_bits((0.1 * rng.standard_normal(N)).astype(np.float32)))
    x0 = rng.standard_normal((M, N)).astype(np.float32)
    gate = rng.standard_normal(N).astype(np.float32)
    y = A.astype(np.float64) @ W.astype(np.float64).T + b
    sem = torch.zeros(4096, dtype=torch.int32, device="cuda")
    ws = torch.empty(64 << 18, dtype=torch.float32, device="cuda")
    outs = []
    for splits in (6, 6, 0):
        x = _f32(x0)
        tsv.op_gemm_split(_bf16(A), _bf16(W), "RESID_GATE", x, sem, ws, splits=splits, bias=_bf16(b), gate=_f32(gate))
        torch.cuda.synchronize()
        assert _rel(_np(x), x0 + gate * y) < 1e-5
        outs.append(x.cpu())
    assert torch.equal(outs[0], outs[1])      # fixed split order: run-to-run bitwise
    assert torch.count_nonzero(sem) == 0


def test_gemm_epilogues_vs_oracle(tsv):
    rng = np.random.default_rng(11)
    M, N, K = 200, 768, 512
    A = synth.bf16_bits_to_f32(synth.bf16_rne_bits(rng.standard_normal((M, K)).astype(np.float32)))
    W = synth.bf16_bits_to_f32(synth.bf16_rne_bits((rng.standard_normal((N, K)) / math.sqrt(K)).astype(np.float32)))
    b = synth.bf16_bits_to_f32(synth.bf16_rne_bits((0.1 * rng.standard_normal(N)).astype(np.float32)))
    y = A.astype(np.float64) @ W.astype(np.float64).T + b
    At, Wt, bt = _bf16(A), _bf16(W), _bf16(b)
    for mode, fn in (("GELU_BF16", F.gelu_tanh), ("SILU_BF16", F.silu)):
        o = torch.zeros(M, N, dtype=torch.bfloat16, device="cuda")
        tsv.op_gemm(At, Wt, mode, o, bias=bt)
        torch.cuda.synchronize()
        assert _rel(_np(o), fn(y)) < 1e-2
    # split: first 512 columns plain, rest GELU into a second buffer with its own stride
    o0 = torch.zeros(M, 512, dtype=torch.bfloat16, device="cuda")
    o1 = torch.zeros(M, 1024, dtype=torch.bfloat16, device="cuda")
    tsv.op_gemm(At, Wt, "SPLIT_GELU", o0, out1=o1[:, 256:], bias=bt, n_split=512, ld1=1024)
    torch.cuda.synchronize()
    assert _rel(_np(o0), y[:, :512]) < 1e-2
    assert _rel(_np(o1[:, 256:512]), F.gelu_tanh(y[:, 512:])) < 1e-2
    assert torch.count_nonzero(o1[:, :256]) == 0
    # gated residual and Euler into fp32 state
    x0 = rng.standard_normal((M, N)).astype(np.float32)
    gate = rng.standard_normal(N).astype(np.float32)
    x = _f32(x0)
    tsv.op_gemm(At, Wt, "RESID_GATE", x, bias=bt, gate=_f32(gate))
    torch.cuda.synchronize()
    assert _rel(_np(x), x0 + gate * y) < 1e-5
    dt = _f32(np.array([-0.05], np.float32))
    x = _f32(x0)
    v = torch.zeros(M, N, dtype=torch.float32, device="cuda")
    tsv.op_gemm(At, Wt, "EULER", x, out1=v, bias=bt, scalar=dt)
    torch.cuda.synchronize()
    assert _rel(_np(v), y) < 1e-5
    assert _rel(_np(x), x0 - 0.05 * y) < 1e-5


def test_gemm_sampled_full_size(tsv):
    """FLUX 512^2 single-block linear1 shape (M = 1536, N = 21504, K = 3072): sampled outputs."""
    rng = np.random.default_rng(12)
    M, N, K = 1536, 21504, 3072
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    W = (torch.randn(N, K, device="cuda") / math.sqrt(K)).to(torch.bfloat16)
    o = torch.zeros(M, N, dtype=torch.float32, device="cuda")
    tsv.op_gemm(A, W, "STORE_F32", o)
    torch.cuda.synchronize()
    rows = rng.integers(0, M, 64)
    cols = rng.integers(0, N, 64)
    An, Wn = _np(A), _np(W)
    ref = np.array([An[r] @ Wn[c] for r, c in zip(rows, cols)])
    got = o.cpu().numpy()[rows, cols].astype(np.float64)
    assert np.max(np.abs(got - ref)) < 1e-3 * np.max(np.abs(ref)) + 1e-4


def test_gemm_rejects_bad_shapes(tsv):
    A = torch.zeros(16, 100, dtype=torch.bfloat16, device="cuda")
    W = torch.zeros(64, 100, dtype=torch.bfloat16, device="cuda")
    o = torch.zeros(16, 64, dtype=torch.float32, device="cuda")
    with pytest.raises(tsv.TsvError):
        tsv.op_gemm(A, W, "STORE_F32", o)


# ----------------------------------------------------------------------------- LN-modulate
@pytest.mark.parametrize("impl", [0, 1, 2])
@pytest.mark.parametrize("M,h", [(1, 256), (333, 256), (1536, 3072), (77, 1536), (5, 640), (13, 3072)])
def test_ln_mod(tsv, M, h, impl):
    rng = np.random.default_rng(M + h)
    x = (rng.standard_normal((M, h)) * 3 + 0.5).astype(np.float32)
    sh = rng.standard_normal(h).astype(np.float32)
    sc = rng.standard_normal(h).astype(np.float32)
    u = torch.zeros(M, h, dtype=torch.bfloat16, device="cuda")
    tsv.op_ln_mod(_f32(x), u, _f32(sh), _f32(sc), impl=impl)
    torch.cuda.synchronize()
    ref = F.ln_modulate(x.astype(np.float64), sh, sc)
    err = np.abs(_np(u) - ref)
    assert np.all(err <= 2 ** -8 * np.abs(ref) + 1e-5 * np.max(np.abs(ref)))


# ----------------------------------------------------------------------------- QK-RMSNorm + RoPE
@pytest.mark.parametrize("H,D,rows,n_first", [(4, 64, 320, 64), (24, 128, 700, 512), (24, 128, 37, 0)])
def test_qk_norm_rope(tsv, H, D, rows, n_first):
    rng = np.random.default_rng(H + D + rows)
    h = H * D
    qkv = rng.standard_normal((rows, 3 * h)).astype(np.float32)
    qkv = synth.bf16_bits_to_f32(synth.bf16_rne_bits(qkv)).astype(np.float64)
    gains = [synth.bf16_bits_to_f32(synth.bf16_rne_bits((1 + 0.1 * rng.standard_normal(D)).astype(np.float32)))
             for _ in range(4)]
    axes = (16, 56, 56) if D == 128 else (8, 28, 28)
    ids = np.stack([np.zeros(rows), rng.integers(0, 64, rows), rng.integers(0, 64, rows)], axis=1).astype(np.float64)
    ang = F.rope_angles(ids, axes, 1e4)
    cosb, sinb = np.cos(ang).astype(np.float32), np.sin(ang).astype(np.float32)
    q, k, v = F.split_qkv(qkv, H, D)
    g_q = np.where(np.arange(rows)[:, None, None] < n_first, gains[0], gains[2])
    g_k = np.where(np.arange(rows)[:, None, None] < n_first, gains[1], gains[3])
    rq = F.apply_rope(F.rms_norm(q, g_q), ang)
    rk = F.apply_rope(F.rms_norm(k, g_k), ang)
    t = _bf16(qkv)
    gt = [_bf16(g) for g in gains]
    tsv.op_qk_norm_rope(t, n_first, H, D, gt[0], gt[1], gt[2], gt[3], _f32(cosb), _f32(sinb))
    torch.cuda.synchronize()
    out = _np(t).reshape(rows, 3, H, D)
    for got, ref in ((out[:, 0], rq), (out[:, 1], rk)):
        assert np.all(np.abs(got - ref) <= 2 ** -8 * np.abs(ref) + 2e-3)
    assert np.array_equal(out[:, 2], v)
    # pack layout [k_sp][rows][3][H/k][D] equals the in-place result permuted, bit for bit
    for k_sp in (2, 4):
        t2 = _bf16(qkv)
        pack = torch.zeros(rows * 3 * h, dtype=torch.bfloat16, device="cuda")
        tsv.op_qk_norm_rope(t2, n_first, H, D, gt[0], gt[1], gt[2], gt[3], _f32(cosb), _f32(sinb), pack=pack, k_sp=k_sp)
        torch.cuda.synchronize()
        p = pack.view(k_sp, rows, 3, H // k_sp, D).permute(1, 2, 0, 3, 4).reshape(rows, 3, H, D)
        assert torch.equal(p.cpu(), t.view(rows, 3, H, D).cpu())
        assert torch.equal(t2.cpu(), _bf16(qkv).cpu())  # source untouched in pack mode


# ----------------------------------------------------------------------------- attention
@pytest.mark.parametrize("impl", [0, 50, 51, 56, 81, 83, 92, 96, 103])
@pytest.mark.parametrize("L,H,D", [(1, 2, 64), (63, 4, 64), (320, 4, 64), (1000, 3, 128), (1536, 2, 128),
                                   (4700, 1, 128), (1357, 3, 64)])
def test_attention(tsv, L, H, D, impl):
    if 90 <= impl and D != 64:
        pytest.skip("rotating S buffers: D = 64 only")
    rng = np.random.default_rng(L + H + D)
    qkv = rng.standard_normal((L, 3, H, D)).astype(np.float32) * np.float32(1.5)
    qkv = synth.bf16_bits_to_f32(synth.bf16_rne_bits(qkv)).astype(np.float64)
    ref = F.attention(qkv[:, 0], qkv[:, 1], qkv[:, 2])
    t = _bf16(qkv.reshape(L, 3 * H * D))
    o = torch.zeros(L, 2 * H * D, dtype=torch.bfloat16, device="cuda")   # strided output (row stride 2HD)
    ld = 3 * H * D
    tsv.op_attention(t, t[:, H * D:], t[:, 2 * H * D:], o, L, H, D, ldq=ld, ldk=ld, ldv=ld, impl=impl)
    torch.cuda.synchronize()
    got = _np(o)[:, :H * D].reshape(L, H, D)
    assert _rel(got, ref) < 1.5e-2
    cos = np.sum(got * ref) / np.linalg.norm(got) / np.linalg.norm(ref)
    assert cos > 0.9999
    assert torch.count_nonzero(o[:, H * D:]) == 0


@pytest.mark.parametrize("L,H,D", [(1000, 3, 128), (1536, 3, 128), (4700, 1, 128), (1357, 2, 64), (4429, 3, 64),
                                   (600, 1, 64)])
@pytest.mark.parametrize("nsplit", [0, 2, 3, 8])
def test_attention_kv_split(tsv, L, H, D, nsplit):
    """KV split: each key range's partial (O, m, l) merged in range order equals softmax attention
    (oracle), is deterministic run to run, and leaves the counters re-armed."""
    rng = np.random.default_rng(L * 3 + H + D + nsplit)
    qkv = rng.standard_normal((L, 3, H, D)).astype(np.float32) * np.float32(1.5)
    qkv = synth.bf16_bits_to_f32(synth.bf16_rne_bits(qkv)).astype(np.float64)
    qkv[L // 2:, 1] += 0.8          # later keys score higher: the ranges' references differ
    qkv = synth.bf16_bits_to_f32(synth.bf16_rne_bits(qkv.astype(np.float32))).astype(np.float64)
    ref = F.attention(qkv[:, 0], qkv[:, 1], qkv[:, 2])
    t = _bf16(qkv.reshape(L, 3 * H * D))
    ld = 3 * H * D
    cnt = torch.zeros(4096, dtype=torch.int32, device="cuda")
    ws = torch.empty(16 << 20, dtype=torch.float32, device="cuda")
    outs = []
    for _ in range(2):
        o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
        tsv.op_attention_split(t, t[:, H * D:], t[:, 2 * H * D:], o, L, H, D, cnt, ws, nsplit=nsplit, ldq=ld, ldk=ld,
                               ldv=ld)
        torch.cuda.synchronize()
        outs.append(o.cpu())
        got = _np(o).reshape(L, H, D)
        assert _rel(got, ref) < 1.5e-2
        assert np.sum(got * ref) / np.linalg.norm(got) / np.linalg.norm(ref) > 0.9999
    assert torch.equal(outs[0], outs[1])
    assert torch.count_nonzero(cnt) == 0


@pytest.mark.parametrize("L,H,D", [(4608, 12, 128), (4429, 12, 64)])
def test_attention_tail_split(tsv, L, H, D):
    """Automatic KV split with a tail (FLUX / SD3 1024^2 at SP = 2: 216 work items on 148 SMs): the
    first items run whole, the last ones in key ranges merged by their last range -- every head
    against the float64 definition, deterministic run to run, counters re-armed."""
    rng = np.random.default_rng(L + H)
    qkv = rng.standard_normal((L, 3, H, D)).astype(np.float32) * np.float32(1.5)
    qkv[L // 2:, 1] += 0.8
    qkv = synth.bf16_bits_to_f32(synth.bf16_rne_bits(qkv)).astype(np.float64)
    ref = F.attention(qkv[:, 0], qkv[:, 1], qkv[:, 2])
    t = _bf16(qkv.reshape(L, 3 * H * D))
    ld = 3 * H * D
    cnt = torch.zeros(4096, dtype=torch.int32, device="cuda")
    ws = torch.empty(32 << 20, dtype=torch.float32, device="cuda")
    outs = []
    for _ in range(2):
        o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
        tsv.op_attention_split(t, t[:, H * D:], t[:, 2 * H * D:], o, L, H, D, cnt, ws, nsplit=0, ldq=ld, ldk=ld,
                               ldv=ld)
        torch.cuda.synchronize()
        outs.append(o.cpu())
        got = _np(o).reshape(L, H, D)
        assert _rel(got, ref) < 1.5e-2
        assert np.sum(got * ref) / np.linalg.norm(got) / np.linalg.norm(ref) > 0.9999
    assert torch.equal(outs[0], outs[1])
    assert torch.count_nonzero(cnt) == 0


@pytest.mark.parametrize("ws_items", [1, 7, 40])
def test_attention_split_workspace_bounds(tsv, ws_items):
    """The automatic KV split stays inside the workspace it is given: a workspace for only ws_items
    split 256-query blocks (2 splits each) and a counter array of 8 x ws_items ints, both followed by
    guard regions (NaN / -1) that must stay untouched; the result still matches the float64 oracle."""
    L, H, D = 4608, 12, 128
    rng = np.random.default_rng(ws_items)
    qkv = rng.standard_normal((L, 3, H, D)).astype(np.float32)
    qkv = synth.bf16_bits_to_f32(synth.bf16_rne_bits(qkv)).astype(np.float64)
    t = _bf16(qkv.reshape(L, 3 * H * D))
    ld = 3 * H * D
    n_ws = ws_items * 2 * 2 * 128 * (D + 2)
    n_cnt = 8 * ws_items
    ws_all = torch.full((n_ws + 65536,), float("nan"), dtype=torch.float32, device="cuda")
    cnt_all = torch.zeros(n_cnt + 1024, dtype=torch.int32, device="cuda")
    cnt_all[n_cnt:] = -1
    o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
    tsv.op_attention_split(t, t[:, H * D:], t[:, 2 * H * D:], o, L, H, D, cnt_all[:n_cnt], ws_all[:n_ws], nsplit=0,
                           ldq=ld, ldk=ld, ldv=ld)
    torch.cuda.synchronize()
    assert torch.isnan(ws_all[n_ws:]).all()
    assert (cnt_all[n_cnt:] == -1).all() and torch.count_nonzero(cnt_all[:n_cnt]) == 0
    hh = [0, H - 1]
    ref = F.attention(qkv[:, 0][:, hh], qkv[:, 1][:, hh], qkv[:, 2][:, hh])
    got = _np(o).reshape(L, H, D)[:, hh]
    assert _rel(got, ref) < 1.5e-2


@pytest.mark.parametrize("L,H,D,split", [(16896, 24, 128, False), (16896, 3, 128, True), (16896, 12, 128, True),
                                         (16717, 24, 64, False), (16717, 6, 64, True), (4429, 3, 64, True)])
def test_attention_sampled_full_size(tsv, L, H, D, split):
    """BASELINE sizes (FLUX 2048^2 joint L = 16 896, SD3 2048^2 / 1024^2 L = 16 717 / 4429; H = 3 is an
    SP = 8 head shard, run with the KV split): sampled query rows of sampled heads against the
    float64 definition over all L keys, in the launch configuration the step uses."""
    g = torch.Generator(device="cuda").manual_seed(L + H + D)
    qkv = (torch.randn(L, 3 * H * D, device="cuda", generator=g) * 1.5).to(torch.bfloat16)
    o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
    ld = 3 * H * D
    if split:
        cnt = torch.zeros(4096, dtype=torch.int32, device="cuda")
        ws = torch.empty(32 << 20, dtype=torch.float32, device="cuda")
        tsv.op_attention_split(qkv, qkv[:, H * D:], qkv[:, 2 * H * D:], o, L, H, D, cnt, ws, nsplit=0, ldq=ld, ldk=ld,
                               ldv=ld)
    else:
        tsv.op_attention(qkv, qkv[:, H * D:], qkv[:, 2 * H * D:], o, L, H, D, ldq=ld, ldk=ld, ldv=ld)
    torch.cuda.synchronize()
    rng = np.random.default_rng(L)
    rows = np.concatenate([[0, L - 1], rng.choice(L, 14, replace=False)])
    heads = sorted(set([0, H - 1] + list(rng.choice(H, min(H, 2), replace=False))))
    t = qkv.view(L, 3, H, D)
    for hh in heads:
        k = t[:, 1, hh].double().cpu().numpy()
        v = t[:, 2, hh].double().cpu().numpy()
        q = t[rows, 0, hh].double().cpu().numpy()
        ref = F.attention(q[:, None, :], k[:, None, :], v[:, None, :])[:, 0]   # oracle: queries x all keys
        got = o.view(L, H, D)[rows, hh].double().cpu().numpy()
        assert _rel(got, ref) < 1.5e-2, hh
        assert np.sum(got * ref) / np.linalg.norm(got) / np.linalg.norm(ref) > 0.9999


def test_attention_special_cases(tsv):
    # identical keys -> mean(V) (S:§8(c) P3)
    L, H, D = 300, 2, 128
    rng = np.random.default_rng(5)
    q = rng.standard_normal((L, H, D))
    k = np.repeat(rng.standard_normal((1, H, D)), L, axis=0)
    v = rng.integers(-3, 4, (L, H, D)).astype(np.float64)
    o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
    tq, tk, tv = _bf16(q.reshape(L, -1)), _bf16(k.reshape(L, -1)), _bf16(v.reshape(L, -1))
    tsv.op_attention(tq, tk, tv, o, L, H, D)
    torch.cuda.synchronize()
    ref = np.repeat(v.mean(axis=0, keepdims=True), L, axis=0)
    assert np.max(np.abs(_np(o).reshape(L, H, D) - ref)) < 2e-2


@pytest.mark.parametrize("impl", [0, 50, 51, 56, 81, 83])
def test_attention_rescale_path(tsv, impl):
    """Scores growing along the key axis force the conditional O rescale (max grows by > 2^8)."""
    L, H, D = 700, 1, 128
    rng = np.random.default_rng(9)
    q = np.ones((L, H, D)) * 0.5
    k = rng.standard_normal((L, H, D)) * 0.1 + np.linspace(0, 3, L)[:, None, None]
    v = rng.standard_normal((L, H, D))
    ref = F.attention(q, k, v)
    o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
    tsv.op_attention(_bf16(q.reshape(L, -1)), _bf16(k.reshape(L, -1)), _bf16(v.reshape(L, -1)), o, L, H, D,
                     impl=impl)
    torch.cuda.synchronize()
    # compare against the oracle on the bf16-rounded inputs
    qb, kb, vb = (synth.bf16_bits_to_f32(synth.bf16_rne_bits(a.astype(np.float32))).astype(np.float64)
                  for a in (q, k, v))
    ref = F.attention(qb, kb, vb)
    assert _rel(_np(o).reshape(L, H, D), ref) < 2e-2


@pytest.mark.parametrize("D,impl", [(64, 0), (64, 51), (64, 83), (64, 92), (64, 96), (64, 103), (128, 0), (128, 51), (128, 56), (128, 81)])
@pytest.mark.parametrize("jump", [3.0, 12.0, 200.0])
def test_attention_score_jump(tsv, D, impl, jump):
    """A later key tile whose scores exceed the running maximum by `jump` (log2 units): small jumps
    stay on the lazy path (p up to 2^jump), large ones overflow the lazy sum bound (or exp2 itself)
    and must take the exact path with an O rescale."""
    L, H = 900, 2
    rng = np.random.default_rng(int(jump))
    q = np.ones((L, H, D)) / np.sqrt(D)
    k = rng.standard_normal((L, H, D)) * 0.3
    k[500:] += jump / np.log2(np.e)           # score(s) = q.k / sqrt(D) -> + jump*ln2 for keys >= 500
    v = rng.standard_normal((L, H, D))
    qb, kb, vb = (synth.bf16_bits_to_f32(synth.bf16_rne_bits(a.astype(np.float32))).astype(np.float64)
                  for a in (q, k, v))
    o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
    tsv.op_attention(_bf16(qb.reshape(L, -1)), _bf16(kb.reshape(L, -1)), _bf16(vb.reshape(L, -1)), o, L, H, D,
                     impl=impl)
    torch.cuda.synchronize()
    ref = F.attention(qb, kb, vb)
    got = _np(o).reshape(L, H, D)
    assert np.all(np.isfinite(got))
    assert _rel(got, ref) < 2e-2


@pytest.mark.parametrize("impl", [0, 83, 92, 96, 103, 51, 56])
def test_attention_large_logits_many_rescales(tsv, impl):
    """Scores with a large spread (q, k ~ 8 N(0, 1)): most key tiles overflow the lazy bound and take
    the exact path with an O rescale, so the softmax warps of a warpgroup drift apart by tiles -- the
    case that exposed a barrier-phase race in the rotating-S variant (impl 92).  SD3 1024^2 shape
    (L = 4429, H = 24), two heads checked against the float64 definition."""
    L, H = 4429, 24
    D = 128 if impl in (51, 56) else 64
    g = torch.Generator(device="cuda").manual_seed(impl)
    qkv = (torch.randn(L, 3 * H * D, device="cuda", generator=g) * 8.0).to(torch.bfloat16)
    o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
    ld = 3 * H * D
    tsv.op_attention(qkv, qkv[:, H * D:], qkv[:, 2 * H * D:], o, L, H, D, ldq=ld, ldk=ld, ldv=ld, impl=impl)
    torch.cuda.synchronize()
    t = qkv.view(L, 3, H, D)
    for hh in (0, H - 1):
        q, k, v = (t[:, i, hh].double().cpu().numpy()[:, None, :] for i in range(3))
        ref = F.attention(q, k, v)[:, 0]
        got = o.view(L, H, D)[:, hh].double().cpu().numpy()
        assert _rel(got, ref) < 2e-2, hh
        assert np.sum(got * ref) / np.linalg.norm(got) / np.linalg.norm(ref) > 0.999
