"""Fused a3+a4 (QKV GEMM with QK-RMSNorm + RoPE + Ulysses pack in the epilogue) vs the oracle."""
import math

import numpy as np
import pytest

import synth
from oracle import flux as F

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def tsv():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_luhtlwm0c26_b200 as m
    return m


def _b(a):
    return synth.bf16_bits_to_f32(synth.bf16_rne_bits(np.asarray(a, dtype=np.float32))).astype(np.float64)


def _t(a, dt=torch.bfloat16):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(dt).cuda()


def _case(H, D, M, F_extra, seed):
    rng = np.random.default_rng(seed)
    h = H * D
    K = 256
    A = _b(rng.standard_normal((M, K)))
    W = _b(rng.standard_normal((3 * h + F_extra, K)) / math.sqrt(K))
    b = _b(0.05 * rng.standard_normal(3 * h + F_extra))
    gq, gk = _b(1 + 0.1 * rng.standard_normal(D)), _b(1 + 0.1 * rng.standard_normal(D))
    axes = (16, 56, 56) if D == 128 else (8, 28, 28)
    ids = np.stack([np.zeros(M), rng.integers(0, 64, M), rng.integers(0, 64, M)], axis=1).astype(np.float64)
    ang = F.rope_angles(ids, axes, 1e4)
    y = A @ W.T + b
    q, k, v = F.split_qkv(y[:, :3 * h], H, D)
    ref = np.stack([F.apply_rope(F.rms_norm(q, gq), ang), F.apply_rope(F.rms_norm(k, gk), ang), v], axis=1)
    return A, W, b, gq, gk, np.cos(ang), np.sin(ang), y, ref


@pytest.mark.parametrize("H,D,M", [(4, 64, 300), (24, 128, 333), (24, 128, 1024)])
def test_fused_qkv_in_place(tsv, H, D, M):
    A, W, b, gq, gk, cs, sn, y, ref = _case(H, D, M, 0, H + M)
    h = H * D
    out = torch.zeros(M, 3 * h, dtype=torch.bfloat16, device="cuda")
    tsv.op_gemm_qkv(_t(A), _t(W), out, h, D, _t(gq), _t(gk), _t(cs, torch.float32), _t(sn, torch.float32),
                    bias=_t(b))
    torch.cuda.synchronize()
    got = out.float().cpu().numpy().astype(np.float64).reshape(M, 3, H, D)
    err = np.abs(got - ref)
    assert np.all(err <= 2 ** -7 * np.abs(ref) + 2e-3 * np.max(np.abs(ref)))


def test_fused_single_block_split_and_pack(tsv):
    """Single-block linear1: [qkv | GELU(mlp)] with the qkv part packed for k_sp = 4 ranks."""
    H, D, M, Fx = 8, 64, 200, 1024
    A, W, b, gq, gk, cs, sn, y, ref = _case(H, D, M, Fx, 7)
    h = H * D
    k_sp, rows, row0 = 4, 260, 37            # pack buffer holds 260 rows; this GEMM writes rows 37..236
    pack = torch.zeros(k_sp * rows * 3 * h // k_sp, dtype=torch.bfloat16, device="cuda")
    mlp = torch.zeros(M, Fx + 64, dtype=torch.bfloat16, device="cuda")
    dummy = torch.zeros(M, 3 * h, dtype=torch.bfloat16, device="cuda")
    tsv.op_gemm_qkv(_t(A), _t(W), dummy, h, D, _t(gq), _t(gk), _t(cs, torch.float32), _t(sn, torch.float32),
                    bias=_t(b), mode="SPLIT_GELU", out1=mlp[:, 64:], ld1=Fx + 64, k_sp=k_sp, pack=pack,
                    pack_rows=rows, pack_row0=row0)
    torch.cuda.synchronize()
    p = pack.view(k_sp, rows, 3, H // k_sp, D).permute(1, 2, 0, 3, 4).reshape(rows, 3, H, D)
    got = p[row0:row0 + M].float().cpu().numpy().astype(np.float64)
    err = np.abs(got - ref)
    assert np.all(err <= 2 ** -7 * np.abs(ref) + 2e-3 * np.max(np.abs(ref)))
    assert torch.count_nonzero(p[:row0]) == 0 and torch.count_nonzero(p[row0 + M:]) == 0
    assert torch.count_nonzero(dummy) == 0                     # packed mode leaves out0 untouched
    g = mlp[:, 64:].float().cpu().numpy().astype(np.float64)
    assert np.max(np.abs(g - F.gelu_tanh(y[:, 3 * h:]))) <= 1e-2 * np.max(np.abs(F.gelu_tanh(y[:, 3 * h:])))
