"""SD3-medium family (config 5) through the C-ABI on the GPU: the CFG step against the float64
oracle (oracle/sd3.py) at tiny and full SD3 shapes, SP=k with the uneven 77/333-token text
stream, step-level SP with reshards, and the per-(res, k) latency table."""
import os

import numpy as np
import pytest

from oracle import sd3 as S3
from oracle.config import MODELS
from oracle.weights import Weights, sd3_request_inputs

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TOL_REL, TOL_COS = 2e-2, 0.999   # BASELINE.json north_star: max rel error 2e-2, cosine >= 0.999


@pytest.fixture(scope="module")
def tsv():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_luhtlwm0c26_b200 as m
    return m


def _metrics(g, o):
    rel = float(np.max(np.abs(g - o)) / np.max(np.abs(o)))
    cos = float(np.sum(g * o) / np.linalg.norm(g) / np.linalg.norm(o))
    return rel, cos


@pytest.mark.parametrize("res,steps,step", [((256, 256), 20, 0), ((208, 240), 4, 0)])
def test_tiny_sd3_step_vs_oracle(tsv, res, steps, step):
    cfg = MODELS["tiny_sd3"]
    H, Wd = res
    eng = tsv.Engine("tiny_sd3", devices=[0])
    g = eng.group_create([0])
    req = eng.request_create(H, Wd, num_steps=steps, seed=1000)
    x, Tc, yc, Tu, yu = sd3_request_inputs(cfg, H, Wd, 1000)
    assert np.array_equal(eng.read_latent(req), x.astype(np.float32))
    eng.event_wait(eng.request_step(req, 0, g))
    v, x1 = eng.read_velocity(req), eng.read_latent(req)
    vo, xo = S3.request_step(cfg, Weights(cfg), x, Tc, yc, Tu, yu, 0, steps, H, Wd)
    for got, ref in ((v, vo), (x1, xo)):
        rel, cos = _metrics(got.astype(np.float64), ref)
        assert rel <= TOL_REL and cos >= TOL_COS, (rel, cos)
    eng.close()


def test_tiny_sd3_inputs_replaced(tsv):
    """tsv_request_set_inputs with the CFG pair layout T = (T_c, T_u), y = (y_c, y_u): equal
    branches make the guidance term vanish (oracle special case)."""
    import synth
    cfg = MODELS["tiny_sd3"]
    eng = tsv.Engine("tiny_sd3", devices=[0])
    g = eng.group_create([0])
    req = eng.request_create(128, 128, num_steps=2, seed=77)
    x, Tc, yc, Tu, yu = sd3_request_inputs(cfg, 128, 128, 77)
    Tb = synth.gen_tensor_bits(77, 2, Tc.size, "x")
    yb = synth.gen_tensor_bits(77, 3, yc.size, "x")
    eng.request_set_inputs(req, T_bits=np.concatenate([Tb, Tb]), y_bits=np.concatenate([yb, yb]))
    eng.event_wait(eng.request_step(req, 0, g))
    vo = S3.forward(cfg, Weights(cfg), x, Tc, yc, S3.schedule(cfg, 2)[0], 128, 128)
    rel, cos = _metrics(eng.read_velocity(req).astype(np.float64), vo)
    assert rel <= TOL_REL and cos >= TOL_COS, (rel, cos)
    eng.close()


@pytest.mark.parametrize("k", [2, 4])
def test_tiny_sd3_sp_vs_oracle(tsv, k):
    """k virtual ranks; 77 text tokens (k = 4: 20/19/19/19) and 195 image tokens: uneven shards."""
    cfg = MODELS["tiny_sd3"]
    eng = tsv.Engine("tiny_sd3", devices=[0] * 4)
    g = eng.group_create(list(range(k))[::-1])
    req = eng.request_create(208, 240, num_steps=3, seed=1003)
    eng.event_wait(eng.request_step(req, 0, g))
    x, Tc, yc, Tu, yu = sd3_request_inputs(cfg, 208, 240, 1003)
    vo, xo = S3.request_step(cfg, Weights(cfg), x, Tc, yc, Tu, yu, 0, 3, 208, 240)
    rel, cos = _metrics(eng.read_velocity(req).astype(np.float64), vo)
    assert rel <= TOL_REL and cos >= TOL_COS, (rel, cos)
    rel, cos = _metrics(eng.read_latent(req).astype(np.float64), xo)
    assert rel <= TOL_REL and cos >= TOL_COS, (rel, cos)
    eng.close()


def test_tiny_sd3_step_level_sp_with_reshard(tsv):
    eng = tsv.Engine("tiny_sd3", devices=[0] * 4)
    groups = [eng.group_create([0, 1]), eng.group_create([0, 1, 2, 3]), eng.group_create([3]), eng.group_create([2, 0])]
    g1 = eng.group_create([0])
    ra = eng.request_create(256, 256, num_steps=4, seed=1004)
    rb = eng.request_create(256, 256, num_steps=4, seed=1004)
    for s, g in enumerate(groups):
        if s > 0:
            before = eng.read_latent(ra)
            eng.event_wait(eng.request_reshard(ra, g))
            assert np.array_equal(before, eng.read_latent(ra))
        eng.request_step(ra, s, g)
        eng.request_step(rb, s, g1)
    rel, cos = _metrics(eng.read_latent(ra).astype(np.float64), eng.read_latent(rb).astype(np.float64))
    assert rel <= 1e-2 and cos >= 0.9999, (rel, cos)
    eng.close()


@pytest.fixture(scope="module")
def sd3_engine(tsv):
    eng = tsv.Engine("sd3", devices=[0] * 8)
    yield eng
    eng.close()


def test_sd3_512_golden(tsv, sd3_engine):
    """Full SD3-medium shapes (24 joint blocks, L = 1024 + 333) at 512^2, step 0 of 20, against the
    oracle's stored result (tests/golden/sd3_512_seed1000_S20.npz, written by tools/make_golden.py
    from oracle/ only)."""
    gold = np.load(os.path.join(ROOT, "tests", "golden", "sd3_512_seed1000_S20.npz"))
    eng = sd3_engine
    for ranks in ([0], [0, 1, 2, 3, 4, 5, 6, 7]):
        g = eng.group_create(ranks)
        req = eng.request_create(512, 512, num_steps=20, seed=1000)
        eng.event_wait(eng.request_step(req, 0, g))
        for got, ref in ((eng.read_velocity(req), gold["v"]), (eng.read_latent(req), gold["x_next"])):
            rel, cos = _metrics(got.astype(np.float64), ref)
            assert rel <= TOL_REL and cos >= TOL_COS, (ranks, rel, cos)
        eng.request_destroy(req)


def test_sd3_1024_golden(tsv, sd3_engine):
    """Config 5's 1024^2 SD3 request (L = 4096 + 333, CFG pair) at step 0 of 20 against the float64
    oracle (tests/golden/sd3_1024_seed1000_S20.npz, tools/make_golden.py sd3_1024), SP = 1 and 8."""
    p = os.path.join(ROOT, "tests", "golden", "sd3_1024_seed1000_S20.npz")
    if not os.path.exists(p):
        pytest.skip("golden sd3_1024_seed1000_S20.npz not generated (tools/make_golden.py sd3_1024)")
    gold = np.load(p)
    eng = sd3_engine
    for ranks in ([0], [0, 1, 2, 3, 4, 5, 6, 7]):
        g = eng.group_create(ranks)
        req = eng.request_create(1024, 1024, num_steps=20, seed=1000)
        eng.event_wait(eng.request_step(req, 0, g))
        for got, ref in ((eng.read_velocity(req), gold["v"]), (eng.read_latent(req), gold["x_next"])):
            rel, cos = _metrics(got.astype(np.float64), ref.astype(np.float64))
            assert rel <= TOL_REL and cos >= TOL_COS, (ranks, rel, cos)
        eng.request_destroy(req)


def test_sd3_latency_table(tsv, sd3_engine):
    ms, cv = sd3_engine.latency_table([512, 1024], [1, 2], warmup=1, iters=3)
    assert ms.shape == (2, 2) and np.all(ms > 0)
    assert ms[1, 0] > ms[0, 0]


def test_mixed_round_tool(tsv, tmp_path):
    """Config 5 machinery end to end at tiny shapes: latency table -> deadlines -> DP packer rounds
    -> disjoint-group placement with reshards -> every request completes all its steps."""
    import json
    import subprocess
    import sys
    out = tmp_path / "round.json"
    subprocess.run([sys.executable, os.path.join(ROOT, "tools", "mixed_round.py"), "--model", "tiny_sd3",
                    "--gpus", "4", "--res", "128", "256", "512", "--steps", "6", "--table-iters", "2",
                    "--out", str(out)], check=True, timeout=600)
    r = json.load(open(out))
    assert len(r["completion"]) == 3 and all(c["finish_s"] > 0 for c in r["completion"])
    assert sum(e["steps"] for rd in r["rounds"] for e in rd["requests"]) == 3 * 6
    for rd in r["rounds"]:
        assert sum(e["gpus"] for e in rd["requests"]) <= 4
