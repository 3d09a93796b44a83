"""NEXT #3 — selective batching: several same-resolution requests, each at its own
step, run as one batched step (every GEMM / LN / all-to-all launch covers all of them).  The
batched step must equal the separate steps (same per-row arithmetic) and the oracle."""
import numpy as np
import pytest

from oracle import flux as F
from oracle import sd3 as S3
from oracle.config import MODELS
from oracle.weights import Weights, request_inputs, sd3_request_inputs

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
TOL_REL, TOL_COS = 2e-2, 0.999


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


@pytest.mark.parametrize("model,n,k", [("tiny2", 3, 1), ("tiny2", 4, 2), ("tiny_sd3", 2, 1), ("tiny_sd3", 3, 4)])
def test_batched_equals_separate(tsv, model, n, k):
    res = (208, 240)
    seeds = [1100 + i for i in range(n)]
    lead = [0, 1, 2, 0][:n]                 # requests at different step indices
    out = []
    for batched in (True, False):
        eng = tsv.Engine(model, devices=[0] * 4)
        g = eng.group_create(list(range(k)))
        reqs = [eng.request_create(*res, num_steps=4, seed=sd) for sd in seeds]
        for r, pre in zip(reqs, lead):      # advance some requests alone first
            for s in range(pre):
                eng.request_step(r, s, g)
        for _ in range(2):
            if batched:
                eng.request_step_batch(reqs, g)
            else:
                for r in reqs:
                    eng.request_step(r, eng.request_info(r)[0], g)
        out.append([(eng.read_latent(r), eng.read_velocity(r)) for r in reqs])
        eng.close()
    bitwise = all(np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1]) for a, b in zip(*out))
    print(f"{model} n={n} k={k}: batched == separate bitwise: {bitwise}")
    for (xa, va), (xb, vb) in zip(*out):
        for got, ref in ((xa, xb), (va, vb)):
            rel, cos = _metrics(got.astype(np.float64), ref.astype(np.float64))
            assert rel <= 1e-2 and cos >= 0.9999, (rel, cos)


def test_batched_vs_oracle(tsv):
    cfg = MODELS["tiny2"]
    eng = tsv.Engine("tiny2", devices=[0])
    g = eng.group_create([0])
    reqs = [eng.request_create(256, 256, num_steps=3, seed=1200 + i) for i in range(2)]
    eng.request_step(reqs[1], 0, g)           # request 1 one step ahead
    eng.event_wait(eng.request_step_batch(reqs, g))
    W = Weights(cfg)
    for i, (r, st) in enumerate(zip(reqs, (0, 1))):
        x, T, y = request_inputs(cfg, 256, 256, 1200 + i)
        if st == 1:
            _, x = F.request_step(cfg, W, x, T, y, 0, 3, 3.5, 256, 256)
        vo, xo = F.request_step(cfg, W, x, T, y, st, 3, 3.5, 256, 256)
        for got, ref in ((eng.read_velocity(r), vo), (eng.read_latent(r), xo)):
            rel, cos = _metrics(got.astype(np.float64), ref)
            assert rel <= TOL_REL and cos >= TOL_COS, (i, rel, cos)
    eng.close()


def test_batched_sd3_vs_oracle(tsv):
    cfg = MODELS["tiny_sd3"]
    eng = tsv.Engine("tiny_sd3", devices=[0])
    g = eng.group_create([0])
    reqs = [eng.request_create(128, 160, num_steps=5, seed=1300 + i) for i in range(3)]
    eng.event_wait(eng.request_step_batch(reqs, g))
    W = Weights(cfg)
    for i, r in enumerate(reqs):
        x, Tc, yc, Tu, yu = sd3_request_inputs(cfg, 128, 160, 1300 + i)
        vo, xo = S3.request_step(cfg, W, x, Tc, yc, Tu, yu, 0, 5, 128, 160)
        rel, cos = _metrics(eng.read_velocity(r).astype(np.float64), vo)
        assert rel <= TOL_REL and cos >= TOL_COS, (i, rel, cos)
    eng.close()


def test_batch_errors(tsv):
    eng = tsv.Engine("tiny2", devices=[0])
    g = eng.group_create([0])
    a = eng.request_create(256, 256, num_steps=2, seed=1)
    b = eng.request_create(128, 256, num_steps=2, seed=2)
    with pytest.raises(tsv.TsvError):
        eng.request_step_batch([a, b], g)        # mixed resolutions
    with pytest.raises(tsv.TsvError):
        eng.request_step_batch([a, a], g)        # repeated request
    with pytest.raises(tsv.TsvError):
        eng.request_step_batch([a] + [eng.request_create(256, 256, num_steps=2, seed=9 + i) for i in range(8)], g)
    eng.close()
