"""The PyTorch hooks of the C-ABI (S:§8(b): tsv_engine_set_allocator / tsv_engine_set_stream;
north_star: "PyTorch is used only for device memory, streams and process groups") and the
non-blocking latent hand-off ("asynchronous, non-blocking" Future)."""
import os
import time

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TOL_REL, TOL_COS = 2e-2, 0.999   # BASELINE.json north_star


@pytest.fixture(scope="module")
def tsv():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_luhtlwm0c26_b200 as m
    return m


def _metrics(g, o):
    return float(np.max(np.abs(g - o)) / np.max(np.abs(o))), float(np.sum(g * o) / np.linalg.norm(g) / np.linalg.norm(o))


def test_torch_allocator_and_stream_reproduce_golden(tsv):
    """An engine whose every buffer comes from PyTorch's caching allocator and whose kernels run on
    a torch stream reproduces the FLUX 512^2 golden (float64 oracle, tools/make_golden.py)."""
    p = os.path.join(ROOT, "tests", "golden", "flux512_seed1000_S1.npz")
    gold = np.load(p)
    torch.cuda.synchronize()
    before = torch.cuda.memory_allocated(0)
    stream = torch.cuda.Stream(device=0)
    eng = tsv.Engine("flux", devices=[0])
    eng.use_torch_allocator()
    eng.set_stream(0, stream)
    g = eng.group_create([0])               # device state (weights: 23.7 GB) is created here
    weights = torch.cuda.memory_allocated(0) - before
    assert weights > 23e9, weights          # the weights live in torch's allocator
    req = eng.request_create(512, 512, num_steps=1, seed=1000)
    ev = eng.request_step(req, 0, g)
    # the step was enqueued on the caller's stream: a torch event recorded behind it on that stream
    # completes only after the step
    done = torch.cuda.Event()
    done.record(stream)
    done.synchronize()
    assert eng.event_query(ev)
    v, x1 = eng.read_velocity(req).astype(np.float64), eng.read_latent(req).astype(np.float64)
    for got, ref in ((v, gold["v"]), (x1, gold["x_next"])):
        rel, cos = _metrics(got, ref)
        assert rel <= TOL_REL and cos >= TOL_COS, (rel, cos)
    per_request = torch.cuda.memory_allocated(0) - before - weights
    assert per_request > 0                  # the request's latent / tables / workspaces too
    eng.request_destroy(req)
    eng.close()
    torch.cuda.synchronize()
    assert torch.cuda.memory_allocated(0) == before   # every buffer went back through free_fn


def test_hooks_only_before_device_state(tsv):
    eng = tsv.Engine("tiny", devices=[0])
    with pytest.raises(tsv.TsvError) as e:
        eng.set_stream(3, torch.cuda.Stream(device=0))
    assert e.value.status == -1                 # device 3 hosts no rank of this engine
    eng.group_create([0])
    with pytest.raises(tsv.TsvError) as e:
        eng.use_torch_allocator()
    assert e.value.status == -2
    with pytest.raises(tsv.TsvError) as e:
        eng.set_stream(0, torch.cuda.Stream(device=0))
    assert e.value.status == -2
    eng.close()


def test_reshard_does_not_block_the_host(tsv):
    """a13: request_reshard returns while the request's previous step is still running on the old
    group (the copies are ordered on the device, old shards are released stream-ordered) -- both on a
    first landing (per-GPU state set up on the new ranks) and on a return to ranks that already hold
    the request (a pure latent move) -- and the moved latent is bit-identical to the one an unmoved
    twin request holds."""
    eng = tsv.Engine("flux", devices=[0] * 4)
    g01, g23 = eng.group_create([0, 1]), eng.group_create([2, 3])
    ra = eng.request_create(2048, 2048, num_steps=20, seed=1600)
    rb = eng.request_create(2048, 2048, num_steps=20, seed=1600)
    for r in (ra, rb):
        eng.event_wait(eng.request_step(r, 0, g01))   # first landing + graph capture
    step = 1
    for dst, bound_ms in ((g23, 50.0), (g01, 5.0), (g23, 5.0)):   # first landing on 2, 3; then returns
        src = g01 if dst == g23 else g23
        ev = eng.request_step(ra, step, src)            # ~0.2-0.4 s of device work
        t0 = time.perf_counter()
        eng.request_reshard(ra, dst)
        host_ms = (time.perf_counter() - t0) * 1e3
        running = not eng.event_query(ev)
        eng.event_wait(eng.request_step(rb, step, g01))
        assert running, "the step finished before reshard returned: the call waited on the device"
        assert host_ms < bound_ms, (step, host_ms)
        assert np.array_equal(eng.read_latent(ra), eng.read_latent(rb))
        step += 1
    eng.event_wait(eng.request_step(ra, step, g23))
    eng.event_wait(eng.request_step(rb, step, g01))
    assert np.array_equal(eng.read_latent(ra), eng.read_latent(rb))   # same kernels, same bits
    eng.close()
