"""NEXT #2 across processes: two processes (one rank each) on one GPU run a k = 2 group with the
fused transport over CUDA-IPC windows and the device barrier (no NCCL).  The result must equal the
in-process fused k = 2 run of the same request bit for bit (same kernels, same arithmetic)."""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("model", ["tiny2", "tiny_sd3"])
def test_two_process_ipc_fused_equals_in_process(model, tmp_path):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_luhtlwm0c26_b200 as tsv
    H, W, steps = 208, 240, 2
    out = str(tmp_path / "ipc.npz")
    port = _port()
    procs = []
    for r in range(2):
        env = dict(os.environ, RANK=str(r), WORLD_SIZE="2", MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        procs.append(subprocess.Popen([sys.executable, os.path.join(ROOT, "tools", "ipc_worker.py"), model, str(H),
                                       str(W), str(steps), out], env=env))
    for p in procs:
        assert p.wait(timeout=300) == 0
    got = np.load(out)
    eng = tsv.Engine(model, devices=[0, 0])
    g = eng.group_create([0, 1])
    req = eng.request_create(H, W, num_steps=steps + 1, seed=1600)
    for s in range(steps):
        eng.request_step(req, s, g)
    x, v = eng.read_latent(req), eng.read_velocity(req)
    eng.close()
    assert np.array_equal(got["x"], x) and np.array_equal(got["v"], v)


def test_bench_two_ranks_one_gpu():
    """bench.py's N > 1 code path (torchrun, two ranks, max-over-ranks timing, e2e, JSON line) on a
    one-GPU box: TSV_BENCH_ONE_GPU=1 puts both ranks on device 0 with the fused CUDA-IPC transport
    (NCCL refuses two ranks on one GPU).  Not a scaling measurement."""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import json
    port = _port()
    env = dict(os.environ, TSV_BENCH_ONE_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(port), os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3",
           "--warmup", "3", "--res", "256", "--no-cpu-baseline"]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["sp"] == 2 and "fused-ipc" in d["config"]["transport"]
    assert d["value"] > 0 and d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    assert d["warmup"] == 3 and d["steps"] == 3
    assert d["comm"]["transport"].startswith("fused-ipc") and d["comm"]["barrier_ms_per_step"] >= 0
    assert d["latency"]["steps"] == 3 and d["latency"]["cv"] >= 0
    assert d["roofline"]["unit"] == "TFLOP/s" and set(d["roofline_kernels"]) == {"gemm", "attention"}
