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
