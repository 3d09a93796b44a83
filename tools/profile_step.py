"""One FLUX step under the CUDA profiler API (for ncu --profile-from-start off).

  python tools/profile_step.py [--res 512] [--k 1] [--steps 1]
Creates the engine, runs 2 warm-up steps, then brackets `--steps` steps with cudaProfilerStart/Stop.
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--res", type=int, default=512)
ap.add_argument("--k", type=int, default=1)
ap.add_argument("--steps", type=int, default=1)
ap.add_argument("--model", default="flux")
a = ap.parse_args()
eng = tsv.Engine(a.model, devices=[0] * a.k)
eng.set_graphs(False)   # direct launches: one ncu record per kernel
g = eng.group_create(list(range(a.k)))
req = eng.request_create(a.res, a.res, num_steps=2 + a.steps, seed=1000)
for s in range(2):
    eng.request_step(req, s, g)
torch.cuda.synchronize()
k0 = eng.kernel_count()
torch.cuda.profiler.start()
for s in range(a.steps):
    eng.request_step(req, 2 + s, g)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print(f"profiled {a.steps} step(s): {eng.kernel_count() - k0} kernel launches")
