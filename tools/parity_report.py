"""Parity of the GPU step against the float64 oracle's goldens (tests/golden, written by
tools/make_golden.py from oracle/ only): max relative error (normwise inf) and cosine of v and x_1,
at the north-star FLUX 2048^2 (SP = 1 and SP = 8 on virtual ranks) and at 512^2 (FLUX, SD3).
One JSON line per case.  python tools/parity_report.py"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402

CASES = [("flux", 2048, 20, 1, "flux2048_seed1000_S20_step0.npz"), ("flux", 2048, 20, 8, "flux2048_seed1000_S20_step0.npz"),
         ("flux", 1024, 20, 1, "flux1024_seed1000_S20_step0.npz"), ("flux", 1024, 20, 8, "flux1024_seed1000_S20_step0.npz"),
         ("flux", 512, 1, 1, "flux512_seed1000_S1.npz"), ("sd3", 512, 20, 1, "sd3_512_seed1000_S20.npz"),
         ("sd3", 1024, 20, 1, "sd3_1024_seed1000_S20.npz"), ("sd3", 1024, 20, 8, "sd3_1024_seed1000_S20.npz")]
for model, res, steps, k, gold in CASES:
    if not os.path.exists(os.path.join(ROOT, "tests", "golden", gold)):
        continue
    g = np.load(os.path.join(ROOT, "tests", "golden", gold))
    eng = tsv.Engine(model, devices=[0] * k)
    grp = eng.group_create(list(range(k)))
    r = eng.request_create(res, res, num_steps=steps, seed=1000)
    eng.event_wait(eng.request_step(r, 0, grp))
    out = {"model": model, "res": res, "sp": k, "golden": gold}
    for name, got, ref in (("v", eng.read_velocity(r), g["v"]), ("x_next", eng.read_latent(r), g["x_next"])):
        a, b = got.astype(np.float64), ref.astype(np.float64)
        out[name] = {"rel": float(np.max(np.abs(a - b)) / np.max(np.abs(b))),
                     "cos": float(np.sum(a * b) / np.linalg.norm(a) / np.linalg.norm(b))}
    out["tolerance"] = {"rel": 2e-2, "cos": 0.999}
    print(json.dumps(out), flush=True)
    eng.close()
