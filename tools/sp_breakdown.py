"""Per-rank kernel-class breakdown of one step at SP degree k on ONE GPU: k virtual ranks serialised
on one stream (TSV_VIRTUAL_SERIAL=1), so every kernel runs alone on the GPU as it would on a rank's
own GPU; the in-step event profile gives device time per class (GEMM / attention / LN-modulate /
other), divided by k = one rank's time.  The NVLink all-to-all is not in it (fused transport: the
exchange is the epilogue stores into the peer buffers of the same device).

  python tools/sp_breakdown.py [--model flux] [--res 512,1024,2048] [--ks 1,2,4,8] [--out file.jsonl]
"""
import argparse
import json
import os
import sys

os.environ["TSV_VIRTUAL_SERIAL"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--model", default="flux")
ap.add_argument("--res", default="512,1024,2048")
ap.add_argument("--ks", default="1,2,4,8")
ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--out", default=None)
a = ap.parse_args()
lines = []
for res in [int(r) for r in a.res.split(",")]:
    for k in [int(x) for x in a.ks.split(",")]:
        eng = tsv.Engine(a.model, devices=[0] * k)
        g = eng.group_create(list(range(k)))
        req = eng.request_create(res, res, num_steps=2 + a.steps, seed=1000)
        for s in range(2):
            eng.request_step(req, s, g)
        torch.cuda.synchronize()
        eng.profile(True)
        for s in range(a.steps):
            eng.request_step(req, 2 + s, g)
        torch.cuda.synchronize()
        prof = eng.profile_read()
        eng.profile(False)
        eng.close()
        per = {c: round(v["ms"] / (a.steps * k), 4) for c, v in prof.items() if v["launches"]}
        tf = {c: round(v["flops"] / max(v["ms"], 1e-9) / 1e9, 1) for c, v in prof.items() if v["flops"] and v["ms"]}
        d = {"model": a.model, "res": res, "k": k, "per_rank_ms": per, "per_rank_total_ms": round(sum(per.values()), 4),
             "tflops": tf, "launches_per_rank_step": {c: v["launches"] // (a.steps * k) for c, v in prof.items()
                                                      if v["launches"]}}
        print(json.dumps(d), flush=True)
        lines.append(d)
if a.out:
    with open(a.out, "w") as f:
        for d in lines:
            f.write(json.dumps(d) + "\n")
