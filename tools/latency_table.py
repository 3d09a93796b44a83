"""Step-latency table T(res, k) through tsv_latency_table: median of `iters` timed steps
after `warmup`, and the CV.  One process drives the ranks of this engine; on one
GPU only k = 1 is physical.  Prints one JSON line per cell and a summary line."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--res", default="256,512,1024,2048")
ap.add_argument("--ks", default="1")
ap.add_argument("--warmup", type=int, default=3)
ap.add_argument("--iters", type=int, default=20)
a = ap.parse_args()
res = [int(r) for r in a.res.split(",")]
ks = [int(k) for k in a.ks.split(",")]
eng = tsv.Engine("flux", devices=[0])
ms, cv = eng.latency_table(res, ks, warmup=a.warmup, iters=a.iters)
for i, r in enumerate(res):
    for j, k in enumerate(ks):
        print(json.dumps({"res": r, "k": k, "ms": round(float(ms[i, j]), 3), "cv": round(float(cv[i, j]), 5)}))
print(json.dumps({"table_ms": ms.tolist(), "cv": cv.tolist(), "res": res, "ks": ks}))
