"""Selective batching (NEXT #3): step time of B same-resolution requests batched into
one step vs B separate steps, per resolution, on one GPU (CUDA-event timed, graphs on).

  python tools/batch_bench.py [--model flux] [--res 256 512 1024] [--batch 1 2 4] [--iters 10]

Prints one JSON line per (res, B): batched ms per step (all B requests), separate ms (B single
steps back to back), and the per-request throughput gain.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import paper_conf_asplos_luhtlwm0c26_b200 as tsv

    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="flux")
    ap.add_argument("--res", type=int, nargs="+", default=[256, 512, 1024])
    ap.add_argument("--batch", type=int, nargs="+", default=[1, 2, 4])
    ap.add_argument("--iters", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    args = ap.parse_args()
    eng = tsv.Engine(args.model, devices=[0])
    g = eng.group_create([0])
    for res in args.res:
        for B in args.batch:
            steps = args.warmup + args.iters
            reqs = [eng.request_create(res, res, num_steps=2 * steps + 2, seed=500 + i) for i in range(B)]

            def run(batched, n):
                for _ in range(n):
                    if batched:
                        eng.request_step_batch(reqs, g)
                    else:
                        for r in reqs:
                            eng.request_step(r, eng.request_info(r)[0], g)

            out = {}
            for batched in (True, False):
                run(batched, args.warmup)
                a = eng.group_record(g)
                run(batched, args.iters)
                b = eng.group_record(g)
                out[batched] = eng.event_elapsed_ms(a, b) / args.iters
            for r in reqs:
                eng.request_destroy(r)
            print(json.dumps({"model": args.model, "res": res, "batch": B, "batched_ms": round(out[True], 3),
                              "separate_ms": round(out[False], 3),
                              "throughput_gain": round(out[False] / out[True], 3)}), flush=True)
    eng.close()


if __name__ == "__main__":
    main()
