"""Reshard overhead (Table 4 analogue): the latent hand-off between GPU groups when a
request's SP degree / group changes between steps, as a fraction of the step latency.

  python tools/reshard_bench.py [--res 256 512 1024 2048] [--bs 1 2 4] [--reps 3]

One B200, four virtual ranks (devices [0] * 4): groups A = [0, 1], B = [2, 3] (k = 2) and
C = [0..3] (k = 4).  For each resolution and batch size BS (BS requests stepped together with
request_step_batch), the requests first land on A, C and B (so every rank holds their
per-GPU state: text rows and embedding, RoPE tables, modulation table), then alternate between the
groups; every move is timed after the previous step completed:
  host_ms  wall time of the request_reshard calls (non-blocking: enqueue only)
  dev_ms   device time of the moves on the destination ranks (group_record before / after)
  step_ms  the following batched step on the destination group
and first landings (per-GPU state set up: modulation table copied from a rank holding it, text
embedding, tables) are reported separately.  On one GPU the row copies are device-local; the same
bytes over NVLink 5 (~700 GB/s achievable per direction) are given as nvlink_us.  One JSON line per
(res, BS, kind).
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--res", type=int, nargs="+", default=[256, 512, 1024, 2048])
    ap.add_argument("--bs", type=int, nargs="+", default=[1, 2, 4])
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    eng = tsv.Engine("flux", devices=[0] * 4)
    gA, gB, gC = eng.group_create([0, 1]), eng.group_create([2, 3]), eng.group_create([0, 1, 2, 3])
    ks = {gA: 2, gB: 2, gC: 4}
    for res in a.res:
        for bs in a.bs:
            n_steps = 3 + 3 * a.reps + 1
            reqs = [eng.request_create(res, res, num_steps=n_steps, seed=2000 + i) for i in range(bs)]
            li = (res // 16) ** 2
            lat_bytes = li * 64 * 4 * bs

            def move_and_step(g):
                t0 = time.perf_counter()
                e0 = eng.group_record(g)
                for r in reqs:
                    eng.request_reshard(r, g)
                e1 = eng.group_record(g)
                host = (time.perf_counter() - t0) * 1e3
                ev = eng.request_step_batch(reqs, g)
                e2 = eng.group_record(g)
                eng.event_wait(ev)
                return host, eng.event_elapsed_ms(e0, e1), eng.event_elapsed_ms(e1, e2)

            first = [move_and_step(g) for g in (gA, gC, gB)]     # first landings on A, then C (ranks 2, 3), B
            moves = [move_and_step(g) for _ in range(a.reps) for g in (gA, gC, gB)]
            for kind, rows in (("first_landing", first[1:]), ("latent_move", moves)):
                host = [r[0] for r in rows]
                dev = [r[1] for r in rows]
                step = [r[2] for r in rows]
                frac = [d / s for d, s in zip(dev, step)]
                print(json.dumps({
                    "op": "reshard", "kind": kind, "res": res, "bs": bs, "moves": len(rows),
                    "host_ms_median": round(statistics.median(host), 4),
                    "dev_ms_median": round(statistics.median(dev), 4),
                    "step_ms_median": round(statistics.median(step), 3),
                    "dev_over_step_pct_median": round(100 * statistics.median(frac), 4),
                    "dev_over_step_pct_max": round(100 * max(frac), 4),
                    "latent_bytes": lat_bytes, "nvlink_us_at_700GBps": round(lat_bytes / 700e9 * 1e6, 2),
                    "note": "one B200, virtual ranks: device-local copies"}), flush=True)
            for r in reqs:
                eng.request_destroy(r)
    eng.close()


if __name__ == "__main__":
    main()
