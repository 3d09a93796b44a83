"""BASELINE.json config 5: a mixed-resolution round of SD3-medium-shaped requests packed across the
GPUs of one box with per-step SP degrees chosen from the measured latency table (SURVEY §8 config
5; paper §4.2).

  python tools/mixed_round.py [--model sd3] [--gpus 8] [--res 512 1024 2048 4096] [--steps 20]
                              [--tau-steps 5] [--out gpurun_out/mixed_round.json]

1. Latency table T(res, k) from tsv_latency_table (median of timed steps).
2. Deadlines: the paper's SLO vector 2.0 / 3.0 / 5.0 s for 512^2 / 1024^2 / 2048^2,
   rescaled so that D(2048^2) = S * T(2048^2, 8) on this box; D(4096^2) = 4 D(2048^2),
   D(256^2) = D(512^2).
3. Rounds of length tau = tau_steps * T(largest res, N): each round the C++ DP packer
   (tsv_sched_round, Alg. 1) chooses (GPUs, steps) per request; requests are placed on disjoint,
   aligned GPU groups (buddy placement of power-of-two blocks) and run concurrently; the latent is
   resharded whenever a request's group changes.  GPUs the packer leaves idle go to
   requests it did not schedule (one GPU each; a work-conserving tool policy outside Alg. 1).
4. Report per round: the plan, makespan, each request's in-round step latency vs the table
   (interference), GPU-busy fraction; and each request's completion time vs its deadline.

With fewer physical GPUs than --gpus, ranks are virtual (several ranks per device): the run is
functionally identical but device time is serialised, so the timing columns are not meaningful
(the report says so).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SLO = {256: 2.0, 512: 2.0, 1024: 3.0, 2048: 5.0}   # seconds; 4096 = 4 x 2048


def buddy_place(plan, N):
    """Disjoint aligned blocks of `g` GPUs for each request (largest first); -> {req: [ranks]}."""
    free = [True] * N
    out = {}
    for i in sorted(range(len(plan)), key=lambda i: -plan[i][0]):
        g = plan[i][0]
        if g <= 0:
            continue
        for start in range(0, N, g):
            if all(free[start:start + g]):
                for r in range(start, start + g):
                    free[r] = False
                out[i] = list(range(start, start + g))
                break
        else:
            raise RuntimeError(f"cannot place {g} GPUs")
    return out


def main():
    import torch

    import paper_conf_asplos_luhtlwm0c26_b200 as tsv
    from paper_conf_asplos_luhtlwm0c26_b200 import sched

    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="sd3")
    ap.add_argument("--gpus", type=int, default=8)
    ap.add_argument("--res", type=int, nargs="+", default=[512, 1024, 2048, 4096])
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--tau-steps", type=int, default=5)
    ap.add_argument("--table-iters", type=int, default=5)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "mixed_round.json"))
    args = ap.parse_args()

    N = args.gpus
    ndev = torch.cuda.device_count()
    devices = [i % ndev for i in range(N)]
    virtual = ndev < N
    eng = tsv.Engine(args.model, devices=devices)
    ks = [k for k in (1, 2, 4, 8) if k <= N]
    res = sorted(args.res)

    t0 = time.perf_counter()
    ms, cv = eng.latency_table(res, ks, warmup=2, iters=args.table_iters)
    T = ms / 1e3                                              # seconds
    table_s = time.perf_counter() - t0

    ref = 2048 if 2048 in res else res[-1]
    scale = args.steps * T[res.index(ref), len(ks) - 1] / SLO.get(ref, 5.0)
    deadline = {}
    for r in res:
        base = SLO.get(r, 4 * SLO[2048] if r > 2048 else SLO[512])
        deadline[r] = base * scale
    tau = args.tau_steps * T[-1, len(ks) - 1]

    reqs = []
    for i, r in enumerate(res):
        rid = eng.request_create(r, r, num_steps=args.steps, seed=2000 + i)
        reqs.append(dict(res=r, row=i, id=rid, done=0, group=None, finish=None))
    groups = {}

    rounds = []
    clock = 0.0     # device-time clock: sum of round makespans
    while any(q["done"] < args.steps for q in reqs):
        live = [q for q in reqs if q["done"] < args.steps]
        sv, plan = sched.schedule_round(T, ks, [(deadline[q["res"]], args.steps - q["done"], q["row"]) for q in live],
                                        clock, tau, N)
        plan = list(plan)
        # work-conserving fill (tool policy, outside Alg. 1): GPUs the packer leaves idle go to
        # requests it did not schedule this round (doomed or late), one GPU each
        used = sum(g for g, _ in plan)
        for j, q in enumerate(live):
            if plan[j][0] == 0 and used < N:
                n = max(1, min(args.steps - q["done"], int(tau // T[q["row"], 0])))
                plan[j] = (1, n)
                used += 1
        place = buddy_place(plan, N)
        evs = []
        for j, q in enumerate(live):
            if j not in place:
                continue
            g_ranks = tuple(place[j])
            if g_ranks not in groups:
                groups[g_ranks] = eng.group_create(list(g_ranks))
            g = groups[g_ranks]
            a = eng.group_record(g)
            if q["group"] is not None and q["group"] != g:
                eng.request_reshard(q["id"], g)
            for _ in range(plan[j][1]):
                eng.request_step(q["id"], q["done"], g)
                q["done"] += 1
            b = eng.group_record(g)
            q["group"] = g
            evs.append((q, plan[j], a, b))
        torch.cuda.synchronize()
        span = 0.0
        busy = 0.0
        entries = []
        for q, (g, n), a, b in evs:
            t = eng.event_elapsed_ms(a, b) / 1e3
            span = max(span, t)
            busy += g * t
            t_tab = T[q["row"], ks.index(g)]
            entries.append(dict(res=q["res"], gpus=g, steps=n, seconds=round(t, 5),
                                step_ms=round(t / n * 1e3, 3), table_step_ms=round(t_tab * 1e3, 3),
                                interference=round(t / n / t_tab, 3)))
        clock += span
        for q, *_ in evs:
            if q["done"] >= args.steps and q["finish"] is None:
                q["finish"] = clock
        rounds.append(dict(survivors=int(sv), makespan_s=round(span, 5),
                           gpu_busy=round(busy / (N * span), 4) if span else None, requests=entries))
        if not evs:
            raise RuntimeError("scheduler returned an empty plan")

    out = dict(model=args.model, gpus=N, devices=ndev, virtual_ranks=bool(virtual),
               note=("ranks are virtual (several per device): device time is serialised, timings are not "
                     "representative of N GPUs") if virtual else "one rank per GPU",
               steps=args.steps, ks=ks, res=res, table_ms=np.round(ms, 3).tolist(), table_cv=np.round(cv, 4).tolist(),
               table_build_s=round(table_s, 1), tau_s=round(tau, 5),
               deadlines_s={str(r): round(d, 4) for r, d in deadline.items()}, rounds=rounds,
               completion=[dict(res=q["res"], finish_s=round(q["finish"], 4), deadline_s=round(deadline[q["res"]], 4),
                                met=bool(q["finish"] <= deadline[q["res"]] + 1e-9)) for q in reqs],
               total_s=round(clock, 4))
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(out, open(args.out, "w"), indent=1)
    print(json.dumps({k: out[k] for k in ("model", "gpus", "virtual_ranks", "table_ms", "deadlines_s", "total_s",
                                          "completion")}))
    eng.close()


if __name__ == "__main__":
    main()
