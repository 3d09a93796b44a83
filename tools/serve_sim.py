"""Synthetic online serving loop (S:§8(f) NEXT #4): SLO attainment ratio (SAR) of TetriServe's
round-based scheduling (Alg. 1 DP + GPU placement preservation + elastic scale-up, all through
libtsv.so's C++ scheduler, include/tsv_sched.h) against fixed-degree sequence parallelism, on a
step-latency table T(res, k), with Poisson arrivals.

  python tools/serve_sim.py --table profiles/r01/latency_table_model.json [--rate 12] [--n 300]
                            [--mix uniform|skewed] [--slo-scale 1.0 1.25 1.5] [--gpus 8]

Workload (paper §5.1): Poisson arrivals at `rate` requests/min; resolutions {256, 512, 1024, 2048}
drawn uniformly ("uniform") or with p_i ∝ exp(alpha L_i / L_max), alpha = 1 ("skewed");
S = 20 steps each; SLOs 1.5 / 2.0 / 3.0 / 5.0 s rescaled to this table so that the
2048^2 SLO equals S T(2048^2, N) (the config-5 rule), times --slo-scale.

Policies:
  tetriserve     rounds of tau = gran * T(largest res, N) (gran = 5 steps); each round
                 tsv_sched_round picks (GPUs, steps) per request, tsv_sched_place keeps requests
                 on their GPUs and scales idle GPUs up; a request whose GPUs change pays
                 a reshard (latent bytes over NVLink).
  tetriserve-np  the same without placement preservation and scale-up (Table 5 ablation analogue).
  tetriserve-wc  the same as tetriserve with Alg. 1's argmax tie taken at the largest capacity
                 (reading S31b: every request that can make progress runs now at its minimal
                 allocation) instead of the smallest (S31: requests with slack are deferred).
  fixed-k        every request runs all its steps at SP degree k on k GPUs, FCFS (xDiT-style).
  rssp           resolution-specific SP: 1 / 1 / 2 / 8 GPUs for 256^2 / 512^2 / 1024^2 / 2048^2, FCFS.

The simulator itself is plain Python; only the scheduling decisions come from the C-ABI.
Timing comes from the table (device-measured per-rank step latencies, see latency_table_model).
"""
from __future__ import annotations

import argparse
import heapq
import json
import math
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

RES = [256, 512, 1024, 2048]
SLO = {256: 1.5, 512: 2.0, 1024: 3.0, 2048: 5.0}   # seconds
NVLINK_BPS = 900e9                                 # per direction per GPU (NVLink 5)


def mix_probs(mix):
    if mix == "uniform":
        p = np.ones(len(RES))
    else:
        L = np.array([(r // 16) ** 2 for r in RES], dtype=float)
        p = np.exp(L / L.max())
    return p / p.sum()


def workload(n, rate_per_min, mix, seed, steps=20):
    rng = np.random.default_rng(seed)
    p = mix_probs(mix)
    t = np.cumsum(rng.exponential(60.0 / rate_per_min, n))
    res = rng.choice(len(RES), size=n, p=p)
    return [dict(id=i, arrival=float(t[i]), row=int(res[i]), steps=steps) for i in range(n)]


def deadlines(T, ks, N, steps, scale):
    ref = steps * T[RES.index(2048), ks.index(N)]
    f = ref / SLO[2048]
    return {r: SLO[r] * f * scale for r in RES}


def reshard_s(row):
    Li = (RES[row] // 16) ** 2
    return Li * 64 * 4 / NVLINK_BPS + 20e-6


def sim_tetriserve(T, ks, N, reqs, dl, gran=5, preserve=True, wc=False):
    """Rounds every tau.  GPUs still busy from earlier work (a best-effort step longer than tau)
    are excluded from the round; the packer and the placement work on the free GPUs (NVSwitch:
    any subset can form a group, S14), mapped to their ids in ascending order."""
    from paper_conf_asplos_luhtlwm0c26_b200 import sched
    tau = gran * T[-1, ks.index(N)]
    pending = sorted(reqs, key=lambda r: r["arrival"])
    live, done = [], {}
    prev = {}
    busy_until = [0.0] * N
    running_until = {}
    now = 0.0
    busy = 0.0
    i = 0
    while i < len(pending) or live:
        while i < len(pending) and pending[i]["arrival"] <= now + 1e-12:
            q = dict(pending[i])
            q["left"] = q["steps"]
            q["deadline"] = q["arrival"] + dl[RES[q["row"]]]
            live.append(q)
            i += 1
        if not live:
            now = pending[i]["arrival"]
            continue
        free = [g for g in range(N) if busy_until[g] <= now + 1e-12]
        cand = [q for q in live if running_until.get(q["id"], 0.0) <= now + 1e-12]
        ran = False
        if free and cand:
            nf = len(free)
            # the packer needs power-of-two degrees <= the free capacity
            ks_r = [k for k in ks if k <= nf]
            Tr = T[:, [ks.index(k) for k in ks_r]]
            sv, plan = sched.schedule_round(Tr, ks_r, [(q["deadline"], q["left"], q["row"]) for q in cand], now, tau, nf,
                                            work_conserving=wc)
            idx = {g: j for j, g in enumerate(free)}
            prv = [{idx[g] for g in prev.get(q["id"], set()) if g in idx} if preserve else set() for q in cand]
            nf2 = 1 << (nf.bit_length() - 1)          # placement works on an aligned pool
            gpus = [min(g, nf2) for g, _ in plan]
            while sum(gpus) > nf2:                     # (only when nf is not a power of two)
                j = max(range(len(gpus)), key=lambda j: gpus[j])
                gpus[j] //= 2
            blocks = sched.place(Tr, ks_r, [q["row"] for q in cand], gpus, prv, nf2, preserve)
            for q, b, (g, n) in zip(cand, blocks, plan):
                if not b:
                    continue
                gids = {free[j] for j in b}
                k = len(gids)
                t_step = T[q["row"], ks.index(k)]
                if k != g:                              # scaled up: more steps fit in the round
                    n = max(n, int(math.floor(tau / t_step + 1e-9)))   # >= 1 step: progress guaranteed
                n = max(1, min(n, q["left"]))
                t = reshard_s(q["row"]) if (q["id"] in prev and prev[q["id"]] != gids) else 0.0
                t += n * t_step
                q["left"] -= n
                busy += k * t
                for g2 in gids:
                    busy_until[g2] = now + t
                running_until[q["id"]] = now + t
                prev[q["id"]] = gids
                ran = True
                if q["left"] == 0:
                    done[q["id"]] = now + t
        live = [q for q in live if q["left"] > 0]
        step = tau
        if not ran and live and all(running_until.get(q["id"], 0.0) <= now + 1e-12 for q in live):
            # nothing ran (every request can still be deferred): skip to the next round in which
            # an arrival happens or some request's latest start (at its fastest degree) is near
            tmin = {q["id"]: min(t for t in T[q["row"]] if t > 0) for q in live}
            wake = min(q["deadline"] - q["left"] * tmin[q["id"]] for q in live) - 2 * tau
            if i < len(pending):
                wake = min(wake, pending[i]["arrival"])
            step = max(step, math.floor((wake - now) / tau) * tau)
        now += step
    return done, busy


def sim_fixed(T, ks, N, reqs, k):
    """FCFS, each request holds k GPUs for all its steps."""
    free_at = [0.0] * (N // k)          # N/k slots of k GPUs
    heapq.heapify(free_at)
    done, busy = {}, 0.0
    for q in sorted(reqs, key=lambda r: r["arrival"]):
        t0 = max(q["arrival"], heapq.heappop(free_at))
        t = q["steps"] * T[q["row"], ks.index(k)]
        done[q["id"]] = t0 + t
        busy += k * t
        heapq.heappush(free_at, t0 + t)
    return done, busy


def sim_rssp(T, ks, N, reqs, degrees):
    """Resolution-specific SP: each resolution has its own fixed degree (profiled offline:
    1 / 1 / 2 / 8 for 256^2 / 512^2 / 1024^2 / 2048^2 in the paper); FCFS, a request starts when its
    degree's worth of GPUs is free (any subset: NVSwitch, S14) and holds them for all its steps."""
    free_at = [0.0] * N
    done, busy = {}, 0.0
    for q in sorted(reqs, key=lambda r: r["arrival"]):
        k = degrees[q["row"]]
        order = sorted(range(N), key=lambda g: free_at[g])[:k]
        t0 = max(q["arrival"], max(free_at[g] for g in order))
        t = q["steps"] * T[q["row"], ks.index(k)]
        for g in order:
            free_at[g] = t0 + t
        done[q["id"]] = t0 + t
        busy += k * t
    return done, busy


def sar(done, reqs, dl):
    ok = sum(1 for q in reqs if done[q["id"]] <= q["arrival"] + dl[RES[q["row"]]] + 1e-9)
    return ok / len(reqs)


def run(T, ks, N=8, n=300, rate=12.0, mix="uniform", scales=(1.0, 1.25, 1.5), seed=0, steps=20, gran=5):
    T = np.asarray(T, dtype=float)
    reqs = workload(n, rate, mix, seed, steps)
    out = []
    for sc in scales:
        dl = deadlines(T, ks, N, steps, sc)
        row = {"mix": mix, "slo_scale": sc, "rate_per_min": round(rate, 3), "n": n}
        d, b = sim_tetriserve(T, ks, N, reqs, dl, gran=gran, preserve=True)
        row["tetriserve"] = round(sar(d, reqs, dl), 4)
        d, b = sim_tetriserve(T, ks, N, reqs, dl, gran=gran, preserve=False)
        row["tetriserve-np"] = round(sar(d, reqs, dl), 4)
        d, b = sim_tetriserve(T, ks, N, reqs, dl, gran=gran, preserve=True, wc=True)
        row["tetriserve-wc"] = round(sar(d, reqs, dl), 4)
        for k in ks:
            d, b = sim_fixed(T, ks, N, reqs, k)
            row[f"fixed-{k}"] = round(sar(d, reqs, dl), 4)
        d, b = sim_rssp(T, ks, N, reqs, [1, 1, 2, 8] if N >= 8 else [1, 1, 2, N])
        row["rssp"] = round(sar(d, reqs, dl), 4)
        out.append(row)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--table", required=True, help="JSON {res: [...], ks: [...], ms: [[...]]}")
    ap.add_argument("--gpus", type=int, default=8)
    ap.add_argument("--n", type=int, default=300)
    ap.add_argument("--rate", type=float, default=12.0, help="requests / min (paper: 12)")
    ap.add_argument("--load", type=float, default=None,
                    help="offered load instead of --rate: rate = load * N / E[S T(res, 1)] (the paper's 12 req/min "
                         "is relative to H100 step times; B200 steps are far shorter)")
    ap.add_argument("--mix", default="both", choices=["uniform", "skewed", "both"])
    ap.add_argument("--slo-scale", type=float, nargs="+", default=[1.0, 1.25, 1.5])
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--gran", type=int, default=5, help="round = gran steps of the largest resolution at k = N (P:562)")
    args = ap.parse_args()
    tab = json.load(open(args.table))
    assert all(r in tab["res"] for r in RES), "the table needs rows 256, 512, 1024, 2048"
    T = np.array([tab["ms"][tab["res"].index(r)] for r in RES], dtype=float) / 1e3
    for mix in (["uniform", "skewed"] if args.mix == "both" else [args.mix]):
        rate = args.rate
        if args.load is not None:
            p = mix_probs(mix)
            rate = args.load * args.gpus / float(np.dot(p, 20 * T[:, 0])) * 60.0
        for row in run(T, tab["ks"], args.gpus, args.n, rate, mix, args.slo_scale, args.seed, gran=args.gran):
            row["load"] = args.load
            row["gran"] = args.gran
            print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
