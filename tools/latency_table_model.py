"""Step-latency table T(res, k) for the serving simulator (tools/serve_sim.py) from ONE GPU.

k = 1: measured (tsv_latency_table, CUDA events, median).  k > 1: the per-rank compute measured
with k virtual ranks on the one device (fused transport: the all-to-alls are epilogue stores plus
an event barrier, so the measured time is the ranks' compute) divided by k, plus a modeled NVLink 5
all-to-all per attention, charged serially (no overlap with compute: conservative for the fused
transport, whose peer stores overlap the epilogues): bytes_r (k - 1) / k / BW + lat, two per block,
BW = 0.8 x 900 GB/s = 720 GB/s per direction and lat = 10 us by default.  The error
bar re-evaluates E(k) at BW = 450 / 900 GB/s and lat = 5 / 20 us.  This is a model for k > 1
(virtual ranks share one GPU's SMs), stated as such in the output; an 8-GPU measurement replaces it.

  python tools/latency_table_model.py [--model flux] [--out profiles/r01/latency_table_model.json]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

RES = [256, 512, 1024, 2048]
KS = [1, 2, 4, 8]


def main():
    import paper_conf_asplos_luhtlwm0c26_b200 as tsv
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="flux")
    ap.add_argument("--iters", type=int, default=5)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02", "latency_table_model.json"))
    ap.add_argument("--res", default=",".join(str(r) for r in RES))
    ap.add_argument("--bw", type=float, default=720.0, help="all-to-all GB/s per direction (model)")
    ap.add_argument("--lat-us", type=float, default=10.0, help="per all-to-all latency (model)")
    ap.add_argument("--serial", action="store_true",
                    help="virtual ranks share one stream (TSV_VIRTUAL_SERIAL=1): each rank's kernels run alone "
                         "on the GPU, so time / k is the per-rank time of a real k-GPU group (minus NVLink)")
    args = ap.parse_args()
    if args.serial:
        os.environ["TSV_VIRTUAL_SERIAL"] = "1"
    res_list = [int(r) for r in args.res.split(",")]
    d = tsv.model_preset(args.model)
    h, Lt = d.hidden, d.text_tokens
    blocks = d.n_double + d.n_single
    B = 2 if d.family == 1 else 1
    eng = tsv.Engine(args.model, devices=[0] * 8)
    ms, cv = eng.latency_table(res_list, KS, warmup=2, iters=args.iters)
    eng.close()
    import importlib.util
    spec = importlib.util.spec_from_file_location("_bench", os.path.join(ROOT, "bench.py"))
    bench = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(bench)
    flops = bench.MODELS[args.model]["flops"]
    peak = bench.peaks()["tflops"] * 1e12
    table = []
    comm = []
    roof = []
    err_lo, err_hi = [], []

    def a2a_ms(Li, k, bw, lat_us):
        rows_r = -(-(Li + Lt) // k)
        bytes_r = B * rows_r * (3 * h + h) * 2 * (k - 1) / k       # a2a #1 (q|k|v) + #2 (o)
        return blocks * (bytes_r / (bw * 1e9) + 2 * lat_us * 1e-6) * 1e3

    for i, r in enumerate(res_list):
        Li = (r // 16) ** 2
        row, crow, lo, hi = [], [], [], []
        for j, k in enumerate(KS):
            if k == 1:
                row.append(float(ms[i, j]))
                crow.append(0.0)
                lo.append(1.0)
                hi.append(1.0)
                continue
            c_ms = a2a_ms(Li, k, args.bw, args.lat_us)
            row.append(float(ms[i, j]) / k + c_ms)
            crow.append(round(c_ms, 4))
            t_worst = float(ms[i, j]) / k + a2a_ms(Li, k, 450.0, 20.0)
            t_best = float(ms[i, j]) / k + a2a_ms(Li, k, 900.0, 5.0)
            lo.append(round(float(ms[i, 0]) / (k * t_worst), 4))
            hi.append(round(float(ms[i, 0]) / (k * t_best), 4))
        table.append([round(x, 4) for x in row])
        comm.append(crow)
        err_lo.append(lo)
        err_hi.append(hi)
        # roofline: per-rank algorithmic GEMM + attention FLOPs at the sustained bf16 peak, plus the
        # modeled all-to-all (the elementwise passes and weight streaming are below 3 % here)
        rrow = []
        for j, k in enumerate(KS):
            g, a = flops(r, k)
            t_roof = (g + a) / peak * 1e3 + crow[j]
            rrow.append(round(t_roof / row[j], 4))
        roof.append(rrow)
    out = {"model": args.model, "res": res_list, "ks": KS, "ms": table, "comm_model_ms": comm,
           "roofline_frac": roof, "roofline_peak_tflops": peak / 1e12,
           "comm_share_model": [[round(c / m, 4) if m > 0 else 0.0 for c, m in zip(cr, mr)] for cr, mr in zip(comm, table)],
           "efficiency_vs_k1": [[round(row[0] / (k * row[j]), 4) for j, k in enumerate(KS)] for row in table],
           "efficiency_range": {"low (450 GB/s, 20 us)": err_lo, "high (900 GB/s, 5 us)": err_hi},
           "a2a_model": {"bw_gbs": args.bw, "lat_us": args.lat_us, "overlap": "none (serial)"},
           "measured_virtual_ms": [[round(float(x), 4) for x in r] for r in ms],
           "measured_cv": [[round(float(x), 5) for x in r] for r in cv],
           "note": "k=1 measured on one B200; k>1 = (k virtual ranks on one B200) / k + modeled NVLink all-to-all"
                   + ("; virtual ranks serialised on one stream (each kernel alone on the GPU, as on a rank's own "
                      "GPU)" if args.serial else "; virtual ranks on concurrent streams (overlap: optimistic for "
                      "small per-rank launches)"),
           "splitk": os.environ.get("TSV_SPLITK", "1") != "0"}
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(out, open(args.out, "w"), indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
