"""Summarise ncu output kept under gpurun_out/ (or profiles/): per-kernel-class share of a step from
a launch list (--metrics gpu__time_duration.sum --csv) and key counters from --set full reports.

  python tools/ncu_summary.py launches <launches.csv>
  python tools/ncu_summary.py report <file.ncu-rep> [...]
"""
import collections
import csv
import io
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__cycles_elapsed.avg.per_second", "sm clock"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram % peak"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe % (active)"),
    ("sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor mem % (active)"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "XU (MUFU) pipe %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("launch__registers_per_thread", "registers"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smem bank conflicts"),
]


def classify(name):
    n = name.split("(")[0]
    for key, cls in (("gemm_tc2", "gemm (CTA pair)"), ("gemm_tc", "gemm"), ("attention", "attention"),
                     ("ln_mod", "ln_mod"), ("qk_norm", "qk_norm_rope"), ("copy2d", "a2a unpack"),
                     ("f32_to_bf16", "cast")):
        if key in n:
            return cls
    return n


def launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h, data = rows[hi], rows[hi + 1:]
    ii, ki, mi, vi, ui = (h.index(c) for c in ("ID", "Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    recs = collections.defaultdict(dict)
    for r in data:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        unit = r[ui]
        v *= {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3,
              "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1.0)
        recs[r[ii]]["name"] = r[ki]
        recs[r[ii]][r[mi]] = v
    tot, cnt, dram = collections.defaultdict(float), collections.Counter(), collections.defaultdict(float)
    for rec in recs.values():
        c = classify(rec["name"])
        tot[c] += rec.get("gpu__time_duration.sum", 0.0)
        dram[c] += rec.get("dram__bytes_read.sum", 0.0) + rec.get("dram__bytes_write.sum", 0.0)
        cnt[c] += 1
    s = sum(tot.values())
    print(f"{'class':24s} {'launches':>8s} {'us':>12s} {'share':>7s} {'DRAM MB/launch':>15s}")
    for k, v in sorted(tot.items(), key=lambda x: -x[1]):
        print(f"{k:24s} {cnt[k]:8d} {v:12.1f} {100 * v / s:6.1f}% {dram[k] / cnt[k] / 1e6:15.2f}")
    print(f"{'total (serialised, cold)':24s} {sum(cnt.values()):8d} {s:12.1f}")
    return tot, cnt, dram


def report(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    for r in rows[2:]:
        print(f"== {path}: {r[h.index('Kernel Name')][:90]}")
        for key, label in KEYS:
            if key in h:
                i = h.index(key)
                print(f"   {label:26s} {r[i]} {units[i]}")


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2])
    else:
        for p in sys.argv[2:]:
            report(p)
