"""Benchmark: one FLUX.1-dev-shaped denoising step (the whole hot path, S:§8(a) a1-a12) under
step-level Ulysses SP, through libtsv.so's C-ABI.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--res 2048] [--model flux|sd3] [--impl ours|reference]

N = 1: the north-star configuration (BASELINE.json north_star: "a FLUX.1-dev-shaped 2048^2
denoising step ... at SP=1"; BASELINE config 4's resolution, 16 384 image + 512 text tokens).
--res 512 gives config 2's line.  N > 1 (torchrun, one process per GPU): the same request at SP = N
on ranks [0..N) (strong scaling: the step's work is fixed); all-to-alls fused into the epilogues
over CUDA-IPC peer memory (default) or NCCL send/recv; a second profiled pass on the NCCL exchange
transport gives the communication share and the all-to-all bus GB/s.  Metric: step latency (ms,
lower is better), CUDA events on the engine's stream around K graph replays, max over ranks; the
per-step latencies give the CV.  Inputs are larger than L2 (23.7 GB of weights
streamed per step), so no L2 flush is needed between timed steps.

--model sd3: the SD3-medium-shaped CFG step of config 5 (24 joint blocks, L_t = 333, batch-2 CFG
pair) instead of FLUX (a secondary line).

--impl reference: the float64 CPU oracle on the box's host cores (the tier's reference arm), timed
on a bounded sample of the same step and extrapolated (see oracle_sample).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "DiT step latency (ms) per resolution at SP=1/2/4/8; attn+GEMM TFLOP/s vs peak"


def ncu_traffic(res: int, pattern: str, model: str = "flux"):
    """Mean DRAM bytes (read + write) per launch of kernels whose name contains `pattern`, from the
    newest committed ncu launch list of one step at this resolution (profiles/rNN/launches_<res>.csv,
    SD3: launches_sd3<res>.csv), or None."""
    import csv
    import glob
    tag = f"sd3{res}" if model == "sd3" else f"{res}"
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*", f"launches_{tag}.csv")))
    if not files:
        return None
    rows = list(csv.reader(open(files[-1])))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ii, ki, mi, vi, ui = (h.index(c) for c in ("ID", "Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    per = {}
    for r in rows[hi + 1:]:
        if len(r) > vi and pattern in r[ki] and r[mi].startswith("dram__bytes"):
            per[r[ii]] = per.get(r[ii], 0.0) + float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
    if not per:
        return None
    return {"bytes_per_launch": round(sum(per.values()) / len(per)), "launches": len(per),
            "source": os.path.relpath(files[-1], ROOT) + " (ncu, cold cache)"}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return dict(tflops=d["bf16_tflops_sustained"], tflops_burst=d["bf16_tflops"], hbm=d["hbm_gbs"],
                    source="measured (MEASURED_PEAKS.json)")
    return dict(tflops=1400.0, tflops_burst=1590.0, hbm=6650.0, source="fallback (B200_PROFILING.md)")


# --------------------------------------------------------------------------- FLOP model (per rank)
def flux_flops(res: int, k: int = 1, Lt: int = 512, h=3072, F=12288, H=24, D=128, nd=19, ns=38, inch=64, ctx=4096):
    Li = (res // 16) ** 2
    lt, li = -(-Lt // k), -(-Li // k)        # largest shard (rank 0)
    L = Lt + Li
    rows = lt + li
    gemm = 2 * li * inch * h + 2 * lt * ctx * h
    gemm += nd * 2 * rows * h * (3 * h + h + 2 * F)
    gemm += ns * (2 * rows * h * (3 * h + F) + 2 * rows * (h + F) * h)
    gemm += 2 * li * h * inch
    attn = (nd + ns) * 4 * L * L * D * (H // k)
    return gemm, attn


def sd3_flops(res: int, k: int = 1, Lt: int = 333, h=1536, F=6144, H=24, D=64, nd=24, inch=64, ctx=4096, B=2):
    """SD3 CFG step per rank: B = 2 evaluations; the last block's txt stream stops at its QKV."""
    Li = (res // 16) ** 2
    lt, li = -(-Lt // k), -(-Li // k)
    L = Lt + Li
    gemm = 2 * li * inch * h + B * 2 * lt * ctx * h
    per_stream = h * (3 * h + h + 2 * F)
    gemm += B * (nd * 2 * li * per_stream + (nd - 1) * 2 * lt * per_stream + 2 * lt * h * 3 * h)
    gemm += B * 2 * li * h * inch
    attn = B * nd * 4 * L * L * D * (H // k)
    return gemm, attn


MODELS = {
    "flux": dict(Lt=512, flops=flux_flops, desc="FLUX.1-dev-shaped denoising step", shapes="FLUX.1-dev shapes",
                 weights_gb=23.7),
    "sd3": dict(Lt=333, flops=sd3_flops, desc="SD3-medium-shaped CFG denoising step (batch-2 CFG pair)",
                shapes="SD3-medium shapes", weights_gb=4.2),
}


# --------------------------------------------------------------------------- clocks sampler
class Clocks:
    def __init__(self, gpu: int):
        self.gpu = gpu
        self.samples = []
        self.stop = threading.Event()
        self.proc = None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            threading.Thread(target=self._read, daemon=True).start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if len(s) > 2 + i and s[2 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


# --------------------------------------------------------------------------- oracle (reference / cpu_baseline)
SAMPLE_ROWS = 1024   # query / token rows of the bounded oracle sample at L > 4096 (~10-20 s of host work)


def oracle_sample(res: int):
    """The float64 oracle (oracle/flux.py, as it stands) timed on a bounded sample of one FLUX step
    and extrapolated.  Weights and inputs are generated first (input synthesis, untimed).
      * L <= 4096 (512^2, 256^2): embed + one double block + one single block + final at full width,
        x 19 / x 38 for the blocks.
      * larger L (1024^2 and up): the oracle's per-row work of one double and one single block on
        n = SAMPLE_ROWS rows -- LN-modulate, the QKV / out / MLP GEMMs, QK-RMSNorm, RoPE, and softmax
        attention of the n query rows against all L keys -- scaled by L / n, then x 19 / x 38.  Every
        op is row-local except attention, whose cost is linear in the query rows for fixed keys, so
        the scaling is exact up to cache effects.
    Returns (ms, detail)."""
    import numpy as np
    from oracle import flux as F
    from oracle.config import FLUX
    from oracle.weights import Weights, request_inputs
    cfg = FLUX
    h, H, D = cfg.hidden, cfg.heads, cfg.head_dim
    W = Weights(cfg, cache_bytes=8 << 30)
    x, T, y = request_inputs(cfg, res, res, 1000)
    Li, Lt = x.shape[0], T.shape[0]
    L = Li + Lt
    for nme in W.table:  # generate the sampled blocks' weights up front (input synthesis, untimed)
        if nme.startswith(("double0.", "single0.", "img_in", "txt_in", "final", "time_in", "guidance_in", "vector_in")):
            W[nme]
    rng = np.random.default_rng(0)
    vec = F.conditioning_vec(cfg, W, 0.5, y, 3.5)
    cores = len(os.sched_getaffinity(0))
    if L <= 4096:
        img = rng.standard_normal((Li, h))
        txt = rng.standard_normal((Lt, h))
        ang = F.rope_angles(F.position_ids(Lt, res, res), cfg.axes_dim, cfg.theta)
        t0 = time.perf_counter()
        F.linear(x, W["img_in.w"], W["img_in.b"])
        F.linear(T, W["txt_in.w"], W["txt_in.b"])
        t1 = time.perf_counter()
        F.double_block(cfg, W, 0, img, txt, vec, ang)
        t2 = time.perf_counter()
        F.single_block(cfg, W, 0, np.concatenate([txt, img]), vec, ang)
        t3 = time.perf_counter()
        F.final_layer(W, img, vec)
        t4 = time.perf_counter()
        ms = ((t1 - t0) + cfg.n_double * (t2 - t1) + cfg.n_single * (t3 - t2) + (t4 - t3)) * 1e3
        return ms, dict(kind="oracle", cores=cores, extrapolated=True,
                        sample=f"float64 numpy oracle: embed + 1 double + 1 single block + final of FLUX {res}x{res} "
                               f"(L={L}) at full width, x19 / x38 blocks; weights pre-generated (untimed); "
                               f"BLAS threads = {cores}")
    n = SAMPLE_ROWS
    u = rng.standard_normal((n, h))
    k_all = rng.standard_normal((L, H, D))   # the keys / values every sampled query row attends to
    v_all = rng.standard_normal((L, H, D))
    ang = F.rope_angles(F.position_ids(Lt, res, res), cfg.axes_dim, cfg.theta)[:n]

    def qk_rope(qkv, p):
        q, k, v = F.split_qkv(qkv, H, D)
        return F.apply_rope(F.rms_norm(q, W[p + "q_norm.g"]), ang), F.apply_rope(F.rms_norm(k, W[p + "k_norm.g"]), ang), v

    t0 = time.perf_counter()   # one double block's per-row work (the img stream's weights for both streams)
    p = "double0.img."
    sh1, sc1, g1, sh2, sc2, g2 = F.modulation(W, p, vec, 6)
    q, _, _ = qk_rope(F.linear(F.ln_modulate(u, sh1, sc1), W[p + "qkv.w"], W[p + "qkv.b"]), p)
    o = F.attention(q, k_all, v_all)
    xr = u + g1 * F.linear(o.reshape(n, h), W[p + "proj.w"], W[p + "proj.b"])
    xr = xr + g2 * F.linear(F.gelu_tanh(F.linear(F.ln_modulate(xr, sh2, sc2), W[p + "fc1.w"], W[p + "fc1.b"])),
                            W[p + "fc2.w"], W[p + "fc2.b"])
    t1 = time.perf_counter()   # one single block's per-row work
    p = "single0."
    sh, sc, g = F.modulation(W, p, vec, 3)
    y1 = F.linear(F.ln_modulate(u, sh, sc), W[p + "lin1.w"], W[p + "lin1.b"])
    q, _, _ = qk_rope(y1[:, :3 * h], p)
    o = F.attention(q, k_all, v_all).reshape(n, h)
    xs = u + g * F.linear(np.concatenate([o, F.gelu_tanh(y1[:, 3 * h:])], axis=1), W[p + "lin2.w"], W[p + "lin2.b"])
    t2 = time.perf_counter()
    ms = (L / n) * (cfg.n_double * (t1 - t0) + cfg.n_single * (t2 - t1)) * 1e3
    return ms, dict(kind="oracle", cores=cores, extrapolated=True,
                    sample=f"float64 numpy oracle (oracle/flux.py ops as they stand): the per-row work of one double "
                           f"and one single block of FLUX {res}x{res} (L={L}) on {n} token rows -- LN-modulate, "
                           f"QKV/out/MLP GEMMs, QK-RMSNorm, RoPE, softmax attention of {n} queries over all {L} keys "
                           f"-- scaled by L/{n} and x19 / x38 blocks (embed/final < 0.1 % omitted); weights "
                           f"pre-generated (untimed); BLAS threads = {cores}")


def oracle_sample_sd3(res: int):
    """SD3: embed + joint block 0 + final of one CFG branch at full width, extrapolated to 24
    joint blocks x 2 branches (weights pre-generated, not timed)."""
    import numpy as np  # noqa: F401
    from oracle import flux as F
    from oracle import sd3 as S3
    from oracle.config import SD3
    from oracle.weights import Weights, sd3_request_inputs
    cfg = SD3
    W = Weights(cfg, cache_bytes=8 << 30)
    x, Tc, yc, _, _ = sd3_request_inputs(cfg, res, res, 1000)
    Li, Lt = x.shape[0], Tc.shape[0]
    for n in W.table:
        if n.startswith(("joint0.", "img_in", "txt_in", "final", "time_in", "vector_in")):
            W[n]
    vec = S3.conditioning_vec(cfg, W, 0.5, yc)
    t0 = time.perf_counter()
    img = F.linear(x, W["img_in.w"], W["img_in.b"]) + S3.pos_embed(cfg, res // 16, res // 16)
    txt = F.linear(Tc, W["txt_in.w"], W["txt_in.b"])
    t1 = time.perf_counter()
    S3.joint_block(cfg, W, 0, img, txt, vec)
    t2 = time.perf_counter()
    S3.final_layer(W, img, vec)
    t3 = time.perf_counter()
    ms = 2 * ((t1 - t0) + cfg.n_double * (t2 - t1) + (t3 - t2)) * 1e3
    cores = len(os.sched_getaffinity(0))
    return ms, dict(kind="oracle", cores=cores, extrapolated=True,
                    sample=f"float64 numpy oracle: embed + joint block 0 + final of one CFG branch of SD3 "
                           f"{res}x{res} (L={Li + Lt}) at full width, extrapolated to 24 blocks x 2 branches; "
                           f"weights pre-generated (untimed); BLAS threads = {cores}")


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    res = args.res
    mdl = MODELS[args.model]
    ms_list = []
    sample = oracle_sample_sd3 if args.model == "sd3" else oracle_sample
    # each step is a bounded sample (~1-2 min of host BLAS at 512^2): at most 1 warm-up and 2 timed
    # samples keep the whole reference run within a few minutes
    warm = min(args.warmup, 1)
    steps = max(1, min(args.steps, 2))
    for _ in range(warm):
        sample(res)
    for _ in range(steps):
        ms, detail = sample(res)
        ms_list.append(ms)
    ms = statistics.median(ms_list)
    detail["value"] = ms
    detail["unit"] = "ms"
    line = {"impl": "reference", "metric": METRIC, "value": ms, "unit": "ms", "n_gpus": args.gpus,
            "steps": steps, "warmup": warm, "ms_per_step": ms, "higher_is_better": False, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic (SYNTH-1 seeded weights and inputs)",
            "config": {"workload": f"{mdl['desc']} {res}x{res} ({(res // 16) ** 2} image + {mdl['Lt']} text tokens)",
                       "sp": 1, "resolution": res},
            "cpu_baseline": detail,
            "e2e": {"value": ms, "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------------- our arm
NOMINAL_DENSE_BF16 = 2250.0   # TFLOP/s per B200 at the 1965 MHz boost clock (B200_PROFILING.md)


def roofline_entry(kind, prof_cls, pk, sm_mhz, traffic, kernel):
    """Roofline of one kernel class from the profiled pass: achieved = algorithmic FLOPs per launch /
    mean device time per launch; peak = the measured sustained bf16 peak (MEASURED_PEAKS.json);
    tensor_util_clock = achieved / (nominal dense peak x in-run SM clock / boost clock), the
    clock-relative tensor-pipe utilisation the north star names."""
    n = prof_cls["launches"]
    if not n or not prof_cls["ms"]:
        return None
    t = prof_cls["ms"] / n * 1e-3
    fl = prof_cls["flops"] / n
    by = prof_cls["bytes"] / n
    achieved = fl / t / 1e12
    at_clock = NOMINAL_DENSE_BF16 * (sm_mhz / 1965.0) if sm_mhz else None
    return {"bound": "tensor", "kernel": kernel, "achieved": round(achieved, 2), "peak": pk["tflops"],
            "unit": "TFLOP/s", "frac": round(achieved / pk["tflops"], 4),
            "traffic": traffic["bytes_per_launch"] if traffic else None, "traffic_detail": traffic,
            "algorithmic_flops_per_launch": round(fl), "algorithmic_bytes_per_launch": round(by),
            "launches_per_step": n // 2, "us_per_launch": round(t * 1e6, 2),
            "tensor_util_clock": round(achieved / at_clock, 4) if at_clock else None,
            "peak_source": pk["source"] + " bf16_tflops_sustained"}


def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_asplos_luhtlwm0c26_b200 as tsv

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    # TSV_BENCH_ONE_GPU=1 (tests only): every rank on device 0, gloo for the host-side collectives and
    # the fused CUDA-IPC transport for the step (NCCL refuses two ranks on one GPU) -- exercises the
    # N > 1 code path of this script on a one-GPU box; the numbers are not a scaling measurement
    one_gpu = os.environ.get("TSV_BENCH_ONE_GPU") == "1" and world > 1
    local = 0 if one_gpu else local
    red_dev = "cpu" if one_gpu else "cuda"
    torch.cuda.set_device(local)
    if world > 1:
        if one_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    mdl = MODELS[args.model]
    res = args.res
    Li = (res // 16) ** 2
    eng = tsv.Engine(args.model, devices=[local], rank_base=rank, world_size=world)
    has_nccl_group = False
    if one_gpu:
        g = eng.group_create(list(range(world)))
        blob = eng.group_ipc_export(g, max_tokens=Li + mdl["Lt"], max_evals=2)
        blobs = [None] * world
        dist.all_gather_object(blobs, blob)
        eng.group_ipc_import(g, blobs)
        eng.set_transport(True)
        transport = "fused-ipc (one GPU, test mode)"
    elif world > 1:
        obj = [tsv.nccl_unique_id() if rank == 0 else None, tsv.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        eng.init_world(obj[0])
        g = eng.group_create(list(range(world)), nccl_id=obj[1])
        has_nccl_group = True
        transport = "nccl-exchange"
        if args.transport == "fused":
            # the product path: all-to-alls fused into the epilogues as stores into the other
            # processes' CUDA-IPC windows (tsv_group_ipc_export / _import); NCCL stays the fallback
            try:
                blob = eng.group_ipc_export(g, max_tokens=Li + mdl["Lt"], max_evals=2)
                blobs = [None] * world
                dist.all_gather_object(blobs, blob)
                eng.group_ipc_import(g, blobs)
                eng.set_transport(True)
                transport = "fused-ipc"
            except tsv.TsvError as ex:
                print(f"[bench] fused IPC transport unavailable ({ex}); using NCCL", file=sys.stderr)
                eng.set_transport(False)
        else:
            eng.set_transport(False)
    else:
        g = eng.group_create([0])
        transport = "none"
    K, Wm = args.steps, args.warmup
    total_steps = Wm + K + 2 + 2 + K + 1   # warm-up + timed + profiled + NCCL-profiled + e2e passes
    req = eng.request_create(res, res, num_steps=total_steps, seed=1000)
    step = 0

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=red_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    for _ in range(Wm):
        eng.request_step(req, step, g)
        step += 1
    barrier()
    kc0 = eng.kernel_count()
    with Clocks(local) as clk:
        barrier()
        evs = [eng.group_record(g)]
        for _ in range(K):
            eng.request_step(req, step, g)
            step += 1
            evs.append(eng.group_record(g))
        total_ms = eng.event_elapsed_ms(evs[0], evs[-1])
        barrier()
    launches = eng.kernel_count() - kc0
    per_step = [eng.event_elapsed_ms(evs[i], evs[i + 1]) for i in range(K)]
    ms = max_over_ranks(total_ms / K)
    mean = statistics.fmean(per_step)
    cv = max_over_ranks(statistics.stdev(per_step) / mean if K > 1 else 0.0)
    median_ms = max_over_ranks(statistics.median(per_step))
    clocks = clk.summary()

    # per-kernel-class device time (a separate profiled pass: events around every launch)
    def profiled(n=2):
        nonlocal step
        eng.profile(True)
        for _ in range(n):
            eng.request_step(req, step, g)
            step += 1
        pr = eng.profile_read()
        eng.profile(False)
        return pr
    prof = profiled()

    # N > 1: the same step on the NCCL exchange transport, profiled: the all-to-alls are then separate
    # NCCL calls whose device time and bytes give the communication share (Fig. 2 analogue)
    # and the all-to-all bus bandwidth ((k-1)/k of each rank's send buffer / time, nccl-tests busbw)
    comm = None
    if world > 1:
        a2a_fused_ms = prof["a2a"]["ms"] / 2
        comm = {"transport": transport, "barrier_ms_per_step": round(max_over_ranks(a2a_fused_ms), 4),
                "barrier_share": round(max_over_ranks(a2a_fused_ms) / ms, 4)}
        if has_nccl_group and transport.startswith("fused"):
            eng.set_transport(False)
            pn = profiled()
            eng.set_transport(True)
            a2a_ms = pn["a2a"]["ms"] / 2
            step_ms = sum(v["ms"] for v in pn.values()) / 2
            comm["nccl_exchange"] = {
                "a2a_ms_per_step": round(max_over_ranks(a2a_ms), 4),
                "a2a_share": round(max_over_ranks(a2a_ms / step_ms), 4),
                "bus_gbs": round(pn["a2a"]["bytes"] / 2 / (a2a_ms * 1e-3) / 1e9, 1) if a2a_ms else None,
                "bus_peak_gbs": 900.0,
                "calls_per_step": pn["a2a"]["launches"] // 2}

    # end to end through the public API with host buffers: H2D latent in, step, D2H latent out
    r0, r1 = tsv.shard_range(Li, world, rank)
    # pinned host buffer (the contract's "host->device copy from pinned host memory")
    host = torch.empty((r1 - r0, 64), dtype=torch.float32, pin_memory=True).numpy()
    host[:] = eng.read_latent(req, r0, r1 - r0)
    barrier()
    e2e_times = []
    for i in range(K + 1):
        t0 = time.perf_counter()
        eng.write_latent(req, host, r0)
        eng.request_step(req, step, g)
        step += 1
        eng.read_latent(req, r0, r1 - r0, out=host)
        if world > 1:
            dist.barrier()
        if i:
            e2e_times.append((time.perf_counter() - t0) * 1e3)
    e2e_ms = max_over_ranks(statistics.median(e2e_times))

    pk = peaks()
    sm = clocks.get("sm_mhz")
    gemm_fl, attn_fl = mdl["flops"](res, world)
    step_prof_ms = sum(v["ms"] for v in prof.values()) / 2
    shares = {c: round(v["ms"] / 2 / step_prof_ms, 4) for c, v in prof.items()} if step_prof_ms else {}
    step_tf = (gemm_fl + attn_fl) / (ms * 1e-3) / 1e12
    one = world == 1
    rl = {
        "gemm": roofline_entry("gemm", prof["gemm"], pk, sm,
                               ncu_traffic(res, "gemm", args.model) if one else None,
                               "gemm_tc2_kernel / gemm_tc_kernel (tcgen05 GEMM, all GEMM launches of the step)"),
        "attention": roofline_entry("attention", prof["attention"], pk, sm,
                                    ncu_traffic(res, "attention", args.model) if one else None,
                                    "attention_fa_kernel (tcgen05/TMEM joint attention)"),
    }
    dominant = max(("gemm", "attention"), key=lambda c: prof[c]["ms"])

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(ms, 4), "unit": "ms", "n_gpus": world, "steps": K, "warmup": Wm,
            "ms_per_step": round(ms, 4), "higher_is_better": False, "scaling": "strong", "vs_baseline": None,
            "dtype": "bf16", "data": f"synthetic (SYNTH-1 seeded weights and inputs, {mdl['shapes']})",
            "config": {"workload": f"{mdl['desc']} {res}x{res} ({Li} image + {mdl['Lt']} text tokens)",
                       "sp": world, "resolution": res, "global_batch": 1, "seq_len": Li + mdl["Lt"],
                       "parallelism": f"ulysses-sp{world}", "transport": transport,
                       "l2": f"inputs larger than L2 ({mdl['weights_gb']} GB of weights streamed per step); no flush"},
            "roofline": dict(rl[dominant], dominant_share=shares.get(dominant)),
            "roofline_kernels": rl,
            "step_tflops": round(step_tf, 2),
            "step_tensor_util": {"vs_sustained_peak": round(step_tf / pk["tflops"], 4),
                                 "clock_relative": round(step_tf / (NOMINAL_DENSE_BF16 * sm / 1965.0), 4) if sm else None,
                                 "note": "algorithmic step FLOPs / step time; clock_relative against 2.25 PF x "
                                         "in-run SM clock / 1965 MHz (ncu tensor-pipe %: profiles/)"},
            "latency": {"median_ms": round(median_ms, 4), "cv": round(cv, 5), "steps": K},
            "time_share": shares,
            "e2e": {"value": round(e2e_ms, 4), "unit": "ms", "h2d_bytes_per_step": int(host.nbytes),
                    "d2h_bytes_per_step": int(host.nbytes)},
            "gpu_launches": int(launches),
            "clocks": clocks,
        }
        if comm:
            line["comm"] = comm
        if world == 1 and not args.no_cpu_baseline:
            ms_cpu, detail = (oracle_sample_sd3 if args.model == "sd3" else oracle_sample)(res)
            detail["value"] = round(ms_cpu, 1)
            detail["unit"] = "ms"
            line["cpu_baseline"] = detail
        print(json.dumps(line), flush=True)
    eng.close()
    if world > 1:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--res", type=int, default=2048)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--model", default="flux", choices=sorted(MODELS))
    ap.add_argument("--transport", default="fused", choices=["fused", "nccl"],
                    help="N > 1: Ulysses all-to-alls fused into the epilogues over CUDA-IPC peer memory (default) "
                         "or NCCL send/recv")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
