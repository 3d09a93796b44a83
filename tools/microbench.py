"""Kernel micro-benchmarks through the kernel-level C-ABI (CUDA events, warm, L2-resident inputs
unless stated).  Prints one JSON line per case.

  python tools/microbench.py [gemm] [attn] [ln] [qk]
"""
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402


def timeit(fn, iters=20, warm=3):
    for _ in range(warm):
        fn()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    s.record()
    for _ in range(iters):
        fn()
    e.record()
    torch.cuda.synchronize()
    return s.elapsed_time(e) / iters


def gemm_cases():
    # FLUX 512^2 (M = 1024 img / 512 txt / 1536 joint) and 2048^2 k=8 shapes
    shapes = [(1024, 9216, 3072), (512, 9216, 3072), (1024, 3072, 3072), (1024, 12288, 3072), (1024, 3072, 12288),
              (1536, 21504, 3072), (1536, 3072, 15360), (4096, 12288, 3072), (8192, 3072, 12288),
              (1536, 3072, 3072), (1536, 3072, 12288), (2714, 1536, 1536), (2714, 1536, 6144),
              (2714, 4608, 1536), (2714, 6144, 1536), (8858, 1536, 1536), (8858, 4608, 1536), (8858, 1536, 6144),
              (576, 3072, 3072), (576, 9216, 3072), (2112, 3072, 12288)]
    if os.environ.get("GEMM_SHAPES") == "small":
        shapes = shapes[-10:]
    for M, N, K in shapes:
        A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
        W = (torch.randn(N, K, device="cuda") / math.sqrt(K)).to(torch.bfloat16)
        o = torch.empty(M, N, dtype=torch.bfloat16, device="cuda")
        for bn, pair in ((0, -1), (128, 0), (256, 0), (256, 1), (128, 1)):
            if N % (bn or 64):
                continue
            ms = timeit(lambda: tsv.op_gemm(A, W, "STORE_BF16", o, force_bn=bn, force_pair=pair))
            print(json.dumps({"op": "gemm", "M": M, "N": N, "K": K, "bn": bn, "pair": pair, "ms": round(ms, 4),
                              "tflops": round(2 * M * N * K / ms / 1e9, 1)}), flush=True)
        ref = timeit(lambda: torch.matmul(A, W.t(), out=o))
        print(json.dumps({"op": "gemm_cublas_ref", "M": M, "N": N, "K": K, "ms": round(ref, 4),
                          "tflops": round(2 * M * N * K / ref / 1e9, 1)}), flush=True)


def qkv_epilogue_cases():
    """QKV GEMM: plain bf16 store vs the fused QK-RMSNorm + RoPE epilogue (a4) at FLUX shapes."""
    for M in (1536, 16896):
        N, K, h, D = 9216, 3072, 3072, 128
        A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
        W = (torch.randn(N, K, device="cuda") / math.sqrt(K)).to(torch.bfloat16)
        o = torch.empty(M, N, dtype=torch.bfloat16, device="cuda")
        g = torch.ones(D, dtype=torch.bfloat16, device="cuda")
        cs = torch.ones(M, D // 2, device="cuda")
        sn = torch.zeros(M, D // 2, device="cuda")
        plain = timeit(lambda: tsv.op_gemm(A, W, "STORE_BF16", o))
        fused = timeit(lambda: tsv.op_gemm_qkv(A, W, o, h, D, g, g, cs, sn))
        print(json.dumps({"op": "qkv_gemm", "M": M, "plain_ms": round(plain, 4), "fused_ms": round(fused, 4),
                          "plain_tflops": round(2 * M * N * K / plain / 1e9, 1),
                          "fused_tflops": round(2 * M * N * K / fused / 1e9, 1)}), flush=True)


def split_cases():
    # small-M fp32-stream GEMMs (text stream, SP = 4/8 shards): split-K vs one K range
    sem = torch.zeros(4096, dtype=torch.int32, device="cuda")
    ws = torch.empty(64 << 18, dtype=torch.float32, device="cuda")
    for M, N, K in ((64, 3072, 12288), (192, 3072, 12288), (192, 3072, 15360), (576, 3072, 15360),
                    (576, 3072, 3072), (288, 3072, 12288), (333, 1536, 6144), (1024, 3072, 3072)):
        A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
        W = (torch.randn(N, K, device="cuda") / math.sqrt(K)).to(torch.bfloat16)
        x = torch.zeros(M, N, device="cuda")
        g = torch.ones(N, device="cuda")
        res = {}
        for splits in (1, 0):
            res[splits] = timeit(lambda: tsv.op_gemm_split(A, W, "RESID_GATE", x, sem, ws, splits=splits, gate=g))
        if os.environ.get("SPLIT_SWEEP"):
            sw = {s_: round(timeit(lambda: tsv.op_gemm_split(A, W, "RESID_GATE", x, sem, ws, splits=s_, gate=g)), 4)
                  for s_ in (2, 3, 4, 6, 8, 12)}
            one = round(timeit(lambda: tsv.op_gemm(A, W, "RESID_GATE", x, gate=g, force_bn=256, force_pair=0)), 4)
            print(json.dumps({"op": "gemm_split_sweep", "M": M, "N": N, "K": K, "ms_by_splits": sw,
                              "ms_1cta_nosplit": one}), flush=True)
        wbytes = N * K * 2
        print(json.dumps({"op": "gemm_split", "M": M, "N": N, "K": K, "ms_nosplit": round(res[1], 4),
                          "ms_auto": round(res[0], 4), "speedup": round(res[1] / res[0], 2),
                          "tflops_auto": round(2 * M * N * K / res[0] / 1e9, 1),
                          "weight_GBps_auto": round(wbytes / res[0] / 1e6, 1)}), flush=True)


def attn_split_cases():
    # SP = 4/8 head shards (few CTAs): KV split (auto) vs one key range
    cnt = torch.zeros(4096, dtype=torch.int32, device="cuda")
    ws = torch.empty(32 << 20, dtype=torch.float32, device="cuda")
    for L, H, D in ((16896, 3, 128), (16896, 6, 128), (4608, 3, 128), (4608, 6, 128), (1536, 3, 128),
                    (1536, 6, 128), (16717, 3, 64), (4429, 3, 64), (1357, 3, 64)):
        qkv = torch.randn(L, 3 * H * D, device="cuda").to(torch.bfloat16)
        o = torch.empty(L, H * D, dtype=torch.bfloat16, device="cuda")
        ld = 3 * H * D
        res = {}
        for ns in (1, 0):
            f = lambda: tsv.op_attention_split(qkv, qkv[:, H * D:], qkv[:, 2 * H * D:], o, L, H, D, cnt, ws,
                                               nsplit=ns, ldq=ld, ldk=ld, ldv=ld)
            res[ns] = timeit(f, iters=10 if L > 8000 else 30)
        fl = 4 * L * L * D * H
        print(json.dumps({"op": "attention_kv_split", "L": L, "H": H, "D": D, "ms_one": round(res[1], 4),
                          "ms_auto": round(res[0], 4), "speedup": round(res[1] / res[0], 2),
                          "tflops_one": round(fl / res[1] / 1e9, 1), "tflops_auto": round(fl / res[0] / 1e9, 1)}),
              flush=True)


def attn_cases():
    sweep = os.environ.get("ATTN_SWEEP")     # "1": also time the kept exp2 variants
    for L, H, D in ((1536, 24, 128), (4608, 24, 128), (16896, 24, 128), (16896, 3, 128), (1357, 24, 64),
                    (4429, 24, 64), (16717, 24, 64)):
        qkv = torch.randn(L, 3 * H * D, device="cuda").to(torch.bfloat16)
        o = torch.empty(L, H * D, dtype=torch.bfloat16, device="cuda")
        ld = 3 * H * D
        impls = (0,) + ((50, 51, 56, 92, 96, 103) if sweep else ())
        if os.environ.get("ATTN_IMPLS"):
            impls = tuple(int(x) for x in os.environ["ATTN_IMPLS"].split(","))
        impls = tuple(i for i in impls if not (i >= 90 and D != 64))   # RS variants: D = 64 only
        fns = {impl: (lambda impl=impl: tsv.op_attention(qkv, qkv[:, H * D:], qkv[:, 2 * H * D:], o, L, H, D,
                                                         ldq=ld, ldk=ld, ldv=ld, impl=impl)) for impl in impls}
        # interleaved rounds (the box is power-capped: clocks drift over a run), median per impl
        times = {impl: [] for impl in impls}
        for _ in range(int(os.environ.get("ATTN_ROUNDS", "3"))):
            for impl in impls:
                times[impl].append(timeit(fns[impl], iters=5 if L > 8000 else 20))
        for impl in impls:
            ms = sorted(times[impl])[len(times[impl]) // 2]
            name = "tcgen05" if impl == 0 else f"tcgen05-impl{impl}"
            print(json.dumps({"op": "attention", "impl": name, "L": L, "H": H, "D": D,
                              "ms": round(ms, 4), "tflops": round(4 * L * L * D * H / ms / 1e9, 1),
                              "all_ms": [round(t, 4) for t in times[impl]]}), flush=True)


def ln_cases():
    for M, h in ((1024, 3072), (1536, 3072), (16896, 3072), (2714, 1536), (8858, 1536)):
        x = torch.randn(M, h, device="cuda")
        u = torch.empty(M, h, dtype=torch.bfloat16, device="cuda")
        sh, sc = torch.randn(h, device="cuda"), torch.randn(h, device="cuda")
        for impl in (0, 1, 2):
            ms = timeit(lambda: tsv.op_ln_mod(x, u, sh, sc, impl=impl))
            print(json.dumps({"op": "ln_mod", "impl": ["cta_per_row", "warp_per_row", "persistent_rows"][impl], "M": M, "h": h,
                              "ms": round(ms, 4), "GBps": round(M * h * 6 / ms / 1e6, 1)}), flush=True)


def qk_cases():
    for rows, H, D in ((1536, 24, 128), (16896, 24, 128)):
        qkv = torch.randn(rows, 3 * H * D, device="cuda").to(torch.bfloat16)
        g = torch.ones(D, device="cuda").to(torch.bfloat16)
        cs = torch.randn(rows, D // 2, device="cuda")
        ms = timeit(lambda: tsv.op_qk_norm_rope(qkv, 0, H, D, g, g, g, g, cs, cs))
        print(json.dumps({"op": "qk_norm_rope", "rows": rows, "ms": round(ms, 4),
                          "GBps": round(rows * H * D * 8 / ms / 1e6, 1)}), flush=True)


if __name__ == "__main__":
    which = sys.argv[1:] or ["gemm", "attn", "ln", "qk"]
    for w in which:
        {"gemm": gemm_cases, "split": split_cases, "attnsplit": attn_split_cases, "attn": attn_cases, "ln": ln_cases, "qk": qk_cases, "qkv": qkv_epilogue_cases}[w]()
