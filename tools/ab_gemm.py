"""Same-box GEMM A/B helper: times the step's GEMM shapes at 512^2 (auto plan) for each epilogue
mode through op_gemm of whichever tree's package is imported (run from that tree's root)."""
import json
import math
import os
import sys

sys.path.insert(0, os.getcwd())
import torch  # noqa: E402

import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402


def timeit(fn, iters=30, warm=5):
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


tag = sys.argv[1] if len(sys.argv) > 1 else "?"
for M, N, K, mode in ((1536, 21504, 3072, "STORE_BF16"), (1536, 3072, 15360, "RESID_GATE"), (1024, 12288, 3072, "GELU_BF16"),
                      (1024, 3072, 12288, "RESID_GATE"), (1024, 3072, 3072, "RESID_GATE"), (1024, 9216, 3072, "STORE_BF16"),
                      (4096, 12288, 3072, "GELU_BF16"), (4096, 3072, 12288, "RESID_GATE")):
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    W = (torch.randn(N, K, device="cuda") / math.sqrt(K)).to(torch.bfloat16)
    if mode == "RESID_GATE":
        o = torch.zeros(M, N, device="cuda")
        g = torch.ones(N, device="cuda")
        f = lambda: tsv.op_gemm(A, W, mode, o, gate=g)
    else:
        o = torch.empty(M, N, dtype=torch.bfloat16, device="cuda")
        f = lambda: tsv.op_gemm(A, W, mode, o)
    ms = min(timeit(f) for _ in range(3))
    print(json.dumps({"tree": tag, "M": M, "N": N, "K": K, "mode": mode, "ms": round(ms, 4),
                      "tflops": round(2 * M * N * K / ms / 1e9, 1)}), flush=True)
