"""Write tests/golden/*.npz from the float64 oracle ONLY (no CUDA path involved).

flux512_seed1000_S1.npz: FLUX.1-dev-shaped step at 512x512, request seed 1000, guidance 3.5,
S = 1 (t_0 = 1 -> t_1 = 0), weights SYNTH-1 seed 0x7E7125E7.  Keys: v, x_next (float64).
Runtime: several minutes on 8 cores (12 B synthetic parameters + ~21 TFLOP of fp64).
"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import flux as F  # noqa: E402
from oracle.config import FLUX  # noqa: E402
from oracle.weights import Weights, request_inputs  # noqa: E402


def main():
    t0 = time.time()
    x, T, y = request_inputs(FLUX, 512, 512, 1000)
    W = Weights(FLUX, cache_bytes=0)
    v, xn = F.request_step(FLUX, W, x, T, y, 0, 1, 3.5, 512, 512)
    out = os.path.join(ROOT, "tests", "golden", "flux512_seed1000_S1.npz")
    np.savez_compressed(out, v=v, x_next=xn)
    print(f"wrote {out} in {time.time() - t0:.1f} s; |v|max={np.abs(v).max():.4f}")


if __name__ == "__main__":
    main()
