"""Write tests/golden/*.npz from the float64 oracle ONLY (no CUDA path involved).

flux512_seed1000_S1.npz: FLUX.1-dev-shaped step at 512x512, request seed 1000, guidance 3.5,
S = 1 (t_0 = 1 -> t_1 = 0), weights SYNTH-1 seed 0x7E7125E7.  Keys: v, x_next (float64).
Runtime: several minutes on 8 cores (12 B synthetic parameters + ~21 TFLOP of fp64).

sd3_512_seed1000_S20.npz: SD3-medium-shaped CFG step 0 of S = 20 at 512x512 (t_0 = 1 ->
t_1 = shift(0.95)), request seed 1000 (inputs ids 1-5), same weight seed.  Keys: v, x_next.

flux2048_seed1000_S20_step0.npz: the north-star configuration (BASELINE.json north_star, SURVEY
§8(d) config 4 "against the oracle at step 0"): FLUX.1-dev-shaped step 0 of S = 20 at 2048x2048
(L_i = 16 384 image + 512 text tokens), request seed 1000, guidance 3.5, same weight seed.  Keys:
v, x_next stored as float32 (the oracle computes in float64; float32 storage keeps the file at
8 MB and its rounding, 2^-24 relative, is far below the 2e-2 tolerance).  Runtime: ~1.5-2 h on
8 cores (~418 TFLOP of fp64 plus 3.9e11 exponentials).

flux1024_seed1000_S20_step0.npz: BASELINE config 3's resolution (1024x1024 = 4096 image + 512
text tokens), step 0 of S = 20, float32 storage as above (~20 min).
sd3_1024_seed1000_S20.npz: SD3-medium CFG step 0 of S = 20 at 1024x1024 (config 5's 1024^2
request), float32 storage.

Usage: python tools/make_golden.py [flux|sd3|flux2048|flux1024|sd3_1024 ...]   (default: flux sd3)
"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import flux as F  # noqa: E402
from oracle import sd3 as S3  # noqa: E402
from oracle.config import FLUX, SD3  # noqa: E402
from oracle.weights import Weights, request_inputs, sd3_request_inputs  # noqa: E402


def sd3():
    t0 = time.time()
    x, Tc, yc, Tu, yu = sd3_request_inputs(SD3, 512, 512, 1000)
    W = Weights(SD3, cache_bytes=20 << 30)     # 2 B parameters: keep them for the second branch
    v, xn = S3.request_step(SD3, W, x, Tc, yc, Tu, yu, 0, 20, 512, 512)
    out = os.path.join(ROOT, "tests", "golden", "sd3_512_seed1000_S20.npz")
    np.savez_compressed(out, v=v, x_next=xn)
    print(f"wrote {out} in {time.time() - t0:.1f} s; |v|max={np.abs(v).max():.4f}")


def flux():
    t0 = time.time()
    x, T, y = request_inputs(FLUX, 512, 512, 1000)
    W = Weights(FLUX, cache_bytes=0)
    v, xn = F.request_step(FLUX, W, x, T, y, 0, 1, 3.5, 512, 512)
    out = os.path.join(ROOT, "tests", "golden", "flux512_seed1000_S1.npz")
    np.savez_compressed(out, v=v, x_next=xn)
    print(f"wrote {out} in {time.time() - t0:.1f} s; |v|max={np.abs(v).max():.4f}")


def flux2048():
    t0 = time.time()
    x, T, y = request_inputs(FLUX, 2048, 2048, 1000)
    W = Weights(FLUX, cache_bytes=0)
    v, xn = F.request_step(FLUX, W, x, T, y, 0, 20, 3.5, 2048, 2048)
    out = os.path.join(ROOT, "tests", "golden", "flux2048_seed1000_S20_step0.npz")
    np.savez_compressed(out, v=v.astype(np.float32), x_next=xn.astype(np.float32))
    print(f"wrote {out} in {time.time() - t0:.1f} s; |v|max={np.abs(v).max():.4f}")


def flux1024():
    t0 = time.time()
    x, T, y = request_inputs(FLUX, 1024, 1024, 1000)
    W = Weights(FLUX, cache_bytes=0)
    v, xn = F.request_step(FLUX, W, x, T, y, 0, 20, 3.5, 1024, 1024)
    out = os.path.join(ROOT, "tests", "golden", "flux1024_seed1000_S20_step0.npz")
    np.savez_compressed(out, v=v.astype(np.float32), x_next=xn.astype(np.float32))
    print(f"wrote {out} in {time.time() - t0:.1f} s; |v|max={np.abs(v).max():.4f}")


def sd3_1024():
    t0 = time.time()
    x, Tc, yc, Tu, yu = sd3_request_inputs(SD3, 1024, 1024, 1000)
    W = Weights(SD3, cache_bytes=20 << 30)
    v, xn = S3.request_step(SD3, W, x, Tc, yc, Tu, yu, 0, 20, 1024, 1024)
    out = os.path.join(ROOT, "tests", "golden", "sd3_1024_seed1000_S20.npz")
    np.savez_compressed(out, v=v.astype(np.float32), x_next=xn.astype(np.float32))
    print(f"wrote {out} in {time.time() - t0:.1f} s; |v|max={np.abs(v).max():.4f}")


def main():
    which = sys.argv[1:] or ["flux", "sd3"]
    for w in which:
        {"flux": flux, "sd3": sd3, "flux2048": flux2048, "flux1024": flux1024, "sd3_1024": sd3_1024}[w]()


if __name__ == "__main__":
    main()
