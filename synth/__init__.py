"""Seeded synthetic inputs shared by the oracle and the tests (spec SYNTH-1).

This module holds NO arithmetic of the method (no DiT math).  It only turns
(seed, tensor id, element index) into numbers, following the counter-hash
specification restated in ``include/tsv.h`` ("SYNTH-1").  The CUDA path has
its own, independent implementations of the same spec (``synth_kernel`` in
``paper_conf_asplos_luhtlwm0c26_b200/csrc/elementwise.cu`` for weights, the
host generator in ``csrc/engine.cu`` for request inputs); they are checked
bit-for-bit against this module in ``tests/test_gpu_kernels.py`` (weights via
``tsv_op_synth`` / ``tsv_debug_read_weight``) and ``tests/test_gpu_step.py``
(request inputs).

SYNTH-1
  key  = seed XOR (tensor_id << 48) XOR idx                    (uint64)
  h    = splitmix64_mix(key + 0x9E3779B97F4A7C15)               (uint64)
  u    = h >> 40                                                (24 bits)
  r    = float32((u - 2**23) * 2**-23)        in [-1, 1), exact
  kind 'w' (weights, sigma = 1/sqrt(fan_in)), 'b' (biases, sigma = 0.02),
       'x' (bf16 inputs, sigma = 1):
           c   = float32(sqrt(3) * sigma)   (rounded from float64)
           val = bf16_rne(float32(r * c))
  kind 'f' (fp32 inputs, sigma = 1): val = float32(r * float32(sqrt(3)))
  kind 'g' (RMSNorm gains):  c = float32(sqrt(3) * 0.1)
           val = bf16_rne(float32(1 + float32(r * c)))
"""
from .counter_hash import (  # noqa: F401
    GOLDEN_GAMMA,
    splitmix64_mix,
    hash_u64,
    uniform_pm1,
    bf16_rne_bits,
    bf16_bits_to_f32,
    gen_tensor,
    gen_tensor_bits,
    scale_for,
)
