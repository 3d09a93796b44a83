"""CPU ORACLE — test infrastructure only.

A plain, slow, obviously-correct float64 numpy implementation of what the
hot path computes: one denoising step (transformer forward + Euler update) of
a FLUX.1-dev-shaped MMDiT on one request's latent, and its simulated Ulysses
sequence-parallel form with k virtual ranks.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import anything under
``oracle/``.  The product path (``paper_conf_asplos_luhtlwm0c26_b200`` and
``libtsv.so``) never imports, links or calls it, and shares no code with it.
The only shared module is ``synth/`` (seeded input generation, SYNTH-1),
which holds none of the method's arithmetic.

Citations:
  P:n     line n of the paper text (TetriServe, ASPLOS '26, PAPER.md).
  S:§     SURVEY.md section (the readings adopted where the paper is silent).
  TT:f:n  local mirror of Black Forest Labs' public FLUX.1 model code under
          site-packages/torchtitan/experiments/flux/model/ (architecture facts
          only; the paper gives no DiT equations).

Pins (tests/test_oracle_*.py, run with -m "not gpu"): see DESIGN.md §Pins.
Parity unpinned: the full FLUX step on random weights has no printed value
in the paper (S:§8(c) P12); it is pinned only through its parts, the
adaLN-Zero closed form (P7), SP invariance (P9) and an independent library
implementation of the blocks (torchtitan's FLUX layers).
"""
