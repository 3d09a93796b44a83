"""Host-side phase timing of a reshard issued while the request's previous step still runs
(TSV_TRACE=1 prints the engine's phase timestamps): python tools/trace_reshard.py"""
import os
import sys
import time

os.environ["TSV_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402

eng = tsv.Engine("flux", devices=[0] * 4)
g01, g23 = eng.group_create([0, 1]), eng.group_create([2, 3])
ra = eng.request_create(2048, 2048, num_steps=20, seed=1600)
eng.event_wait(eng.request_step(ra, 0, g01))
for trial in range(3):
    t0 = time.perf_counter()
    ev = eng.request_step(ra, 1 + 2 * trial, g01 if trial % 2 == 0 else g23)
    t1 = time.perf_counter()
    print(f"step enqueue {1e3 * (t1 - t0):.2f} ms", file=sys.stderr, flush=True)
    eng.request_reshard(ra, g23 if trial % 2 == 0 else g01)
    t2 = time.perf_counter()
    print(f"reshard call {1e3 * (t2 - t1):.2f} ms, step still running: {not eng.event_query(ev)}", file=sys.stderr,
          flush=True)
    eng.event_wait(eng.request_step(ra, 2 + 2 * trial, g23 if trial % 2 == 0 else g01))
eng.close()
