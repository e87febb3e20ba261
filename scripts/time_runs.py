"""Sweep time of repeated simulates (CUDA events, profile=True) for a config / shard.
    python scripts/time_runs.py --config 5 --shard-of 8 [--capacity C] [--runs N] [--flush]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_date_schneiderw20_b200 import Context, load_workload, shard_pairs  # noqa: E402
from workloads import make_config  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=4)
ap.add_argument("--capacity", type=int, default=0)
ap.add_argument("--runs", type=int, default=5)
ap.add_argument("--shard-of", type=int, default=0)
ap.add_argument("--flush", action="store_true")
a = ap.parse_args()
w = make_config(a.config)
ctx = Context(0)
load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
ctx.set_options(capacity=a.capacity or w.capacity, profile=True)
if a.shard_of > 1:
    ctx.set_pair_range(*shard_pairs(w.stimuli.n_pairs, 0, a.shard_of))
s = torch.cuda.Stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for r in range(a.runs):
    if a.flush:
        flush.fill_(r & 255)
    ctx.simulate(s)
    ctx.sync()
    st = ctx.stats()
    print(f"run {r}: sweep {st['sweep_ms']:.2f} ms, spill {st['spill_bytes'] / 1e9:.1f} GB, "
          f"heap {st.get('spill_heap_bytes', 0) / 1e9:.1f} GB, reruns {st['rerun_rounds']}", flush=True)
