"""One warm-up + one profiled simulate of a config (for ncu -k regex:sweep -s 1 -c 1)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_date_schneiderw20_b200 import Context, load_workload  # noqa: E402
from workloads import make_config  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=4)
ap.add_argument("--capacity", type=int, default=0)
ap.add_argument("--warps-per-cta", type=int, default=0)
ap.add_argument("--runs", type=int, default=2)
ap.add_argument("--shard-of", type=int, default=0)
a = ap.parse_args()
w = make_config(a.config)
ctx = Context(0)
load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
ctx.set_options(capacity=a.capacity or w.capacity, warps_per_cta=a.warps_per_cta, profile=True)
if a.shard_of > 1:
    from paper_conf_date_schneiderw20_b200 import shard_pairs
    ctx.set_pair_range(*shard_pairs(w.stimuli.n_pairs, 0, a.shard_of))
s = torch.cuda.Stream()
for _ in range(a.runs):
    ctx.simulate(s)
print(ctx.stats())
