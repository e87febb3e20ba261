"""Per-evaluation sweep throughput of a config for different (pairs, Vdd points) splits of about
the same slot count: how much the pair-major groups gain when a group holds one pair's points
(V = 32 / 64) against groups that straddle pairs (config 5's 51 points).
    python scripts/vdd_pack_ab.py --config 5 --splits 128x51,204x32,102x64"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_date_schneiderw20_b200 import Context, load_workload  # noqa: E402
from workloads import make_config  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--splits", default="128x51,204x32,102x64")
ap.add_argument("--runs", type=int, default=4)
a = ap.parse_args()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()
for sp in a.splits.split(","):
    P, V = (int(x) for x in sp.split("x"))
    w = make_config(a.config, n_pairs=P, n_vdd=V)
    ctx = Context(0)
    load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
    ctx.set_options(capacity=w.capacity, profile=True)
    for r in range(a.runs):                  # the first run learns the spill heap (reruns)
        flush.fill_(r & 255)
        ctx.simulate(s)
        ctx.sync()
    st = ctx.stats()
    best = st["sweep_ms"]
    ev = w.netlist.n_gates * P * V
    print(f"cfg {a.config} {P} pairs x {V} Vdd: sweep {best:.2f} ms, {ev / best * 1e3:.3e} evals/s, "
          f"spill {st['spill_bytes'] / 1e9:.1f} GB, groups {st['slot_warps']}", flush=True)
    del ctx
    torch.cuda.empty_cache()
