"""Phase timing of the sweep (needs a -DAVFS_PROF_PHASES build): one warm-up simulate, reset, one simulate."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_date_schneiderw20_b200 import Context, load_workload
from paper_conf_date_schneiderw20_b200.avfs import debug_phase_cycles
from workloads import make_config
ap = argparse.ArgumentParser(); ap.add_argument("--config", type=int, default=4); a = ap.parse_args()
w = make_config(a.config)
ctx = Context(0); load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
ctx.set_options(capacity=w.capacity, profile=True)
s = torch.cuda.Stream(); ctx.simulate(s); ctx.sync(); debug_phase_cycles(reset=True); ctx.simulate(s); ctx.sync()
c = debug_phase_cycles().astype(np.float64)
names = {1: "phaseA", 2: "item setup", 3: "merge", 4: "item finish", 5: "phaseB total", 6: "barrier"}
tot = c[1] + c[5] + c[6]
st = ctx.stats()
print(f"cfg{a.config} sweep {st['sweep_ms']:.1f} ms; warp-cycles total {tot:.3e}")
for k, n in names.items():
    print(f"  {n:14s} {c[k]:.3e}  {100*c[k]/tot:5.1f}%")
