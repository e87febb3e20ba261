"""Small end-to-end runs for compute-sanitizer (c17 keep-all, multiplier with spills and reruns, random DAG)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_date_schneiderw20_b200 import Context, load_workload
from workloads import make_config

for cfg, kw in ((1, dict(n_pairs=64)), (2, dict(n_pairs=64, n_vdd=2)), (3, dict(n_pairs=64, n_vdd=2, scale=0.02))):
    w = make_config(cfg, **kw)
    for cap, spill in ((1, 0), (1, -1), (1, 4096), (8, 0)):
        ctx = Context(0)
        load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
        ctx.set_options(capacity=cap, keep_all=(cfg == 1), max_rerun_rounds=4, spill_bytes=spill,
                        delay_in_sweep=(cap == 8))
        ctx.simulate()
        a = ctx.activity()
        ctx.waveforms(w.netlist.po_sig, 0, w.n_slots, cap=8)
        ctx.capture(np.full(len(w.vdd), 50.0, np.float32))
        ctx.switching_energy()
        st = ctx.stats()
        print(cfg, cap, spill, int(a.sum()), st["rerun_rounds"], st["spill_bytes"], flush=True)
        ctx.close()

# work-distribution variants: G slot groups per CTA (named barriers), S CTAs per group
w = make_config(3, n_pairs=96, n_vdd=2, scale=0.05)
for env in ({"AVFS_GROUPS_PER_CTA": "4"}, {"AVFS_GROUPS_PER_CTA": "1", "AVFS_SPLIT": "2"},
            {"AVFS_GROUPS_PER_CTA": "1", "AVFS_SPLIT": "8"}):
    os.environ.pop("AVFS_GROUPS_PER_CTA", None)
    os.environ.pop("AVFS_SPLIT", None)
    os.environ.update(env)
    ctx = Context(0)
    load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
    ctx.set_options(capacity=4)
    ctx.simulate()
    print(env, int(ctx.activity().sum()), flush=True)
    ctx.close()
os.environ.pop("AVFS_GROUPS_PER_CTA", None)
os.environ.pop("AVFS_SPLIT", None)
# 2-D (v, c) delay model, voltage islands
w = make_config(3, n_pairs=64, n_vdd=2, scale=0.03, deg_c=3)
ctx = Context(0)
load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
ctx.set_options(capacity=2, quantum_ps=2.0 ** -8)
ctx.simulate()
print("2d", int(ctx.activity().sum()), flush=True)
ctx.close()
