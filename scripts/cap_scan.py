"""Overflow statistics vs capacity for a config (GPU)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_date_schneiderw20_b200 import Context, load_workload
from workloads import make_config
cfg = int(sys.argv[1])
caps = [int(x) for x in sys.argv[2].split(",")]
shard = int(sys.argv[3]) if len(sys.argv) > 3 else 1
w = make_config(cfg)
for cap in caps:
    ctx = Context(0)
    load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
    ctx.set_options(capacity=cap, profile=True)
    if shard > 1:
        ctx.set_slot_range(0, w.n_slots // shard)
    s = torch.cuda.Stream()
    ctx.simulate(s)
    torch.cuda.synchronize()
    t0 = time.time(); ctx.simulate(s); torch.cuda.synchronize(); t = time.time() - t0
    st = ctx.stats()
    print(f"cfg{cfg} cap{cap}: wall {t*1e3:.1f} ms sweep {st['sweep_ms']:.1f} ms ovf {st['overflow_slot_warps']}/{st['slot_warps']} rounds {st['rerun_rounds']} arena {st['arena_bytes']/1e9:.1f} GB evals/s {st['evals']/t:.3e}", flush=True)
    ctx.close()
