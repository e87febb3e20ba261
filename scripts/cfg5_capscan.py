"""Config 5 (1/8 shard) overflow scan: round-0 overflowed slot groups per capacity."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_date_schneiderw20_b200 import Context, load_workload, shard_range
from paper_conf_date_schneiderw20_b200.avfs import AvfsError
from workloads import make_config
w = make_config(5)
first, cnt = shard_range(w.n_slots, 0, 8)
s = torch.cuda.Stream()
for C in [int(x) for x in sys.argv[1:]]:
    for rr in (0, 3):
        ctx = Context(0)
        load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
        ctx.set_options(capacity=C, max_rerun_rounds=rr, profile=True)
        ctx.set_slot_range(first, cnt)
        t = time.time()
        try:
            ctx.simulate(s); torch.cuda.synchronize()
            st = ctx.stats()
            print(f"C={C} rr={rr} ok sweep_ms={st.get('sweep_ms')} ovf={st['overflow_slot_warps']} rounds={st['rerun_rounds']} arena={st['arena_bytes']/1e9:.1f}GB wall={time.time()-t:.1f}s", flush=True)
        except AvfsError as e:
            print(f"C={C} rr={rr} err {e} wall={time.time()-t:.1f}s", flush=True)
        ctx.close()
