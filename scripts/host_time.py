import sys, time, os
sys.path.insert(0, '/root/repo')
import numpy as np, torch
from paper_conf_date_schneiderw20_b200 import Context, load_workload
from workloads import make_config
w = make_config(4)
ctx = Context(0); load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
ctx.set_options(capacity=w.capacity, profile=True)
s = torch.cuda.Stream()
for i in range(6):
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(s)
    t0 = time.perf_counter(); ctx.simulate(s); t1 = time.perf_counter(); ctx.sync(); t2 = time.perf_counter()
    e1.record(s); torch.cuda.synchronize()
    st = ctx.stats()
    print(f"simulate host {1e3*(t1-t0):.2f} ms, sync {1e3*(t2-t1):.2f} ms, events {e0.elapsed_time(e1):.2f} ms, sweep {st['sweep_ms']:.2f} ms")
