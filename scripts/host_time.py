"""Per-step host vs device timing of simulate + sync on config 4 (diagnostic):
where does step time beyond the sweep kernel go?  Optional nvidia-smi sampling
in the background (--smi) as in bench.py."""
import argparse, os, subprocess, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_date_schneiderw20_b200 import Context, load_workload
from workloads import make_config
ap = argparse.ArgumentParser(); ap.add_argument("--smi", action="store_true"); ap.add_argument("--n", type=int, default=20)
a = ap.parse_args()
w = make_config(4)
ctx = Context(0); load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
ctx.set_options(capacity=w.capacity, profile=True)
s = torch.cuda.Stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
smi = subprocess.Popen(["nvidia-smi", "-i", "0", "--query-gpu=clocks.sm", "--format=csv,noheader", "-lms", "250"],
                       stdout=subprocess.DEVNULL) if a.smi else None
for i in range(a.n):
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        flush.zero_()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(s)
    t0 = time.perf_counter(); ctx.simulate(s); t1 = time.perf_counter(); ctx.sync(); t2 = time.perf_counter()
    e1.record(s); torch.cuda.synchronize()
    sw, _ = ctx.timing()
    print(f"step {e0.elapsed_time(e1):7.2f} ms  sweep {sw:7.2f}  simulate-call {1e3*(t1-t0):6.2f}  sync-call {1e3*(t2-t1):7.2f}")
if smi: smi.terminate()
