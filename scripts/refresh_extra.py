"""Copy a gpu_extra.sh / gpu_multirank.sh / gpu_checks.sh run (gpurun_out/) into profiles/ (run
here, no GPU): the delay A/B table, the capped-heap overflow line, the 2-rank line, the
bounds-checked build summary.    python scripts/refresh_extra.py [--round r02]"""
import argparse
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G = os.path.join(ROOT, "gpurun_out")
ap = argparse.ArgumentParser()
ap.add_argument("--round", default="r02")
R = ap.parse_args().round


def last_json(name):
    with open(os.path.join(G, name)) as f:
        return json.loads(f.read().strip().split("\n")[-1])


P = os.path.join(ROOT, "profiles")
# delay table vs in-sweep evaluation
f = os.path.join(P, f"{R}_delay_ab_cfg4.txt")
s = open(f).read()
rows = {n: last_json(f"delay_{n}.log") for n in ("t0", "s0", "t3", "s3")}
ms = {n: (d["ms_per_step"], d["roofline"]["kernel_ms"]) for n, d in rows.items()}
table = ("model                         delays                               step ms   sweep ms\n"
         f"N_v = 3, N_c = 0 (configs)    table (delay_kernel, 205 MB)          {ms['t0'][0]:6.1f}    {ms['t0'][1]:6.1f}\n"
         f"N_v = 3, N_c = 0              in sweep (FP64 Horner per slot)       {ms['s0'][0]:6.1f}    {ms['s0'][1]:6.1f}\n"
         f"N_v = N_c = 3 (Table I model) table                                 {ms['t3'][0]:6.1f}    {ms['t3'][1]:6.1f}\n"
         f"N_v = N_c = 3                 in sweep (16-coef 2-D Horner)         {ms['s3'][0]:6.1f}    {ms['s3'][1]:6.1f}\n\n")
a, b = s.index("model "), s.index("The in-sweep variant")
open(f, "w").write(s[:a] + table + s[b:])
# overflow stress and the 2-rank path
for src, dst in (("bench_cfg5_overflow.log", f"{R}_bench_cfg5_shard_overflow_stress.json"),
                 ("bench_2rank.log", f"{R}_bench_2rank_shared_gpu_cfg3.json")):
    with open(os.path.join(P, dst), "w") as o:
        o.write(json.dumps(last_json(src)) + "\n")
# bounds-checked build
hdr = ("Bounds-checked build (final kernel): scripts/gpu_checks.sh -- the stand-in for\n"
       "compute-sanitizer, which the GPU pool closed late in round 2.  libavfs.so compiled with\n"
       "-DAVFS_CHECKS: device asserts in the sweep that (1) every observable input of a slot has an entry\n"
       "there (its bit in the input's A) with >= 1 event, (2) a gate's outputs stay inside the extent\n"
       "reserved for it (in-place region capacity or its heap allocation), (3) every heap allocation lies\n"
       "inside the heap.  A failed assert traps the kernel (sticky CUDA error -> the test / bench fails).\n\n")
tail = open(os.path.join(G, "checks_pytest.log")).read().strip().split("\n")[-1]
lines = [f"pytest -m gpu (all GPU tests, checks build): {tail}"]
for n in ("cfg4", "cfg2", "cfg5", "cfg5_capped"):
    d = last_json(f"checks_{n}.log")
    st = d["stats"]
    lines.append(f"bench.py {n}: {d['ms_per_step']:.1f} ms/step, {d['value']:.3e} evals/s, spill {st['spill_bytes'] / 1e9:.1f} GB, "
                 f"groups rerun {st['overflow_slot_warps']}, rerun rounds {st['rerun_rounds']}")
open(os.path.join(P, f"{R}_bounds_checks.txt"), "w").write(hdr + "\n".join(lines) + "\n")
print("ok")
