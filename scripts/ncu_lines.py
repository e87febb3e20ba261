"""Per-CUDA-source-line warp instructions and stall samples from an ncu report
(source page, cuda,sass view).  python scripts/ncu_lines.py rep [--evals E] [--top N]"""
import argparse, csv, io, subprocess, collections
ap = argparse.ArgumentParser(); ap.add_argument("rep"); ap.add_argument("--evals", type=float, default=13107200000)
ap.add_argument("--top", type=int, default=60); a = ap.parse_args()
out = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = None; inst = collections.Counter(); samp = collections.Counter(); src = {}; cur = None; fname = None
for r in rows:
    if r and r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r and r[0] == "Line No": hdr = r; continue
    if not hdr or len(r) < len(hdr): continue
    if r[0]:  # cuda line row
        cur = (fname, int(r[0])); src[cur] = r[1].strip()[:90]
        ie = hdr.index("Instructions Executed") - len(hdr); ws = hdr.index("Warp Stall Sampling (All Samples)") - len(hdr)
        f = lambda x: float(x) if x not in ("", "-") else 0.0
        inst[cur] += f(r[ie]); samp[cur] += f(r[ws])
tot = sum(inst.values()); ts = sum(samp.values()); gw = a.evals / 32
# the cuda-line rows of the source page attribute inlined code to several
# lines; scale to the kernel's executed warp instructions (sass view total)
raw = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
srows = list(csv.reader(io.StringIO(raw)))
sh = next(r for r in srows if r and "Source" in r and "Instructions Executed" in r)
k = sh.index("Instructions Executed")
sass_tot = sum(float(r[k]) for r in srows if len(r) > k and r is not sh and r[k].replace(".", "").isdigit())
f = sass_tot / tot if tot else 1.0
print(f"executed warp instructions {sass_tot:.4e} = {sass_tot/gw:.1f} per gate-warp (per-line counts below scaled "
      f"by {f:.3f} from the cuda-line attribution sum {tot:.4e}); stall samples {ts:.0f}")
inst = collections.Counter({key: v * f for key, v in inst.items()}); tot = sass_tot
for k, v in sorted(inst.items(), key=lambda x: -x[1])[:a.top]:
    print(f"{k[0]}:{k[1]:5d} {v/gw:7.1f}/gw {100*v/tot:5.1f}%  samp {100*samp[k]/max(ts,1):5.1f}%  {src[k]}")
