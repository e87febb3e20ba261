"""Top CUDA source lines by warp-stall samples (with the dominant stall reasons) from an ncu report.
    python scripts/ncu_stall_lines.py rep [--top N]"""
import argparse, csv, io, subprocess, collections
ap = argparse.ArgumentParser(); ap.add_argument("rep"); ap.add_argument("--top", type=int, default=30); a = ap.parse_args()
out = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = None; samp = collections.Counter(); src = {}; fname = None; reasons = collections.defaultdict(collections.Counter)
for r in rows:
    if r and r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r and r[0] == "Line No": hdr = r; continue
    if not hdr or len(r) < len(hdr) or not r[0]: continue
    cur = (fname, int(r[0])); src[cur] = r[1].strip()[:80]
    f = lambda x: float(x) if x not in ("", "-") else 0.0
    samp[cur] += f(r[hdr.index("Warp Stall Sampling (All Samples)") - len(hdr)])
    for i, h in enumerate(hdr):
        if h.startswith("stall_") or h.startswith("smsp__pcsamp_warps_issue_stalled_"):
            reasons[cur][h.replace("smsp__pcsamp_warps_issue_stalled_", "")] += f(r[i - len(hdr)])
ts = sum(samp.values())
for k, v in sorted(samp.items(), key=lambda x: -x[1])[:a.top]:
    top = ", ".join(f"{n}:{100*c/max(v,1):.0f}%" for n, c in reasons[k].most_common(2) if c)
    print(f"{k[0]}:{k[1]:5d} {100*v/max(ts,1):5.1f}%  [{top}]  {src[k]}")
