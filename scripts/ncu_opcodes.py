"""Dynamic SASS opcode histogram (warp instructions executed per opcode) of the
profiled kernel, from an ncu report's source page (sass view).
    python scripts/ncu_opcodes.py rep [--gw GATE_WARPS]"""
import argparse, collections, csv, io, re, subprocess
ap = argparse.ArgumentParser(); ap.add_argument("rep"); ap.add_argument("--gw", type=float, default=200000 * 2048)
a = ap.parse_args()
out = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(r for r in rows if r and "Source" in r and "Instructions Executed" in r)
si, ie = hdr.index("Source"), hdr.index("Instructions Executed")
cnt = collections.Counter()
for r in rows:
    if len(r) <= ie or r is hdr or not r[ie].replace(".", "").isdigit():
        continue
    m = re.match(r"\s*(@!?U?P[T0-9]+\s+)?([A-Z][A-Z0-9_]*)", r[si])
    if m:
        cnt[m.group(2)] += float(r[ie])
tot = sum(cnt.values())
print(f"{a.rep}: {tot:.4e} warp instructions = {tot / a.gw:.1f} per gate x 32-slot group")
for k, v in cnt.most_common(40):
    print(f"{k:12s} {v:14.4e}  {100 * v / tot:5.1f}%  {v / a.gw:7.2f}/gw")
