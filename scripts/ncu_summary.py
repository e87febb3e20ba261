"""Summarise an ncu report (run here, no GPU): key metrics + stall mix + traffic JSON.

    python scripts/ncu_summary.py gpurun_out/prof.ncu-rep --config 4 --tag r01 [--alg-bytes B] [--evals E]
"""
import argparse
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "smsp__inst_executed.sum", "sm__inst_executed.sum.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "launch__grid_size", "launch__block_size",
        "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return [{k: (u, v) for k, u, v in zip(rows[0], rows[1], row)} for row in rows[2:]]


def stalls(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    body = out.split("\n", 1)[1] if out.startswith('"Kernel Name"') else out
    rows = list(csv.DictReader(io.StringIO(body)))
    if not rows:
        return {}, 0
    st = [k for k in rows[0] if k and k.startswith("stall_") and "Not Issued" not in k]
    tot = {k[6:]: sum(int(r[k] or 0) for r in rows) for k in st}
    T = sum(tot.values()) or 1
    return {k: round(v / T, 3) for k, v in sorted(tot.items(), key=lambda x: -x[1]) if v / T >= 0.01}, len(rows)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--tag", default="r01")
    ap.add_argument("--alg-bytes", type=float, default=None)
    ap.add_argument("--evals", type=float, default=None)
    a = ap.parse_args()
    rs = raw(a.rep)
    lines = [f"source: {os.path.basename(a.rep)} (ncu --set full --clock-control none --import-source on)"]
    for i, r in enumerate(rs):
        lines.append(f"launch {i}: {r.get('Kernel Name', ('', '?'))[1]}")
        for k in KEYS:
            if k in r:
                lines.append(f"  {k} = {r[k][1]} {r[k][0]}")
    st, nsass = stalls(a.rep)
    lines.append(f"stall mix (share of warp-stall samples): {st}")
    lines.append(f"SASS instructions in kernel: {nsass}")
    r = rs[0]

    def val(k):
        u, v = r[k]
        return float(v.replace(",", "")) * SCALE.get(u, 1)
    traffic = val("dram__bytes_read.sum") + val("dram__bytes_write.sum")
    u, v = r["gpu__time_duration.sum"]
    dur_ms = float(v.replace(",", "")) * {"ns": 1e-6, "us": 1e-3, "ms": 1.0, "s": 1e3}.get(u, 1.0)
    summary = {"config": a.config, "tag": a.tag, "kernel": r.get("Kernel Name", ("", ""))[1],
               "dram_bytes_per_launch": traffic, "dram_read": val("dram__bytes_read.sum"),
               "dram_write": val("dram__bytes_write.sum"), "duration_ms_under_ncu": dur_ms,
               "alg_bytes_per_launch": a.alg_bytes, "stall_mix": st}
    if a.alg_bytes:
        summary["traffic_over_alg"] = traffic / a.alg_bytes
        lines.append(f"traffic / algorithmic bytes = {traffic / a.alg_bytes:.3f}")
    if a.evals:
        ipg = float(r["smsp__inst_executed.sum"][1].replace(",", "")) / (a.evals / 32)
        summary["warp_instructions_per_gate_warp"] = ipg
        lines.append(f"warp instructions per gate-warp (32 evals) = {ipg:.1f}")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"{a.tag}_sweep_cfg{a.config}_ncu_summary.txt"), "w") as f:
        f.write("\n".join(lines) + "\n")
    json.dump(summary, open(os.path.join(ROOT, "profiles", "ncu_sweep_traffic.json"), "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
