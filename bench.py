#!/usr/bin/env python
"""Benchmark: gate-waveform evals/s (gates x pairs x Vdd) and % of the HBM roofline.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 4] [--impl avfs|reference]

One step = one avfs_simulate over the whole slot space of the workload
(stimulus expansion, PI activity, the persistent level sweep, overflow reruns,
on-device activity / latest-arrival reductions) plus, for N > 1, the NCCL
reduce of the activity counters.  Inputs are resident in HBM before timing;
L2 is flushed (256 MiB write) between timed steps.  The `e2e` figure repeats
the measurement through the public API with host buffers (H2D of the stimuli,
D2H of activity + latest arrival inside the timed region).
For N > 1 launch with torchrun (one rank per GPU).  Slots are independent
problems, so they shard with no data-path exchange; by default the
scaling is strong: BASELINE's config at every N, its stimulus pairs split into
N contiguous ranges, each simulated at every Vdd point (whole operating-point
sweeps per slot group; "--scaling weak" grows the pairs N-fold instead).  Config 5
(specified on 8 x B200) runs as one shard of 8 per GPU with --gpus 8, or
--shard-of 8 on one GPU.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]
UNIT = "evals/s"


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def traffic_per_launch(cfg):
    p = os.path.join(ROOT, "profiles", "ncu_sweep_traffic.json")
    if os.path.exists(p):
        d = json.load(open(p))
        if int(d.get("config", -1)) == cfg:
            return d.get("dram_bytes_per_launch")
    return None


class ClockSampler:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, dev: int):
        self.dev = dev
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", os.environ.get("AVFS_SMI_MS", "250")], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(2)
        except Exception:
            self.proc.kill()
        self.t.join(1)
        sm = [float(r[0]) for r in self.rows if len(r) >= 6 and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) >= 6 and r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows if len(r) >= 6 for i in range(4) if r[2 + i] == "Active"})
        if not sm:
            return None
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(sm)}


# AVFS_BENCH_SHARE_GPU=1: every rank uses cuda:0 and gloo collectives on CPU
# tensors -- exercises the multi-rank path on a single-GPU box (testing only).
SHARE_GPU = os.environ.get("AVFS_BENCH_SHARE_GPU", "0") == "1"


def dist_setup(n_gpus):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = 0 if SHARE_GPU else int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch
        import torch.distributed as dist
        if SHARE_GPU:
            dist.init_process_group("gloo")
        else:
            torch.cuda.set_device(local)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return world, rank, local


def _reduce(t, op):
    """dist.reduce to rank 0 (on the collective's device)."""
    import torch.distributed as dist
    if SHARE_GPU:
        c = t.cpu()
        dist.reduce(c, dst=0, op=op)
        t.copy_(c)
    else:
        dist.reduce(t, dst=0, op=op)


def _max_over_ranks(x, dev):
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cpu" if SHARE_GPU else dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def host_cores() -> int:
    """All cores this process may run on (torchrun sets OMP_NUM_THREADS=1; the
    oracle runs on rank 0 only, so it takes every core explicitly)."""
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def collective_info(world, args):
    """What the multi-GPU step exchanges: nothing during the
    simulation; one reduce of the activity counters (SUM) and of the latest
    arrival (MAX) to rank 0 per step."""
    if world <= 1:
        return None
    import torch
    import torch.distributed as dist
    info = {"backend": dist.get_backend(), "world_size": dist.get_world_size(),
            "ops": ["reduce(activity u64 [signals x Vdd], SUM)", "reduce(latest f32 [Vdd], MAX)"],
            "scaling": args.scaling}
    try:
        info["nccl_version"] = ".".join(str(x) for x in torch.cuda.nccl.version())
    except Exception:
        pass
    return info


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.lower().startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def parity_sample(w):
    """BASELINE.md / SURVEY §8(d) deterministic oracle sample (also the GPU
    parity set): cfgs 1-2 every slot; cfg 3 pairs j mod 64 = 0; cfg 4 pairs
    j mod 256 = 0; cfg 5 pair 0 at all 51 Vdd points.  Returns (pairs, vdd
    indices, description)."""
    P, V = w.stimuli.n_pairs, len(w.vdd)
    step = {1: 1, 2: 1, 3: 64, 4: 256}.get(w.cfg)
    if step is None:                                    # cfg 5
        j = np.zeros(V, np.int64)
        k = np.arange(V, dtype=np.int32)
        return j, k, f"pair 0 x all {V} Vdd points"
    jj = np.arange(0, P, step, dtype=np.int64)
    k, j = np.meshgrid(np.arange(V, dtype=np.int32), jj, indexing="ij")
    return j.ravel(), k.ravel(), (f"pairs j mod {step} = 0 ({len(jj)} pairs) x {V} Vdd" if step > 1
                                  else f"every slot ({P} pairs x {V} Vdd)")


def cpu_baseline(w):
    """The oracle as it stands, on this host's cores and on one core, on the
    deterministic sample of BASELINE.md's CPU-baseline plan."""
    import oracle
    threads = host_cores()
    j, k, desc = parity_sample(w)

    def run(nth, jj, kk):
        t0 = time.perf_counter()
        oracle.simulate(w.netlist, w.library, w.stimuli, w.vdd, jj, kk, quantum=0.0, cap=0,
                        out_sig=w.netlist.po_sig, threads=nth)
        return time.perf_counter() - t0

    t_all = run(threads, j, k)
    # 1 thread: the whole sample if it takes <= ~20 s at the all-core rate x cores, else a prefix
    n1 = int(min(len(j), max(1, 20.0 / max(t_all * threads / len(j), 1e-6))))
    t_one = run(1, j[:n1], k[:n1])
    G = w.netlist.n_gates
    return {"value": G * len(j) / t_all, "unit": UNIT, "cores": threads, "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": f"{desc}: {len(j)} slots (all {G} gates each), {t_all:.2f} s wall, OpenMP over slots",
            "one_thread": {"value": G * n1 / t_one, "unit": UNIT, "cores": 1,
                           "sample": f"first {n1} slots of that sample, {t_one:.2f} s wall"}}


def run_reference(args, w, world, rank):
    """--impl reference: the oracle (FP64 event-driven, C/OpenMP) on the host cores."""
    if rank != 0:
        return
    import oracle
    P, V = w.stimuli.n_pairs, len(w.vdd)
    threads = host_cores()
    # each step: the deterministic parity sample, or an evenly
    # spaced subset of it that keeps the whole --steps K --warmup W run within
    # a few minutes
    js, ks, desc = parity_sample(w)
    probe = np.linspace(0, len(js) - 1, min(len(js), max(threads, 4))).astype(int)
    t0 = time.perf_counter()
    oracle.simulate(w.netlist, w.library, w.stimuli, w.vdd, js[probe], ks[probe], cap=0,
                    out_sig=w.netlist.po_sig, threads=threads)
    per_slot = (time.perf_counter() - t0) / len(probe)
    budget = 150.0 / max(1, args.steps + args.warmup)
    n = int(max(len(probe), min(len(js), budget / max(per_slot, 1e-6))))
    sel = np.linspace(0, len(js) - 1, n).astype(int)
    times = []
    for it in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.simulate(w.netlist, w.library, w.stimuli, w.vdd, js[sel], ks[sel], cap=0,
                        out_sig=w.netlist.po_sig, threads=threads)
        if it >= args.warmup:
            times.append(time.perf_counter() - t0)
    t = float(np.sum(times))
    value = w.netlist.n_gates * n * args.steps / t
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t / args.steps,
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": config_dict(w, args),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "cpu_model": cpu_model(),
                         "sample": f"{n} slots per step of the parity sample ({desc}) of {P * V}"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def config_dict(w, args):
    d = w.describe()
    n = getattr(args, "shard_slots", None) or w.n_slots
    d.update({"slots": n, "evals_per_step": w.netlist.n_gates * n,
              "mode": "F (FP64 delay polynomials, FP32 times)" if args.quantum == 0 else f"Q (quantum {args.quantum} ps)",
              "delays": "evaluated in the sweep" if getattr(args, "delay_in_sweep", False) else "delay table",
              "l2": "flushed by a 256 MiB write between timed steps; waveform arena >> L2",
              "parallelism": (f"one pair shard of {args.shard_of} (rank 0, all Vdd points), 1 GPU"
                              if args.shard_of > 1 else f"pair-shard x{args.gpus} ({args.scaling}, all Vdd points per rank)")})
    return d


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--capacity", type=int, default=0)
    ap.add_argument("--quantum", type=float, default=0.0)
    ap.add_argument("--warps-per-cta", type=int, default=0)
    ap.add_argument("--impl", default="avfs", choices=["avfs", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--scaling", default="strong", choices=["weak", "strong"],
                    help="strong (default): BASELINE's config at every N, slots sharded over ranks; "
                         "weak: N x the pairs")
    ap.add_argument("--deg-c", type=int, default=0,
                    help="N_c of the delay polynomial (3 = the paper's 2-D Table I model, N_v = N_c = 3)")
    ap.add_argument("--spill-bytes", type=int, default=0,
                    help="pass-0 spill heap bytes (0 auto, <0 none): a capped heap forces overflow reruns (H7)")
    ap.add_argument("--delay-in-sweep", action="store_true",
                    help="evaluate Eq. (4)/(9) inside the sweep instead of tabulating delays")
    ap.add_argument("--shard-of", type=int, default=0,
                    help="N=1 only: simulate rank 0's shard of an N-GPU run (e.g. config 5, "
                         "specified on 8 x B200, does not fit one GPU whole)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl == "avfs" else args.warmup

    from workloads import make_config
    world, rank, local = dist_setup(args.gpus)
    w = make_config(args.config, deg_c=args.deg_c)
    if args.scaling == "weak" and world > 1:
        w = make_config(args.config, n_pairs=w.stimuli.n_pairs * world, deg_c=args.deg_c)
    if args.impl == "reference":
        run_reference(args, w, world, rank)
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()
        return

    import torch
    from paper_conf_date_schneiderw20_b200 import Context, load_workload, shard_pairs
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    stream = torch.cuda.Stream(dev)
    ctx = Context(local)
    load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
    cap = args.capacity or w.capacity
    ctx.set_options(capacity=cap, quantum_ps=args.quantum, warps_per_cta=args.warps_per_cta, profile=True,
                    delay_in_sweep=args.delay_in_sweep, spill_bytes=args.spill_bytes)
    total_slots = w.n_slots
    P, V = w.stimuli.n_pairs, len(w.vdd)
    first, n_local = shard_pairs(P, rank, world)
    if args.shard_of > 1 and world == 1:
        first, n_local = shard_pairs(P, 0, args.shard_of)
        total_slots = n_local * V
        args.shard_slots = total_slots
    ctx.set_pair_range(first, n_local)
    n_sig, V = w.netlist.n_signals, len(w.vdd)
    act_dev = torch.zeros((n_sig, V), dtype=torch.int64, device=dev)
    lat_dev = torch.zeros(V, dtype=torch.float32, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def step():
        ctx.simulate(stream)      # asynchronous; sync settles overflow reruns (none expected)
        ctx.sync()
        if world > 1:
            import torch.distributed as dist
            ctx.activity(act_dev)
            ctx.latest_arrival(lat_dev)                       # device copy, no host round trip
            with torch.cuda.stream(stream):
                _reduce(act_dev, dist.ReduceOp.SUM)          # the only collective
                _reduce(lat_dev, dist.ReduceOp.MAX)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    stats = ctx.stats()
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.synchronize()
    clocks = ClockSampler(local)
    clocks.start()
    import gc
    gc.collect()
    gc.disable()                    # no collector pauses between the stream's events
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    sweep_ms, rerun_ms = [], []
    for i in range(args.steps):
        with torch.cuda.stream(stream):
            flush.zero_()
        ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
        sw_i, rr_i = ctx.timing()
        sweep_ms.append(sw_i)
        rerun_ms.append(rr_i)
    torch.cuda.synchronize()
    gc.enable()
    ck = clocks.stop()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    t_total = float(np.sum(step_ms))
    if world > 1:
        import torch.distributed as dist
        t_total = _max_over_ranks(t_total, dev)
        dist.barrier()
    stats = ctx.stats()
    evals_total = w.netlist.n_gates * total_slots
    value = evals_total * args.steps / (t_total / 1e3)

    # roofline of the dominant kernel (the pass-0 sweep) on this rank
    peak, peak_src = peaks()
    sweep_avg = float(np.mean(sweep_ms))
    alg_b = stats["alg_bytes"]
    achieved = alg_b / (sweep_avg / 1e3) / 1e9
    traffic = traffic_per_launch(args.config) if world == 1 else None

    # e2e through the public API with host buffers (pinned), H2D + D2H in the region
    e2e = None
    if not args.no_e2e:
        p1h = torch.from_numpy(w.stimuli.p1.view(np.int32)).pin_memory().numpy().view(np.uint32)
        p2h = torch.from_numpy(w.stimuli.p2.view(np.int32)).pin_memory().numpy().view(np.uint32)
        h2d = int(p1h.nbytes + p2h.nbytes)
        d2h = int(n_sig * V * 8 + V * 4)
        act_h = torch.empty((n_sig, V), dtype=torch.int64).pin_memory().numpy().view(np.uint64)
        e2e_ms = []
        for i in range(args.steps + 1):
            with torch.cuda.stream(stream):
                flush.zero_()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            ctx.set_stimuli(p1h, p2h)
            ctx.simulate(stream)
            a = ctx.activity(act_h)
            lat = ctx.latest_arrival()
            if world > 1:
                import torch.distributed as dist
                ta = torch.from_numpy(a.view(np.int64)).to(dev)
                tl = torch.from_numpy(lat).to(dev)
                _reduce(ta, dist.ReduceOp.SUM)
                _reduce(tl, dist.ReduceOp.MAX)
                a = ta.cpu()
            if i > 0:
                e2e_ms.append((time.perf_counter() - t0) * 1e3)
        te = float(np.sum(e2e_ms))
        if world > 1:
            te = _max_over_ranks(te, dev)
        e2e = {"value": evals_total * args.steps / (te / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(w)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_total / args.steps, "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "f32",
            "data": "synthetic", "config": config_dict(w, args),
            "step_ms_each": [round(x, 3) for x in step_ms],
            "sweep_ms_each": [round(x, 3) for x in sweep_ms],
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                         "kernel": "avfs::sweep_kernel", "kernel_ms": sweep_avg,
                         "alg_bytes_per_launch": alg_b,
                         "sweep_share_of_step": sweep_avg / (t_total / args.steps)},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(stats["launches"] * args.steps),
            "collective": collective_info(world, args),
            "clocks": ck,
            "stats": {k: stats[k] for k in ("evals", "slot_warps", "overflow_slot_warps", "rerun_rounds", "spill_bytes", "batches",
                                            "grid", "warps_per_cta", "n_scratch_buffers", "n_pinned",
                                            "arena_bytes", "launches", "enc_bytes")},
            "overflow": {"groups_rerun": stats["overflow_slot_warps"], "groups": stats["slot_warps"],
                         "rerun_fraction": stats["overflow_slot_warps"] / max(stats["slot_warps"], 1),
                         "rerun_ms": float(np.mean(rerun_ms)),
                         "rerun_share_of_step": float(np.mean(rerun_ms)) / (t_total / args.steps)},
            "paper_context": "P100 (CUDA 10): 1186 MEPS average at one Vdd, 310-1785x over a serial "
                             "commercial event-driven simulator on a Xeon E5-2687W v2 core (PAPER.md L203)",
        }
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
