"""GPU <-> oracle parity through the C-ABI (-m gpu).

Small cases compare every (signal, slot); they span several 32-slot groups,
ragged pair counts (not multiples of 32), 1..4-input cells, dangling gates,
overflow reruns and slot-range shards.
"""
import numpy as np
import pytest

import oracle
from workloads import make_config, make_library, make_stimuli, random_dag, exhaustive_pairs, c17
from workloads.configs import Workload
from workloads.netlists import _Builder
from tests.parity import Q, gpu_run, gpu_waveforms, compare, activity_ref

pytestmark = pytest.mark.gpu


def full_compare(w, quantum, capacity=None, cap=None, label="", **kw):
    nl = w.netlist
    j, k = oracle.all_slots(w.stimuli.n_pairs, len(w.vdd))
    ref = oracle.simulate(nl, w.library, w.stimuli, w.vdd, j, k, quantum=quantum, cap=cap or 64)
    cap = cap or max(1, int(ref.count.max()))
    ctx = gpu_run(w, quantum=quantum, capacity=capacity, **kw)
    sig = np.arange(nl.n_signals, dtype=np.int32)
    init, cnt, times = gpu_waveforms(ctx, sig, 0, len(j), cap)
    st = compare(ref, init, cnt, times, quantum, label)
    act = ctx.activity().astype(np.int64)
    ra, ok = activity_ref(ref, len(w.vdd), nl.n_signals)
    assert np.array_equal(act[ok], ra[ok]), f"{label}: activity differs"
    lat = ctx.latest_arrival()
    if quantum > 0:
        po = nl.po_sig
        n = ref.count[:, po]
        last = np.take_along_axis(ref.times[:, po, :], np.maximum(n - 1, 0)[:, :, None], 2)[:, :, 0]
        last = np.where(n > 0, last, 0.0).reshape(len(w.vdd), -1).max(1)
        assert np.array_equal(lat.astype(np.float64), last), f"{label}: latest arrival differs"
    st["stats"] = ctx.stats()
    ctx.close()
    return st


@pytest.mark.parametrize("quantum", [Q, 0.0])
def test_c17_config1(quantum):
    st = full_compare(make_config(1), quantum, label="c17")
    assert st["events"] > 0


@pytest.mark.parametrize("quantum", [Q, 0.0])
def test_c17_exhaustive_1024_pairs(quantum):
    w = make_config(1)
    w.stimuli = exhaustive_pairs(5)
    full_compare(w, quantum, label="c17-exh")


@pytest.mark.parametrize("quantum", [Q, 0.0])
def test_multiplier_ragged(quantum):
    w = make_config(2, n_pairs=100, n_vdd=3)
    st = full_compare(w, quantum, capacity=32, label="mult")
    assert st["events"] > 10000


@pytest.mark.parametrize("quantum", [Q, 0.0])
def test_random_dag_four_input_cells(quantum):
    mix = {"NAND2": .2, "NOR2": .1, "XOR2": .1, "INV": .15, "BUF": .05, "AOI21": .1, "OAI21": .1,
           "NAND4": .05, "NOR4": .05, "AOI22": .05, "OAI22": .05}
    nl = random_dag(4242, 3000, 64, 25, mix=mix)
    w = Workload(0, "rdag4", nl, make_library(77, deg_v=3), make_stimuli(78, nl.n_pi, 200),
                 np.array([0.6, 0.75, 0.9, 1.1]), 8)
    full_compare(w, quantum, label="rdag4")


@pytest.mark.parametrize("quantum,in_sweep", [(Q, False), (0.0, False), (Q, True), (0.0, True)])
def test_2d_polynomial_on_device(quantum, in_sweep):
    """NEXT-2: the full 2-D (v, c) polynomial of Eq. (4) (N_v = N_c = 3, the
    paper's 16 coefficients) evaluated on the device -- by the
    delay kernel or inside the sweep -- on a mid-size DAG: Q mode bit-exact,
    F mode within the time tolerance."""
    nl = random_dag(99, 6000, 120, 30)
    w = Workload(0, "rdag-2d", nl, make_library(98, deg_v=3, deg_c=3), make_stimuli(97, nl.n_pi, 96),
                 np.array([0.62, 0.8, 1.05]), 8)
    full_compare(w, quantum, label=f"2d-{'sweep' if in_sweep else 'table'}", delay_in_sweep=in_sweep)


@pytest.mark.parametrize("quantum", [Q, 0.0])
def test_delay_in_sweep_identical_to_table(quantum):
    """On-the-fly delays in the sweep give bit-identical results to
    the delay table, with islands, reruns and several groups per CTA."""
    w = make_config(3, n_pairs=96, n_vdd=4, scale=0.1)
    outs = []
    for in_sweep in (False, True):
        ctx = gpu_run(w, quantum=quantum, capacity=2, delay_in_sweep=in_sweep, spill_bytes=4096)
        sig = np.arange(w.netlist.n_signals, dtype=np.int32)
        outs.append((ctx.activity(), ctx.latest_arrival(), *ctx.waveforms(sig, 0, w.n_slots, cap=24)))
        ctx.close()
    for a, b in zip(*outs):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("quantum", [Q, 0.0])
def test_overflow_reruns_equal_large_capacity(quantum):
    """Reading C17: the result is independent of capacity and of how overflow is handled.
    No spill heap: capacity 1 forces reruns 1 -> 4 -> 16 -> 64.  A 4 KiB heap: it runs
    out, the affected slot groups are rerun with larger heaps.  Default heap: every
    oversize region spills, no rerun.  All equal capacity 64 and the oracle."""
    w = make_config(2, n_pairs=64, n_vdd=2)
    st = full_compare(w, quantum, capacity=1, label="cap1-nospill", spill_bytes=-1)
    assert st["stats"]["rerun_rounds"] >= 2 and st["stats"]["overflow_slot_warps"] > 0
    assert st["stats"]["spill_bytes"] == 0
    st = full_compare(w, quantum, capacity=1, label="cap1-smallheap", spill_bytes=4096)
    assert st["stats"]["rerun_rounds"] >= 1 and st["stats"]["spill_bytes"] > 0
    st = full_compare(w, quantum, capacity=1, label="cap1-spill")
    assert st["stats"]["rerun_rounds"] == 0 and st["stats"]["spill_bytes"] > 0
    full_compare(w, quantum, capacity=64, label="cap64")


@pytest.mark.parametrize("spill_bytes", [-1, 0, 8192])
def test_overflow_exact_across_runs(spill_bytes):
    w = make_config(2, n_pairs=96, n_vdd=2)
    sig = np.arange(w.netlist.n_signals, dtype=np.int32)
    out = []
    for cap in (2, 64):
        ctx = gpu_run(w, quantum=0.0, capacity=cap, spill_bytes=spill_bytes if cap == 2 else 0)
        out.append((ctx.activity(), ctx.latest_arrival(), *ctx.waveforms(sig, 0, 192, cap=48)))
        ctx.close()
    for a, b in zip(out[0], out[1]):
        assert np.array_equal(a, b)


def test_capacity_exhausted_reports_error():
    from paper_conf_date_schneiderw20_b200 import AvfsError
    w = make_config(2, n_pairs=32, n_vdd=1)
    # simulate is asynchronous: the capacity error surfaces on sync
    with pytest.raises(AvfsError) as e:
        gpu_run(w, capacity=1, max_rerun_rounds=0, spill_bytes=-1).sync()
    assert e.value.status == 7
    with pytest.raises(AvfsError) as e:
        gpu_run(w, capacity=1, max_rerun_rounds=0, spill_bytes=64).sync()
    assert e.value.status == 7
    # ... and so does any call that reads the results
    ctx = gpu_run(w, capacity=1, max_rerun_rounds=0, spill_bytes=-1)
    with pytest.raises(AvfsError) as e:
        ctx.activity()
    assert e.value.status == 7


def test_determinism_bitwise():
    w = make_config(3, n_pairs=64, n_vdd=2, scale=0.1)
    runs = []
    for _ in range(2):
        ctx = gpu_run(w, keep_all=False)
        runs.append((ctx.activity(), ctx.latest_arrival(),
                     *ctx.waveforms(w.netlist.po_sig, 0, 128, cap=16)))
        ctx.close()
    for a, b in zip(*runs):
        assert np.array_equal(a, b)


def test_slot_range_shards_sum_to_full():
    """Disjoint slot ranges (the multi-GPU shards) reproduce the full run exactly."""
    from paper_conf_date_schneiderw20_b200 import shard_range
    w = make_config(3, n_pairs=150, n_vdd=3, scale=0.05)
    total = w.n_slots
    full = gpu_run(w, keep_all=False)
    act_full, lat_full = full.activity(), full.latest_arrival()
    po = w.netlist.po_sig
    wf_full = full.waveforms(po, 0, total, cap=16)
    full.close()
    acc = np.zeros_like(act_full)
    lat = np.zeros_like(lat_full)
    for r in range(3):
        first, n = shard_range(total, r, 3)
        ctx = gpu_run(w, keep_all=False, slot_range=(first, n))
        acc += ctx.activity()
        lat = np.maximum(lat, ctx.latest_arrival())
        wf = ctx.waveforms(po, first, n, cap=16)
        for a, b in zip(wf, wf_full):
            assert np.array_equal(a, b[:, first:first + n])
        ctx.close()
    assert np.array_equal(acc, act_full)
    assert np.array_equal(lat, lat_full)


@pytest.mark.parametrize("first,n", [(130, 40), (100, 160), (10, 430), (149, 2)])
def test_slot_range_boxes(first, n):
    """Slot ranges whose slot box wraps around the pairs (two partial rows),
    spans whole rows, or is a single row: every kept waveform and the
    activity restricted to the range equal the full run's (Q mode)."""
    w = make_config(3, n_pairs=150, n_vdd=3, scale=0.05)
    P, V = w.stimuli.n_pairs, len(w.vdd)
    po = w.netlist.po_sig
    full = gpu_run(w, keep_all=True, quantum=Q)
    sig = np.arange(w.netlist.n_signals, dtype=np.int32)
    wf_full = full.waveforms(sig, 0, w.n_slots, cap=16)
    full.close()
    ctx = gpu_run(w, keep_all=True, quantum=Q, slot_range=(first, n))
    assert ctx.stats()["slots"] == n
    wf = ctx.waveforms(sig, first, n, cap=16)
    for a, b in zip(wf, wf_full):
        assert np.array_equal(a, b[:, first:first + n])
    # activity per (signal, Vdd) = the full run's counts summed over the range
    cnt = wf_full[1][:, first:first + n].astype(np.int64)
    k = np.arange(first, first + n) // P
    want = np.zeros((w.netlist.n_signals, V), np.int64)
    for kv in range(V):
        want[:, kv] = cnt[:, k == kv].sum(1)
    assert np.array_equal(ctx.activity().astype(np.int64), want)
    ctx.close()


def test_pair_range_shards_sum_to_full():
    """Pair ranges at every operating point (the bench's multi-GPU shards,
    avfs_set_pair_range) reproduce the full run exactly: activity sums,
    latest arrival maxima, PO waveforms of the shard's slots; activity equals
    the oracle's (Q mode); slots of other pairs are refused; capture's fail
    bits cover exactly the shard's slots."""
    from paper_conf_date_schneiderw20_b200 import AvfsError, shard_pairs
    w = make_config(3, n_pairs=150, n_vdd=3, scale=0.05)
    P, V = w.stimuli.n_pairs, len(w.vdd)
    po = w.netlist.po_sig
    full = gpu_run(w, keep_all=False, quantum=Q)
    act_full, lat_full = full.activity(), full.latest_arrival()
    wf_full = full.waveforms(po, 0, w.n_slots, cap=16)
    t_clk = np.full(V, 150.0, np.float32)
    cap_full = full.capture(t_clk)
    full.close()
    acc = np.zeros_like(act_full)
    lat = np.zeros_like(lat_full)
    fails = np.zeros(V, np.int64)
    for r in range(3):
        first, n = shard_pairs(P, r, 3)
        ctx = gpu_run(w, keep_all=False, quantum=Q, pair_range=(first, n))
        st = ctx.stats()
        assert st["slots"] == n * V and st["evals"] == w.netlist.n_gates * n * V
        acc += ctx.activity()
        lat = np.maximum(lat, ctx.latest_arrival())
        for k in range(V):
            wf = ctx.waveforms(po, k * P + first, n, cap=16)
            for a, b in zip(wf, wf_full):
                assert np.array_equal(a, b[:, k * P + first:k * P + first + n])
        other = (first + n) % P
        with pytest.raises(AvfsError):
            ctx.waveforms(po, other, 1, cap=16)
        c = ctx.capture(t_clk)
        fails += c["fail_pairs"]
        fb = c["fail_bits"].reshape(V, n)                # [k][j - first]
        assert np.array_equal(fb, cap_full["fail_bits"].reshape(V, P)[:, first:first + n])
        ctx.close()
    assert np.array_equal(acc, act_full)
    assert np.array_equal(lat, lat_full)
    assert np.array_equal(fails, cap_full["fail_pairs"])
    j, k = oracle.all_slots(P, V)
    ref = oracle.simulate(w.netlist, w.library, w.stimuli, w.vdd, j, k, quantum=Q, cap=0)
    ra, ok = activity_ref(ref, V, w.netlist.n_signals)
    assert ok.all() and np.array_equal(acc.astype(np.int64), ra)


def test_permuted_gate_order_same_results():
    w = make_config(3, n_pairs=64, n_vdd=2, scale=0.05)
    perm = w.netlist.permuted(5)
    a = gpu_run(w, keep_all=True)
    b = gpu_run(w, keep_all=True, netlist=perm)
    G = w.netlist.n_gates
    n_pi = w.netlist.n_pi
    new_of_old = np.empty(G, np.int64)
    new_of_old[perm.meta["gate_perm"]] = np.arange(G)
    sig_old = np.arange(n_pi + G)
    sig_new = np.concatenate([np.arange(n_pi), n_pi + new_of_old])
    wa = a.waveforms(sig_old, 0, 128, cap=16)
    wb = b.waveforms(sig_new, 0, 128, cap=16)
    for x, y in zip(wa, wb):
        assert np.array_equal(x, y)
    assert np.array_equal(a.activity(), b.activity()[sig_new])


def test_bench_text_path_equals_array_path():
    from paper_conf_date_schneiderw20_b200 import Context
    from workloads import c17_bench_text
    w = make_config(1)
    a = gpu_run(w)
    ctx = Context(0)
    lib = w.library
    ctx.load_library(lib.names, lib.n_inputs, lib.tt, lib.deg_v, lib.deg_c, lib.beta)
    ctx.load_bench(c17_bench_text(), w.netlist.d_nom)
    ctx.set_operating_points(w.vdd)
    ctx.set_stimuli(w.stimuli.p1, w.stimuli.p2)
    ctx.set_options(capacity=8, keep_all=True)
    ctx.simulate()
    sig = np.arange(11, dtype=np.int32)
    for x, y in zip(a.waveforms(sig, 0, 96, cap=8), ctx.waveforms(sig, 0, 96, cap=8)):
        assert np.array_equal(x, y)
    assert ctx.find_signal("22") == 9


def test_edge_cases_single_pair_dup_inputs_pi_po_dangling():
    b = _Builder(3)
    g0 = b.gate("NAND2", 0, 0)          # duplicate input signal
    g1 = b.gate("XOR2", g0, 1)
    g2 = b.gate("INV", g1)               # dangling (no reader, not PO)
    g3 = b.gate("AOI21", g1, 2, 0)
    nl = b.build("edge", [g3, 2])        # PI 2 is also a PO
    nl.d_nom = np.random.default_rng(1).uniform(2, 8, size=(nl.n_edges, 2))
    nl.c_load = np.ones(nl.n_gates)
    for P in (1, 33):
        w = Workload(0, "edge", nl, make_library(3, deg_v=2), make_stimuli(4, 3, P), np.array([0.7, 1.0]), 4)
        full_compare(w, Q, label=f"edge{P}")
        full_compare(w, 0.0, label=f"edge{P}")


def test_nonpositive_delay_reported():
    from paper_conf_date_schneiderw20_b200 import AvfsError
    w = make_config(1)
    w.library = make_library(0, deg_v=1, const=-2.0)     # d' = -d_nom
    with pytest.raises(AvfsError) as e:
        gpu_run(w).sync()                                   # surfaced on sync (asynchronous simulate)
    assert e.value.status == 6


def test_api_errors_and_state():
    from paper_conf_date_schneiderw20_b200 import Context, AvfsError
    ctx = Context(0)
    with pytest.raises(AvfsError) as e:
        ctx.simulate()
    assert e.value.status == 3
    w = make_config(1)
    from paper_conf_date_schneiderw20_b200 import load_workload
    load_workload(ctx, w.netlist, w.library, w.stimuli, w.vdd)
    with pytest.raises(AvfsError):
        ctx.activity()                     # before simulate
    ctx.set_options(capacity=8)
    ctx.simulate()
    with pytest.raises(AvfsError):         # internal signal not kept
        ctx.waveforms([6], 0, 4)
    with pytest.raises(AvfsError):         # outside simulated range
        ctx.waveforms([9], 90, 10)
    ctx.close()


def test_device_stimuli_and_torch_stream():
    import torch
    from paper_conf_date_schneiderw20_b200 import Context, load_workload
    w = make_config(3, n_pairs=96, n_vdd=2, scale=0.05)
    a = gpu_run(w, keep_all=False)
    ctx = Context(0)
    load_workload(ctx, w.netlist, w.library, None, w.vdd)
    p1 = torch.from_numpy(w.stimuli.p1.view(np.int32)).cuda()
    p2 = torch.from_numpy(w.stimuli.p2.view(np.int32)).cuda()
    ctx.set_stimuli(p1, p2)
    ctx.set_options(capacity=8)
    s = torch.cuda.Stream()
    ctx.simulate(s)
    out = torch.zeros((w.netlist.n_signals, 2), dtype=torch.int64, device="cuda")
    ctx.activity(out)
    assert np.array_equal(out.cpu().numpy().astype(np.uint64), a.activity())
    # host readback into a caller-owned pinned buffer (bench.py's e2e path)
    pinned = torch.empty((w.netlist.n_signals, 2), dtype=torch.int64).pin_memory().numpy().view(np.uint64)
    assert ctx.activity(pinned) is pinned
    assert np.array_equal(pinned, a.activity())


def test_groups_per_cta_invariance(monkeypatch):
    """Narrow netlists sweep several slot groups per CTA (warps split between
    them); the result must not depend on the split (incl. idle tail warps)."""
    w = make_config(2, n_pairs=200, n_vdd=3)
    sig = np.arange(w.netlist.n_signals, dtype=np.int32)
    out = []
    for g in ("1", "2", "8", "32"):
        monkeypatch.setenv("AVFS_GROUPS_PER_CTA", g)
        ctx = gpu_run(w, quantum=0.0, capacity=8)
        out.append((ctx.activity(), ctx.latest_arrival(), *ctx.waveforms(sig, 0, w.n_slots, cap=32)))
        ctx.close()
    for o in out[1:]:
        for a, b in zip(out[0], o):
            assert np.array_equal(a, b)


def test_split_groups_invariance(monkeypatch):
    """Few slot groups: S co-resident CTAs share one group (each a 1/S slice of
    every level, cross-CTA level barrier); results must equal S = 1."""
    w = make_config(3, n_pairs=64, n_vdd=2, scale=0.1)
    sig = np.arange(w.netlist.n_signals, dtype=np.int32)
    out = []
    for sp in ("1", "2", "4"):
        monkeypatch.setenv("AVFS_SPLIT", sp)
        ctx = gpu_run(w, quantum=0.0, capacity=4)
        out.append((ctx.activity(), ctx.latest_arrival(), *ctx.waveforms(sig, 0, w.n_slots, cap=16)))
        ctx.close()
    for o in out[1:]:
        for a, b in zip(out[0], o):
            assert np.array_equal(a, b)


@pytest.mark.parametrize("quantum", [Q, 0.0])
def test_slot_batching(quantum):
    """SURVEY H5 batching: slot groups run in batches on one reused arena.
    Activity and latest arrival equal the unbatched run (and the oracle);
    the last batch's waveforms are kept, earlier ones are refused, as is capture."""
    from paper_conf_date_schneiderw20_b200 import AvfsError
    w = make_config(3, n_pairs=96, n_vdd=3, scale=0.05)
    sig = np.arange(w.netlist.n_signals, dtype=np.int32)
    a = gpu_run(w, quantum=quantum, capacity=4)
    b = gpu_run(w, quantum=quantum, capacity=4, max_batch_slots=64)      # 2 groups per batch
    assert b.stats()["batches"] == 5 and a.stats()["batches"] == 1
    assert np.array_equal(a.activity(), b.activity())
    assert np.array_equal(a.latest_arrival(), b.latest_arrival())
    # the last slot group holds the box's last 32 slots in pair-major order
    # (internal i = j * n_vdd + k): pairs 85..95 at their Vdd points
    P, V = w.stimuli.n_pairs, len(w.vdd)
    last = [(i % V) * P + i // V for i in range(P * V - 32, P * V)]
    for s in last:
        wa, wb = a.waveforms(sig, s, 1, cap=16), b.waveforms(sig, s, 1, cap=16)
        for x, y in zip(wa, wb):
            assert np.array_equal(x, y)
    with pytest.raises(AvfsError):
        b.waveforms(sig, 0, 32, cap=16)
    with pytest.raises(AvfsError):
        b.capture(np.full(3, 100.0, np.float32))
    j, k = oracle.all_slots(w.stimuli.n_pairs, len(w.vdd))
    ref = oracle.simulate(w.netlist, w.library, w.stimuli, w.vdd, j, k, quantum=quantum, cap=0)
    ra, ok = activity_ref(ref, len(w.vdd), w.netlist.n_signals)
    assert np.array_equal(b.activity().astype(np.int64)[ok], ra[ok])
    a.close()
    b.close()


def test_repeated_heap_exhaustion_counts_activity_once(monkeypatch):
    """a gate counted in round r-1 that is poisoned again in round
    r must not be counted twice.  A 4 KiB pass-0 heap and no floor on the
    rerun heaps force several heap-exhausting rerun rounds; activity, latest
    arrival and waveforms equal the run without any heap (capacity reruns)
    and the run with an ample heap."""
    monkeypatch.setenv("AVFS_RERUN_HEAP_MIN_BYTES", "16")
    w = make_config(3, n_pairs=64, n_vdd=3, scale=0.08)
    sig = np.arange(w.netlist.n_signals, dtype=np.int32)
    outs, stats = [], []
    for spill in (4096, -1, 0):
        ctx = gpu_run(w, quantum=Q, capacity=1, spill_bytes=spill, max_rerun_rounds=6)
        outs.append((ctx.activity(), ctx.latest_arrival(), *ctx.waveforms(sig, 0, w.n_slots, cap=40)))
        stats.append(ctx.stats())
        ctx.close()
    assert stats[0]["rerun_rounds"] >= 2, stats[0]
    for other in outs[1:]:
        for a, b in zip(outs[0], other):
            assert np.array_equal(a, b)
