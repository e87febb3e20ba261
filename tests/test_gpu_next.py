"""NEXT rows on the GPU vs the oracle (-m gpu): capture / test-response
analysis (NEXT-1) and switching energy (NEXT-4)."""
import numpy as np
import pytest

import oracle
from workloads import make_config
from tests.parity import Q, gpu_run

pytestmark = pytest.mark.gpu


def capture_ref(ref, nl, P, V, t_clk, lo, width, n_bins):
    """From oracle PO waveforms: fail flags, per-PO fail counts, slack histogram."""
    n = ref.count                      # [slot][po]
    T = np.repeat(np.asarray(t_clk, np.float64), P)[:, None]
    cap = ref.times.shape[2]
    idx = np.arange(cap)[None, None, :]
    valid = idx < n[:, :, None]
    c = ((ref.times <= T[:, :, None]) & valid).sum(2)
    fail_po_slot = ((ref.init ^ (c & 1)) != (ref.init ^ (n & 1)))
    fail = fail_po_slot.any(1)
    last = np.where(valid, ref.times, 0.0).max(2).max(1)
    slack = T[:, 0] - last
    k = np.arange(P * V) // P
    fail_pairs = np.bincount(k, weights=fail, minlength=V).astype(np.int64)
    fail_po = np.stack([np.bincount(k, weights=fail_po_slot[:, o], minlength=V) for o in range(n.shape[1])]).astype(np.int64)
    b = np.clip(np.floor((slack - lo) / width).astype(np.int64), 0, n_bins - 1)
    hist = np.zeros((V, n_bins), np.int64)
    np.add.at(hist, (k, b), 1)
    return fail, fail_pairs, fail_po, hist


@pytest.mark.parametrize("cfg", [2, 3])
def test_capture_matches_oracle_q_mode(cfg):
    w = make_config(cfg, n_pairs=70, n_vdd=3, scale=0.1)
    nl = w.netlist
    P, V = w.stimuli.n_pairs, len(w.vdd)
    j, k = oracle.all_slots(P, V)
    ref = oracle.simulate(nl, w.library, w.stimuli, w.vdd, j, k, quantum=Q, cap=128, out_sig=nl.po_sig)
    assert ref.count.max() < 128
    ctx = gpu_run(w, quantum=Q, keep_all=False, capacity=32)
    lat = ctx.latest_arrival().astype(np.float64)
    # capture at the per-Vdd median of the pairs' last PO transition, on the
    # quantum grid (comparisons are then exact in binary32)
    valid = np.arange(ref.times.shape[2])[None, None, :] < ref.count[:, :, None]
    last = np.where(valid, ref.times, 0.0).max(2).max(1).reshape(V, P)
    t_clk = np.round(np.median(last, axis=1) / Q) * Q + Q / 2
    lo, width, nb = -256.0, 8.0, 96
    out = ctx.capture(t_clk.astype(np.float32), n_bins=nb, lo_ps=lo, width_ps=width)
    fail, fp, fpo, hist = capture_ref(ref, nl, P, V, t_clk, lo, width, nb)
    assert np.array_equal(out["fail_bits"].astype(bool), fail)
    assert np.array_equal(out["fail_pairs"].astype(np.int64), fp)
    assert np.array_equal(out["fail_po"].astype(np.int64), fpo)
    assert np.array_equal(out["slack_hist"].astype(np.int64), hist)
    assert fp.sum() > 0 and fp.sum() < P * V        # the clock actually separates pairs
    # a generous clock passes everything
    out2 = ctx.capture((lat + 10.0).astype(np.float32), n_bins=nb, lo_ps=lo, width_ps=width)
    assert out2["fail_pairs"].sum() == 0
    ctx.close()


def test_switching_energy_matches_oracle_counts():
    w = make_config(3, n_pairs=64, n_vdd=4, scale=0.05)
    nl = w.netlist
    P, V = w.stimuli.n_pairs, len(w.vdd)
    j, k = oracle.all_slots(P, V)
    ref = oracle.simulate(nl, w.library, w.stimuli, w.vdd, j, k, quantum=Q, cap=0)
    act = ref.count.reshape(V, P, -1).sum(1)[:, nl.n_pi:]          # [V][G]
    want = 0.5 * (act * nl.c_load[None, :]).sum(1) * w.vdd ** 2
    ctx = gpu_run(w, quantum=Q, keep_all=False)
    got = ctx.switching_energy()
    assert np.allclose(got, want, rtol=1e-12, atol=0)
    assert np.all(want > 0) and np.all(np.diff(want / w.vdd ** 2) != 0)   # per-Vdd activity differs
    ctx.close()


@pytest.mark.parametrize("quantum", [Q, 0.0])
def test_voltage_islands_parity(quantum):
    """NEXT-2: per-gate supplies (3 islands x 4 operating points) vs the oracle."""
    from paper_conf_date_schneiderw20_b200 import Context, load_workload
    from tests.parity import gpu_waveforms, compare, activity_ref
    w = make_config(3, n_pairs=72, n_vdd=4, scale=0.05)
    nl = w.netlist
    rng = np.random.default_rng(11)
    island = rng.integers(0, 3, size=nl.n_gates).astype(np.int32)
    vdd = np.array([[0.6, 0.8, 1.1], [0.7, 0.7, 0.7], [1.0, 0.65, 0.9], [1.1, 1.1, 0.6]])
    P, V = w.stimuli.n_pairs, vdd.shape[0]
    j, k = oracle.all_slots(P, V)
    ref = oracle.simulate(nl, w.library, w.stimuli, vdd, j, k, quantum=quantum, cap=64, island=island)
    ctx = Context(0)
    load_workload(ctx, nl, w.library, w.stimuli, vdd[:, 0])
    ctx.set_voltage_islands(island, vdd)
    ctx.set_options(capacity=8, quantum_ps=quantum, keep_all=True)
    ctx.simulate()
    init, cnt, times = gpu_waveforms(ctx, np.arange(nl.n_signals), 0, P * V, int(ref.count.max()) or 1)
    compare(ref, init, cnt, times, quantum, "islands")
    act = ctx.activity().astype(np.int64)
    ra, ok = activity_ref(ref, V, nl.n_signals)
    assert np.array_equal(act[ok], ra[ok])
    e = ctx.switching_energy()
    vg = vdd[:, island]                                  # [V][G]
    want = 0.5 * (ra[nl.n_pi:].T * nl.c_load[None, :] * vg ** 2).sum(1)
    if quantum > 0:
        assert np.allclose(e, want, rtol=1e-12)
    ctx.close()
