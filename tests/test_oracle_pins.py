"""Pins of the oracle against what the paper and mathematics fix (-m "not gpu").

Each test names the pin of SURVEY.md §8(c) / DESIGN.md it implements.  None
of them re-types the oracle's formula: they use numpy's polyval2d, closed
forms, brute force, or the independent merge-sweep formulation in
tests/merge_sweep.py.
"""
import numpy as np
import pytest

from workloads import make_config, make_library, random_dag, make_stimuli, exhaustive_pairs
from workloads.cells import CELL_INDEX, BASE_BETA_QUAD, BASE_BETA_CUBIC
from workloads.netlists import _Builder, c17, array_multiplier
from workloads.stimuli import Stimuli, pack_bits
from tests.merge_sweep import merge_sweep, static_eval, topo_order

Q = 2.0 ** -8


def phi_v(v, lo=0.55, hi=1.1):
    return (v - lo) / (hi - lo)


def poly_delay(lib, nl, g, pin, pol, v):
    """Eq. (4)+(9) via numpy.polyval2d (test-side, independent of the oracle's Horner)."""
    b = lib.beta[nl.gate_cell[g], pin, pol]
    x = phi_v(v, lib.v_min, lib.v_max)
    z = 0.0
    if lib.deg_c:
        c = nl.c_load[g]
        z = (np.log2(c) - np.log2(lib.c_min)) / (np.log2(lib.c_max) - np.log2(lib.c_min))
    f = np.polynomial.polynomial.polyval2d(x, z, b)
    return nl.d_nom[nl.fanin_ptr[g] + pin, pol] * (1.0 + f)


# ---------------------------------------------------------------- T1
@pytest.mark.parametrize("dv,dc", [(0, 0), (1, 0), (2, 0), (3, 0), (3, 3), (2, 1), (5, 2)])
def test_t1_delay_matches_polyval2d(oracle_mod, dv, dc):
    rng = np.random.default_rng(100 + 10 * dv + dc)
    eps = np.finfo(np.float64).eps
    for _ in range(300):
        beta = rng.normal(size=(dv + 1, dc + 1)) * 0.5
        v = rng.uniform(0.55, 1.1)
        c = 2.0 ** rng.uniform(-1, 7)
        dnom = rng.uniform(1, 20)
        x = phi_v(v)
        z = (np.log2(c) - np.log2(0.5)) / (np.log2(128.0) - np.log2(0.5))
        ref = dnom * (1.0 + np.polynomial.polynomial.polyval2d(x, z, beta))
        got = oracle_mod.delay(beta, dnom, v, c)
        bound = 16 * eps * dnom * (1.0 + np.abs(beta).sum())
        assert abs(got - ref) <= bound, (got, ref)


def test_t1_special_points(oracle_mod):
    # v = V_min: phi_V = 0 so f = beta_00 exactly (Horner with x = 0).
    b = np.array([[0.25], [3.0], [-7.0]])
    assert oracle_mod.delay(b, 8.0, 0.55) == 8.0 * 1.25
    # v = V_max: phi_V = 1, f = sum(beta) (exact for these dyadic values)
    assert oracle_mod.delay(b, 8.0, 1.1) == 8.0 * (1 + 0.25 + 3.0 - 7.0)
    # Q mode rounds half to even on the quantum grid
    assert oracle_mod.delay(np.zeros((1, 1)), 3 * Q + Q / 2, 0.8, quantum=Q) == 4 * Q
    assert oracle_mod.delay(np.zeros((1, 1)), 2 * Q + Q / 2, 0.8, quantum=Q) == 2 * Q


@pytest.mark.parametrize("base", [BASE_BETA_QUAD, BASE_BETA_CUBIC])
def test_t1_calibration_matches_table2_ratios(oracle_mod, base):
    """Synthetic beta reproduce the s38584 delay ratios of Table II."""
    b = np.array(base)[:, None]
    r = [oracle_mod.delay(b, 1.0, v) for v in (0.55, 0.8, 1.1)]
    assert abs(r[0] - 846.0 / 590.1) < 2e-3
    assert abs(r[1] - 1.0) < 1e-3
    assert abs(r[2] - 485.0 / 590.1) < 2e-3


# ---------------------------------------------------------------- helpers
def small_dag(seed, G=200, n_pi=16, depth=12, mix=None):
    return random_dag(seed, G, n_pi, depth, mix=mix, delay_seed=seed + 1)


def run_all(oracle_mod, nl, lib, stim, vdd, quantum=0.0, cap=16):
    j, k = oracle_mod.all_slots(stim.n_pairs, len(vdd))
    return oracle_mod.simulate(nl, lib, stim, vdd, j, k, quantum=quantum, cap=cap)


# ---------------------------------------------------------------- T2
def test_t2_degree0_static_and_vdd_invariant(oracle_mod):
    nl = small_dag(7)
    lib = make_library(1, deg_v=0, zero=True)
    stim = make_stimuli(11, nl.n_pi, 24)
    vdd = np.array([0.6, 0.8, 1.1])
    r = run_all(oracle_mod, nl, lib, stim, vdd, cap=32)
    assert r.count.max() < 32
    P = stim.n_pairs
    for k in (1, 2):                      # identical across operating points
        assert np.array_equal(r.count[k * P:(k + 1) * P], r.count[:P])
        assert np.array_equal(r.times[k * P:(k + 1) * P], r.times[:P])
    order = topo_order(nl)
    b1, b2 = stim.bits(1), stim.bits(2)
    for j in range(P):                    # equal to static-delay simulation (d = d_nom)
        init, wf = merge_sweep(nl, lib, b1[j], b2[j],
                               lambda g, p, y: nl.d_nom[nl.fanin_ptr[g] + p, y], order)
        assert np.array_equal(r.init[j], init)
        for s in range(nl.n_signals):
            assert r.count[j, s] == len(wf[s])
            assert np.array_equal(r.times[j, s, :len(wf[s])], np.array(wf[s]))


# ---------------------------------------------------------------- T3
def test_t3_uniform_scale_doubles_times(oracle_mod):
    nl = small_dag(8, mix={"NAND2": 0.4, "XOR2": 0.3, "INV": 0.3})
    nl.d_nom = np.round(nl.d_nom / Q) * Q           # on the quantum grid
    stim = make_stimuli(12, nl.n_pi, 32)
    vdd = np.array([0.7, 1.0])
    r0 = run_all(oracle_mod, nl, make_library(1, deg_v=2, zero=True), stim, vdd, quantum=Q, cap=40)
    r1 = run_all(oracle_mod, nl, make_library(1, deg_v=2, const=1.0), stim, vdd, quantum=Q, cap=40)
    assert r0.count.max() < 40
    assert np.array_equal(r0.count, r1.count)
    assert np.array_equal(r0.init, r1.init)
    assert np.array_equal(2.0 * r0.times, r1.times)
    assert r0.count.sum() > 0


# ---------------------------------------------------------------- T4
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_t4_inv_buf_chain_closed_form(oracle_mod, seed):
    rng = np.random.default_rng(seed)
    n = 40
    b = _Builder(1)
    s = 0
    kinds = rng.choice(["INV", "BUF"], size=n)
    for kd in kinds:
        s = b.gate(str(kd), s)
    nl = b.build("chain", [s])
    nl.d_nom = rng.uniform(2.0, 12.0, size=(n, 2))
    lib = make_library(seed, deg_v=3)
    vdd = np.array([0.6, 0.8, 1.05])
    for start in (0, 1):
        stim = Stimuli(1, pack_bits(np.array([[start]], np.uint8)), pack_bits(np.array([[1 - start]], np.uint8)))
        r = run_all(oracle_mod, nl, lib, stim, vdd, cap=2)
        for k, v in enumerate(vdd):
            assert r.count[k, 0] == 1 and r.times[k, 0, 0] == 0.0
            t, val = 0.0, 1 - start
            for g in range(n):
                val = 1 - val if kinds[g] == "INV" else val
                t += poly_delay(lib, nl, g, 0, val, v)
                assert r.count[k, 1 + g] == 1
                assert abs(r.times[k, 1 + g, 0] - t) <= 1e-9 * t


# ---------------------------------------------------------------- T5
def _pulse_net(d_buf0_r, d_inv_f, d_and_r0, d_and_f1, d_buf3_r):
    b = _Builder(1)
    g0 = b.gate("BUF", 0)          # delta
    g1 = b.gate("INV", g0)
    g2 = b.gate("AND2", 0, g1)     # pulse generator
    g3 = b.gate("BUF", g2)         # single-input pulse filter
    nl = b.build("pulse", [g2, g3])
    big = 50.0
    nl.d_nom = np.array([[big, d_buf0_r], [d_inv_f, big], [big, d_and_r0], [d_and_f1, big],
                         [big, d_buf3_r]], dtype=np.float64)
    return nl


def test_t5_pulse_threshold_equality_kept(oracle_mod):
    lib = make_library(0, deg_v=1, zero=True)
    stim = Stimuli(1, pack_bits(np.array([[0]], np.uint8)), pack_bits(np.array([[1]], np.uint8)))
    vdd = np.array([0.8])
    d_inv_f, d_and_r0, d_and_f1 = 3 * 256 * Q, 9 * 256 * Q, 4 * 256 * Q
    thr = d_and_r0 - d_inv_f                       # cancel iff d_and_r0 > delta + d_inv_f
    for m, expect in ((-2, 0), (-1, 0), (0, 2), (1, 2)):
        delta = thr + m * Q
        nl = _pulse_net(delta, d_inv_f, d_and_r0, d_and_f1, 1.0)
        r = run_all(oracle_mod, nl, lib, stim, vdd, quantum=Q, cap=4)
        g2 = 1 + 2
        assert r.count[0, g2] == expect, (m, r.count[0])
        if expect:
            assert r.times[0, g2, 0] == d_and_r0
            assert r.times[0, g2, 1] == delta + d_inv_f + d_and_f1
    # BUF passes a rising pulse iff width >= d_rise (reading C3 ii)
    delta = thr + 8 * Q
    w = delta + d_inv_f + d_and_f1 - d_and_r0
    for m, expect in ((-1, 2), (0, 2), (1, 0)):
        nl = _pulse_net(delta, d_inv_f, d_and_r0, d_and_f1, w + m * Q)
        r = run_all(oracle_mod, nl, lib, stim, vdd, quantum=Q, cap=4)
        assert r.count[0, 1 + 3] == expect, (m, r.count[0])


# ---------------------------------------------------------------- T6
def test_t6_c17_exhaustive(oracle_mod):
    nl = c17()
    lib = make_library(2001, deg_v=2, spread=0.1)
    stim = exhaustive_pairs(5)
    vdd = np.array([0.8, 0.9, 1.0])
    r = run_all(oracle_mod, nl, lib, stim, vdd, cap=8)
    assert r.count.max() <= 8
    b1, b2 = stim.bits(1), stim.bits(2)
    order = topo_order(nl)
    e1 = np.array([static_eval(nl, lib, b, order) for b in b1])
    e2 = np.array([static_eval(nl, lib, b, order) for b in b2])
    P = stim.n_pairs
    for k in range(3):
        sl = slice(k * P, (k + 1) * P)
        assert np.array_equal(r.init[sl], e1)
        assert np.array_equal(r.final[sl], e2)
        assert np.array_equal((r.count[sl] & 1).astype(np.uint8), e1 ^ e2)
    # times strictly increasing and > 0 for gate outputs, == 0 for PIs
    for s in range(nl.n_signals):
        for i in range(len(r.count)):
            n = r.count[i, s]
            t = r.times[i, s, :n]
            if s < nl.n_pi:
                assert n <= 1 and (n == 0 or t[0] == 0.0)
            else:
                assert np.all(t > 0) and np.all(np.diff(t) > 0)


# ---------------------------------------------------------------- T7
def test_oracle_sta_matches_path_enumeration(oracle_mod):
    nl = small_dag(21, G=14, n_pi=4, depth=4)
    lib = make_library(3, deg_v=3)
    vdd = np.array([0.65, 1.0])
    amax, amin = oracle_mod.sta(nl, lib, vdd)
    n_pi = nl.n_pi

    def paths(s, v):      # all path sums into signal s (brute force)
        if s < n_pi:
            return [0.0]
        g = s - n_pi
        out = []
        for p, src in enumerate(nl.fanin_sig[nl.fanin_ptr[g]:nl.fanin_ptr[g + 1]]):
            for a in paths(src, v):
                for pol in (0, 1):
                    out.append(a + poly_delay(lib, nl, g, p, pol, v))
        return out
    for k, v in enumerate(vdd):
        for s in range(nl.n_signals):
            ps = paths(s, v)
            assert abs(amax[k, s] - max(ps)) <= 1e-9 * max(1.0, max(ps))
            assert abs(amin[k, s] - min(ps)) <= 1e-9 * max(1.0, min(ps))


def test_t7_transitions_within_sta_bounds(oracle_mod):
    nl = small_dag(22, G=400, n_pi=24, depth=20, mix={"NAND2": .3, "XOR2": .2, "NOR2": .2, "INV": .1, "AOI21": .2})
    lib = make_library(4, deg_v=3)
    vdd = np.array([0.6, 0.8, 1.1])
    stim = make_stimuli(5, nl.n_pi, 32)
    r = run_all(oracle_mod, nl, lib, stim, vdd, cap=64)
    assert r.count.max() <= 64
    amax, amin = oracle_mod.sta(nl, lib, vdd)
    P = stim.n_pairs
    for i in range(len(r.count)):
        k = i // P
        n = r.count[i]
        has = n > 0
        first = r.times[i, :, 0]
        last = r.times[i, np.arange(nl.n_signals), np.maximum(n - 1, 0)]
        assert np.all(last[has] <= amax[k][has])
        assert np.all(first[has] >= amin[k][has])


# ---------------------------------------------------------------- T8
def test_t8_event_queue_equals_merge_sweep(oracle_mod):
    """3-4 hundred tiny DAGs with integer delays (exact ties are common)."""
    lib = make_library(0, deg_v=0, zero=True)
    mix = {"NAND2": .2, "NOR2": .1, "XOR2": .2, "XNOR2": .1, "INV": .1, "AOI21": .1, "OAI21": .1, "NAND4": .05, "AOI22": .05}
    multi = 0
    for case in range(300):
        rng = np.random.default_rng(5000 + case)
        G = int(rng.integers(3, 26))
        nl = random_dag(7000 + case, G, int(rng.integers(4, 7)), int(rng.integers(2, 7)), mix=mix)
        nl.d_nom = rng.integers(1, 7, size=nl.d_nom.shape).astype(np.float64)
        stim = make_stimuli(9000 + case, nl.n_pi, 4)
        r = run_all(oracle_mod, nl, lib, stim, np.array([0.8]), quantum=1.0, cap=64)
        order = topo_order(nl)
        b1, b2 = stim.bits(1), stim.bits(2)
        for j in range(stim.n_pairs):
            init, wf = merge_sweep(nl, lib, b1[j], b2[j],
                                   lambda g, p, y: nl.d_nom[nl.fanin_ptr[g] + p, y], order)
            assert np.array_equal(r.init[j], init), case
            for s in range(nl.n_signals):
                assert r.count[j, s] == len(wf[s]), (case, j, s)
                assert np.array_equal(r.times[j, s, :len(wf[s])], wf[s]), (case, j, s)
                multi += len(wf[s]) > 1
    assert multi > 100          # glitches actually exercised


# ---------------------------------------------------------------- T9
def test_t9_structural_invariants(oracle_mod):
    nl = small_dag(31, G=300, n_pi=20, depth=15)
    lib = make_library(6, deg_v=3)
    vdd = np.array([0.6, 1.1])
    stim = make_stimuli(7, nl.n_pi, 32)
    r = run_all(oracle_mod, nl, lib, stim, vdd, cap=64)
    assert r.count.max() <= 64
    P = stim.n_pairs
    for i in range(len(r.count)):
        v = vdd[i // P]
        assert np.all(r.count[i, :nl.n_pi] <= 1)
        for g in range(nl.n_gates):
            ins = nl.fanin_sig[nl.fanin_ptr[g]:nl.fanin_ptr[g + 1]]
            n = r.count[i, nl.n_pi + g]
            assert n <= r.count[i, ins].sum()
            if n > 1:     # inertial filter: consecutive outputs >= min arc delay apart
                dmin = min(poly_delay(lib, nl, g, p, pol, v) for p in range(len(ins)) for pol in (0, 1))
                assert np.all(np.diff(r.times[i, nl.n_pi + g, :n]) >= dmin * (1 - 1e-12))


# ---------------------------------------------------------------- multiplier brute force
def test_multiplier_final_values_are_products(oracle_mod):
    nl = array_multiplier(16)
    lib = make_library(2002, deg_v=3)
    stim = make_stimuli(3002, nl.n_pi, 48)
    vdd = np.array([0.6, 1.1])
    r = oracle_mod.simulate(nl, lib, stim, vdd, *oracle_mod.all_slots(48, 2), cap=0, out_sig=nl.po_sig)
    for which, vals in ((1, r.init), (2, r.final)):
        bits = stim.bits(which).astype(np.int64)
        a = (bits[:, :16] << np.arange(16)).sum(1)
        b = (bits[:, 16:] << np.arange(16)).sum(1)
        prod = a * b
        got = (vals.astype(np.int64) << np.arange(32)).sum(1)
        assert np.array_equal(got, np.tile(prod, 2))
    assert r.count.max() > 2          # glitch-heavy


def test_oracle_fmode_flags_are_rare_and_counted(oracle_mod):
    w = make_config(2, n_pairs=32, n_vdd=2)
    r = oracle_mod.simulate(w.netlist, w.library, w.stimuli, w.vdd, *oracle_mod.all_slots(32, 2), cap=0)
    assert r.taint.mean() < 0.1
    rq = oracle_mod.simulate(w.netlist, w.library, w.stimuli, w.vdd, *oracle_mod.all_slots(32, 2), cap=0, quantum=Q)
    assert rq.flags == 0 and rq.taint.sum() == 0


# ---------------------------------------------------------------- NEXT-2 islands
def test_islands_chain_closed_form(oracle_mod):
    """Per-gate supplies: each stage of a chain uses its own island's voltage."""
    rng = np.random.default_rng(9)
    n = 24
    b = _Builder(1)
    s = 0
    kinds = rng.choice(["INV", "BUF"], size=n)
    for kd in kinds:
        s = b.gate(str(kd), s)
    nl = b.build("chain", [s])
    nl.d_nom = rng.uniform(2.0, 12.0, size=(n, 2))
    lib = make_library(5, deg_v=3)
    island = rng.integers(0, 3, size=n).astype(np.int32)
    vdd = np.array([[0.6, 0.9, 1.1], [1.0, 0.7, 0.8]])
    stim = Stimuli(1, pack_bits(np.array([[0]], np.uint8)), pack_bits(np.array([[1]], np.uint8)))
    j, k = oracle_mod.all_slots(1, 2)
    r = oracle_mod.simulate(nl, lib, stim, vdd, j, k, cap=2, island=island)
    for kk in range(2):
        t, val = 0.0, 1
        for g in range(n):
            val = 1 - val if kinds[g] == "INV" else val
            t += poly_delay(lib, nl, g, 0, val, vdd[kk, island[g]])
            assert abs(r.times[kk, 1 + g, 0] - t) <= 1e-9 * t


def test_islands_equal_supplies_reduce_to_single_supply(oracle_mod):
    nl = small_dag(41, G=300, n_pi=16, depth=12)
    lib = make_library(7, deg_v=3)
    stim = make_stimuli(8, nl.n_pi, 16)
    vdd = np.array([0.65, 0.95])
    island = (np.arange(nl.n_gates) % 4).astype(np.int32)
    j, k = oracle_mod.all_slots(16, 2)
    a = oracle_mod.simulate(nl, lib, stim, vdd, j, k, cap=32)
    b = oracle_mod.simulate(nl, lib, stim, np.repeat(vdd[:, None], 4, axis=1), j, k, cap=32, island=island)
    assert np.array_equal(a.count, b.count) and np.array_equal(a.times, b.times)
