"""Pins of the oracle's near-threshold flag / taint logic (O6, reading C13).

north_star: "the rare pulses whose width lies within tolerance of the filter
threshold are flagged and counted, not silently excluded"; PAPER.md L133
(§III-D) is why the two sides differ at all (FP64 delay model, binary32 times
on the GPU).

Reading C13 fixes the window: a binary32 time after one gate driven by a PI
event at t = 0 can be off from the FP64 time by at most
(1 + 2^-20) u (|d| + |t_out|) = (1 + 2^-20) u 2d  (u = 2^-24: one rounding of
d, one of the sum), and two events compare differently in binary32 only if
their FP64 times lie within the sum of their windows.  The tests below put the
separation of two decisive events at fractions of that window:

  * 0, 0.5 and 0.99 windows must be flagged -- a zero (or missing) window
    fails here;
  * 1.5 windows must NOT be flagged -- a window twice too wide fails here;

for both decision kinds (input order of two pins, and the inertial filter's
cancel-or-keep), plus the truth-table exemption and taint propagation.  The
last test checks soundness against an independent binary32 emulation of the
method (tests/merge_sweep.py run in numpy float32): every (signal, slot) whose
binary32 waveform differs from the FP64 oracle must be tainted.
"""
import numpy as np
import pytest

from workloads import make_library, random_dag
from workloads.netlists import _Builder
from workloads.stimuli import Stimuli, pack_bits
from tests.merge_sweep import merge_sweep, topo_order

U = 2.0 ** -24
BIG = 50.0


def _window(d):
    """Worst-case binary32 error of the output time of a gate of delay d
    driven by a PI edge at t = 0 (reading C13, stated in the module doc)."""
    return (1.0 + 2.0 ** -20) * U * 2.0 * d


def _run(oracle_mod, nl, lib, p1, p2):
    stim = Stimuli(nl.n_pi, pack_bits(np.array([p1], np.uint8)), pack_bits(np.array([p2], np.uint8)))
    return oracle_mod.simulate(nl, lib, stim, np.array([0.8]), np.array([0], np.int64),
                               np.array([0], np.int32), quantum=0.0, cap=4)


def _reconvergent(cell, d_x, d_y, with_const):
    """PI 0 rises; X = BUF(0) (rise d_x), Y = BUF(0) (rise d_y); Z = cell(X, Y[, PI 1]);
    W = BUF(Z) downstream, V = BUF(PI 1) off the cone."""
    b = _Builder(2)
    x = b.gate("BUF", 0)
    y = b.gate("BUF", 0)
    z = b.gate(cell, x, y, 1) if with_const else b.gate(cell, x, y)
    w = b.gate("BUF", z)
    v = b.gate("BUF", 1)
    nl = b.build("reconv", [w, v])
    k = 3 if with_const else 2
    nl.d_nom = np.array([[BIG, d_x], [BIG, d_y]] + [[7.0, 7.0]] * k + [[5.0, 5.0], [5.0, 5.0]], np.float64)
    return nl, (x, y, z, w, v)


LIB0 = None


def _lib0():
    global LIB0
    if LIB0 is None:
        LIB0 = make_library(0, deg_v=1, zero=True)        # d = d_nom exactly (f = 0)
    return LIB0


@pytest.mark.parametrize("frac,flagged", [(0.0, True), (0.5, True), (0.99, True), (1.5, False), (4.0, False)])
def test_o6_input_order_near_tie(oracle_mod, frac, flagged):
    d_x = 10.0
    d_y = d_x + frac * (_window(d_x) + _window(d_x + frac * _window(d_x)))
    nl, (x, y, z, w, v) = _reconvergent("AND2", d_x, d_y, with_const=False)
    r = _run(oracle_mod, nl, _lib0(), [0, 0], [1, 0])
    # the AND output rises once in every case (no filter decision involved)
    assert r.count[0, z] == 1
    assert r.flags == (1 if flagged else 0)
    assert r.taint[0, z] == flagged and r.taint[0, w] == flagged       # propagates downstream
    assert r.taint[0, x] == 0 and r.taint[0, y] == 0 and r.taint[0, v] == 0


@pytest.mark.parametrize("const,flagged", [(0, False), (1, True)])
def test_o6_truth_table_exemption(oracle_mod, const, flagged):
    """AND3 with its third input stable at 0 cannot depend on the order of
    the other two (all four truth-table values equal): exact tie, no flag.
    Stable at 1 it is an AND2: the same tie is flagged."""
    nl, (x, y, z, w, v) = _reconvergent("AND3", 10.0, 10.0, with_const=True)
    r = _run(oracle_mod, nl, _lib0(), [0, const], [1, const])
    assert r.count[0, z] == const
    assert r.flags == (1 if flagged else 0)
    assert r.taint[0, z] == flagged


def _pulse(d_inv, d_and):
    """PI 0 rises; X = INV(0) falls after d_inv; Z = AND2(0, X) rises (pin 0)
    after d_and unless X's fall cancels it first (reading C3: cancel iff the
    pending output lies after the input event); W = BUF(Z)."""
    b = _Builder(1)
    x = b.gate("INV", 0)
    z = b.gate("AND2", 0, x)
    w = b.gate("BUF", z)
    nl = b.build("pulse", [w])
    nl.d_nom = np.array([[d_inv, BIG], [BIG, d_and], [3.0, 3.0], [2.0, 2.0]], np.float64)
    return nl, (x, z, w)


@pytest.mark.parametrize("frac,flagged", [(-4.0, False), (-1.5, False), (-0.5, True), (0.0, True),
                                          (0.5, True), (0.99, True), (1.5, False), (4.0, False)])
def test_o6_filter_decision_near_threshold(oracle_mod, frac, flagged):
    d_inv = 10.0
    win = _window(d_inv) + _window(d_inv)
    d_and = d_inv + frac * win
    nl, (x, z, w) = _pulse(d_inv, d_and)
    r = _run(oracle_mod, nl, _lib0(), [0], [1])
    # the decision itself follows reading C3 exactly in FP64
    assert r.count[0, z] == (0 if d_and > d_inv else 2)
    assert r.flags == (1 if flagged else 0)
    assert r.taint[0, z] == flagged and r.taint[0, w] == flagged
    assert r.taint[0, x] == 0


def test_o6_q_mode_never_flags(oracle_mod):
    nl, _ = _pulse(10.0, 10.0)
    stim = Stimuli(1, pack_bits(np.array([[0]], np.uint8)), pack_bits(np.array([[1]], np.uint8)))
    r = oracle_mod.simulate(nl, _lib0(), stim, np.array([0.8]), np.array([0], np.int64),
                            np.array([0], np.int32), quantum=2.0 ** -8, cap=4)
    assert r.flags == 0 and r.taint.sum() == 0


def test_o6_sound_against_binary32_emulation(oracle_mod):
    """Random DAGs with tie-prone decimal delays (0.1 + 0.2 != 0.3 in FP64,
    == in binary32): simulate every slot with the independent merge-sweep
    formulation in numpy float32 (d rounded once to binary32, binary32 sums,
    as the GPU path computes).  Every (signal, slot) whose binary32 waveform
    differs from the FP64 oracle (count, or a time beyond the north_star
    tolerance) must be tainted; and such differences must occur."""
    lib = make_library(0, deg_v=0, zero=True)
    mix = {"NAND2": .2, "NOR2": .1, "XOR2": .2, "XNOR2": .1, "INV": .1, "AOI21": .1, "OAI21": .1, "AND2": .1}
    steps = np.array([0.1, 0.2, 0.3, 0.4, 0.6, 0.7])
    differ = tainted_differ = untainted = tainted = 0
    for case in range(60):
        rng = np.random.default_rng(8100 + case)
        nl = random_dag(8200 + case, int(rng.integers(8, 30)), int(rng.integers(3, 6)), int(rng.integers(3, 7)),
                        mix=mix)
        nl.d_nom = rng.choice(steps, size=nl.d_nom.shape)
        P = 16
        b1 = (rng.random((P, nl.n_pi)) < 0.5).astype(np.uint8)
        b2 = b1 ^ (rng.random((P, nl.n_pi)) < 0.6).astype(np.uint8)
        stim = Stimuli(nl.n_pi, pack_bits(b1), pack_bits(b2))
        r = oracle_mod.simulate(nl, lib, stim, np.array([0.8]), np.arange(P, dtype=np.int64),
                                np.zeros(P, np.int32), quantum=0.0, cap=64)
        assert r.count.max() < 64
        order = topo_order(nl)
        for j in range(P):
            _, wf = merge_sweep(nl, lib, b1[j], b2[j],
                                lambda g, p, y: np.float32(nl.d_nom[nl.fanin_ptr[g] + p, y]), order)
            for s in range(nl.n_signals):
                t32 = np.array(wf[s], np.float64)
                n = r.count[j, s]
                same = len(t32) == n and np.all(np.abs(t32 - r.times[j, s, :n]) <= 1e-5 * np.abs(r.times[j, s, :n]) + 1e-3)
                if r.taint[j, s]:
                    tainted += 1
                    tainted_differ += not same
                else:
                    untainted += 1
                    assert same, (case, j, s, wf[s], r.times[j, s, :n])
                differ += not same
    assert differ >= 10, differ                 # binary32 really flips decisions here
    assert tainted_differ == differ
    assert untainted > 2 * tainted              # the window is not so wide that it taints everything
