"""Second, independent formulation of the waveform semantics (pin T8).

The oracle processes a global event queue (O4).  This module instead sweeps
the netlist gate by gate in topological order and, per gate, merges the
already-complete input waveforms by (time, pin) -- the "waveform processing
loop" view of P:L160 / [25] -- applying reading C3 (cancel the last output
event iff it lies after the input event, equality kept), C4 (no reschedule on
confirming events) and C5 (ascending pin order on ties).  Pure Python, for
small cases only.  Used only by tests to pin the oracle.
"""
from __future__ import annotations

import numpy as np


def topo_order(nl) -> list:
    """Gates in topological order by repeated relaxation of levels."""
    G, n_pi = nl.n_gates, nl.n_pi
    lvl = np.zeros(nl.n_signals, dtype=np.int64)
    for _ in range(G + 1):
        changed = False
        for g in range(G):
            ins = nl.fanin_sig[nl.fanin_ptr[g]:nl.fanin_ptr[g + 1]]
            v = 1 + max(lvl[s] for s in ins)
            if v != lvl[n_pi + g]:
                lvl[n_pi + g] = v
                changed = True
        if not changed:
            break
    else:
        raise ValueError("cycle")
    return sorted(range(G), key=lambda g: (lvl[n_pi + g], g))


def static_eval(nl, lib, pi_bits, order=None) -> np.ndarray:
    """Boolean value of every signal for one input vector."""
    order = order if order is not None else topo_order(nl)
    val = np.zeros(nl.n_signals, dtype=np.uint8)
    val[:nl.n_pi] = pi_bits
    for g in order:
        ins = nl.fanin_sig[nl.fanin_ptr[g]:nl.fanin_ptr[g + 1]]
        b = sum(int(val[s]) << p for p, s in enumerate(ins))
        val[nl.n_pi + g] = (int(lib.tt[nl.gate_cell[g]]) >> b) & 1
    return val


def merge_sweep(nl, lib, p1_bits, p2_bits, delay_fn, order=None):
    """Waveforms (init, [times]) of every signal for one slot.

    delay_fn(g, pin, pol) -> delay in ps (pol 1 = output rises).
    """
    order = order if order is not None else topo_order(nl)
    init = static_eval(nl, lib, p1_bits, order)
    wf = [[] for _ in range(nl.n_signals)]
    for i in range(nl.n_pi):
        if p1_bits[i] != p2_bits[i]:
            wf[i] = [0.0]
    for g in order:
        ins = list(nl.fanin_sig[nl.fanin_ptr[g]:nl.fanin_ptr[g + 1]])
        tt = int(lib.tt[nl.gate_cell[g]])
        bits = sum(int(init[s]) << p for p, s in enumerate(ins))
        proj = (tt >> bits) & 1
        events = sorted((t, p) for p, s in enumerate(ins) for t in wf[s])
        out = []
        for t, p in events:
            bits ^= 1 << p
            y = (tt >> bits) & 1
            if y == proj:
                continue
            proj = y
            if out and out[-1] > t:
                out.pop()
            else:
                out.append(t + delay_fn(g, p, y))
        wf[nl.n_pi + g] = out
    return init, wf
