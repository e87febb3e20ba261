"""The five BASELINE.json configurations (SURVEY.md §8(d) input recipes).

Seeds: netlist 1000+i, library/delays 2000+i, stimuli 3000+i for config i.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .cells import Library, make_library
from .netlists import Netlist, c17, array_multiplier, random_dag
from .stimuli import Stimuli, make_stimuli

CONFIG_NAMES = {
    1: "c17",
    2: "c6288-shaped",
    3: "b17-shaped",
    4: "b19-shaped",
    5: "synthetic-2M",
}


@dataclass
class Workload:
    cfg: int
    name: str
    netlist: Netlist
    library: Library
    stimuli: Stimuli
    vdd: np.ndarray          # float64 [n_vdd] volts
    capacity: int            # waveform capacity parameter C (transitions / slot, per slot-warp average)

    @property
    def n_slots(self) -> int:
        return self.stimuli.n_pairs * len(self.vdd)

    @property
    def evals(self) -> int:
        return self.netlist.n_gates * self.n_slots

    def describe(self) -> dict:
        return {
            "workload": self.name, "cfg": self.cfg, "gates": self.netlist.n_gates,
            "pis": self.netlist.n_pi, "pos": int(len(self.netlist.po_sig)),
            "pairs": self.stimuli.n_pairs, "vdd_points": int(len(self.vdd)),
            "deg_v": self.library.deg_v, "deg_c": self.library.deg_c, "capacity": self.capacity,
        }


def make_config(i: int, n_pairs: int | None = None, n_vdd: int | None = None,
                scale: float = 1.0, deg_c: int = 0) -> Workload:
    """Build config i (1..5).  n_pairs / n_vdd / scale shrink it for tests.
    deg_c > 0 (configs 2-5): the paper's 2-D (v, c) delay model with N_c =
    deg_c (Table I uses N_v = N_c = 3)."""
    if i == 1:
        nl = c17(seed=2001)
        lib = make_library(2001, deg_v=2, spread=0.1)
        P = n_pairs or 32
        stim = make_stimuli(3001, nl.n_pi, P, toggle=0.5)
        vdd = np.array([0.8, 0.9, 1.0])
        cap = 8
    elif i == 2:
        nl = array_multiplier(16, seed=2002)
        lib = make_library(2002, deg_v=3, deg_c=deg_c, spread=0.2)
        P = n_pairs or 10_000
        stim = make_stimuli(3002, nl.n_pi, P, toggle=0.5)
        vdd = np.linspace(0.6, 1.1, 8)
        cap = 32
    elif i in (3, 4, 5):
        G, PI, PO, L, P0, V0, cap = {
            3: (30_000, 1452, 1512, 60, 4096, 16, 8),
            4: (200_000, 6663, 6672, 80, 2048, 32, 12),   # pilot: C = 8 overflows 42/2048 groups
            5: (2_000_000, 50_000, 50_000, 120, 1024, 51, 4),
        }[i]
        G = max(64, int(G * scale))
        PI = max(8, int(PI * scale))
        PO = max(4, int(PO * scale))
        mix = None
        if i == 5:
            from .netlists import DEFAULT_MIX
            mix = dict(DEFAULT_MIX)
            mix["XOR2"] += 0.01
            mix["XNOR2"] += 0.01
        nl = random_dag(1000 + i, G, PI, L, n_po_min=PO, mix=mix,
                        delay_seed=2000 + i, name=CONFIG_NAMES[i])
        lib = make_library(2000 + i, deg_v=3, deg_c=deg_c, spread=0.2)
        P = n_pairs or P0
        stim = make_stimuli(3000 + i, nl.n_pi, P, toggle=0.5)
        vdd = (np.linspace(0.6, 1.1, V0) if i != 5 else 0.6 + 0.01 * np.arange(51))
    else:
        raise ValueError(f"unknown config {i}")
    if n_vdd is not None:
        vdd = vdd[np.linspace(0, len(vdd) - 1, n_vdd).round().astype(int)]
    return Workload(cfg=i, name=CONFIG_NAMES[i], netlist=nl, library=lib,
                    stimuli=stim, vdd=np.ascontiguousarray(vdd, dtype=np.float64),
                    capacity=cap)
