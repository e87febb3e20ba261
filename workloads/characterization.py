"""Synthetic cell-delay ground truth for the regression pre-process (NEXT-3).

The paper characterises cells by SPICE sweeps (Fig. 1 step A) on the
grid V in [0.55, 1.1] V step 0.05, C_load in {2^-1 .. 2^7} fF.  No SPICE
or cell library is available, so the ground truth here is the alpha-power law
(Eq. 1) times the logical-effort model (Eq. 2):
    d(v, c) = k * v / (v - V_th)^alpha * (g * c / c_in + p)
with per-arc parameters drawn from plausible ranges.  Inputs only: the fit
itself lives in the library (avfs_fit_delay_polynomial) and the oracle.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

PAPER_V = np.round(np.arange(0.55, 1.1 + 1e-9, 0.05), 10)     # 12 points
PAPER_C = 2.0 ** np.arange(-1, 8)                              # 0.5 .. 128 fF, 9 points
V_NOM = 0.8                                                    # nominal supply


@dataclass
class Arc:
    k: float
    v_th: float
    alpha: float
    g: float
    p: float
    c_in: float

    def delay(self, v, c):
        v = np.asarray(v, np.float64)
        c = np.asarray(c, np.float64)
        return self.k * v / (v - self.v_th) ** self.alpha * (self.g * c / self.c_in + self.p)

    def d_nom(self, c):
        """nominal delay at load c (the SDF annotation of a gate driving c)"""
        return self.delay(V_NOM, c)


def make_arcs(seed: int, n: int) -> list:
    rng = np.random.default_rng(seed)
    return [Arc(k=float(rng.uniform(1.0, 3.0)), v_th=float(rng.uniform(0.25, 0.33)),
                alpha=float(rng.uniform(1.2, 1.7)), g=float(rng.uniform(1.0, 2.2)),
                p=float(rng.uniform(0.6, 2.0)), c_in=float(rng.uniform(0.8, 2.0))) for _ in range(n)]


def paper_grid_samples(arc: Arc):
    """(v, c, y) on the paper's 12 x 9 characterisation grid, with
    y = d(v, c) / d(V_nom, c) - 1: the deviation from the nominal-voltage delay
    at the same load (reading C7: Eq. 9 scales the gate's own annotated delay)."""
    vv, cc = np.meshgrid(PAPER_V, PAPER_C, indexing="ij")
    v, c = vv.ravel(), cc.ravel()
    return v, c, arc.delay(v, c) / arc.delay(V_NOM, c) - 1.0


def eval_grid(n: int = 64, v_min=0.55, v_max=1.1, c_min=0.5, c_max=128.0):
    """n x n grid equidistant in the normalised coordinates (phi_V, phi_C)."""
    x = np.linspace(0.0, 1.0, n)
    v = v_min + x * (v_max - v_min)
    c = 2.0 ** (np.log2(c_min) + x * (np.log2(c_max) - np.log2(c_min)))
    vv, cc = np.meshgrid(v, c, indexing="ij")
    return vv.ravel(), cc.ravel()
