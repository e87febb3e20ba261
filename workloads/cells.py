"""Synthetic truth-table cell set and polynomial delay-coefficient library.

The paper characterises NanGate 15 nm cells by SPICE + regression
(§III-A, Fig. 1); those data are not available, so the
coefficients here are synthetic, calibrated to the delay-vs-Vdd ratios
Table II prints for s38584 (846.0 / 590.1 / 485.0 ps at
0.55 / 0.8 / 1.1 V, i.e. ratios 1.434 / 1.0 / 0.822).  SURVEY.md §8(d).

Coefficient layout (reading C9): beta[cell][pin<4][pol][i][j],
pol 0 = output falls, 1 = output rises; i = power of phi_V(v), j = power of
phi_C(c) (Eq. 4; L117 normalisations).
"""
from __future__ import annotations

from dataclasses import dataclass
from itertools import product

import numpy as np

V_MIN, V_MAX = 0.55, 1.1          # PAPER.md L179 (regression range), reading C10
C_MIN, C_MAX = 0.5, 128.0         # fF

# Base f(phi_V) with f(0)=0.434, f(phi_V(0.8))~0, f(1)=-0.178 (s38584 ratios,
# PAPER.md L238).  Quadratic for config 1 (N_v=2), cubic for configs 2-5.
BASE_BETA_QUAD = (0.434, -1.24047, 0.62847)
BASE_BETA_CUBIC = (0.43363, -1.49901, 1.45832, -0.57104)


def _tt(n: int, fn) -> int:
    """Truth table: bit b is fn(inputs) with input pin p = bit p of b."""
    tt = 0
    for b in range(1 << n):
        bits = [(b >> p) & 1 for p in range(n)]
        tt |= (int(bool(fn(bits))) << b)
    return tt


# (name, n_inputs, logic function)
_CELL_DEFS = [
    ("INV", 1, lambda x: not x[0]),
    ("BUF", 1, lambda x: x[0]),
    ("NAND2", 2, lambda x: not (x[0] and x[1])),
    ("NOR2", 2, lambda x: not (x[0] or x[1])),
    ("AND2", 2, lambda x: x[0] and x[1]),
    ("OR2", 2, lambda x: x[0] or x[1]),
    ("XOR2", 2, lambda x: x[0] ^ x[1]),
    ("XNOR2", 2, lambda x: not (x[0] ^ x[1])),
    ("NAND3", 3, lambda x: not (x[0] and x[1] and x[2])),
    ("NOR3", 3, lambda x: not (x[0] or x[1] or x[2])),
    ("AND3", 3, lambda x: x[0] and x[1] and x[2]),
    ("OR3", 3, lambda x: x[0] or x[1] or x[2]),
    ("AOI21", 3, lambda x: not ((x[0] and x[1]) or x[2])),
    ("OAI21", 3, lambda x: not ((x[0] or x[1]) and x[2])),
    ("NAND4", 4, lambda x: not (x[0] and x[1] and x[2] and x[3])),
    ("NOR4", 4, lambda x: not (x[0] or x[1] or x[2] or x[3])),
    ("AOI22", 4, lambda x: not ((x[0] and x[1]) or (x[2] and x[3]))),
    ("OAI22", 4, lambda x: not ((x[0] or x[1]) and (x[2] or x[3]))),
]

CELLS = [(name, n, _tt(n, fn)) for name, n, fn in _CELL_DEFS]
CELL_INDEX = {name: i for i, (name, _, _) in enumerate(CELLS)}

# intrinsic nominal delay per cell type in ps (SURVEY.md §8(d) random-DAG rules)
INTRINSIC_PS = {
    "INV": 3.0, "BUF": 6.0, "NAND2": 5.0, "NOR2": 6.0, "AND2": 8.0, "OR2": 9.0,
    "XOR2": 10.0, "XNOR2": 10.0, "NAND3": 6.0, "NOR3": 7.5, "AND3": 8.0,
    "OR3": 8.0, "AOI21": 7.0, "OAI21": 7.0, "NAND4": 7.0, "NOR4": 8.5,
    "AOI22": 7.5, "OAI22": 7.5,
}


@dataclass
class Library:
    names: list
    n_inputs: np.ndarray      # int32 [n_cells]
    tt: np.ndarray            # uint16 [n_cells]
    deg_v: int
    deg_c: int
    beta: np.ndarray          # float64 [n_cells][4][2][deg_v+1][deg_c+1]
    v_min: float = V_MIN
    v_max: float = V_MAX
    c_min: float = C_MIN
    c_max: float = C_MAX

    @property
    def n_cells(self) -> int:
        return len(self.names)


def make_library(seed: int, deg_v: int = 3, deg_c: int = 0,
                 spread: float = 0.2, zero: bool = False,
                 const: float | None = None) -> Library:
    """Per (cell, pin, pol): base polynomial x U(1-spread, 1+spread).

    deg_v=2 uses BASE_BETA_QUAD, 3 the cubic; other degrees pad/truncate the
    cubic.  deg_c>0 adds a small synthetic load dependence in phi_C (the paper's
    general 2-D model, Eq. 4); the configs use deg_c=0 (reading C8).
    zero=True gives beta == 0 (static delays, test T2); const=x gives
    beta_00 = x and all else 0 (test T3).
    """
    rng = np.random.default_rng(seed)
    n = len(CELLS)
    beta = np.zeros((n, 4, 2, deg_v + 1, deg_c + 1), dtype=np.float64)
    if zero:
        pass
    elif const is not None:
        beta[..., 0, 0] = const
    else:
        base = BASE_BETA_QUAD if deg_v == 2 else BASE_BETA_CUBIC
        base = np.array([base[i] if i < len(base) else 0.0 for i in range(deg_v + 1)])
        scale = rng.uniform(1.0 - spread, 1.0 + spread, size=(n, 4, 2))
        beta[..., 0] = scale[..., None] * base[None, None, None, :]
        if deg_c > 0:
            # heavier loads slow the cell: +0..30 % across phi_C in [0,1],
            # stronger at low voltage.  Synthetic; only shapes the test inputs.
            cj = rng.uniform(0.05, 0.15, size=(n, 4, 2, deg_c))
            for j in range(1, deg_c + 1):
                beta[..., 0, j] = cj[..., j - 1] / j
                if deg_v >= 1:
                    beta[..., 1, j] = -0.5 * cj[..., j - 1] / j
    return Library(
        names=[c[0] for c in CELLS],
        n_inputs=np.array([c[1] for c in CELLS], dtype=np.int32),
        tt=np.array([c[2] for c in CELLS], dtype=np.uint16),
        deg_v=deg_v, deg_c=deg_c, beta=beta,
    )


def all_input_vectors(n: int):
    return list(product((0, 1), repeat=n))
