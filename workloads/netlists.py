"""Seeded combinational netlists shaped like the paper's workloads.

Signal numbering used everywhere (library, oracle, tests): primary inputs are
signals 0..n_pi-1, gate g drives signal n_pi+g.  Gates need not be in
topological order (the library levelises; the oracle sorts on its own).

* c17: the textbook ISCAS'85 netlist (6 NAND2), config 1.
* array_multiplier: a c6288-shaped 16x16 array multiplier built from AND2
  partial products and NOR2 full/half adders (c6288 itself is a NOR-based
  array multiplier of 2406 gates; its file is not available here), config 2.
* random_dag: levelised random DAG with the SURVEY.md §8(d) cell mix and
  fan-in rules, configs 3-5 (b17/b19-shaped and the 2M synthetic).

Nominal delays follow SURVEY.md §8(d): per fan-in edge and output polarity
(pin-to-pin with polarity).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from .cells import CELLS, CELL_INDEX, INTRINSIC_PS

C17_BENCH = """# c17 (ISCAS'85)
INPUT(1)
INPUT(2)
INPUT(3)
INPUT(6)
INPUT(7)
OUTPUT(22)
OUTPUT(23)
10 = NAND(1, 3)
11 = NAND(3, 6)
16 = NAND(2, 11)
19 = NAND(11, 7)
22 = NAND(10, 16)
23 = NAND(16, 19)
"""


def c17_bench_text() -> str:
    return C17_BENCH


@dataclass
class Netlist:
    name: str
    n_pi: int
    gate_cell: np.ndarray      # int32 [G]
    fanin_ptr: np.ndarray      # int64 [G+1]
    fanin_sig: np.ndarray      # int32 [E]
    po_sig: np.ndarray         # int32 [n_po]
    d_nom: np.ndarray = None   # float64 [E][2]  (pol 0 = output falls, 1 = rises)
    c_load: np.ndarray = None  # float64 [G] fF
    meta: dict = field(default_factory=dict)

    @property
    def n_gates(self) -> int:
        return int(self.gate_cell.shape[0])

    @property
    def n_signals(self) -> int:
        return self.n_pi + self.n_gates

    @property
    def n_edges(self) -> int:
        return int(self.fanin_sig.shape[0])

    def fanout_counts(self) -> np.ndarray:
        """Number of gate input pins reading each signal [n_signals]."""
        return np.bincount(self.fanin_sig, minlength=self.n_signals).astype(np.int64)

    def permuted(self, seed: int) -> "Netlist":
        """Same circuit with gates stored in a random order (signal ids remapped)."""
        rng = np.random.default_rng(seed)
        G = self.n_gates
        perm = rng.permutation(G)            # new gate i = old gate perm[i]
        inv = np.empty(G, dtype=np.int64)
        inv[perm] = np.arange(G)
        remap = np.concatenate([np.arange(self.n_pi), self.n_pi + inv]).astype(np.int32)
        k = np.diff(self.fanin_ptr)
        new_ptr = np.zeros(G + 1, dtype=np.int64)
        new_ptr[1:] = np.cumsum(k[perm])
        new_sig = np.empty_like(self.fanin_sig)
        new_dn = None if self.d_nom is None else np.empty_like(self.d_nom)
        for i, g in enumerate(perm):
            a, b = self.fanin_ptr[g], self.fanin_ptr[g + 1]
            new_sig[new_ptr[i]:new_ptr[i + 1]] = remap[self.fanin_sig[a:b]]
            if new_dn is not None:
                new_dn[new_ptr[i]:new_ptr[i + 1]] = self.d_nom[a:b]
        return Netlist(
            name=self.name + "-perm", n_pi=self.n_pi,
            gate_cell=self.gate_cell[perm].copy(), fanin_ptr=new_ptr, fanin_sig=new_sig,
            po_sig=remap[self.po_sig], d_nom=new_dn,
            c_load=None if self.c_load is None else self.c_load[perm].copy(),
            meta=dict(self.meta, gate_perm=perm),
        )


class _Builder:
    def __init__(self, n_pi: int):
        self.n_pi = n_pi
        self.cells, self.fanins = [], []

    def gate(self, cell: str, *ins: int) -> int:
        assert len(ins) == CELLS[CELL_INDEX[cell]][1]
        self.cells.append(CELL_INDEX[cell])
        self.fanins.append(list(ins))
        return self.n_pi + len(self.cells) - 1

    def build(self, name: str, po: list) -> Netlist:
        k = np.array([len(f) for f in self.fanins], dtype=np.int64)
        ptr = np.zeros(len(k) + 1, dtype=np.int64)
        ptr[1:] = np.cumsum(k)
        sig = np.array([s for f in self.fanins for s in f], dtype=np.int32)
        return Netlist(name=name, n_pi=self.n_pi,
                       gate_cell=np.array(self.cells, dtype=np.int32),
                       fanin_ptr=ptr, fanin_sig=sig,
                       po_sig=np.array(po, dtype=np.int32))


def c17(seed: int = 2001) -> Netlist:
    """ISCAS'85 c17; PIs 1,2,3,6,7 -> 0..4; gates 10,11,16,19,22,23 -> 5..10.

    Nominal delays: NAND2 fall 6 ps, rise 8 ps,
    each (edge, pol) x U(0.9, 1.1).
    """
    b = _Builder(5)
    s = {"1": 0, "2": 1, "3": 2, "6": 3, "7": 4}
    s["10"] = b.gate("NAND2", s["1"], s["3"])
    s["11"] = b.gate("NAND2", s["3"], s["6"])
    s["16"] = b.gate("NAND2", s["2"], s["11"])
    s["19"] = b.gate("NAND2", s["11"], s["7"])
    s["22"] = b.gate("NAND2", s["10"], s["16"])
    s["23"] = b.gate("NAND2", s["16"], s["19"])
    nl = b.build("c17", [s["22"], s["23"]])
    rng = np.random.default_rng(seed)
    base = np.array([6.0, 8.0])
    nl.d_nom = base[None, :] * rng.uniform(0.9, 1.1, size=(nl.n_edges, 2))
    nl.c_load = _c_load(nl)
    nl.meta["names"] = {v: k for k, v in s.items()}
    return nl


def _nor_xnor(b: _Builder, x: int, y: int):
    n1 = b.gate("NOR2", x, y)
    n2 = b.gate("NOR2", x, n1)
    n3 = b.gate("NOR2", y, n1)
    return n1, b.gate("NOR2", n2, n3)          # (NOR(x,y), XNOR(x,y))


def _full_adder(b: _Builder, x: int, y: int, z: int):
    """9-NOR full adder: sum = x^y^z, carry = maj(x,y,z)."""
    n1, xn = _nor_xnor(b, x, y)
    n5 = b.gate("NOR2", xn, z)
    n6 = b.gate("NOR2", xn, n5)
    n7 = b.gate("NOR2", z, n5)
    s = b.gate("NOR2", n6, n7)
    c = b.gate("NOR2", n1, n5)
    return s, c


def _half_adder(b: _Builder, x: int, y: int):
    """NOR half adder: 4 NOR2 XNOR, INV, carry = NOR(NOR(x,y), sum)."""
    n1, xn = _nor_xnor(b, x, y)
    s = b.gate("INV", xn)
    c = b.gate("NOR2", n1, s)
    return s, c


def array_multiplier(n: int = 16, seed: int = 2002) -> Netlist:
    """c6288-shaped n x n carry-save array multiplier.

    PIs: a_0..a_{n-1} (signals 0..n-1), b_0..b_{n-1} (n..2n-1).
    POs: product bits p_0..p_{2n-1} (LSB first).
    """
    b = _Builder(2 * n)
    A = list(range(n))
    B = list(range(n, 2 * n))
    pp = [[b.gate("AND2", A[j], B[i]) for j in range(n)] for i in range(n)]
    sums = list(pp[0])                  # weight j
    carries = [None] * n                # carries[j] of row i has weight i+j+1
    out = [sums[0]]

    def add(*xs):
        xs = [x for x in xs if x is not None]
        if len(xs) == 3:
            return _full_adder(b, *xs)
        if len(xs) == 2:
            return _half_adder(b, *xs)
        return xs[0], None

    for i in range(1, n):
        ns, nc = [], []
        for j in range(n):
            s_in = sums[j + 1] if j + 1 < n else None
            s, c = add(pp[i][j], s_in, carries[j])
            ns.append(s)
            nc.append(c)
        out.append(ns[0])
        sums, carries = ns, nc
    rc = None
    for j in range(n):
        s_in = sums[j + 1] if j + 1 < n else None
        s, rc = add(s_in, carries[j], rc)
        out.append(s)
    assert rc is None or len(out) == 2 * n
    nl = b.build(f"mult{n}x{n}", out[:2 * n])
    assign_delays(nl, seed)
    return nl


DEFAULT_MIX = {
    "INV": 0.20, "BUF": 0.05, "NAND2": 0.25, "NOR2": 0.15, "AND2": 0.10,
    "OR2": 0.08, "NAND3": 0.035, "NOR3": 0.035, "AOI21": 0.03, "OAI21": 0.03,
    "XOR2": 0.02, "XNOR2": 0.02,
}


def random_dag(seed: int, n_gates: int, n_pi: int, depth: int, n_po_min: int = 0,
               mix: dict | None = None, pi_prob: float = 0.05,
               delay_seed: int | None = None, name: str = "rdag") -> Netlist:
    """Levelised random DAG (SURVEY.md §8(d) random-DAG rules).

    Pin 0 of a level-L gate reads level L-1 (fixing the level) through a
    permutation so every level-(L-1) signal gets a reader when widths allow;
    the other pins read level L-1-Geom(0.5) (PIs with prob pi_prob).  Level
    widths follow a tapered diamond.  POs: every unread gate output, topped
    up from the deepest levels to n_po_min.
    """
    rng = np.random.default_rng(seed)
    depth = max(1, min(depth, n_gates))
    mix = mix or DEFAULT_MIX
    names = list(mix)
    probs = np.array([mix[k] for k in names], dtype=np.float64)
    probs /= probs.sum()
    cell_ids = np.array([CELL_INDEX[k] for k in names], dtype=np.int32)
    n_in_of = np.array([c[1] for c in CELLS], dtype=np.int64)

    lv = np.arange(1, depth + 1)
    prof = 0.3 + np.sin(np.pi * (lv - 0.5) / depth)
    w = np.maximum(1, np.floor(prof / prof.sum() * n_gates)).astype(np.int64)
    diff = n_gates - int(w.sum())
    mid = np.argsort(-prof)
    i = 0
    while diff != 0:
        j = mid[i % depth]
        if diff > 0:
            w[j] += 1
            diff -= 1
        elif w[j] > 1:
            w[j] -= 1
            diff += 1
        i += 1
    start = np.zeros(depth + 1, dtype=np.int64)
    start[1:] = np.cumsum(w)            # gates of level l (1-based) are start[l-1]..start[l]-1

    cell = cell_ids[rng.choice(len(names), size=n_gates, p=probs)]
    k = n_in_of[cell]
    kmax = int(k.max())
    F = np.full((n_gates, kmax), -1, dtype=np.int64)
    for l in range(1, depth + 1):
        a, b_ = start[l - 1], start[l]
        m = b_ - a
        kk = k[a:b_]
        if l == 1:
            for r in range(m):
                F[a + r, :kk[r]] = rng.choice(n_pi, size=kk[r], replace=False)
            continue
        pa, pb = start[l - 2], start[l - 1]     # previous level gate range
        pw = pb - pa
        reps = -(-m // pw)
        perm = np.concatenate([rng.permutation(pw) for _ in range(reps)])[:m]
        F[a:b_, 0] = n_pi + pa + perm
        for p in range(1, kmax):
            act = kk > p
            back = rng.geometric(0.5, size=m) - 1          # 0,1,2,... w.p. 1/2,1/4,..
            src_lvl = np.maximum(l - 1 - back, 0)
            src_lvl[rng.random(m) < pi_prob] = 0
            sig = np.empty(m, dtype=np.int64)
            is_pi = src_lvl == 0
            sig[is_pi] = rng.integers(0, n_pi, size=int(is_pi.sum()))
            g_l = src_lvl[~is_pi]
            lo, hi = start[g_l - 1], start[g_l]
            sig[~is_pi] = n_pi + lo + (rng.random(len(g_l)) * (hi - lo)).astype(np.int64)
            for _ in range(4):   # redraw duplicates among this gate's pins from level L-1
                dup = act & np.any(F[a:b_, :p] == sig[:, None], axis=1)
                if not dup.any():
                    break
                sig[dup] = n_pi + pa + rng.integers(0, pw, size=int(dup.sum()))
            F[a:b_, p] = np.where(act, sig, -1)
    fanin_sig = F[F >= 0].astype(np.int32)          # row-major keeps pin order
    ptr = np.zeros(n_gates + 1, dtype=np.int64)
    ptr[1:] = np.cumsum(k)
    nl = Netlist(name=name, n_pi=n_pi, gate_cell=cell.astype(np.int32),
                 fanin_ptr=ptr, fanin_sig=fanin_sig, po_sig=np.zeros(0, np.int32))
    fo = nl.fanout_counts()
    unread = np.nonzero(fo[n_pi:] == 0)[0] + n_pi
    po = list(unread)
    if len(po) < n_po_min:
        cand = np.arange(n_pi + start[max(0, depth - max(2, depth // 5))], n_pi + n_gates)
        cand = np.setdiff1d(cand, unread)
        extra = rng.choice(cand, size=min(len(cand), n_po_min - len(po)), replace=False)
        po += list(extra)
    nl.po_sig = np.sort(np.array(po, dtype=np.int32))
    nl.meta["level_widths"] = w
    assign_delays(nl, seed + 1000 if delay_seed is None else delay_seed)
    return nl


def _c_load(nl: Netlist) -> np.ndarray:
    fo = nl.fanout_counts()[nl.n_pi:]
    return np.clip(0.6 * fo + 0.2, 0.5, 128.0)


def assign_delays(nl: Netlist, seed: int) -> None:
    """Synthetic SDF-like annotation.

    d_nom(edge, pol) = (intrinsic(cell) + 0.8 ps x fanout) x U(0.85,1.15)[gate,pol]
                       x U(0.95,1.05)[edge] x lognormal(0, 0.05)[edge,pol]
    c_load = 0.6 fF x fanout + 0.2 fF clipped to [0.5, 128] fF.
    """
    rng = np.random.default_rng(seed)
    G = nl.n_gates
    fo = nl.fanout_counts()[nl.n_pi:]
    intr = np.array([INTRINSIC_PS[CELLS[c][0]] for c in nl.gate_cell])
    base = intr + 0.8 * fo                                   # [G]
    asym = rng.uniform(0.85, 1.15, size=(G, 2))
    k = np.diff(nl.fanin_ptr)
    gate_of_edge = np.repeat(np.arange(G), k)
    skew = rng.uniform(0.95, 1.05, size=nl.n_edges)
    jit = rng.lognormal(0.0, 0.05, size=(nl.n_edges, 2))
    nl.d_nom = (base[gate_of_edge, None] * asym[gate_of_edge] * skew[:, None] * jit)
    nl.c_load = _c_load(nl)
