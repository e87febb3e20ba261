"""ORACLE -- TEST INFRASTRUCTURE ONLY.

FP64 event-driven CPU reference for the hot path of Schneider & Wunderlich,
DATE'20 (see oracle.c for the per-function citations).  Only `tests/`,
`__graft_entry__.smoke()` and `bench.py` (cpu_baseline / --impl reference)
may import this package.  The product path
(`paper_conf_date_schneiderw20_b200`) must never import it, and it never
imports the product path.  It consumes the plain numpy inputs of
`workloads/` (generators only; no method arithmetic there).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-std=c11", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
               "-shared", "-fPIC", "-Wall", "-o", _LIB, _SRC, "-lm"]
        subprocess.check_call(cmd)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = C.CDLL(_LIB)
        P = C.c_void_p
        lib.oracle_delay.restype = C.c_double
        lib.oracle_delay.argtypes = [P, C.c_int, C.c_int, C.c_double, C.c_double, C.c_double,
                                     C.c_double, C.c_double, C.c_double, C.c_double, C.c_double]
        lib.oracle_sta.restype = C.c_int
        lib.oracle_sta.argtypes = [C.c_int32, C.c_int32, P, P, P, P, P, P, P, C.c_int32, C.c_int32, P,
                                   C.c_double, C.c_double, C.c_double, C.c_double,
                                   C.c_int32, P, C.c_double, P, C.c_int32, P, P]
        lib.oracle_simulate.restype = C.c_int
        lib.oracle_simulate.argtypes = [C.c_int32, C.c_int32, P, P, P, P, P, P, P, C.c_int32, C.c_int32, P,
                                        C.c_double, C.c_double, C.c_double, C.c_double,
                                        C.c_int32, P, P, P, C.c_double, P, C.c_int32,
                                        C.c_int64, P, P, C.c_int32, P, C.c_int32,
                                        P, P, P, P, P, C.c_int32]
        lib.oracle_max_threads.restype = C.c_int
        _lib = lib
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def delay(beta_cpp, d_nom, v, c=1.0, v_min=0.55, v_max=1.1, c_min=0.5, c_max=128.0, quantum=0.0):
    """Eq. (4)+(9) for one arc; beta_cpp is [deg_v+1][deg_c+1] float64."""
    b = _c(beta_cpp, np.float64)
    dv, dc = b.shape[0] - 1, b.shape[1] - 1
    return float(_load().oracle_delay(_p(b), dv, dc, float(d_nom), float(v), float(c),
                                      v_min, v_max, c_min, c_max, float(quantum)))


def _net_args(nl, lib):
    keep = [_c(nl.gate_cell, np.int32), _c(nl.fanin_ptr, np.int64), _c(nl.fanin_sig, np.int32),
            _c(nl.d_nom, np.float64),
            None if (nl.c_load is None or lib.deg_c == 0) else _c(nl.c_load, np.float64),
            _c(lib.n_inputs, np.int32), _c(lib.tt, np.uint16), _c(lib.beta, np.float64)]
    args = [nl.n_pi, nl.n_gates, _p(keep[0]), _p(keep[1]), _p(keep[2]), _p(keep[3]), _p(keep[4]),
            _p(keep[5]), _p(keep[6]), lib.deg_v, lib.deg_c, _p(keep[7]),
            lib.v_min, lib.v_max, lib.c_min, lib.c_max]
    return keep, args


def _islands(vdd, island):
    """vdd [n_points] (one supply) or [n_points][n_isl] with island[gate]."""
    v = _c(vdd, np.float64)
    if v.ndim == 1:
        return v, None, 1
    isl = _c(island, np.int32)
    return v, isl, int(v.shape[1])


def sta(nl, lib, vdd, quantum=0.0, island=None):
    """Longest / shortest path arrival per (Vdd, signal): (arr_max, arr_min)."""
    vdd, isl, n_isl = _islands(vdd, island)
    amax = np.zeros((len(vdd), nl.n_signals))
    amin = np.zeros((len(vdd), nl.n_signals))
    keep, args = _net_args(nl, lib)
    rc = _load().oracle_sta(*args, len(vdd), _p(vdd), float(quantum), _p(isl), n_isl, _p(amax), _p(amin))
    if rc:
        raise RuntimeError(f"oracle_sta failed: {rc}")
    return amax, amin


@dataclass
class OracleResult:
    count: np.ndarray     # int32 [n_slots][n_out]
    init: np.ndarray      # uint8 [n_slots][n_out]
    times: np.ndarray     # float64 [n_slots][n_out][cap] (0-padded) or None
    taint: np.ndarray     # uint8 [n_slots][n_out]
    flags: int
    out_sig: np.ndarray   # signals in column order

    @property
    def final(self) -> np.ndarray:
        return self.init ^ (self.count & 1).astype(np.uint8)


def simulate(nl, lib, stim, vdd, slot_pair, slot_vdd, quantum=0.0, cap=8,
             out_sig=None, threads=0, island=None) -> OracleResult:
    """Simulate slots (pair slot_pair[s], operating point slot_vdd[s]).
    vdd: [n_points] volts, or [n_points][n_isl] with island[gate] (NEXT-2)."""
    vdd, isl, n_isl = _islands(vdd, island)
    sp = _c(slot_pair, np.int64)
    sv = _c(slot_vdd, np.int32)
    n_slots = len(sp)
    if out_sig is None:
        out_sig = np.arange(nl.n_signals, dtype=np.int32)
    out_sig = _c(out_sig, np.int32)
    n_out = len(out_sig)
    count = np.zeros((n_slots, n_out), np.int32)
    init = np.zeros((n_slots, n_out), np.uint8)
    taint = np.zeros((n_slots, n_out), np.uint8)
    times = np.zeros((n_slots, n_out, cap), np.float64) if cap > 0 else None
    flags = np.zeros(1, np.int64)
    p1, p2 = _c(stim.p1, np.uint32), _c(stim.p2, np.uint32)
    keep, args = _net_args(nl, lib)
    rc = _load().oracle_simulate(*args, stim.words, _p(p1), _p(p2), _p(vdd), float(quantum), _p(isl), n_isl,
                                 n_slots, _p(sp), _p(sv), n_out, _p(out_sig), int(cap),
                                 _p(count), _p(init), _p(times), _p(taint), _p(flags), int(threads))
    if rc:
        raise RuntimeError(f"oracle_simulate failed: {rc}")
    return OracleResult(count, init, times, taint, int(flags[0]), out_sig)


def all_slots(n_pairs: int, n_vdd: int):
    """Every (pair, Vdd) slot, Vdd-major (slot = k*n_pairs + j)."""
    k, j = np.divmod(np.arange(n_pairs * n_vdd), n_pairs)
    return j.astype(np.int64), k.astype(np.int32)
