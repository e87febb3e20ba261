"""Thin ctypes binding of libavfs (include/avfs.h).  Argument marshalling only:
every step of the simulation runs in the library's CUDA kernels.  Fails loudly
(ImportError / AvfsError) when the extension is missing -- there is no CPU
fallback on the product path.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libavfs.so")

STATUS = {0: "AVFS_OK", 1: "AVFS_ERR_ARG", 2: "AVFS_ERR_PARSE", 3: "AVFS_ERR_STATE", 4: "AVFS_ERR_CUDA",
          5: "AVFS_ERR_NOMEM", 6: "AVFS_ERR_DELAY_NONPOS", 7: "AVFS_ERR_CAPACITY"}

# every symbol include/avfs.h declares
EXPORTS = [
    "avfs_create", "avfs_destroy", "avfs_last_error", "avfs_status_string", "avfs_version",
    "avfs_load_library", "avfs_load_netlist", "avfs_load_bench", "avfs_find_signal",
    "avfs_get_netlist_info", "avfs_get_levels", "avfs_get_buffer_map",
    "avfs_set_operating_points", "avfs_set_voltage_islands", "avfs_set_stimuli", "avfs_set_slot_range", "avfs_set_pair_range",
    "avfs_set_options", "avfs_default_options", "avfs_simulate", "avfs_sync",
    "avfs_get_activity", "avfs_get_latest_arrival", "avfs_get_final_values",
    "avfs_get_waveforms", "avfs_get_stats", "avfs_capture", "avfs_get_switching_energy",
    "avfs_fit_delay_polynomial", "avfs_debug_phase_cycles", "avfs_get_timing",
]


class AvfsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class avfs_cell(C.Structure):
    _fields_ = [("name", C.c_char_p), ("n_inputs", C.c_int32), ("truth_table", C.c_uint16)]


class avfs_netlist_info(C.Structure):
    _fields_ = [("n_pi", C.c_int32), ("n_gates", C.c_int32), ("n_po", C.c_int32), ("depth", C.c_int32),
                ("max_fanin", C.c_int32), ("n_scratch_buffers", C.c_int32), ("n_pinned", C.c_int32),
                ("n_dangling", C.c_int32), ("n_edges", C.c_int64)]


class avfs_options(C.Structure):
    _fields_ = [("capacity", C.c_int32), ("quantum_ps", C.c_double), ("n_probe", C.c_int32),
                ("probe_sig", C.POINTER(C.c_int32)), ("keep_all", C.c_int32),
                ("max_rerun_rounds", C.c_int32), ("warps_per_cta", C.c_int32), ("profile", C.c_int32),
                ("spill_bytes", C.c_int64), ("max_batch_slots", C.c_int64), ("delay_in_sweep", C.c_int32)]


class avfs_stats(C.Structure):
    _fields_ = [("evals", C.c_int64), ("slots", C.c_int64), ("slot_warps", C.c_int64),
                ("overflow_slot_warps", C.c_int64), ("rerun_rounds", C.c_int64), ("launches", C.c_int64),
                ("arena_bytes", C.c_int64), ("alg_bytes", C.c_int64), ("grid", C.c_int32),
                ("warps_per_cta", C.c_int32), ("n_scratch_buffers", C.c_int32), ("n_pinned", C.c_int32),
                ("sim_ms", C.c_double), ("sweep_ms", C.c_double), ("spill_bytes", C.c_int64),
                ("spill_heap_bytes", C.c_int64), ("batches", C.c_int64), ("enc_bytes", C.c_int64),
                ("rerun_ms", C.c_double)]

    def as_dict(self) -> dict:
        return {f: getattr(self, f) for f, _ in self._fields_}


_lib = None


def load_library(path: str = LIB_PATH):
    """Load libavfs.so (raises if it has not been built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(path):
            raise ImportError(f"libavfs.so not built at {path}; run __graft_entry__.build()")
        lib = C.CDLL(path)
        P, I32, I64, D = C.c_void_p, C.c_int32, C.c_int64, C.c_double
        sig = {
            "avfs_create": ([C.c_int, C.POINTER(P)], C.c_int),
            "avfs_destroy": ([P], None),
            "avfs_last_error": ([P], C.c_char_p),
            "avfs_status_string": ([C.c_int], C.c_char_p),
            "avfs_version": ([], C.c_char_p),
            "avfs_load_library": ([P, I32, P, I32, I32, P, D, D, D, D], C.c_int),
            "avfs_load_netlist": ([P, I32, I32, P, P, P, P, P, I32, P], C.c_int),
            "avfs_load_bench": ([P, C.c_char_p, C.c_size_t, P, P], C.c_int),
            "avfs_find_signal": ([P, C.c_char_p, C.POINTER(I32)], C.c_int),
            "avfs_get_netlist_info": ([P, P], C.c_int),
            "avfs_get_levels": ([P, P], C.c_int),
            "avfs_get_buffer_map": ([P, P], C.c_int),
            "avfs_set_operating_points": ([P, I32, P], C.c_int),
            "avfs_set_voltage_islands": ([P, I32, P, I32, P], C.c_int),
            "avfs_set_stimuli": ([P, I64, P, P, I32], C.c_int),
            "avfs_set_slot_range": ([P, I64, I64], C.c_int),
            "avfs_set_pair_range": ([P, I64, I64], C.c_int),
            "avfs_set_options": ([P, P], C.c_int),
            "avfs_default_options": ([P], C.c_int),
            "avfs_simulate": ([P, P], C.c_int),
            "avfs_sync": ([P], C.c_int),
            "avfs_get_activity": ([P, P, I32], C.c_int),
            "avfs_get_latest_arrival": ([P, P, I32], C.c_int),
            "avfs_get_final_values": ([P, I32, P, I64, I64, P], C.c_int),
            "avfs_get_waveforms": ([P, I32, P, I64, I64, I32, P, P, P], C.c_int),
            "avfs_get_stats": ([P, P], C.c_int),
            "avfs_capture": ([P, P, I32, C.c_float, C.c_float, P, P, P, P], C.c_int),
            "avfs_get_switching_energy": ([P, P], C.c_int),
            "avfs_fit_delay_polynomial": ([I64, P, P, P, I32, I32, D, D, D, D, P, P], C.c_int),
            "avfs_debug_phase_cycles": ([P, I32], C.c_int32),
            "avfs_get_timing": ([P, P, P], C.c_int),
        }
        for name, (args, res) in sig.items():
            f = getattr(lib, name)
            f.argtypes = args
            f.restype = res
        _lib = lib
    return _lib


def debug_phase_cycles(reset: bool = False) -> np.ndarray:
    """Per-phase warp clock sums of the sweep (diagnostic builds, -DAVFS_PROF_PHASES)."""
    out = np.zeros(16, np.uint64)
    n = load_library().avfs_debug_phase_cycles(C.c_void_p(out.ctypes.data), int(reset))
    return out if n > 0 else np.zeros(0, np.uint64)


def _p(a):
    return None if a is None else C.c_void_p(a.ctypes.data)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


class Context:
    """One libavfs context (one CUDA device, or device=-1 for host-only)."""

    def __init__(self, device: int = 0):
        self.lib = load_library()
        h = C.c_void_p()
        st = self.lib.avfs_create(int(device), C.byref(h))
        if st:
            raise AvfsError(st, f"avfs_create({device}) failed")
        self.h = h
        self.n_vdd = 0
        self.n_signals = 0
        self.n_pairs = 0

    def close(self):
        if getattr(self, "h", None):
            self.lib.avfs_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def _ck(self, st: int):
        if st:
            msg = self.lib.avfs_last_error(self.h)
            raise AvfsError(st, msg.decode() if msg else "")

    # ------------------------------------------------------------ (1')
    def load_library(self, names, n_inputs, truth_tables, deg_v, deg_c, beta,
                     v_min=0.55, v_max=1.1, c_min=0.5, c_max=128.0):
        n = len(names)
        cells = (avfs_cell * n)()
        self._names = [s.encode() for s in names]
        for i in range(n):
            cells[i].name = self._names[i]
            cells[i].n_inputs = int(n_inputs[i])
            cells[i].truth_table = int(truth_tables[i])
        b = _c(beta, np.float64)
        self._ck(self.lib.avfs_load_library(self.h, n, cells, int(deg_v), int(deg_c), _p(b),
                                            float(v_min), float(v_max), float(c_min), float(c_max)))

    # ------------------------------------------------------------ (1)
    def load_netlist(self, n_pi, gate_cell, fanin_ptr, fanin_sig, d_nom, c_load, po_sig):
        gc = _c(gate_cell, np.int32)
        fp = _c(fanin_ptr, np.int64)
        fs = _c(fanin_sig, np.int32)
        dn = _c(d_nom, np.float64)
        cl = None if c_load is None else _c(c_load, np.float64)
        po = _c(po_sig, np.int32)
        self._ck(self.lib.avfs_load_netlist(self.h, int(n_pi), len(gc), _p(gc), _p(fp), _p(fs), _p(dn),
                                            _p(cl), len(po), _p(po)))
        self.n_signals = int(n_pi) + len(gc)

    def load_bench(self, text: str, d_nom, c_load=None):
        t = text.encode()
        dn = _c(d_nom, np.float64)
        cl = None if c_load is None else _c(c_load, np.float64)
        self._ck(self.lib.avfs_load_bench(self.h, t, len(t), _p(dn), _p(cl)))
        info = self.netlist_info()
        self.n_signals = info["n_pi"] + info["n_gates"]

    def find_signal(self, name: str) -> int:
        s = C.c_int32()
        self._ck(self.lib.avfs_find_signal(self.h, name.encode(), C.byref(s)))
        return s.value

    def netlist_info(self) -> dict:
        i = avfs_netlist_info()
        self._ck(self.lib.avfs_get_netlist_info(self.h, C.byref(i)))
        return {f: getattr(i, f) for f, _ in i._fields_}

    def levels(self) -> np.ndarray:
        out = np.zeros(self.n_signals, np.int32)
        self._ck(self.lib.avfs_get_levels(self.h, _p(out)))
        return out

    def buffer_map(self) -> np.ndarray:
        out = np.zeros(self.n_signals, np.int32)
        self._ck(self.lib.avfs_get_buffer_map(self.h, _p(out)))
        return out

    # ------------------------------------------------------------ (2), (3)
    def set_operating_points(self, vdd):
        v = _c(vdd, np.float64)
        self._ck(self.lib.avfs_set_operating_points(self.h, len(v), _p(v)))
        self.n_vdd = len(v)

    def set_voltage_islands(self, island_of_gate, vdd_matrix):
        """NEXT-2: vdd_matrix [n_points][n_islands] volts, island_of_gate [n_gates]."""
        v = _c(vdd_matrix, np.float64)
        isl = None if island_of_gate is None else _c(island_of_gate, np.int32)
        self._ck(self.lib.avfs_set_voltage_islands(self.h, int(v.shape[1]), _p(isl), int(v.shape[0]), _p(v)))
        self.n_vdd = int(v.shape[0])

    def set_stimuli(self, p1, p2):
        """p1, p2: numpy uint32 [n_pairs][words] (host) or torch CUDA tensors (device)."""
        if hasattr(p1, "data_ptr"):
            n = int(p1.shape[0])
            self._ck(self.lib.avfs_set_stimuli(self.h, n, C.c_void_p(p1.data_ptr()),
                                               C.c_void_p(p2.data_ptr()), 1))
        else:
            a, b = _c(p1, np.uint32), _c(p2, np.uint32)
            n = int(a.shape[0])
            self._ck(self.lib.avfs_set_stimuli(self.h, n, _p(a), _p(b), 0))
        self.n_pairs = n

    def set_slot_range(self, first: int, n: int = -1):
        self._ck(self.lib.avfs_set_slot_range(self.h, int(first), int(n)))

    def set_pair_range(self, first: int, n: int):
        """Simulate pairs [first, first + n) at every operating point."""
        self._ck(self.lib.avfs_set_pair_range(self.h, int(first), int(n)))

    def set_options(self, capacity=8, quantum_ps=0.0, probes=None, keep_all=False,
                    max_rerun_rounds=3, warps_per_cta=0, profile=False, spill_bytes=0, max_batch_slots=0,
                    delay_in_sweep=False):
        o = avfs_options()
        self._ck(self.lib.avfs_default_options(C.byref(o)))
        o.capacity = int(capacity)
        o.quantum_ps = float(quantum_ps)
        self._probes = None if probes is None else _c(probes, np.int32)
        o.n_probe = 0 if self._probes is None else len(self._probes)
        if self._probes is not None and len(self._probes):
            o.probe_sig = self._probes.ctypes.data_as(C.POINTER(C.c_int32))
        o.keep_all = int(bool(keep_all))
        o.max_rerun_rounds = int(max_rerun_rounds)
        o.warps_per_cta = int(warps_per_cta)
        o.profile = int(bool(profile))
        o.spill_bytes = int(spill_bytes)
        o.max_batch_slots = int(max_batch_slots)
        o.delay_in_sweep = int(bool(delay_in_sweep))
        self._ck(self.lib.avfs_set_options(self.h, C.byref(o)))

    def simulate(self, stream=None):
        """stream: a torch.cuda.Stream, a raw cudaStream_t int, or None (legacy default)."""
        s = getattr(stream, "cuda_stream", stream)
        self._ck(self.lib.avfs_simulate(self.h, None if not s else C.c_void_p(int(s))))

    def sync(self):
        self._ck(self.lib.avfs_sync(self.h))

    # ------------------------------------------------------------ (4)
    def activity(self, out=None) -> np.ndarray:
        """[n_signals][n_vdd] uint64; `out` may be a torch CUDA int64/uint64 tensor
        (device copy) or a C-contiguous uint64 numpy array (e.g. pinned host memory)."""
        if out is not None and hasattr(out, "data_ptr"):
            import torch
            if (not out.is_cuda or out.dtype not in (torch.int64, torch.uint64)
                    or tuple(out.shape) != (self.n_signals, self.n_vdd) or not out.is_contiguous()):
                raise ValueError("activity out tensor must be a contiguous CUDA int64/uint64 [n_signals][n_vdd]")
            self._ck(self.lib.avfs_get_activity(self.h, C.c_void_p(out.data_ptr()), 1))
            return out
        if out is not None:
            if out.dtype != np.uint64 or out.shape != (self.n_signals, self.n_vdd) or not out.flags.c_contiguous:
                raise ValueError("activity out must be C-contiguous uint64 [n_signals][n_vdd]")
            self._ck(self.lib.avfs_get_activity(self.h, _p(out), 0))
            return out
        a = np.zeros((self.n_signals, self.n_vdd), np.uint64)
        self._ck(self.lib.avfs_get_activity(self.h, _p(a), 0))
        return a

    def timing(self):
        """(pass-0 sweep ms, rerun ms) of the last simulate (profile=True); no readback."""
        a, b = C.c_double(), C.c_double()
        self._ck(self.lib.avfs_get_timing(self.h, C.byref(a), C.byref(b)))
        return a.value, b.value

    def latest_arrival(self, out=None) -> np.ndarray:
        """[n_vdd] float32 ps; `out` may be a contiguous CUDA float32 tensor (device copy)."""
        if out is not None:
            import torch
            if not out.is_cuda or out.dtype != torch.float32 or tuple(out.shape) != (self.n_vdd,) or not out.is_contiguous():
                raise ValueError("latest_arrival out tensor must be a contiguous CUDA float32 [n_vdd]")
            self._ck(self.lib.avfs_get_latest_arrival(self.h, C.c_void_p(out.data_ptr()), 1))
            return out
        a = np.zeros(self.n_vdd, np.float32)
        self._ck(self.lib.avfs_get_latest_arrival(self.h, _p(a), 0))
        return a

    def final_values(self, sig, slot0: int, n_slots: int) -> np.ndarray:
        s = _c(sig, np.int32)
        out = np.zeros((len(s), n_slots), np.uint8)
        self._ck(self.lib.avfs_get_final_values(self.h, len(s), _p(s), int(slot0), int(n_slots), _p(out)))
        return out

    def waveforms(self, sig, slot0: int, n_slots: int, cap: int = 16):
        s = _c(sig, np.int32)
        init = np.zeros((len(s), n_slots), np.uint8)
        count = np.zeros((len(s), n_slots), np.int32)
        times = np.zeros((len(s), n_slots, max(cap, 1)), np.float32)
        self._ck(self.lib.avfs_get_waveforms(self.h, len(s), _p(s), int(slot0), int(n_slots), int(cap),
                                             _p(init), _p(count), _p(times)))
        return init, count, times[:, :, :cap]

    def capture(self, t_clk, n_bins=64, lo_ps=-500.0, width_ps=25.0):
        """NEXT-1: sample every PO at t_clk[k]; returns dict with fail_pairs [n_vdd],
        fail_po [n_po][n_vdd], slack_hist [n_vdd][n_bins], fail_bits [n_sim_slots]."""
        t = _c(t_clk, np.float32)
        V = self.n_vdd
        n_po = int(self.netlist_info()["n_po"])
        st = self.stats()
        fp = np.zeros(V, np.uint32)
        fpo = np.zeros((max(n_po, 1), V), np.uint32)
        hist = np.zeros((V, n_bins), np.uint32)
        bits = np.zeros(max(int(st["slots"]), 1), np.uint8)
        self._ck(self.lib.avfs_capture(self.h, _p(t), int(n_bins), float(lo_ps), float(width_ps), _p(fp), _p(fpo),
                                       _p(hist), _p(bits)))
        return {"fail_pairs": fp, "fail_po": fpo[:n_po], "slack_hist": hist, "fail_bits": bits[:int(st["slots"])]}

    def switching_energy(self) -> np.ndarray:
        """NEXT-4: 1/2 sum act * c_load * v^2 per operating point, fJ."""
        out = np.zeros(self.n_vdd, np.float64)
        self._ck(self.lib.avfs_get_switching_energy(self.h, _p(out)))
        return out

    def stats(self) -> dict:
        st = avfs_stats()
        self._ck(self.lib.avfs_get_stats(self.h, C.byref(st)))
        return st.as_dict()


def fit_delay_polynomial(v, c, y, deg_v, deg_c, v_min=0.55, v_max=1.1, c_min=0.5, c_max=128.0):
    """NEXT-3: OLS fit of Eq. (4) (normal equation, Eq. 8).  Returns (beta [deg_v+1][deg_c+1], rms)."""
    lib = load_library()
    vv = _c(v, np.float64)
    cc = None if c is None else _c(c, np.float64)
    yy = _c(y, np.float64)
    beta = np.zeros((deg_v + 1) * (deg_c + 1), np.float64)
    rms = np.zeros(1, np.float64)
    st = lib.avfs_fit_delay_polynomial(len(vv), _p(vv), _p(cc), _p(yy), int(deg_v), int(deg_c), float(v_min),
                                       float(v_max), float(c_min), float(c_max), _p(beta), _p(rms))
    if st:
        raise AvfsError(st, "avfs_fit_delay_polynomial failed")
    return beta.reshape(deg_v + 1, deg_c + 1), float(rms[0])


def load_workload(ctx: Context, netlist, library, stimuli, vdd):
    """Marshal generator objects (workloads/) into the four setup calls."""
    ctx.load_library(library.names, library.n_inputs, library.tt, library.deg_v, library.deg_c,
                     library.beta, library.v_min, library.v_max, library.c_min, library.c_max)
    ctx.load_netlist(netlist.n_pi, netlist.gate_cell, netlist.fanin_ptr, netlist.fanin_sig,
                     netlist.d_nom, netlist.c_load, netlist.po_sig)
    ctx.set_operating_points(vdd)
    if stimuli is not None:
        ctx.set_stimuli(stimuli.p1, stimuli.p2)
