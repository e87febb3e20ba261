"""C-ABI library on CPU (-m "not gpu"): symbol exports, parser, levelizer,
liveness allocator, argument / state errors.  Uses a host-only context
(avfs_create(-1)); no compute call runs without a GPU."""
import ctypes
import os
import re

import numpy as np
import pytest

from workloads import make_config, make_library, random_dag, c17_bench_text
from workloads.cells import CELLS

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def pkg():
    from paper_conf_date_schneiderw20_b200 import _build
    _build.build()
    import paper_conf_date_schneiderw20_b200 as P
    return P


def lib_args(lib):
    return (lib.names, lib.n_inputs, lib.tt, lib.deg_v, lib.deg_c, lib.beta)


def host_ctx(P, nl, lib, **opt):
    c = P.Context(-1)
    c.load_library(*lib_args(lib))
    c.load_netlist(nl.n_pi, nl.gate_cell, nl.fanin_ptr, nl.fanin_sig, nl.d_nom,
                   nl.c_load if lib.deg_c else None, nl.po_sig)
    c.set_options(**opt)
    return c


def test_exports_match_header(pkg):
    hdr = open(os.path.join(ROOT, "include", "avfs.h")).read()
    declared = set(re.findall(r"\b(avfs_[a-z_]+)\s*\(", hdr))
    assert declared == set(pkg.EXPORTS)
    so = ctypes.CDLL(pkg.LIB_PATH)
    for name in declared:
        assert hasattr(so, name), name


def test_version_and_status_strings(pkg):
    lib = pkg.load_library()
    assert lib.avfs_version().decode().endswith("sm_100a")
    assert lib.avfs_status_string(7) == b"AVFS_ERR_CAPACITY"


def independent_levels(nl):
    lv = np.zeros(nl.n_signals, np.int64)
    changed = True
    while changed:
        changed = False
        for g in range(nl.n_gates):
            ins = nl.fanin_sig[nl.fanin_ptr[g]:nl.fanin_ptr[g + 1]]
            v = 1 + lv[ins].max()
            if v != lv[nl.n_pi + g]:
                lv[nl.n_pi + g] = v
                changed = True
    return lv


@pytest.mark.parametrize("seed", [1, 2])
def test_levelizer_on_permuted_netlists(pkg, seed):
    nl = random_dag(seed, 800, 30, 14).permuted(seed)
    c = host_ctx(pkg, nl, make_library(1))
    assert np.array_equal(c.levels(), independent_levels(nl))
    info = c.netlist_info()
    assert info["depth"] == independent_levels(nl).max()
    assert info["n_edges"] == nl.n_edges


def check_liveness(nl, levels, bmap):
    """No scratch buffer is rewritten while a reader still needs its value."""
    last = np.full(nl.n_signals, -1)
    for g in range(nl.n_gates):
        for s in nl.fanin_sig[nl.fanin_ptr[g]:nl.fanin_ptr[g + 1]]:
            last[s] = max(last[s], levels[nl.n_pi + g])
    by_buf = {}
    for s in range(nl.n_pi, nl.n_signals):
        if bmap[s] >= 0:
            by_buf.setdefault(bmap[s], []).append((levels[s], max(levels[s], last[s])))
    for b, iv in by_buf.items():
        iv.sort()
        for (a0, a1), (b0, b1) in zip(iv, iv[1:]):
            assert a1 < b0, f"buffer {b}: [{a0},{a1}] overlaps [{b0},{b1}]"
    return len(by_buf)


@pytest.mark.parametrize("cfg,scale", [(2, 1.0), (3, 0.2)])
def test_liveness_allocator(pkg, cfg, scale):
    w = make_config(cfg, n_pairs=32, n_vdd=1, scale=scale)
    nl = w.netlist
    c = host_ctx(pkg, nl, w.library, capacity=8)
    bm = c.buffer_map()
    nbuf = check_liveness(nl, c.levels(), bm)
    info = c.netlist_info()
    assert nbuf == info["n_scratch_buffers"]
    assert info["n_pinned"] == len(set(nl.po_sig) - set(range(nl.n_pi)))
    assert nbuf < nl.n_gates // 2          # liveness actually reuses buffers
    assert np.all(bm[:nl.n_pi] == -1)
    assert set(np.nonzero(bm <= -2)[0]) == set(nl.po_sig) - set(range(nl.n_pi))
    # keep_all pins every gate; probes pin exactly the probes
    c.set_options(keep_all=True)
    assert c.netlist_info()["n_scratch_buffers"] == 0
    probes = np.array([nl.n_pi + 3, nl.n_pi + 10], np.int32)
    c.set_options(probes=probes)
    bm = c.buffer_map()
    assert np.all(bm[probes] <= -2)
    check_liveness(nl, c.levels(), bm)


def test_bench_parser_c17(pkg):
    w = make_config(1)
    c = pkg.Context(-1)
    c.load_library(*lib_args(w.library))
    c.load_bench(c17_bench_text(), w.netlist.d_nom)
    info = c.netlist_info()
    assert (info["n_pi"], info["n_gates"], info["n_po"], info["depth"]) == (5, 6, 2, 3)
    assert [c.find_signal(n) for n in ("1", "2", "3", "6", "7", "10", "22", "23")] == [0, 1, 2, 3, 4, 5, 9, 10]
    assert np.array_equal(c.levels(), [0, 0, 0, 0, 0, 1, 1, 2, 2, 3, 3])


def test_bench_parser_dff_cut_and_aliases(pkg):
    text = """# s27-like
INPUT(G0)
INPUT(G1)
OUTPUT(G17)
G5 = DFF(G10)
G10 = NOR(G14, G11)
G11 = NOT(G5)
G14 = BUFF(G0)
G17 = AND(G11, G1)
"""
    lib = make_library(1, deg_v=1)
    c = pkg.Context(-1)
    c.load_library(*lib_args(lib))
    d = np.full((7, 2), 5.0)
    c.load_bench(text, d)
    info = c.netlist_info()
    assert info["n_pi"] == 3 and info["n_gates"] == 4       # G5 is a pseudo PI
    assert c.find_signal("G5") == 2
    assert info["n_po"] == 2                                 # G17 and pseudo PO G10
    lv = c.levels()
    assert lv[c.find_signal("G10")] == 2 and lv[c.find_signal("G11")] == 1


@pytest.mark.parametrize("text,code", [
    ("INPUT(a)\nOUTPUT(b)\nb = NAND(a, c)\n", 2),            # undriven net
    ("INPUT(a)\nOUTPUT(b)\nb = FOO(a, a)\n", 2),             # unknown cell
    ("INPUT(a)\nOUTPUT(b)\nb = NAND(a, c)\nc = NAND(a, b)\n", 2),  # cycle
    ("INPUT(a)\nOUTPUT(b)\nb = NAND a, a\n", 2),             # malformed
])
def test_bench_parser_errors(pkg, text, code):
    c = pkg.Context(-1)
    c.load_library(*lib_args(make_library(1)))
    with pytest.raises(pkg.AvfsError) as e:
        c.load_bench(text, np.full((8, 2), 5.0))
    assert e.value.status == code


def test_netlist_argument_errors(pkg):
    lib = make_library(1)
    c = pkg.Context(-1)
    with pytest.raises(pkg.AvfsError) as e:      # library first
        c.load_netlist(2, [2], [0, 2], [0, 1], np.ones((2, 2)), None, [2])
    assert e.value.status == 3
    c.load_library(*lib_args(lib))
    nand2 = [n for n, _, _ in CELLS].index("NAND2")
    with pytest.raises(pkg.AvfsError) as e:      # arity mismatch
        c.load_netlist(2, [nand2], [0, 1], [0], np.ones((1, 2)), None, [2])
    assert e.value.status == 1
    with pytest.raises(pkg.AvfsError) as e:      # non-positive nominal delay
        c.load_netlist(2, [nand2], [0, 2], [0, 1], np.array([[1.0, 0.0], [1.0, 1.0]]), None, [2])
    assert e.value.status == 1
    with pytest.raises(pkg.AvfsError) as e:      # cycle through two gates
        c.load_netlist(1, [nand2, nand2], [0, 2, 4], [0, 2, 0, 1], np.ones((4, 2)), None, [2])
    assert e.value.status == 2
    with pytest.raises(pkg.AvfsError) as e:      # host-only context cannot take stimuli
        c.load_netlist(2, [nand2], [0, 2], [0, 1], np.ones((2, 2)), None, [2])
        c.set_stimuli(np.zeros((1, 1), np.uint32), np.zeros((1, 1), np.uint32))
    assert e.value.status == 3
    with pytest.raises(pkg.AvfsError):
        c.set_options(capacity=0)


def test_product_path_has_no_oracle_or_cpu_fallback():
    """The product package never imports the oracle (and vice versa)."""
    pkg_dir = os.path.join(ROOT, "paper_conf_date_schneiderw20_b200")
    for dp, _, fs in os.walk(pkg_dir):
        for f in fs:
            if f.endswith((".py", ".cpp", ".cu", ".h")):
                src = open(os.path.join(dp, f)).read()
                assert "import oracle" not in src and "oracle." not in src.replace("oracle.c", ""), f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            src = open(os.path.join(ROOT, "oracle", f)).read()
            assert "paper_conf_date_schneiderw20_b200 import" not in src and "import paper_conf" not in src
            assert "avfs_internal" not in src and "avfs.h" not in src


def test_missing_library_fails_loudly(tmp_path):
    from paper_conf_date_schneiderw20_b200 import avfs as A
    saved = A._lib
    A._lib = None
    try:
        with pytest.raises(ImportError):
            A.load_library(str(tmp_path / "nope.so"))
    finally:
        A._lib = saved
