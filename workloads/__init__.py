"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

This package generates INPUTS only (netlists, a truth-table cell library with
polynomial delay coefficients, nominal delays, two-pattern stimuli, Vdd
points).  It contains none of the method's arithmetic: no delay evaluation,
no event processing, no filtering.  Both the C-ABI library (`avfs`) and the
oracle (`oracle/`) consume the plain numpy arrays it returns.

Recipes follow SURVEY.md §8(d) "Concrete synthetic inputs"; DESIGN.md restates
them.  Every random draw goes through numpy's PCG64 `default_rng(seed)`.
"""
from .cells import CELLS, CELL_INDEX, Library, make_library
from .netlists import Netlist, c17, c17_bench_text, array_multiplier, random_dag
from .stimuli import Stimuli, make_stimuli, exhaustive_pairs
from .configs import Workload, make_config, CONFIG_NAMES

__all__ = [
    "CELLS", "CELL_INDEX", "Library", "make_library",
    "Netlist", "c17", "c17_bench_text", "array_multiplier", "random_dag",
    "Stimuli", "make_stimuli", "exhaustive_pairs",
    "Workload", "make_config", "CONFIG_NAMES",
]
