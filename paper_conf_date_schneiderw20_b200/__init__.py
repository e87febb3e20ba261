"""B200-native (sm_100a) waveform-accurate logic time simulation under many
supply-voltage operating points (Schneider & Wunderlich, DATE'20).

The product is the C-ABI library libavfs.so (include/avfs.h, csrc/); this
package holds its thin ctypes binding and the multi-GPU slot sharding.  There
is no CPU fallback: without the built library, Context() raises.
"""
from .avfs import (AvfsError, Context, EXPORTS, LIB_PATH, fit_delay_polynomial, load_library, load_workload)
from .parallel import shard_range, shard_pairs, reduce_results

__all__ = ["AvfsError", "Context", "EXPORTS", "LIB_PATH", "fit_delay_polynomial", "load_library", "load_workload",
           "shard_range", "shard_pairs", "reduce_results"]
