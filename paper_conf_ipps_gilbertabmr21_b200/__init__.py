"""B200-native (sm_100a) hot path of iterated Heavy Edge Coarsening (HEC),
Gilbert, Acer, Boman, Madduri, Rajamanickam, IPDPS 2021.

The product is libhec.so (C-ABI in include/hec.h, CUDA sources in csrc/); this
package is its thin Python binding.  There is no CPU fallback: importing works
without a GPU, but every call needs the CUDA library and a B200.
"""
from ._lib import (HEC_EINVAL, HEC_ENOMEM, HEC_ECUDA, HEC_EOVERFLOW, HEC_OK, STOP_CUTOFF,  # noqa: F401
                   STOP_DISCARD, STOP_MAX_LEVELS, STOP_STALL, HecError, load)
from .hec import (CoarseGraph, Context, DeviceGraph, Hierarchy, Level, build_coarse_graph,  # noqa: F401
                  coarsen_hierarchy, hec_debug_heavy, hec_debug_roots, hec_find_mapping,
                  hec_find_mapping_method, hec_find_mapping_prio, hec_prio, spectral_bisection)

__all__ = [
    "Context", "DeviceGraph", "CoarseGraph", "Hierarchy", "Level", "hec_find_mapping",
    "hec_find_mapping_prio", "hec_find_mapping_method", "build_coarse_graph", "coarsen_hierarchy", "hec_debug_heavy",
    "hec_debug_roots", "hec_prio", "HecError", "load", "spectral_bisection",
]
