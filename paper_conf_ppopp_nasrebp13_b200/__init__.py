"""B200-native Boruvka minimum-spanning-forest hot path (Nasre, Burtscher, Pingali,
"Morph Algorithms on GPUs", PPoPP'13, §5).

The method runs in ``libmst.so`` (hand-written CUDA for sm_100a behind the C ABI of
``include/mst.h``); this package is the thin Python binding with the same names.
"""
from .mst import (MSTError, MSTGraph, mst_get_unique_id, mst_solve_host, mst_version,  # noqa: F401
                  minimum_spanning_forest, load, lib_path, EXPORTS)

__all__ = ["MSTError", "MSTGraph", "mst_get_unique_id", "mst_solve_host", "mst_version",
           "minimum_spanning_forest", "load", "lib_path", "EXPORTS"]
