"""B200-native explicit Lagrangian hydro cycle (Pearce, ICPP'18 workload) -- Python package.

The compute path is the CUDA library ``libhydro_b200.so`` (include/hydro.h); ``hydro`` is its
thin binding and ``inputs`` the seeded synthetic input generators.  Importing the package does
not load the library; constructing ``Hydro`` does, and fails loudly if it is missing.
"""
from .hydro import (ALL_FIELDS, Hydro, HydroConfig, HydroError, comm_plan_export,  # noqa
                    decompose_hierarchical, dom_to_rank, layout_export, load_library,
                    rebalance_plan, weighted_slabs)

__all__ = ["Hydro", "HydroConfig", "HydroError", "layout_export", "decompose_hierarchical",
           "weighted_slabs", "load_library", "ALL_FIELDS", "comm_plan_export", "rebalance_plan",
           "dom_to_rank"]
