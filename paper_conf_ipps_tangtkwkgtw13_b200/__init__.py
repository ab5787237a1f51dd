"""B200-native in-plane 3D star-stencil sweeps (Tang et al., IPDPS 2013).

The product is ``libstencil.so`` (C ABI, include/stencil.h) built from
``csrc/`` for sm_100a; this package is its thin Python binding.  Importing it
fails loudly if the library has not been built -- there is no CPU fallback.
"""
from ._lib import StencilError, lib  # noqa: F401  (raises ImportError if libstencil.so is missing)
from .plan import (DistPlan, DivGrad, LocalRankGroup, P2PSlab, Plan, exchange_plan, layout_compute, nccl_unique_id, p2p_targets,  # noqa: F401
                   slab_partition)

__all__ = ["Plan", "DistPlan", "DivGrad", "LocalRankGroup", "P2PSlab", "p2p_targets", "layout_compute", "slab_partition", "exchange_plan", "nccl_unique_id",
           "StencilError", "lib"]
