"""B200-native DGCL halo exchange (Cai et al., EuroSys '21): planner + sm_100a plan executor.

The compute path is libdgcl.so (C ABI in include/dgcl.h); this package is its Python binding.
"""
from ._abi import DGCLError, LOOPBACK_FUSED, LOOPBACK_PER_RANK, LIB_PATH, SYMBOLS
from .dgcl import Context, init, loopback, setup_distributed, GraphAllgather, graph_allgather

__all__ = ["DGCLError", "Context", "init", "loopback", "setup_distributed", "GraphAllgather",
           "graph_allgather", "LOOPBACK_FUSED", "LOOPBACK_PER_RANK", "LIB_PATH", "SYMBOLS"]
