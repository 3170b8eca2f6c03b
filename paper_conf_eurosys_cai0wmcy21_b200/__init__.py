"""B200-native DGCL halo exchange (Cai et al., EuroSys '21): planner + sm_100a plan executor.

The compute path is libdgcl.so (C ABI in include/dgcl.h); this package is its Python binding.
"""
from ._abi import DGCLError, LOOPBACK_FUSED, LOOPBACK_PER_RANK, LIB_PATH, SYMBOLS
from .dgcl import (Context, init, loopback, setup_distributed, GraphAllgather, graph_allgather,
                   multicast_supported, multicast_selftest)

__all__ = ["DGCLError", "Context", "init", "loopback", "setup_distributed", "GraphAllgather",
           "graph_allgather", "multicast_supported", "multicast_selftest", "LOOPBACK_FUSED",
           "LOOPBACK_PER_RANK", "LIB_PATH", "SYMBOLS"]
