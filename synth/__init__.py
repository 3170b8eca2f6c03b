"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This package holds none of DGCL's arithmetic.  It generates the method's INPUTS only:
R-MAT graphs shaped like the paper's datasets (Table 4), a balanced random
partition (stand-in for METIS), the required lists R_d (V^r_d of §4.1),
hash-defined fp32 row values and the link-cost topology descriptors the planner takes as input
(D(V', E') with bandwidths, §5.1).
"""
from .graph import (Graph, rmat_edges, partition, permutation, required_lists, make_graph,
                    required_lists_numpy)
from .values import fill_values, fill_values_numpy, MODES
from .topology import Topology, uniform_nvswitch, dgx1_like, ring, fig6, fig6_pcie, ticks_of
from .configs import CONFIGS, Config, get_config
