"""Oracle: the staged cost model t(S) of §5.1.  TEST INFRASTRUCTURE ONLY.

Rules:
  * a communication's stage is its number of links from the source GPU;
  * a direct link L_i in stage k costs t_i^k = c_i^k(S) / b_i;
  * a multi-hop link costs t_i^k = max_j c_ij^k(S) / b_ij, where c_ij^k is the AGGREGATE data that
    goes through physical hop L_ij at stage k (so hops shared by several links model contention);
  * a stage costs t^k = max_i t_i^k; the plan costs t(S) = sum_{k=1}^{m-1} t^k.
Reading (R7): data is counted in rows and 1/b_h is the integer tick w_h per row
(topology.hop_ticks), so every cost is an exact integer.
"""
import numpy as np


def hop_loads(topo, edges):
    """c_h^k: rows through physical hop h at stage k.  edges: iterable of (u, parent, child, stage).
    Returns int64 array [m x n_hops]; row k holds stage k (row 0 unused)."""
    m = topo.m
    load = np.zeros((m, len(topo.hop_gbps)), dtype=np.int64)
    for (_u, p, c, k) in edges:
        hops = topo.link(int(p), int(c))
        assert hops is not None, "edge on a missing link %d->%d" % (p, c)
        for h in hops:
            load[int(k), h] += 1
    return load


def stage_times(topo, load):
    """t^k = max over links of max over their hops of c_h^k * w_h  (== max over used hops)."""
    w = np.asarray(topo.hop_ticks, dtype=np.int64)
    m = topo.m
    t = np.zeros(m, dtype=np.int64)
    for k in range(1, m):
        best = 0
        for (i, j), hops in topo.links.items():
            # t_i^k for link i->j: its slowest physical hop under the aggregate hop load
            tik = max(int(load[k, h]) * int(w[h]) for h in hops)
            best = max(best, tik)
        t[k] = best
    return t


def plan_cost(topo, edges):
    """t(S) = sum_k t^k.  Returns (total, per-stage array)."""
    load = hop_loads(topo, edges)
    t = stage_times(topo, load)
    return int(t.sum()), t
