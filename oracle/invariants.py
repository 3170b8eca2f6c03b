"""Oracle: plan invariants.  TEST INFRASTRUCTURE ONLY.

(i)   each T_u is a tree rooted at s_u, stage = depth <= m-1;
(ii)  halo deliveries = {(u, d) : d in D_u}, each exactly once;
(iii) no delivery to a GPU outside D_u except as a pure relay (relay staging, not the halo);
(iv)  every edge uses an existing link of the topology;
(v)   recomputing t(S) from the edges gives the planner's reported cost (§5.1).
"""
from collections import defaultdict

from .cost import plan_cost


def check_plan(topo, edges, owner, D, reported_cost=None):
    m = topo.m
    by_u = defaultdict(list)
    for (u, p, c, k) in edges:
        by_u[int(u)].append((int(p), int(c), int(k)))
    assert set(by_u) == {u for u in D if D[u]}, "planned vertex set != {u : D_u non-empty}"
    n_relay = 0
    for u, te in by_u.items():
        su = owner[u]
        parent = {}
        depth = {su: 0}
        for (p, c, k) in te:
            assert c != su, "edge into the root"
            assert c not in parent, "vertex %d reaches GPU %d twice" % (u, c)       # (ii)
            parent[c] = p
            assert topo.link(p, c) is not None, "missing link %d->%d" % (p, c)   # (iv)
        # depths follow parents; every node reaches the root (tree, (i))
        def dep(x, seen=()):
            if x in depth:
                return depth[x]
            assert x in parent and x not in seen, "not a tree"
            depth[x] = dep(parent[x], seen + (x,)) + 1
            return depth[x]
        for (p, c, k) in te:
            assert dep(c) == k, "stage != depth for u=%d" % u
            assert 1 <= k <= m - 1
        reached = set(parent)
        assert set(D[u]) <= reached, "missing delivery"                          # (ii)
        extra = reached - set(D[u])
        for x in extra:                                                            # (iii)
            assert any(pp == x for (pp, _c, _k) in te), "leaf outside D_u (useless delivery)"
        n_relay += len(extra)
    if reported_cost is not None:
        total, _ = plan_cost(topo, edges)
        assert total == reported_cost, (total, reported_cost)                       # (v)
    return n_relay
