"""Pins for oracle/cost.py and oracle/spst.py (-m "not gpu").

* the Fig. 6 worked example and §5.1 hand calculations (tests/golden/fig6_example.json)
* brute-force optimum over all feasible trees on tiny instances (eq. 2)
* derived properties: uniform NVSwitch => single-stage direct plan; plans are trees with
  stage = depth <= m-1; exactly-once delivery; cost recomputation
"""
import itertools
import json
import os

import numpy as np
import pytest

from oracle import cost, invariants, spst
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _fig6():
    with open(os.path.join(GOLD, "fig6_example.json")) as f:
        return json.load(f)


def test_ticks_table1():
    g = _fig6()
    assert synth.ticks_of(synth.topology.NV1) == g["ticks"]["NV1"]
    assert synth.ticks_of(synth.topology.PCIE) == g["ticks"]["PCIe"]
    assert synth.ticks_of(synth.topology.QPI) == g["ticks"]["QPI"]


def test_cost_stage_example():
    g = _fig6()["stage_example"]
    t = synth.fig6()
    edges = [("a", p, c, k) for (p, c, k) in g["trees"]["a"]] + \
            [("g", p, c, k) for (p, c, k) in g["trees"]["g"]]
    total, per = cost.plan_cost(t, edges)
    assert total == g["cost"]
    assert list(per[1:4]) == [4129, 4129, 4129]   # stage-1 links run concurrently, not summed


def test_cost_contention_example():
    g = _fig6()["contention_example"]
    t = synth.fig6_pcie()
    edges = [(i, p, c, k) for i, (p, c, k) in enumerate(g["edges_parent_child_stage"])]
    total, per = cost.plan_cost(t, edges)
    assert per[1] == g["stage1"] == 4 * 10460
    assert total == g["stage1"]


def test_spst_fig6_T_a():
    g = _fig6()["T_a_alone"]
    t = synth.fig6()
    edges, c = spst.spst(t, {"a": 0}, {"a": set(g["D"])}, seed=0, order=["a"])
    assert [(p, ch, k) for (_u, p, ch, k) in edges] == [tuple(x) for x in g["edges_parent_child_stage"]]
    assert c == g["cost"]
    # second step alternatives (after adding 0->1->2)
    st = spst.CostState(t)
    st.add(1, (0, 1))
    st.add(2, (1, 2))
    alt = g["second_step_alternative_costs"]
    assert st.incremental(1, (0, 3)) == alt["0->3 stage 1"]
    assert st.incremental(2, (1, 3)) == alt["1->3 stage 2"]
    assert st.incremental(3, (2, 3)) == alt["2->3 stage 3"]


def _all_trees(topo, root, must):
    """Every tree rooted at `root` over a node subset containing `must`, edges on existing links,
    as lists of (parent, child, stage)."""
    m = topo.m
    others = [x for x in range(m) if x != root]
    out = []
    for r in range(len(others) + 1):
        for subset in itertools.combinations(others, r):
            if not set(must) <= set(subset):
                continue
            nodes = (root,) + subset
            for parents in itertools.product(nodes, repeat=len(subset)):
                par = dict(zip(subset, parents))
                if any(par[x] == x or topo.link(par[x], x) is None for x in subset):
                    continue
                depth = {root: 0}
                ok = True
                for x in subset:
                    seen, y, dd = set(), x, 0
                    while y != root:
                        if y in seen:
                            ok = False
                            break
                        seen.add(y)
                        y, dd = par[y], dd + 1
                    if not ok:
                        break
                    depth[x] = dd
                if ok:
                    out.append([(par[x], x, depth[x]) for x in subset])
    return out


def _opt(topo, owner, D):
    verts = sorted(D)
    choices = [_all_trees(topo, owner[u], D[u]) for u in verts]
    best = None
    for combo in itertools.product(*choices):
        edges = [(u, p, c, k) for u, tr in zip(verts, combo) for (p, c, k) in tr]
        tot, _ = cost.plan_cost(topo, edges)
        best = tot if best is None else min(best, tot)
    return best


def test_fig6_T_a_is_optimal_by_brute_force():
    t = synth.fig6()
    assert _opt(t, {"a": 0}, {"a": {2, 3}}) == _fig6()["T_a_alone"]["cost"]


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_spst_bounded_by_bruteforce_opt(seed):
    """SPST is greedy: its cost is >= OPT of eq. 2; equal when every D_u is a single GPU and
    vertices are planned one at a time on empty links (shortest paths)."""
    t = synth.fig6()
    rng = np.random.RandomState(seed)
    owner, D = {}, {}
    for u in range(3):
        owner[u] = int(rng.randint(4))
        D[u] = set(int(x) for x in rng.choice([d for d in range(4) if d != owner[u]],
                                               size=rng.randint(1, 3), replace=False))
    edges, c = spst.spst(t, owner, D, seed=seed)
    invariants.check_plan(t, edges, owner, D, c)
    assert c >= _opt(t, owner, D)
    one = {0: {3}}
    e1, c1 = spst.spst(t, {0: 0}, one, seed=0)
    assert c1 == _opt(t, {0: 0}, one)


def test_fig6_full_relation_balances_links():
    """Fig. 6 relation: d1->d3 {a,b,c,d}, d1->d4 {a,b,e,f}, d2->d3 {g,h,i},
    d2->d4 {g,i,k,l}.  SPST uses both the direct PCIe-QPI-PCIe links and NVLink forwarding
    (load balancing and fast-link intuitions)."""
    t = synth.fig6()
    names = "abcdefghijkl"
    rel = {0: {2: "abcd", 3: "abef"}, 1: {2: "ghi", 3: "gikl"}}
    owner, D = {}, {}
    for s, dd in rel.items():
        for d, vs in dd.items():
            for v in vs:
                u = names.index(v)
                owner[u] = s
                D.setdefault(u, set()).add(d)
    for seed in range(4):
        edges, c = spst.spst(t, owner, D, seed=seed)
        invariants.check_plan(t, edges, owner, D, c)
        qpi = [e for e in edges if len(t.link(e[1], e[2])) == 3]
        relayed = [e for e in edges if e[3] >= 2]
        assert qpi and relayed
        all_direct = [(u, owner[u], d, 1) for u in D for d in D[u]]
        assert c < cost.plan_cost(t, all_direct)[0]


def _random_relation(n, m, seed, p=0.4):
    rng = np.random.RandomState(seed)
    part = rng.randint(m, size=n)
    owner, D = {}, {}
    for u in range(n):
        owner[u] = int(part[u])
        ds = {d for d in range(m) if d != part[u] and rng.rand() < p}
        if ds:
            D[u] = ds
    return owner, D


def test_spst_uniform_is_single_stage_direct():
    t = synth.uniform_nvswitch(8)
    owner, D = _random_relation(120, 8, 3, p=0.6)
    edges, c = spst.spst(t, owner, D, seed=7)
    invariants.check_plan(t, edges, owner, D, c)
    assert all(k == 1 and p == owner[u] for (u, p, _c, k) in edges)
    assert len(edges) == sum(len(v) for v in D.values())


@pytest.mark.parametrize("topo_name,min_stages", [("dgx1_like", 2), ("ring", 3)])
def test_spst_forced_topologies_emit_relays(topo_name, min_stages):
    t = synth.topology.by_name(topo_name)
    owner, D = _random_relation(60, 8, 11, p=0.5)
    edges, c = spst.spst(t, owner, D, seed=1)
    n_relay = invariants.check_plan(t, edges, owner, D, c)
    assert max(k for (_u, _p, _c, k) in edges) >= min_stages
    assert len(edges) >= sum(len(v) for v in D.values())
    assert n_relay >= 0


def test_shuffle_is_a_permutation_and_seeded():
    a = spst.shuffle_order(range(50), 9)
    assert sorted(a) == list(range(50))
    assert a == spst.shuffle_order(range(50), 9)
    assert a != spst.shuffle_order(range(50), 10)


# ---- negative pins of oracle.invariants.check_plan: each invariant broken once ----------------
# A checker that let a broken plan pass would let every planner test pass silently; each case
# below breaks exactly one of (i)-(v) of SURVEY §8(c) step 7 on a known-good plan and must fail.

def _chain3():
    """3 GPUs on a chain 0 -> 1 -> 2 (links 0->1, 1->0, 1->2, 2->1 only: 0->2 does not exist)."""
    t = synth.Topology("chain3", 3, [100.0] * 4, ["h01", "h10", "h12", "h21"])
    t.links = {(0, 1): [0], (1, 0): [1], (1, 2): [2], (2, 1): [3]}
    return t


def _good_chain_plan():
    """u=0 owned by GPU 0, requested by 1 and 2: T = 0->1 (stage 1), 1->2 (stage 2);
    u=1 owned by GPU 2, requested by 0 through the relay 1 (1 did not ask): 2->1, 1->0."""
    owner = {0: 0, 1: 2}
    D = {0: [1, 2], 1: [0]}
    edges = [(0, 0, 1, 1), (0, 1, 2, 2), (1, 2, 1, 1), (1, 1, 0, 2)]
    total, _ = cost.plan_cost(_chain3(), edges)
    return owner, D, edges, total


def test_check_plan_accepts_the_good_plan():
    owner, D, edges, total = _good_chain_plan()
    # by hand: every hop is 100 GB/s = 1000 ticks per row; stage 1 carries 0->1 and 2->1 (one row
    # on each of two hops), stage 2 carries 1->2 and 1->0 (likewise): t(S) = 1000 + 1000
    assert total == 2000
    assert invariants.check_plan(_chain3(), edges, owner, D, total) == 1   # one relay (u=1 on 1)


@pytest.mark.parametrize("case", [
    "stage_not_depth",       # (i)  stage label != tree depth
    "stage_too_deep",        # (i)  a stage-3 edge in a 3-GPU plan (> m - 1, and != its depth)
    "edge_into_root",        # (i)  the owner receives its own vertex
    "cycle",                 # (i)  nodes that never reach the root
    "duplicate_delivery",    # (ii) a GPU reached twice
    "missing_delivery",      # (ii) a requester never reached
    "useless_leaf",          # (iii) a leaf outside D_u (delivery to a GPU that did not ask)
    "missing_link",          # (iv) an edge on a link the topology does not have
    "wrong_cost",            # (v)  reported t(S) != recomputed
    "unplanned_vertex",      # planned set != {u : D_u non-empty}
    "planned_extra_vertex",  # a vertex nobody requested gets a tree
])
def test_check_plan_rejects(case):
    t = _chain3()
    owner, D, edges, total = _good_chain_plan()
    reported = None          # structural cases: the cost check is not what must fire
    if case == "stage_not_depth":
        edges[1] = (0, 1, 2, 1)
    elif case == "stage_too_deep":
        edges[1] = (0, 1, 2, 3)
    elif case == "edge_into_root":
        edges.append((0, 1, 0, 2))
    elif case == "cycle":
        edges[0:2] = [(0, 2, 1, 1), (0, 1, 2, 2)]     # u=0: 1 and 2 point at each other
    elif case == "duplicate_delivery":
        edges.append((0, 2, 1, 3))                     # 1 reached again, from 2
    elif case == "missing_delivery":
        del edges[1]                                   # 2 asked for u=0, never gets it
    elif case == "useless_leaf":
        D[0] = [1]                                     # 2 no longer asks for u=0: 1->2 is useless
    elif case == "missing_link":
        edges[0:2] = [(0, 0, 1, 1), (0, 0, 2, 1)]     # 0->2 does not exist
    elif case == "wrong_cost":
        reported = total + 1
    elif case == "unplanned_vertex":
        D[5] = [1]
        owner[5] = 0
    elif case == "planned_extra_vertex":
        edges.append((7, 0, 1, 1))
        owner[7] = 0
    with pytest.raises(AssertionError):
        invariants.check_plan(t, edges, owner, D, reported)
