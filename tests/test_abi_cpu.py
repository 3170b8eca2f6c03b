"""CPU tests of libdgcl (no GPU): exports, argument validation, SPST parity with the oracle's
reference planner, plan invariants, and the lowered tables run by the host interpreter against
the oracle (forward bit-exact, backward bit-exact in tree order)."""
import ctypes
import re

import numpy as np
import pytest

import synth
from oracle import halo, invariants, spst

pytestmark = pytest.mark.usefixtures("built")


def _D():
    import paper_conf_eurosys_cai0wmcy21_b200 as D
    return D


def test_library_exports_every_header_symbol(built):
    import os
    D = _D()
    hdr = open(os.path.join(built, "include", "dgcl.h")).read()
    declared = set(re.findall(r"\b(dgcl_[a-z_]+)\s*\(", hdr))
    declared = {s for s in declared if s not in ("dgcl_status",)}
    lib = ctypes.CDLL(D.LIB_PATH)
    for s in sorted(declared):
        assert hasattr(lib, s), s
    assert declared == set(D.SYMBOLS)


def _ctx(g, dims, topo=None, seed=0, device=-1, options=None):
    D = _D()
    c = D.loopback(g.m, g.part, dims, device=device)
    for k, v in (options or {}).items():
        c.set_option(k, v)
    c.build_plan(g.req_ptr, g.req_ids, seed=seed, topology=topo)
    return c


def test_init_validation():
    D = _D()
    part = np.array([0, 1, 2], np.int32)
    with pytest.raises(D.DGCLError):
        D.loopback(2, part, [4], device=-1)           # part out of range
    with pytest.raises(D.DGCLError):
        D.loopback(3, part, [0], device=-1)           # dim < 1
    with pytest.raises(D.DGCLError):
        D.init(part, [4], rank=3, world=3, device=-1)  # rank >= world
    with pytest.raises(D.DGCLError):
        D.loopback(17, np.zeros(3, np.int32), [4], device=-1)


def test_build_plan_validation():
    D = _D()
    part = np.array([0, 1, 0, 1], np.int32)
    c = D.loopback(2, part, [4], device=-1)
    with pytest.raises(D.DGCLError) as e:
        c.build_plan([0, 1, 1], [2])                   # GPU 0 requires its own vertex 2
    assert e.value.status == 1
    c = D.loopback(2, part, [4], device=-1)
    with pytest.raises(D.DGCLError):
        c.build_plan([0, 2, 2], [1, 1])                # duplicate
    c = D.loopback(2, part, [4], device=-1)
    with pytest.raises(D.DGCLError):
        c.build_plan([0, 1, 1], [9])                   # out of range
    c = D.loopback(2, part, [4], device=-1)
    c.build_plan([0, 1, 2], [1, 0])
    with pytest.raises(D.DGCLError) as e:
        c.build_plan([0, 1, 2], [1, 0])                # twice
    assert e.value.status == 2
    from paper_conf_eurosys_cai0wmcy21_b200 import _abi
    assert c.workspace_bytes() > 0                     # host-side layout is known
    # device calls on a host-only context are state errors (no memory is touched)
    assert _abi.lib().dgcl_register_workspace(c.handle, ctypes.c_void_p(1 << 20), 1 << 30) == 2
    with pytest.raises(D.DGCLError) as e:
        c.ipc_export()
    assert e.value.status == 2
    assert _abi.lib().dgcl_dispatch_forward(c.handle, 0, ctypes.c_void_p(1 << 20), 4, None,
                                            None) == 2


def test_unreachable_gpu_is_eplan():
    D = _D()
    part = np.array([0, 1], np.int32)
    t = synth.Topology("broken", 2, [100.0], ["h"], {})   # no links at all
    c = D.loopback(2, part, [4], device=-1)
    with pytest.raises(D.DGCLError) as e:
        c.build_plan([0, 1, 1], [1], topology=t)
    assert e.value.status == 6


def _check_lowering(g, dims, topo, seed, options=None):
    m = g.m
    R = [g.R(d) for d in range(m)]
    loc, _ = halo.local_rows(g.part, m)
    c = _ctx(g, dims, topo, seed, options=options)
    info = c.plan_info()
    E = c.plan_export()
    owner, Dd = spst.relation_from_lists(R, g.part)
    topo_o = topo if topo is not None else synth.uniform_nvswitch(m)
    edges, cost = spst.spst(topo_o, owner, Dd, seed=seed)
    assert [tuple(x) for x in E.tolist()] == [tuple(x) for x in edges]
    assert cost == info["model_cost_ticks"]
    invariants.check_plan(topo_o, [tuple(x) for x in E.tolist()], owner, Dd, cost)
    counts = c.plan_counts()
    assert counts.sum() == info["n_tree_edges"] == len(edges)
    for layer, dim in enumerate(dims):
        pitch = c.halo_view(layer)[2]
        emb = synth.fill_values(g.n, dim, pitch, keys=np.argsort(g.part, kind="stable"), seed=3)
        H = np.zeros((int(g.req_ptr[-1]), pitch), np.float32)
        c.debug_hostsim_forward(layer, emb, H)
        local = [emb[c.row_off[d]:c.row_off[d + 1], :dim] for d in range(m)]
        Ho = halo.forward(local, R, g.part, loc)
        for d in range(m):
            got = H[g.req_ptr[d]:g.req_ptr[d + 1], :dim]
            assert np.array_equal(got.view(np.uint32), Ho[d].view(np.uint32))
        G = synth.fill_values(int(g.req_ptr[-1]), dim, pitch, seed=4)
        L = synth.fill_values(g.n, dim, pitch, seed=5)
        EG = L.copy()
        c.debug_hostsim_backward(layer, G, EG)
        Ls = [L[c.row_off[d]:c.row_off[d + 1], :dim] for d in range(m)]
        Gs = [G[g.req_ptr[d]:g.req_ptr[d + 1], :dim] for d in range(m)]
        Bt = halo.backward_tree(Ls, Gs, R, g.part, loc, E)
        for d in range(m):
            got = EG[c.row_off[d]:c.row_off[d + 1], :dim]
            assert np.array_equal(got.view(np.uint32), Bt[d].view(np.uint32))
        if info["n_stages"] == 1:
            Bf = halo.backward_flat(Ls, Gs, R, g.part, loc)
            for d in range(m):
                got = EG[c.row_off[d]:c.row_off[d + 1], :dim]
                assert np.array_equal(got.view(np.uint32), Bf[d].view(np.uint32))
    return info


@pytest.mark.parametrize("m,direct", [(2, 1), (3, 1), (8, 1), (3, 0), (8, 0), (3, 2), (8, 2)])
def test_uniform_plan_and_lowering(m, direct):
    """direct=1: loopback in-place reduce program; direct=0: push to slots + owner reduce;
    direct=2: the atomic-add ablation's groups (one per (requester, owner), run by the host in
    requester order, i.e. the flat order)."""
    g = synth.make_graph(1500, 12000, m, graph_seed=m, part_seed=50 + m)
    opts = {"atomic_backward": 1} if direct == 2 else {"direct_reduce": direct}
    info = _check_lowering(g, [16, 5], None, seed=3, options=opts)
    assert info["n_stages"] == 1 and info["n_relay_rows"] == 0


@pytest.mark.parametrize("m,opts", [(2, {}), (8, {}), (8, {"stage_fold": 0}),
                                    (4, {"direct_reduce": 0}),
                                    (8, {"direct_reduce": 0, "item_bytes": 2048}),
                                    (3, {"gather4": 0, "stage_fold": 0}),
                                    (8, {"geometry": 1}), (8, {"geometry": 2}),
                                    (4, {"geometry": 2, "direct_reduce": 0}),
                                    (8, {"fanout": 1}), (3, {"fanout": 1, "geometry": 2}),
                                    (8, {"lsu_gather": 1}), (4, {"lsu_gather": 1, "geometry": 1}),
                                    (8, {"multicast": 1, "lsu_gather": 1})])
def test_work_items_host(m, opts):
    """The fused program's WORK ITEMS (not the groups) moved the way the bulk-copy executor moves
    them — COPY row runs, staged FOLD segments read back through the staged-term table — on the
    host, against the oracle: checks build_items (item cuts, runs, segments, staged rows)."""
    g = synth.make_graph(1500, 14000, m, graph_seed=20 + m, part_seed=60 + m)
    _check_lowering(g, [16, 5, 602], None, seed=3, options=dict(opts, hostsim_items=1))


@pytest.mark.parametrize("name,sf,fan,nb", [("dgx1_like", 1, 0, 4), ("ring", 1, 0, 4),
                                           ("ring", 0, 0, 4), ("dgx1_like", 1, 1, 1),
                                           ("ring", 1, 1, 1), ("ring", 1, 0, 8),
                                           ("dgx1_like", 0, 0, 1), ("ring", 1, 0, -1),
                                           ("dgx1_like", 0, 0, -4)])
def test_work_items_host_relay(name, sf, fan, nb):
    """nb: vertex blocks of the stage chaining (fan-out stage 1 needs nb = 1); nb < 0: the staged
    reversed-plan backward (direct_reduce = 0) with |nb| blocks instead of the loopback
    tree-order programs."""
    g = synth.make_graph(500, 2500, 8, graph_seed=9, part_seed=19)
    _check_lowering(g, [12, 3], synth.topology.by_name(name), seed=5,
                    options={"hostsim_items": 1, "stage_fold": sf, "fanout": fan,
                             "pipeline_blocks": abs(nb), "direct_reduce": int(nb > 0)})


def test_work_items_host_shuffled():
    g = synth.make_graph(800, 6000, 4, graph_seed=2, part_seed=3)
    g.req_ids = synth.graph.shuffle_lists(g.req_ptr, g.req_ids, 77)
    _check_lowering(g, [8, 64], None, seed=1, options={"hostsim_items": 1})


@pytest.mark.parametrize("name", ["dgx1_like", "ring"])
def test_relay_plan_and_lowering(name):
    g = synth.make_graph(500, 2500, 8, graph_seed=9, part_seed=19)
    info = _check_lowering(g, [12, 3], synth.topology.by_name(name), seed=5)
    assert info["n_stages"] >= 2 and info["n_relay_rows"] > 0


def test_shuffled_halo_order():
    g = synth.make_graph(800, 6000, 4, graph_seed=2, part_seed=3)
    g.req_ids = synth.graph.shuffle_lists(g.req_ptr, g.req_ids, 77)
    _check_lowering(g, [8], None, seed=1)


@pytest.mark.parametrize("topo_name", [None, "dgx1_like", "ring"])
def test_plan_save_and_resume(topo_name):
    """Checkpoint/resume of the planning step: plan_export -> build_plan(trees=...) in a fresh
    context gives the same plan, cost and lowered program (host interpreter vs the oracle)."""
    g = synth.make_graph(700, 5000, 8, graph_seed=31, part_seed=32)
    topo = synth.topology.by_name(topo_name) if topo_name else None
    a = _ctx(g, [12, 5], topo, seed=4)
    E = a.plan_export()
    D = _D()
    b = D.loopback(g.m, g.part, [12, 5], device=-1)
    b.build_plan(g.req_ptr, g.req_ids, topology=topo, trees=E)
    assert np.array_equal(b.plan_export(), E)
    ia, ib = a.plan_info(), b.plan_info()
    for k in ("n_stages", "n_tree_edges", "n_relay_rows", "model_cost_ticks", "n_fwd_groups",
              "n_bwd_groups"):
        assert ia[k] == ib[k], k
    # the resumed plan through the lowering, on the host, against the oracle
    m = g.m
    R = [g.R(d) for d in range(m)]
    loc, _ = halo.local_rows(g.part, m)
    pitch = b.halo_view(0)[2]
    emb = synth.fill_values(g.n, 12, pitch, keys=np.argsort(g.part, kind="stable"), seed=3)
    H = np.zeros((int(g.req_ptr[-1]), pitch), np.float32)
    b.debug_hostsim_forward(0, emb, H)
    Ho = halo.forward([emb[b.row_off[d]:b.row_off[d + 1], :12] for d in range(m)], R, g.part, loc)
    for d in range(m):
        assert np.array_equal(H[g.req_ptr[d]:g.req_ptr[d + 1], :12], Ho[d])


def test_saved_plan_is_validated():
    """Invalid trees are rejected with EPLAN (each §8(c) tree invariant broken once)."""
    D = _D()
    g = synth.make_graph(300, 2000, 4, graph_seed=41, part_seed=42)
    topo = synth.fig6()
    E = _ctx(g, [4], topo, seed=1).plan_export()
    assert (E[:, 3] > 1).any()          # the Fig. 6 model relays

    def rejected(E2):
        c = D.loopback(g.m, g.part, [4], device=-1)
        with pytest.raises(D.DGCLError) as e:
            c.build_plan(g.req_ptr, g.req_ids, topology=topo, trees=E2)
        assert e.value.status == 6, e.value     # DGCL_EPLAN

    deep = int(np.nonzero(E[:, 3] > 1)[0][0])
    bad = E.copy(); bad[deep, 3] += 1; rejected(bad)               # stage != tree depth
    bad = E.copy(); bad[0, 1] = bad[0, 2]; rejected(bad)           # parent not in the tree
    first = E[E[:, 0] == E[0, 0]]
    rejected(E[len(first):])                                       # a requested vertex missing
    bad = np.concatenate([E[len(first):], first, first[:1]])
    rejected(bad)                                                  # a vertex's edges split
    # an extra leaf on a GPU that did not request the vertex
    for v in np.unique(E[:, 0]):
        rows = E[E[:, 0] == v]
        nodes = set(rows[:, 1]) | set(rows[:, 2])
        free = [x for x in range(4) if x not in nodes]
        if free:
            k = int(np.nonzero(E[:, 0] == v)[0][-1])
            extra = np.array([[v, g.part[v], free[0], 1]], E.dtype)
            rejected(np.concatenate([E[:k + 1], extra, E[k + 1:]]))
            break
    else:
        pytest.fail("no vertex with a GPU outside its tree")


def test_fig6_plan_from_library():
    """The Fig. 6 worked example through the C planner (T_a = d1-d2-d3-d4)."""
    D = _D()
    part = np.array([0, 1, 2, 3], np.int32)  # vertex 0 = 'a' owned by GPU 0
    c = D.loopback(4, part, [4], device=-1)
    c.build_plan([0, 0, 0, 1, 2], [0, 0], seed=0, topology=synth.fig6())
    E = c.plan_export()
    assert E.tolist() == [[0, 0, 1, 1], [0, 1, 2, 2], [0, 2, 3, 3]]
    assert c.plan_info()["model_cost_ticks"] == 12387


def test_empty_and_single_rank():
    D = _D()
    part = np.zeros(5, np.int32)
    c = D.loopback(1, part, [4], device=-1)
    c.build_plan([0, 0], [])
    assert c.plan_info()["n_tree_edges"] == 0
    part = np.array([0, 1, 0, 1], np.int32)
    c = D.loopback(2, part, [4], device=-1)
    c.build_plan([0, 0, 0], [])   # nobody requires anything
    info = c.plan_info()
    assert info["n_deliveries"] == 0 and info["n_stages"] == 0


def test_plan_is_dim_independent():
    """the plan does not depend on the feature dimension."""
    g = synth.make_graph(600, 4000, 4, graph_seed=4, part_seed=4)
    a = _ctx(g, [3], synth.dgx1_like() if False else None, seed=2).plan_export()
    b = _ctx(g, [602, 256], None, seed=2).plan_export()
    assert np.array_equal(a, b)


@pytest.mark.parametrize("topo_name", ["dgx1_like", "ring"])
def test_single_shared_hop_cost_closed_form(topo_name):
    """tools/cost_fit.py's loopback model: when every link is the same single hop of w ticks per
    row, the §5.1 rules (a stage costs the max over hops of load x w, stages add)
    reduce to t(S) = (number of tree edges) x w for any plan — checked on relay plans re-costed
    through dgcl_build_plan_from_trees, and against the oracle's plan_cost."""
    from oracle import cost
    from synth.topology import Topology
    D = _D()
    g = synth.make_graph(900, 7000, 8, graph_seed=51, part_seed=52)
    a = _ctx(g, [8], synth.topology.by_name(topo_name), seed=2)
    E = a.plan_export()
    assert a.plan_info()["n_stages"] >= 2
    one = Topology("one_hop", 8, [123.0], ["hbm"])
    one.links = {(i, j): [0] for i in range(8) for j in range(8) if i != j}
    w = one.hop_ticks[0]
    b = D.loopback(g.m, g.part, [8], device=-1)
    b.build_plan(g.req_ptr, g.req_ids, topology=one, trees=E)
    assert b.plan_info()["model_cost_ticks"] == len(E) * w
    assert cost.plan_cost(one, [(int(u), int(p), int(c), int(k)) for u, p, c, k in E])[0] == len(E) * w


@pytest.mark.parametrize("m,mc", [(2, 1), (4, 1), (8, 1), (8, 5), (3, 2)])
def test_multicast_lowering_host(m, mc):
    """Option multicast (NEXT-1): rows of vertices requested by >= k GPUs (1: every peer) leave
    by one multicast group per owner + per-requester unpack groups.  The host interpreter runs the
    groups and the work items (a multicast store reaching every rank's region copy) and the halos
    equal oracle.halo.forward bit for bit; the number of multicast rows is the number of vertices
    whose fan-out, counted by the oracle, reaches the threshold; the backward is untouched."""
    import paper_conf_eurosys_cai0wmcy21_b200 as D
    g = synth.make_graph(3000, 60000, m, graph_seed=3 + m, part_seed=4)
    ctx = D.loopback(m, g.part, [24], device=-1)
    ctx.set_option("multicast", mc)
    ctx.build_plan(g.req_ptr, g.req_ids)
    k = m - 1 if mc == 1 else mc
    R = [g.R(d) for d in range(m)]
    assert ctx.plan_info()["n_multicast_rows"] == int((halo.fanout(R, g.n) >= k).sum()) > 0
    order = np.argsort(g.part, kind="stable")
    loc, nl = halo.local_rows(g.part, m)
    ro = np.concatenate([[0], np.cumsum(nl)])
    emb = synth.fill_values(g.n, 24, keys=order)
    Ho = halo.forward([emb[ro[d]:ro[d + 1]] for d in range(m)], R, g.part, loc)
    for items in (0, 1):
        ctx.set_option("hostsim_items", items)
        H = np.zeros((int(g.req_ptr[-1]), 24), np.float32)
        ctx.debug_hostsim_forward(0, emb, H)
        for d in range(m):
            a, b = int(g.req_ptr[d]), int(g.req_ptr[d + 1])
            assert np.array_equal(H[a:b].view(np.uint32), Ho[d].view(np.uint32))
    Gr = synth.fill_values(int(g.req_ptr[-1]), 24, seed=4)
    L = synth.fill_values(g.n, 24, keys=order, seed=5)
    out = L.copy()
    ctx.debug_hostsim_backward(0, Gr, out)
    Bf = halo.backward_flat([L[ro[d]:ro[d + 1]] for d in range(m)],
                            [Gr[g.req_ptr[d]:g.req_ptr[d + 1]] for d in range(m)], R, g.part, loc)
    for d in range(m):
        assert np.array_equal(out[ro[d]:ro[d + 1]].view(np.uint32), Bf[d].view(np.uint32))


@pytest.mark.parametrize("m,explicit", [(2, False), (4, False), (8, False), (8, True), (16, False)])
def test_uniform_closed_form_equals_spst_loop(m, explicit):
    """Planning at scale (NEXT-4): on the uniform switch model SPST's result is the direct star of
    every vertex (DESIGN.md §11 proof), computed in parallel.  It must equal Algorithm 1's loop
    (option spst_fast = 0) edge for edge, with the same t(S); the topology may also be given
    explicitly (dgcl_set_topology with synth.uniform_nvswitch)."""
    import paper_conf_eurosys_cai0wmcy21_b200 as D
    g = synth.make_graph(4000, 50000, m, graph_seed=70 + m, part_seed=71)
    plans, costs = [], []
    for fast in (1, 0):
        ctx = D.loopback(m, g.part, [8], device=-1)
        ctx.set_option("spst_fast", fast)
        ctx.build_plan(g.req_ptr, g.req_ids, seed=13,
                       topology=synth.uniform_nvswitch(m) if explicit else None)
        plans.append(ctx.plan_export())
        costs.append(ctx.plan_info()["model_cost_ticks"])
        ctx.destroy()
    assert np.array_equal(plans[0], plans[1]) and costs[0] == costs[1]
    assert np.all(plans[0][:, 3] == 1)


@pytest.mark.parametrize("seed", range(16))
def test_random_lowering_host(seed):
    """Seeded random sweep of the planning + lowering options (ranks, topology, dims, item sizes,
    geometry, staged folds, reduce form, multicast, fan-out, vertex blocks): the host interpreter
    of the fused program's work items and groups against the oracle, the plan against the
    oracle's SPST and invariants."""
    rng = np.random.RandomState(1000 + seed)
    m = int(rng.choice([2, 3, 4, 6, 8]))
    topo = synth.topology.by_name("ring", m) if (m >= 4 and rng.rand() < 0.4) else None
    opts = {"hostsim_items": int(rng.rand() < 0.7)}
    for key, vals in (("geometry", [0, 1, 2]), ("stage_fold", [0, 1]),
                      ("direct_reduce", [0, 1]), ("align_sources", [0, 1]),
                      ("item_bytes", [1024, 8192, 65536]), ("owner_major", [0, 1]),
                      ("relay_lead_kb", [-1, 0, 1, 196608])):
        opts[key] = int(rng.choice(vals))
    if topo is None:
        r = rng.rand()
        if r < 0.3:
            opts["multicast"] = int(rng.choice([1, 2]))
        elif r < 0.5:
            opts["fanout"] = 1
    else:
        opts["pipeline_blocks"] = int(rng.choice([1, 2, 4]))
    dims = [int(rng.choice([3, 12, 64, 257])) for _ in range(int(rng.randint(1, 3)))]
    n = int(rng.choice([300, 900, 2000]))
    g = synth.make_graph(n, 8 * n, m, graph_seed=300 + seed, part_seed=400 + seed)
    _check_lowering(g, dims, topo, seed=seed, options=opts)


# ---- the flag protocol of the lowered programs, checked on the host ----------------------------
_PROTO_OPTS = [{"leaf_split": 0}, {"leaf_split": 1}, {"leaf_split": 2}, {"pipeline_blocks": 4},
               {"fanout": 1}, {"fanout": 1, "leaf_split": 1}, {"direct_reduce": 0},
               {"stage_fold": 0}, {"geometry": 2}, {"relay_lead_kb": -1}, {"relay_lead_kb": 0},
               {"relay_lead_kb": 1}, {"leaf_split": 2, "relay_lead_kb": 1},
               {"leaf_split": 2, "fanout": 1, "relay_lead_kb": 2}, {"owner_major": 1}]


@pytest.mark.parametrize("topo", ["dgx1_like", "ring", None])
@pytest.mark.parametrize("per_rank", [0, 1])
def test_protocol_check(topo, per_rank):
    """Every lowered program passes the host protocol check (dgcl_debug_check_protocol): wait
    targets equal the rows signalled on their counters, no deadlock in list order, every row read
    in the launch it is written is read only after waiting on its writer's counter,
    each halo row written once.  Relay plans under every stage-chaining variant (leaf split off /
    stages >= 2 / every stage, vertex blocks, per-pair stage 1, staged backward)."""
    D = _D()
    g = synth.make_graph(4000, 20000, 8, graph_seed=5, part_seed=6)
    flags = D.LOOPBACK_PER_RANK if per_rank else D.LOOPBACK_FUSED
    opts_list = _PROTO_OPTS + ([{"multicast": 1}, {"multicast": 3}] if topo is None else [])
    for opts in opts_list:
        ctx = D.loopback(8, g.part, [40, 3], device=-1, flags=flags)
        for k, v in opts.items():
            ctx.set_option(k, v)
        ctx.build_plan(g.req_ptr, g.req_ids, seed=9,
                       topology=synth.topology.by_name(topo) if topo else None)
        for layer in range(2):
            for d in range(2):
                assert ctx.debug_check_protocol(layer, d).startswith("ok"), (opts, layer, d)


@pytest.mark.parametrize("per_rank", [0, 1])
def test_protocol_check_rejects(per_rank):
    """The checker's negative pins: a stage-chained item that stops waiting (race), the same item
    moved before its producers (deadlock in one list; across per-rank lists it only waits), a
    repeated data item (row written twice / counter overshoot), a producer that stops signalling
    (target never reached)."""
    D = _D()
    g = synth.make_graph(4000, 20000, 8, graph_seed=5, part_seed=6)
    flags = D.LOOPBACK_PER_RANK if per_rank else D.LOOPBACK_FUSED
    for topo in ("dgx1_like", "ring"):
        ctx = D.loopback(8, g.part, [40], device=-1, flags=flags)
        ctx.build_plan(g.req_ptr, g.req_ids, seed=9, topology=synth.topology.by_name(topo))
        assert ctx.debug_check_protocol(0, 0).startswith("ok")
        for mu, what in ((1, "without waiting|before it is written"), (2, "deadlock"),
                         (3, "written twice|ever signalled"), (4, "ever signalled")):
            if mu == 2 and per_rank:
                assert ctx.debug_check_protocol(0, 0, mu).startswith("ok")
                continue
            with pytest.raises(D.DGCLError, match=what):
                ctx.debug_check_protocol(0, 0, mu)
        if per_rank:  # staged backward: slot reads chained the same way
            with pytest.raises(D.DGCLError, match="before it is written|without waiting"):
                ctx.debug_check_protocol(0, 1, 1)


@pytest.mark.parametrize("name", ["google8_ring", "google8_dgx1", "reddit_dgx1", "google8"])
def test_protocol_check_full_size(name):
    """The BASELINE configs' programs at full size (fused and per-rank) pass the protocol check."""
    D = _D()
    c = synth.get_config(name)
    g = synth.make_graph(c.n, c.e, c.m, c.graph_seed, c.part_seed, keep_edges=False)
    topo = synth.topology.by_name(c.topology, c.m) if c.topology != "uniform_nvswitch" else None
    for flags in (D.LOOPBACK_FUSED, D.LOOPBACK_PER_RANK):
        ctx = D.loopback(c.m, g.part, list(c.dims), device=-1, flags=flags)
        ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo)
        for layer in range(len(c.dims)):
            for d in range(2):
                assert ctx.debug_check_protocol(layer, d).startswith("ok"), (flags, layer, d)
