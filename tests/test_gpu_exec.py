"""GPU parity tests of the sm_100a executor through the C ABI (-m gpu).

Every case compares the CUDA path with the oracle element by element on seeded inputs:
  * forward halos bit-exact (uint32 view);
  * backward bit-exact against the flat oracle for single-stage plans and against the tree-order
    oracle for relay plans; the flat oracle within |gpu - ref| <= 1e-6 * sum|terms| (R6);
  * determinism (repeat -> identical bits), the G = 1 closed form, both loopback modes (fused and
    per-rank with the full ready/done flag protocol), 16-B and 4-B paths, ragged tails, empty
    halos, the host-buffer (e2e) entry points, the watchdog (ETIMEOUT) and argument errors.
Full-size configs (BASELINE.json) are checked on sampled rows the oracle recomputes one by one
from the hash-defined inputs, plus properties that hold at any size.
"""
import os

import numpy as np
import pytest

import synth
from oracle import halo

pytestmark = [pytest.mark.gpu, pytest.mark.usefixtures("built")]


def _torch():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def _D():
    import paper_conf_eurosys_cai0wmcy21_b200 as D
    return D


class Case:
    """Loopback job: graph + a context + device inputs in the loopback layouts."""

    def __init__(self, g, dims, topo=None, seed=0, flags=0, emb_pitch=None, mode="uniform",
                 options=None):
        torch = _torch()
        D = _D()
        self.g, self.m, self.dims = g, g.m, list(dims)
        self.ctx = D.loopback(g.m, g.part, dims, device=0, flags=flags)
        # test graphs are small: force the bulk-copy executor unless a case asks otherwise (the
        # default hands launches under small_launch_bytes to the register executor)
        for k, v in dict({"small_launch_bytes": 0}, **(options or {})).items():
            self.ctx.set_option(k, v)
        self.ctx.build_plan(g.req_ptr, g.req_ids, seed=seed, topology=topo)
        self.ctx.register_workspace()
        self.order = np.argsort(g.part, kind="stable")   # loopback row -> global vertex id
        self.S = int(g.req_ptr[-1])
        self.mode = mode
        self.emb_pitch = emb_pitch
        self.loc, _ = halo.local_rows(g.part, g.m)
        self.R = [g.R(d) for d in range(g.m)]
        self.torch = torch

    def pitch(self, layer):
        return self.ctx.halo_view(layer)[2]

    def emb(self, layer, seed=3):
        p = self.emb_pitch or self.pitch(layer)
        return synth.fill_values(self.g.n, self.dims[layer], p, keys=self.order, seed=seed,
                                 stream=synth.values.STREAM_EMB + layer, mode=self.mode)

    def grads(self, layer, seed=4, mode=None):
        mode = mode or self.mode
        p = self.emb_pitch or self.pitch(layer)
        G = synth.fill_values(self.S, self.dims[layer], p, seed=seed,
                              stream=synth.values.STREAM_HGRAD + layer, mode=mode)
        L = synth.fill_values(self.g.n, self.dims[layer], p, keys=self.order, seed=seed,
                              stream=synth.values.STREAM_EGRAD + layer, mode=mode)
        return G, L

    def dev(self, a):
        return self.torch.from_numpy(a).cuda()

    def run_forward(self, layer, emb):
        out = self.ctx.forward(layer, self.dev(emb))
        self.torch.cuda.synchronize()
        self.ctx.check()
        return out.cpu().numpy()

    def run_backward(self, layer, G, L):
        eg = self.dev(L)
        self.ctx.backward(layer, self.dev(G), eg)
        self.torch.cuda.synchronize()
        self.ctx.check()
        return eg.cpu().numpy()

    # oracle views
    def local(self, a, dim):
        ro = self.ctx.row_off
        return [a[ro[d]:ro[d + 1], :dim] for d in range(self.m)]

    def halos(self, a, dim):
        ho = self.g.req_ptr
        return [a[ho[d]:ho[d + 1], :dim] for d in range(self.m)]


def _eq(a, b):
    return np.array_equal(np.ascontiguousarray(a).view(np.uint32),
                          np.ascontiguousarray(b).view(np.uint32))


def _check_case(c, layers=None, bwd=True):
    layers = range(len(c.dims)) if layers is None else layers
    info = c.ctx.plan_info()
    E = c.ctx.plan_export()
    for layer in layers:
        dim = c.dims[layer]
        emb = c.emb(layer)
        H = c.run_forward(layer, emb)
        Ho = halo.forward(c.local(emb, dim), c.R, c.g.part, c.loc)
        for d in range(c.m):
            assert _eq(c.halos(H, dim)[d], Ho[d]), "forward mismatch layer %d rank %d" % (layer, d)
        if not bwd:
            continue
        G, L = c.grads(layer)
        out = c.run_backward(layer, G, L)
        Bt = halo.backward_tree(c.local(L, dim), c.halos(G, dim), c.R, c.g.part, c.loc, E)
        for d in range(c.m):
            assert _eq(c.local(out, dim)[d], Bt[d]), "backward (tree order) rank %d" % d
        Bf = halo.backward_flat(c.local(L, dim), c.halos(G, dim), c.R, c.g.part, c.loc)
        if info["n_stages"] <= 1:
            for d in range(c.m):
                assert _eq(c.local(out, dim)[d], Bf[d]), "backward (flat order) rank %d" % d
        else:
            # plan-agnostic oracle: |gpu - ref| <= 1e-6 * sum|terms|
            absL = [np.abs(x) for x in c.local(L, dim)]
            absG = [np.abs(x) for x in c.halos(G, dim)]
            bound = halo.backward_flat(absL, absG, c.R, c.g.part, c.loc)
            for d in range(c.m):
                diff = np.abs(c.local(out, dim)[d].astype(np.float64) - Bf[d])
                assert np.all(diff <= 1e-6 * bound[d] + 0.0), "flat tolerance rank %d" % d
        # determinism: identical bits on a second run
        out2 = c.run_backward(layer, G, L)
        assert _eq(out, out2)


@pytest.mark.parametrize("small", [0, 4 << 20])
def test_tiny_config_bit_exact(small):
    """configs[0]: 10k vertices, 100k edges, random 2-way, dim 16, one layer fwd + bwd — through
    the bulk-copy executor (small=0) and through the default latency choice (register executor
    below 4 MiB per launch)."""
    cfg = synth.get_config("tiny")
    g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed)
    _check_case(Case(g, cfg.dims, options={"small_launch_bytes": small}))


@pytest.mark.parametrize("m,opts", [
    (3, {}), (4, {}), (8, {}),
    (8, {"bulk_store": 0}),
    (4, {"tma": 0}), (8, {"tma": 0}),
    (8, {"direct_reduce": 0}), (3, {"tma": 0, "direct_reduce": 0}),
    (4, {"direct_reduce": 0, "bulk_store": 0}),
    (8, {"gather4": 0}),
    (4, {"direct_copy_rows": 4}),
    # direct COPY items on the register path (a launch of direct copies + folds must
    # not reach the fold-only instance), forced (tma=0) and by the default latency choice
    (4, {"direct_copy_rows": 4, "tma": 0}), (4, {"direct_copy_rows": 4, "tma": 0, "direct_reduce": 0}),
    (8, {"direct_copy_rows": 4, "small_launch_bytes": 4 << 20, "direct_reduce": 0}),
    (8, {"direct_copy_rows": 4, "small_launch_bytes": 4 << 20}),
    (8, {"stage_fold": 0}), (4, {"stage_fold": 0, "direct_reduce": 0}),
    (8, {"direct_reduce": 0, "item_bytes": 4096}),
    (8, {"geometry": 1}), (8, {"geometry": 2}), (4, {"geometry": 2, "direct_reduce": 0}),
    (3, {"geometry": 1, "stage_fold": 0}),
    # two producer warps (simple copy launches on the WIDE geometry) and one
    (8, {"geometry": 1, "gather4": 0}), (3, {"geometry": 1, "gather4": 0, "item_bytes": 4096}),
    (8, {"geometry": 1, "gather4": 0, "dual_producer": 0}),
    # dual producers with dynamic claims (each claims its own batches)
    (4, {"geometry": 1, "claim_batch": 2}), (8, {"claim_batch": 3, "item_bytes": 4096}),
    (2, {"geometry": 1, "claim_batch": 1, "dual_claims": 0}),
    # item order of fused forwards: chunk-major / group-major (default owner-major)
    (8, {"owner_major": 0}), (8, {"owner_major": 2}), (4, {"owner_major": 2, "align_sources": 0}),
    (8, {"fanout": 1}), (4, {"fanout": 1, "tma": 0}), (8, {"fanout": 1, "geometry": 2}),
    (3, {"fanout": 1, "bulk_store": 0}), (4, {"fanout": 1, "geometry": 1}),
    # NVSwitch multicast of high-fan-out rows, emulated on one GPU (one store per virtual rank's
    # region copy): send + unpack groups, multicast done counters
    (8, {"multicast": 1}), (4, {"multicast": 2}), (4, {"multicast": 1, "tma": 0}),
    (3, {"multicast": 1, "geometry": 2}), (8, {"multicast": 3, "small_launch_bytes": 4 << 20}),
    # consumer cp.async gathers for short-run items (option lsu_gather), both geometries
    (8, {"lsu_gather": 1}), (4, {"lsu_gather": 1, "geometry": 1}),
    (3, {"lsu_gather": 1, "bulk_store": 0}), (4, {"lsu_gather": 1, "direct_reduce": 0}),
])
def test_uniform_loopback_fused(m, opts):
    """Executor variants: tma (bulk-copy executor vs the register LDG executor), direct_reduce
    (loopback in-place reduce vs push to slots + owner reduce, the multi-GPU form), bulk_store
    (TMA stores vs 16-B st.global), gather4 (TMA row gather of 4 rows per instruction vs one bulk
    copy per run), direct_copy_rows (consumer-side gathers for short runs), stage_fold (backward
    folds with every operand row bulk-copied into shared memory vs consumer gathers), fanout
    (forward stage 1 as per-owner fan-out items vs one COPY group per (owner, receiver))."""
    g = synth.make_graph(6000, 60000, m, graph_seed=m, part_seed=7 * m)
    _check_case(Case(g, [64, 5, 602, 32], options=opts))


@pytest.mark.parametrize("m,fanout,mc", [(2, 1, 0), (8, 1, 0), (8, 0, 0), (8, 0, 1), (4, 0, 2)])
def test_per_rank_flag_protocol(m, fanout, mc):
    """Every virtual rank is its own launch on its own stream: ready handshake, done counters,
    forward completion waits — the multi-GPU protocol on one device; several calls in a row.
    mc: the (emulated) multicast path, whose sends wait on every peer's ready word and whose
    unpacks wait on the owners' multicast counters."""
    D = _D()
    g = synth.make_graph(5000, 40000, m, graph_seed=11, part_seed=12)
    c = Case(g, [32, 7], flags=D.LOOPBACK_PER_RANK, options={"fanout": fanout, "multicast": mc})
    if mc:
        assert c.ctx.plan_info()["n_multicast_rows"] > 0
    for _ in range(2):
        _check_case(c)


@pytest.mark.parametrize("name,flags,tma,sf", [("dgx1_like", 0, 1, 1), ("ring", 0, 1, 1),
                                               ("dgx1_like", 1, 1, 1), ("ring", 1, 1, 1),
                                               ("ring", 0, 0, 1), ("dgx1_like", 1, 0, 1),
                                               ("ring", 1, 1, 0), ("dgx1_like", 0, 1, 0),
                                               ("ring", 0, 1, 2), ("dgx1_like", 1, 1, 3),
                                               ("dgx1_like", 0, 1, 4), ("ring", 1, 1, 4),
                                               ("ring", 0, 1, 5), ("dgx1_like", 1, 1, 6),
                                               ("ring", 1, 0, 6), ("ring", 0, 1, 7),
                                               ("dgx1_like", 0, 1, 7), ("ring", 1, 1, 7),
                                               ("dgx1_like", 0, 0, 7), ("ring", 0, 1, 8),
                                               ("dgx1_like", 1, 1, 8), ("ring", 0, 1, 9),
                                               ("dgx1_like", 0, 0, 9), ("ring", 1, 1, 9),
                                               ("dgx1_like", 0, 1, 10), ("ring", 0, 1, 11),
                                               ("ring", 0, 1, 12), ("ring", 0, 1, 13),
                                               ("dgx1_like", 1, 1, 13)])
def test_relay_plans(name, flags, tma, sf):
    """sf: stage_fold 0/1; 2, 3 = stage_fold with the DUAL / WIDE geometry forced; 4 = fan-out
    stage 1 (first hops into halos and relay staging, done counts per receiver); 5, 6 = one /
    eight vertex blocks in the stage chaining (default 1); 7 = the staged reversed-plan backward
    (direct_reduce = 0: pushes into slots stage by stage, the multi-GPU form) instead of the
    loopback tree-order programs; 8 / 9 = the relay item order off (relay_lead_kb -1) / with a
    1-KB lead (forwarded rows of the next stage right behind a few leaves); 10 = no leaf split;
    11 / 12 = chunk-major / group-major stage 1 (owner_major 0 / 2); 13 = dims 256 / 602 (rows
    >= 1 KB: relay stages store scattered rows with one bulk store per row)."""
    g = synth.make_graph(4000, 20000, 8, graph_seed=5, part_seed=6)
    opts = {"tma": tma, "stage_fold": min(sf, 1)}
    if sf in (2, 3):
        opts["geometry"] = 2 if sf == 2 else 1
    if sf == 4:
        opts["fanout"] = 1
    if sf in (5, 6):
        opts["pipeline_blocks"] = 1 if sf == 5 else 8
    if sf == 7:
        opts["direct_reduce"] = 0
    if sf in (8, 9):
        opts["relay_lead_kb"] = -1 if sf == 8 else 1
    if sf == 10:
        opts["leaf_split"] = 0
    if sf in (11, 12):
        opts["owner_major"] = 0 if sf == 11 else 2
    dims = [256, 602] if sf == 13 else [40, 3]
    c = Case(g, dims, topo=synth.topology.by_name(name), seed=9, flags=flags, options=opts)
    assert c.ctx.plan_info()["n_stages"] >= 2
    _check_case(c)


@pytest.mark.parametrize("tma,flags,blocks,leaf", [(1, 0, 4, 2), (0, 0, 4, 2), (1, 1, 4, 2),
                                                   (1, 0, 1, 0), (1, 0, 1, 2), (1, 1, 1, 2),
                                                   (0, 1, 1, 1)])
def test_trace_stage_causality(tma, flags, blocks, leaf):
    """Option "trace": per-item timelines of a relay plan's forward.  Stage chaining on device
    flags means no stage-k item of GPU r passes its waits before every stage-(k-1) item of the
    same vertex block into r has stored its rows; every item is traced once, in
    order start <= ready <= done; with blocks, later blocks' stage k-1 may still be running.
    Leaf split (one block): the stage-(k-1) rows r forwards are block 0; r's stage-k items wait
    for those, not for the leaf deliveries (block 1) of stage k-1."""
    D = _D()
    g = synth.make_graph(4000, 20000, 8, graph_seed=5, part_seed=6)
    c = Case(g, [40], topo=synth.topology.by_name("dgx1_like"), seed=9, flags=flags,
             options={"tma": tma, "trace": 1, "pipeline_blocks": blocks, "leaf_split": leaf})
    K = c.ctx.plan_info()["n_stages"]
    assert K >= 2
    _check_case(c, bwd=False)
    ranks = range(c.m) if flags == D.LOOPBACK_PER_RANK else [0]
    T = [c.ctx.trace(0, 0, r) for r in ranks]
    T = {k: np.concatenate([t[k] for t in T]) for k in T[0]}
    data = (T["op"] <= 1) | (T["op"] == 6)  # COPY, FOLD, FANOUT
    assert data.sum() > 0 and np.all(T["t_start"][data] > 0)
    assert np.all(T["t_start"][data] <= T["t_ready"][data])
    assert np.all(T["t_ready"][data] <= T["t_done"][data])
    split = blocks == 1 and leaf > 0
    if split:
        assert (T["block"][data] == 1).any()  # leaf deliveries exist on this plan
    for r in range(c.m):
        for k in range(2, K + 1):
            for b in range(8):
                after = data & (T["exec"] == r) & (T["stage"] == k) & (T["block"] == b)
                before = data & (T["dst"] == r) & (T["stage"] == k - 1) & \
                    (T["block"] == (0 if split else b))
                if after.any() and before.any():
                    assert T["t_ready"][after].min() >= T["t_done"][before].max(), (r, k, b)


def test_unaligned_pitch_scalar_path():
    g = synth.make_graph(3000, 20000, 4, graph_seed=2, part_seed=2)
    _check_case(Case(g, [5], emb_pitch=5))   # 20-B rows: not 16-B aligned -> 4-B path


def test_small_items_many_chunks():
    g = synth.make_graph(3000, 20000, 4, graph_seed=3, part_seed=3)
    _check_case(Case(g, [37], options={"item_bytes": 64, "ctas_per_sm": 1, "threads": 128}))


def test_shuffled_halo_order_idx_lists():
    g = synth.make_graph(3000, 25000, 4, graph_seed=8, part_seed=8)
    g.req_ids = synth.graph.shuffle_lists(g.req_ptr, g.req_ids, 5)
    _check_case(Case(g, [24]))


def test_empty_halo_rank_and_no_requests():
    part = np.array([0, 1, 2, 0, 1, 2], np.int32)
    g = synth.Graph(6, 3, None, None, part, np.array([0, 2, 2, 3], np.int64),
                    np.array([1, 5, 0], np.int64))   # GPU 1 requires nothing
    _check_case(Case(g, [4]))


@pytest.mark.parametrize("topo,flags,opts", [(None, 0, {}), ("ring", 0, {}), ("dgx1_like", 1, {}),
                                             ("ring", 0, {"direct_reduce": 0}),
                                             (None, 1, {"tma": 0})])
def test_closed_form_ones_and_integer_inputs(topo, flags, opts):
    """Backward closed forms on direct and relay plans: G = 1, L = 0 gives |D_u| (counted by the
    oracle from the required lists) in every column; integer-valued inputs (|x| <= 8, every
    partial sum exact in fp32) make every summation order exact, so the result must equal the
    flat oracle bit for bit whatever the tree."""
    g = synth.make_graph(5000, 50000, 8 if topo else 4, graph_seed=21, part_seed=22)
    t = synth.topology.by_name(topo) if topo else None
    c = Case(g, [16], topo=t, seed=2, flags=flags, options=opts)
    G, L = c.grads(0, mode="ones")
    out = c.run_backward(0, G, np.zeros_like(L))
    fan = halo.fanout(c.R, g.n)
    want = fan[c.order].astype(np.float32)
    assert np.array_equal(out[:, 0], want) and np.array_equal(out[:, 15], want)
    Gi, Li = c.grads(0, mode="int")
    outi = c.run_backward(0, Gi, Li)
    Bf = halo.backward_flat(c.local(Li, 16), c.halos(Gi, 16), c.R, g.part, c.loc)
    for d in range(c.m):
        assert _eq(c.local(outi, 16)[d], Bf[d]), "integer inputs rank %d" % d


def test_host_buffer_entry_points():
    g = synth.make_graph(2000, 15000, 2, graph_seed=31, part_seed=32)
    c = Case(g, [16])
    emb = c.emb(0)
    H = np.zeros((c.S, c.pitch(0)), np.float32)
    c.ctx.forward_host(0, emb, H)
    Ho = halo.forward(c.local(emb, 16), c.R, g.part, c.loc)
    for d in range(2):
        assert _eq(c.halos(H, 16)[d], Ho[d])
    G, L = c.grads(0)
    out = L.copy()
    c.ctx.backward_host(0, G, out)
    Bf = halo.backward_flat(c.local(L, 16), c.halos(G, 16), c.R, g.part, c.loc)
    for d in range(2):
        assert _eq(c.local(out, 16)[d], Bf[d])


def test_host_buffer_calls_pipelined():
    """host_async: a queue of host-buffer calls (inputs copied in while the previous outputs are
    copied out, per-layer staging) gives the same bits as the oracle once the stream is synced;
    the same layer twice in a row exercises the staging / halo reuse ordering."""
    torch = _torch()
    g = synth.make_graph(3000, 25000, 4, graph_seed=33, part_seed=34)
    c = Case(g, [16, 40])
    c.ctx.set_option("host_async", 1)
    pin = lambda a: torch.from_numpy(a).pin_memory()
    embs = [pin(c.emb(0, seed=3)), pin(c.emb(1, seed=5)), pin(c.emb(0, seed=7))]
    layers = [0, 1, 0]
    Hs = [torch.zeros(c.S, c.pitch(l), dtype=torch.float32).pin_memory() for l in layers]
    G, L = c.grads(1)
    Gp, out = pin(G), pin(L.copy())
    s = torch.cuda.current_stream()
    for l, e, H in zip(layers, embs, Hs):
        c.ctx.forward_host(l, e, H, stream=s)
    c.ctx.backward_host(1, Gp, out, stream=s)
    s.synchronize()
    for l, e, H in zip(layers, embs, Hs):
        dim = c.dims[l]
        Ho = halo.forward(c.local(e.numpy(), dim), c.R, g.part, c.loc)
        for d in range(c.m):
            assert _eq(c.halos(H.numpy(), dim)[d], Ho[d])
    Bf = halo.backward_flat(c.local(L, 40), c.halos(G, 40), c.R, g.part, c.loc)
    for d in range(c.m):
        assert _eq(c.local(out.numpy(), 40)[d], Bf[d])


def test_watchdog_timeout_when_a_rank_never_arrives():
    D = _D()
    g = synth.make_graph(2000, 15000, 4, graph_seed=41, part_seed=42)
    c = Case(g, [8], flags=D.LOOPBACK_PER_RANK)
    c.ctx.set_option("timeout_ms", 300)
    c.ctx.set_option("debug_skip_rank", 2)
    emb = c.dev(c.emb(0))
    c.ctx.forward(0, emb)
    c.torch.cuda.synchronize()
    with pytest.raises(D.DGCLError) as e:
        c.ctx.check()
    assert e.value.status == 5
    with pytest.raises(D.DGCLError) as e:   # the context stays unusable
        c.ctx.forward(0, emb)
    assert e.value.status == 5


def test_argument_errors():
    D = _D()
    g = synth.make_graph(1000, 8000, 2, graph_seed=51, part_seed=52)
    c = Case(g, [16])
    torch = c.torch
    emb = torch.zeros(g.n, 16, device="cuda")
    with pytest.raises(D.DGCLError) as e:
        c.ctx.forward(0, emb, halo=torch.zeros(4, 16, device="cuda"))  # not the registered view
    assert e.value.status == 1
    with pytest.raises(D.DGCLError) as e:
        c.ctx.forward(3, emb)
    assert e.value.status == 1
    with pytest.raises(D.DGCLError) as e:
        c.ctx.forward(0, torch.zeros(g.n, 8, device="cuda"))            # pitch < dim
    assert e.value.status == 1
    # what only the binding can see (the C side gets a pointer and a pitch): dtype, device,
    # column stride, row count
    for bad in (torch.zeros(g.n, 16, device="cuda", dtype=torch.bfloat16),
                torch.zeros(g.n, 16),                                   # host tensor
                torch.zeros(16, g.n, device="cuda").t(),                # column-strided
                torch.zeros(g.n - 1, 16, device="cuda")):               # too few rows
        with pytest.raises(D.DGCLError) as e:
            c.ctx.forward(0, bad)
        assert e.value.status == 1
    hg = torch.zeros(c.S, 16, device="cuda")
    with pytest.raises(D.DGCLError) as e:
        c.ctx.backward(0, hg[:-1], torch.zeros(g.n, 16, device="cuda"))  # halo_grad too short
    assert e.value.status == 1
    with pytest.raises(D.DGCLError) as e:
        c.ctx.backward(0, hg, torch.zeros(g.n, 16, device="cuda", dtype=torch.float16))
    assert e.value.status == 1


def test_autograd_graph_allgather():
    torch = _torch()
    D = _D()
    g = synth.make_graph(1500, 10000, 2, graph_seed=61, part_seed=62)
    c = Case(g, [16])
    emb = torch.from_numpy(c.emb(0)).cuda().requires_grad_(True)
    out = D.graph_allgather(c.ctx, 0, emb)
    assert out.shape[0] == g.n + c.S
    w = torch.from_numpy(synth.fill_values(out.shape[0], 16, seed=8, stream=3)).cuda()
    (out * w).sum().backward()
    wn = w.cpu().numpy()
    Bf = halo.backward_flat(c.local(wn[:g.n], 16), c.halos(wn[g.n:], 16), c.R, g.part, c.loc)
    got = emb.grad.cpu().numpy()
    for d in range(2):
        assert _eq(c.local(got, 16)[d], Bf[d])


# ---- full-size configs (BASELINE.json): every row against oracle/halo ---------------------

def _r6_bound(c, L, G, dim):
    """R6: |gpu - flat| <= 1e-6 * sum|terms| per element, the terms folded in the
    flat order by the oracle itself on |L|, |G| (every partial sum of non-negative terms)."""
    absL = [np.abs(x) for x in c.local(L, dim)]
    absG = [np.abs(x) for x in c.halos(G, dim)]
    return halo.backward_flat(absL, absG, c.R, c.g.part, c.loc)


def _full_size(name):
    """Every halo row and every owner row of a BASELINE config (in the configuration bench.py
    times: fused loopback, bulk-copy executor) against the oracle:
      * the exported plan passes oracle.invariants.check_plan (trees, exactly-once delivery,
        links exist, t(S) recomputed = the library's reported cost);
      * forward: each rank's halo bit-exact (uint32 view) vs oracle.halo.forward, one rank at a
        time (the other ranks' lists empty), so host memory holds one rank's halo;
      * backward (the config's backward layers): bit-exact vs oracle.halo.backward_tree (the
        plan's fixed order) always; vs backward_flat bit-exact on single-stage plans, within the
        R6 bound on relay plans; a second run gives identical bits."""
    from oracle import invariants
    cfg = synth.get_config(name)
    g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
    topo = synth.topology.by_name(cfg.topology, cfg.m)
    c = Case(g, list(cfg.dims), topo=None if cfg.topology == "uniform_nvswitch" else topo, seed=0)
    info = c.ctx.plan_info()
    E = c.ctx.plan_export()
    D = {}
    for d in range(c.m):
        for u in c.R[d].tolist():
            D.setdefault(u, []).append(d)
    invariants.check_plan(topo, E.tolist(), g.part, D, reported_cost=info["model_cost_ticks"])
    del D
    empty = np.zeros(0, np.int64)
    for layer, dim in enumerate(cfg.dims):
        emb = c.emb(layer)
        c.ctx.forward(layer, c.dev(emb))
        c.torch.cuda.synchronize()
        c.ctx.check()
        Hdev = c.ctx.halo(layer)
        loc_emb = c.local(emb, dim)
        for d in range(c.m):
            Rq = [c.R[q] if q == d else empty for q in range(c.m)]
            want = halo.forward(loc_emb, Rq, g.part, c.loc)[d]
            got = Hdev[int(g.req_ptr[d]):int(g.req_ptr[d + 1]), :dim].cpu().numpy()
            assert _eq(got, want), "forward mismatch (%s layer %d rank %d)" % (name, layer, d)
            del got, want
        del Hdev, emb, loc_emb
        if layer not in cfg.backward_layers:
            continue
        G, L = c.grads(layer)
        out = c.run_backward(layer, G, L)
        Bt = halo.backward_tree(c.local(L, dim), c.halos(G, dim), c.R, g.part, c.loc, E)
        for d in range(c.m):
            assert _eq(c.local(out, dim)[d], Bt[d]), "backward (tree order) %s rank %d" % (name, d)
        del Bt
        Bf = halo.backward_flat(c.local(L, dim), c.halos(G, dim), c.R, g.part, c.loc)
        if info["n_stages"] <= 1:
            for d in range(c.m):
                assert _eq(c.local(out, dim)[d], Bf[d]), "backward (flat) %s rank %d" % (name, d)
        else:
            bound = _r6_bound(c, L, G, dim)
            for d in range(c.m):
                diff = np.abs(c.local(out, dim)[d].astype(np.float64) - Bf[d])
                assert np.all(diff <= 1e-6 * bound[d]), "R6 bound %s rank %d" % (name, d)
            del bound
        del Bf
        out2 = c.run_backward(layer, G, L)
        assert _eq(out, out2), "backward not reproducible (%s)" % name
    return c


FULL_CONFIGS = ["tiny", "reddit", "google2", "google4", "google8", "orkut", "google8_dgx1",
                "google8_ring", "reddit_dgx1"]


@pytest.mark.parametrize("name", FULL_CONFIGS)
def test_full_size_every_row(name):
    _full_size(name)


def test_single_rank_is_noop():
    """world = 1: nothing to exchange — forward leaves the (empty) halo alone, backward leaves
    emb_grad unchanged, and no executor launch happens."""
    D = _D()
    torch = _torch()
    part = np.zeros(100, np.int32)
    ctx = D.loopback(1, part, [8], device=0)
    ctx.build_plan([0, 0], [])
    ctx.register_workspace()
    emb = torch.randn(100, 8, device="cuda")
    ctx.forward(0, emb)
    eg = torch.randn(100, 8, device="cuda")
    before = eg.clone()
    ctx.backward(0, torch.zeros(1, 8, device="cuda"), eg)
    torch.cuda.synchronize()
    assert torch.equal(eg, before) and ctx.launch_count() == 0


@pytest.mark.parametrize("flags,topo,opts", [
    (0, None, {}),
    # per-rank launches and relay plans need done counts from exec ranks 14 and 15 published
    # (the FLUSH/END publish covered only the first T of 256 (source, receiver) slots)
    (1, None, {}), (1, None, {"threads": 128}), (0, "ring", {}), (1, "ring", {}),
    (0, "ring", {"direct_reduce": 0}),
])
def test_sixteen_virtual_ranks(flags, topo, opts):
    g = synth.make_graph(8000, 60000, 16, graph_seed=71, part_seed=72)
    t = synth.topology.by_name(topo, 16) if topo else None
    c = Case(g, [24, 64], topo=t, seed=3, flags=flags, options=opts)
    if topo:
        assert c.ctx.plan_info()["n_stages"] >= 2
    _check_case(c)


@pytest.mark.parametrize("dims", [[4000], [20000]])
def test_wide_rows(dims):
    """4000 floats: a few rows per bulk-copy stage; 20000 floats (80 KB rows): wider than a
    stage, so the register executor runs the launch."""
    g = synth.make_graph(600, 3000, 3, graph_seed=81, part_seed=82)
    _check_case(Case(g, dims))


@pytest.mark.parametrize("small,dims", [(0, [64, 602]), (4 << 20, [16]), (0, [5])])
def test_atomic_backward_ablation(small, dims):
    """Option "atomic_backward" (ablation: the paper's Atomic baseline, Table 9):
    requesters add their halo-gradient rows into the owners' rows with atomic reductions (TMA
    bulk reduce-add; fp32 atomics for partial chunks and on the register path).  The order of
    the adds is not fixed, so random inputs are held to the R6 tolerance against the flat
    oracle; integer-valued inputs (every partial sum exact) must match bit for bit, and the
    caller's emb_grad padding (pitch > dim) is never touched."""
    g = synth.make_graph(6000, 60000, 4, graph_seed=21, part_seed=22)
    c = Case(g, dims, seed=1, options={"atomic_backward": 1, "small_launch_bytes": small})
    for layer, dim in enumerate(dims):
        G, L = c.grads(layer)
        p = c.pitch(layer)
        if p > dim:
            L[:, dim:] = 7.0
        out = c.run_backward(layer, G, L)
        if p > dim:
            assert np.all(out[:, dim:] == 7.0)
        Bf = halo.backward_flat(c.local(L, dim), c.halos(G, dim), c.R, c.g.part, c.loc)
        absL = [np.abs(x) for x in c.local(L, dim)]
        absG = [np.abs(x) for x in c.halos(G, dim)]
        bound = halo.backward_flat(absL, absG, c.R, c.g.part, c.loc)
        for d in range(c.m):
            diff = np.abs(c.local(out, dim)[d].astype(np.float64) - Bf[d])
            assert np.all(diff <= 1e-6 * bound[d]), "atomic tolerance rank %d" % d
        Gi, Li = c.grads(layer, mode="int")
        outi = c.run_backward(layer, Gi, Li)
        Bi = halo.backward_flat(c.local(Li, dim), c.halos(Gi, dim), c.R, c.g.part, c.loc)
        for d in range(c.m):
            assert _eq(c.local(outi, dim)[d], Bi[d]), "atomic integer inputs rank %d" % d


@pytest.mark.parametrize("flags,opts", [(1, {}), (0, {"signal_all": 1}),
                                        (1, {"tma": 0}), (0, {"signal_all": 1, "multicast": 1})])
def test_wait_arrival_per_source(flags, opts):
    """dgcl_stream_wait_arrival (overlap, NEXT-2): on a second stream, after the wait for
    (receiver d, source s), the halo rows d received from s equal the oracle's — the halo was
    zeroed before the call, so a read ahead of the rows would show; a device start barrier
    precedes each call (dgcl_device_barrier)."""
    torch = _torch()
    g = synth.make_graph(6000, 60000, 4, graph_seed=91, part_seed=92)
    c = Case(g, [64], flags=flags, options=dict({"sm_budget": 100}, **opts))
    emb = c.emb(0)
    Ho = halo.forward(c.local(emb, 64), c.R, g.part, c.loc)
    e = c.dev(emb)
    side = torch.cuda.Stream()
    for rep in range(2):
        c.ctx.halo(0).zero_()
        torch.cuda.synchronize()
        main = torch.cuda.current_stream()
        c.ctx.device_barrier(main)
        c.ctx.forward(0, e, stream=main)
        got = {}
        with torch.cuda.stream(side):
            for d in range(c.m):
                for s in range(c.m):
                    if s == d:
                        continue
                    c.ctx.wait_arrival(src=s, dst=d, stream=side)
                    a, b = int(g.req_ptr[d]), int(g.req_ptr[d + 1])
                    got[(d, s)] = c.ctx.halo(0)[a:b, :64].clone()
        torch.cuda.synchronize()
        c.ctx.check()
        for (d, s), h in got.items():
            sel = g.part[c.R[d]] == s
            assert _eq(h.cpu().numpy()[sel], Ho[d][sel]), (rep, d, s)


def _random_option_case(seed):
    """A seeded random combination of graph size, ranks, topology, loopback mode, dims and executor
    options (the option interactions the fixed cases do not enumerate)."""
    rng = np.random.RandomState(seed)
    m = int(rng.choice([2, 3, 4, 5, 8]))
    topo = None
    if m == 8 and rng.rand() < 0.5:
        topo = str(rng.choice(["ring", "dgx1_like"]))
    elif m in (4, 5) and rng.rand() < 0.3:
        topo = "ring"
    flags = int(rng.rand() < 0.35)
    dims = [int(rng.choice([4, 16, 37, 64, 128, 256, 602]))
            for _ in range(int(rng.randint(1, 3)))]
    opts = {"small_launch_bytes": int(rng.choice([0, 0, 4 << 20]))}
    for key, vals in (("tma", [0, 1, 1, 1]), ("geometry", [0, 0, 1, 2]),
                      ("claim_batch", [-1, 0, 1, 3]), ("stage_fold", [0, 1, 1]),
                      ("direct_reduce", [0, 1, 1]), ("gather4", [0, 1, 1]),
                      ("bulk_store", [0, 1, 1]), ("l2_policy", [0, 1, 3]),
                      ("align_sources", [0, 1])):
        opts[key] = int(rng.choice(vals))
    if topo is None and rng.rand() < 0.3:
        opts["multicast"] = int(rng.choice([1, 2]))
    elif rng.rand() < 0.2:
        opts["fanout"] = 1
    if rng.rand() < 0.2:
        opts["item_bytes"] = int(rng.choice([2048, 8192]))
    n = int(rng.choice([800, 3000, 7000]))
    # (drawn last: the earlier draws, hence the earlier cases, are unchanged)
    for key, vals in (("owner_major", [0, 1, 1, 2]), ("relay_lead_kb", [-1, 0, 1, 196608]),
                      ("leaf_split", [0, 1, 1, 2]), ("dual_producer", [0, 1, 1]),
                      ("dual_claims", [0, 1, 1])):
        opts[key] = int(rng.choice(vals))
    return m, topo, flags, dims, opts, n


@pytest.mark.parametrize("seed", range(int(os.environ.get("DGCL_RANDOM_CASES", "48"))))
def test_random_option_combinations(seed):
    """Seeded random sweep over executor options, ranks, topologies and loopback modes; every case
    element by element against the oracle (forward bit-exact, backward bit-exact in tree order, flat
    order on single-stage plans, R6 bound otherwise, reproducible)."""
    m, topo, flags, dims, opts, n = _random_option_case(seed)
    g = synth.make_graph(n, 10 * n, m, graph_seed=100 + seed, part_seed=200 + seed)
    t = synth.topology.by_name(topo, m) if topo else None
    _check_case(Case(g, dims, topo=t, seed=seed, flags=flags, options=opts))
