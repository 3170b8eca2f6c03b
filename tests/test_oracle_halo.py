"""Pins for oracle/halo.py against things other than itself (-m "not gpu").

* literal worked example (tests/golden/h2_example.json)
* brute force (explicit loops) on tiny random graphs
* closed form: G = 1, L = 0  =>  out[u] = |D_u|, with |D_u| counted from the EDGES
* integer-valued inputs: every summation order is exact, so a differently ordered float64 sum
  must agree bit-for-bit (pins dropped / duplicated / misindexed terms)
* fp32 order sensitivity: the fixed order of DESIGN.md R6 is observable and pinned
* complete relation: forward == torch.distributed all_gather, backward == all_reduce slice
"""
import json
import os

import numpy as np
import pytest

from oracle import halo
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _h2():
    with open(os.path.join(GOLD, "h2_example.json")) as f:
        g = json.load(f)
    part = np.array([v % 3 for v in range(g["n"])], dtype=np.int32)
    return g, part


def test_h2_required_sets_and_loc():
    g, part = _h2()
    R = halo.required_bruteforce(g["n"], g["edges"], part, g["m"])
    assert [list(r) for r in R] == g["R"]
    loc, n_local = halo.local_rows(part, g["m"])
    for v, r in g["loc"].items():
        assert loc[int(v)] == r
    assert list(n_local) == [3, 3, 3]


def test_h2_forward_halo_sources():
    g, part = _h2()
    loc, n_local = halo.local_rows(part, 3)
    # marker values encode (owner, row): 100*owner + row
    local = [np.array([[100.0 * d + r] for r in range(n_local[d])], dtype=np.float32)
             for d in range(3)]
    H = halo.forward(local, g["R"], part, loc)
    for d in range(3):
        want = [100.0 * o + r for (o, r) in g["halo_sources_owner_row"][d]]
        assert H[d][:, 0].tolist() == want
    assert sum(len(r) for r in g["R"]) == g["n_deliveries"]


def test_h2_all_ones_backward():
    g, part = _h2()
    loc, n_local = halo.local_rows(part, 3)
    L = [np.zeros((n_local[d], 1), np.float32) for d in range(3)]
    G = [np.ones((len(g["R"][d]), 1), np.float32) for d in range(3)]
    out = halo.backward_flat(L, G, g["R"], part, loc)
    assert [o[:, 0].tolist() for o in out] == g["all_ones_backward_owner_rows"]


def test_h2_flat_order_is_observable():
    """(L + G_1) + G_2 with L = 1, G = 2^-24: sequential fp32 gives 1.0 (ties-to-even twice);
    the other association L + (G_1 + G_2) would give 1 + 2^-23.  Pins the R6 order for v0."""
    g, part = _h2()
    loc, n_local = halo.local_rows(part, 3)
    L = [np.zeros((n_local[d], 1), np.float32) for d in range(3)]
    L[0][0, 0] = 1.0
    G = [np.zeros((len(g["R"][d]), 1), np.float32) for d in range(3)]
    G[1][0, 0] = 2.0 ** -24       # R_1[0] = v0
    G[2][0, 0] = 2.0 ** -24       # R_2[0] = v0
    out = halo.backward_flat(L, G, g["R"], part, loc)
    assert out[0][0, 0] == np.float32(1.0)
    assert np.float32(1.0) + (np.float32(2.0 ** -24) + np.float32(2.0 ** -24)) != np.float32(1.0)


def _tiny(n=300, e=2500, m=3, seed=5):
    src, dst = synth.rmat_edges(n, e, seed)
    part = synth.partition(n, m, seed + 1)
    edges = list(zip(src.tolist(), dst.tolist()))
    R = halo.required_bruteforce(n, edges, part, m)
    return n, m, part, edges, R


def test_generator_required_lists_match_bruteforce():
    """The input helper (synth.required_lists) agrees with the §4.1 definition by loops."""
    n, m, part, edges, R = _tiny()
    src = np.array([a for a, _ in edges], np.int32)
    dst = np.array([b for _, b in edges], np.int32)
    ptr, ids = synth.required_lists(src, dst, part, m)
    for d in range(m):
        assert ids[ptr[d]:ptr[d + 1]].tolist() == sorted(R[d], key=lambda u: (part[u], u))


@pytest.mark.parametrize("m", [2, 3, 4])
def test_forward_and_backward_match_loops(m):
    n, m, part, edges, R = _tiny(m=m, seed=10 + m)
    loc, n_local = halo.local_rows(part, m)
    dim = 3
    local = [synth.fill_values(n_local[d], dim, seed=3, stream=50 + d) for d in range(m)]
    # shuffled halo order: the oracle must read R_d as given
    Rs = [list(np.random.RandomState(d).permutation(r)) for d, r in enumerate(R)]
    F = halo.forward(local, Rs, part, loc)
    Fl = halo.forward_loops(local, Rs, part, loc)
    for d in range(m):
        assert np.array_equal(F[d].view(np.uint32), Fl[d].view(np.uint32))
    G = [synth.fill_values(len(Rs[d]), dim, seed=4, stream=90 + d) for d in range(m)]
    L = [synth.fill_values(n_local[d], dim, seed=4, stream=70 + d) for d in range(m)]
    B = halo.backward_flat(L, G, Rs, part, loc)
    Bl = halo.backward_flat_loops(L, G, Rs, part, loc)
    for d in range(m):
        assert np.array_equal(B[d].view(np.uint32), Bl[d].view(np.uint32))


def test_backward_closed_form_fanout_from_edges():
    n, m, part, edges, R = _tiny(m=4, seed=21)
    loc, n_local = halo.local_rows(part, m)
    L = [np.zeros((n_local[d], 2), np.float32) for d in range(m)]
    G = [np.ones((len(R[d]), 2), np.float32) for d in range(m)]
    out = halo.backward_flat(L, G, R, part, loc)
    # |D_u| straight from the edge list: distinct foreign GPUs among u's out-neighbours
    fan = np.zeros(n, np.int64)
    for u in range(n):
        fan[u] = len({int(part[v]) for (a, v) in edges if a == u and part[v] != part[u]})
    for u in range(n):
        assert out[part[u]][loc[u], 0] == fan[u] and out[part[u]][loc[u], 1] == fan[u]


def test_fanout_is_edge_counted_requesters():
    """halo.fanout (|D_u|, which drives the GPU closed-form test) against |D_u| counted from the
    EDGE LIST by explicit loops (distinct foreign GPUs among u's out-neighbours, R3), and against
    the H2 literal (its all-ones backward owner rows are exactly the fan-outs)."""
    for m, seed in ((2, 61), (4, 62), (5, 63)):
        n, m, part, edges, R = _tiny(m=m, seed=seed)
        f = halo.fanout(R, n)
        for u in range(n):
            want = len({int(part[v]) for (a, v) in edges if a == u and part[v] != part[u]})
            assert f[u] == want, (m, u)
    g, part = _h2()
    loc, _ = halo.local_rows(part, 3)
    f = halo.fanout(g["R"], g["n"])
    for v in range(g["n"]):
        assert f[v] == g["all_ones_backward_owner_rows"][part[v]][loc[v]]


def test_backward_integer_inputs_any_order():
    n, m, part, edges, R = _tiny(m=4, seed=33)
    loc, n_local = halo.local_rows(part, m)
    dim = 5
    G = [synth.fill_values(len(R[d]), dim, seed=4, stream=d, mode="int") for d in range(m)]
    L = [synth.fill_values(n_local[d], dim, seed=4, stream=9 + d, mode="int") for d in range(m)]
    out = halo.backward_flat(L, G, R, part, loc)
    # float64 accumulation in DESCENDING contributor order (a different order): exact for ints
    acc = [L[d].astype(np.float64) for d in range(m)]
    for c in reversed(range(m)):
        for i, u in enumerate(R[c]):
            acc[part[u]][loc[u]] += G[c][i]
    for d in range(m):
        assert np.array_equal(out[d], acc[d].astype(np.float32))


def test_tree_order_equals_flat_for_direct_trees():
    n, m, part, edges, R = _tiny(m=3, seed=44)
    loc, n_local = halo.local_rows(part, m)
    G = [synth.fill_values(len(R[d]), 4, seed=4, stream=d) for d in range(m)]
    L = [synth.fill_values(n_local[d], 4, seed=4, stream=20 + d) for d in range(m)]
    direct = [(int(u), int(part[u]), d, 1) for d in range(m) for u in R[d]]
    T = halo.backward_tree(L, G, R, part, loc, np.array(direct))
    B = halo.backward_flat(L, G, R, part, loc)
    for d in range(m):
        assert np.array_equal(T[d].view(np.uint32), B[d].view(np.uint32))


def test_tree_order_relay_by_hand():
    """u owned by 0, D_u = {1, 2}, tree 0->3->1, 3->2 (3 a pure relay):
    out = L + ((G_1 + G_2))  with the relay starting from val(y1) = G_1 then + G_2."""
    part = np.array([0, 1, 2, 3], np.int32)       # vertex v owned by GPU v
    loc, n_local = halo.local_rows(part, 4)
    R = [[], [0], [0], []]
    L = [np.array([[1.0]], np.float32)] + [np.zeros((1, 1), np.float32)] * 3
    G = [np.zeros((0, 1), np.float32), np.array([[2.0 ** -24]], np.float32),
         np.array([[2.0 ** -24]], np.float32), np.zeros((0, 1), np.float32)]
    edges = np.array([(0, 0, 3, 1), (0, 3, 1, 2), (0, 3, 2, 2)])
    T = halo.backward_tree(L, G, R, part, loc, edges)
    assert T[0][0, 0] == np.float32(1.0) + np.float32(2.0 ** -23)   # relay summed first
    B = halo.backward_flat(L, G, R, part, loc)
    assert B[0][0, 0] == np.float32(1.0)                              # flat: ((1 + e) + e) = 1


def _complete_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n = 12
    part = np.array([v % world for v in range(n)], np.int32)
    loc, n_local = halo.local_rows(part, world)
    dim = 3
    local = [synth.fill_values(n_local[d], dim, seed=3, keys=np.nonzero(part == d)[0])
             for d in range(world)]
    # complete relation: every GPU requires every non-local vertex, ordered by (owner, id)
    R = [sorted([u for u in range(n) if part[u] != d], key=lambda u: (part[u], u))
         for d in range(world)]
    H = halo.forward(local, R, part, loc)
    bufs = [torch.zeros(n_local[d], dim) for d in range(world)]
    dist.all_gather(bufs, torch.from_numpy(local[rank]))
    want = np.concatenate([bufs[d].numpy() for d in range(world) if d != rank])
    ok_fwd = np.array_equal(H[rank].view(np.uint32), want.view(np.uint32))
    # backward: integer inputs; owner s receives sum over c != s of G_c rows for s's vertices
    G = [synth.fill_values(len(R[d]), dim, seed=4, stream=d, mode="int") for d in range(world)]
    L = [synth.fill_values(n_local[d], dim, seed=4, stream=40 + d, mode="int")
         for d in range(world)]
    out = halo.backward_flat(L, G, R, part, loc)
    # contribution tensor of this rank: its halo grads scattered back into owner blocks, plus L
    contrib = [torch.zeros(n_local[d], dim) for d in range(world)]
    contrib[rank] += torch.from_numpy(L[rank])
    for i, u in enumerate(R[rank]):
        contrib[part[u]][loc[u]] += torch.from_numpy(G[rank][i])
    full = torch.cat(contrib)
    dist.all_reduce(full)
    off = int(sum(n_local[:rank]))
    mine = full[off:off + n_local[rank]].numpy()
    ok_bwd = np.array_equal(out[rank], mine)
    q.put((rank, ok_fwd, ok_bwd))
    dist.destroy_process_group()


def test_complete_relation_is_allgather_and_allreduce():
    import socket
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    world = 2
    procs = [ctx.Process(target=_complete_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(ok_f and ok_b for (_r, ok_f, ok_b) in res), res
