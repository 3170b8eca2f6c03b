"""The peer-to-peer baseline arm (bench_p2p.py) against the oracle (-m "not gpu").

PAPER.md §7.1: the baseline the paper compares against packs rows by send list,
sends them point to point and unpacks them.  Its pack / unpack index lists are derived from the
partition and the required lists; here every rank of a gloo job (world 2 and 3, CPU tensors) runs
the forward and the backward, and each rank's halo must equal oracle.halo.forward and its owner
rows oracle.halo.backward_flat bit for bit (the backward adds requesters in ascending id, the
fixed order of DESIGN.md R6)."""
import os
import socket

import numpy as np
import pytest

import synth
from oracle import halo


def _worker(rank, world, port, q, shuffled):
    try:
        import torch
        import torch.distributed as dist

        import bench_p2p
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        g = synth.make_graph(1500, 12000, world, graph_seed=90 + world, part_seed=91)
        if shuffled:
            g.req_ids = synth.graph.shuffle_lists(g.req_ptr, g.req_ids, 3)
        ex = bench_p2p.P2PExchange(g.part, g.req_ptr, g.req_ids, rank, world, "cpu")
        loc, n_local = halo.local_rows(g.part, world)
        R = [g.R(d) for d in range(world)]
        dim, pitch = 6, 8
        order = [np.nonzero(g.part == d)[0] for d in range(world)]
        local = [synth.fill_values(n_local[d], dim, pitch, keys=order[d], seed=3) for d in range(world)]
        H = torch.zeros(len(R[rank]), pitch)
        ex.forward(torch.from_numpy(local[rank]), H)
        want = halo.forward([x[:, :dim] for x in local], R, g.part, loc)[rank]
        ok_f = np.array_equal(H.numpy()[:, :dim].view(np.uint32), want.view(np.uint32))
        ptr = g.req_ptr
        Gall = synth.fill_values(int(ptr[-1]), dim, pitch, seed=4, stream=synth.values.STREAM_HGRAD)
        G = [Gall[ptr[d]:ptr[d + 1]] for d in range(world)]
        L = [synth.fill_values(n_local[d], dim, pitch, keys=order[d], seed=4, stream=7)
             for d in range(world)]
        eg = torch.from_numpy(L[rank].copy())
        ex.backward(torch.from_numpy(G[rank]), eg)
        Bf = halo.backward_flat([x[:, :dim] for x in L], [x[:, :dim] for x in G], R, g.part, loc)
        ok_b = np.array_equal(eg.numpy()[:, :dim].view(np.uint32), Bf[rank].view(np.uint32))
        dist.destroy_process_group()
        q.put((rank, ok_f, ok_b, ""))
    except Exception:
        import traceback
        q.put((rank, False, False, traceback.format_exc()))


@pytest.mark.parametrize("world,shuffled", [(2, False), (3, True)])
def test_p2p_baseline_matches_oracle(world, shuffled):
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, shuffled)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(f and b for (_r, f, b, _e) in res), res


def test_p2p_lists_are_the_direct_plan():
    """The send lists are exactly the direct plan's stage-1 tuples: the H2 worked example
    (tests/golden/h2_example.json, direct_tuples_src_dst_vertices)."""
    import json
    import bench_p2p
    with open(os.path.join(os.path.dirname(__file__), "golden", "h2_example.json")) as f:
        gd = json.load(f)
    part = np.array([v % 3 for v in range(gd["n"])], np.int32)
    ptr = np.concatenate([[0], np.cumsum([len(r) for r in gd["R"]])]).astype(np.int64)
    ids = np.concatenate([np.asarray(r, np.int64) for r in gd["R"]])
    loc, _ = halo.local_rows(part, 3)
    tuples = {(s, d): v for (s, d, v) in gd["direct_tuples_src_dst_vertices"]}
    for me in range(3):
        send, recv = bench_p2p.p2p_lists(part, ptr, ids, me, 3)
        for d in range(3):
            want = [loc[u] for u in tuples.get((me, d), [])]
            assert send[d].tolist() == want
        for s in range(3):
            want = [i for i, u in enumerate(gd["R"][me]) if part[u] == s and s != me]
            assert recv[s].tolist() == want
