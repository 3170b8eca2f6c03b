"""Multi-process test of the real multi-GPU path on ONE device (-m gpu).

One process per rank (torch.multiprocessing, gloo process group for setup), each with its own
context built by `setup_distributed`: required lists all-gathered, identical plans, workspaces
allocated by torch and mapped into every peer with CUDA IPC, then forward and backward through the
per-rank programs (ready handshake, done counters, completion waits) with peer-pointer stores.
All ranks share cuda:0 here (this run has one GPU); the kernels time-slice, which exercises the
flag protocol under arbitrary interleavings.  Every rank checks its rows against oracle/halo on
the hash-defined inputs of all ranks: forward bit-exact; backward bit-exact against the tree-order
oracle (the plan's fixed order) and against the flat oracle on single-stage plans, within the R6
bound (1e-6 * sum|terms|) on relay plans; a repeated backward gives identical bits.
"""
import os
import socket

import numpy as np
import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.usefixtures("built")]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, n, e, dims, topo_name, cfg_name=None, opts=None):
    try:
        import torch
        import torch.distributed as dist

        import paper_conf_eurosys_cai0wmcy21_b200 as D
        import synth
        from oracle import halo
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        if cfg_name:
            cfg = synth.get_config(cfg_name)
            g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed)
        else:
            g = synth.make_graph(n, e, world, graph_seed=77, part_seed=78)
        topo = synth.topology.by_name(topo_name, world) if topo_name else None
        ctx = D.setup_distributed(g.part, dims, g.R(rank), topology=topo, seed=5, device=0,
                                  options=dict({"small_launch_bytes": 0},  # the bulk-copy path
                                               **(opts or {})))
        ctx.set_option("timeout_ms", 120000)
        E = ctx.plan_export()
        multi_stage = ctx.plan_info()["n_stages"] > 1
        loc, n_local = halo.local_rows(g.part, world)
        R = [g.R(d) for d in range(world)]
        ptr = g.req_ptr
        order = [np.nonzero(g.part == d)[0] for d in range(world)]   # each rank's ids, loc order
        eq = lambda a, b: np.array_equal(np.ascontiguousarray(a).view(np.uint32),
                                         np.ascontiguousarray(b).view(np.uint32))
        ok = True
        msgs = []
        for layer, dim in enumerate(dims):
            pitch = ctx.pitch(layer)
            # every rank's inputs from the hash definition (the oracle needs all of them)
            embs = [synth.fill_values(len(order[d]), dim, pitch, keys=order[d], seed=3,
                                      stream=synth.values.STREAM_EMB + layer) for d in range(world)]
            Ho = halo.forward([x[:, :dim] for x in embs], R, g.part, loc)[rank]
            for rep in range(2):
                H = ctx.forward(layer, torch.from_numpy(embs[rank]).cuda())
                torch.cuda.synchronize()
                ctx.check()
                if not eq(H.cpu().numpy()[:, :dim], Ho):
                    ok = False
                    msgs.append("forward layer %d rep %d" % (layer, rep))
            # backward: halo gradients keyed by the global halo row index
            Gs = [synth.fill_values(len(R[d]), dim, pitch, keys=np.arange(ptr[d], ptr[d + 1]),
                                    seed=4, stream=synth.values.STREAM_HGRAD + layer)
                  for d in range(world)]
            Ls = [synth.fill_values(len(order[d]), dim, pitch, keys=order[d], seed=4,
                                    stream=synth.values.STREAM_EGRAD + layer) for d in range(world)]
            outs = []
            for rep in range(2):
                eg = torch.from_numpy(Ls[rank].copy()).cuda()
                ctx.backward(layer, torch.from_numpy(Gs[rank]).cuda(), eg)
                torch.cuda.synchronize()
                ctx.check()
                outs.append(eg.cpu().numpy()[:, :dim])
            out = outs[0]
            if not eq(outs[0], outs[1]):
                ok = False
                msgs.append("backward not reproducible layer %d" % layer)
            Lc, Gc = [x[:, :dim] for x in Ls], [x[:, :dim] for x in Gs]
            Bt = halo.backward_tree(Lc, Gc, R, g.part, loc, E)[rank]
            if not eq(out, Bt):
                ok = False
                msgs.append("backward (tree order) layer %d" % layer)
            Bf = halo.backward_flat(Lc, Gc, R, g.part, loc)[rank]
            if not multi_stage:
                same = eq(out, Bf)
            else:   # R6: |gpu - flat| <= 1e-6 * sum|terms|
                bound = halo.backward_flat([np.abs(x) for x in Lc], [np.abs(x) for x in Gc], R,
                                           g.part, loc)[rank]
                same = bool(np.all(np.abs(out.astype(np.float64) - Bf) <= 1e-6 * bound))
            if not same:
                ok = False
                msgs.append("backward (flat order) layer %d" % layer)
        launches = ctx.launch_count()
        ctx.destroy()
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, ok, msgs, launches))
    except Exception as ex:  # report instead of hanging the parent
        import traceback
        q.put((rank, False, [traceback.format_exc()], 0))


def _run(world, n, e, dims, topo_name=None, timeout=600, cfg_name=None, opts=None):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, n, e, dims, topo_name, cfg_name,
                                                     opts))
             for r in range(world)]
    for p in procs:
        p.start()
    res = []
    try:
        for _ in range(world):
            res.append(q.get(timeout=timeout))
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    bad = [r for r in res if not r[1]]
    assert not bad, bad
    return res


def test_two_processes_ipc_uniform():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    _run(2, 3000, 20000, [32, 5])


def test_four_processes_ipc_relay_ring():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    _run(4, 2000, 12000, [16], topo_name="ring")


def test_tiny_config_two_processes_ipc():
    """BASELINE configs[0] (10k vertices, 100k edges, 2-way, dim 16) over the real multi-process
    path: two ranks, IPC-mapped workspaces, per-rank programs, every row against the oracle."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    _run(2, 0, 0, [16], cfg_name="tiny")


def test_four_processes_ipc_relay_ring_two_layers():
    """4 ranks, relay plan from a ring model, two layers (one with a ragged dim)."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    _run(4, 3000, 20000, [24, 7], topo_name="ring")


@pytest.mark.parametrize("world,topo", [(2, None), (4, "ring")])
def test_bulk_store_peer_ipc(world, topo):
    """Option bulk_store_peer: TMA bulk stores of packed contiguous rows into IPC-mapped peer
    memory (the multi-GPU form of the loopback's bulk stores), on the same-device IPC path."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    _run(world, 3000, 20000, [64, 256], topo_name=topo, opts={"bulk_store_peer": 1})
