"""Multi-process test of the real multi-GPU path on ONE device (-m gpu).

One process per rank (torch.multiprocessing, gloo process group for setup), each with its own
context built by `setup_distributed`: required lists all-gathered, identical plans, workspaces
allocated by torch and mapped into every peer with CUDA IPC, then forward and backward through the
per-rank programs (ready handshake, done counters, completion waits) with peer-pointer stores.
All ranks share cuda:0 here (this run has one GPU); the kernels time-slice, which exercises the
flag protocol under arbitrary interleavings.  Results are checked against values recomputed from
the hash definition (forward bit-exact, backward in the fixed flat order, bit-exact).
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


def _worker(rank, world, port, q, n, e, dims, topo_name):
    try:
        import torch
        import torch.distributed as dist

        import paper_conf_eurosys_cai0wmcy21_b200 as D
        import synth
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        g = synth.make_graph(n, e, world, graph_seed=77, part_seed=78)
        topo = synth.topology.by_name(topo_name, world) if topo_name else None
        ctx = D.setup_distributed(g.part, dims, g.R(rank), topology=topo, seed=5, device=0,
                                  options={"small_launch_bytes": 0})  # the bulk-copy path
        ctx.set_option("timeout_ms", 120000)
        mine = np.nonzero(g.part == rank)[0]           # my global ids, loc order
        ok = True
        msgs = []
        for layer, dim in enumerate(dims):
            pitch = ctx.pitch(layer)
            emb = synth.fill_values(len(mine), dim, pitch, keys=mine, seed=3,
                                    stream=synth.values.STREAM_EMB + layer)
            for rep in range(2):
                H = ctx.forward(layer, torch.from_numpy(emb).cuda())
                torch.cuda.synchronize()
                ctx.check()
                Rm = g.R(rank)
                want = synth.fill_values_numpy(Rm, np.arange(dim), seed=3,
                                               stream=synth.values.STREAM_EMB + layer)
                got = H.cpu().numpy()[:, :dim]
                if not np.array_equal(got.view(np.uint32), want.view(np.uint32)):
                    ok = False
                    msgs.append("forward layer %d rep %d" % (layer, rep))
            # backward: my halo gradients are hash rows keyed by the global halo row index
            base = int(g.req_ptr[rank])
            G = synth.fill_values(len(g.R(rank)), dim, pitch,
                                  keys=np.arange(base, base + len(g.R(rank))), seed=4,
                                  stream=synth.values.STREAM_HGRAD + layer)
            L = synth.fill_values(len(mine), dim, pitch, keys=mine, seed=4,
                                  stream=synth.values.STREAM_EGRAD + layer)
            eg = torch.from_numpy(L.copy()).cuda()
            ctx.backward(layer, torch.from_numpy(G).cuda(), eg)
            torch.cuda.synchronize()
            ctx.check()
            out = eg.cpu().numpy()[:, :dim]
            # expected: L + contributions of requesting GPUs in ascending id (flat order)
            acc = L[:, :dim].copy()
            loc = {int(u): i for i, u in enumerate(mine)}
            for d in range(world):
                Rd = g.R(d)
                sel = np.nonzero(g.part[Rd] == rank)[0]
                if sel.size == 0:
                    continue
                rows = np.array([loc[int(u)] for u in Rd[sel]])
                contrib = synth.fill_values_numpy(int(g.req_ptr[d]) + sel, np.arange(dim), seed=4,
                                                  stream=synth.values.STREAM_HGRAD + layer)
                acc[rows] = (acc[rows] + contrib).astype(np.float32)
            if ctx.plan_info()["n_stages"] <= 1:
                same = np.array_equal(out.view(np.uint32), acc.view(np.uint32))
            else:
                same = np.allclose(out, acc, rtol=0, atol=2e-5)
            if not same:
                ok = False
                msgs.append("backward layer %d" % layer)
        launches = ctx.launch_count()
        ctx.destroy()
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, ok, msgs, launches))
    except Exception as ex:  # report instead of hanging the parent
        import traceback
        q.put((rank, False, [traceback.format_exc()], 0))


def _run(world, n, e, dims, topo_name=None, timeout=600):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, n, e, dims, topo_name))
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
