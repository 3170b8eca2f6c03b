"""Multi-process host logic of the N>1 path on CPU (gloo, world size 2 and 4; -m "not gpu").

Each rank knows only its own required list; `build_plan_distributed` all-gathers them and every
rank plans independently.  Checks: identical plans on every rank (deterministic, no
master), the plan equals the oracle's reference SPST, and each rank's per-rank programs see the
same halo sizes.  Device steps (workspace, IPC, dispatch) are covered by -m gpu tests.
"""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.usefixtures("built")


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, topo_name):
    try:
        import torch.distributed as dist

        import paper_conf_eurosys_cai0wmcy21_b200 as D
        import synth
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        g = synth.make_graph(800, 5000, world, graph_seed=31, part_seed=32)
        topo = synth.topology.by_name(topo_name, world) if topo_name else None
        ctx = D.init(g.part, [8], rank, world, -1)          # host-only context
        ptr, ids = D.dgcl.build_plan_distributed(ctx, g.R(rank), topology=topo, seed=9)
        E = ctx.plan_export()
        info = ctx.plan_info()
        plans = [None] * world
        dist.all_gather_object(plans, (E.tolist(), info["model_cost_ticks"]))
        same = all(p == plans[0] for p in plans)
        ok_lists = np.array_equal(ptr, g.req_ptr) and np.array_equal(ids, g.req_ids)
        dist.destroy_process_group()
        q.put((rank, same and ok_lists, E.tolist(), info["model_cost_ticks"]))
    except Exception:
        import traceback
        q.put((rank, False, traceback.format_exc(), 0))


@pytest.mark.parametrize("world,topo_name", [(2, None), (4, "ring")])
def test_identical_plans_over_gloo(world, topo_name):
    import torch.multiprocessing as mp

    import synth
    from oracle import spst
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, topo_name))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in range(world)]
    for p in procs:
        p.join(timeout=30)
    assert all(r[1] for r in res), res
    g = synth.make_graph(800, 5000, world, graph_seed=31, part_seed=32)
    topo = synth.topology.by_name(topo_name, world) if topo_name else synth.uniform_nvswitch(world)
    owner, Dd = spst.relation_from_lists([g.R(d) for d in range(world)], g.part)
    edges, cost = spst.spst(topo, owner, Dd, seed=9)
    assert [tuple(e) for e in res[0][2]] == [tuple(e) for e in edges]
    assert res[0][3] == cost
