"""Small executor cases for compute-sanitizer (memcheck / synccheck): bulk-copy executor with
dynamic claims, relay plans (fused + per-rank), multicast emulation, lsu gathers, register path;
each checked against the oracle so a silent corruption also shows."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth
from oracle import halo

CASES = [  # (ranks, topology, per-rank flags, dim, options)
    (4, None, 0, 24, {"small_launch_bytes": 0, "claim_batch": 2}),
    (8, "ring", 0, 24, {"small_launch_bytes": 0}),
    (8, "dgx1_like", 1, 24, {"small_launch_bytes": 0}),
    (4, None, 1, 24, {"small_launch_bytes": 0, "multicast": 1}),
    (8, None, 0, 24, {"small_launch_bytes": 0, "multicast": 1, "lsu_gather": 1}),
    (4, None, 0, 24, {"tma": 0, "multicast": 2}),
    (8, "ring", 0, 24, {"small_launch_bytes": 0, "direct_reduce": 0}),
    # rows of 1 KB: per-row bulk stores of relay stages, fan-out bulk stores, item orders
    (8, "ring", 0, 256, {"small_launch_bytes": 0}),
    (8, "dgx1_like", 1, 256, {"small_launch_bytes": 0, "relay_lead_kb": 1}),
    (8, None, 0, 256, {"small_launch_bytes": 0, "fanout": 1}),
    (8, None, 0, 256, {"small_launch_bytes": 0, "owner_major": 0}),
    (8, "ring", 0, 256, {"small_launch_bytes": 0, "leaf_split": 2, "owner_major": 2}),
]
bad = 0
for m, topo, flags, dim, opts in CASES:
    g = synth.make_graph(1500, 12000, m, graph_seed=m, part_seed=m + 1)
    ctx = D.loopback(m, g.part, [dim], device=0, flags=flags)
    for k, v in opts.items():
        ctx.set_option(k, v)
    ctx.build_plan(g.req_ptr, g.req_ids, seed=1,
                   topology=synth.topology.by_name(topo, m) if topo else None)
    ctx.register_workspace()
    order = np.argsort(g.part, kind="stable")
    loc, nl = halo.local_rows(g.part, m)
    ro = np.concatenate([[0], np.cumsum(nl)])
    R = [g.R(d) for d in range(m)]
    p = ctx.pitch(0)
    emb = synth.fill_values(g.n, dim, p, keys=order)
    H = ctx.forward(0, torch.from_numpy(emb).cuda())
    torch.cuda.synchronize()
    ctx.check()
    Hh = H.cpu().numpy()
    Ho = halo.forward([emb[ro[d]:ro[d + 1], :dim] for d in range(m)], R, g.part, loc)
    ok = all(np.array_equal(Hh[g.req_ptr[d]:g.req_ptr[d + 1], :dim].view(np.uint32),
                            Ho[d].view(np.uint32)) for d in range(m))
    S = int(g.req_ptr[-1])
    G = synth.fill_values(S, dim, p, seed=4)
    L = synth.fill_values(g.n, dim, p, keys=order, seed=5)
    eg = torch.from_numpy(L.copy()).cuda()
    ctx.backward(0, torch.from_numpy(G).cuda(), eg)
    torch.cuda.synchronize()
    ctx.check()
    Bt = halo.backward_tree([L[ro[d]:ro[d + 1], :dim] for d in range(m)],
                            [G[g.req_ptr[d]:g.req_ptr[d + 1], :dim] for d in range(m)], R, g.part,
                            loc, ctx.plan_export())
    out = eg.cpu().numpy()
    okb = all(np.array_equal(out[ro[d]:ro[d + 1], :dim].view(np.uint32), Bt[d].view(np.uint32))
              for d in range(m))
    print(m, topo, flags, opts, "forward", ok, "backward", okb, flush=True)
    bad += (not ok) + (not okb)
    ctx.destroy()
sys.exit(1 if bad else 0)
