"""Stage timeline of a relay-plan launch (1 GPU loopback, option "trace").

usage: python tools/relay_trace.py CONFIG [geometry]
Prints, per (direction, stage): items, first start, first ready, last done (us from the launch's
first item) and the summed item busy time, so the serial stage chain can be read off directly.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth

name = sys.argv[1]
geo = int(sys.argv[2]) if len(sys.argv) > 2 else 0
cfg = synth.get_config(name)
g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
topo = synth.topology.by_name(cfg.topology, cfg.m) if cfg.topology != "uniform_nvswitch" else None
ctx = D.loopback(cfg.m, g.part, list(cfg.dims), device=0)
ctx.set_option("geometry", geo)
ctx.set_option("trace", 1)
ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo)
ctx.register_workspace()
p = ctx.pitch(0)
S = int(g.req_ptr[-1])
emb = torch.randn(cfg.n, p, device="cuda")
hg = torch.randn(S, p, device="cuda")
eg = torch.zeros(cfg.n, p, device="cuda")
for direction in (0, 1):
    ts = []
    for _ in range(5):
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record()
        if direction == 0:
            ctx.forward(0, emb)
        else:
            ctx.backward(0, hg, eg)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ctx.check()
    tr = ctx.trace(0, direction)
    t0 = int(tr["t_start"].min())
    print("%s %s geo %d: launch %.3f ms (median of 5), %d items, %d SMs" %
          (name, "fwd" if direction == 0 else "bwd", geo, float(np.median(ts)), len(tr["tag"]),
           len(np.unique(tr["sm"]))))
    for st, op in sorted(set(zip(tr["stage"].tolist(), tr["op"].tolist()))):
        m = (tr["stage"] == st) & (tr["op"] == op)
        busy = (tr["t_done"][m] - tr["t_ready"][m]).astype(np.int64)
        print("    stage %d op %d: %5d items, ready->done busy sum %.0f us, med %.1f us" %
              (st, op, m.sum(), busy.sum() / 1e3, np.median(busy) / 1e3))
    for st in np.unique(tr["stage"]):
        m = tr["stage"] == st
        busy = (tr["t_done"][m] - tr["t_start"][m]).astype(np.int64)
        wait = (tr["t_ready"][m] - tr["t_start"][m]).astype(np.int64)
        print("  stage %d ops %s: %5d items  start %7.1f  ready %7.1f  done %7.1f us  "
              "item busy med %.1f us  wait sum %.0f us" %
              (st, sorted(set(tr["op"][m].tolist())), m.sum(),
               (tr["t_start"][m].min() - t0) / 1e3, (tr["t_ready"][m].min() - t0) / 1e3,
               (tr["t_done"][m].max() - t0) / 1e3, np.median(busy) / 1e3, wait.sum() / 1e3))
ctx.destroy()
