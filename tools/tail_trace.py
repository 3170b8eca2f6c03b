"""Per-SM timeline of one loopback launch (option "trace"): when each SM started its first item
and finished its last, and how much of the launch it was busy — ramp and tail of a persistent
launch.  usage: python tools/tail_trace.py CONFIG [dir] [key=value ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth

name = sys.argv[1]
direction = int(sys.argv[2]) if len(sys.argv) > 2 else 0
opts = dict(kv.split("=") for kv in sys.argv[3:])
cfg = synth.get_config(name)
g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
topo = synth.topology.by_name(cfg.topology, cfg.m) if cfg.topology != "uniform_nvswitch" else None
ctx = D.loopback(cfg.m, g.part, list(cfg.dims), device=0)
ctx.set_option("trace", 1)
for k, v in opts.items():
    ctx.set_option(k, int(v))
ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo)
ctx.register_workspace()
layer = len(cfg.dims) - 1
p = ctx.pitch(layer)
S = int(g.req_ptr[-1])
emb = torch.randn(cfg.n, p, device="cuda")
hg = torch.randn(S, p, device="cuda")
eg = torch.zeros(cfg.n, p, device="cuda")
ts = []
for _ in range(5):
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    if direction == 0:
        ctx.forward(layer, emb)
    else:
        ctx.backward(layer, hg, eg)
    b.record()
    torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
ctx.check()
tr = ctx.trace(layer, direction)
data = tr["op"] <= 1
t0 = int(tr["t_start"][data].min())
T = int(tr["t_done"][data].max()) - t0
sm = tr["sm"][data]
first = np.array([tr["t_start"][data][sm == s].min() - t0 for s in np.unique(sm)]) / 1e3
last = np.array([tr["t_done"][data][sm == s].max() - t0 for s in np.unique(sm)]) / 1e3
n_items = np.array([(sm == s).sum() for s in np.unique(sm)])
print("%s dir %d layer %d opts %s: launch %.3f ms (median of 5), traced span %.1f us, %d items, "
      "%d SMs" % (name, direction, layer, opts, float(np.median(ts)), T / 1e3, data.sum(),
                  len(np.unique(sm))))
for q in (0, 10, 50, 90, 100):
    print("  p%-3d first start %7.1f us   last done %7.1f us   items/SM %d" % (
        q, np.percentile(first, q), np.percentile(last, q), np.percentile(n_items, q)))
busy = (tr["t_done"][data] - tr["t_ready"][data]) / 1e3
print("  item ready->done us: median %.1f p90 %.1f max %.1f" % (
    np.median(busy), np.percentile(busy, 90), busy.max()))
ctx.destroy()
