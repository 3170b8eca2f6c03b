"""Occupancy timeline of a relay-plan forward (1 GPU loopback, option "trace").

usage: python tools/relay_timeline.py CONFIG [bin_us] [key=value options...]
Per time bin (us from the launch's first item): how many items were waiting for their sources
(t_start..t_ready: stage chaining) and how many were moving rows (t_ready..t_done), split by
stage, so the cost of each stage boundary can be read off: bins where few items move rows.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth

name = sys.argv[1]
binus = float(sys.argv[2]) if len(sys.argv) > 2 else 10.0
opts = dict(kv.split("=") for kv in sys.argv[3:])
cfg = synth.get_config(name)
g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
topo = synth.topology.by_name(cfg.topology, cfg.m) if cfg.topology != "uniform_nvswitch" else None
ctx = D.loopback(cfg.m, g.part, list(cfg.dims), device=0)
for k, v in opts.items():
    ctx.set_option(k, int(v))
ctx.set_option("trace", 1)
ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo)
ctx.register_workspace()
p = ctx.pitch(0)
emb = torch.randn(cfg.n, p, device="cuda")
ts = []
for _ in range(5):
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    ctx.forward(0, emb)
    b.record()
    torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
ctx.check()
tr = ctx.trace(0, 0)
t0 = int(tr["t_start"].min())
s = (tr["t_start"].astype(np.int64) - t0) / 1e3
r = (tr["t_ready"].astype(np.int64) - t0) / 1e3
d = (tr["t_done"].astype(np.int64) - t0) / 1e3
st = tr["stage"]
end = float(d.max())
print("%s fwd %s: launch %.3f ms (median of 5), %d items, last done %.1f us" %
      (name, opts, float(np.median(ts)), len(st), end))
stages = sorted(np.unique(st).tolist())
print("  bin(us)  waiting  " + "  ".join("busy_s%d" % k for k in stages) + "  busy_all")
nb = int(np.ceil(end / binus))
low = 0.0
for i in range(nb):
    a, b = i * binus, (i + 1) * binus
    mid = (a + b) / 2
    waiting = int(((s <= mid) & (r > mid)).sum())
    busy = [int(((st == k) & (r <= mid) & (d > mid)).sum()) for k in stages]
    tot = sum(busy)
    print("  %6.0f  %7d  " % (a, waiting) + "  ".join("%7d" % x for x in busy) + "  %7d" % tot)
print("  per stage: items, start min/max, ready min/med/max, done min/med/max, busy (ready->done) "
      "p50/p90/max, wait (start->ready) p50/p90/max  [us]")
bl = tr["block"]
for k, b_ in sorted(set(zip(st.tolist(), bl.tolist()))):
    m = (st == k) & (bl == b_)
    busy, wait = d[m] - r[m], r[m] - s[m]
    q = lambda x, p: float(np.percentile(x, p))
    print("    s%d b%d %6d  start %6.1f/%6.1f  ready %6.1f/%6.1f/%6.1f  done %6.1f/%6.1f/%6.1f  "
          "busy %5.1f/%5.1f/%5.1f  wait %5.1f/%5.1f/%5.1f" %
          (k, b_, m.sum(), s[m].min(), s[m].max(), r[m].min(), q(r[m], 50), r[m].max(), d[m].min(),
           q(d[m], 50), d[m].max(), q(busy, 50), q(busy, 90), busy.max(), q(wait, 50), q(wait, 90),
           wait.max()))
