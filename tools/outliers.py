"""Per-launch time distribution (min / median / p99 / max over many launches, each between its own
events, launched back to back) — looks for rare slow launches.
usage: python tools/outliers.py CONFIG [reps] [key=value options...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth

name = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 200
opts = dict(kv.split("=") for kv in sys.argv[3:])
cfg = synth.get_config(name)
g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
topo = synth.topology.by_name(cfg.topology, cfg.m) if cfg.topology != "uniform_nvswitch" else None
ctx = D.loopback(cfg.m, g.part, list(cfg.dims), device=0)
for k, v in opts.items():
    ctx.set_option(k, int(v))
ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo)
ctx.register_workspace()
S = int(g.req_ptr[-1])
emb = {l: torch.randn(cfg.n, ctx.pitch(l), device="cuda") for l in range(len(cfg.dims))}
hg = {l: torch.randn(S, ctx.pitch(l), device="cuda") for l in cfg.backward_layers}
eg = {l: torch.zeros(cfg.n, ctx.pitch(l), device="cuda") for l in cfg.backward_layers}
calls = [("fwd%d_d%d" % (l, cfg.dims[l]), (lambda l=l: ctx.forward(l, emb[l])))
         for l in range(len(cfg.dims))]
calls += [("bwd%d_d%d" % (l, cfg.dims[l]), (lambda l=l: ctx.backward(l, hg[l], eg[l])))
          for l in cfg.backward_layers]
for _ in range(5):
    for _, fn in calls:
        fn()
torch.cuda.synchronize()
ev = [[(torch.cuda.Event(True), torch.cuda.Event(True)) for _ in calls] for _ in range(reps)]
for r in range(reps):
    for i, (_, fn) in enumerate(calls):
        ev[r][i][0].record()
        fn()
        ev[r][i][1].record()
torch.cuda.synchronize()
ctx.check()
for i, (n, _) in enumerate(calls):
    t = np.array([ev[r][i][0].elapsed_time(ev[r][i][1]) for r in range(reps)])
    print("%s %s %s: min %.4f med %.4f p99 %.4f max %.4f ms, launches > 1.2x median: %d" %
          (name, opts, n, t.min(), np.median(t), np.percentile(t, 99), t.max(),
           int((t > 1.2 * np.median(t)).sum())))
