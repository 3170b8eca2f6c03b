"""A/B of runtime executor options on one loopback context (one GPU): the plan is built once,
the option sets (dgcl_set_option keys that may change at any time: l2_policy, sys_scope,
sm_budget, ...) are interleaved over several rounds, and each launch's median time is reported.
usage: python tools/ab_rt.py CONFIG "k=v,k=v" "k=v" ...   (build-time options: --build k=v,...)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth

args = sys.argv[1:]
build = {}
if "--build" in args:
    i = args.index("--build")
    build = dict(kv.split("=") for kv in args[i + 1].split(","))
    del args[i:i + 2]
name, sets = args[0], [dict(kv.split("=") for kv in s.split(",") if kv) for s in args[1:]]
cfg = synth.get_config(name)
g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
topo = synth.topology.by_name(cfg.topology, cfg.m) if cfg.topology != "uniform_nvswitch" else None
ctx = D.loopback(cfg.m, g.part, list(cfg.dims), device=0)
for k, v in build.items():
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
res = {i: {n: [] for n, _ in calls} for i in range(len(sets))}
for rnd in range(4):
    for i, st in enumerate(sets):
        for k, v in st.items():
            ctx.set_option(k, int(v))
        for n, fn in calls:
            for _ in range(2):
                fn()
            for _ in range(8):
                a, b = torch.cuda.Event(True), torch.cuda.Event(True)
                a.record()
                fn()
                b.record()
                torch.cuda.synchronize()
                res[i][n].append(a.elapsed_time(b))
        ctx.check()
out = {"config": name, "build": build,
       "sets": [{"opts": st, "ms": {n: round(float(np.median(v)), 4) for n, v in res[i].items()}}
                for i, st in enumerate(sets)]}
print(json.dumps(out))
ctx.destroy()
