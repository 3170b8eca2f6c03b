"""Run one config's launch (layer, direction) `reps` times — a target for ncu.
usage: python tools/one_launch.py CONFIG LAYER DIR [reps] [key=value options...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth

name, layer, direction = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
opts = dict(kv.split("=") for kv in sys.argv[5:])
cfg = synth.get_config(name)
g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
topo = synth.topology.by_name(cfg.topology, cfg.m) if cfg.topology != "uniform_nvswitch" else None
ctx = D.loopback(cfg.m, g.part, list(cfg.dims), device=0)
for k, v in opts.items():
    ctx.set_option(k, int(v))
ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo)
ctx.register_workspace()
S = int(g.req_ptr[-1])
p = ctx.pitch(layer)
if direction == 0:
    emb = torch.randn(cfg.n, p, device="cuda")
    fn = lambda: ctx.forward(layer, emb)
else:
    hg = torch.randn(S, p, device="cuda")
    eg = torch.zeros(cfg.n, p, device="cuda")
    fn = lambda: ctx.backward(layer, hg, eg)
for _ in range(reps):
    fn()
torch.cuda.synchronize()
ctx.check()
print("ok", name, layer, direction, reps)
