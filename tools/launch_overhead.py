"""Fixed per-launch cost of the executor (1 GPU loopback): one launch between two CUDA events
(as bench.py times it) vs N launches back to back between one pair, vs an empty torch kernel.

usage: python tools/launch_overhead.py CONFIG [N]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth

name = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 20
cfg = synth.get_config(name)
g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
topo = synth.topology.by_name(cfg.topology, cfg.m) if cfg.topology != "uniform_nvswitch" else None
ctx = D.loopback(cfg.m, g.part, list(cfg.dims), device=0)
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


def timed(fn, reps):
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize()
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


x = torch.zeros(1, device="cuda")
for _ in range(3):
    timed(lambda: x.add_(1), 1)
empty = np.median([timed(lambda: x.add_(1), 1) for _ in range(20)])
print("%s: empty torch kernel between events %.4f ms" % (name, empty))
for n, fn in calls:
    for _ in range(3):
        fn()
    one = np.median([timed(fn, 1) for _ in range(20)])
    many = np.median([timed(fn, N) for _ in range(5)])
    print("  %-10s one launch %.4f ms   %d back to back %.4f ms each   difference %.1f us" %
          (n, one, N, many, (one - many) * 1e3))

# the bench's step pattern: every launch bracketed by its own event pair, launches back to back
evs = [[torch.cuda.Event(True), torch.cuda.Event(True)] for _ in range(N * len(calls))]
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
torch.cuda.synchronize()
e0.record()
k = 0
for _ in range(N):
    for n, fn in calls:
        evs[k][0].record()
        fn()
        evs[k][1].record()
        k += 1
e1.record()
torch.cuda.synchronize()
with_ev = e0.elapsed_time(e1) / N
per = {n: np.mean([evs[j * len(calls) + i][0].elapsed_time(evs[j * len(calls) + i][1])
                   for j in range(N)]) for i, (n, _) in enumerate(calls)}
torch.cuda.synchronize()
e0.record()
for _ in range(N):
    for n, fn in calls:
        fn()
e1.record()
torch.cuda.synchronize()
no_ev = e0.elapsed_time(e1) / N
print("  step of %d launches: %.4f ms with per-launch events (%s), %.4f ms without" %
      (len(calls), with_ev, ", ".join("%s %.4f" % kv for kv in per.items()), no_ev))
