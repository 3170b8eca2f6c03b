"""Per-launch timing distribution of a relay-plan forward (variance study), 1 GPU loopback."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
import paper_conf_eurosys_cai0wmcy21_b200 as D
name = sys.argv[1]
geo = int(sys.argv[2]) if len(sys.argv) > 2 else 0
cfg = synth.get_config(name)
g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
ctx = D.loopback(cfg.m, g.part, list(cfg.dims), device=0)
ctx.set_option("geometry", geo)
ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=synth.topology.by_name(cfg.topology, cfg.m))
ctx.register_workspace()
p = ctx.pitch(0)
emb = torch.randn(cfg.n, p, device="cuda")
ts = []
for i in range(30):
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(); ctx.forward(0, emb); b.record(); torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
ctx.check()
print(name, "geo", geo, "fwd ms: min %.3f med %.3f max %.3f" % (min(ts), np.median(ts), max(ts)), [round(t, 2) for t in ts[:12]])
