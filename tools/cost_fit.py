#!/usr/bin/env python3
"""Cost model against measured exchange time — the analogue of the paper's Fig. 10 (P:2358-2366:
"we plot the estimated cost and actual communication time of one graphAllgather operation").
Host only: the measured times come from a bench JSONL (default profiles/r1_bench_all_configs.jsonl,
one B200, 1-GPU loopback); the estimates are the §5.1 cost model t(S) recomputed by
the library for the plan that was actually executed.

On one GPU every virtual link i->j is the same physical resource, HBM: a delivered row is read once
and written once.  So the "loopback topology" has ONE hop shared by all ordered pairs, costing
w = round(1e5 / (HBM_GBps / 2)) ticks per row (R7 tick convention; half the copy
bandwidth because the copy figure counts read + write).  Under the §5.1 rules t(S) is then the sum
over stages of (rows in the stage) x w — the stage-serialised byte count, which is what the model
predicts for this hardware.  Each plan is the SPST plan of the config's own topology (uniform,
dgx1_like, ring), exported and re-costed through dgcl_build_plan_from_trees (no re-planning).

Reported per forward launch: model ms, measured ms, measured / model, and the least-squares fit
measured = a * model + b over all points (slope, intercept, R^2) — the paper's claim is a linear
relation (Fig. 10), not equality.

usage: python tools/cost_fit.py [bench.jsonl] [--out profiles/r1_cost_fit.txt]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth
from synth.topology import Topology


def loopback_topology(m, hbm_gbs):
    t = Topology("loopback_hbm", m, [hbm_gbs / 2.0], ["hbm"])
    for i in range(m):
        for j in range(m):
            if i != j:
                t.links[(i, j)] = [0]
    return t


def ticks_to_ms(ticks, row_bytes):
    return ticks * row_bytes / 1e14 * 1e3  # one tick = row_bytes / 1e14 s (see tools/plan_model.py)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("bench", nargs="?", default=os.path.join(ROOT, "profiles/r1_bench_all_configs.jsonl"))
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    hbm = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    pts, lines = [], []
    graphs = {}
    for line in open(args.bench):
        d = json.loads(line)
        c = d["config"]
        if c["config"] == "tiny":  # latency-bound (12 us launches): off the bandwidth line
            continue
        cfg = synth.get_config(c["config"])
        key = (cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed)
        if key not in graphs:
            graphs = {key: synth.make_graph(*key, keep_edges=False)}
        g = graphs[key]
        topo = synth.topology.by_name(c["topology"], cfg.m)
        ctx = D.loopback(cfg.m, g.part, [cfg.dims[-1]], device=-1)
        ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo)
        E = ctx.plan_export()
        stages = ctx.plan_info()["n_stages"]
        ctx.destroy()
        ctx = D.loopback(cfg.m, g.part, [cfg.dims[-1]], device=-1)
        ctx.build_plan(g.req_ptr, g.req_ids, topology=loopback_topology(cfg.m, hbm), trees=E)
        ticks = ctx.plan_info()["model_cost_ticks"]
        ctx.destroy()
        for k, ms in d["ms_per_layer"].items():
            if not k.startswith("fwd"):
                continue
            dim = int(k.split("_d")[1])
            est = ticks_to_ms(ticks, 4 * dim)
            pts.append((est, ms, stages))
            lines.append("%-13s %-16s %-10s stages %d  tree edges %9d  model %.3f ms  measured %.3f ms"
                         "  ratio %.2f" % (c["config"], c["topology"], k, stages, len(E), est, ms,
                                           ms / est))
            print(lines[-1], flush=True)
    x = np.array([p[0] for p in pts])
    y = np.array([p[1] for p in pts])
    a, b = np.polyfit(x, y, 1)
    r2 = 1 - np.sum((y - (a * x + b)) ** 2) / np.sum((y - y.mean()) ** 2)
    lines.append("fit over %d forward launches: measured = %.3f * model %+.4f ms, R^2 = %.3f "
                 "(HBM %.1f GB/s, MEASURED_PEAKS.json)" % (len(pts), a, b, r2, hbm))
    print(lines[-1])
    # the §5.1 model has no per-stage term; in loopback a stage boundary is a device-wide drain
    st = np.array([p[2] for p in pts], np.float64)
    (a2, c2), *_ = np.linalg.lstsq(np.stack([x, st], 1), y, rcond=None)
    r22 = 1 - np.sum((y - (a2 * x + c2 * st)) ** 2) / np.sum((y - y.mean()) ** 2)
    lines.append("with a per-stage term: measured = %.3f * model + %.4f ms * stages, R^2 = %.3f"
                 % (a2, c2, r22))
    print(lines[-1])
    if args.out:
        with open(args.out, "w") as f:
            f.write("# tools/cost_fit.py %s\n" % os.path.relpath(args.bench, ROOT))
            f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
