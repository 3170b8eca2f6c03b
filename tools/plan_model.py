#!/usr/bin/env python3
"""SPST against the direct (peer-to-peer) plan in the §5.1 cost model — the model-space analogue of
the paper's planner evaluation (per-link balance, Table 7; the
P2P baseline of Figs. 7-8).  Host only (no GPU).

For each (graph, topology): the SPST plan (Algorithm 1) and the direct plan (every delivery
owner -> requester in stage 1, loaded through dgcl_build_plan_from_trees so the library recomputes
t(S) with the same rules), their model time t(S) (ticks -> ms for the config's row size), stages,
tree edges, and the load balance of the busiest stage: max / mean rows per used physical hop.

usage: python tools/plan_model.py [config ...]     (default: google8 reddit)
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np

import paper_conf_eurosys_cai0wmcy21_b200 as D
import synth


def ticks_to_ms(ticks, row_bytes):
    # a hop of G GB/s costs w = 1e5 / G ticks per row (R7): one tick = row_bytes / 1e14 s
    return ticks * row_bytes / 1e14 * 1e3


def hop_balance(E, topo, stage=1):
    """max / mean rows over the physical hops used in `stage` (per-link balance, Table 7)."""
    load = {}
    for (_, p, c, k) in E:
        if k != stage:
            continue
        for h in topo.links[(int(p), int(c))]:
            load[h] = load.get(h, 0) + 1
    v = np.array(list(load.values()), np.float64)
    return (v.max() / v.mean()) if v.size else 0.0, int(v.max()) if v.size else 0


def main(names):
    rows = []
    for name in names:
        cfg = synth.get_config(name)
        g = synth.make_graph(cfg.n, cfg.e, cfg.m, cfg.graph_seed, cfg.part_seed, keep_edges=False)
        row_bytes = 4 * cfg.dims[-1]
        # direct plan: every (u, d) delivery straight from the owner in stage 1
        ids = np.asarray(g.req_ids, np.int64)
        dsts = np.repeat(np.arange(cfg.m), np.diff(g.req_ptr))
        direct = np.stack([ids, g.part[ids], dsts, np.ones_like(ids)], axis=1)
        direct = direct[np.lexsort((direct[:, 2], direct[:, 0]))]  # grouped per vertex
        for tname in ("uniform_nvswitch", "dgx1_like", "ring"):
            topo = synth.topology.by_name(tname, cfg.m)
            out = {}
            for kind in ("spst", "direct"):
                c = D.loopback(cfg.m, g.part, [cfg.dims[-1]], device=-1)
                c.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo,
                             trees=direct if kind == "direct" else None)
                info = c.plan_info()
                E = c.plan_export()
                bal, mx = hop_balance(E, topo)
                out[kind] = (info["model_cost_ticks"], info["n_stages"], info["n_tree_edges"], bal,
                             info["planner_seconds"])
                c.destroy()
            s, d = out["spst"], out["direct"]
            rows.append((name, tname, ticks_to_ms(s[0], row_bytes), ticks_to_ms(d[0], row_bytes),
                         d[0] / s[0], s[1], s[2], d[2], s[3], d[3], s[4]))
            print("%-8s %-16s model ms SPST %.3f direct %.3f (x%.2f)  stages %d  tree edges %d "
                  "(direct %d)  stage-1 hop max/mean SPST %.2f direct %.2f  plan %.2f s" % rows[-1],
                  flush=True)
    return rows


if __name__ == "__main__":
    main(sys.argv[1:] or ["google8", "reddit"])
