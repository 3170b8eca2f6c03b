#!/usr/bin/env python3
"""A 2-layer GCN trained on graph partitions with graphAllgather, checked against the full graph.

PAPER.md Listing 1 and §4: each GPU runs the GNN in single-GPU mode on its
partition plus the halo rows graph_allgather delivers; remote rows are dropped before the dense
ops.  Here all `m` partitions are virtual ranks of a 1-GPU loopback context, so the
per-partition sparse aggregation matrices stack into one [N x (N + S)] matrix over
[local rows ; halo rows] — exactly the computation m GPUs would do, block by block.

Model (mean aggregation over in-neighbours and self, eq. 1):
    H1 = relu(Agg(X) W0),   Y = Agg(H1) W1,   loss = sum(Y * T)
Agg on a partition reads halo rows from graph_allgather; its backward is the library's
fixed-order backward kernel.  The reference runs the same model on the whole graph.
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def build_matrices(g, order, device):
    """(M [N x (N+S)] partition-local aggregation, A [N x N] full-graph aggregation), both in the
    loopback row order (row r <-> vertex order[r])."""
    import torch
    n, m = g.n, g.m
    inv = np.empty(n, np.int64)
    inv[order] = np.arange(n)
    src = g.src.astype(np.int64)
    dst = g.dst.astype(np.int64)
    indeg = np.bincount(dst, minlength=n) + 1
    w_e = 1.0 / indeg[dst]
    # halo position of (vertex u, requesting GPU d): global halo row in the loopback layout
    hpos = {}
    for d in range(m):
        for i, u in enumerate(g.R(d)):
            hpos[(int(u), d)] = int(g.req_ptr[d]) + i
    rows_full = inv[dst]
    cols_full = inv[src]
    cols_part = np.empty_like(cols_full)
    for k in range(src.shape[0]):
        u, v = int(src[k]), int(dst[k])
        d = int(g.part[v])
        cols_part[k] = inv[u] if g.part[u] == d else n + hpos[(u, d)]
    self_rows = np.arange(n)
    self_w = 1.0 / indeg[order]
    S = int(g.req_ptr[-1])

    def sp(rows, cols, vals, shape):
        idx = torch.from_numpy(np.stack([rows, cols]))
        return torch.sparse_coo_tensor(idx, torch.from_numpy(vals.astype(np.float32)), shape,
                                       device=device).coalesce()

    M = sp(np.concatenate([rows_full, self_rows]), np.concatenate([cols_part, self_rows]),
           np.concatenate([w_e, self_w]), (n, n + S))
    A = sp(np.concatenate([rows_full, self_rows]), np.concatenate([cols_full, self_rows]),
           np.concatenate([w_e, self_w]), (n, n))
    return M, A


def run(n=3000, e=24000, m=4, dims=(16, 8), out_dim=4, seed=7, device=0):
    import torch

    import paper_conf_eurosys_cai0wmcy21_b200 as D
    import synth
    torch.manual_seed(seed)
    dev = torch.device("cuda", device)
    g = synth.make_graph(n, e, m, graph_seed=seed, part_seed=seed + 1)
    order = np.argsort(g.part, kind="stable")
    ctx = D.loopback(m, g.part, list(dims), device=device)
    ctx.build_plan(g.req_ptr, g.req_ids, seed=0)
    ctx.register_workspace()
    M, A = build_matrices(g, order, dev)
    X0 = torch.randn(n, dims[0], device=dev)
    W0 = torch.randn(dims[0], dims[1], device=dev) * 0.3
    W1 = torch.randn(dims[1], out_dim, device=dev) * 0.3
    T = torch.randn(n, out_dim, device=dev)

    def model(agg):
        X = X0.clone().requires_grad_(True)
        w0 = W0.clone().requires_grad_(True)
        w1 = W1.clone().requires_grad_(True)
        h1 = torch.relu(agg(X, 0) @ w0)
        y = agg(h1, 1) @ w1
        loss = (y * T).sum()
        loss.backward()
        return y.detach(), X.grad, w0.grad, w1.grad

    # distributed: graph_allgather -> [local rows; halo rows], then the partition matrices
    dist = model(lambda h, layer: torch.sparse.mm(M, D.graph_allgather(ctx, layer, h.contiguous())))
    ref = model(lambda h, layer: torch.sparse.mm(A, h))
    torch.cuda.synchronize()
    ctx.check()
    errs = {}
    for name, a, b in zip(["y", "grad_x", "grad_w0", "grad_w1"], dist, ref):
        errs[name] = float((a - b).abs().max() / (b.abs().max() + 1e-30))
    launches = ctx.launch_count()
    ctx.destroy()
    return errs, launches


if __name__ == "__main__":
    errs, launches = run()
    print("max relative error vs the full graph:", errs, "executor launches:", launches)
