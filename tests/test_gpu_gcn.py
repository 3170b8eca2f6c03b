"""Integration: a 2-layer GCN on 4 loopback partitions through
graph_allgather (forward + the fixed-order backward kernel) equals the same GCN on the whole
graph, outputs and all gradients, to fp32 summation-order tolerance (-m gpu)."""
import os
import sys

import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.usefixtures("built")]


def test_gcn_partitions_match_full_graph():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(__file__)), "examples"))
    import gcn_loopback
    errs, launches = gcn_loopback.run()
    assert launches >= 4                       # 2 forward + 2 backward executor launches
    for k, v in errs.items():
        assert v < 1e-5, (k, v)


def test_gcn_unaligned_dims_match_full_graph():
    """The same with feature dims that are not multiples of 4 floats (contiguous [n, 602] / [n, 7]
    activations: graph_allgather lays them out at the library pitch, bulk-copy executor)."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(__file__)), "examples"))
    import gcn_loopback
    errs, launches = gcn_loopback.run(dims=(602, 7), out_dim=3)
    assert launches >= 4
    for k, v in errs.items():
        assert v < 1e-5, (k, v)


def test_gcn_aggregation_overlapped_with_exchange():
    """NEXT-2: the aggregation's local part runs on a second stream while the executor (with
    sm_budget) moves the halo; each (receiver, source) block waits on its arrival counter
    (dgcl_stream_wait_arrival).  Same result as the full-graph aggregation and as the sequential
    form, from a zeroed halo."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(__file__)), "examples"))
    import gcn_overlap
    out = gcn_overlap.run(n=20000, e=200000, m=4, dim=64, sm_budget=100, reps=2)
    for mode in ("sequential", "overlapped"):
        assert out[mode]["max_rel_err_vs_full_graph"] < 1e-5, out


def test_wait_arrival_needs_signals_in_fused_loopback():
    import numpy as np
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_eurosys_cai0wmcy21_b200 as D
    import synth
    g = synth.make_graph(2000, 15000, 2, graph_seed=1, part_seed=2)
    ctx = D.loopback(2, g.part, [8], device=0)
    ctx.build_plan(g.req_ptr, g.req_ids)
    ctx.register_workspace()
    ctx.forward(0, torch.zeros(g.n, 8, device="cuda"))
    with pytest.raises(D.DGCLError) as e:
        ctx.wait_arrival(src=1, dst=0)
    assert e.value.status == 2
    with pytest.raises(D.DGCLError) as e:
        ctx.wait_arrival(src=0, dst=0)
    torch.cuda.synchronize()
    ctx.destroy()
