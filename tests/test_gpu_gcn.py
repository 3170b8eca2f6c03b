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
