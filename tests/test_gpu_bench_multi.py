"""The N > 1 leg of bench.py end to end (-m gpu): torchrun with two ranks, one process per rank,
both on cuda:0 (--share-gpu: this run has one GPU; the ranks' kernels time-slice), gloo process
group for setup, CUDA IPC peer mapping, per-rank programs with the ready/done protocol.  Checks
the JSON line the driver reads (keys, max-over-ranks timing, e2e with host copies, launches)."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.usefixtures("built")]

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _check_line(d, world, steps, warmup):
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "dtype", "config", "roofline", "e2e",
              "gpu_launches", "cpu_baseline", "clocks"):
        assert k in d, k
    assert d["n_gpus"] == world and d["steps"] == steps and d["warmup"] == warmup
    assert d["value"] > 0 and d["ms_per_step"] > 0
    assert d["gpu_launches"] >= world * steps * 2          # ranks x steps x (fwd + bwd)
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    r = d["roofline"]
    assert r["peak"] == 900.0 and r["bound"] == "nvlink" and 0 < r["frac"]
    for name, k in r["per_kernel"].items():
        st = k["per_call_ms_max_over_ranks"]
        assert st["calls"] >= 10 and st["p10"] <= st["median"] <= st["p90"]
        assert st["mean_first10"] > 0 and k["t_lb_ms"] > 0
        assert len(k["per_rank"]) == world
        assert sum(x["rows_in"] for x in k["per_rank"]) == d["config"]["halo_rows_total"]
        assert sum(x["rows_out"] for x in k["per_rank"]) == d["config"]["halo_rows_total"]
    acct = d["plan_accounting"]
    assert len(acct["rows_out"]) == acct["stages"] >= 1
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["value"] > 0 and c["cores"] >= 1


def test_bench_two_ranks_shared_gpu():
    """torchrun launch (the driver's form), two ranks on cuda:0."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py",
           "--gpus", "2", "--share-gpu", "--config", "tiny", "--steps", "2", "--warmup", "3",
           "--e2e-steps", "1", "--calls", "10", "--cpu-budget", "1"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]           # rank 0 prints ONE line
    _check_line(json.loads(lines[0]), 2, 2, 3)


def test_bench_gpus_flag_spawns_ranks():
    """`bench.py --gpus 2` without torchrun starts the ranks itself (here on one shared GPU), and
    refuses to run with fewer visible GPUs than asked for (no silent 1-GPU fallback)."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    base = [sys.executable, "bench.py", "--gpus", "2", "--config", "tiny", "--steps", "2",
            "--warmup", "3", "--e2e-steps", "1", "--calls", "10", "--cpu-budget", "1"]
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run(base + ["--share-gpu"], cwd=ROOT, capture_output=True, text=True,
                       timeout=600, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    _check_line(json.loads(lines[0]), 2, 2, 3)
    if torch.cuda.device_count() < 2:
        r = subprocess.run(base, cwd=ROOT, capture_output=True, text=True, timeout=600, env=env)
        assert r.returncode != 0 and not [l for l in r.stdout.splitlines() if l.startswith("{")]
