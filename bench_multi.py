"""Multi-GPU leg of bench.py (N > 1 under torchrun, one process per GPU).

The configured graph is partitioned N-way (one partition per GPU, the paper's setting P:379-387);
rank 0 builds the graph and the required lists and broadcasts them; every rank builds the
identical plan, allocates its workspace, and maps its peers with CUDA IPC (setup, torch process
group).  The timed steps run the same executor as N=1 over NVLink peer memory.  Per-launch and
per-step times are CUDA events on the launching stream, max over ranks.
"""
import statistics
import time

import numpy as np

NVLINK_PEER_GBS = 770.0  # measured peer copy per direction (B200_PROFILING.md); 900 nominal


def run_multi(args, metric, unit, rank, world, local_rank, ClockSampler):
    import torch
    import torch.distributed as dist

    import paper_conf_eurosys_cai0wmcy21_b200 as D
    import synth

    share = args.share_gpu
    dev = 0 if share else local_rank
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo" if share else "nccl")
    cfg = synth.get_config(args.config)
    dims = list(cfg.dims)
    fwd_layers = list(range(len(dims)))
    bwd_layers = list(cfg.backward_layers)
    t0 = time.time()
    obj = [None]
    if rank == 0:
        src, dst = synth.rmat_edges(cfg.n, cfg.e, cfg.graph_seed)
        part = synth.partition(cfg.n, world, cfg.part_seed)
        ptr, ids = synth.required_lists(src, dst, part, world)
        del src, dst
        obj = [(part, ptr, ids)]
    dist.broadcast_object_list(obj, src=0)
    part, ptr, ids = obj[0]
    gen_s = time.time() - t0
    topo = None
    if cfg.topology != "uniform_nvswitch":
        topo = synth.topology.by_name(cfg.topology, world)
    ctx = D.init(part, dims, rank, world, dev)
    ctx.build_plan(ptr, ids, seed=0, topology=topo)
    ctx.register_workspace()
    blobs = [None] * world
    dist.all_gather_object(blobs, ctx.ipc_export())
    ctx.ipc_import(blobs)
    dist.barrier()
    info = ctx.plan_info()
    mine = np.nonzero(part == rank)[0]
    n_halo = int(ptr[rank + 1] - ptr[rank])
    emb, hg, eg = {}, {}, {}
    for l in fwd_layers:
        p = ctx.pitch(l)
        emb[l] = torch.from_numpy(synth.fill_values(len(mine), dims[l], p, keys=mine,
                                                    seed=cfg.emb_seed,
                                                    stream=synth.values.STREAM_EMB + l)).cuda()
    for l in bwd_layers:
        p = ctx.pitch(l)
        keys = np.arange(int(ptr[rank]), int(ptr[rank]) + n_halo)
        hg[l] = torch.from_numpy(synth.fill_values(n_halo, dims[l], p, keys=keys,
                                                   seed=cfg.grad_seed,
                                                   stream=synth.values.STREAM_HGRAD + l)).cuda()
        eg[l] = torch.from_numpy(synth.fill_values(len(mine), dims[l], p, keys=mine,
                                                   seed=cfg.grad_seed,
                                                   stream=synth.values.STREAM_EGRAD + l)).cuda()
    stream = torch.cuda.current_stream()
    names = ["fwd%d_d%d" % (l, dims[l]) for l in fwd_layers] + \
            ["bwd%d_d%d" % (l, dims[l]) for l in bwd_layers]

    def step(evs=None):
        i = 0
        for l in fwd_layers:
            if evs is not None:
                evs[i][0].record(stream)
            ctx.forward(l, emb[l], stream=stream)
            if evs is not None:
                evs[i][1].record(stream)
            i += 1
        for l in bwd_layers:
            if evs is not None:
                evs[i][0].record(stream)
            ctx.backward(l, hg[l], eg[l], stream=stream)
            if evs is not None:
                evs[i][1].record(stream)
            i += 1

    clk = ClockSampler(dev) if rank == 0 else None
    if clk:
        clk.start()
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    ctx.check()
    K = args.steps
    evs = [[[torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)]
            for _ in names] for _ in range(K)]
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    l0 = ctx.launch_count()
    dist.barrier()
    torch.cuda.synchronize()
    tw0 = time.time()
    e0.record(stream)
    for k in range(K):
        step(evs[k])
    e1.record(stream)
    torch.cuda.synchronize()
    dist.barrier()
    tw1 = time.time()
    ctx.check()
    launches = ctx.launch_count() - l0

    # ---- e2e through the host-buffer C-ABI calls: every step copies this rank's inputs from
    # pinned host memory and its halos / gradients back (inside the timed region) ----
    e2e_ms, h2d, d2h = 0.0, 0, 0
    if args.e2e_steps > 0:
        pin = lambda t: t.cpu().pin_memory()
        emb_p = {l: pin(a) for l, a in emb.items()}
        hg_p = {l: pin(a) for l, a in hg.items()}
        eg_p = {l: pin(a) for l, a in eg.items()}
        halo_p = {l: torch.empty(n_halo, ctx.pitch(l), dtype=torch.float32).pin_memory()
                  for l in fwd_layers}
        h2d = sum(a.numel() * 4 for d_ in (emb_p, hg_p, eg_p) for a in d_.values())
        d2h = sum(a.numel() * 4 for d_ in (halo_p, eg_p) for a in d_.values())
        ctx.set_option("host_async", 1)

        def e2e_step():
            for l in fwd_layers:
                ctx.forward_host(l, emb_p[l], halo_p[l], stream=stream)
            for l in bwd_layers:
                ctx.backward_host(l, hg_p[l], eg_p[l], stream=stream)

        e2e_step()
        torch.cuda.synchronize()
        dist.barrier()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        for _ in range(args.e2e_steps):
            e2e_step()
        a1.record(stream)
        torch.cuda.synchronize()
        dist.barrier()
        ctx.check()
        e2e_ms = a0.elapsed_time(a1) / args.e2e_steps
    t = torch.tensor([e0.elapsed_time(e1)] + [statistics.mean(
        evs[k][i][0].elapsed_time(evs[k][i][1]) for k in range(K)) for i in range(len(names))] +
        [e2e_ms], dtype=torch.float64)
    hb = torch.tensor([float(h2d), float(d2h)], dtype=torch.float64)
    if not share:
        hb = hb.cuda()
    dist.all_reduce(hb)
    if not share:
        t = t.cuda()
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    lt = torch.tensor([float(launches)], dtype=torch.float64)
    if not share:
        lt = lt.cuda()
    dist.all_reduce(lt)
    t = t.cpu()
    if clk:
        clk.stop()
    counts = ctx.plan_counts()
    ctx.destroy()
    if rank != 0:
        return None
    ms_step = float(t[0]) / K
    per_op = {n: float(t[1 + i]) for i, n in enumerate(names)}
    S = int(ptr[-1])
    payload = S * 4 * (sum(dims[l] for l in fwd_layers) + sum(dims[l] for l in bwd_layers))
    value = payload / (ms_step * 1e-3) / 1e9
    out_rows = counts.sum(axis=(0, 2))
    in_rows = counts.sum(axis=(0, 1))
    maxport = int(max(out_rows.max(), in_rows.max())) if counts.size else 0
    kernels = {}
    for i, n in enumerate(names):
        l = (fwd_layers + bwd_layers)[i]
        alg = maxport * dims[l] * 4
        ach = alg / (per_op[n] * 1e-3) / 1e9
        kernels[n] = {"ms": per_op[n], "algorithmic_bytes_max_port": alg, "achieved_gbs": ach,
                      "frac": ach / NVLINK_PEER_GBS}
    dom = max(names, key=lambda n: per_op[n])
    e2e = None
    if args.e2e_steps > 0:
        e2e_ms = float(t[1 + len(names)])
        hb = hb.cpu()
        e2e = {"value": payload / (e2e_ms * 1e-3) / 1e9, "unit": unit, "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": int(hb[0]), "d2h_bytes_per_step": int(hb[1]),
               "note": "all ranks' host copies, max over ranks of the step time"}
    clocks = clk.summary(tw0, tw1) if clk else None
    if clocks and clocks["samples"] == 0:
        clocks = clk.summary()
    return {
        "metric": metric, "value": value, "unit": unit, "n_gpus": world, "steps": K,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "impl": "ours",
        "config": {"workload": "%s-shaped R-MAT, %d-way partition over %d B200 (NVLink 5)%s" %
                               (cfg.name, world, world, " [shared GPU test mode]" if share else ""),
                   "config": cfg.name, "dims": dims, "world": world,
                   "fwd_layers": fwd_layers, "bwd_layers": bwd_layers, "halo_rows_total": S,
                   "parallelism": "graph-partition x%d" % world,
                   "l2": "inputs larger than L2 (no flush needed)"},
        "ms_per_layer": per_op,
        "gbs_per_gpu": value / world,
        "roofline": {"bound": "nvlink", "kernel": "executor_tma_kernel (%s)" % dom,
                     "achieved": kernels[dom]["achieved_gbs"], "peak": NVLINK_PEER_GBS,
                     "unit": "GB/s", "frac": kernels[dom]["frac"], "traffic": None,
                     "nominal_peak": 900.0,
                     "algorithmic_bytes_per_launch": kernels[dom]["algorithmic_bytes_max_port"],
                     "per_kernel": kernels},
        "cpu_baseline": None, "e2e": e2e, "gpu_launches": int(lt[0]),
        "clocks": clocks, "plan": dict(info, graph_gen_s=gen_s),
    }
