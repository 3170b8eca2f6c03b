"""Multi-GPU leg of bench.py (N > 1, one process per GPU; launched by torchrun, or spawned by
`bench.py --gpus N` itself).

The configured graph is partitioned N-way (one partition per GPU, the paper's setting P:379-387);
rank 0 builds the graph and the required lists and broadcasts them; every rank builds the
identical plan, allocates its workspace and maps its peers with CUDA IPC (setup, torch process
group).  The timed steps run the same executor as N = 1, storing into peers' memory over NVLink.

Timing (SURVEY §8(d) "timing protocol", a13; PAPER.md times communication after warm-up, mean of
10 runs):
  * the driver's step: W warm-up steps, then K steps between a barrier + synchronize on both
    sides, CUDA events on the launching stream, max over ranks -> value, ms_per_step;
  * per call, per launch (forward of every layer, backward of the backward layers): 5 warm-up
    calls, then `--calls` timed calls, each = device start barrier (dgcl_device_barrier: every
    rank has arrived) -> event -> dispatch -> event; the per-call time is the max over ranks;
    reported as median, p10 / p90 and the mean of the first 10 calls;
  * accounting per rank and stage: rows / bytes out and in (the plan's tuples), achieved GB/s per
    rank; t_lb = max_d max(out_d, in_d) * dim * 4 / 900 GB/s (NVLink 5 per direction, the
    north-star denominator); frac = t_lb / t_median; the measured 770 GB/s peer copy
    (B200_PROFILING.md) is reported beside it as context;
  * NVLink data counters (NVML field values, TX / RX KiB summed over links) read before and
    after each launch's timed calls: bytes per call on the wire, the roofline's `traffic`;
  * the NCCL peer-to-peer baseline (bench_p2p.py: pack by send list, grouped send / recv,
    unpack; §7.1) timed with the same per-call protocol when the process
    group is NCCL (one GPU per rank);
  * the CPU oracle on rank 0 after the timed region (bounded sample) -> cpu_baseline.
"""
import statistics
import time

import numpy as np

NVLINK_GBS = 900.0        # NVLink 5 per direction per GPU (north_star's denominator)
NVLINK_PEER_GBS = 770.0   # measured peer copy per direction (B200_PROFILING.md), context only


class NvlinkCounters:
    """NVLink data TX / RX counters of one device (NVML, KiB, summed over the links)."""
    MAX_LINKS = 18

    def __init__(self, device_index):
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.ids = []
            for f in (pynvml.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_TX,
                      pynvml.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_RX):
                for link in range(self.MAX_LINKS):
                    self.ids.append((f, link))
            self.read()
            self.ok = True
        except Exception as e:  # no NVML / no NVLink: reported as unavailable
            self.err = str(e)

    def read(self):
        """(tx_bytes, rx_bytes, links that answered)."""
        vals = self.nv.nvmlDeviceGetFieldValues(self.h, self.ids)
        tx = rx = 0
        links = set()
        for (f, link), v in zip(self.ids, vals):
            if v.nvmlReturn != 0:
                continue
            x = int(v.value.ullVal) * 1024
            links.add(link)
            if f == self.nv.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_TX:
                tx += x
            else:
                rx += x
        return tx, rx, len(links)


def _stats(ms):
    a = np.asarray(ms, np.float64)
    return {"median": float(np.median(a)), "p10": float(np.percentile(a, 10)),
            "p90": float(np.percentile(a, 90)), "mean_first10": float(a[:10].mean()),
            "mean": float(a.mean()), "min": float(a.min()), "calls": int(a.size)}


def _per_call(fn, barrier, stream, calls, warm=5):
    """Per-call device times: barrier -> event -> fn -> event (ms, this rank)."""
    import torch
    for _ in range(warm):
        barrier()
        fn()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(calls)]
    for a, b in evs:
        barrier()
        a.record(stream)
        fn()
        b.record(stream)
    torch.cuda.synchronize()
    return [a.elapsed_time(b) for a, b in evs]


def plan_accounting(counts, dims_bytes):
    """Per rank and stage rows out / in from the plan's (stage, src, dst) row counts."""
    K = counts.shape[0]
    out = counts.sum(axis=2)   # [K x m]: rows rank s sends at stage k
    inn = counts.sum(axis=1)   # [K x m]: rows rank d receives at stage k
    return {"stages": K, "rows_out": out.tolist(), "rows_in": inn.tolist(),
            "rows_out_total": out.sum(axis=0).tolist(), "rows_in_total": inn.sum(axis=0).tolist()}


def run_multi(args, metric, unit, rank, world, local_rank, ClockSampler, make_workload=None,
              oracle_sample=None, host_inputs=None):
    import torch
    import torch.distributed as dist

    import paper_conf_eurosys_cai0wmcy21_b200 as D
    import synth

    share = args.share_gpu
    dev = 0 if share else local_rank
    torch.cuda.set_device(dev)
    backend = "gloo" if share else "nccl"
    if backend == "nccl":
        dist.init_process_group(backend, device_id=torch.device("cuda", dev))
    else:
        dist.init_process_group(backend)
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
    for kv in args.opt:
        k, v = kv.split("=")
        ctx.set_option(k, int(v))
    ctx.build_plan(ptr, ids, seed=0, topology=topo)
    ctx.register_workspace()
    blobs = [None] * world
    dist.all_gather_object(blobs, ctx.ipc_export())
    ctx.ipc_import(blobs)
    dist.barrier()
    if ctx.multicast_bytes()[1] > 0:  # option multicast: NVSwitch multicast object
        from paper_conf_eurosys_cai0wmcy21_b200.dgcl import _setup_multicast
        _setup_multicast(ctx)
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
    calls_of = {}
    for l in fwd_layers:
        calls_of["fwd%d_d%d" % (l, dims[l])] = (lambda l=l: ctx.forward(l, emb[l], stream=stream))
    for l in bwd_layers:
        calls_of["bwd%d_d%d" % (l, dims[l])] = (lambda l=l: ctx.backward(l, hg[l], eg[l],
                                                                         stream=stream))

    def step(evs=None):
        for i, n in enumerate(names):
            if evs is not None:
                evs[i][0].record(stream)
            calls_of[n]()
            if evs is not None:
                evs[i][1].record(stream)

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

    # ---- per-call protocol with the device start barrier, NVLink counters around each ----
    nvl = NvlinkCounters(dev)
    barrier = lambda: ctx.device_barrier(stream)
    per_call_ms, nvl_bytes = {}, {}
    for n in names:
        c0 = nvl.read() if nvl.ok else None
        per_call_ms[n] = _per_call(calls_of[n], barrier, stream, args.calls)
        if nvl.ok:
            c1 = nvl.read()
            nvl_bytes[n] = {"tx_per_call": (c1[0] - c0[0]) / (args.calls + 5),
                            "rx_per_call": (c1[1] - c0[1]) / (args.calls + 5), "links": c1[2]}
    ctx.check()

    # ---- NCCL peer-to-peer baseline (pack + grouped send/recv + unpack), same protocol ----
    p2p_ms = None
    if backend == "nccl" and not args.no_p2p_baseline:
        import bench_p2p
        ex = bench_p2p.P2PExchange(part, ptr, ids, rank, world, torch.device("cuda", dev))
        halos = {l: torch.zeros(n_halo, ctx.pitch(l), dtype=torch.float32, device="cuda")
                 for l in fwd_layers}
        eg2 = {l: eg[l].clone() for l in bwd_layers}
        p2p_calls = {}
        for l in fwd_layers:
            p2p_calls["fwd%d_d%d" % (l, dims[l])] = (lambda l=l: ex.forward(emb[l], halos[l]))
        for l in bwd_layers:
            p2p_calls["bwd%d_d%d" % (l, dims[l])] = (lambda l=l: ex.backward(hg[l], eg2[l]))
        p2p_ms = {n: _per_call(p2p_calls[n], barrier, stream, args.calls) for n in names}
        # the baseline computes the same halos (bit-exact forward)
        ok = all(torch.equal(halos[l][:, :dims[l]], ctx.halo(l)[:, :dims[l]]) for l in fwd_layers)
        p2p_ok = torch.tensor([1.0 if ok else 0.0], device="cuda")
        dist.all_reduce(p2p_ok, op=dist.ReduceOp.MIN)
        p2p_ok = bool(p2p_ok.item() > 0)
        del halos, eg2

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

    # ---- max over ranks ----
    def allmax(vals):
        t = torch.tensor(vals, dtype=torch.float64)
        if not share:
            t = t.cuda()
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return t.cpu().tolist()

    def allsum(vals):
        t = torch.tensor(vals, dtype=torch.float64)
        if not share:
            t = t.cuda()
        dist.all_reduce(t)
        return t.cpu().tolist()

    t = allmax([e0.elapsed_time(e1)] + [statistics.mean(
        evs[k][i][0].elapsed_time(evs[k][i][1]) for k in range(K)) for i in range(len(names))] +
        [e2e_ms])
    calls_max = {n: allmax(per_call_ms[n]) for n in names}
    p2p_max = {n: allmax(p2p_ms[n]) for n in names} if p2p_ms else None
    per_rank_call = {n: np.asarray(allsum([0.0] * rank + [float(np.median(per_call_ms[n]))] +
                                          [0.0] * (world - rank - 1))) for n in names}
    hb = allsum([float(h2d), float(d2h)])
    lt = allsum([float(launches)])
    nvl_all = None
    if nvl_bytes:
        nvl_all = {n: allsum([0.0] * (2 * rank) + [nvl_bytes[n]["tx_per_call"],
                                                   nvl_bytes[n]["rx_per_call"]] +
                             [0.0] * (2 * (world - rank - 1))) for n in names}
    counts = ctx.plan_counts()
    if clk:
        clk.stop()
    clocks = clk.summary(tw0, tw1) if clk else None
    if clocks and clocks["samples"] == 0:
        clocks = clk.summary()

    # ---- CPU oracle on rank 0 (after every timed region; the other ranks wait) ----
    cpu = None
    if rank == 0 and not args.no_cpu_baseline and make_workload is not None:
        w = make_workload(cfg, world, part, ptr, ids)
        pitches = {l: synth.configs.pitch_of(dims[l]) for l in range(len(dims))}
        emb_h, hg_h, eg_h = host_inputs(w, pitches)
        gbs, secs, used, thr = oracle_sample(w, emb_h, hg_h, eg_h, budget_s=args.cpu_budget)
        cpu = {"value": gbs, "unit": unit, "cores": thr, "kind": "oracle",
               "sample": "oracle forward (all layers) + flat backward for destination/owner "
                         "ranks %s of %d (%.1f s of CPU work, rank 0's host)" % (used, world, secs)}
        del emb_h, hg_h, eg_h
    dist.barrier()
    ctx.destroy()
    if rank != 0:
        return None

    # ---- accounting ----
    ms_step = float(t[0]) / K
    per_op = {n: float(t[1 + i]) for i, n in enumerate(names)}
    S = int(ptr[-1])
    payload = S * 4 * (sum(dims[l] for l in fwd_layers) + sum(dims[l] for l in bwd_layers))
    value = payload / (ms_step * 1e-3) / 1e9
    acct = plan_accounting(counts, None)
    # deliveries (the direct minimum): out_d = sum over my vertices of |D_u|, in_d = |R_d|
    in_del = np.diff(ptr).astype(np.int64)
    owner_of = part[ids]
    out_del = np.bincount(owner_of, minlength=world).astype(np.int64)
    maxport_del = int(max(in_del.max(), out_del.max()))
    out_plan = np.asarray(acct["rows_out_total"], np.int64)
    in_plan = np.asarray(acct["rows_in_total"], np.int64)
    maxport_plan = int(max(out_plan.max(), in_plan.max())) if counts.size else 0
    kernels = {}
    for i, n in enumerate(names):
        l = (fwd_layers + bwd_layers)[i]
        row = dims[l] * 4
        st = _stats(calls_max[n])
        t_lb = maxport_del * row / (NVLINK_GBS * 1e9) * 1e3
        ach = maxport_del * row / (st["median"] * 1e-3) / 1e9
        med_r = per_rank_call[n]
        kernels[n] = {
            "ms_step_mean": per_op[n], "per_call_ms_max_over_ranks": st,
            "t_lb_ms": t_lb, "frac": t_lb / st["median"], "achieved_gbs_max_port": ach,
            "frac_vs_measured_peer_copy": ach / NVLINK_PEER_GBS,
            "algorithmic_bytes_max_port": maxport_del * row,
            "plan_bytes_max_port": maxport_plan * row,
            "per_rank": [{"rank": d, "rows_out": int(out_del[d]), "rows_in": int(in_del[d]),
                          "bytes_out": int(out_del[d]) * row, "bytes_in": int(in_del[d]) * row,
                          "plan_rows_out": int(out_plan[d]), "plan_rows_in": int(in_plan[d]),
                          "median_ms": float(med_r[d]),
                          "gbs_out": int(out_plan[d]) * row / (med_r[d] * 1e-3) / 1e9,
                          "gbs_in": int(in_plan[d]) * row / (med_r[d] * 1e-3) / 1e9}
                         for d in range(world)],
        }
        if nvl_all is not None:
            v = nvl_all[n]
            kernels[n]["nvlink_counter_bytes_per_call"] = {
                "tx": [v[2 * d] for d in range(world)], "rx": [v[2 * d + 1] for d in range(world)]}
        if p2p_max is not None:
            ps = _stats(p2p_max[n])
            kernels[n]["nccl_p2p_baseline"] = dict(ps, frac=t_lb / ps["median"],
                                                   speedup_of_ours=ps["median"] / st["median"])
    dom = max(names, key=lambda n: kernels[n]["per_call_ms_max_over_ranks"]["median"])
    traffic = None
    if nvl_all is not None:
        v = nvl_all[dom]
        traffic = max(max(v[0::2]), max(v[1::2])) or None
    e2e = None
    if args.e2e_steps > 0:
        e2e_ms = float(t[1 + len(names)])
        e2e = {"value": payload / (e2e_ms * 1e-3) / 1e9, "unit": unit, "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": int(hb[0]), "d2h_bytes_per_step": int(hb[1]),
               "note": "all ranks' host copies, max over ranks of the step time"}
    return {
        "metric": metric, "value": value, "unit": unit, "n_gpus": world, "steps": K,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "impl": "ours",
        "config": {"workload": "%s-shaped R-MAT, %d-way partition over %d B200 (NVLink 5)%s" %
                               (cfg.name, world, world, " [shared GPU test mode]" if share else ""),
                   "config": cfg.name, "dims": dims, "world": world,
                   "fwd_layers": fwd_layers, "bwd_layers": bwd_layers, "halo_rows_total": S,
                   "halo_rows_per_rank": in_del.tolist(),
                   "parallelism": "graph-partition x%d" % world, "backend_setup": backend,
                   "options": list(args.opt),
                   "l2": "inputs larger than L2 (no flush needed)"},
        "ms_per_layer": per_op,
        "gbs_per_gpu": value / world,
        "roofline": {"bound": "nvlink", "kernel": "executor_tma_kernel (%s)" % dom,
                     "achieved": kernels[dom]["achieved_gbs_max_port"], "peak": NVLINK_GBS,
                     "unit": "GB/s", "frac": kernels[dom]["frac"], "traffic": traffic,
                     "traffic_source": ("NVML NVLink data TX/RX counters, max over ranks, bytes "
                                        "per call" if traffic else
                                        "unavailable (%s)" % getattr(nvl, "err", "no NVLink "
                                                                     "traffic counted")),
                     "peak_source": "NVLink 5 nominal 900 GB/s per direction (north_star); "
                                    "measured peer copy %.0f GB/s as context" % NVLINK_PEER_GBS,
                     "algorithmic_bytes_per_launch": kernels[dom]["algorithmic_bytes_max_port"],
                     "per_kernel": kernels},
        "plan_accounting": acct,
        "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(lt[0]),
        "nccl_p2p_check": (p2p_ok if p2p_ms else None),
        "clocks": clocks, "plan": dict(info, graph_gen_s=gen_s),
    }
