#!/usr/bin/env python3
"""Benchmark of the DGCL halo-exchange hot path on B200 (BASELINE.json metric).

metric: per-layer embedding-exchange ms and NVLink GB/s/GPU at 1/2/4/8 B200 vs 900 GB/s
A STEP is one GCN training step's communication on the configured graph: graphAllgather forward
of every layer, then the backward of the layers that need gradients (for the Reddit-shaped config:
forward dim 602 and dim 256, backward dim 256).  value = halo payload delivered by the whole job
per second (sum over layers of sum_d |R_d| x dim x 4 bytes, forward and backward) in GB/s;
per-layer ms and per-GPU GB/s are reported beside it.

N = 1: the 1-GPU loopback configuration (all 8 virtual ranks of the 8-way partition on one
B200, fused executor launch; bound by HBM).  N > 1 (torchrun, one process per GPU): the real
multi-GPU path over NVLink peer memory (bound by NVLink).  --impl reference times the CPU oracle
(the reference arm of this tier) on a bounded sample.

Timing: W warm-up steps, then K steps between device barriers with CUDA events on the launching
stream; max over ranks.  Every input (embeddings 563 MB, halos 3.8 GB for Reddit dim 602) is far
larger than the 126 MB L2, so no explicit flush is needed (config.l2 says so).
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "per-layer embedding-exchange ms and NVLink GB/s/GPU at 1/2/4/8 B200 vs 900 GB/s"
UNIT = "GB/s"


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ---------------------------------------------------------------------------------------------
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms while running."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index):
        self.dev = device_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), "--query-gpu=" + self.Q,
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append((time.time(), line.strip()))

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self, t0=None, t1=None):
        sms, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for (t, line) in self.lines:
            if t0 is not None and (t < t0 - 0.25 or t > t1 + 0.25):
                continue
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sms.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sms:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sms), "sm_max_mhz": max(mx),
                "reasons": sorted(reasons), "samples": len(sms)}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f), "measured"
    return {"hbm_gbs": 6650.0}, "fallback"


def profiled_traffic(key):
    """dram bytes per launch from the committed ncu --set full summary (profiles/traffic.json)."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f).get(key)
    return None


# ---------------------------------------------------------------------------------------------
class Workload:
    """Synthetic inputs of one BASELINE.json config (seeded; shared with the oracle)."""

    def __init__(self, cfg_name):
        import synth
        self.cfg = synth.get_config(cfg_name)
        c = self.cfg
        t = time.time()
        self.g = synth.make_graph(c.n, c.e, c.m, c.graph_seed, c.part_seed, keep_edges=False)
        self.gen_s = time.time() - t
        self.S = int(self.g.req_ptr[-1])
        self.order = np.argsort(self.g.part, kind="stable")
        self.fwd_layers = list(range(len(c.dims)))
        self.bwd_layers = list(c.backward_layers)

    @classmethod
    def from_parts(cls, cfg, world, part, req_ptr, req_ids):
        """The same workload re-partitioned `world`-way (the N > 1 leg's partition)."""
        import dataclasses
        import synth
        w = cls.__new__(cls)
        w.cfg = dataclasses.replace(cfg, m=world)
        w.g = synth.Graph(cfg.n, world, None, None, part, req_ptr, req_ids)
        w.gen_s = 0.0
        w.S = int(req_ptr[-1])
        w.order = np.argsort(part, kind="stable")
        w.fwd_layers = list(range(len(cfg.dims)))
        w.bwd_layers = list(cfg.backward_layers)
        return w

    def step_payload_bytes(self, ranks=None):
        """Halo payload one step delivers (forward) and returns (backward), algorithmic bytes."""
        ptr = self.g.req_ptr
        S = self.S if ranks is None else sum(int(ptr[d + 1] - ptr[d]) for d in ranks)
        dims = self.cfg.dims
        return S * 4 * (sum(dims[l] for l in self.fwd_layers) +
                        sum(dims[l] for l in self.bwd_layers))


def host_inputs(w, pitches, rows_order=None):
    """Hash-defined host arrays in the loopback layouts (see synth/values.py)."""
    import synth
    c = w.cfg
    emb, hg, eg = {}, {}, {}
    for l in w.fwd_layers:
        emb[l] = synth.fill_values(c.n, c.dims[l], pitches[l], keys=w.order, seed=c.emb_seed,
                                   stream=synth.values.STREAM_EMB + l)
    for l in w.bwd_layers:
        hg[l] = synth.fill_values(w.S, c.dims[l], pitches[l], seed=c.grad_seed,
                                  stream=synth.values.STREAM_HGRAD + l)
        eg[l] = synth.fill_values(c.n, c.dims[l], pitches[l], keys=w.order, seed=c.grad_seed,
                                  stream=synth.values.STREAM_EGRAD + l)
    return emb, hg, eg


# ---------------------------------------------------------------------------------------------
def oracle_sample(w, emb, hg, eg, budget_s=15.0, ranks=None, threads=1):
    """Time the CPU oracle (as it stands) on destination/owner ranks until the budget is spent.

    A unit of work is (rank d, chunk j of J): the forward of halo rows R_d[chunk j] (every
    layer) and the flat backward of the owner-d vertices in vertex-id chunk j (the backward
    layers) — oracle.halo calls on sub-lists, nothing re-implemented.  threads == 1: J = 1, ranks
    in order until the budget is spent.  threads > 1: J chunks per rank so that there are >= 2
    units per thread, every unit of the given ranks run in a thread pool over `threads` host
    cores (numpy's gathers and adds release the GIL), wall-clock timed.
    Returns (GB/s, seconds, ranks used, threads)."""
    from oracle import halo
    c = w.cfg
    g = w.g
    m = c.m
    loc, n_local = halo.local_rows(g.part, m)
    ro = np.concatenate([[0], np.cumsum(n_local)])
    R = [g.R(d) for d in range(m)]
    ptr = g.req_ptr
    empty = np.zeros(0, np.int64)

    def unit(d, j, J):
        nb = 0
        a, b = int(ptr[d]), int(ptr[d + 1])
        lo, hi = a + (b - a) * j // J, a + (b - a) * (j + 1) // J
        for l in w.fwd_layers:
            dim = c.dims[l]
            local = [emb[l][ro[s]:ro[s + 1], :dim] for s in range(m)]
            Rd = [g.req_ids[lo:hi] if q == d else empty for q in range(m)]
            halo.forward(local, Rd, g.part, loc)
            nb += (hi - lo) * 4 * dim
        vlo, vhi = g.n * j // J, g.n * (j + 1) // J
        for l in w.bwd_layers:
            dim = c.dims[l]
            L = [eg[l][ro[s]:ro[s + 1], :dim] if s == d else np.zeros((0, dim), np.float32)
                 for s in range(m)]
            G = [hg[l][ptr[q]:ptr[q + 1], :dim] for q in range(m)]
            # owner d's rows in the chunk: every contributor's rows for those vertices
            sel = [(g.part[R[q]] == d) & (R[q] >= vlo) & (R[q] < vhi) for q in range(m)]
            Rd = [R[q][sel[q]] for q in range(m)]
            Gd = [G[q][sel[q]] for q in range(m)]
            halo.backward_flat(L, Gd, Rd, g.part, loc)
            nb += sum(len(r) for r in Rd) * 4 * dim
        return nb

    rk = list(ranks if ranks is not None else range(m))
    if threads > 1:
        from concurrent.futures import ThreadPoolExecutor
        J = max(1, -(-2 * threads // len(rk)))
        units = [(d, j, J) for d in rk for j in range(J)]
        with ThreadPoolExecutor(max_workers=threads) as ex:
            t = time.perf_counter()
            nbytes = sum(ex.map(lambda u: unit(*u), units))
            secs = time.perf_counter() - t
        return nbytes / secs / 1e9, secs, rk, threads
    done_bytes, t_total, used = 0, 0.0, []
    for d in rk:
        t = time.perf_counter()
        done_bytes += unit(d, 0, 1)
        t_total += time.perf_counter() - t
        used.append(d)
        if t_total >= budget_s:
            break
    return done_bytes / t_total / 1e9, t_total, used, 1


# ---------------------------------------------------------------------------------------------
def torch_gather_baseline(w, emb, hg, eg, stream, reps=5):
    """The same loopback exchange with stock PyTorch ops on the same GPU (context for the
    executor's numbers, not our kernels): forward = one torch.index_select of every halo row;
    backward = torch.index_add_ of the halo gradients into the owner rows (atomic scatter-add,
    order not fixed — the Table 9 'atomic' alternative)."""
    import torch
    g = w.g
    inv = np.empty(g.n, np.int64)
    inv[w.order] = np.arange(g.n)
    src = torch.from_numpy(inv[g.req_ids]).cuda()
    out = {}

    def timed(fn):
        fn()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(reps):
            fn()
        b.record(stream)
        torch.cuda.synchronize()
        return a.elapsed_time(b) / reps

    for l in w.fwd_layers:
        buf = torch.empty(w.S, emb[l].shape[1], dtype=torch.float32, device="cuda")
        out["fwd%d_d%d" % (l, w.cfg.dims[l])] = timed(
            lambda: torch.index_select(emb[l], 0, src, out=buf))
        del buf
    for l in w.bwd_layers:
        e2 = eg[l].clone()
        out["bwd%d_d%d" % (l, w.cfg.dims[l])] = timed(lambda: e2.index_add_(0, src, hg[l]))
        del e2
    return {"ms_per_layer": out, "ops": "torch.index_select (forward), torch.index_add_ "
            "(backward, atomic)", "note": "stock PyTorch on the same B200, same layouts"}


def per_rank_loopback(w, emb, hg, eg, stream, topo, reps=10):
    """Context for the multi-GPU path: the same plan run as one launch per virtual rank on its own
    stream (DGCL_LOOPBACK_PER_RANK) — every rank's program with the ready handshake, done counters
    and completion waits of the multi-GPU protocol, sharing this GPU's SMs (each launch gets
    1/m of them) — against the fused launch the bench times.  Per-launch ms, mean of `reps`."""
    import torch
    import paper_conf_eurosys_cai0wmcy21_b200 as D
    c = w.cfg
    ctx = D.loopback(c.m, w.g.part, list(c.dims), device=0, flags=D.LOOPBACK_PER_RANK)
    ctx.build_plan(w.g.req_ptr, w.g.req_ids, seed=0, topology=topo)
    ctx.register_workspace()
    out = {}

    def timed(fn):
        for _ in range(2):
            fn()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(reps):
            fn()
        b.record(stream)
        torch.cuda.synchronize()
        return a.elapsed_time(b) / reps

    for l in w.fwd_layers:
        out["fwd%d_d%d" % (l, c.dims[l])] = timed(lambda: ctx.forward(l, emb[l], stream=stream))
    for l in w.bwd_layers:
        e2 = eg[l].clone()
        out["bwd%d_d%d" % (l, c.dims[l])] = timed(lambda: ctx.backward(l, hg[l], e2, stream=stream))
    ctx.check()
    ctx.destroy()
    return {"ms_per_layer": out, "note": "one launch per virtual rank on its own stream with the "
            "multi-GPU flag protocol (ready / done / completion waits), on one GPU; context, not "
            "the bench value"}


def run_ours_single(args, w):
    import torch
    import paper_conf_eurosys_cai0wmcy21_b200 as D
    torch.cuda.set_device(0)
    c = w.cfg
    g = w.g
    topo = None
    if c.topology != "uniform_nvswitch":
        import synth
        topo = synth.topology.by_name(c.topology, c.m)
    ctx = D.loopback(c.m, g.part, list(c.dims), device=0)
    if args.item_bytes:
        ctx.set_option("item_bytes", args.item_bytes)
    opts = {}
    for kv in args.opt:  # executor options (dgcl_set_option), for A/B runs
        k, v = kv.split("=")
        ctx.set_option(k, int(v))
        opts[k] = int(v)
    t = time.time()
    ctx.build_plan(g.req_ptr, g.req_ids, seed=0, topology=topo)
    plan_s = time.time() - t
    ctx.register_workspace()
    info = ctx.plan_info()
    pitches = {l: ctx.pitch(l) for l in range(len(c.dims))}
    emb_h, hg_h, eg_h = host_inputs(w, pitches)
    emb = {l: torch.from_numpy(a).cuda() for l, a in emb_h.items()}
    hg = {l: torch.from_numpy(a).cuda() for l, a in hg_h.items()}
    eg = {l: torch.from_numpy(a).cuda() for l, a in eg_h.items()}
    stream = torch.cuda.current_stream()
    names = ["fwd%d_d%d" % (l, c.dims[l]) for l in w.fwd_layers] + \
            ["bwd%d_d%d" % (l, c.dims[l]) for l in w.bwd_layers]

    def step(evs=None):
        i = 0
        for l in w.fwd_layers:
            if evs is not None:
                evs[i][0].record(stream)
            ctx.forward(l, emb[l], stream=stream)
            if evs is not None:
                evs[i][1].record(stream)
            i += 1
        for l in w.bwd_layers:
            if evs is not None:
                evs[i][0].record(stream)
            ctx.backward(l, hg[l], eg[l], stream=stream)
            if evs is not None:
                evs[i][1].record(stream)
            i += 1

    clk = ClockSampler(torch.cuda.current_device())
    clk.start()
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    # keep the GPU under load for >= 1 s before timing (clock sampling, steady state)
    t_soak = time.time()
    while time.time() - t_soak < 1.0:
        step()
        torch.cuda.synchronize()
    ctx.check()
    K = args.steps
    evs = [[[torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)]
            for _ in names] for _ in range(K)]
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    # per-launch durations: K steps with an event pair around every launch; then the step
    # itself: K steps back to back with events only at the two ends (an event between two
    # launches delays the second one's start by a few us, ~1 % of a step)
    torch.cuda.synchronize()
    tw0 = time.time()
    for k in range(K):
        step(evs[k])
    torch.cuda.synchronize()
    launches0 = ctx.launch_count()
    e0.record(stream)
    for k in range(K):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    tw1 = time.time()
    launches = ctx.launch_count() - launches0
    ctx.check()
    total_ms = e0.elapsed_time(e1)
    ms_step = total_ms / K
    per_op = {n: statistics.mean(evs[k][i][0].elapsed_time(evs[k][i][1]) for k in range(K))
              for i, n in enumerate(names)}
    clocks = clk.summary(tw0, tw1)
    if clocks["samples"] == 0:
        clocks = clk.summary()

    # ---- e2e through the host-buffer C-ABI calls (pinned host memory) ----
    e2e = None
    if args.e2e_steps > 0:
        pin = lambda a: torch.from_numpy(a).pin_memory()
        emb_p = {l: pin(a) for l, a in emb_h.items()}
        hg_p = {l: pin(a) for l, a in hg_h.items()}
        eg_p = {l: pin(a) for l, a in eg_h.items()}
        halo_p = {l: torch.empty(w.S, pitches[l], dtype=torch.float32).pin_memory()
                  for l in w.fwd_layers}
        h2d = sum(a.numel() * 4 for a in emb_p.values()) + \
            sum(a.numel() * 4 for a in hg_p.values()) + sum(a.numel() * 4 for a in eg_p.values())
        d2h = sum(a.numel() * 4 for a in halo_p.values()) + sum(a.numel() * 4 for a in eg_p.values())

        # pipelined host calls: each call's input copy overlaps the previous call's output copy
        # (host_async); the step ends when the stream is synchronized (the timed events below)
        ctx.set_option("host_async", 1)

        def e2e_step():
            for l in w.fwd_layers:
                ctx.forward_host(l, emb_p[l], halo_p[l], stream=stream)
            for l in w.bwd_layers:
                ctx.backward_host(l, hg_p[l], eg_p[l], stream=stream)

        e2e_step()
        torch.cuda.synchronize()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        for _ in range(args.e2e_steps):
            e2e_step()
        a1.record(stream)
        torch.cuda.synchronize()
        e2e_ms = a0.elapsed_time(a1) / args.e2e_steps
        e2e = {"value": w.step_payload_bytes() / (e2e_ms * 1e-3) / 1e9, "unit": UNIT,
               "ms_per_step": e2e_ms, "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h)}
    clk.stop()

    # ---- roofline: every launch is HBM-bound in loopback.  Algorithmic bytes = the minimum DRAM
    # traffic of the operation: forward reads each sent source row once and writes every halo
    # row (S rows); the backward (in-place reduce) reads every halo-gradient row and
    # read-modify-writes every owner row that has requesters.
    peaks, src = measured_peaks()
    nv = info["n_vertices_planned"]
    # relay plans (several stages) must move more than the direct minimum: every tree edge writes
    # a row and every forwarding GPU re-reads the row it forwards; the staged backward
    # (direct_reduce = 0) pushes one partial-sum row per tree edge into a slot that the parent
    # reads back.  Reported next to the direct minimum as plan_algorithmic_bytes / plan_frac.
    # (The default loopback backward of a relay plan folds each owner row's tree in one pass:
    # its bytes are the direct minimum.)
    plan_rows = None
    if info["n_stages"] > 1:
        E = ctx.plan_export()                       # (u, parent, child, stage)
        owner = g.part[E[:, 0]]
        fwd_pairs = np.unique(E[E[:, 1] != owner][:, [0, 1]], axis=0).shape[0]
        ne = int(info["n_tree_edges"])
        staged_bwd = opts.get("direct_reduce", 1) == 0
        plan_rows = {"fwd": nv + fwd_pairs + ne,
                     "bwd": w.S + 2 * ne + 2 * nv if staged_bwd else w.S + 2 * nv}
    kernels = {}
    for i, n in enumerate(names):
        l = (w.fwd_layers + w.bwd_layers)[i]
        row = c.dims[l] * 4
        if n.startswith("fwd"):
            alg = (nv + w.S) * row
        else:
            alg = (w.S + 2 * nv) * row
        ach = alg / (per_op[n] * 1e-3) / 1e9
        # SURVEY §8(d)'s loopback formula, HBM r+w = 2 x deliveries x row (every delivery read
        # AND written), reported beside it: it counts a row sent to k receivers as k DRAM reads,
        # which L2 serves after the first (R20), so its "fraction" can exceed 1
        survey = 2 * w.S * row
        kernels[n] = {"ms": per_op[n], "algorithmic_bytes": int(alg), "achieved_gbs": ach,
                      "frac": ach / peaks["hbm_gbs"],
                      "survey_formula_bytes": int(survey),
                      "survey_formula_frac": survey / (per_op[n] * 1e-3) / 1e9 / peaks["hbm_gbs"],
                      "traffic": profiled_traffic("%s/%s" % (c.name, n))}
        if plan_rows is not None:
            pb = plan_rows["fwd" if n.startswith("fwd") else "bwd"] * row
            kernels[n]["plan_algorithmic_bytes"] = int(pb)
            kernels[n]["plan_frac"] = pb / (per_op[n] * 1e-3) / 1e9 / peaks["hbm_gbs"]
    dom = max(names, key=lambda n: per_op[n])
    roofline = {"bound": "hbm", "kernel": "executor_tma_kernel (%s)" % dom,
                "achieved": kernels[dom]["achieved_gbs"], "peak": peaks["hbm_gbs"],
                "unit": "GB/s", "frac": kernels[dom]["frac"], "traffic": kernels[dom]["traffic"],
                "algorithmic_bytes_per_launch": kernels[dom]["algorithmic_bytes"],
                "algorithmic_bytes_definition": "compulsory DRAM bytes (DESIGN.md R20): unique "
                                                "source rows read once + every destination row "
                                                "written once (backward: halo-gradient rows read "
                                                "+ owner rows with requesters read and written)",
                "survey_formula_frac": kernels[dom]["survey_formula_frac"],
                "peak_source": src + " (MEASURED_PEAKS.json hbm_gbs: copy read+write)",
                "per_kernel": kernels}

    value = w.step_payload_bytes() / (ms_step * 1e-3) / 1e9
    torch_base = None if args.no_torch_baseline else torch_gather_baseline(w, emb, hg, eg, stream)
    per_rank = None if args.no_per_rank else per_rank_loopback(w, emb, hg, eg, stream, topo)
    cpu = None
    if not args.no_cpu_baseline:
        gbs, secs, used, thr = oracle_sample(w, emb_h, hg_h, eg_h, budget_s=args.cpu_budget)
        cpu = {"value": gbs, "unit": UNIT, "cores": thr, "kind": "oracle",
               "sample": "oracle forward (all layers) + flat backward for destination/owner "
                         "ranks %s of %d (%.1f s of CPU work)" % (used, c.m, secs)}
        ncores = len(os.sched_getaffinity(0))
        if ncores > 1 and not args.no_cpu_threads:
            gbs_t, secs_t, used_t, thr_t = oracle_sample(w, emb_h, hg_h, eg_h, ranks=range(c.m),
                                                         threads=ncores)
            cpu["threaded"] = {"value": gbs_t, "unit": UNIT, "cores": thr_t,
                               "host_cores": ncores,
                               "sample": "all %d ranks' oracle work as (rank, row-chunk) units on "
                                         "%d threads (%.1f s wall)" % (c.m, thr_t, secs_t)}
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 1, "steps": K,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "impl": "ours",
        "config": {"workload": "%s-shaped R-MAT, %d-way partition, 1-GPU loopback (all %d "
                               "virtual ranks on one B200)" % (c.name, c.m, c.m),
                   "config": c.name, "n_vertices": c.n, "n_edges": c.e, "world": c.m,
                   "dims": list(c.dims), "fwd_layers": w.fwd_layers, "bwd_layers": w.bwd_layers,
                   "halo_rows_total": w.S, "halo_rows_per_rank": np.diff(g.req_ptr).tolist(),
                   "topology": c.topology, "parallelism": "loopback%d" % c.m,
                   "options": opts,
                   "backward": ("staged reversed plan (slots, stage by stage)"
                                if opts.get("direct_reduce", 1) == 0 or c.m < 2 else
                                "tree-order fold per owner row, one pass (loopback)"
                                if info["n_stages"] > 1 else "fixed-order fold per owner row"),
                   "l2": "inputs larger than L2 (no flush needed)"},
        "ms_per_layer": per_op,
        "gbs_per_gpu": value,
        "roofline": roofline,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": int(launches),
        "clocks": clocks,
        "plan": dict(info, planner_wall_s=plan_s, graph_gen_s=w.gen_s),
        "torch_gather_baseline": torch_base,
        "per_rank_loopback": per_rank,
    }
    ctx.destroy()
    return out


def run_reference(args, w):
    """The reference arm of this tier: the CPU oracle as it stands, timed per step on a bounded
    sample of the same workload (one destination/owner rank per step)."""
    import synth
    c = w.cfg
    pitches = {l: synth.configs.pitch_of(c.dims[l]) for l in range(len(c.dims))}
    emb_h, hg_h, eg_h = host_inputs(w, pitches)
    for k in range(args.warmup):
        oracle_sample(w, emb_h, hg_h, eg_h, budget_s=0.0, ranks=[k % c.m])
    vals, secs = [], []
    for k in range(args.steps):
        gbs, s, used, thr = oracle_sample(w, emb_h, hg_h, eg_h, budget_s=0.0, ranks=[k % c.m])
        vals.append(gbs)
        secs.append(s)
    value = sum(vals) / len(vals)
    ms = 1e3 * sum(secs) / len(secs)
    return {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 0, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": "%s-shaped R-MAT, %d-way partition; CPU oracle, one rank's "
                                   "halo + owner rows per step" % (c.name, c.m), "config": c.name},
            "cpu_baseline": {"value": value, "unit": UNIT, "kind": "oracle", "cores": 1,
                             "sample": "one destination/owner rank of %d per step" % c.m},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}


def spawn_ranks(args):
    """`bench.py --gpus N` outside torchrun: start N ranks (one process per GPU) through
    torch.distributed.run on 127.0.0.1 with the same arguments; rank 0's JSON line is the
    output.  Refuses to run with fewer visible GPUs than N (unless --share-gpu, test mode)."""
    import socket
    import torch
    n_dev = torch.cuda.device_count()
    if n_dev < args.gpus and not args.share_gpu:
        log("bench.py: --gpus %d but only %d CUDA device(s) visible" % (args.gpus, n_dev))
        return 2
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           "--nproc-per-node", str(args.gpus), "--master-addr", "127.0.0.1",
           "--master-port", str(port), os.path.join(ROOT, "bench.py")] + sys.argv[1:]
    subprocess.check_call(["make", "-s", "-C", ROOT, "all"])
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="reddit")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-torch-baseline", action="store_true")
    ap.add_argument("--no-per-rank", action="store_true",
                    help="N = 1: skip the per-rank loopback context measurement")
    ap.add_argument("--cpu-budget", type=float, default=12.0)
    ap.add_argument("--no-cpu-threads", action="store_true")
    ap.add_argument("--item-bytes", type=int, default=0)
    ap.add_argument("--opt", action="append", default=[], metavar="KEY=VALUE",
                    help="executor option (dgcl_set_option) before planning, e.g. stage_fold=0")
    ap.add_argument("--calls", type=int, default=50,
                    help="N > 1: timed calls per launch in the per-call protocol (device start "
                         "barrier, max over ranks, median / p10 / p90 / mean of the first 10)")
    ap.add_argument("--no-p2p-baseline", action="store_true",
                    help="N > 1: skip the NCCL pack + send/recv + unpack baseline")
    ap.add_argument("--share-gpu", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "ours":
        sys.exit(spawn_ranks(args))
    if args.impl == "ours" and world != args.gpus and "WORLD_SIZE" in os.environ:
        raise SystemExit("bench.py: --gpus %d but WORLD_SIZE=%d" % (args.gpus, world))
    subprocess.check_call(["make", "-s", "-C", ROOT, "all"]) if rank == 0 and world == 1 else None

    if args.impl == "reference":
        if rank != 0:
            return
        w = Workload(args.config)
        print(json.dumps(run_reference(args, w)), flush=True)
        return

    if world == 1:
        w = Workload(args.config)
        out = run_ours_single(args, w)
        print(json.dumps(out), flush=True)
        return

    from bench_multi import run_multi
    out = run_multi(args, METRIC, UNIT, rank, world, local_rank, ClockSampler,
                    make_workload=Workload.from_parts, oracle_sample=oracle_sample,
                    host_inputs=host_inputs)
    if rank == 0:
        print(json.dumps(out), flush=True)
    import torch.distributed as dist
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
