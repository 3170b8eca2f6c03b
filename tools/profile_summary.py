#!/usr/bin/env python3
"""profiles/<tag>_ncu_<config>.md + profiles/traffic.json from tools/ncu_all.sh output.

Per captured executor launch (first warm-up step of `bench.py --config C`, one launch per
(layer, direction)): ncu time (cold, serialised), DRAM read / write bytes against the launch's
algorithmic bytes (bench line roofline.per_kernel), L2 read hit rate, SM issue activity, warps
active and the top stall reasons (per issued instruction)."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
UNIT = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "ms": 1e-3, "us": 1e-6,
        "ns": 1e-9, "s": 1.0, "msecond": 1e-3, "usecond": 1e-6, "nsecond": 1e-9}


def raw(rep):
    """Rows of the raw page: from the report (ncu -i), or from its saved CSV (<rep>.raw.csv)."""
    if os.path.exists(rep):
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                             text=True).stdout
        open(rep[:-len(".ncu-rep")] + ".raw.csv", "w").write(out)
    else:
        out = open(rep[:-len(".ncu-rep")] + ".raw.csv").read()
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return [{h: (r[i], units[i]) for i, h in enumerate(hdr)} for r in rows[2:]]


def num(d, k):
    if k not in d:
        return None
    v, u = d[k]
    try:
        return float(v.replace(",", "")) * UNIT.get(u, 1.0)
    except ValueError:
        return None


def summarize(tag, cfg):
    rep = os.path.join(ROOT, "gpurun_out", "%s_%s_prof.ncu-rep" % (tag, cfg))
    bj = os.path.join(ROOT, "gpurun_out", "%s_%s_bench.json" % (tag, cfg))
    csvp = rep[:-len(".ncu-rep")] + ".raw.csv"
    if not (os.path.exists(rep) or os.path.exists(csvp)) or not os.path.exists(bj):
        return None, {}
    bench = json.loads(open(bj).read().strip().splitlines()[-1])
    names = list(bench["ms_per_layer"])
    pk = bench["roofline"]["per_kernel"]
    L = raw(rep)
    rows, traffic = [], {}
    for n, d in zip(names, L):
        rd, wr = num(d, "dram__bytes_read.sum"), num(d, "dram__bytes_write.sum")
        t = num(d, "gpu__time_duration.sum")
        alg = pk[n]["algorithmic_bytes"]
        plan = pk[n].get("plan_algorithmic_bytes")
        stalls = sorted(((k.split("stalled_")[1].split("_per_issue")[0], num(d, k))
                         for k in d if k.startswith("smsp__average_warps_issue_stalled_") and
                         k.endswith("_per_issue_active.ratio") and num(d, k)),
                        key=lambda x: -x[1])[:4]
        traffic["%s/%s" % (cfg, n)] = int(rd + wr)
        rows.append("| %s | `%s` | %.1f | %.3f | %.3f | %.3f | %s | %.2f | %.1f | %.1f | %.1f | %s | %s |" % (
            n, d["Kernel Name"][0].split("executor_tma_kernel")[-1].split("(")[0][:14] or
            d["Kernel Name"][0][:24], t * 1e6, rd / 1e9, wr / 1e9, alg / 1e9,
            "%.3f" % (plan / 1e9) if plan else "-", (rd + wr) / alg,
            num(d, "lts__t_sector_op_read_hit_rate.pct") or 0,
            num(d, "sm__issue_active.avg.pct_of_peak_sustained_elapsed") or 0,
            num(d, "sm__warps_active.avg.pct_of_peak_sustained_active") or 0,
            ", ".join("%s %.2f" % s for s in stalls), d["launch__registers_per_thread"][0]))
    bench_ms = {n: round(v, 4) for n, v in bench["ms_per_layer"].items()}
    fr = {n: round(v["frac"], 3) for n, v in pk.items()}
    pfr = {n: round(v["plan_frac"], 3) for n, v in pk.items() if "plan_frac" in v}
    head = ["### %s (%d-way, dims %s, %d stage(s))" % (cfg, bench["config"]["world"],
                                                       bench["config"]["dims"],
                                                       bench["plan"]["n_stages"]), "",
            "bench (same box, warm, CUDA events): ms %s; HBM frac of the direct minimum %s%s" % (
                bench_ms, fr, ("; of the plan's bytes %s" % pfr) if pfr else ""), "",
            "| launch | instance | ncu us | DRAM rd GB | DRAM wr GB | alg GB | plan GB | DRAM/alg | "
            "L2 rd hit % | issue active % | warps active % | top stalls (per issue) | regs |",
            "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    return "\n".join(head + rows) + "\n", traffic


def main(tag, cfgs, outdir=None):
    outdir = outdir or os.path.join(ROOT, "profiles")
    out = ["# ncu --set full, every executor launch of one step (%s)" % tag, "",
           "`tools/ncu_all.sh`: `ncu --set full --clock-control none --import-source on -k "
           "regex:executor -c <launches per step> python bench.py --config C --steps 1 --warmup 3` "
           "(the first step's launches; cold-cache, serialised under replay: compare DRAM bytes "
           "and shares, not absolute times).  alg = the launch's algorithmic bytes "
           "(DESIGN.md §4: unique source rows read once + every destination row written once; "
           "backward: halo-gradient rows read + owner rows with requesters read and written); "
           "plan = the relay plan's own minimum (every tree edge written, forwarded rows read).", ""]
    tp = os.path.join(outdir, "traffic.json")
    if not os.path.exists(tp) and os.path.exists(os.path.join(ROOT, "profiles", "traffic.json")):
        tp0 = os.path.join(ROOT, "profiles", "traffic.json")
        json.dump(json.load(open(tp0)), open(tp, "w"))
    traffic = json.load(open(tp)) if os.path.exists(tp) else {}
    for c in cfgs:
        s, t = summarize(tag, c)
        if s:
            out.append(s)
            traffic.update(t)
    path = os.path.join(outdir, "%s_ncu_all_configs.md" % tag)
    open(path, "w").write("\n".join(out))
    json.dump(traffic, open(tp, "w"), indent=1, sort_keys=True)
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2].split(",") if len(sys.argv) > 2 and sys.argv[2] else
         "tiny,reddit,google2,google4,google8,orkut,google8_dgx1,google8_ring,reddit_dgx1".split(","),
         sys.argv[3] if len(sys.argv) > 3 else None)
