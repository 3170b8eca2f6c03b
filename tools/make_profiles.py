#!/usr/bin/env python3
"""Write profiles/<tag>_ncu_summary.md, profiles/<tag>_launches.csv summary and profiles/traffic.json
from an ncu --set full report and an ncu launch list (gpurun_out/)."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return [{h: (r[i], units[i]) for i, h in enumerate(hdr)} for r in rows[2:]]


def val(d, k, scale=1.0):
    v, u = d[k]
    v = float(v.replace(",", ""))
    mult = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "ms": 1e-3, "us": 1e-6,
            "ns": 1e-9, "s": 1.0}.get(u, 1.0)
    return v * mult * scale


def main(tag, names, config="reddit"):
    rep = os.path.join(ROOT, "gpurun_out", "%s_prof.ncu-rep" % tag)
    launches = raw(rep)
    lines = ["# ncu --set full summary (%s)" % tag, "",
             "Command: `ncu --set full --clock-control none --import-source on -k regex:executor "
             "-c 3 python bench.py --config %s --steps 1 --warmup 3` (tools/ncu_bench.sh).  "
             "Per-launch times are cold-cache and serialised under replay." % config, "",
             "| launch | kernel | time | DRAM read | DRAM write | DRAM % of peak | regs | smem/CTA |",
             "|---|---|---|---|---|---|---|---|"]
    traffic = {}
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        traffic = json.load(open(p))
    for n, d in zip(names, launches):
        rd = val(d, "dram__bytes_read.sum")
        wr = val(d, "dram__bytes_write.sum")
        t = val(d, "gpu__time_duration.sum")
        lines.append("| %s | %s | %.1f us | %.3f GB | %.3f GB | %s %% | %s | %s %s |" % (
            n, d["Kernel Name"][0][:40], t * 1e6, rd / 1e9, wr / 1e9,
            d["gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"][0][:5],
            d["launch__registers_per_thread"][0],
            d["launch__shared_mem_per_block_dynamic"][0],
            d["launch__shared_mem_per_block_dynamic"][1]))
        traffic["%s/%s" % (config, n)] = int(rd + wr)
    lc = os.path.join(ROOT, "gpurun_out", "%s_launches.csv" % tag)
    if os.path.exists(lc):
        rows = list(csv.reader(open(lc)))
        h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        hdr = rows[h]
        ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
        ks = [(r[ki], float(r[vi].replace(",", ""))) for r in rows[h + 1:] if len(r) > vi]
        tot = sum(v for _, v in ks)
        by = {}
        for k, v in ks:
            short = k.split("(")[0][-60:]
            n, t = by.get(short, (0, 0.0))
            by[short] = (n + 1, t + v)
        lines += ["", "Launch list (`--metrics gpu__time_duration.sum`, whole process: input "
                  "generation, warm-up and timed steps): %d launches; executor launches = %.1f %% "
                  "of all GPU time (the other kernels are input fills and copies outside the "
                  "timed region; inside it only executor launches run, three per step)." % (
                      len(ks), 100.0 * sum(v for k, v in ks if "executor" in k) / max(tot, 1)),
                  "", "| kernel | launches | total us |", "|---|---|---|"]
        for short, (n, t) in sorted(by.items(), key=lambda x: -x[1][1]):
            lines.append("| `%s` | %d | %.1f |" % (short, n, t / 1e3))
        with open(os.path.join(ROOT, "profiles", "%s_launches.csv" % tag), "w") as f:
            f.write("kernel,gpu__time_duration_ns\n")
            for k, v in ks:
                f.write('"%s",%d\n' % (k, v))
    with open(os.path.join(ROOT, "profiles", "%s_ncu_summary.md" % tag), "w") as f:
        f.write("\n".join(lines) + "\n")
    with open(p, "w") as f:
        json.dump(traffic, f, indent=1, sort_keys=True)
    print("\n".join(lines))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2].split(","), *(sys.argv[3:4]))
