"""Summarise an ncu launch-list CSV of `bench.py` into markdown.

    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
        --clock-control none -c 600 --csv --log-file gpurun_out/launches.csv \
        python bench.py --steps 3 --warmup 3 --no-cpu
    python tools/launch_list.py gpurun_out/launches.csv profiles/ncu_launches_rNN.md "<command>"

Takes the last `--last` libfop launches (the steady-state passes after the
auto-tuner's candidate timings) and reports per kernel: launches, mean time,
share of the step, DRAM bytes per launch next to the algorithmic bytes.
ncu times are cold-cache and serialised: compare SHARES with bench.py's live
per-op times, not absolutes.
"""
import csv
import io
import os
import re
import sys
from collections import OrderedDict

ALG = {"ew": ("cfg2", 616563712), "transpose": ("cfg3", 822083584), "row_reduce": ("cfg4a", 100926976),
       "col_reduce": ("cfg4b", 134221824)}


def main():
    src, out = sys.argv[1], sys.argv[2]
    cmd = sys.argv[3] if len(sys.argv) > 3 else ""
    last = 32
    text = open(src).read()
    body = text[text.index('"ID"'):]
    rows = list(csv.DictReader(io.StringIO(body)))
    launches = OrderedDict()
    for r in rows:
        key = int(r["ID"])
        e = launches.setdefault(key, {"name": r["Kernel Name"]})
        e[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    fop = [v for v in launches.values() if v["name"].startswith("fop_")]
    tail = fop[-last:]
    agg = OrderedDict()
    for v in tail:
        a = agg.setdefault(v["name"], {"n": 0, "t": 0.0, "rd": 0.0, "wr": 0.0})
        a["n"] += 1
        a["t"] += v.get("gpu__time_duration.sum", 0.0)
        a["rd"] += v.get("dram__bytes_read.sum", 0.0)
        a["wr"] += v.get("dram__bytes_write.sum", 0.0)
    total = sum(a["t"] for a in agg.values())
    unit_us = 1e-3   # gpu__time_duration.sum is reported in ns by --csv
    lines = [f"# ncu launch list ({os.path.basename(src)})", "",
             f"Command: `{cmd}`" if cmd else "", "",
             f"{len(launches)} launches captured, {len(fop)} of them libfop kernels (the first are the auto-tuner's "
             "candidate timings, `_vN` = candidate N); the table covers the last "
             f"{len(tail)} libfop launches (steady-state suite passes, the geometry the tuner kept).",
             "ncu per-launch times are cold-cache and serialised, so compare SHARES with bench.py's live per-op "
             "times, not absolutes.", "",
             "| kernel (chosen variant) | op | launches | mean us (ncu) | share of step | DRAM read MB | DRAM write MB "
             "| alg MB |", "|---|---|---|---|---|---|---|---|"]
    for name, a in agg.items():
        cls = re.match(r"fop_(ew|transpose|row_reduce|col_reduce)", name)
        op, alg = ALG.get(cls.group(1) if cls else "", ("?", 0))
        n = a["n"]
        lines.append(f"| {name} | {op} | {n} | {a['t'] / n * unit_us:.1f} | {100 * a['t'] / total:.1f}% | "
                     f"{a['rd'] / n / 1e6:.1f} | {a['wr'] / n / 1e6:.1f} | {alg / 1e6:.1f} |")
    with open(out, "w") as fh:
        fh.write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
