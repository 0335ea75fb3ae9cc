"""Summarise an `ncu --set full` report of libfop kernels into markdown + JSON.

    python tools/ncu_summary.py gpurun_out/prof_r01_v4.ncu-rep profiles/ncu_r01_summary.md

Also writes profiles/ncu_dram_bytes.json (DRAM read+write bytes per launch by
op), which bench.py reports as roofline.traffic.
"""
import csv
import io
import json
import os
import re
import subprocess
import sys

OPS = {"ew": ("cfg2", 616563712), "transpose": ("cfg3", 822083584), "row_reduce": ("cfg4a", 100926976),
       "col_reduce": ("cfg4b", 134221824)}
KEEP = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__bytes.sum.per_second",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "smsp__inst_executed.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum"]


def main():
    rep, out = sys.argv[1], sys.argv[2]
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, data = rows[0], rows[2:]
    res, traffic = {}, {}
    lines = [f"# ncu --set full summary ({os.path.basename(rep)})", "",
             "Command (gpurun, 1x B200): `ncu --set full --clock-control none --import-source on --profile-from-start off "
             "-k regex:fop_ -c 4 -o prof python tools/profile_ops.py --reps 1` — the kernels the auto-tuner kept, one "
             "launch each, cold L2 (ncu flushes), serialised.  DRAM write bytes exclude output still dirty in the 126 MB "
             "L2 when the kernel ends.", "",
             "| kernel | op | time us | DRAM rd MB | DRAM wr MB | alg MB | DRAM TB/s | dram % pk | regs | grid x block | warps act % | issue act % | FMA pipe % | XU pipe % | long-sb stall/issue |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for r in data:
        g = lambda m: r[hdr.index(m)] if m in hdr else ""  # noqa: E731
        k = g("Kernel Name")
        cls = re.match(r"fop_(ew|transpose|row_reduce|col_reduce)", k).group(1)
        op, alg = OPS[cls]
        res[op] = {"kernel": k, "alg_bytes": alg, **{m: g(m) for m in KEEP}}
        rd, wr = float(g("dram__bytes_read.sum")), float(g("dram__bytes_write.sum"))
        traffic[op] = (rd + wr) * 1e6
        f = lambda m: float(g(m) or 0)  # noqa: E731
        lines.append(f"| {k} | {op} | {f('gpu__time_duration.sum'):.1f} | {rd:.1f} | {wr:.1f} | {alg / 1e6:.1f} | "
                     f"{f('dram__bytes.sum.per_second'):.2f} | {f('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed'):.1f} | "
                     f"{g('launch__registers_per_thread')} | {g('launch__grid_size')} x {g('launch__block_size')} | "
                     f"{f('sm__warps_active.avg.pct_of_peak_sustained_active'):.1f} | {f('smsp__issue_active.avg.pct_of_peak_sustained_active'):.1f} | "
                     f"{f('sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active'):.1f} | {f('sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active'):.1f} | "
                     f"{f('smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio'):.2f} |")
    with open(out, "w") as fh:
        fh.write("\n".join(lines) + "\n")
    with open(os.path.splitext(out)[0] + ".json", "w") as fh:
        json.dump(res, fh, indent=1)
    with open(os.path.join(os.path.dirname(out), "ncu_dram_bytes.json"), "w") as fh:
        json.dump(traffic, fh, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
