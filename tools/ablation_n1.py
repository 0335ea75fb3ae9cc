"""the paper's novec vs infl ablation on B200 (Table II).

"novec" = influenced schedule, coalescing only (no explicit vector types):
force_width=1, every access a scalar 2/4-byte LDG/STG across consecutive
threads.  "infl" = explicit vector types: widths 2, 4, 8 elements (16 B =
LDG/STG.128 for fp16) and 32 B (LDG/STG.256).  Same planner, same thread
order, same grid rules; only the vector width changes.

    python tools/ablation_n1.py > profiles/ablation_n1_r01.md

Timing as tools/sweep.py (rotating input copies > 3x L2, 5 batches of 40).
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from bench import to_device  # noqa: E402
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp  # noqa: E402

L2 = 126 << 20
VARIANTS = [("novec (W=1)", {"force_width": 1}), ("W=2", {"force_width": 2}), ("W=4", {"force_width": 4}),
            ("W=8 / 16 B (default)", {}), ("32 B vectors", {"max_vec_bytes": 32}),
            ("paper thread order", {"coalesce_order": "paper"})]


def time_op(op, sets):
    for i in range(5):
        op.run(sets[i % len(sets)])
    torch.cuda.synchronize()
    per = []
    for _ in range(5):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        for i in range(40):
            op.run(sets[i % len(sets)])
        e.record()
        torch.cuda.synchronize()
        per.append(s.elapsed_time(e) / 40)
    return statistics.median(per)


def main():
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    rows = {}
    for name in ("cfg2", "cfg3", "cfg4a", "cfg4b"):
        d = W.CONFIGS[name]()
        x = W.make_inputs(d)
        o = W.alloc_outputs(d, fill_nan=False)
        nb = W.algorithmic_bytes(d)
        copies = max(1, min(16, -(-3 * L2 // nb)))
        sets = [{n: to_device(x[n] if t["role"] in ("in", "inout") else o[n], t["dtype"], "cuda")
                 for n, t in d["tensors"].items() if t["role"] != "temp"} for _ in range(copies)]
        for label, opts in VARIANTS:
            op = FusedOp(d, **opts)
            ms = time_op(op, sets)
            li = op.info()["launches"][0]
            rows.setdefault(name, []).append((label, nb / ms / 1e6, li["width"], li.get("read_width", 0)))
            print(json.dumps({"op": name, "variant": label, "GBs": nb / ms / 1e6, "us": ms * 1e3,
                              "width": li["width"], "read_width": li["read_width"]}), file=sys.stderr, flush=True)
        del sets
        torch.cuda.empty_cache()
    print("# N1 ablation: explicit vector types vs coalescing only (novec), 1x B200\n")
    print("GB/s of algorithmic bytes; speedup = variant / novec (the paper's Table II infl/novec geomean is 1.09x")
    print(f"on V100, P:397-403).  Peak for the % column: {peak:.1f} GB/s (measured copy).\n")
    print("| op | " + " | ".join(v[0] for v in VARIANTS) + " |")
    print("|---|" + "---|" * len(VARIANTS))
    for name, r in rows.items():
        base = r[0][1]
        print(f"| {name} | " + " | ".join(f"{g:.0f} ({g / base:.2f}x, {100 * g / peak:.0f}%)" for _, g, _, _ in r) + " |")
    import math
    gm = lambda i: math.exp(sum(math.log(r[i][1] / r[0][1]) for r in rows.values()) / len(rows))  # noqa: E731
    print("\ngeomean speedup over novec: " + ", ".join(f"{VARIANTS[i][0]} {gm(i):.2f}x" for i in range(len(VARIANTS))))


if __name__ == "__main__":
    main()
