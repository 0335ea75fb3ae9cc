"""One-off fuzz campaign: N random operators (tests/fuzz_gen.py) on the GPU
against the oracle with the checks of tests/test_fuzz.py; failing
descriptors are written to gpurun_out/fuzz_fail_<seed>.json.

    python tools/fuzz_campaign.py --seed 1 --count 1000
"""
import argparse
import json
import os
import sys
import traceback

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402
from fuzz_gen import random_op  # noqa: E402
from harness import run_gpu, assert_bitexact, assert_ulp, assert_normwise, abs_terms_desc  # noqa: E402
from oracle import oracle as O  # noqa: E402


def check(d, repeat=False, variants=False):
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    ref = O.run(d, x, outputs=W.alloc_outputs(d))
    compare(d, x, got, ref)
    if variants:   # every auto-tuning candidate forced in turn (opts.variant), not only the tuner's pick
        nv = max(li["nvariants"] for li in op.info()["launches"])
        for k in range(1, nv):
            got, _ = run_gpu(d, x, variant=k)
            compare(d, x, got, ref)
    if repeat:   # the same plan again (tuned geometry), a misaligned run (narrow variant), aligned again
        import torch
        from harness import device_tensors, to_host
        for off in (0, 1, 0):
            dev = device_tensors(d, x, offset=off)
            op.run(dev)
            torch.cuda.synchronize()
            got = {n: to_host(dev[n], d["tensors"][n]["dtype"]) for n, t in d["tensors"].items()
                   if t["role"] in ("out", "inout")}
            compare(d, x, got, ref)
    return [li["class"] for li in op.info()["launches"]]


def compare(d, x, got, ref):
    for si, st in enumerate(d["stmts"]):
        n = st["write"][0]
        t = d["tensors"][n]
        if t["role"] != "out":
            continue
        from_sum = any(q["kind"] == "reduce" and q.get("op", "sum") == "sum" and
                       any(r[0] == q["write"][0] for r in st["reads"]) for q in d["stmts"][:si])
        if st["kind"] == "reduce" and st.get("op", "sum") == "sum" and t["dtype"] != "i32":   # (i32: exact)
            assert_normwise(got[n], ref[n], O.run(abs_terms_desc(d, si), x)[n], 1e-5, n)
        elif from_sum and t["dtype"] == "f32":
            g, r = got[n].astype(np.float64), ref[n].astype(np.float64)
            assert np.all((np.abs(g - r) <= 1e-5 * np.abs(r) + 1e-30) | (np.isnan(g) & np.isnan(r))), n
        elif t["dtype"] != "f32" and from_sum:   # (÷ is IEEE-exact in every form, fast 16-bit ones included)
            assert_ulp(got[n], ref[n], 1, n)
        else:
            assert_bitexact(got[n], ref[n], n)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--count", type=int, default=500)
    ap.add_argument("--repeat", action="store_true", help="also re-run each plan (aligned, misaligned, aligned)")
    ap.add_argument("--trace", action="store_true", help="print each case index before running it (crash triage)")
    ap.add_argument("--variants-every", type=int, default=0,
                    help="every N-th operator also runs each auto-tuning candidate forced (0: never)")
    a = ap.parse_args()
    rng = np.random.default_rng(a.seed)
    fails, classes = [], {}
    for i in range(a.count):
        d = random_op(rng)
        if a.trace:
            print("case", i, d["name"], flush=True)
        try:
            for c in check(d, a.repeat, a.variants_every > 0 and i % a.variants_every == 0):
                classes[c] = classes.get(c, 0) + 1
        except Exception as e:  # noqa: BLE001
            fails.append({"case": i, "error": f"{type(e).__name__}: {str(e)[:300]}", "desc": d,
                          "trace": traceback.format_exc()[-800:]})
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", f"fuzz_fail_{a.seed}.json"), "w") as fh:
        json.dump(fails, fh, indent=1, default=str)
    print(json.dumps({"seed": a.seed, "count": a.count, "failures": len(fails), "classes": classes}))
    for f in fails[:10]:
        print(f["case"], f["desc"]["name"], f["error"][:200])


if __name__ == "__main__":
    main()
