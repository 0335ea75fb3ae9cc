"""Re-run one fuzz descriptor (a tests/fuzz_regressions/*.json file or one entry of a
gpurun_out/fuzz_fail_<seed>.json list) through the campaign's sequence — a first
(tuning) run, then aligned / misaligned / aligned re-runs of the same plan — printing
each run's base pointers, the launch the runtime selected and whether it matched the
oracle.  Run with FOP_DEBUG_RUN=1 FOP_TUNE_LOG=1 for the runtime's own trace.

    python tools/repro_fuzz.py tests/fuzz_regressions/tma_seed41_case273.json
    python tools/repro_fuzz.py gpurun_out/fuzz_fail_51.json 0
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import torch  # noqa: E402

import workloads as W  # noqa: E402
from harness import device_tensors, to_host  # noqa: E402
from oracle import oracle as O  # noqa: E402
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp  # noqa: E402


def main():
    d = json.load(open(sys.argv[1]))
    if isinstance(d, list):
        d = d[int(sys.argv[2]) if len(sys.argv) > 2 else 0]["desc"]
    x = W.make_inputs(d)
    ref = O.run(d, x, outputs=W.alloc_outputs(d))
    op = FusedOp(d)
    print(op.info()["launches"])
    for off in (0, 0, 1, 0, 1, 0):
        dev = device_tensors(d, x, offset=off)
        print("run offset", off, {n: hex(t.data_ptr()) for n, t in dev.items()}, flush=True)
        try:
            op.run(dev)
            torch.cuda.synchronize()
        except Exception as e:  # noqa: BLE001
            print("  FAIL", e, flush=True)
            continue
        for n, t in d["tensors"].items():
            if t["role"] in ("out", "inout"):
                got = to_host(dev[n], t["dtype"])
                same = (got.view("u1") == ref[n].view("u1")).all()
                print(f"  {n}: selected {op.selected(0)} {'bit-identical to the oracle' if same else 'DIFFERS'}",
                      flush=True)


if __name__ == "__main__":
    main()
