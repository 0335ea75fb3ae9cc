"""A plan run many times must give the same results every time, whatever
geometry the auto-tuner picked and when aligned and misaligned pointers
alternate (the narrow variant).  Regression: tuning variants and the narrow
variant of a COL_REDUCE shared the default's workspace region, so one
geometry's partial sums overwrote another's arrival counters and the
reduction stopped writing its output after tuning."""
import numpy as np
import pytest
import torch

import workloads as W
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp

CASES = {
    "cfg4b": lambda: W.cfg4b(8192, 1024),
    "cfg4b_ragged": lambda: W.cfg4b(3001, 1000),
    "cfg4a": lambda: W.cfg4a(4, 64, 768),
    "cfg2": lambda: W.cfg2(2, 64, 28, 28),
}


def test_variant_workspace_regions_disjoint_cpu():
    # the workspace grows with every tuned COL geometry (own region each)
    d = W.cfg4b(8192, 1024)
    plain = FusedOp(d, autotune=0).workspace_bytes
    tuned = FusedOp(d).workspace_bytes
    assert tuned > plain


@pytest.mark.gpu
@pytest.mark.parametrize("case", list(CASES))
def test_repeated_runs_identical(case):
    from oracle import oracle as O
    from harness import device_tensors, to_host, assert_normwise, abs_terms_desc, assert_bitexact
    d = CASES[case]()
    x = W.make_inputs(d)
    op = FusedOp(d)
    aligned = device_tensors(d, x)
    shifted = device_tensors(d, x, offset=1)
    outs = [n for n, t in d["tensors"].items() if t["role"] == "out"]
    first = None
    for k in range(6):
        dev = shifted if k % 3 == 2 else aligned
        for n in outs:
            dev[n].fill_(float("nan"))
        op.run(dev)
        torch.cuda.synchronize()
        got = {n: to_host(dev[n], d["tensors"][n]["dtype"]) for n in outs}
        for n in outs:
            assert not np.isnan(got[n].astype(np.float32)).any(), (k, n)
        if first is None:
            first = got
            ref = O.run(d, x)
            for si, s in enumerate(d["stmts"]):
                n = s["write"][0]
                if n not in outs:
                    continue
                if s["kind"] == "reduce":
                    assert_normwise(got[n], ref[n], O.run(abs_terms_desc(d, si), x)[n], 2e-3, n)
        elif dev is aligned:
            for n in outs:
                assert_bitexact(got[n], first[n], f"run {k} {n}")
