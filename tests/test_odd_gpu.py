"""Odd innermost extents under a broadcast (round-2 cliff fix): no vector
width divides E[d_v] and a broadcast along d_v (bias[c]) keeps (c, r) from
collapsing, so the kernel flattens (c, r) into one loop of full-width vectors
and reads the broadcast access per element at c = flat index mod E[c]
(§V: vector and scalar accesses mixed in one statement).
Bit-exact against the oracle, aligned and misaligned, plus per-channel
BatchNorm on NHWC with an odd channel count (the scale/shift cone tabulated
over c and looked up per element)."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import oracle as O

from harness import assert_bitexact, run_gpu

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)


@pytest.mark.parametrize("R,C,dtype", [(1000, 1001, "f16"), (333, 13, "f32"), (64, 1001, "bf16"), (7, 9, "f16"),
                                       (5, 3, "f16"), (4099, 255, "f16")])
@pytest.mark.parametrize("offset", [0, 1])
def test_bias_add_over_odd_rows(R, C, dtype, offset):
    d = W.bias_add_rows(R, C, dtype)
    d["tensors"]["x"]["init"] = ("special", 63)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x, offset=offset)
    li = op.info()["launches"][0]
    if offset == 0 and C >= 8:
        assert li["width"] >= 4 and "PC_0" in op.source(), li      # flattened, full-width vectors
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


@pytest.mark.parametrize("dims", [(2, 7, 9, 255), (3, 5, 5, 13), (1, 4, 4, 1001)])
def test_nhwc_bn_odd_channels(dims):
    d = W.cfg2_nhwc(*dims)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert_bitexact(got["y"], O.run(d, x)["y"], "y")


def test_bias_add_full_size_every_candidate():
    """[65536, 1001] f16 (a 1001-class classifier's logits over 65536 tokens), every tuning candidate."""
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    from harness import device_tensors, to_host
    d = W.bias_add_rows(65536, 1001, "f16")
    x = W.make_inputs(d)
    ref = O.run(d, x)["out"]
    nv = FusedOp(d).info()["launches"][0]["nvariants"]
    for k in range(nv):
        op = FusedOp(d, variant=k)
        dev = device_tensors(d, x)
        op.run(dev)
        torch.cuda.synchronize()
        assert_bitexact(to_host(dev["out"], "f16"), ref, f"candidate {k} {op.selected(0)[0]}")
