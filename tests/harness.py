"""Shared helpers for the tests: run the product (CUDA path through the C ABI)
and the oracle on the same seeded inputs, and compare with the tolerances of
BASELINE.json's north_star."""
import numpy as np
import torch

import workloads as W

TORCH_DT = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16, "i32": torch.int32}


def to_device(buf, dtype, device="cuda"):
    if dtype == "bf16":
        return torch.from_numpy(np.ascontiguousarray(buf).view(np.int16)).to(device).view(torch.bfloat16)
    return torch.from_numpy(np.ascontiguousarray(buf)).to(device)


def to_host(t, dtype):
    if dtype == "bf16":
        return t.view(torch.int16).cpu().numpy().view(np.uint16)
    return t.cpu().numpy()


def device_tensors(desc, inputs, device="cuda", offset=0):
    """Device buffers for all non-TEMP tensors; outputs NaN-filled.
    offset > 0 shifts every base pointer by `offset` elements (misalignment tests)."""
    outs = W.alloc_outputs(desc)
    dev = {}
    for n, t in desc["tensors"].items():
        if t["role"] == "temp":
            continue
        buf = inputs[n] if t["role"] in ("in", "inout") else outs[n]
        if offset:
            pad = np.zeros(offset, buf.dtype)
            full = to_device(np.concatenate([pad, buf]), t["dtype"], device)
            dev[n] = full[offset:]
        else:
            dev[n] = to_device(buf, t["dtype"], device)
    return dev


def run_gpu(desc, inputs, offset=0, **opts):
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    op = FusedOp(desc, **opts)
    dev = device_tensors(desc, inputs, offset=offset)
    op.run(dev)
    torch.cuda.synchronize()
    res = {n: to_host(dev[n], desc["tensors"][n]["dtype"]) for n, t in desc["tensors"].items()
           if t["role"] in ("out", "inout")}
    return res, op


def ordered16(h):
    i = h.view(np.uint16).astype(np.int32)
    return np.where(i & 0x8000, -(i & 0x7FFF), i)


def ordered32(f):
    i = f.view(np.int32).astype(np.int64)
    return np.where(i < 0, -(i & 0x7FFFFFFF), i)


def _isnan(a):
    """NaN mask; uint16 arrays hold raw bf16 bit patterns."""
    if a.dtype == np.uint16:
        return ((a & 0x7F80) == 0x7F80) & ((a & 0x007F) != 0)
    return np.isnan(a.astype(np.float32))


def assert_bitexact(got, ref, name=""):
    got, ref = np.asarray(got), np.asarray(ref)
    assert got.shape == ref.shape, (name, got.shape, ref.shape)
    if got.dtype.kind == "f" or got.dtype == np.uint16:
        view = np.uint16 if got.itemsize == 2 else np.uint32
        same = (got.view(view) == ref.view(view)) | (_isnan(got) & _isnan(ref))
    else:
        same = got == ref
    bad = np.flatnonzero(~same)
    assert bad.size == 0, f"{name}: {bad.size} of {got.size} differ, first at {bad[:5]}: " \
                          f"got {got.reshape(-1)[bad[:5]]} ref {ref.reshape(-1)[bad[:5]]}"


def assert_ulp(got, ref, max_ulp, name=""):
    """fp16/bf16/fp32 outputs within max_ulp (NaN == NaN)."""
    got, ref = np.asarray(got), np.asarray(ref)
    if got.dtype in (np.float16, np.uint16):   # f16, or raw bf16 bit patterns (same ordering)
        d = np.abs(ordered16(got) - ordered16(ref))
    else:
        d = np.abs(ordered32(got.astype(np.float32)) - ordered32(ref.astype(np.float32)))
    nan = _isnan(got) & _isnan(ref)
    d = np.where(nan, 0, d)
    assert d.max(initial=0) <= max_ulp, f"{name}: max {d.max()} ulp at {np.argmax(d)} " \
                                        f"(got {got.reshape(-1)[np.argmax(d)]}, ref {ref.reshape(-1)[np.argmax(d)]})"
    return int(d.max(initial=0))


def abs_terms_desc(desc, stmt_index):
    """Same operator, with |term| in the reduce statement: the oracle then
    returns fin(sum |term|) — the normwise error scale (reading R16)."""
    import copy
    d = copy.deepcopy(desc)
    s = d["stmts"][stmt_index]
    n = len(s["expr"])
    s["expr"] = list(s["expr"]) + [("abs", n - 1)]
    return d


def assert_normwise(got, ref, scale, tol, name=""):
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    scale = np.asarray(scale, np.float64)
    # non-finite results must match exactly (NaN where the oracle has NaN, the same infinities);
    # a NaN would otherwise pass every `err > bound` test
    nf = ~np.isfinite(ref) | ~np.isfinite(got)
    same_nf = (np.isnan(got) & np.isnan(ref)) | (got == ref)
    bad_nf = np.flatnonzero(nf & ~same_nf)
    assert bad_nf.size == 0, f"{name}: non-finite mismatch at {bad_nf[:5]}: got {got.reshape(-1)[bad_nf[:5]]} " \
                             f"ref {ref.reshape(-1)[bad_nf[:5]]}"
    got, ref, scale = np.where(nf, 0, got), np.where(nf, 0, ref), np.where(nf, 0, scale)
    err = np.abs(got - ref)
    bound = tol * np.maximum(scale, np.finfo(np.float32).tiny)
    bad = np.flatnonzero(err > bound)
    assert bad.size == 0, f"{name}: {bad.size} exceed tol*sum|t| (worst ratio " \
                          f"{(err / bound).max():.3g}) first {bad[:5]}"
    return float((err / np.maximum(scale, 1e-30)).max(initial=0))


def check_rowstats(d, x, got, ulp_y=1):
    """cfg4a-shaped operators (y = f16(gelu(x + b)), mean/var over y): y within
    `ulp_y` of the oracle; the statistics against the oracle run on the GPU's
    OWN y (isolates the reduction from y's last-bit rounding: R16's 1e-5
    normwise bound) and end to end against the oracle (2e-3 for fp16 data)."""
    import copy
    from oracle import oracle as O
    ref = O.run(d, x)
    assert_ulp(got["y"], ref["y"], ulp_y, "y")
    d2 = copy.deepcopy(d)
    d2["tensors"]["y"]["role"] = "in"
    xin = dict(x)
    xin["y"] = got["y"]
    ref2 = O.run(d2, xin, stmts=[1, 2])
    for si, name in [(1, "mean"), (2, "var")]:
        scale = O.run(abs_terms_desc(d2, si), xin, stmts=[1, 2])[name]
        assert_normwise(got[name], ref2[name], scale, 1e-5, name)
        assert_normwise(got[name], ref[name], O.run(abs_terms_desc(d, si), x)[name], 2e-3, name)
