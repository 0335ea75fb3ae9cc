"""Seeded synthetic inputs for the fused operators (no method arithmetic).

Every tensor is materialised as a flat 1-D numpy buffer covering its strided
span (``tensor_span``); descriptors carry the strides.  fp16 buffers are
``np.float16``; bf16 buffers are ``np.uint16`` bit patterns (numpy has no
bfloat16); i32 buffers are ``np.int32``.

Recipes (``tensor["init"]``), each drawn with ``numpy.random.default_rng``:
  ("uniform", lo, hi, seed)   U[lo, hi)
  ("normal", mu, sigma, seed) N(mu, sigma^2)
  ("randint", lo, hi, seed)   integers in [lo, hi) (exact in every dtype used)
  ("ones",) / ("const", v)    constant fill (closed-form pins)
  ("arange", start, step)     start + step * flat_index
  ("special", seed)           uniform U[-4,4) salted with +-0, subnormals,
                              +-inf, NaN and near-overflow values (bit tests)
Values are drawn in float32 and rounded to the tensor dtype (RNE).
"""

import numpy as np
import torch

NP_DTYPE = {"f32": np.float32, "f16": np.float16, "bf16": np.uint16, "i32": np.int32}


def contiguous_strides(shape):
    st, acc = [], 1
    for s in reversed(shape):
        st.append(acc)
        acc *= s
    return list(reversed(st))


def tensor_strides(t):
    return list(t["strides"]) if t.get("strides") else contiguous_strides(t["shape"])


def tensor_span(t):
    """Number of elements the flat buffer of tensor ``t`` must hold."""
    shape, st = t["shape"], tensor_strides(t)
    if any(s == 0 for s in shape):
        return 0
    return 1 + sum((s - 1) * abs(k) for s, k in zip(shape, st))


def _to_dtype(vals_f32, dtype):
    if dtype == "f32":
        return vals_f32.astype(np.float32)
    if dtype == "f16":
        return vals_f32.astype(np.float16)
    if dtype == "bf16":
        return torch.from_numpy(np.ascontiguousarray(vals_f32, dtype=np.float32)) \
            .to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    if dtype == "i32":
        return vals_f32.astype(np.int32)
    raise ValueError(dtype)


def draw(init, n, dtype, seed_offset=0):
    kind = init[0]
    if kind == "uniform":
        rng = np.random.default_rng(init[3] + seed_offset)
        v = rng.uniform(init[1], init[2], n).astype(np.float32)
    elif kind == "normal":
        rng = np.random.default_rng(init[3] + seed_offset)
        v = rng.standard_normal(n, dtype=np.float32) * np.float32(init[2]) + np.float32(init[1])
    elif kind == "randint":
        rng = np.random.default_rng(init[3] + seed_offset)
        v = rng.integers(init[1], init[2], n).astype(np.float32)
    elif kind == "ones":
        v = np.ones(n, np.float32)
    elif kind == "const":
        v = np.full(n, init[1], np.float32)
    elif kind == "arange":
        v = (np.float32(init[1]) + np.float32(init[2]) * np.arange(n, dtype=np.float64)).astype(np.float32)
    elif kind == "special":
        rng = np.random.default_rng(init[1] + seed_offset)
        v = rng.uniform(-4.0, 4.0, n).astype(np.float32)
        specials = np.array([0.0, -0.0, np.inf, -np.inf, np.nan, 1e-6, -1e-6, 6e-8, -6e-8,
                             65504.0, -65504.0, 65519.0, 70000.0, 1e-30, 3.0e38],
                            dtype=np.float32)
        idx = rng.integers(0, n, max(1, n // 16))
        v[idx] = specials[rng.integers(0, len(specials), len(idx))]
    else:
        raise ValueError(f"unknown init recipe {init!r}")
    return _to_dtype(v, dtype)


def make_inputs(desc, seed_offset=0):
    """Flat buffers for every IN / INOUT tensor, keyed by tensor name."""
    out = {}
    for name, t in desc["tensors"].items():
        if t["role"] in ("in", "inout"):
            init = t.get("init") or ("uniform", -1.0, 1.0, 0)
            out[name] = draw(init, tensor_span(t), t["dtype"], seed_offset)
    return out


def alloc_outputs(desc, fill_nan=True):
    """Flat buffers for OUT tensors, pre-filled with a NaN / 0xFF pattern so
    that an element nobody writes cannot pass a comparison."""
    out = {}
    for name, t in desc["tensors"].items():
        if t["role"] == "out":
            n = tensor_span(t)
            dt = NP_DTYPE[t["dtype"]]
            if fill_nan:
                buf = np.full(n * np.dtype(dt).itemsize, 0xFF, np.uint8).view(dt)
            else:
                buf = np.zeros(n, dt)
            out[name] = buf
    return out
