"""Random fused operators for the fuzz tests (descriptions only: no method
arithmetic here).  Shapes, layouts and DAGs are drawn from a seeded numpy
generator:

  * 1-4 loops, extents from a mix of powers of two, odd and ragged sizes;
  * every input indexes a random subset of the loops (broadcast along the
    rest) in a random dim order, f32/f16/bf16, contiguous or padded strides;
  * the output indexes all loops (ASSIGN) or the non-reduced ones (REDUCE)
    in a random dim order — transposes included;
  * expressions use ops whose GPU result is IEEE-exact (add, sub, mul, div,
    max, min, neg, abs, sqrt, relu, cast), so ASSIGN outputs compare bit for
    bit; REDUCE sums compare normwise (R16), max reductions bit for bit;
  * patterns: one ASSIGN, one REDUCE, a TEMP producer over a subset of the
    loops consumed by an ASSIGN (cfg2's shape), a row REDUCE whose value an
    ASSIGN over the same loops consumes (softmax/LayerNorm's shape), and an
    integer ASSIGN over i32 tensors (reading R30, bit-exact).
"""
import numpy as np

EXTENTS = [1, 2, 3, 5, 7, 8, 13, 16, 24, 31, 32, 33, 48, 64, 100, 128, 257]
DTYPES = ["f32", "f16", "bf16"]
EXACT_UNARY = ["neg", "abs", "relu", "sqrt"]
EXACT_BINARY = ["add", "sub", "mul", "div", "max", "min"]
INT_UNARY = ["neg", "abs", "relu"]                       # reading R30: integer statements
INT_BINARY = ["add", "sub", "mul", "max", "min"]


def _loops(rng, max_elems=120_000):
    while True:
        n = int(rng.integers(1, 5))
        ext = [int(rng.choice(EXTENTS)) for _ in range(n)]
        if np.prod(ext) <= max_elems and np.prod(ext) >= 2:
            return {f"l{i}": e for i, e in enumerate(ext)}


def _tensor(rng, loops, names, dtype, role, seed, pad=True):
    """Tensor over `names` (dim order as given) with optional padded strides."""
    shape = [loops[n] for n in names]
    strides = None
    if pad and names and rng.random() < 0.35:
        st, acc = [], 1
        for s in reversed(shape):
            st.append(acc)
            acc *= s + int(rng.integers(0, 3))
        strides = list(reversed(st))
    init = ("normal", 0.0, 1.0, seed) if role in ("in", "inout") else None
    return {"shape": shape, "dtype": dtype, "role": role, "init": init, "strides": strides}


def _dag(rng, nloads, nodes_max=6):
    """Random expression DAG over load 0..nloads-1; returns the node list."""
    expr = [("load", k) for k in range(nloads)]
    if rng.random() < 0.5:
        expr.append(("const", float(rng.choice([0.5, 2.0, -1.5, 3.0, 0.125]))))
    for _ in range(int(rng.integers(1, nodes_max))):
        n = len(expr)
        if rng.random() < 0.3:
            op = str(rng.choice(EXACT_UNARY))
            a = int(rng.integers(0, n))
            if op == "sqrt":      # keep sqrt's argument non-negative
                expr.append(("abs", a))
                expr.append(("sqrt", len(expr) - 1))
            else:
                expr.append((op, a))
        else:
            op = str(rng.choice(EXACT_BINARY))
            expr.append((op, int(rng.integers(0, n)), int(rng.integers(0, n))))
    # make sure every load is used: fold unused ones in with adds
    used = set()
    for e in expr[nloads:]:
        for x in e[1:]:
            if isinstance(x, int) and e[0] != "const":
                used.add(x)
    last = len(expr) - 1
    for k in range(nloads):
        if k not in used and k != last:
            expr.append(("add", last, k))
            last = len(expr) - 1
    if rng.random() < 0.2:
        expr.append(("cast", len(expr) - 1, str(rng.choice(["f16", "bf16"]))))
    return expr


def random_op(rng):
    loops = _loops(rng)
    names = list(loops)
    pat = rng.choice(["assign", "reduce", "producer", "rowstat", "integer"], p=[0.35, 0.25, 0.12, 0.18, 0.1])
    tensors, stmts = {}, []
    seed = int(rng.integers(1000, 100000))

    def inputs(k, over=None):
        reads = []
        for i in range(k):
            sub = [n for n in names if rng.random() < 0.75] or [str(rng.choice(names))]
            if over is not None:
                sub = [n for n in sub if n in over] or list(over)
            sub = list(rng.permutation(sub)) if rng.random() < 0.4 else sub
            nm = f"x{i}"
            tensors[nm] = _tensor(rng, loops, sub, str(rng.choice(DTYPES)), "in", seed + i)
            reads.append((nm, list(sub)))
        return reads

    out_dt = str(rng.choice(DTYPES))
    if pat == "integer":
        # reading R30: i32 tensors only, wrap-around integer DAG, any layout (transposes included)
        reads = []
        for i in range(int(rng.integers(1, 4))):
            sub = [n for n in names if rng.random() < 0.75] or [str(rng.choice(names))]
            sub = list(rng.permutation(sub)) if rng.random() < 0.4 else sub
            t = _tensor(rng, loops, sub, "i32", "in", seed + i)
            t["init"] = ("randint", -2 ** 30, 2 ** 30, seed + i)
            tensors[f"x{i}"] = t
            reads.append((f"x{i}", list(sub)))
        perm = list(rng.permutation(names)) if rng.random() < 0.5 else names
        tensors["out"] = _tensor(rng, loops, perm, "i32", "out", 0)
        expr = [("load", k) for k in range(len(reads))]
        if rng.random() < 0.5:
            expr.append(("const", float(rng.choice([3.0, -7.0, 65537.0, 0.0]))))
        for _ in range(int(rng.integers(1, 6))):
            n = len(expr)
            if rng.random() < 0.3:
                expr.append((str(rng.choice(INT_UNARY)), int(rng.integers(0, n))))
            else:
                expr.append((str(rng.choice(INT_BINARY)), int(rng.integers(0, n)), int(rng.integers(0, n))))
        last = len(expr) - 1
        for k in range(len(reads)):   # every load used
            expr.append(("add", last, k))
            last = len(expr) - 1
        if rng.random() < 0.35 and len(names) > 1:   # an integer REDUCE over some loops (wrap-around, exact)
            red = [n for n in names if rng.random() < 0.5] or [names[-1]]
            keep = [n for n in names if n not in red] or [names[0]]
            red = [n for n in names if n not in keep]
            tensors["out"] = _tensor(rng, loops, keep, "i32", "out", 0, pad=False)
            stmts.append({"kind": "reduce", "op": "max" if rng.random() < 0.3 else "sum", "loops": names,
                          "write": ("out", list(keep)), "reads": reads, "expr": expr})
        else:
            stmts.append({"kind": "assign", "loops": names, "write": ("out", list(perm)), "reads": reads,
                          "expr": expr})
    elif pat == "assign":
        reads = inputs(int(rng.integers(1, 4)))
        perm = list(rng.permutation(names)) if rng.random() < 0.5 else names
        tensors["out"] = _tensor(rng, loops, perm, out_dt, "out", 0)
        stmts.append({"kind": "assign", "loops": names, "write": ("out", list(perm)), "reads": reads,
                      "expr": _dag(rng, len(reads))})
    elif pat == "reduce" or len(names) == 1:
        red = [n for n in names if rng.random() < 0.5] or [names[-1]]
        keep = [n for n in names if n not in red]
        perm = list(rng.permutation(keep)) if rng.random() < 0.5 else keep
        reads = inputs(int(rng.integers(1, 3)))
        op = "max" if rng.random() < 0.35 else "sum"
        tensors["out"] = _tensor(rng, loops, perm, "f32", "out", 0, pad=False)
        st = {"kind": "reduce", "op": op, "loops": names, "write": ("out", list(perm)), "reads": reads,
              "expr": _dag(rng, len(reads), nodes_max=3)}
        if rng.random() < 0.4:
            st["finalize"] = [("acc",), ("const", float(rng.choice([3.0, 0.25, 768.0]))), ("div", 0, 1)]
        stmts.append(st)
        pat = "reduce"
    elif pat == "producer":
        # TEMP p[sub] = f(params[sub]);  out[all] = g(x[all], p[sub])
        sub = [n for n in names if rng.random() < 0.5] or [names[0]]
        preads = inputs(2, over=sub)
        tensors["p"] = {"shape": [loops[n] for n in sub], "dtype": "f32", "role": "temp", "init": None,
                        "strides": None}
        stmts.append({"kind": "assign", "loops": sub, "write": ("p", list(sub)), "reads": preads,
                      "expr": _dag(rng, 2, nodes_max=3)})
        tensors["y"] = _tensor(rng, loops, names, str(rng.choice(DTYPES)), "in", seed + 9)
        perm = list(rng.permutation(names)) if rng.random() < 0.3 else names
        tensors["out"] = _tensor(rng, loops, perm, out_dt, "out", 0)
        stmts.append({"kind": "assign", "loops": names, "write": ("out", list(perm)),
                      "reads": [("y", names), ("p", list(sub))], "expr": _dag(rng, 2, nodes_max=4)})
    else:
        # row statistic over the innermost loop, then a normalisation using it
        row, keep = names[-1], names[:-1]
        tensors["x"] = _tensor(rng, loops, names, str(rng.choice(["f16", "f32"])), "in", seed + 5, pad=False)
        tensors["s"] = {"shape": [loops[n] for n in keep], "dtype": "f32",
                        "role": "temp" if rng.random() < 0.5 else "out", "init": None, "strides": None}
        op = "max" if rng.random() < 0.5 else "sum"
        stmts.append({"kind": "reduce", "op": op, "loops": names, "write": ("s", keep),
                      "reads": [("x", names)], "expr": [("load", 0), ("abs", 0)]})
        tensors["out"] = _tensor(rng, loops, names, out_dt, "out", 0, pad=False)
        stmts.append({"kind": "assign", "loops": names, "write": ("out", names),
                      "reads": [("x", names), ("s", keep)],
                      "expr": [("load", 0), ("load", 1), ("const", 1.0), ("add", 1, 2), ("div", 0, 3)]})
    return {"name": f"fuzz_{pat}", "loops": loops, "tensors": tensors, "stmts": stmts}
