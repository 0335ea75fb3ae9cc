"""One named pin per case of the oracle's expression evaluator
(oracle/fop_oracle.c: apply() for float statements, apply_int() for integer
statements), each against something other than the oracle: exact rational or
60-digit decimal arithmetic, numpy's IEEE float32 / int32 routines, closed
forms and hand-worked special values.  DESIGN.md §3 lists these pins.

The paper's statement DAG is abstract (the f and g of Fig. 2, PAPER.md P:54,
P:59), so every opcode the ABI accepts needs its own definition and pin;
readings R12 (transcendentals in double, rounded once to fp32), R15 (relu),
R24 (max/min of +-0 and NaN), R29 (GELU at +-inf) and R30 (i32 arithmetic)
are the definitions pinned here.
"""
import decimal
from decimal import Decimal

import numpy as np
import pytest

from oracle import oracle as O

F32 = np.float32
PI = Decimal("3.14159265358979323846264338327950288419716939937510582097494459230781640628620899862803")


@pytest.fixture(autouse=True)
def _decimal_precision():
    """80 significant digits for every decimal reference (other modules set their own)."""
    with decimal.localcontext() as ctx:
        ctx.prec = 80
        yield


# ---------------------------------------------------------------- helpers
def run_ew(expr, cols, out_dtype="f32", in_dtype="f32"):
    """The oracle on out[i] = expr(a[i], b[i], ...) over one loop."""
    n = len(cols[0])
    names = "abcd"[:len(cols)]
    d = {"name": "op", "loops": {"i": n},
         "tensors": {**{k: {"shape": [n], "dtype": in_dtype, "role": "in", "init": None, "strides": None}
                        for k in names},
                     "out": {"shape": [n], "dtype": out_dtype, "role": "out", "init": None, "strides": None}},
         "stmts": [{"kind": "assign", "loops": ["i"], "write": ("out", ["i"]),
                    "reads": [(k, ["i"]) for k in names], "expr": expr}]}
    np_in = {"f32": np.float32, "i32": np.int32, "f16": np.float16}[in_dtype]
    return O.run(d, {k: np.asarray(c, np_in) for k, c in zip(names, cols)})["out"]


def unary(op, v, out_dtype="f32"):
    return run_ew([("load", 0), (op, 0)], [v], out_dtype)


def binary(op, a, b):
    return run_ew([("load", 0), ("load", 1), (op, 0, 1)], [a, b])


def bits(x):
    x = np.asarray(x)
    return x.view(np.uint32 if x.itemsize == 4 else np.uint16)


def ordered(f):
    i = np.asarray(f, F32).view(np.int32).astype(np.int64)
    return np.where(i < 0, -(i & 0x7FFFFFFF), i)


def rn32(D):
    """Decimal -> nearest float32 (ties to even), decided in exact decimal arithmetic."""
    if D.is_nan():
        return F32(np.nan)
    f = F32(float(D))
    if not np.isfinite(f):
        return f
    cands = [np.nextafter(f, F32(-np.inf)), f, np.nextafter(f, F32(np.inf))]
    best = min(cands, key=lambda c: (abs(Decimal(float(c)) - D), int(bits(np.array([c], F32))[0]) & 1))
    return F32(best)


def dexp(x):
    return Decimal(float(x)).exp()


def erf_dec(z):
    """erf(z) by its Maclaurin series in 80-digit arithmetic (|z| <= 10)."""
    z = Decimal(z)
    term, s, n = z, z, 0
    while True:
        n += 1
        term = -term * z * z / n
        add = term / (2 * n + 1)
        s += add
        if abs(add) < Decimal(10) ** -70:
            break
    return 2 / PI.sqrt() * s


def sample(lo, hi, n, seed):
    return np.random.default_rng(seed).uniform(lo, hi, n).astype(F32)


def assert_within_one_ulp_mostly_exact(got, ref, min_exact=0.99):
    d = np.abs(ordered(got) - ordered(ref))
    assert d.max() <= 1, (d.max(), got[np.argmax(d)], ref[np.argmax(d)])
    assert (d == 0).mean() >= min_exact


# ---------------------------------------------------------------- IEEE arithmetic (apply: ADD SUB MUL DIV SQRT)
SPECIAL = np.array([0.0, -0.0, 1.0, -1.0, np.inf, -np.inf, np.nan, 3e38, -3e38, 1e-40, -1e-45, 6e4, 0.1],
                   F32)


def _pairs():
    rng = np.random.default_rng(3)
    a = np.concatenate([rng.standard_normal(4000).astype(F32) * F32(2.0) ** rng.integers(-60, 60, 4000).astype(F32),
                        np.repeat(SPECIAL, len(SPECIAL))]).astype(F32)
    b = np.concatenate([rng.standard_normal(4000).astype(F32) * F32(2.0) ** rng.integers(-60, 60, 4000).astype(F32),
                        np.tile(SPECIAL, len(SPECIAL))]).astype(F32)
    return a, b


@pytest.mark.parametrize("op,fn", [("add", np.add), ("sub", np.subtract), ("mul", np.multiply),
                                   ("div", np.divide)])
def test_arith_vs_numpy_ieee_float32(op, fn):
    """+ - * / are IEEE correctly rounded fp32 (no contraction): numpy's float32 ufuncs."""
    a, b = _pairs()
    with np.errstate(all="ignore"):
        ref = fn(a, b)
    got = binary(op, a, b)
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(got), nan)
    assert np.array_equal(bits(got[~nan]), bits(ref[~nan]))


def test_arith_exact_rational_spot_checks():
    """Correct rounding against exact rational arithmetic on random normal operands."""
    from fractions import Fraction as Fr
    rng = np.random.default_rng(4)
    a = rng.standard_normal(300).astype(F32)
    b = rng.standard_normal(300).astype(F32)
    for op, f in (("add", lambda x, y: x + y), ("mul", lambda x, y: x * y), ("div", lambda x, y: x / y)):
        got = binary(op, a, b)
        for x, y, g in zip(a, b, got):
            q = f(Fr(float(x)), Fr(float(y)))
            assert F32(g) == rn32(Decimal(q.numerator) / Decimal(q.denominator))


def test_sqrt_vs_numpy_and_squares():
    v = np.concatenate([sample(0, 1e6, 3000, 5), SPECIAL]).astype(F32)
    with np.errstate(invalid="ignore"):
        ref = np.sqrt(v)
    got = unary("sqrt", v)
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(got), nan)
    assert np.array_equal(bits(got[~nan]), bits(ref[~nan]))
    k = np.arange(1, 4097, dtype=F32)
    assert np.array_equal(unary("sqrt", k * k), k)                  # exact squares
    assert bits(unary("sqrt", np.array([-0.0], F32)))[0] == 0x80000000  # sqrt(-0) = -0 (IEEE)


def test_neg_abs_flip_and_clear_the_sign_bit_only():
    v = np.concatenate([sample(-5, 5, 200, 6), SPECIAL]).astype(F32)
    assert np.array_equal(bits(unary("neg", v)), bits(v) ^ np.uint32(0x80000000))
    assert np.array_equal(bits(unary("abs", v)), bits(v) & np.uint32(0x7FFFFFFF))


def test_const_is_the_fp32_immediate():
    got = run_ew([("load", 0), ("const", 0.1), ("add", 0, 1)], [np.zeros(3, F32)])
    assert np.all(got == F32(0.1))


# ---------------------------------------------------------------- MAX / MIN (reading R24)
def test_max_min_vs_numpy_fmax_fmin():
    """NaN operands are ignored (IEEE 754-2019 maximumNumber / C fmaxf): numpy fmax/fmin."""
    a, b = _pairs()
    zero_pair = (a == 0) & (b == 0)
    for op, fn in (("max", np.fmax), ("min", np.fmin)):
        got = binary(op, a, b)
        ref = fn(a, b)
        nan = np.isnan(ref)
        assert np.array_equal(np.isnan(got), nan)
        m = ~nan & ~zero_pair
        assert np.array_equal(bits(got[m]), bits(ref[m]))


def test_max_min_signed_zero_and_nan_hand_cases():
    P, N, Q = 0.0, -0.0, np.nan
    a = np.array([P, N, N, P, Q, 1.0, Q, N, -2.0], F32)
    b = np.array([N, P, N, P, 1.0, Q, Q, -1.0, N], F32)
    mx = binary("max", a, b)
    mn = binary("min", a, b)
    # max(+-0) = +0 unless both are -0; min(+-0) = -0 unless both are +0
    assert bits(mx)[:4].tolist() == [0, 0, 0x80000000, 0]
    assert bits(mn)[:4].tolist() == [0x80000000, 0x80000000, 0x80000000, 0]
    assert mx[4] == 1.0 and mx[5] == 1.0 and np.isnan(mx[6])
    assert mn[4] == 1.0 and mn[5] == 1.0 and np.isnan(mn[6])
    assert bits(mx)[7] == 0x80000000 and mn[7] == -1.0                       # -0 vs -1
    assert bits(mx)[8] == 0x80000000 and mn[8] == -2.0


# ---------------------------------------------------------------- transcendentals (reading R12)
def test_exp_vs_decimal_and_special_values():
    v = np.concatenate([sample(-87, 88, 400, 7), sample(-1, 1, 100, 8)]).astype(F32)
    got = unary("exp", v)
    ref = np.array([rn32(dexp(x)) for x in v], F32)
    assert_within_one_ulp_mostly_exact(got, ref)
    s = unary("exp", np.array([0.0, -0.0, np.inf, -np.inf, np.nan, 89.0, -104.0], F32))
    assert s[0] == 1 and s[1] == 1 and s[2] == np.inf and bits(s[3:4])[0] == 0 and np.isnan(s[4])
    assert s[5] == np.inf and s[6] == 0


def test_log_vs_decimal_closed_forms_and_special_values():
    v = np.concatenate([sample(0, 1e4, 300, 9), sample(0, 2, 100, 10),
                        (np.float32(2.0) ** sample(-126, 127, 100, 11)).astype(F32)]).astype(F32)
    v = v[v > 0]
    got = unary("log", v)
    ref = np.array([rn32(Decimal(float(x)).ln()) for x in v], F32)
    assert_within_one_ulp_mostly_exact(got, ref)
    k = np.arange(-126, 128)
    pw = unary("log", (2.0 ** k).astype(F32))
    ln2 = Decimal(2).ln()
    assert np.array_equal(pw, np.array([rn32(int(j) * ln2) for j in k], F32))   # log 2^k = k ln 2
    s = unary("log", np.array([1.0, 0.0, -0.0, -1.0, np.inf, -np.inf, np.nan, 1e-45], F32))
    assert bits(s[:1])[0] == 0                                                  # log 1 = +0
    assert s[1] == -np.inf and s[2] == -np.inf and np.isnan(s[3]) and s[4] == np.inf
    assert np.isnan(s[5]) and np.isnan(s[6])
    assert s[7] == rn32(Decimal(float(F32(1e-45))).ln())                         # smallest subnormal


def _tanh_dec(x):
    e = (2 * Decimal(float(x))).exp()
    return (e - 1) / (e + 1)


def test_tanh_vs_decimal_odd_and_limits():
    v = np.concatenate([sample(-10, 10, 400, 12), sample(-0.01, 0.01, 50, 13)]).astype(F32)
    got = unary("tanh", v)
    ref = np.array([rn32(_tanh_dec(x)) for x in v], F32)
    assert_within_one_ulp_mostly_exact(got, ref)
    assert np.array_equal(unary("tanh", -v), -got)                              # odd
    s = unary("tanh", np.array([0.0, -0.0, np.inf, -np.inf, 20.0, np.nan], F32))
    assert bits(s[:2]).tolist() == [0, 0x80000000] and s[2] == 1 and s[3] == -1 and s[4] == 1
    assert np.isnan(s[5])


def test_sigmoid_vs_decimal_symmetry_and_limits():
    v = np.concatenate([sample(-30, 30, 400, 14), sample(-100, -80, 20, 15)]).astype(F32)
    got = unary("sigmoid", v)
    ref = np.array([rn32(1 / (1 + (-Decimal(float(x))).exp())) for x in v], F32)
    assert_within_one_ulp_mostly_exact(got, ref)
    s = unary("sigmoid", np.array([0.0, np.inf, -np.inf, np.nan, 200.0, -200.0], F32))
    assert s[0] == 0.5 and s[1] == 1 and bits(s[2:3])[0] == 0 and np.isnan(s[3]) and s[4] == 1
    assert s[5] == 0
    w = sample(-5, 5, 200, 16)
    assert np.allclose(unary("sigmoid", w) + unary("sigmoid", -w), 1, rtol=0, atol=1.2e-7)   # s(x)+s(-x)=1


def _gelu_erf_dec(x):
    z = Decimal(float(x)) / Decimal(2).sqrt()
    return Decimal(float(x)) * (1 + erf_dec(z)) / 2


def test_gelu_erf_vs_decimal_series_including_the_tail():
    """0.5 v (1 + erf(v / sqrt 2)) against its Maclaurin series in 80 digits, over
    [-13, 13] (the negative tail, 0.5 v erfc(|v|/sqrt 2) down to ~1e-38, included)."""
    v = np.concatenate([sample(-6, 6, 300, 17), sample(-13, -6, 60, 18), sample(6, 13, 20, 19)]).astype(F32)
    got = unary("gelu_erf", v)
    ref = np.array([rn32(_gelu_erf_dec(x)) for x in v], F32)
    assert_within_one_ulp_mostly_exact(got, ref)


def test_gelu_erf_identities_and_special_values():
    v = sample(-4, 4, 300, 20)
    g, gm = unary("gelu_erf", v), unary("gelu_erf", -v)
    assert np.allclose(g.astype(np.float64) - gm, v, rtol=0, atol=4e-7 * np.maximum(1, np.abs(v)))  # g(v)-g(-v)=v
    s = unary("gelu_erf", np.array([0.0, -0.0, np.inf, -np.inf, np.nan, 1.0, 30.0], F32))
    assert bits(s[:2]).tolist() == [0, 0x80000000]
    assert s[2] == np.inf
    assert np.isnan(s[3])        # R29: -inf * (1 + erf(-inf)) = -inf * 0 = NaN (IEEE; torch gelu agrees)
    assert np.isnan(s[4])
    assert s[5] == rn32(Decimal("0.841344746068542948585232545632034"))          # Phi(1) to 33 digits
    assert s[6] == 30.0


def test_gelu_tanh_special_values():
    s = unary("gelu_tanh", np.array([0.0, -0.0, np.inf, -np.inf, np.nan, 30.0], F32))
    assert bits(s[:2]).tolist() == [0, 0x80000000] and s[2] == np.inf
    assert np.isnan(s[3]) and np.isnan(s[4]) and s[5] == 30.0


def test_cast_nodes_round_like_numpy():
    v = np.concatenate([sample(-7e4, 7e4, 500, 21), SPECIAL]).astype(F32)
    got = run_ew([("load", 0), ("cast", 0, "f16")], [v])
    with np.errstate(over="ignore"):
        ref = v.astype(np.float16).astype(F32)
    nan = np.isnan(ref)
    assert np.array_equal(bits(got[~nan]), bits(ref[~nan])) and np.all(np.isnan(got[nan]))


# ---------------------------------------------------------------- integer statements (reading R30)
I32 = np.int32


def _irand(n, seed):
    rng = np.random.default_rng(seed)
    v = rng.integers(-2 ** 31, 2 ** 31, n, dtype=np.int64).astype(I32)
    v[:8] = [0, 1, -1, 2 ** 31 - 1, -2 ** 31, -2 ** 31, 2 ** 31 - 1, 65536]
    return v


def run_int(expr, cols):
    n = len(cols[0])
    names = "abcd"[:len(cols)]
    d = {"name": "iop", "loops": {"i": n},
         "tensors": {**{k: {"shape": [n], "dtype": "i32", "role": "in", "init": None, "strides": None}
                        for k in names},
                     "out": {"shape": [n], "dtype": "i32", "role": "out", "init": None, "strides": None}},
         "stmts": [{"kind": "assign", "loops": ["i"], "write": ("out", ["i"]),
                    "reads": [(k, ["i"]) for k in names], "expr": expr}]}
    return O.run(d, {k: np.asarray(c, I32) for k, c in zip(names, cols)})["out"]


@pytest.mark.parametrize("op,fn", [("add", np.add), ("sub", np.subtract), ("mul", np.multiply),
                                   ("max", np.maximum), ("min", np.minimum)])
def test_int_binary_wraps_like_numpy_int32(op, fn):
    a, b = _irand(5000, 30), _irand(5000, 31)[::-1].copy()
    with np.errstate(over="ignore"):
        ref = fn(a, b)                                   # numpy int32: two's complement wrap-around
    assert np.array_equal(run_int([("load", 0), ("load", 1), (op, 0, 1)], [a, b]), ref)


def test_int_unary_and_const():
    a = _irand(3000, 32)
    with np.errstate(over="ignore"):
        assert np.array_equal(run_int([("load", 0), ("neg", 0)], [a]), -a)      # -INT_MIN wraps to INT_MIN
        assert np.array_equal(run_int([("load", 0), ("abs", 0)], [a]), np.abs(a))
        assert np.array_equal(run_int([("load", 0), ("relu", 0)], [a]), np.maximum(a, 0))
        ref = (a * I32(3) + I32(-7)).astype(I32)
    got = run_int([("load", 0), ("const", 3.0), ("mul", 0, 1), ("const", -7.0), ("add", 2, 3)], [a])
    assert np.array_equal(got, ref)
    # closed form: (2^31 - 1) + 1 = -2^31
    assert run_int([("load", 0), ("const", 1.0), ("add", 0, 1)], [np.array([2 ** 31 - 1], I32)])[0] == -2 ** 31


def test_int_reduce_sum_wraps_and_max_vs_numpy():
    R, Cn = 300, 7
    x = _irand(R * Cn, 33)
    for op, fn in (("sum", lambda m: m.sum(0, dtype=np.int64)), ("max", lambda m: m.max(0))):
        d = {"name": "ired", "loops": {"r": R, "c": Cn},
             "tensors": {"x": {"shape": [R, Cn], "dtype": "i32", "role": "in", "init": None, "strides": None},
                         "out": {"shape": [Cn], "dtype": "i32", "role": "out", "init": None, "strides": None}},
             "stmts": [{"kind": "reduce", "op": op, "loops": ["r", "c"], "write": ("out", ["c"]),
                        "reads": [("x", ["r", "c"])], "expr": [("load", 0)]}]}
        got = O.run(d, {"x": x})["out"]
        ref = fn(x.reshape(R, Cn).astype(np.int64))
        ref = ((ref + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(I32)        # modulo 2^32 into int32
        assert np.array_equal(got, ref), op


@pytest.mark.parametrize("expr,dt,msg", [
    ([("load", 0), ("const", 1.0), ("div", 0, 1)], "i32", "not defined on i32"),
    ([("load", 0), ("exp", 0)], "i32", "not defined on i32"),
    ([("load", 0), ("const", 0.5), ("add", 0, 1)], "i32", "not defined on i32"),
    ([("load", 0), ("const", 1.0), ("add", 0, 1)], "f32", "float statement reads an i32"),
])
def test_int_rejections(expr, dt, msg):
    n = 4
    d = {"name": "bad", "loops": {"i": n},
         "tensors": {"a": {"shape": [n], "dtype": "i32", "role": "in", "init": None, "strides": None},
                     "out": {"shape": [n], "dtype": dt, "role": "out", "init": None, "strides": None}},
         "stmts": [{"kind": "assign", "loops": ["i"], "write": ("out", ["i"]), "reads": [("a", ["i"])],
                    "expr": expr}]}
    with pytest.raises(ValueError, match=msg):
        O.run(d, {"a": np.zeros(n, I32)})


def test_int_move_keeps_bits():
    a = _irand(100, 34)
    assert np.array_equal(run_int([("load", 0)], [a]), a)


def test_every_abi_opcode_has_a_named_pin_here():
    """Every expression opcode include/fop.h declares (FOP_OP_*) is exercised by a pin in
    this file (or, for ACC, tests/test_oracle.py) under its descriptor name, so a new opcode
    cannot reach the ABI unpinned."""
    import os
    import re
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    ops = set(re.findall(r"FOP_OP_([A-Z0-9_]+)", open(os.path.join(root, "include", "fop.h")).read()))
    ops -= {"_COUNT"}
    # descriptor names are the lower-case opcodes; ACC (a REDUCE's finalize input) is pinned
    # with the finalize expressions in tests/test_oracle.py
    src = open(os.path.abspath(__file__)).read() + open(os.path.join(root, "tests", "test_oracle.py")).read()
    missing = [op for op in sorted(ops) if f'"{op.lower()}"' not in src and f"'{op.lower()}'" not in src]
    assert not missing, f"opcodes without a pin in tests/test_oracle_ops.py: {missing}"
