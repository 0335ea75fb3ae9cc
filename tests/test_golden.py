"""Fixtures of values the paper prints (tests/golden/, each with its citation), checked against
the planner oracle and against the numbers this repo quotes from the paper."""
import math
import os

import workloads as W
from oracle import planner_oracle as P

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _rows(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return [l.strip() for l in f if l.strip() and not l.startswith("#")]


def test_fig2_schedules_from_the_paper():
    """Algorithm 2 + cost on Fig. 2's running example reaches Fig. 2(c)."""
    want = {}
    for line in _rows("fig2_schedules.txt"):
        key, val = line.split(":", 1)
        want[key.strip()] = val.strip()
    for N in (8, 64, 512):
        d = W.fig2_running_example(N)
        X, Y = d["stmts"]
        for stmt, key in ((X, "X"), (Y, "Y")):
            order, vec = (p.split() for p in want[key].split("|"))
            got = P.algorithm2(d, stmt)
            assert got == order and got[-1] == vec[0], (N, key, got)
        sc = P.innermost_scores(d, Y)
        assert max(sc, key=sc.get) != want["Y_rejected_innermost"]


def test_table2_geomeans_quoted_in_this_repo():
    """The context numbers the bench line and BASELINE.md quote: geomean infl speedup 1.78 (printed as
    "1.7x") and the explicit-vector gain infl/novec 1.09."""
    rows = _rows("table2_all_fused_speedups.csv")[1:]
    infl = [float(r.split(",")[5]) for r in rows]
    novec = [float(r.split(",")[4]) for r in rows]
    g = math.exp(sum(map(math.log, infl)) / len(infl))
    gv = math.exp(sum(math.log(a / b) for a, b in zip(infl, novec)) / len(infl))
    assert abs(g - 1.78) < 0.01 and int(g * 10) / 10 == 1.7
    assert abs(gv - 1.09) < 0.01
