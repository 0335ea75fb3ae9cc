"""Pins of the Algorithm-2 oracle (oracle/planner_oracle.py) to the paper.

The paper prints the outcome its optimizer must reach on the running example:
Fig. 2(c) runs Y as ``forall i / for k / forvec j`` and X with k
innermost; Fig. 3(b)'s prose asks for "exactly a coefficient 1 for j on the
third dimension"; Fig. 2(b)'s innermost k, with long jumps in D, is
the bad schedule.  P:353 fixes write-over-read priority and "if
multiple candidate dimensions enable strides of size 1, we favor the one with
more accesses with stride 1".  The numeric scores are hand evaluations of
P:338 under the readings of DESIGN.md.
"""
import pytest

import workloads as W
from oracle import planner_oracle as P


@pytest.mark.parametrize("N", [4, 16, 64, 256, 1000])
def test_fig2_Y_is_fig2c_order_for_any_N(N):
    d = W.fig2_running_example(N)
    X, Y = d["stmts"]
    assert P.algorithm2(d, Y) == ["i", "k", "j"]          # Fig. 2(c)
    assert P.algorithm2(d, X)[-1] == "k"                   # X: k innermost (Fig. 2(c))
    sc = P.innermost_scores(d, Y)
    assert sc["j"] > sc["k"] > sc["i"]                     # Fig. 2(b)'s innermost k rejected


def test_fig2_scores_hand_evaluated():
    d = W.fig2_running_example(64)
    X, Y = d["stmts"]
    sy = P.innermost_scores(d, Y)
    assert sy["j"] == pytest.approx(5 + 3 * 3 + 1 + 3 + 64 / 1024)
    assert sy["k"] == pytest.approx(5 + 3 * 2 + 1 + 1 + 64 / 1024)
    assert sy["i"] == pytest.approx(1 / 64 + 64 / 1024)
    sx = P.innermost_scores(d, X)
    assert sx["k"] == pytest.approx(5 + 3 + 1 + 2 + 64 / 1024)


def test_write_over_read_priority_transpose():
    d = W.transpose2d(64, 96)
    s = d["stmts"][0]
    sc = P.innermost_scores(d, s)
    assert sc["i"] == pytest.approx(7.0625) and sc["j"] == pytest.approx(5.09375)
    assert P.algorithm2(d, s) == ["j", "i"]     # vector loop i: the store-contiguous one


def test_more_stride1_accesses_wins():
    # two candidate loops both reach stride 1; the one with more stride-1 accesses wins
    d = {"loops": {"p": 32, "q": 32},
         "tensors": {"a": {"shape": [32, 32], "dtype": "f32", "role": "in"},
                     "b": {"shape": [32, 32], "dtype": "f32", "role": "in"},
                     "c": {"shape": [32, 32], "dtype": "f32", "role": "in"},
                     "o": {"shape": [32], "dtype": "f32", "role": "out"}},
         "stmts": [{"kind": "reduce", "op": "sum", "loops": ["p", "q"],
                    "write": ("o", [0]), "reads": [("a", ["p", "q"]), ("b", ["p", "q"]),
                                                    ("c", ["q", "p"])],
                    "expr": [("load", 0)]}]}
    d["tensors"]["o"]["shape"] = [1]
    s = d["stmts"][0]
    sc = P.innermost_scores(d, s)
    assert sc["q"] > sc["p"]                    # a, b contiguous along q; only c along p


@pytest.mark.parametrize("name,expect,inner", [
    ("cfg1", ["a", "b", "c"], {"c": 19.015625, "b": 3.0703125, "a": 3.01171875}),
    ("cfg3", ["h", "w", "c"], {"c": 7.25, "w": 5.0546875, "n": 0.25 + 1 / 802816}),
    ("cfg4b", ["r", "c"], {"c": 15.0, "r": 8.0 + 1 / 1024}),
])
def test_config_scenarios(name, expect, inner):
    d = W.CONFIGS[name]()
    s = d["stmts"][-1]
    assert P.algorithm2(d, s) == expect
    sc = P.innermost_scores(d, s)
    for k, v in inner.items():
        assert sc[k] == pytest.approx(v, abs=1e-9)


def test_cfg2_and_cfg4a_scenarios():
    d = W.cfg2()
    assert P.algorithm2(d, d["stmts"][2]) == ["h", "c", "w"]
    d = W.cfg4a()
    for s in d["stmts"]:
        assert P.algorithm2(d, s) == ["b", "s", "h"]
    sc = P.innermost_scores(d, d["stmts"][1])
    assert sc["h"] == pytest.approx(13.75) and sc["s"] == pytest.approx(11.5)


def test_printed_thread_term_flips_cfg1():
    """Evidence for reading R1: the printed w5*F*L/N vectorises the extent-4 loop."""
    d = W.cfg1()
    assert P.algorithm2(d, d["stmts"][0], readings=0)[-1] == "a"
    assert P.algorithm2(d, d["stmts"][0])[-1] == "c"


def test_scenario_list_bounded_and_distinct():
    d = W.cfg2()
    sc = P.scenarios(d, d["stmts"][2])
    assert 1 <= len(sc) <= 8
    assert sc[0] == P.algorithm2(d, d["stmts"][2])
    assert len({tuple(s) for s in sc}) == len(sc)
    assert all(len(s) == 3 for s in sc)
