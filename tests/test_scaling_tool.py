"""tools/scaling.py: eq. 4 efficiencies from bench lines (host logic, no GPU)."""
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
import scaling  # noqa: E402


def line(m, v, kind="weak"):
    return {"metric": "x", "n_gpus": m, "value": v, "insert_gops": v / 2, "query_gops": v * 2,
            "scaling": kind}


def test_weak_efficiency_is_eq4():
    # tau(n,1) = 2n / v1, tau(mn, m) = 2mn / vm  ->  E_w = vm / (m v1)
    e = scaling.efficiencies([line(1, 10.0), line(2, 19.0), line(8, 72.0)])["weak"]
    assert abs(e[1]["value"] - 1.0) < 1e-12
    assert abs(e[2]["value"] - 0.95) < 1e-12
    assert abs(e[8]["value"] - 0.9) < 1e-12
    assert abs(e[8]["insert_gops"] - 0.9) < 1e-12


def test_strong_separate_and_reference_lines_ignored():
    lines = [line(1, 10.0, "strong"), line(4, 30.0, "strong"), line(1, 10.0),
             dict(line(4, 1.0), impl="reference")]
    e = scaling.efficiencies(lines)
    assert abs(e["strong"][4]["value"] - 0.75) < 1e-12
    assert list(e["weak"]) == [1]
