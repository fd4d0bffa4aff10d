"""Host-side checks of bench.py's accounting (CPU, no GPU): the roofline object follows SURVEY
§8(d) -- max(T_work, T_span, T_mem) with the binding term named and its fraction of the measured
time -- for every bench workload, and the C5 column-strip T(P) model is only
emitted for lcs16 plans and reproduces the single-GPU time at P = 1."""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402

# measured ms per step on one B200 (profiles/round2_bench.json) and the binding term expected
MEASURED = {"C1": (0.0511, "span"), "C2": (0.852, "span"), "C3": (1.564, "span"), "C4": (1.522, "hbm"),
            "C5": (4.034, "alu"), "C6": (0.680, "hbm"), "C7": (1.500, "hbm"), "C8": (1.617, "span")}


@pytest.mark.parametrize("name", sorted(MEASURED))
def test_roofline_terms(name):
    ms, bound = MEASURED[name]
    peaks = bench.load_peaks()
    r = bench.roofline(name, ms, peaks, 1, 1965)
    assert r["bound"] == bound, r
    terms = r["terms_ms"]
    assert set(terms) == {"work", "span", "mem"}
    # the binding term is the largest, and the reported fraction is that term over the measured time
    key = {"hbm": "mem", "alu": "work", "fma": "work", "span": "span"}[r["bound"]]
    assert terms[key] == max(terms.values())
    assert 0.0 < r["frac"] <= 1.0
    assert r["frac"] == pytest.approx(terms[key] / ms, rel=2e-3)
    assert r["frac"] == pytest.approx(r["achieved"] / r["peak"], rel=2e-3)


def test_roofline_hbm_peak_is_measured():
    peaks = bench.load_peaks()
    r = bench.roofline("C6", 0.68, peaks, 1, 1965)
    assert r["peak"] == pytest.approx(peaks["hbm_gbs"], rel=1e-3)
    assert "measured" in str(r["hbm_peak_source"]).lower() or r["hbm_peak_source"]


def test_scaling_model_only_for_lcs16():
    assert bench.scaling_model(1.5, {"kernel": "prevrow_hx", "variant": 2}, 32768) is None
    plan = {"kernel": "lcs16", "strips": 261, "chunks": 3125, "extra_lag": 2}
    m = bench.scaling_model(4.03, plan, 100000)
    assert m["P1"]["strong_ms"] == pytest.approx(4.03, rel=1e-3)
    # strong scaling is capped near 1x by the strip pipeline; weak-scaling efficiency falls with P
    for P in (2, 4, 8):
        assert 0.9 < m[f"P{P}"]["strong_speedup"] <= 1.0
    assert m["P2"]["weak_efficiency"] > m["P4"]["weak_efficiency"] > m["P8"]["weak_efficiency"]
