"""Pins for oracle/config.py against the paper's printed adaptive-scheme numbers (P8)."""
import pytest

from oracle import config as cfg
from sknn_testutil import load_golden

G = load_golden("adaptive_config.json")


def test_k20c_thresholds():
    k = G["k20c"]
    assert cfg.th1(k["smem_per_sm"], k["max_threads_per_sm"]) == k["th1"]
    assert cfg.th2(k["max_regs_per_thread"]) == k["th2_formula"]
    # the paper prints 1024: within one register of the formula (reading R14)
    assert abs(k["th2_printed"] - cfg.th2(k["max_regs_per_thread"])) <= 4


def test_k20c_threads_per_query():
    k = G["k20c"]
    mc = cfg.max_cur(k["num_sms"], k["max_threads_per_sm"])
    for name in ("arcene", "dor"):
        c = k[name]
        raw = cfg.threads_per_query_raw(c["nq"], k["r"], mc)
        assert raw == pytest.approx(c["raw"], rel=1e-3)
        assert cfg.threads_per_query(c["nq"], k["r"], mc) == c["tpq"]


def test_b200_numbers():
    b = G["b200"]
    assert cfg.th1(b["smem_per_sm"], b["max_threads_per_sm"]) == b["th1"]
    assert cfg.th2(b["max_regs_per_thread"]) == b["th2"]
    assert b["r"] * cfg.max_cur(b["num_sms"], b["max_threads_per_sm"]) == b["r_max_cur"]
    # placement per Fig. 8: k <= 28 in smem, k <= 255 in registers
    assert cfg.knearests_placement(28, b["th1"], b["th2"]) == "shared"
    assert cfg.knearests_placement(29, b["th1"], b["th2"]) == "registers"
    assert cfg.knearests_placement(255, b["th1"], b["th2"]) == "registers"
    assert cfg.knearests_placement(256, b["th1"], b["th2"]) == "global"


def test_filter_strength():
    for k, d, want in G["filter_strength"]["cases"]:
        assert cfg.filter_strength(k, d) == want
