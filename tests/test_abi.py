"""C-ABI library checks that need no GPU: the library loads, exports every
symbol include/sknn.h declares, validates arguments before touching a device,
and its adaptive-scheme arithmetic matches the oracle's on the paper's fixtures."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_icde_chends17_b200 as sknn
from oracle import config as ocfg
from sknn_testutil import load_golden, ROOT

HEADER = os.path.join(ROOT, "include", "sknn.h")


@pytest.fixture(scope="module")
def L():
    from paper_conf_icde_chends17_b200 import buildlib as b
    b.build()
    return sknn.lib()


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sknn_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_abi():
    names = declared_functions()
    assert set(names) == set(sknn.ABI_SYMBOLS), names


def test_exports_every_symbol(L):
    for name in declared_functions():
        assert hasattr(L, name), name


def test_library_is_sm100a_only():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", sknn.LIB_PATH], capture_output=True,
                         text=True).stdout
    archs = set(re.findall(r"sm_(\d+a?)", out))
    assert archs == {"100a"}, archs


def test_version_and_error_strings(L):
    assert sknn.version() == (0, 1)
    assert L.sknn_error_string(-1) == b"SKNN_ERR_INVALID_ARG"
    assert L.sknn_error_string(0) == b"SKNN_OK"


@pytest.mark.parametrize("nq,nt,d,k,msg", [
    (4, 4, 2, 5, "k > nt"), (4, 4, 2, 0, "k <= 0"), (4, 4, 0, 1, "d <= 0"), (-1, 4, 2, 1, "nq < 0"),
    (4, 0, 2, 1, "nt <= 0")])
def test_invalid_arguments_rejected_before_device(L, nq, nt, d, k, msg):
    Q = np.zeros((max(nq, 1), max(d, 1)), np.float32)
    out = np.zeros((max(nq, 1), max(k, 1)), np.float32)
    st = L.sknn_join(Q.ctypes.data, nq, Q.ctypes.data, nt, d, k, None, out.ctypes.data, None)
    assert st == -1
    assert msg in L.sknn_last_error().decode()


def test_null_pointers_rejected(L):
    out = np.zeros((1, 1), np.float32)
    assert L.sknn_join(None, 1, None, 1, 1, 1, None, out.ctypes.data, None) == -1
    assert L.sknn_query(None, None, 1, 1, None, None, None, None, None) == -1
    assert L.sknn_index_free(None) == 0


def test_k_above_max_unsupported(L):
    Q = np.zeros((1000, 2), np.float32)
    out = np.zeros((1000, 513), np.float32)
    assert L.sknn_join(Q.ctypes.data, 1000, Q.ctypes.data, 1000, 2, 513, None, out.ctypes.data, None) == -5


def test_nq_zero_is_noop(L):
    T = np.zeros((4, 2), np.float32)
    out = np.zeros((1, 1), np.float32)
    assert L.sknn_join(T.ctypes.data, 0, T.ctypes.data, 4, 2, 1, None, out.ctypes.data, None) == 0


def test_config_decide_matches_oracle_k20c(L):
    g = load_golden("adaptive_config.json")["k20c"]
    props = dict(num_sms=g["num_sms"], max_threads_per_sm=g["max_threads_per_sm"], smem_per_sm=g["smem_per_sm"],
                 max_regs_per_thread=g["max_regs_per_thread"])
    for name in ("arcene", "dor"):
        c = sknn.config_decide(g[name]["nq"], g[name]["nq"], 4, 20, props=props, r_factor=g["r"])
        assert c["th1_bytes"] == g["th1"] == ocfg.th1(g["smem_per_sm"], g["max_threads_per_sm"])
        assert c["th2_bytes"] == g["th2_formula"] == ocfg.th2(g["max_regs_per_thread"])
        assert c["threads_per_query"] == g[name]["tpq"]
        mc = ocfg.max_cur(g["num_sms"], g["max_threads_per_sm"])
        assert c["tpq_raw"] == pytest.approx(ocfg.threads_per_query_raw(g[name]["nq"], g["r"], mc))


def test_config_decide_matches_oracle_b200(L):
    g = load_golden("adaptive_config.json")["b200"]
    props = dict(num_sms=g["num_sms"], max_threads_per_sm=g["max_threads_per_sm"], smem_per_sm=g["smem_per_sm"],
                 max_regs_per_thread=g["max_regs_per_thread"])
    for (nq, d, k) in [(434_874, 4, 20), (65_554, 28, 16), (1_000_000, 128, 16), (4_000_000, 16, 32), (1024, 4, 8)]:
        c = sknn.config_decide(nq, nq, d, k, props=props)
        assert c["th1_bytes"] == g["th1"] and c["th2_bytes"] == g["th2"]
        assert c["r_max_cur"] == g["r_max_cur"]
        placement = ["shared", "registers", "global"][c["placement"]]
        assert placement == ocfg.knearests_placement(k, g["th1"], g["th2"])
        assert bool(c["partial_filter"]) == (ocfg.filter_strength(k, d) == "partial")
        assert c["threads_per_query"] == ocfg.threads_per_query(nq, 0.25, ocfg.max_cur(148, 2048))
        assert c["mq"] == min(8192, int(np.floor(3 * np.sqrt(nq))))
    # mapping (B200 rule): thread-per-query for dp <= 32 (C1, C2, C3, C5), warp-per-query for C4 (dp = 128)
    assert sknn.config_decide(434_874, 434_874, 4, 20, props=props)["mapping"] == 1
    assert sknn.config_decide(4_000_000, 4_000_000, 16, 32, props=props)["mapping"] == 1
    assert sknn.config_decide(65_554, 65_554, 28, 16, props=props)["mapping"] == 1  # B200 rule: dp <= 32
    assert sknn.config_decide(1_000_000, 1_000_000, 128, 16, props=props)["mapping"] == 2


def test_struct_layouts_match_the_header(L):
    """The ctypes mirrors of sknn_options / sknn_stats have the C sizes
    (sknn_options_default writes sizeof(sknn_options) into struct_size)."""
    o = sknn.make_options()
    assert o.struct_size == ctypes.sizeof(sknn.Options)
    # sknn_stats: the last field (dense_terms + pad) closes an 8-byte-aligned struct
    assert ctypes.sizeof(sknn.Stats) % 8 == 0
    assert sknn.Stats.dense_terms.offset == sknn.Stats.rows_loaded.offset + 8
