"""The paper's adaptive-scheme arithmetic (Fig. 8, §IV-D), written out.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py). The product computes the
same decisions in C++ (``sknn_config_decide`` in
paper_conf_icde_chends17_b200/csrc/api.cu); tests pin this module to the
numbers the paper prints for the K20c and to the B200
fixture, and compare the product with it on both.

Citations: P:L<n> = PAPER.md line n.
"""
from __future__ import annotations

import math


def th1(smem_per_sm_bytes: int, max_threads_per_sm: int) -> int:
    """th1 = shared mem size / max currPerSM (§IV-D2). K20c: 48KB/2048 = 24."""
    return smem_per_sm_bytes // max_threads_per_sm


def th2(max_regs_per_thread: int) -> int:
    """th2 = max regPerThread * 4 bytes. K20c: 255*4 = 1020; the paper prints 1024 (reading R14)."""
    return max_regs_per_thread * 4


def knearests_placement(k: int, th1_bytes: int, th2_bytes: int) -> str:
    """Fig. 8 lower branch: k*4 <= th1 -> shared; k*4 > th2 -> global; otherwise registers."""
    if k * 4 <= th1_bytes:
        return "shared"
    if k * 4 > th2_bytes:
        return "global"
    return "registers"


def filter_strength(k: int, d: int) -> str:
    """Fig. 8 top and §IV-D1: partial level-2 filter iff k/d > 8 (reading R13)."""
    return "partial" if k > 8 * d else "full"


def max_cur(num_sms: int, max_threads_per_sm: int) -> int:
    """max_cur: threads concurrently active on the GPU, at full occupancy."""
    return num_sms * max_threads_per_sm


def threads_per_query_raw(nq: int, r: float, maxcur: int) -> float:
    """|Q| >= r*max_cur -> 1 (query-level parallelism); else r*max_cur/|Q| threads per query."""
    if nq >= r * maxcur:
        return 1.0
    return r * maxcur / nq


def round_pow2_log(x: float) -> int:
    """Reading R15: nearest power of two in log2 (66.56 -> 64, 3.41 -> 4)."""
    if x <= 1.0:
        return 1
    return 1 << int(round(math.log2(x)))


def threads_per_query(nq: int, r: float, maxcur: int, cap: int | None = None) -> int:
    t = round_pow2_log(threads_per_query_raw(nq, r, maxcur))
    return min(t, cap) if cap else t

