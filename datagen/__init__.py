"""Seeded synthetic workload generators (C1-C5 of BASELINE.json).

This module holds NONE of the method's arithmetic: it only draws point sets.
It is the one module both the oracle side (tests, bench cpu_baseline) and the
CUDA side (tests, bench) use for inputs. Recipes are stated in DESIGN.md §4
and follow SURVEY.md §8(d) d.2 (shapes of the paper's UCI workloads, Table III
P:L655-687). All generators use ``numpy.random.default_rng(seed)`` and return
fp32 row-major arrays.
"""
from __future__ import annotations

import numpy as np

CONFIGS = {
    # name: (n, d, k, description)
    "C1": dict(n=1024, d=4, k=8, desc="tiny self-join, integer coords [0,255]^4"),
    "C2": dict(n=434_874, d=4, k=20, desc="3D road-network-shaped self-join (3DNet 434,874 x 4)"),
    "C3": dict(n=65_554, d=28, k=16, desc="KEGG-shaped self-join (65,554 x 28), 30% duplicate rows"),
    "C4": dict(n=1_000_000, d=128, k=16, desc="SIFT-like clustered Gaussian join, integer [0,255]"),
    "C5": dict(n=4_000_000, d=16, k=32, desc="large clustered join, integer [0,1023]"),
}


def c1_uniform_int(n: int = 1024, d: int = 4, seed: int = 1, hi: int = 255) -> np.ndarray:
    """C1: uniform integers in [0, hi]^d (d*hi^2 < 2^24 keeps squared distances exact in fp32)."""
    rng = np.random.default_rng(seed)
    return rng.integers(0, hi + 1, size=(n, d)).astype(np.float32)


def sphere_ties() -> np.ndarray:
    """C1-ties: all sign/permutation variants of (1,2,3,4)
    (384 points at distance sqrt(30) from the origin) followed by the origin."""
    import itertools
    pts = set()
    for perm in itertools.permutations((1, 2, 3, 4)):
        for signs in itertools.product((1, -1), repeat=4):
            pts.add(tuple(s * p for s, p in zip(signs, perm)))
    arr = np.array(sorted(pts), dtype=np.float32)
    assert arr.shape == (384, 4)
    return np.concatenate([arr, np.zeros((1, 4), np.float32)], axis=0)


def c2_road(n: int = 434_874, seed: int = 2) -> np.ndarray:
    """C2: 3D-road-network-shaped points (UCI 3D spatial network, 434,874 x 4).

    ~n/62 random-walk polylines ("roads", length 1+Poisson(61)) in a 3.2 x 1.3
    lon/lat-like box, step 3e-4 with heading noise 0.2 rad; z = smooth altitude
    field (6 random sinusoids, amplitude 0.05) + N(0, 2e-5); w = per-road
    constant U[0, 0.05]; 1% of points are exact duplicates (junctions).
    """
    rng = np.random.default_rng(seed)
    nroads = max(1, int(round(n / 62.0)))
    lengths = 1 + rng.poisson(61, size=nroads)
    while lengths.sum() < n:
        lengths = np.concatenate([lengths, 1 + rng.poisson(61, size=max(1, nroads // 10))])
    lengths = lengths[: np.searchsorted(np.cumsum(lengths), n) + 1]
    nroads = len(lengths)
    x0 = rng.uniform(0.0, 3.2, size=nroads)
    y0 = rng.uniform(0.0, 1.3, size=nroads)
    h0 = rng.uniform(0.0, 2 * np.pi, size=nroads)
    w_road = rng.uniform(0.0, 0.05, size=nroads)
    total = int(lengths.sum())
    road_id = np.repeat(np.arange(nroads), lengths)
    starts = np.concatenate([[0], np.cumsum(lengths)[:-1]])
    step_in_road = np.arange(total) - np.repeat(starts, lengths)
    dh = rng.normal(0.0, 0.2, size=total)
    dh[step_in_road == 0] = 0.0
    # heading = h0 + cumulative heading noise within each road
    cum = np.cumsum(dh)
    cum -= np.repeat(cum[starts], lengths)
    heading = h0[road_id] + cum
    stepx = 3e-4 * np.cos(heading)
    stepy = 3e-4 * np.sin(heading)
    stepx[step_in_road == 0] = 0.0
    stepy[step_in_road == 0] = 0.0
    cx = np.cumsum(stepx)
    cy = np.cumsum(stepy)
    cx -= np.repeat(cx[starts], lengths)
    cy -= np.repeat(cy[starts], lengths)
    x = x0[road_id] + cx
    y = y0[road_id] + cy
    # smooth altitude field: sum of 6 random sinusoids
    z = np.zeros(total)
    for _ in range(6):
        fx, fy = rng.uniform(0.5, 4.0, size=2)
        ph = rng.uniform(0, 2 * np.pi)
        z += np.sin(fx * x + fy * y + ph)
    z = 0.05 * z / 6.0 + rng.normal(0.0, 2e-5, size=total)
    w = w_road[road_id]
    X = np.stack([x, y, z, w], axis=1)[:n]
    # 1% exact duplicates at junctions
    ndup = n // 100
    dst = rng.choice(n, size=ndup, replace=False)
    src = rng.integers(0, n, size=ndup)
    X[dst] = X[src]
    return np.ascontiguousarray(X.astype(np.float32))


def c3_kegg(n: int = 65_554, d: int = 28, seed: int = 3, integer: bool = False) -> np.ndarray:
    """C3: KEGG-network-shaped heavy-tailed features (65,554 x 28, reading R18).

    latent s ~ LogNormal(2.5, 1); column c = a_c * s^{b_c} * LogNormal(0, 0.25)
    with b_c ~ U[0.5, 1.5], a_c log-uniform in [1e-2, 1e2]; columns 0..13 are
    rounded (counts), 14..27 real; 30% of rows are copies of random other rows.
    integer=True (C3-int): clip to [0, 700] and round (28*700^2 < 2^24).
    """
    rng = np.random.default_rng(seed)
    s = rng.lognormal(2.5, 1.0, size=n)
    b = rng.uniform(0.5, 1.5, size=d)
    a = 10.0 ** rng.uniform(-2.0, 2.0, size=d)
    X = a[None, :] * s[:, None] ** b[None, :] * rng.lognormal(0.0, 0.25, size=(n, d))
    X[:, : min(14, d)] = np.round(X[:, : min(14, d)])
    ndup = int(0.3 * n)
    dst = rng.choice(n, size=ndup, replace=False)
    src = rng.integers(0, n, size=ndup)
    X[dst] = X[src]
    if integer:
        X = np.round(np.clip(X, 0, 700))
    return np.ascontiguousarray(X.astype(np.float32))


def gaussian_blobs(n: int, d: int, nblobs: int, lo: float, hi: float, sig_lo: float,
                   sig_hi: float, clip_hi: float, centers_seed: int, seed: int,
                   margin: float = 0.0) -> np.ndarray:
    """Integer-valued Gaussian mixture: blob centers U[lo+margin, hi-margin]^d,
    sigma_c ~ U[sig_lo, sig_hi], weights ~ Dirichlet(2); samples rounded and
    clipped to [0, clip_hi]."""
    crng = np.random.default_rng(centers_seed)
    centers = crng.uniform(lo + margin, hi - margin, size=(nblobs, d))
    sig = crng.uniform(sig_lo, sig_hi, size=nblobs)
    wts = crng.dirichlet(np.full(nblobs, 2.0))
    rng = np.random.default_rng(seed)
    lab = rng.choice(nblobs, size=n, p=wts)
    X = np.empty((n, d), dtype=np.float32)
    chunk = 1 << 18
    for s0 in range(0, n, chunk):
        s1 = min(n, s0 + chunk)
        l = lab[s0:s1]
        v = centers[l] + sig[l, None] * rng.standard_normal((s1 - s0, d))
        X[s0:s1] = np.round(np.clip(v, 0, clip_hi))
    return X


def c4_sift(n: int = 1_000_000, d: int = 128, which: str = "T") -> np.ndarray:
    """C4: SIFT-like clustered Gaussian, 1000 blobs, centers U[20,235]^128,
    sigma U[8,24], integer in [0,255] (128*255^2 < 2^24). Q and T are
    independent draws (seeds 40 / 41; centers seed 4)."""
    return gaussian_blobs(n, d, 1000, 20.0, 235.0, 8.0, 24.0, 255.0, 4,
                          40 if which == "Q" else 41)


def c5_blobs(n: int = 4_000_000, d: int = 16, which: str = "T") -> np.ndarray:
    """C5: 4000 blobs, centers U[0,1023]^16, sigma U[10,40], integer in
    [0,1023] (16*1023^2 < 2^24). Q / T seeds 50 / 51; centers seed 5."""
    return gaussian_blobs(n, d, 4000, 0.0, 1023.0, 10.0, 40.0, 1023.0, 5,
                          50 if which == "Q" else 51)


def workload(name: str, scale: float = 1.0):
    """Return (Q, T, k, self_join) for a named config; ``scale`` < 1 shrinks n
    (parity tests at sizes the oracle finishes in seconds)."""
    if name[0] in "GK" and name[1:].isdigit():
        # ablation shapes (not bench configs): G<d> = 200,000-point integer blob
        # self-join (C5 recipe, 1,000 blobs), K<d> = C3's KEGG recipe at dimension d
        d = int(name[1:])
        if name[0] == "G":
            X = gaussian_blobs(max(16, int(round(200_000 * scale))), d, 1000, 0.0, 1023.0, 10.0, 40.0, 1023.0, 7, 70)
        else:
            X = c3_kegg(max(16, int(round(65_554 * scale))), d=d)
        return X, X, 16, True
    if name in ("ARC", "DOR"):
        # high-d shapes of Table III, not bench configs: arcene-like
        # 100 x 10,000 (dense integer intensities 0..999, a few latent
        # prototypes) and dorothea-like 1,950 x 100,000 (sparse binary, ~1%
        # ones, rows near a few prototypes); integer-valued, self-joins, k = 8
        X = high_d(name, scale)
        return X, X, 8, True
    cfg = CONFIGS[name.replace("int", "")]
    n = max(16, int(round(cfg["n"] * scale)))
    k = cfg["k"]
    if name == "C1":
        X = c1_uniform_int(n)
        return X, X, k, True
    if name == "C2":
        X = c2_road(n)
        return X, X, k, True
    if name == "C3":
        X = c3_kegg(n)
        return X, X, k, True
    if name == "C3int":
        X = c3_kegg(n, integer=True)
        return X, X, k, True
    if name == "C4":
        return c4_sift(n, which="Q"), c4_sift(n, which="T"), k, False
    if name == "C5":
        return c5_blobs(n, which="Q"), c5_blobs(n, which="T"), k, False
    raise KeyError(name)


def high_d(name: str, scale: float = 1.0, seed: int = 11) -> np.ndarray:
    """ARC (arcene-like) or DOR (dorothea-like) rows; see workload()."""
    rng = np.random.default_rng(seed)
    if name == "ARC":
        n, d = max(16, int(round(100 * scale))), 10_000
        protos = rng.integers(0, 1000, size=(4, d))
        X = protos[rng.integers(0, 4, size=n)] + rng.integers(-60, 61, size=(n, d))
        return np.clip(X, 0, 999).astype(np.float32)
    n, d = max(16, int(round(1950 * scale))), 100_000
    protos = rng.random((8, d)) < 0.01
    X = protos[rng.integers(0, 8, size=n)]
    flip = rng.random((n, d)) < 0.002
    return np.logical_xor(X, flip).astype(np.float32)
