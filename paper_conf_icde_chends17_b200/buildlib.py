"""Build libsweetknn.so (the C-ABI library) in-tree with nvcc for sm_100a.

    python -m paper_conf_icde_chends17_b200.buildlib [--verbose] [--force]

Every kernel is compiled for `-gencode arch=compute_100a,code=sm_100a` with
-lineinfo (so ncu source pages map to the .cu lines). No fast-math: the
distance arithmetic relies on IEEE fp32 sqrt and explicit fma.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(os.path.dirname(HERE), "include")
LIB = os.path.join(HERE, "libsweetknn.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        glob.glob(os.path.join(INCLUDE, "*.h"))
    return any(os.path.getmtime(p) > t for p in deps)


def build(force: bool = False, verbose: bool = False, out: str = None) -> str:
    """Build the library (to `out`, default in-tree). NVCC_EXTRA adds compiler
    flags, e.g. -D tuning macros for an A/B variant built into abl/."""
    extra = os.environ.get("NVCC_EXTRA", "").split()
    lib = out or LIB
    if not force and not extra and lib == LIB and not _stale():
        return LIB
    objdir = os.path.join(HERE, "build" + ("_" + str(abs(hash(" ".join(extra))) % 10**8) if extra else ""))
    os.makedirs(objdir, exist_ok=True)
    common = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-I", INCLUDE,
                     "--expt-relaxed-constexpr"] + extra
    if verbose:
        common += ["-Xptxas", "-v"]
    objs = []
    procs = []
    hdr = glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        glob.glob(os.path.join(INCLUDE, "*.h")) + [os.path.abspath(__file__)]
    hdr_t = max(os.path.getmtime(h) for h in hdr)
    for src in sources():
        obj = os.path.join(objdir, os.path.basename(src)[:-3] + ".o")
        objs.append(obj)
        # incremental: an object newer than its source and every header is kept
        # (flags are part of objdir's name, so a flag change never reuses one)
        if not force and os.path.exists(obj) and os.path.getmtime(obj) > max(os.path.getmtime(src), hdr_t):
            continue
        cmd = [NVCC, "-c", src, "-o", obj] + common
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
    failed = False
    for cmd, p in procs:
        out, _ = p.communicate()
        if out and (verbose or p.returncode):
            sys.stderr.write(out.decode(errors="replace"))
        if p.returncode:
            sys.stderr.write("FAILED: %s\n" % " ".join(cmd))
            failed = True
    if failed:
        raise RuntimeError("nvcc failed building libsweetknn.so")
    tmp = lib + ".tmp.%d" % os.getpid()
    subprocess.check_call([NVCC] + ARCH + ["-shared", "-o", tmp] + objs + ["-lcudart_static"])
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    out = None
    if "--out" in sys.argv:
        out = os.path.abspath(sys.argv[sys.argv.index("--out") + 1])
        os.makedirs(os.path.dirname(out), exist_ok=True)
    print(build(force="--force" in sys.argv, verbose="--verbose" in sys.argv, out=out))
