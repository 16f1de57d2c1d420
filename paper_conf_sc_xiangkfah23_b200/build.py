"""Build libcualign_bp.so in-tree for sm_100a (nvcc; no torch in the library).

    python -m paper_conf_sc_xiangkfah23_b200.build [--verbose] [--probes]

--probes builds lib/libcualign_bp_probes.so instead: the same sources with
-DCUALIGN_PROBES, which reads measurement knobs (timing probes that skip work,
alternative launch shapes; see probe_knob in csrc/internal.cuh) from the
environment.  Only tools/ load it (CUALIGN_LIB=...); the product library never
reads the environment.

--fmad=false: products and sums are rounded as written (no FMA contraction),
the same arithmetic as the oracle's -ffp-contract=off.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIBDIR = os.path.join(HERE, "lib")
LIB = os.path.join(LIBDIR, "libcualign_bp.so")
PROBE_LIB = os.path.join(LIBDIR, "libcualign_bp_probes.so")
INCLUDE = os.path.join(os.path.dirname(HERE), "include")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "--fmad=false", "-std=c++17",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-O2",
    "--expt-relaxed-constexpr",
]


def nvcc() -> str:
    for cand in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if cand and (os.path.sep not in cand or os.path.exists(cand)):
            return cand
    return "nvcc"


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale(lib) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(INCLUDE, "cualign_bp.h")]
    return any(os.path.getmtime(p) > t for p in deps)


def build(force: bool = False, verbose: bool = False, probes: bool = False) -> str:
    lib = PROBE_LIB if probes else LIB
    if not force and not _stale(lib):
        return lib
    os.makedirs(LIBDIR, exist_ok=True)
    objs = []
    cmds = []
    tag = ".probes" if probes else ""
    for src in sources():
        obj = os.path.join(LIBDIR, os.path.basename(src)[:-3] + tag + ".o")
        cmd = [nvcc(), *NVCC_FLAGS, *(["-DCUALIGN_PROBES"] if probes else []), "-I", INCLUDE, "-c", src, "-o", obj]
        if verbose:
            cmd += ["-Xptxas", "-v"]
            print(" ".join(cmd), flush=True)
        cmds.append(cmd)
        objs.append(obj)
    # translation units are independent: compile them concurrently
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=min(len(cmds), os.cpu_count() or 1)) as ex:
        for f in [ex.submit(subprocess.check_call, c) for c in cmds]:
            f.result()
    tmp = lib + ".tmp%d" % os.getpid()
    cmd = [nvcc(), "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, *objs,
           "-Xcompiler", "-fPIC", "-ldl"]
    if verbose:
        print(" ".join(cmd), flush=True)
    subprocess.check_call(cmd)
    os.replace(tmp, lib)
    for o in objs:
        os.remove(o)
    return lib


if __name__ == "__main__":
    print(build(force=True, verbose="--verbose" in sys.argv, probes="--probes" in sys.argv))
