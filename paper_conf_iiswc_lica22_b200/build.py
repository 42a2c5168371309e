"""Build libmg.so in-tree: nvcc for sm_100a (cross-compiles without a GPU).

    python -m paper_conf_iiswc_lica22_b200.build [--verbose] [--ptxas-v]

Output: paper_conf_iiswc_lica22_b200/libmg.so (statically linked CUDA runtime).
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(ROOT, "build", "mg")
LIB = os.path.join(PKG, "libmg.so")
# diagnostics variants: libmg_<name>.so with the matching -D flags, loaded via MG_LIB_VARIANT=<name>
VARIANTS = {"base": [],   # (a plain build under another name: A/B against a stashed source tree)
            "watchdog": ["-DMG_WATCHDOG"], "timeline": ["-DMG_TIMELINE"], "trace": ["-DMG_TRACE"],
            # A/B of the share of exponentials emulated on the FMA pipe (pairs of 16 per chunk)
            "e0": ["-DMG_EXP_EMU=0"], "e1": ["-DMG_EXP_EMU=1"], "e2": ["-DMG_EXP_EMU=2"], "e3": ["-DMG_EXP_EMU=3"], "e4": ["-DMG_EXP_EMU=4"], "e8": ["-DMG_EXP_EMU=8"],
            "maxpass": ["-DMG_SKIP_MAX=0"],
            # coarse softmax: 32-column chunks whose exponentials precede the P.V(n-1) wait
            "pre0": ["-DMG_PRE_CHUNKS=0"], "pre1": ["-DMG_PRE_CHUNKS=1"], "pre2": ["-DMG_PRE_CHUNKS=2"],
            # fine tensor-core kernel: cp.async ring stages per warp (default 2), min blocks per SM
            "fs3": ["-DMG_FINE_STAGES=3"], "fs4": ["-DMG_FINE_STAGES=4"], "fs3b4": ["-DMG_FINE_STAGES=3", "-DMG_FINE_MINB=4"], "fs3b6": ["-DMG_FINE_STAGES=3", "-DMG_FINE_MINB=6"], "fb4": ["-DMG_FINE_MINB=4"], "fb6": ["-DMG_FINE_MINB=6"],
            "fb8": ["-DMG_FINE_MINB=8"], "fp2": ["-DMG_FINE_PAIRS=2"], "fp2b3": ["-DMG_FINE_PAIRS=2", "-DMG_FINE_MINB=3"],
            "fw8": ["-DMG_FINE_WARPS=8", "-DMG_FINE_MINB=3"], "fw2": ["-DMG_FINE_WARPS=2", "-DMG_FINE_MINB=10"],
            "fw1": ["-DMG_FINE_WARPS=1", "-DMG_FINE_MINB=20"],
            # skeleton cost: no exponentials / no MMAs / no loads (results are garbage)
            "dbg1": ["-DMG_DBG=1"], "dbg2": ["-DMG_DBG=2"], "dbg3": ["-DMG_DBG=3"], "dbg7": ["-DMG_DBG=7"],
            "dbg8": ["-DMG_DBG=8"], "dbg16": ["-DMG_DBG=16"], "dbg24": ["-DMG_DBG=24"], "dbg25": ["-DMG_DBG=25"],
            "dbg31": ["-DMG_DBG=31"], "tl7": ["-DMG_TIMELINE", "-DMG_DBG=7"], "tl1": ["-DMG_TIMELINE", "-DMG_DBG=1"],
            "iq1": ["-DMG_IDLE_QUARTERS=1"], "ia0": ["-DMG_FINE_IDX_AHEAD=0"], "late1": ["-DMG_PV_LATE=1"], "ring0": ["-DMG_MASK_RING=0"], "cs128off": ["-DMG_CSPLIT128=0"], "tlate": ["-DMG_TIMELINE"], "swap0": ["-DMG_FINE_SWAP=0"], "vote0": ["-DMG_FINE_VOTE=0"], "items4": ["-DMG_ITEMS=4"], "fch4": ["-DMG_FINE_CHUNK=4"], "fch16": ["-DMG_FINE_CHUNK=16"], "fch64": ["-DMG_FINE_CHUNK=64"], "items3": ["-DMG_ITEMS=3"], "movm0": ["-DMG_FINE_MOVM=0"], "nsw": ["-DMG_DIAG_NO_STORE_WAIT"], "nswb": ["-DMG_DIAG_NO_STORE_WAIT", "-DMG_DIAG_NO_EPI_BAR"], "f2s3b2": ["-DMG_FINE_STAGES=3", "-DMG_FINE_MINB2=2"], "f2s2b2": ["-DMG_FINE_MINB2=2"], "f2s3b2w5": ["-DMG_FINE_STAGES=3", "-DMG_FINE_MINB2=2", "-DMG_FINE_WARPS=5"]}
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

SOURCES = ["plan.cpp", "api.cu", "coarse_pp_sm100.cu", "fine_rows.cu", "fine_mma.cu", "staged.cu", "selftest_umma.cu"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-fvisibility=hidden",
          "-I", os.path.join(ROOT, "include"), "-I", CSRC]


def _compile(src: str, extra: list[str], verbose: bool, bdir: str = BUILD) -> tuple[str, str]:
    obj = os.path.join(bdir, os.path.splitext(src)[0] + ".o")
    cmd = [NVCC, *ARCH, *COMMON, *extra, "-c", os.path.join(CSRC, src), "-o", obj]
    if verbose:
        print(" ".join(cmd))
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    return obj, r.stderr


def build(verbose: bool = False, ptxas_v: bool = False, variant: str = "") -> str:
    bdir = os.path.join(BUILD, variant) if variant else BUILD
    lib = os.path.join(PKG, f"libmg_{variant}.so") if variant else LIB
    os.makedirs(bdir, exist_ok=True)
    extra = ["-Xptxas", "-v"] if ptxas_v else []
    if variant:
        extra += VARIANTS[variant]
    if os.environ.get("MG_TIMELINE"):
        extra += ["-DMG_TIMELINE"]  # diagnostics build: per-item event clocks (tools/timeline_coarse.py)
    if os.environ.get("MG_WATCHDOG"):
        extra += ["-DMG_WATCHDOG"]  # diagnostics build: barrier waits trap with a report instead of hanging
    if os.environ.get("MG_TRACE"):
        extra += ["-DMG_TRACE"]  # diagnostics build: device event trace (tools/trace_coarse.py)
    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        results = list(ex.map(lambda s: _compile(s, extra, verbose, bdir), SOURCES))
    if ptxas_v:
        for _, log in results:
            if log.strip():
                print(log)
    objs = [o for o, _ in results]
    tmp = lib + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs,
           "-Xlinker", "--exclude-libs,ALL", "-lrt", "-ldl", "-lpthread"]
    if verbose:
        print(" ".join(cmd))
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--verbose", action="store_true")
    ap.add_argument("--ptxas-v", action="store_true")
    ap.add_argument("--variant", default="", choices=[""] + sorted(VARIANTS))
    a = ap.parse_args()
    print(build(a.verbose, a.ptxas_v, a.variant))
    sys.exit(0)
