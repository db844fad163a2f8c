"""Build libks.so (the C-ABI library) in-tree with nvcc for sm_100a.

    python -m paper_conf_icppw_wangkbgj16_b200.build [--force]

Every .cu under csrc/ is compiled with
``-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo`` and linked into
``paper_conf_icppw_wangkbgj16_b200/libks.so`` (cudart static, so the library
only needs the driver at run time).  Objects are rebuilt when a source or any
header is newer.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libks.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
         "--expt-relaxed-constexpr", "-I", os.path.join(ROOT, "include"), "-I", CSRC] + \
    os.environ.get("KS_EXTRA_NVCC", "").split()  # e.g. -DKS_PROF=1 (phase profiling build)


def _headers():
    return glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + \
        glob.glob(os.path.join(ROOT, "include", "*.h"))


def build(force: bool = False, verbose: bool = False, extra=None, lib: str = None, build_dir: str = None) -> str:
    """Compile csrc/*.cu (in parallel) and link the library.  `extra` adds nvcc flags (the
    measurement library: build_debug()); `lib` / `build_dir` default to libks.so / _build."""
    from concurrent.futures import ThreadPoolExecutor
    lib = lib or LIB
    build_dir = build_dir or BUILD
    flags = FLAGS + list(extra or [])
    os.makedirs(build_dir, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    hdr_mtime = max([os.path.getmtime(h) for h in _headers()] + [0])
    objs, cmds = [], []
    for s in srcs:
        o = os.path.join(build_dir, os.path.basename(s)[:-3] + ".o")
        objs.append(o)
        if force or not os.path.exists(o) or os.path.getmtime(o) < max(os.path.getmtime(s), hdr_mtime):
            cmd = [NVCC, *ARCH, *flags, "-c", s, "-o", o]
            if verbose:
                cmd.insert(1, "-Xptxas=-v")
                print(" ".join(cmd), flush=True)
            cmds.append(cmd)
    if cmds:
        with ThreadPoolExecutor(max_workers=min(len(cmds), os.cpu_count() or 1)) as ex:
            for f in [ex.submit(subprocess.check_call, c) for c in cmds]:
                f.result()
    if force or not os.path.exists(lib) or os.path.getmtime(lib) < max(os.path.getmtime(o) for o in objs):
        tmp = lib + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, *ARCH, "-shared", "-cudart", "static", *objs, "-o", tmp])
        os.replace(tmp, lib)
    return lib


DBG_LIB = os.path.join(PKG, "libks_dbg.so")


def build_debug(debug: int = 1, prof: int = 0, trace: int = 0, force: bool = False) -> str:
    """The measurement library libks_dbg.so (never the shipped libks.so; selected with
    KS_LIB=libks_dbg.so): KS_DEBUG work-dropping knobs and bounded waits, KS_PROF phase clocks,
    KS_TRACE unit timeline.  Objects are rebuilt when the flags change."""
    flags = [f"-DKS_DEBUG={debug}", f"-DKS_PROF={prof}", f"-DKS_TRACE={trace}"]
    bdir = BUILD + "_dbg"
    stamp = os.path.join(bdir, "flags")
    os.makedirs(bdir, exist_ok=True)
    old = open(stamp).read() if os.path.exists(stamp) else ""
    if old != " ".join(flags):
        force = True
    lib = build(force=force, extra=flags, lib=DBG_LIB, build_dir=bdir)
    with open(stamp, "w") as f:
        f.write(" ".join(flags))
    return lib


if __name__ == "__main__":
    if "--debug" in sys.argv:
        print(build_debug(force="--force" in sys.argv))
    else:
        print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
