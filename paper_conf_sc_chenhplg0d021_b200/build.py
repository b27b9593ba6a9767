"""Build libet.so (the C-ABI library) in-tree for sm_100a.

    python paper_conf_sc_chenhplg0d021_b200/build.py      (or __graft_entry__.build())

Every .cu under csrc/ is compiled with
    nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC
(NOT -arch=sm_100a: that emits compute_100 PTX and ptxas rejects tcgen05) and linked into
paper_conf_sc_chenhplg0d021_b200/libet.so with the static CUDA runtime.  Objects are cached
by source/header mtime in build/.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
DIAG = os.path.join(PKG, "diag")
INCLUDE = os.path.join(ROOT, "include")
BUILD = os.path.join(ROOT, "build", "et")
LIB = os.path.join(PKG, "libet.so")
DIAG_LIB = os.path.join(PKG, "libet_diag.so")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
         "--expt-relaxed-constexpr", "-I", INCLUDE, "-I", CSRC]


def _nvcc() -> str:
    for cand in (os.environ.get("NVCC"), shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found")


def _headers() -> list[str]:
    return glob.glob(os.path.join(CSRC, "**", "*.cuh"), recursive=True) + \
        glob.glob(os.path.join(CSRC, "**", "*.h"), recursive=True) + \
        glob.glob(os.path.join(INCLUDE, "*.h"))


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "**", "*.cu"), recursive=True))


def diag_sources() -> list[str]:
    return sorted(glob.glob(os.path.join(DIAG, "*.cu")))


def build_diag(verbose: bool = False) -> str:
    """Microbenchmark probes (diag/*.cu: M1 tcgen05 shapes, M1b issue / TMEM fill rates, TMA pull)
    in their own libet_diag.so, linked against libet.so; never loaded by the product path."""
    nvcc = _nvcc()
    bdir = BUILD + "_diag"
    os.makedirs(bdir, exist_ok=True)
    hdr_mtime = max([os.path.getmtime(h) for h in _headers()] + [0.0])
    objs = []
    for src in diag_sources():
        obj = os.path.join(bdir, os.path.basename(src) + ".o")
        objs.append(obj)
        if not os.path.exists(obj) or os.path.getmtime(obj) < max(os.path.getmtime(src), hdr_mtime):
            r = subprocess.run([nvcc, *ARCH, *FLAGS, "-c", src, "-o", obj], capture_output=True, text=True)
            if r.returncode != 0:
                raise RuntimeError("compile failed: " + src + "\n" + r.stdout + r.stderr)
    r = subprocess.run([nvcc, *ARCH, "-shared", "-o", DIAG_LIB, *objs, "-L", PKG, "-let", "-Xlinker",
                        "-rpath=$ORIGIN", "-lcudart_static", "-ldl", "-lrt", "-lpthread"],
                       capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("link failed: " + r.stdout + r.stderr)
    return DIAG_LIB


def build(verbose: bool = False, force: bool = False, debug: bool = False, variant: str | None = None,
          defines: tuple[str, ...] = (), only: str | None = None) -> str:
    """Compile every .cu and link libet.so (debug=True: -DET_WATCHDOG build into build/et_dbg/libet_dbg.so;
    variant=NAME: an experiment build with extra -D defines into build/et_var_NAME/libet.so; only=SUBSTR:
    compile just the sources whose name contains SUBSTR with those defines and link the main build's
    objects for the rest)."""
    nvcc = _nvcc()
    if variant:
        bdir = BUILD + "_var_" + variant
        lib = os.path.join(bdir, "libet.so")
    else:
        bdir = BUILD + ("_dbg" if debug else "")
        lib = os.path.join(bdir, "libet_dbg.so") if debug else LIB
    flags = FLAGS + (["-DET_WATCHDOG", "-DET_TIMELINE"] if debug else []) + ["-D" + d for d in defines]
    os.makedirs(bdir, exist_ok=True)
    hdr_mtime = max([os.path.getmtime(h) for h in _headers()] + [0.0])
    jobs = []
    objs = []
    for src in sources():
        rel = os.path.relpath(src, CSRC).replace(os.sep, "_")
        if variant and only and only not in rel:
            objs.append(os.path.join(BUILD, rel + ".o"))   # the main build's object
            continue
        obj = os.path.join(bdir, rel + ".o")
        objs.append(obj)
        if force or not os.path.exists(obj) or os.path.getmtime(obj) < max(os.path.getmtime(src), hdr_mtime):
            jobs.append([nvcc, *ARCH, *flags, "-c", src, "-o", obj])

    def run(cmd):
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("compile failed:\n" + " ".join(cmd) + "\n" + r.stdout + r.stderr)
        if verbose and (r.stdout or r.stderr):
            print(r.stdout + r.stderr, file=sys.stderr)

    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        list(ex.map(run, jobs))
    if jobs or force or not os.path.exists(lib) or os.path.getmtime(lib) < max(os.path.getmtime(o) for o in objs):
        tmp = lib + ".tmp"
        run([nvcc, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart_static", "-ldl",
             "-lrt", "-lpthread"])
        os.replace(tmp, lib)
    # the source revision the library was built from (bench.py reports it; the GPU box has no .git)
    try:
        sha = subprocess.run(["git", "rev-parse", "--short", "HEAD"], cwd=ROOT, capture_output=True, text=True,
                             timeout=5).stdout.strip()
        dirty = subprocess.run(["git", "status", "--porcelain", "--untracked-files=no"], cwd=ROOT,
                               capture_output=True, text=True, timeout=5).stdout.strip()
        if sha:
            with open(os.path.join(ROOT, "build", "BUILD_SHA"), "w") as fh:
                fh.write(sha + ("-dirty" if dirty else "") + "\n")
    except Exception:
        pass
    return lib


if __name__ == "__main__":
    var = sys.argv[sys.argv.index("--variant") + 1] if "--variant" in sys.argv else None
    defs = tuple(a[2:] for a in sys.argv if a.startswith("-D"))
    only = sys.argv[sys.argv.index("--only") + 1] if "--only" in sys.argv else None
    print(build(verbose=True, force="--force" in sys.argv, debug="--debug" in sys.argv, variant=var, defines=defs,
                only=only))
    if "--diag" in sys.argv:
        print(build_diag(verbose=True))
