"""Build the sm_100a C-ABI library libeirene.so in-tree with nvcc.

    python -m paper_conf_ppopp_zhangz0lzl23_b200.build [--force] [--verbose]

Every .cu under csrc/ is compiled with
  -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -Xcompiler -fPIC
and linked (static cudart) into paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
OBJ = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libeirene.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC", "-I", INCLUDE, "-I", CSRC]


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _deps():
    return _sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(INCLUDE, "eirene.h")]


def _stale(target: str, deps) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, variant: str = "", defines: tuple = ()) -> str:
    """Build libeirene.so; a `variant` (A/B or diagnostic build, e.g. -DEIRENE_PHASE_PROF) goes to
    _build_<variant>/ and libeirene_<variant>.so, selected at run time with EIRENE_LIB."""
    OBJ = os.path.join(PKG, "_build" + (f"_{variant}" if variant else ""))
    LIB = os.path.join(PKG, {"": "libeirene.so", "32": "libeirene32.so"}.get(variant, f"libeirene_{variant}.so"))
    flags = FLAGS + [f"-D{d}" for d in defines]
    os.makedirs(OBJ, exist_ok=True)
    headers = glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(INCLUDE, "eirene.h")]
    jobs = []
    objs = []
    for src in _sources():
        obj = os.path.join(OBJ, os.path.basename(src)[:-3] + ".o")
        objs.append(obj)
        if force or _stale(obj, [src] + headers):
            cmd = [NVCC, *ARCH, *flags, "-Xptxas", "-v", "-c", src, "-o", obj]
            jobs.append((src, cmd))

    def run(job):
        src, cmd = job
        p = subprocess.run(cmd, capture_output=True, text=True)
        with open(os.path.join(OBJ, os.path.basename(src) + ".ptxas.log"), "w") as f:
            f.write(p.stdout + p.stderr)
        if p.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{p.stdout}\n{p.stderr}")
        return src

    if jobs:
        with cf.ThreadPoolExecutor(max_workers=min(8, len(jobs))) as ex:
            for src in ex.map(run, jobs):
                if verbose:
                    print("compiled", os.path.relpath(src, ROOT))
    if force or jobs or _stale(LIB, objs):
        tmp = LIB + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-cudart", "static"]
        p = subprocess.run(cmd, capture_output=True, text=True)
        if p.returncode != 0:
            raise RuntimeError(f"link failed:\n{p.stdout}\n{p.stderr}")
        os.replace(tmp, LIB)
        if verbose:
            print("linked", os.path.relpath(LIB, ROOT))
    return LIB


def build_all(force: bool = False, verbose: bool = False) -> list[str]:
    """The product libraries: libeirene.so (64-bit keys / values) and libeirene32.so
    (-DEIRENE_KEY32: 32-bit keys / values)."""
    return [build(force, verbose), build(force, verbose, variant="32", defines=("EIRENE_KEY32",))]


if __name__ == "__main__":
    # python -m paper_conf_ppopp_zhangz0lzl23_b200.build [--force] [--variant NAME -DX ...]
    a = sys.argv[1:]
    var = a[a.index("--variant") + 1] if "--variant" in a else ""
    if var or any(x.startswith("-D") for x in a):
        build(force="--force" in a, verbose=True, variant=var, defines=tuple(x[2:] for x in a if x.startswith("-D")))
    else:
        build_all(force="--force" in a, verbose=True)
