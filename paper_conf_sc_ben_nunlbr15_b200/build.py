"""Build libmapsm.so in-tree (sm_100a only) with nvcc.

Used by ``__graft_entry__.build()`` and runnable as ``python -m
paper_conf_sc_ben_nunlbr15_b200.build``.  Rebuilds only when a source or
header is newer than the library.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libmapsm.so")
OBJ = os.path.join(PKG, "_build")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
# No --use_fast_math: the fp32 path must keep IEEE fmaf semantics (reading c11).
NVFLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
           "--fmad=true", "-Xptxas", "-O3"]


def _nccl_include() -> str:
    import importlib.util

    spec = importlib.util.find_spec("nvidia")
    for base in list(spec.submodule_search_locations or []):
        inc = os.path.join(base, "nccl", "include")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc
    if os.path.exists("/usr/include/nccl.h"):
        return "/usr/include"
    raise RuntimeError("nccl.h not found")


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def _deps():
    return (_sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh"))
            + [os.path.join(INCLUDE, "mapsm.h"), __file__])


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in _deps())


def build(force: bool = False, verbose: bool = False, out: str | None = None, csrc: str | None = None,
          extra: list[str] | None = None) -> str:
    """Build the library.  ``out``/``csrc``/``extra`` build a tuning variant
    from another source tree with extra nvcc flags (tools/ only)."""
    lib_path = out or LIB
    if out is None and not force and not needs_build():
        return LIB
    src_dir = csrc or CSRC
    obj_dir = os.path.join(os.path.dirname(lib_path), "_build") if out else OBJ
    os.makedirs(obj_dir, exist_ok=True)
    nvcc = os.environ.get("NVCC", "nvcc")
    incs = ["-I", INCLUDE, "-I", src_dir, "-I", _nccl_include()]
    srcs = sorted(glob.glob(os.path.join(src_dir, "*.cu")) + glob.glob(os.path.join(src_dir, "*.cpp")))
    # incremental: a translation unit recompiles when it is newer than its
    # object or any shared header / build flag source changed
    hdr_t = max(os.path.getmtime(p) for p in
                glob.glob(os.path.join(src_dir, "*.h")) + glob.glob(os.path.join(src_dir, "*.cuh"))
                + [os.path.join(INCLUDE, "mapsm.h"), __file__])
    objs, cmds = [], []
    for src in srcs:
        obj = os.path.join(obj_dir, os.path.basename(src) + ".o")
        objs.append(obj)
        if (not force and os.path.exists(obj)
                and os.path.getmtime(obj) > max(os.path.getmtime(src), hdr_t)):
            continue
        cmds.append([nvcc, *ARCH, *NVFLAGS, *(extra or []), *incs, "-c", src, "-o", obj])
    # translation units compile in parallel (the conv radii are the slow ones)
    from concurrent.futures import ThreadPoolExecutor

    def run(cmd):
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        return subprocess.run(cmd, capture_output=not verbose, text=True)

    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        results = list(ex.map(run, cmds))
    for cmd, res in zip(cmds, results):
        if res.returncode != 0:
            if not verbose:
                sys.stderr.write(res.stdout or "")
                sys.stderr.write(res.stderr or "")
            raise subprocess.CalledProcessError(res.returncode, cmd)
    tmp = lib_path + ".tmp"
    cmd = [nvcc, *ARCH, "-shared", "-o", tmp, *objs, "-ldl", "-lpthread"]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, lib_path)
    return lib_path


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
