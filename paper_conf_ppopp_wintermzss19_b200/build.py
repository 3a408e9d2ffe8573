"""Build libacspgemm.so in-tree for sm_100a (nvcc; no JIT, no torch extension).

The .so is loaded with ctypes by the binding (`_lib.py`); it exports the C ABI of
include/acspgemm.h.  Objects are compiled in parallel, then linked with nvcc.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
# ACS_BUILD_TAG builds a variant (with ACS_EXTRA_NVCC_FLAGS) into build_<tag>/libacspgemm_<tag>.so
_TAG = os.environ.get("ACS_BUILD_TAG", "")
BUILD = os.path.join(HERE, "build" + (f"_{_TAG}" if _TAG else ""))
SO = os.path.join(HERE, "libacspgemm" + (f"_{_TAG}" if _TAG else "") + ".so")
SOURCES = ["glb.cu", "scan.cu", "esc.cu", "esc_small.cu", "hash.cu", "dict.cu", "rows.cu", "merge.cu", "copy.cu", "plan.cu"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr", "-ftz=false", "-prec-div=true",
         "-prec-sqrt=true", "-fmad=true"] + os.environ.get("ACS_EXTRA_NVCC_FLAGS", "").split()


def _stale(obj: str, deps) -> bool:
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return any(os.path.getmtime(d) > t for d in deps)


def _flags_changed() -> bool:
    """True when the nvcc flags differ from the ones the objects in BUILD were built with
    (a -D knob in ACS_EXTRA_NVCC_FLAGS must not reuse objects of another variant)."""
    stamp = os.path.join(BUILD, "FLAGS")
    want = " ".join(FLAGS)
    have = open(stamp).read() if os.path.exists(stamp) else None
    return have != want


def build(verbose: bool = False, ptxas_v: bool = False, force: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    force = force or _flags_changed()
    headers = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".cuh")]
    headers.append(os.path.join(os.path.dirname(HERE), "include", "acspgemm.h"))
    jobs = []
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(BUILD, src.replace(".cu", ".o"))
        if force or ptxas_v or _stale(o, [s] + headers):
            cmd = [NVCC] + FLAGS + (["-Xptxas", "-v"] if ptxas_v else []) + ["-c", s, "-o", o]
            jobs.append(cmd)
    def run(cmd):
        r = subprocess.run(cmd, capture_output=True, text=True)
        return cmd, r
    with cf.ThreadPoolExecutor(max_workers=min(8, max(1, len(jobs)))) as ex:
        for cmd, r in ex.map(run, jobs):
            if verbose or ptxas_v or r.returncode:
                sys.stderr.write(r.stdout + r.stderr)
            if r.returncode:
                raise RuntimeError("nvcc failed: " + " ".join(cmd))
    with open(os.path.join(BUILD, "FLAGS"), "w") as f:
        f.write(" ".join(FLAGS))
    objs = [os.path.join(BUILD, s.replace(".cu", ".o")) for s in SOURCES]
    if force or jobs or _stale(SO, objs):
        cmd = [NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", SO] + objs + ["-lcudart"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("link failed")
    return SO


if __name__ == "__main__":
    build(verbose=True, ptxas_v="-v" in sys.argv, force="-f" in sys.argv)
    print(SO)
