"""Build libgraffix.so in-tree with nvcc for sm_100a (no torch dependency).

    python -m paper_conf_icpp_0001n20_b200.build [--force] [--jobs N]
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import hashlib
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
OUT = os.environ.get("GX_BUILD_OUT") or os.path.join(HERE, "libgraffix.so")
OBJ = os.environ.get("GX_BUILD_OBJ") or os.path.join(HERE, "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-fopenmp,-O3", "-I" + os.path.join(HERE, "..", "include")] + \
    os.environ.get("GX_NVCC_EXTRA", "").split()


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def _headers():
    return glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        glob.glob(os.path.join(HERE, "..", "include", "*.h"))


def _compile(src: str, force: bool, extra) -> str:
    obj = os.path.join(OBJ, os.path.basename(src) + ".o")
    hdr_t = max((os.path.getmtime(h) for h in _headers()), default=0)
    if not force and os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(src), hdr_t):
        return obj
    cmd = [NVCC] + ARCH + COMMON + list(extra) + ["-c", src, "-o", obj]
    if src.endswith(".cu"):
        cmd += ["-Xptxas", "-v"] if os.environ.get("GX_PTXAS_V") else []
    else:
        cmd += ["-x", "cu"] if False else []
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    if r.stderr.strip() and os.environ.get("GX_VERBOSE"):
        print(r.stderr, file=sys.stderr)
    return obj


def _flags_stamp(extra) -> str:
    """Hash of everything that changes the objects besides the sources: the
    compiler, the arch and the full flag set (GX_NVCC_EXTRA and ``extra``)."""
    return hashlib.sha256(repr((NVCC, ARCH, COMMON, list(extra))).encode()).hexdigest()


def build(force: bool = False, jobs: int | None = None, extra=()) -> str:
    os.makedirs(OBJ, exist_ok=True)
    # objects built with other flags (an A/B variant's -D...) are never reused
    stamp_path = os.path.join(OBJ, "flags.stamp")
    stamp = _flags_stamp(extra)
    old = open(stamp_path).read().strip() if os.path.exists(stamp_path) else ""
    if old != stamp:
        force = True
    srcs = _sources()
    with cf.ThreadPoolExecutor(max_workers=jobs or min(16, os.cpu_count() or 4)) as ex:
        objs = list(ex.map(lambda s: _compile(s, force, extra), srcs))
    if force or not os.path.exists(OUT) or os.path.getmtime(OUT) < max(os.path.getmtime(o) for o in objs):
        tmp = OUT + f".tmp{os.getpid()}"
        cmd = [NVCC] + ARCH + ["-shared", "-o", tmp] + objs + ["-Xcompiler", "-fopenmp", "-ldl", "-cudart", "static"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
        os.replace(tmp, OUT)
    if old != stamp:
        with open(stamp_path, "w") as f:
            f.write(stamp + "\n")
    return OUT


if __name__ == "__main__":
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--jobs", type=int, default=None)
    a = ap.parse_args()
    print(build(a.force, a.jobs))
