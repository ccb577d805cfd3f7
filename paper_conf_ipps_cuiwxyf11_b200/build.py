"""Build libblas3.so (the C-ABI library) in-tree for sm_100a.

nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo, cudart linked
statically, one object per .cu compiled in parallel, then linked.  Every
step is keyed by a SHA-256 of its inputs (sources, headers, flags), stored
beside the output as <file>.sha256.  The .so
lives next to this file so it travels with the repo snapshot to the GPU box.
"""
from __future__ import annotations

import concurrent.futures as cf
import hashlib
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
OUT = os.path.join(HERE, "libblas3.so")
BUILD = os.path.join(HERE, "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
         "--expt-relaxed-constexpr", "-I", os.path.join(os.path.dirname(HERE), "include")]


def sources():
    return sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".cu"))


def _headers():
    hs = sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".h"))
    hs.append(os.path.join(os.path.dirname(HERE), "include", "blas3.h"))
    return hs


REPO = os.path.dirname(HERE)


def _digest(paths, extra):
    """Content hash of the inputs of one build step (sources, every header,
    compiler and flags): rebuilds follow content, never file times, so a
    stale object or library shipped with a snapshot is never reused.  Paths
    enter relative to the repository, so the same sources give the same
    digest wherever the checkout lives (the GPU box's copy included)."""
    h = hashlib.sha256()
    for p in paths:
        h.update(os.path.relpath(p, REPO).encode())
        with open(p, "rb") as f:
            h.update(f.read())
    h.update(repr(extra).replace(REPO, "<repo>").encode())
    return h.hexdigest()


def _stamp_ok(out, digest):
    try:
        with open(out + ".sha256") as f:
            return os.path.exists(out) and f.read().strip() == digest
    except OSError:
        return False


def _write_stamp(out, digest):
    with open(out + ".sha256", "w") as f:
        f.write(digest + "\n")


def _compile(src, verbose):
    obj = os.path.join(BUILD, os.path.basename(src) + ".o")
    digest = _digest([src, *_headers()], (NVCC, ARCH, FLAGS))
    if _stamp_ok(obj, digest):
        return obj, digest
    cmd = [NVCC, *ARCH, *FLAGS, "-c", src, "-o", obj]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed on {src}:\n{r.stdout}\n{r.stderr}")
    if verbose and r.stderr:
        print(r.stderr, file=sys.stderr)
    _write_stamp(obj, digest)
    return obj, digest


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    if force:
        for f in os.listdir(BUILD):
            os.remove(os.path.join(BUILD, f))
        if os.path.exists(OUT + ".sha256"):
            os.remove(OUT + ".sha256")
    with cf.ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
        res = list(ex.map(lambda s: _compile(s, verbose), sources()))
    objs = [o for o, _ in res]
    link_digest = hashlib.sha256("".join(d for _, d in res).encode()).hexdigest()
    if not _stamp_ok(OUT, link_digest):
        tmp = OUT + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
        os.replace(tmp, OUT)
        _write_stamp(OUT, link_digest)
    return OUT


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
