"""Build libmx.so in-tree for sm_100a (nvcc cross-compiles without a GPU).

    python -m paper_conf_sc_dhakalrwercfm23_b200.build [--force] [-v]

Objects go to paper_conf_sc_dhakalrwercfm23_b200/build/, the shared library to
paper_conf_sc_dhakalrwercfm23_b200/libmx.so (git-ignored, travels with gpurun).
cudart is linked statically; the driver is reached through
cudaGetDriverEntryPointByVersion, so the library loads on GPU-less hosts.
"""
from __future__ import annotations

import argparse
import glob
import os
import shutil
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libmx.so")
EXTRA_DEFS = [d for d in os.environ.get("MX_DEFS", "").split() if d]   # variant builds (-DMX_...)
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nvcc() -> str:
    p = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    if not os.path.exists(p):
        raise RuntimeError("nvcc not found")
    return p


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cpp")) + glob.glob(os.path.join(CSRC, "kernels", "*.cu")))


def headers():
    return (glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "kernels", "*.h"))
            + glob.glob(os.path.join(CSRC, "kernels", "*.cuh")) + [os.path.join(ROOT, "include", "mx.h")])


def build(force: bool = False, verbose: bool = False, out: str | None = None,
          build_dir: str | None = None) -> str:
    lib = out or LIB
    bdir = build_dir or BUILD
    os.makedirs(bdir, exist_ok=True)
    hdr_mtime = max(os.path.getmtime(h) for h in headers())
    # objects are only reused when built with the same flags (a variant build
    # with MX_DEFS must never leak its objects into the product library)
    stamp = os.path.join(bdir, "flags.stamp")
    flags = " ".join(ARCH + EXTRA_DEFS)
    if not os.path.exists(stamp) or open(stamp).read() != flags:
        force = True
    lib_stamp = lib + ".flags"
    if not os.path.exists(lib_stamp) or open(lib_stamp).read() != flags:
        force = True
    objs, jobs = [], []
    common = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-Wall", "-I", CSRC,
              "-I", os.path.join(ROOT, "include")] + EXTRA_DEFS
    for src in sources():
        rel = os.path.relpath(src, CSRC).replace(os.sep, "_")
        obj = os.path.join(bdir, rel + ".o")
        objs.append(obj)
        if (not force and os.path.exists(obj) and os.path.getmtime(obj) > os.path.getmtime(src)
                and os.path.getmtime(obj) > hdr_mtime):
            continue
        cmd = [nvcc()] + ARCH + common + ["-c", src, "-o", obj]
        if verbose and src.endswith(".cu"):
            cmd += ["-Xptxas", "-v"]
        jobs.append((src, cmd))

    def compile_one(job):
        src, cmd = job
        if verbose:
            print(" ".join(cmd), flush=True)
        return src, subprocess.run(cmd, capture_output=True, text=True)

    # translation units compile in parallel (the decode kernel is one TU per batch size)
    with ThreadPoolExecutor(max_workers=max(1, min(len(jobs), os.cpu_count() or 1))) as ex:
        for src, r in ex.map(compile_one, jobs):
            if r.returncode != 0:
                sys.stderr.write(r.stdout + r.stderr)
                raise RuntimeError(f"compile failed: {src}")
            if verbose and r.stderr:
                sys.stderr.write(r.stderr)
    lib_mtime = os.path.getmtime(lib) if os.path.exists(lib) else 0
    if force or lib_mtime < max(os.path.getmtime(o) for o in objs):
        cmd = [nvcc()] + ARCH + ["-shared", "-o", lib] + objs + ["-lpthread", "-ldl", "-lrt"]
        if verbose:
            print(" ".join(cmd), flush=True)
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("link failed")
    for path in (stamp, lib_stamp):
        with open(path, "w") as f:
            f.write(flags)
    return lib


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-v", "--verbose", action="store_true")
    ap.add_argument("--out", default=None, help="library path (variant builds)")
    ap.add_argument("--build-dir", default=None)
    a = ap.parse_args()
    print(build(a.force, a.verbose, a.out, a.build_dir))
