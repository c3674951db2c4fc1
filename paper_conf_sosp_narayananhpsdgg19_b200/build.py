"""Builds libpipedream.so in-tree: every CUDA/C++ source of csrc/ compiled for sm_100a
(-gencode arch=compute_100a,code=sm_100a), static CUDA runtime, no link-time dependency
on libcuda.so (driver entry points are resolved at run time)."""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libpipedream.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def headers():
    return sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(HERE, "..", "include", "*.h")))


def up_to_date() -> bool:
    if not os.path.exists(LIB):
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(f) <= t for f in sources() + headers() + [__file__])


def build(force: bool = False, verbose: bool = False, jobs: int = 8) -> str:
    if not force and up_to_date():
        return LIB
    objdir = os.path.join(HERE, "build")
    os.makedirs(objdir, exist_ok=True)
    common = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
              "-I", CSRC, "-I", os.path.join(HERE, "..", "include")] + ARCH
    if verbose:
        common += ["-Xptxas", "-v"]
    procs, objs = [], []
    for src in sources():
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        objs.append(obj)
        cmd = [NVCC, "-c", src, "-o", obj] + common
        if src.endswith(".cpp"):
            cmd += ["-x", "cu"]  # compile host-only sources with the same toolchain
        procs.append((src, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
        while len([p for _, p in procs if p.poll() is None]) >= jobs:
            procs[0][1].wait()
    failed = False
    for src, p in procs:
        out, _ = p.communicate()
        text = out.decode()
        if p.returncode != 0:
            failed = True
            sys.stderr.write(f"--- {os.path.basename(src)}\n{text}\n")
        elif verbose and text:
            sys.stderr.write(text)
    if failed:
        raise RuntimeError("libpipedream build failed")
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, "-shared", "-o", tmp] + objs + ARCH + ["-cudart", "static", "-lpthread", "-ldl", "-lrt"])
    os.replace(tmp, LIB)
    return LIB


# Fault-injected variants of the library (tests only, never loaded by the product path):
# runtime.cu recompiled with one PD_FAULT_* define, linked with the product's other objects
# into build/<name>/libpipedream.so.  The negative-control tests load them through
# PD_LIBRARY in a subprocess and require the parity / slot-ownership checks to FAIL.
FAULTS = {
    "fault_stash": "PD_FAULT_STASH",            # backward reads the latest weight version
    "fault_no_dxwait": "PD_FAULT_NO_DXWAIT",    # side-stream dW + update not ordered after dX / G
    "fault_recv_depth": "PD_FAULT_RECV_DEPTH",  # activation receive rings one slot too shallow
}


def fault_lib(name: str) -> str:
    return os.path.join(HERE, "build", name, "libpipedream.so")


def build_faults(force: bool = False) -> None:
    build()
    objdir = os.path.join(HERE, "build")
    common = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
              "-I", CSRC, "-I", os.path.join(HERE, "..", "include")] + ARCH
    rt = os.path.join(CSRC, "runtime.cu")
    others = [os.path.join(objdir, os.path.basename(f) + ".o") for f in sources() if f != rt]
    procs = []
    for name, define in FAULTS.items():
        out = fault_lib(name)
        if not force and os.path.exists(out) and os.path.getmtime(out) >= os.path.getmtime(LIB):
            continue
        os.makedirs(os.path.dirname(out), exist_ok=True)
        obj = os.path.join(os.path.dirname(out), "runtime.cu.o")
        procs.append((out, obj, subprocess.Popen([NVCC, "-c", rt, "-o", obj, "-D" + define] + common)))
    for out, obj, p in procs:
        if p.wait() != 0:
            raise RuntimeError(f"fault variant build failed: {out}")
        tmp = out + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, "-shared", "-o", tmp, obj] + others + ARCH +
                              ["-cudart", "static", "-lpthread", "-ldl", "-lrt"])
        os.replace(tmp, out)


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    if "--faults" in sys.argv:
        build_faults(force="--force" in sys.argv)
    print(LIB)
