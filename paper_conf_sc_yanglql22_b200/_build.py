"""Build libwg.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with
the repository snapshot to the GPU box)."""

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libwg.so")
SOURCES = ["dsm.cu", "sample.cu", "unique.cu", "gather.cu", "micro.cu", "spmm.cu", "exchange.cu"]
HEADERS = ["wg_internal.cuh", "device_util.cuh", "hash.cuh", "scan.cuh", "sample_warp.cuh"]

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-O2", "--expt-relaxed-constexpr",
         "-I", INCLUDE]
# extra compile-time knobs for A/B builds, e.g. WG_NVCC_DEFS="-DWG_LB_SLEEP_NS=0" (default build: none)
FLAGS += os.environ.get("WG_NVCC_DEFS", "").split()


STAMP = LIB + ".stamp"   # the nvcc command line the library was built with


def _stamp_text(lib_path=LIB):
    import hashlib
    with open(lib_path, "rb") as f:
        digest = hashlib.sha256(f.read()).hexdigest()
    return " ".join([NVCC, *ARCH, *FLAGS, *SOURCES]) + "\n" + digest


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    if any(os.path.getmtime(d) > t for d in deps):
        return True
    # a build with other flags (e.g. WG_NVCC_DEFS A/B defines) or a copied-in binary is never current
    try:
        with open(STAMP) as f:
            return f.read() != _stamp_text(target)
    except OSError:
        return True


def build_lib(force=False, verbose=False) -> str:
    deps = [os.path.join(CSRC, s) for s in SOURCES + HEADERS] + [os.path.join(INCLUDE, "wg.h")]
    if not force and not _stale(LIB, deps):
        return LIB
    objdir = os.path.join(PKG, "build")
    os.makedirs(objdir, exist_ok=True)
    objs = []
    procs = []
    for s in SOURCES:
        o = os.path.join(objdir, s.replace(".cu", ".o"))
        cmd = [NVCC, *ARCH, *FLAGS, "-c", os.path.join(CSRC, s), "-o", o]
        if verbose:
            cmd += ["-Xptxas", "-v"]
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
        objs.append(o)
    for cmd, p in procs:
        out, _ = p.communicate()
        if p.returncode != 0:
            sys.stderr.write(out.decode())
            raise RuntimeError("nvcc failed: " + " ".join(cmd))
        if verbose:
            sys.stderr.write(out.decode())
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-cudart", "static", *objs, "-o", tmp])
    os.replace(tmp, LIB)
    with open(STAMP, "w") as f:
        f.write(_stamp_text())
    return LIB


if __name__ == "__main__":
    build_lib(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
