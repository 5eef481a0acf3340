"""Build libbqr.so in-tree with nvcc for sm_100a (no fast math: IEEE sqrt/div)."""
from __future__ import annotations

import os
import re
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libbqr.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

FLAGS = [
    "-O3", "-std=c++17", "-lineinfo",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-prec-div=true", "-prec-sqrt=true", "-ftz=false", "-fmad=true",
    "-Xcompiler", "-fPIC,-O2", "-shared",
]


def cutlass_flags():
    """CUTLASS / CuTe headers vendored in the image (flashinfer's copy): used
    by bqr_wy.cu's tensor-core GEMMs; without them that translation unit
    compiles to stubs (the blocked WY entry point then falls back)."""
    import site
    for sp in site.getsitepackages():
        inc = os.path.join(sp, "flashinfer", "data", "cutlass", "include")
        if os.path.isdir(os.path.join(inc, "cutlass")):
            util = os.path.join(sp, "flashinfer", "data", "cutlass", "tools", "util", "include")
            return ["-I" + inc, "-I" + util, "--expt-relaxed-constexpr", "-diag-suppress", "20012"]
    return ["-DBQR_NO_CUTLASS"]


def sources():
    out = []
    for d, _, files in os.walk(CSRC):
        out += [os.path.join(d, f) for f in files if f.endswith((".cu", ".cuh", ".h"))]
    out.append(os.path.join(os.path.dirname(HERE), "include", "bqr.h"))
    return out


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


def deps(path, seen=None):
    """The translation unit and every quoted #include it reaches."""
    seen = set() if seen is None else seen
    if path in seen or not os.path.exists(path):
        return seen
    seen.add(path)
    with open(path) as f:
        for inc in re.findall(r'^\s*#\s*include\s+"([^"]+)"', f.read(), re.M):
            deps(os.path.normpath(os.path.join(os.path.dirname(path), inc)), seen)
    return seen


def build(force: bool = False, verbose: bool = False, extra=()) -> str:
    """Compile the csrc/*.cu translation units whose object is older than the
    unit or a header it includes (all of them with force / extra flags) in
    parallel, link libbqr.so."""
    if not force and not stale():
        return LIB
    units = sorted(f for f in os.listdir(CSRC) if f.endswith(".cu"))
    objdir = os.path.join(HERE, "build_obj")
    os.makedirs(objdir, exist_ok=True)
    cflags = [f for f in FLAGS if f != "-shared"]
    procs = []
    for u in units:
        obj = os.path.join(objdir, u[:-3] + ".o")
        src = os.path.join(CSRC, u)
        if (not force and not extra and os.path.exists(obj)
                and all(os.path.getmtime(d) <= os.path.getmtime(obj) for d in deps(src))):
            procs.append((u, obj, None))
            continue
        cmd = [NVCC, *cflags, *(cutlass_flags() if u == "bqr_wy.cu" else []), *extra, "-c", "-o", obj,
               os.path.join(CSRC, u)]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
            print(" ".join(cmd), file=sys.stderr)
        procs.append((u, obj, subprocess.Popen(cmd)))
    objs = []
    for u, obj, pr in procs:
        if pr is not None and pr.wait() != 0:
            raise subprocess.CalledProcessError(pr.returncode, f"nvcc {u}")
        objs.append(obj)
    link = [NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-Xcompiler", "-fPIC",
            "-o", LIB + ".tmp", *objs, "-lcuda"]
    subprocess.check_call(link)
    os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
