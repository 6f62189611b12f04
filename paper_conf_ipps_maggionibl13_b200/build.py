"""Build libcme.so in-tree with nvcc for sm_100a (no JIT, no torch extension cache).

    python paper_conf_ipps_maggionibl13_b200/build.py [--force] [-v]

(Run it by path: importing the package loads libcme.so.)
"""
from __future__ import annotations

import glob
import hashlib
import os
import shutil
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libcme.so")
OBJ = os.path.join(PKG, "build")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_include() -> str:
    try:
        import nvidia.nccl  # the NCCL torch ships (2.28.x); one libnccl per process
        for base in nvidia.nccl.__path__:
            inc = os.path.join(base, "include")
            if os.path.exists(os.path.join(inc, "nccl.h")):
                return inc
    except ImportError:
        pass
    return "/usr/include"


def nvcc() -> str:
    for cand in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found")


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cpp")) + glob.glob(os.path.join(CSRC, "*.cu")))


def _deps():
    return _sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(ROOT, "include", "cme.h")]


def _common_flags(defines=()):
    return ["-std=c++17", "-O3", "-lineinfo", "-I", os.path.join(ROOT, "include"), "-I", CSRC,
            "-I", nccl_include(), "-Xcompiler", "-fPIC,-fopenmp,-ffp-contract=off,-Wall"] + [f"-D{d}" for d in defines]


def source_hash(defines=()) -> str:
    """sha256 over every source/header byte, the compiler flags and the nvcc
    version: the library is rebuilt whenever any of them differs from the hash
    recorded beside it (file mtimes are not trusted: a shipped libcme.so newer
    than its sources would otherwise be reused unbuilt)."""
    h = hashlib.sha256()
    for p in sorted(_deps()):
        h.update(os.path.relpath(p, ROOT).encode())
        with open(p, "rb") as f:
            h.update(f.read())
    h.update(" ".join(ARCH + _common_flags(defines)).replace(ROOT, "<root>").encode())
    try:
        h.update(subprocess.run([nvcc(), "--version"], capture_output=True, text=True).stdout.encode())
    except (OSError, RuntimeError):
        pass
    return h.hexdigest()


def _stamp(lib: str) -> str:
    return lib + ".sha256"


def up_to_date(lib: str = LIB, defines=()) -> bool:
    if not os.path.exists(lib) or not os.path.exists(_stamp(lib)):
        return False
    with open(_stamp(lib)) as f:
        return f.read().strip() == source_hash(tuple(defines))


SANITIZE = ["-Xcompiler", "-fsanitize=address", "-Xcompiler", "-fsanitize=undefined", "-Xcompiler",
            "-fno-omit-frame-pointer", "-Xcompiler", "-fno-sanitize-recover=undefined"]   # (nvcc splits -Xcompiler at commas)


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines=(), sanitize=False) -> str:
    """Compile libcme.so (or `out` with extra -D`defines`, for kernel A/B builds;
    `sanitize`: the host code instrumented with ASan + UBSan, tools/asan_host.py)."""
    lib = out or LIB
    digest = source_hash(tuple(defines) + (("SANITIZE",) if sanitize else ()))
    if not force and up_to_date(lib, defines):
        return lib
    obj_dir = OBJ if out is None else OBJ + "_" + os.path.basename(out).replace(".so", "")
    os.makedirs(obj_dir, exist_ok=True)
    common = _common_flags(defines) + (SANITIZE if sanitize else [])

    def compile_one(src):
        obj = os.path.join(obj_dir, os.path.basename(src) + ".o")
        cmd = [nvcc()] + ARCH + common + ["-c", src, "-o", obj]
        if src.endswith(".cu"):
            cmd += ["-Xptxas", "-v"] if verbose else []
        else:
            cmd += ["-x", "cu"] if False else []
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
        if verbose and r.stderr:
            print(r.stderr, file=sys.stderr)
        return obj

    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        objs = list(ex.map(compile_one, _sources()))
    tmp = lib + f".tmp{os.getpid()}"
    cmd = [nvcc()] + ARCH + ["-shared", "-o", tmp] + objs + ["-Xcompiler", "-fopenmp", "-lgomp", "-ldl"] + \
        (SANITIZE if sanitize else [])
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stderr}")
    os.replace(tmp, lib)
    with open(_stamp(lib), "w") as f:
        f.write(digest + "\n")
    return lib


if __name__ == "__main__":
    args = sys.argv[1:]
    out = args[args.index("--out") + 1] if "--out" in args else None
    defs = [a[2:] for a in args if a.startswith("-D")]
    print(build(force="--force" in args, verbose="-v" in args, out=out, defines=defs, sanitize="--sanitize" in args))
