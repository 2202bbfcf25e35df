"""Builds libac.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

Each translation unit is compiled to an object in parallel (the per-tier
kernel instantiations dominate), then linked into one shared library that
lives next to this file so it travels with the repository snapshot to the
GPU box.  Rebuilds only when a source is newer than the .so.
"""
from __future__ import annotations

import os
import subprocess
from concurrent.futures import ThreadPoolExecutor
from pathlib import Path

PKG = Path(__file__).resolve().parent
ROOT = PKG.parent
CSRC = PKG / "csrc"
LIB = PKG / "libac.so"
INCLUDE = ROOT / "include"
OBJ = ROOT / "build" / "obj"

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CFLAGS = ["-std=c++17", "-O3", "-lineinfo", *ARCH, "-Xcompiler", "-fPIC,-O2", "--expt-relaxed-constexpr"]


def sources() -> list[Path]:
    return sorted(list(CSRC.glob("*.cu")) + list(CSRC.glob("*.cpp")))


def _stale() -> bool:
    if not LIB.exists():
        return True
    t = LIB.stat().st_mtime
    deps = sources() + list(CSRC.glob("*.h")) + list(CSRC.glob("*.cuh")) + list(INCLUDE.glob("*.h"))
    return any(p.stat().st_mtime > t for p in deps)


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc"):
        if c and Path(c).exists():
            return c
    return "nvcc"


def build(force: bool = False, verbose: bool = False) -> Path:
    if not force and not _stale():
        return LIB
    OBJ.mkdir(parents=True, exist_ok=True)
    extra = ["-Xptxas=-v"] if verbose else []

    def compile_one(src: Path) -> Path:
        obj = OBJ / (src.name + ".o")
        # AC_EXTRA_NVCC_FLAGS: experiment switches (e.g. -DAC_TEXT_EVICT_NORMAL), empty by default
        exp = os.environ.get("AC_EXTRA_NVCC_FLAGS", "").split()
        cmd = [nvcc(), *CFLAGS, *extra, *exp, f"-I{INCLUDE}", f"-I{CSRC}", "-c", str(src), "-o", str(obj)]
        if verbose:
            print(" ".join(cmd), flush=True)
        subprocess.check_call(cmd)
        return obj

    with ThreadPoolExecutor(max_workers=max(1, min(8, os.cpu_count() or 1))) as ex:
        objs = list(ex.map(compile_one, sources()))
    tmp = LIB.with_suffix(f".so.tmp{os.getpid()}")
    subprocess.check_call([nvcc(), *ARCH, "-shared", "-o", str(tmp), *map(str, objs), "-ldl"])  # -ldl: NVTX3
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    import sys
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
