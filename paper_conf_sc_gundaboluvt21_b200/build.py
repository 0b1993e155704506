"""Build libfastz.so (in-tree) with nvcc for sm_100a."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libfastz.so")
SOURCES = ["api.cu", "kernels.cu", "intpeak.cu", "seeds.cu", "dedup.cu"]
HEADERS = ["dp.cuh", "side.cuh", "pair.cuh", "internal.h"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
         "-Xcompiler", "-fPIC", "-shared", "-Xptxas", "-warn-spills", "-diag-suppress", "177"]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "fastz.h"),
                                                                  os.path.abspath(__file__)]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines=()) -> str:
    """Compile libfastz.so in-tree (``out``/``defines``: an A/B variant of the same sources, e.g.
    ``-DEXECUTE_MIN_BLOCKS=5`` into ab_libs/, loaded with FASTZ_LIB=...)."""
    lib = os.path.abspath(out) if out else LIB
    if not force and out is None and not _stale():
        return lib
    cmd = [NVCC] + FLAGS + list(defines) + ["-o", lib + ".tmp"] + [os.path.join(CSRC, s) for s in SOURCES]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd, cwd=CSRC)
    os.replace(lib + ".tmp", lib)
    return lib


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
