"""Build libstm.so (nvcc, sm_100a) in-tree.  Also used by __graft_entry__.build()."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libstm.so")
SOURCES = ["kernel.cu", "kernel_instr.cu", "kernel_list.cu", "kernel_multi.cu", "runtime.cu", "compiler.cpp", "order.cpp", "motif.cpp"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)]
    deps.append(os.path.join(HERE, "..", "include", "stm.h"))
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, out: str = LIB, defines=()) -> str:
    """defines: extra -D flags for A/B variant libraries (loaded via STM_LIB_PATH)."""
    if out == LIB and not defines and not force and not needs_build():
        return LIB
    cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3", "-shared",
           *[f"-D{d}" for d in defines],
           "-Xptxas", "-v", "-o", out + ".tmp", *[os.path.join(CSRC, s) for s in SOURCES], "-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed building libstm.so")
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(out + ".tmp", out)
    return out


if __name__ == "__main__":
    # usage: build.py [--force] [--out=PATH] [NAME=VALUE ...]   (NAME=VALUE -> -DNAME=VALUE)
    defs = [a for a in sys.argv[1:] if not a.startswith("--")]
    outs = [a[len("--out="):] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose=True, out=outs[0] if outs else LIB, defines=defs))
