"""Build the in-tree CUDA library libtopk_b200.so for sm_100a (nvcc cross-compiles
without a GPU).  Invoked by __graft_entry__.build() and by the binding on first use
if the .so is missing or stale."""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libtopk_b200.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17", "--shared", "-Xcompiler", "-fPIC",
    "-Xptxas", "-v", "-diag-suppress", "177",
]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cuh"))
                  + glob.glob(os.path.join(CSRC, "*.h"))
                  + [os.path.join(INCLUDE, "topk.h")])


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


def _run(cmd):
    return subprocess.run(cmd, capture_output=True, text=True)


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile every csrc/*.cu to an object (in parallel: the select kernel's
    instantiations live in one translation unit per key type), then link the .so."""
    if not force and not stale():
        return LIB
    from concurrent.futures import ThreadPoolExecutor

    cus = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    objdir = os.path.join(PKG, "build")
    os.makedirs(objdir, exist_ok=True)
    objs = [os.path.join(objdir, os.path.basename(c)[:-3] + ".o") for c in cus]
    cmds = [[NVCC, *FLAGS, "-c", "-I", INCLUDE, "-o", o, c] for c, o in zip(cus, objs)]
    # largest TUs first
    order = sorted(range(len(cmds)), key=lambda i: -os.path.getsize(cus[i]))
    with ThreadPoolExecutor(max_workers=max(1, min(len(cmds), os.cpu_count() or 1))) as ex:
        results = dict(zip(order, ex.map(lambda i: _run(cmds[i]), order)))
    log = []
    for i in range(len(cmds)):
        r = results[i]
        log.append(f"== {os.path.basename(cus[i])}\n" + r.stdout + r.stderr)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed on {cus[i]}:\n" + r.stdout + r.stderr)
    r = _run([NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "--shared", "-o",
              LIB + ".tmp", *objs, "-ldl"])
    if r.returncode != 0:
        raise RuntimeError("nvcc link failed:\n" + r.stdout + r.stderr)
    os.replace(LIB + ".tmp", LIB)
    with open(os.path.join(PKG, "ptxas_info.txt"), "w") as f:
        f.write("\n".join(log))
    if verbose:
        print("\n".join(log))
    return LIB


if __name__ == "__main__":
    print(build(force=True))
