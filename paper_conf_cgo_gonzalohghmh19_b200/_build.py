"""In-tree build of libreduce_b200.so (sm_100a only).

Each CUDA / C++ source is compiled by nvcc with
``-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo`` (in parallel), then
linked into ``paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so`` with the
static CUDA runtime.  NCCL is not linked: reduce_multi.cpp dlopens it at run
time (only its header is needed here, from the torch wheel's nvidia-nccl).
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libreduce_b200.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nvcc() -> str:
    for p in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc"):
        if p and os.path.exists(p):
            return p
    return "nvcc"


def _nccl_include() -> str:
    import site
    cands = []
    for sp in site.getsitepackages() + [site.getusersitepackages()]:
        cands.append(os.path.join(sp, "nvidia", "nccl", "include"))
    cands.append("/usr/include")
    for c in cands:
        if os.path.exists(os.path.join(c, "nccl.h")):
            return c
    raise RuntimeError("nccl.h not found (expected the torch wheel's nvidia/nccl/include)")


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def _deps() -> list[str]:
    return (sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h"))
            + glob.glob(os.path.join(CSRC, "*.inc")) + [os.path.join(ROOT, "include", "reduce.h"), __file__])


STAMP = os.path.join(BUILD, "flags.stamp")  # the experiment flags the in-tree library was built with


def _extra_flags() -> str:
    return " ".join(os.environ.get("REDUCE_B200_NVCC_FLAGS", "").split())


def up_to_date() -> bool:
    """The in-tree library is newer than every source AND was built with the
    current experiment flags (an A/B build with -D... flags is never reused by a
    default build, and the reverse)."""
    if not os.path.exists(LIB):
        return False
    try:
        with open(STAMP) as fh:
            if fh.read().strip() != _extra_flags():
                return False
    except OSError:
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(d) <= t for d in _deps())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and up_to_date():
        return LIB
    os.makedirs(BUILD, exist_ok=True)
    nvcc = _nvcc()
    inc = ["-I", os.path.join(ROOT, "include"), "-I", CSRC, "-I", _nccl_include()]
    common = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", "-Xptxas", "-warn-spills"] + inc
    # experiment hook (tools/probes A/B builds), e.g. REDUCE_B200_NVCC_FLAGS="-DRB_SEG_PIPE=2"
    common += os.environ.get("REDUCE_B200_NVCC_FLAGS", "").split()

    def compile_one(src: str) -> str:
        obj = os.path.join(BUILD, os.path.basename(src) + ".o")
        cmd = [nvcc] + common + ["-c", src, "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
        if verbose and (r.stderr.strip() or r.stdout.strip()):
            print(r.stdout, r.stderr, file=sys.stderr)
        return obj

    with ThreadPoolExecutor(max_workers=max(2, os.cpu_count() or 2)) as ex:
        objs = list(ex.map(compile_one, sources()))
    tmp = LIB + ".tmp"
    cmd = [nvcc] + ARCH + ["-shared", "-o", tmp] + objs + ["-ldl", "-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, LIB)
    with open(STAMP, "w") as fh:
        fh.write(_extra_flags() + "\n")
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
