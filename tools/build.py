"""Build every native library of the repo in-tree (sm_100a only).

* ``oracle/liblouvain_oracle.so``  -- gcc, plain C (test infrastructure)
* ``graphgen/libgraphgen.so``      -- nvcc, seeded input generators (host + device)
* ``paper_conf_ipps_naimmht17_b200/liblouvain.so`` -- nvcc, the product C-ABI

Rebuilds a target only when one of its sources is newer than the .so.
"""
from __future__ import annotations

import glob
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NVCC = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _site_nccl() -> str:
    for p in sys.path:
        cand = os.path.join(p, "nvidia", "nccl")
        if os.path.isdir(os.path.join(cand, "include")):
            return cand
    return ""


def _stale(target: str, sources: list[str]) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def _run(cmd: list[str]) -> None:
    print("+", " ".join(cmd), flush=True)
    subprocess.run(cmd, check=True, cwd=ROOT)


def build_oracle(force: bool = False) -> str:
    src = [os.path.join(ROOT, "oracle", "louvain_oracle.c")]
    hdr = [os.path.join(ROOT, "oracle", "louvain_oracle.h")]
    out = os.path.join(ROOT, "oracle", "liblouvain_oracle.so")
    if force or _stale(out, src + hdr + [__file__]):
        _run(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-ffp-contract=off", "-Wall", "-Wextra",
              "-o", out] + src)
    return out


def build_graphgen(force: bool = False) -> str:
    d = os.path.join(ROOT, "graphgen", "csrc")
    srcs = sorted(glob.glob(os.path.join(d, "*.cpp")) + glob.glob(os.path.join(d, "*.cu")))
    hdrs = glob.glob(os.path.join(d, "*.h"))
    out = os.path.join(ROOT, "graphgen", "libgraphgen.so")
    if force or _stale(out, srcs + hdrs + [__file__]):
        _run([NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-shared",
              "-Xcompiler", "-fPIC,-ffp-contract=off", "-o", out] + srcs)
    return out


def build_louvain(force: bool = False, d: str = "", out: str = "", objdir: str = "", defines=()) -> str:
    """The product library; d/out/objdir name another source tree and target (tools/ab_build.py)."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_naimmht17_b200")
    d = d or os.path.join(pkg, "csrc")
    srcs = sorted(glob.glob(os.path.join(d, "*.cu")) + glob.glob(os.path.join(d, "*.cpp")))
    hdrs = glob.glob(os.path.join(d, "*.h")) + glob.glob(os.path.join(d, "*.cuh")) + \
        glob.glob(os.path.join(ROOT, "include", "*.h"))
    out = out or os.path.join(pkg, "liblouvain.so")
    if not srcs:
        return out
    nccl = _site_nccl()
    nccl_flags = []
    if nccl:
        nccl_flags = ["-I", os.path.join(nccl, "include"), "-DLOUVAIN_HAVE_NCCL_HEADERS=1"]
    # one object per translation unit (compiled in parallel, only when stale), then one link
    objdir = objdir or os.path.join(ROOT, "build", "louvain")
    os.makedirs(objdir, exist_ok=True)
    flags = [NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xptxas", "-v",
             "-Xcompiler", "-fPIC,-ffp-contract=off,-fvisibility=hidden",
             "-I", os.path.join(ROOT, "include"), *nccl_flags, *[f"-D{x}" for x in defines]]
    objs, procs = [], []
    for src in srcs:
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        objs.append(obj)
        if force or _stale(obj, [src] + hdrs + [__file__]):
            cmd = flags + ["-c", "-o", obj, src]
            print("+", " ".join(cmd), flush=True)
            procs.append((src, subprocess.Popen(cmd, cwd=ROOT)))
    for src, pr in procs:
        if pr.wait() != 0:
            raise subprocess.CalledProcessError(pr.returncode, f"nvcc {src}")
    if force or procs or _stale(out, objs):
        _run([NVCC, *ARCH, "-shared", "-o", out] + objs + ["-ldl"])
    return out


def build_micro(force: bool = False) -> str:
    """tools/micro/libgather_sol.so: the gather speed-of-light kernel bench.py times beside the sweep."""
    src = os.path.join(ROOT, "tools", "micro", "gather_sol.cu")
    out = os.path.join(ROOT, "tools", "micro", "libgather_sol.so")
    if force or _stale(out, [src, __file__]):
        _run([NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-shared", "-Xcompiler", "-fPIC", "-o", out, src])
    return out


def build_all(force: bool = False) -> None:
    build_oracle(force)
    build_graphgen(force)
    build_louvain(force)
    build_micro(force)


if __name__ == "__main__":
    build_all(force="--force" in sys.argv)
