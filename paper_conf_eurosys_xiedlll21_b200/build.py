"""Build libtahoe.so in-tree with nvcc for sm_100a (no fast-math: IEEE compares and fp64 sums).

    python -m paper_conf_eurosys_xiedlll21_b200.build [--force] [--verbose]
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libtahoe.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_include() -> str:
    """Headers of the NCCL (>= 2.28, device API) that torch ships; the library is dlopen'ed at run
    time, so only the headers are needed to build."""
    try:
        import nvidia.nccl as m  # type: ignore
        for base in list(getattr(m, "__path__", [])):
            inc = os.path.join(base, "include")
            if os.path.exists(os.path.join(inc, "nccl_device.h")):
                return inc
    except ImportError:
        pass
    raise RuntimeError("NCCL >= 2.28 headers (nccl_device.h) not found (python package nvidia-nccl)")


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cpp")) + glob.glob(os.path.join(CSRC, "*.cu")))


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.hpp")) + [os.path.join(INCLUDE, "tahoe.h")]
    return any(os.path.getmtime(p) > t for p in deps)


def build(force: bool = False, verbose: bool = False, out: str | None = None,
          defines: list[str] | None = None) -> str:
    """out / defines: another in-tree build with extra -D flags (same-box A/B experiments,
    selected at run time by $TAHOE_LIB_AB)."""
    if out is None and not force and not _stale():
        return LIB
    dst = out or LIB
    tmp = dst + f".tmp{os.getpid()}"
    cmd = [NVCC, *ARCH, "-lineinfo", "-O3", "-std=c++17", "-shared", "-cudart", "static",
           "-Xcompiler", "-fPIC,-fvisibility=hidden,-O3", "-I", nccl_include(), "-I", INCLUDE, "-I", CSRC,
           *[f"-D{d}" for d in (defines or [])], "-o", tmp, *sources(), "-lpthread", "-ldl"]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed building libtahoe.so")
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(tmp, dst)
    return dst


if __name__ == "__main__":
    # --out NAME -DX=Y ...: an A/B variant next to libtahoe.so
    args = sys.argv[1:]
    out = os.path.join(PKG, args[args.index("--out") + 1]) if "--out" in args else None
    print(build(force="--force" in args, verbose="--verbose" in args, out=out,
                defines=[a[2:] for a in args if a.startswith("-D")]))
