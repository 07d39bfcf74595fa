"""Build libmsp.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

``python paper_conf_ipps_daltonbmog15_b200/_build.py`` or
``__graft_entry__.build()`` (run it by path: importing the package loads
libmsp.so first).  Objects are compiled in parallel and linked
into ``paper_conf_ipps_daltonbmog15_b200/libmsp.so`` with static cudart and a
version script that exports only the ``msp_*`` C ABI of include/msp.h.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys
from pathlib import Path

PKG = Path(__file__).resolve().parent
CSRC = PKG / "csrc"
ROOT = PKG.parent
LIB = Path(os.environ.get("MSP_LIB_OUT", PKG / "libmsp.so"))  # experiment builds may go elsewhere
BUILD = Path(os.environ.get("MSP_BUILD_DIR", ROOT / "build" / "msp"))

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
         "--expt-relaxed-constexpr", "-I", str(ROOT / "include")] + os.environ.get("MSP_NVCC_EXTRA", "").split()


def sources() -> list[Path]:
    return sorted(CSRC.glob("*.cu"))


def headers() -> list[Path]:
    return sorted(CSRC.glob("*.cuh")) + sorted(CSRC.glob("*.h")) + [ROOT / "include" / "msp.h"]


def _stale(out: Path, deps: list[Path]) -> bool:
    if not out.exists():
        return True
    t = out.stat().st_mtime
    return any(d.stat().st_mtime > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> Path:
    BUILD.mkdir(parents=True, exist_ok=True)
    srcs = sources()
    hdrs = headers()
    objs = [BUILD / (s.stem + ".o") for s in srcs]

    def compile_one(src: Path, obj: Path):
        if not force and not _stale(obj, [src] + hdrs):
            return ""
        cmd = [NVCC, *ARCH, *FLAGS, "-Xptxas", "-v", "-c", str(src), "-o", str(obj)]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src.name}:\n{r.stdout}\n{r.stderr}")
        return r.stderr

    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        logs = list(ex.map(compile_one, srcs, objs))
    if verbose:
        for s, lg in zip(srcs, logs):
            if lg:
                print(f"--- {s.name}\n{lg}", file=sys.stderr)
    if force or _stale(LIB, objs):
        tmp = LIB.with_suffix(f".so.{os.getpid()}")
        cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", str(tmp), *map(str, objs),
               "-Xlinker", f"--version-script={CSRC / 'msp.map'}"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
    print(LIB)
