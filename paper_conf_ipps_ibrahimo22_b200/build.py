"""Build libspp.so in-tree with nvcc for sm_100a (no JIT cache, no torch extension).

The .so lands next to this file so it travels to the GPU box with the repo
snapshot (it is git-ignored, not gpurun-ignored).
"""
from __future__ import annotations

import os
import subprocess
import sys
from pathlib import Path

PKG = Path(__file__).resolve().parent
ROOT = PKG.parent
CSRC = PKG / "csrc"
LIB = PKG / "libspp.so"
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

GENCODE = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = ["-O3", "-std=c++17", "-lineinfo", *GENCODE, "-Xptxas", "-v",
              "-Xcompiler", "-fPIC,-O3,-ffp-contract=off,-fno-fast-math",
              f"-I{ROOT / 'include'}", f"-I{CSRC}"]
# NB: no --use_fast_math / -ftz=true: fp32 subnormals are real results here (FORMAT.md 2.3)


def sources():
    return sorted(CSRC.glob("*.cu")) + sorted(CSRC.glob("*.cpp"))


def _stale() -> bool:
    if not LIB.exists():
        return True
    t = LIB.stat().st_mtime
    deps = sources() + list(CSRC.glob("*.h")) + list(CSRC.glob("*.cuh")) + [ROOT / "include" / "spp.h", Path(__file__)]
    return any(p.stat().st_mtime > t for p in deps)


def build(force: bool = False, verbose: bool = False, defines=(), out: Path | None = None) -> Path:
    """Build libspp.so (or, for experiments, a variant with extra -D defines at `out`)."""
    target = Path(out) if out else LIB
    if not force and not defines and out is None and not _stale():
        return LIB
    objdir = PKG / ("_build" if not defines else "_build_" + "_".join(d.replace("=", "") for d in defines))
    objdir.mkdir(exist_ok=True)
    objs = []
    for src in sources():
        obj = objdir / (src.name + ".o")
        cmd = [NVCC, *NVCC_FLAGS, *[f"-D{d}" for d in defines], "-c", str(src), "-o", str(obj)]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError(f"nvcc failed on {src.name}")
        (objdir / (src.name + ".ptxas.log")).write_text(r.stderr)
        if verbose:
            sys.stderr.write(r.stderr)
        objs.append(str(obj))
    tmp = target.with_suffix(".so.tmp")
    cmd = [NVCC, *GENCODE, "-shared", "-cudart", "shared", "-o", str(tmp), *objs,
           "-Xlinker", "-rpath,/usr/local/cuda/lib64"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc link failed")
    tmp.replace(target)
    return target


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
