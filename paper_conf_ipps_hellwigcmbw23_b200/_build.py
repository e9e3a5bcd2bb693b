"""Build libcdscreen.so in-tree with nvcc for sm_100a (B200)."""
from __future__ import annotations

import os
import subprocess
from pathlib import Path

PKG = Path(__file__).resolve().parent
ROOT = PKG.parent
CSRC = PKG / "csrc"
LIB = PKG / "libcdscreen.so"
NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
              "-Xcompiler", "-fPIC", "-shared", f"-I{ROOT / 'include'}"]


def sources():
    return sorted(CSRC.glob("*.cu"))


def _inputs():
    return sources() + sorted(CSRC.glob("*.cuh")) + sorted(CSRC.glob("*.h")) + \
        [ROOT / "include" / "cdscreen.h"]


def up_to_date() -> bool:
    if not LIB.exists():
        return False
    t = LIB.stat().st_mtime
    return all(p.stat().st_mtime <= t for p in _inputs())


def build(force: bool = False, verbose: bool = False) -> Path:
    """Compile every translation unit in parallel (nvcc, sm_100a), then link the shared
    library (no device code crosses translation units, so no relocatable device code)."""
    if not force and up_to_date():
        return LIB
    import tempfile
    nvcc = os.environ.get("NVCC", "nvcc")
    compile_flags = [f for f in NVCC_FLAGS if f != "-shared"]
    tmp = LIB.with_suffix(f".so.tmp{os.getpid()}")
    with tempfile.TemporaryDirectory(prefix="cdbuild") as td:
        objs, procs = [], []
        for src in sources():
            obj = Path(td) / (src.stem + ".o")
            cmd = [nvcc] + compile_flags + ["-c", "-o", str(obj), str(src)]
            if verbose:
                print(" ".join(cmd))
            procs.append((cmd, subprocess.Popen(cmd)))
            objs.append(str(obj))
        for cmd, p in procs:
            if p.wait() != 0:
                raise subprocess.CalledProcessError(p.returncode, cmd)
        link = [nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", str(tmp)] + objs
        if verbose:
            print(" ".join(link))
        subprocess.run(link, check=True)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force=True, verbose=True)
