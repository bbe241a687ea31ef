"""Builds libcrk.so in-tree for sm_100a (nvcc cross-compiles without a GPU)."""
from __future__ import annotations

import concurrent.futures
import glob
import os
import shutil
import subprocess
import sys
import tempfile

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "lib", "libcrk.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
         "--expt-relaxed-constexpr"]
# Per-file extra device-code flags (experiments; e.g. {"k_server.cu": ["-Xcicc", "-O1"]} made the persistent
# server's step 3.5x slower: less inlining, more local-memory traffic).
FILE_FLAGS: dict[str, list[str]] = {}


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def deps() -> list[str]:
    return sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + [
        os.path.join(ROOT, "include", "crk.h"), os.path.abspath(__file__)]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in deps())


def _compile_link(out: str, defines: list[str] = (), file_flags: dict | None = None, verbose: bool = False) -> str:
    """Each source to an object (in parallel, with its FILE_FLAGS), then one shared library -> out."""
    file_flags = FILE_FLAGS if file_flags is None else file_flags
    os.makedirs(os.path.dirname(out), exist_ok=True)
    tmp = tempfile.mkdtemp(prefix="crk_build_")
    try:
        def one(src: str) -> tuple[str, subprocess.CompletedProcess]:
            obj = os.path.join(tmp, os.path.basename(src) + ".o")
            cmd = [NVCC, *FLAGS, *file_flags.get(os.path.basename(src), []), *[f"-D{d}" for d in defines], "-c",
                   "-o", obj, src]
            if verbose:
                cmd.insert(1, "-Xptxas=-v")
            return obj, subprocess.run(cmd, capture_output=True, text=True)

        with concurrent.futures.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
            results = list(ex.map(one, sources()))
        for _, r in results:
            if r.returncode != 0:
                sys.stderr.write(r.stdout + r.stderr)
                raise RuntimeError(f"nvcc failed building {out}")
            if verbose:
                sys.stderr.write(r.stderr)
        r = subprocess.run([NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", out + ".tmp",
                            *[o for o, _ in results]], capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError(f"nvcc failed linking {out}")
        os.replace(out + ".tmp", out)
    finally:
        shutil.rmtree(tmp, ignore_errors=True)
    return out


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not stale():
        return LIB
    return _compile_link(LIB, verbose=verbose)


def build_trace() -> str:
    """Diagnostic variant with the scan's per-round clock trace (-DCRK_SCAN_TRACE); tools/scan_trace.py."""
    return build_variant("trace", ["CRK_SCAN_TRACE"])


def build_variant(name: str, defines: list[str], file_flags: dict | None = None) -> str:
    """Experiment build with extra -D defines (e.g. scan prefetch knobs) -> lib/libcrk_<name>.so."""
    out = os.path.join(PKG, "lib", f"libcrk_{name}.so")
    if os.path.exists(out) and all(os.path.getmtime(d) <= os.path.getmtime(out) for d in deps()):
        return out
    return _compile_link(out, defines, file_flags)


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
