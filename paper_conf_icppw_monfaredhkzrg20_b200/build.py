"""Build libbsrng.so (the C-ABI library, include/bsrng.h) in-tree for sm_100a.

The library is five translation units (csrc/bsrng.cu: the C ABI; csrc/
cipher_{mickey2,grain,lfsr,aes}.cu: each cipher's kernels and launchers),
compiled in parallel with nvcc and linked into one shared object.
"""
from __future__ import annotations

import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libbsrng.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
UNITS = ["bsrng.cu", "cipher_mickey2.cu", "cipher_grain.cu", "cipher_lfsr.cu", "cipher_aes.cu"]
# --compress-mode=size: the fatbin (SASS + the -lineinfo debug sections) is
# stored compressed and unpacked at module load: 15 MB -> ~3 MB on disk
FLAGS = [*ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "--compress-mode=size"]


def _sources():
    out = [os.path.join(ROOT, "include", "bsrng.h"), os.path.abspath(__file__)]
    for f in sorted(os.listdir(CSRC)):
        if f.endswith((".cu", ".cuh", ".h", ".inc")):
            out.append(os.path.join(CSRC, f))
    return out


def _compile(unit: str, objdir: str, verbose: bool) -> str:
    obj = os.path.join(objdir, unit.replace(".cu", ".o"))
    cmd = [NVCC, *FLAGS, *_DEFINES, "-Xptxas", "-v", "-c", "-o", obj, os.path.join(CSRC, unit)]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError(f"nvcc failed on {unit}")
    if verbose:
        sys.stderr.write(r.stderr)
    return obj


def build(force: bool = False, verbose: bool = False, out: str = LIB, defines=()) -> str:
    """Compile libbsrng.so (or `out`, with extra -D `defines`, for A/B builds)."""
    srcs = _sources()
    if (not force and not defines and out == LIB and os.path.exists(LIB)
            and all(os.path.getmtime(LIB) >= os.path.getmtime(s) for s in srcs)):
        return LIB
    global _DEFINES
    _DEFINES = [f"-D{d}" for d in defines]
    objdir = os.path.join(CSRC, f".obj{os.getpid()}")
    os.makedirs(objdir, exist_ok=True)
    try:
        # the MICKEY unit dominates (its clock loop is ~1.2k LOP3 per 4 clocks);
        # submitting it first keeps the wall time at its compile time
        with ThreadPoolExecutor(max_workers=len(UNITS)) as ex:
            objs = list(ex.map(lambda u: _compile(u, objdir, verbose), UNITS))
        tmp = out + f".tmp{os.getpid()}"
        r = subprocess.run([NVCC, *ARCH, "-shared", "-o", tmp, *objs], capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("nvcc failed linking libbsrng.so")
        os.replace(tmp, out)
    finally:
        for f in os.listdir(objdir):
            os.remove(os.path.join(objdir, f))
        os.rmdir(objdir)
    return out


_DEFINES: list = []

if __name__ == "__main__":
    defs = [a[2:] for a in sys.argv[1:] if a.startswith("-D")]
    outs = [a[6:] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, out=outs[0] if outs else LIB, defines=defs))
