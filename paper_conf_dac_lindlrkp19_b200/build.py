"""Build libdp.so in-tree for sm_100a with nvcc (no JIT cache: the .so travels with the repo).

    python -m paper_conf_dac_lindlrkp19_b200.build [--force]
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIBDIR = os.path.join(HERE, "lib")
LIB = os.path.join(LIBDIR, "libdp.so")
INCLUDE = os.path.join(os.path.dirname(HERE), "include")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC",
    "-Xptxas", "-v",
    "--expt-relaxed-constexpr",
] + os.environ.get("DP_NVCC_EXTRA", "").split()   # A/B builds only (e.g. -DDP_WA_PPL=8)


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + _headers()
    return any(os.path.getmtime(p) > t for p in deps)


def _headers() -> list[str]:
    return (glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh"))
            + [os.path.join(INCLUDE, "dp.h")])


def build(force: bool = False, verbose: bool = False) -> str:
    """One object per .cu (compiled in parallel, rebuilt when it or a header is newer), then
    one nvcc link into lib/libdp.so."""
    if not force and not _stale():
        return LIB
    os.makedirs(LIBDIR, exist_ok=True)
    nvcc = os.environ.get("NVCC", "nvcc")
    hdr_t = max(os.path.getmtime(p) for p in _headers())
    jobs = []
    for src in sources():
        obj = os.path.join(LIBDIR, os.path.basename(src)[:-3] + ".o")
        if force or not os.path.exists(obj) or os.path.getmtime(obj) < max(hdr_t, os.path.getmtime(src)):
            jobs.append((src, obj))
    from concurrent.futures import ThreadPoolExecutor

    def compile_one(job):
        src, obj = job
        tmp_o = obj + f".tmp{os.getpid()}"
        cmd = [nvcc, *NVCC_FLAGS, "-I", INCLUDE, "-c", "-o", tmp_o, src]
        res = subprocess.run(cmd, capture_output=True, text=True)
        if res.returncode == 0:
            os.replace(tmp_o, obj)
        return src, cmd, res

    log_path = os.path.join(LIBDIR, "build.log")
    with ThreadPoolExecutor(max_workers=max(1, min(len(jobs), os.cpu_count() or 4))) as ex:
        results = list(ex.map(compile_one, jobs))
    with open(log_path, "a" if not force else "w") as log:
        for src, cmd, res in results:
            log.write(" ".join(cmd) + "\n" + res.stdout + res.stderr)
    failed = [r for r in results if r[2].returncode != 0]
    if failed:
        for _, _, res in failed:
            sys.stderr.write(res.stderr[-8000:])
        raise RuntimeError(f"nvcc failed (see {log_path})")
    if verbose:
        for _, _, res in results:
            sys.stderr.write(res.stderr)
    tmp = LIB + f".tmp{os.getpid()}"
    objs = [os.path.join(LIBDIR, os.path.basename(s)[:-3] + ".o") for s in sources()]
    cmd = [nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, *objs, "-ldl"]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stderr[-8000:])
        raise RuntimeError("nvcc link failed")
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
