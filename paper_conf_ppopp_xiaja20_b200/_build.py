"""Build libfsmspec.so in-tree with nvcc for sm_100a (no JIT cache; the .so travels with the repo)."""
from __future__ import annotations

import glob
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
SO = os.environ.get("FSMSPEC_BUILD_SO") or os.path.join(HERE, "libfsmspec.so")  # override: experiments only
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-Xptxas", "-v", "--expt-relaxed-constexpr"]
UNITS = ["fsmspec", "kernels_p4", "kernels_p8", "kernels_b", "kernels_g", "kernels_hs", "kernels_cl", "kernels_n8", "kernels_r16", "kernels_rg"]


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cuh"))
                  + glob.glob(os.path.join(CSRC, "*.h")) + [os.path.join(ROOT, "include", "fsmspec.h")])


def stale() -> bool:
    if not os.path.exists(SO):
        return True
    t = os.path.getmtime(SO)
    return any(os.path.getmtime(s) > t for s in sources())


OBJ = os.path.join(HERE, "build")  # per-unit objects (git-ignored), reused when their inputs are unchanged


def _unit_stale(u: str, obj: str) -> bool:
    """A kernel unit depends on its .cu and every header; fsmspec.cu (host side) on itself, the
    headers and the public header.  Host-only edits therefore relink without recompiling kernels."""
    if not os.path.exists(obj):
        return True
    deps = [os.path.join(CSRC, u + ".cu")] + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        glob.glob(os.path.join(CSRC, "*.h")) + [os.path.join(ROOT, "include", "fsmspec.h"), __file__]
    t = os.path.getmtime(obj)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile the translation units in parallel (one per table variant) and link the .so."""
    if not force and not stale():
        return SO
    import concurrent.futures as cf

    os.makedirs(OBJ, exist_ok=True)
    log = os.path.join(HERE, "build.log")
    extra = os.environ.get("FSMSPEC_EXTRA_FLAGS", "").split()  # experiments only

    def unit(u):
        obj = os.path.join(OBJ, u + ".o")
        cmd = [NVCC, *FLAGS, *extra, "-I", os.path.join(ROOT, "include"), "-c", "-o", obj, os.path.join(CSRC, u + ".cu")]
        if not (force or extra) and not _unit_stale(u, obj):
            return u, obj, cmd, None
        res = subprocess.run(cmd, capture_output=True, text=True)
        if res.returncode != 0 and os.path.exists(obj):
            os.remove(obj)
        return u, obj, cmd, res

    with cf.ThreadPoolExecutor(len(UNITS)) as ex:
        results = list(ex.map(unit, UNITS))
    with open(log, "a" if not force else "w") as fh:
        for u, obj, cmd, res in results:
            if res is not None:
                fh.write(" ".join(cmd) + "\n" + res.stdout + res.stderr)
    results = [(u, o, c, r if r is not None else subprocess.CompletedProcess(c, 0, "", "")) for u, o, c, r in results]
    bad = [(u, r) for u, _, _, r in results if r.returncode != 0]
    if bad:
        raise RuntimeError(f"nvcc failed for {bad[0][0]} (see {log}):\n{bad[0][1].stderr[-4000:]}")
    cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", SO + ".tmp",
           *[o for _, o, _, _ in results]]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        raise RuntimeError(f"link failed:\n{res.stderr[-4000:]}")
    os.replace(SO + ".tmp", SO)
    if verbose:
        print(open(log).read()[-2000:])
    return SO


if __name__ == "__main__":
    import time

    t = time.time()
    build(force=True)
    print(f"built {SO} in {time.time() - t:.1f}s")
