#!/usr/bin/env python
"""Time the oracle loop (oracle/fsm_oracle.c) built with -O3 and with -O3 -march=native on this
host (1 core), on the bench's default C5 workload sample -- the evidence for the oracle build flags
(SURVEY 8.d.6 asks for -march=native; the oracle library built in-tree travels to the GPU box)."""
import ctypes
import json
import os
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

from fsmgen import dfas, streams  # noqa: E402


def main():
    os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
    d = dfas.random_dfa(8, 2, seed=streams.MASTER_SEED + 5)
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 30
    data = streams.splitmix_bytes(streams.MASTER_SEED + 5, 0, n)
    t = np.ascontiguousarray(d.table, np.uint32)
    acc = np.ascontiguousarray(d.accept, np.uint8)
    out = {"bytes": n, "cpu": open("/proc/cpuinfo").read().split("model name")[1].split("\n")[0].strip(": ")}
    for name, flags in (("O3", ["-O3"]), ("O3_march_native", ["-O3", "-march=native"])):
        so = os.path.join(tempfile.mkdtemp(), "lib.so")
        subprocess.check_call(["gcc", *flags, "-shared", "-fPIC", "-o", so, os.path.join(ROOT, "oracle", "fsm_oracle.c")])
        lib = ctypes.CDLL(so)
        q, c = ctypes.c_uint32(), ctypes.c_uint64()
        best = None
        for _ in range(3):
            t0 = time.perf_counter()
            lib.oracle_run(ctypes.c_void_p(t.ctypes.data), ctypes.c_uint32(256), ctypes.c_uint32(0),
                           ctypes.c_void_p(acc.ctypes.data), ctypes.c_void_p(data.ctypes.data), ctypes.c_uint64(n),
                           ctypes.c_int(0), ctypes.byref(q), ctypes.byref(c))
            dt = time.perf_counter() - t0
            best = dt if best is None else min(best, dt)
        out[name] = {"gbs": round(n / best / 1e9, 4), "result": [q.value, c.value]}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
