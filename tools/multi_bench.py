#!/usr/bin/env python
"""NEXT-4 measurement: M DFAs over one resident input (the NIDS case).

Times fsm_run_multi (fused per variant/K group: the input is read from HBM about once) against M
back-to-back fsm_run_spec_k_async calls (the input is read M times), on the C5 counter-based byte
stream, and prints one JSON line per M.  Results of both are checked equal (and, on a prefix
sample, equal to the oracle).  Usage: python tools/multi_bench.py [--size-gib 8] [--ms 1,2,4,8]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from fsmgen import dfas, streams  # noqa: E402
from paper_conf_ppopp_xiaja20_b200 import fsmspec  # noqa: E402
from paper_conf_ppopp_xiaja20_b200.fsmspec import FSM  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--size-gib", type=float, default=8.0)
    ap.add_argument("--ms", default="1,2,4,8")
    ap.add_argument("--n-states", type=int, default=8)
    ap.add_argument("--m", type=int, default=2)
    ap.add_argument("--k", type=int, default=2)
    ap.add_argument("--steps", type=int, default=5)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    n = int(a.size_gib * (1 << 30))
    seed = streams.MASTER_SEED + 5
    buf = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
    streams.splitmix_fill_device(buf.data_ptr(), seed, 0, n, torch.cuda.current_stream().cuda_stream)
    stream = torch.cuda.current_stream()
    res = torch.zeros(4, dtype=torch.int32, device="cuda")
    mmax = max(int(x) for x in a.ms.split(","))
    ds = [dfas.random_dfa(a.n_states, a.m, seed=seed + 100 * i) for i in range(mmax)]
    fs = [FSM.from_dfa(d) for d in ds]
    for f in fs:
        f.set_stream(stream.cuda_stream)
    # parity on a prefix sample against the oracle
    from oracle import seq
    sample = 64 << 20
    host = streams.splitmix_bytes(seed, 0, sample)
    got = fsmspec.run_multi(fs, buf.data_ptr(), sample, [a.k] * mmax)
    ok = got == [seq.run(d, host) for d in ds]

    def timed(fn):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(a.steps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            out = fn()
            e1.record(stream)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        return statistics.median(ts), out

    for M in (int(x) for x in a.ms.split(",")):
        t_fused, r_fused = timed(lambda: fsmspec.run_multi(fs[:M], buf.data_ptr(), n, [a.k] * M))

        def separate():
            out = []
            for f in fs[:M]:
                f.run_spec_k_async(buf.data_ptr(), n, a.k, res.data_ptr())
            return out
        t_sep, _ = timed(separate)
        r_sep = [f.run_spec_k(buf.data_ptr(), n, a.k) for f in fs[:M]]
        print(json.dumps({
            "metric": "input GB/s with M DFAs per pass (NEXT-4)", "M": M,
            "workload": f"C5 random DFAs N={a.n_states} m={a.m} (seeds differ), spec-{a.k}, {n / 2**30:g} GiB",
            "fused_input_gbs": round(n / t_fused / 1e9, 1), "fused_dfa_gbs": round(M * n / t_fused / 1e9, 1),
            "separate_input_gbs": round(n / t_sep / 1e9, 1), "separate_dfa_gbs": round(M * n / t_sep / 1e9, 1),
            "fused_over_separate": round(t_sep / t_fused, 3), "same_result": r_fused == r_sep,
            "oracle_prefix_ok": ok}), flush=True)
    for f in fs:
        f.close()


if __name__ == "__main__":
    main()
