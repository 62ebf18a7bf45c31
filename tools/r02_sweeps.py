#!/usr/bin/env python
"""Round-2 measurement sweeps on one B200 (device time, CUDA events, median of 5; results checked
against a first run and, for the smaller configs, the oracle).  One JSON line per point.

  --sweep r5     delayed re-execution across tiles: fsm_options.preresolve (R5) in {all, top-1,
                 none} x k on C2 (Huffman bits) and C4 (HTML): GB/s and the split counters
  --sweep check  Alg. 1 (nested loop) vs Alg. 2 (hash) runtime check at k = 12 / 16 (a5)
  --sweep grid   a11: parallel vs sequential merge at 37 / 74 / 148 SMs (Figs. 7-11 vary the
                 number of thread blocks)
"""
from __future__ import annotations

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

GiB = 1 << 30
SEED = streams.MASTER_SEED


def workload(name, gib):
    if name == "c2":
        w = dfas.zipf_weights(256, seed=SEED + 2)
        d, codes = dfas.huffman(w.tolist())
        n = int(gib * GiB)
        data, _ = streams.huffman_stream(codes, w, n * 8, SEED + 2)
        return d, data[:n], n * 8, 32
    if name == "c4":
        n = int(gib * GiB)
        return dfas.html_tokenizer(), streams.html_bytes(n, SEED + 4), n, 64
    if name.startswith("rand"):
        nn, m = (int(x) for x in name[4:].split("_"))
        n = int(gib * GiB)
        return dfas.random_dfa(nn, m, seed=SEED + 5), None, n, 0
    raise SystemExit(name)


def device_input(data, n):
    buf = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
    if data is None:
        streams.splitmix_fill_device(buf.data_ptr(), SEED + 5, 0, n, torch.cuda.current_stream().cuda_stream)
    else:
        buf[:n] = torch.from_numpy(data[:n]).cuda()
    torch.cuda.synchronize()
    return buf


def timed(f, ptr, nsym, k, reps=5):
    res = torch.zeros(4, dtype=torch.int32, device="cuda")
    s = torch.cuda.current_stream()
    f.set_stream(s.cuda_stream)
    f.run_spec_k_async(ptr, nsym, k, res.data_ptr())
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        f.run_spec_k_async(ptr, nsym, k, res.data_ptr())
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    r = res.cpu().numpy().view(np.uint32)
    return statistics.median(ts), (int(r[0]), int(r[2]) | (int(r[3]) << 32)), f.stats()


def emit(out, **kv):
    line = json.dumps(kv)
    print(line, flush=True)
    out.write(line + "\n")
    out.flush()


def sweep_r5(out, gib):
    for cfg in ("c4", "c2"):
        d, data, nsym, lb = workload(cfg, gib)
        nbytes = nsym // 8 if d.bit_mode else nsym
        buf = device_input(data, nbytes)
        ref = None
        with FSM.from_dfa(d) as f:
            for k in (1, 2, 4, 8, 16):
                for pre, name in ((0, "all"), (1, "top1"), (fsmspec.FSM_PRERESOLVE_NONE, "none")):
                    f.set_options(lookback_len=lb, preresolve=pre)
                    t, got, st = timed(f, buf.data_ptr(), nsym, k)
                    ref = ref or got
                    emit(out, sweep="r5", config=cfg, gib=gib, k=k, preresolve=name, gbs=round(nbytes / t / 1e9, 1),
                         ok=got == ref, chunks=st["chunks"], reexec_true=st["reexec_true"],
                         reexec_candidate=st["reexec_candidate"], boundary_misses=st["boundary_misses"],
                         eager_resolved=st["eager_resolved"], max_miss_chain=st["max_miss_chain"],
                         reexec_rate=round(st["reexec_true"] / max(1, st["chunks"]), 5), variant=st["variant"])


def sweep_check(out, gib):
    for cfg, var in (("c4", 6), ("rand64_16", 2), ("rand16_16", 8), ("rand1000_16", 3), ("rand255_16", 2)):
        d, data, nsym, lb = workload(cfg, gib)
        buf = device_input(data, nsym)
        ref = None
        with FSM.from_dfa(d) as f:
            for k in (12, 16):
                if k > d.n_states:
                    continue
                for chk, name in ((fsmspec.FSM_CHECK_NESTED, "alg1_nested"), (fsmspec.FSM_CHECK_HASH, "alg2_hash")):
                    f.set_options(lookback_len=lb, check=chk, variant=var)
                    t, got, st = timed(f, buf.data_ptr(), nsym, k)
                    ref = ref or got
                    emit(out, sweep="check", config=cfg, gib=gib, k=k, check=name, used=st["check"],
                         variant=st["variant"], T=st["threads_per_tile"], gbs=round(nsym / t / 1e9, 1), ok=got == ref)
            ref = None


def sweep_grid(out, gib, scaled=False):
    """scaled=False: the library's fixed 4 KiB chunks at every grid size.  scaled=True: the number
    of chunks grows with the grid like the paper's one-chunk-per-thread kernel (chunk bytes =
    2048 x 148 / SMs), so the sequential merge walks more chunks on bigger grids (Figs. 7-11)."""
    for cfg, ks in (("c4", (1, 4)), ("c2", (4,))):
        d, data, nsym, lb = workload(cfg, gib)
        nbytes = nsym // 8 if d.bit_mode else nsym
        buf = device_input(data, nbytes)
        with FSM.from_dfa(d) as f:
            for k in ks:
                ref = None
                for sms in (37, 74, 148):
                    row = {}
                    chunk = 2048 * 148 // sms if scaled else 0
                    for merge, name in ((fsmspec.FSM_MERGE_PARALLEL, "parallel"), (fsmspec.FSM_MERGE_SEQUENTIAL, "sequential")):
                        f.set_options(lookback_len=lb, merge=merge, grid_sms=sms, chunk_bytes=chunk)
                        t, got, st = timed(f, buf.data_ptr(), nsym, k, reps=3)
                        ref = ref or got
                        row[name] = (round(nbytes / t / 1e9, 1), got == ref)
                    emit(out, sweep="grid_scaled" if scaled else "grid", config=cfg, gib=gib, k=k, sms=sms,
                         chunk_bytes=st["chunk_bytes"], parallel_gbs=row["parallel"][0],
                         sequential_gbs=row["sequential"][0], ratio=round(row["parallel"][0] / row["sequential"][0], 2),
                         ok=row["parallel"][1] and row["sequential"][1],
                         paper_v100="parallel/sequential 2.02-6.74x best vs best (P:11); Huffman 289.72/355.32/407.23 vs "
                                    "60.44/55.07/39.70 x at 20/40/80 blocks (P:290, P:304-305)")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sweep", required=True, choices=["r5", "check", "grid", "grid_scaled"])
    ap.add_argument("--gib", type=float, default=1.0)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweeps.jsonl"))
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "a") as out:
        {"r5": sweep_r5, "check": sweep_check, "grid": sweep_grid,
         "grid_scaled": lambda o, g: sweep_grid(o, g, True)}[a.sweep](out, a.gib)


if __name__ == "__main__":
    main()
