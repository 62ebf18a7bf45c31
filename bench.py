#!/usr/bin/env python
"""bench.py -- input GB/s of spec-k FSM execution on B200 (BASELINE.json metric), one JSON line.

Default workload = BASELINE configs[4] (C5, the config the metric is quoted on at 1/2/4/8 B200):
a random (N, m) DFA over 64 GiB of counter-based i.i.d. bytes generated in place in HBM, sharded
contiguously over the ranks (strong scaling).  --config picks another BASELINE config.

A step = one pass of the whole hot path over the whole input: look-back speculation, local
spec-k processing, warp/block/grid parallel merge, delayed re-execution and (N > 1) the NCCL
all-gather of shard maps + compose + fix-up.  `value` = input bytes of all ranks / max-over-ranks
device time per step (CUDA events on the library's stream), inputs resident in HBM.
`e2e` = the same metric through fsm_run_spec_k_host from pinned HOST memory (H2D inside).
`--impl reference` times the oracle (oracle/, plain sequential loop of Fig. 1c) on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import re
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

GiB = 1 << 30
METRIC = "input GB/s (final state+accept count bit-exact)"


# ----------------------------------------------------------------------------- workloads
def make_workload(args):
    """Returns dict(dfa, k, name, total, bits, and either data (host array, generated once) or
    fill(dev_ptr, lo, n, stream) + host(lo, n) for the counter-based C5 stream)."""
    from fsmgen import dfas, streams

    seed = streams.MASTER_SEED
    cfg = args.config
    gib = args.size_gib
    if cfg == "c5":
        d = dfas.random_dfa(args.n_states, args.m, seed=seed + 5)
        total = int((gib or 64.0) * GiB)
        sseed = seed + 5

        def fill(ptr, lo, n, stream=0):
            streams.splitmix_fill_device(ptr, sseed, lo, n, stream)

        def host(lo, n, out=None):
            # multi-threaded host regeneration of the same counter-based stream
            import concurrent.futures as cf

            if out is None:
                out = np.empty(n, dtype=np.uint8)
            piece = 1 << 28
            with cf.ThreadPoolExecutor(os.cpu_count()) as ex:
                list(ex.map(lambda o: streams.splitmix_bytes(sseed, lo + o, min(piece, n - o), out=out[o:]),
                            range(0, n, piece)))
            return out[:n]

        name = (f"C5 random DFA N={args.n_states} m={args.m} (|image(c)|=m), spec-{args.k}, "
                f"{total / GiB:g} GiB i.i.d. bytes")
        return dict(dfa=d, k=args.k, name=name, total=total, fill=fill, host=host, bits=False)
    if cfg == "c1":
        d = dfas.c_comment(True)
        total = int((gib or 1.0 / 1024) * GiB)
        data = streams.c_source(total, seed=seed + 1)
        k = args.k_override or 1
        return dict(dfa=d, k=k, name=f"C1 C-comment FSM (Fig. 1, 4 states x 3 classes) on {total} B synthetic C, spec-{k}",
                    total=total, data=data, bits=False)
    if cfg == "c2":
        w = dfas.zipf_weights(256, seed=seed + 2)
        d, codes = dfas.huffman(w.tolist())
        nbytes = int((gib or 1.0) * GiB)
        data, _ = streams.huffman_stream(codes, w, nbytes * 8, seed + 2)
        k = args.k_override or 4
        return dict(dfa=d, k=k, name=f"C2 Huffman decoder (Zipf-1, 256 symbols, {d.n_states} states, bit alphabet) "
                    f"on {nbytes / GiB:g} GiB encoded bitstream, spec-{k}", total=nbytes, data=data, bits=True)
    if cfg == "c3":
        pats = dfas.snort_patterns(args.ac_states, seed=seed + 3)
        d = dfas.aho_corasick(pats)
        total = int((gib or 4.0) * GiB)
        data = streams.ac_payload(total, seed + 3, pats)
        k = args.k_override or 1
        return dict(dfa=d, k=k, name=f"C3 Snort-style Aho-Corasick DFA ({d.n_states} states, 256 symbols) on "
                    f"{total / GiB:g} GiB synthetic packet payloads, spec-{k}", total=total, data=data, bits=False)
    if cfg == "c4":
        d = dfas.html_tokenizer()
        total = int((gib or 8.0) * GiB)
        data = streams.html_bytes(total, seed + 4)
        k = args.k_override or 1
        return dict(dfa=d, k=k, name=f"C4 HTML tokenizer (38 states) on {total / GiB:g} GiB synthetic HTML, spec-{k}",
                    total=total, data=data, bits=False)
    raise SystemExit(f"unknown config {cfg}")


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []      # (arrival time, fields)
        self.proc = None
        self.window = None  # (start, end) of the timed region, time.monotonic()

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "20"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            t0 = time.monotonic()
            while not self.rows and time.monotonic() - t0 < 5.0:  # sampler running before timing starts
                time.sleep(0.01)
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append((time.monotonic(), [x.strip() for x in line.split(",")]))

    def start(self):
        self.window = [time.monotonic(), None]

    def stop(self):
        time.sleep(0.05)  # let the sample covering the end arrive
        self.window[1] = time.monotonic()

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            self.proc.wait()

    def summary(self):
        rows = self.rows
        if self.window and self.window[1]:
            inside = [r for t, r in rows if self.window[0] <= t <= self.window[1]]
            rows = inside if inside else [r for _, r in rows[-2:]]
        else:
            rows = [r for _, r in rows]
        sm = [float(r[0]) for r in rows if r and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if len(r) > 1 and r[1].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            for i, nme in enumerate(names):
                if len(r) > 4 + i and r[4 + i].lower() == "active":
                    reasons.add(nme)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------------------- reference arm
def cpu_oracle_rate(w, budget_s: float = 12.0, max_bytes: int = 4 * GiB):
    """Time the oracle (plain sequential loop, 1 core) on a bounded prefix sample."""
    from oracle import seq

    d = w["dfa"]
    n = min(w["total"], max_bytes)
    probe = min(n, 64 << 20)
    data = w["data"][:probe] if "data" in w else w["host"](0, probe)
    t = time.perf_counter()
    seq.run(d, data)
    dt = time.perf_counter() - t
    rate = probe / dt
    n = int(min(n, max(probe, rate * budget_s)))
    data = w["data"][:n] if "data" in w else w["host"](0, n)
    t = time.perf_counter()
    res = seq.run(d, data)
    dt = time.perf_counter() - t
    return dict(bytes=n, seconds=dt, gbs=n / dt / 1e9, result=res)


def run_reference(args, w):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    try:
        os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
    except (AttributeError, OSError):
        pass
    rates = []
    for i in range(args.warmup + args.steps):
        r = cpu_oracle_rate(w, budget_s=min(10.0, 120.0 / (args.warmup + args.steps)), max_bytes=2 * GiB)
        if i >= args.warmup:
            rates.append(r)
    gbs = statistics.median(r["gbs"] for r in rates)
    line = {"impl": "reference", "metric": METRIC, "value": round(gbs, 4), "unit": "GB/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(statistics.median(r["seconds"] for r in rates) * 1e3, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic", "config": config_json(args, w),
            "cpu_baseline": {"value": round(gbs, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": f"first {rates[0]['bytes']} bytes of the workload per step"},
            "e2e": {"value": round(gbs, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def config_key(args, w):
    """Key of this workload in profiles/ncu_metrics.json (the ncu capture of the same config)."""
    if args.config == "c5":
        return f"c5_n{args.n_states}_m{args.m}_k{w['k']}"
    return f"{args.config}_k{w['k']}" + (f"_ac{args.ac_states}" if args.config == "c3" else "")


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def config_json(args, w):
    return {"workload": w["name"], "input_bytes": w["total"], "k": w["k"], "lookback_len": w.get("lookback"),
            "input_offset": args.offset,
            "eager_window": w.get("eager", 0), "lookback_width": w.get("width", 0),
            "n_states": int(w["dfa"].n_states), "parallelism": f"shard{args.gpus}",
            "l2": "input >> L2 (126 MB), no flush needed" if w["total"] > 4 * 126e6 else "L2 flushed between steps"}


def certify_full(args, w, f, buf, n, k, final):
    """Full-length parity of the timed configuration, part of the CPU-baseline leg.
    The GPU claims the state at G segment boundaries (chained fsm_run_shard maps + fixups); every
    host core runs the plain sequential loop (oracle) over its segment from the claimed start,
    streaming the regenerated input; the check passes iff segment 0 starts in q0, each segment
    ends where the next one claims to start, and the chained (end, count) equals the fused
    kernel's result.  By induction that is the sequential oracle over the whole input."""
    from fsmgen import streams
    from oracle import seq
    from paper_conf_ppopp_xiaja20_b200.fsmspec import compose_from

    t0 = time.perf_counter()
    d = w["dfa"]
    G = max(1, min(os.cpu_count() or 1, 32))
    bounds = [n * g // G // 32 * 32 for g in range(G)] + [n]
    claims, x = [], d.start
    for g in range(G):
        lo, hi = bounds[g], bounds[g + 1]
        claims.append(x)
        m, sh = f.run_shard(buf.data_ptr() + lo, hi - lo, halo=(buf.data_ptr() + lo - 1) if g else None,
                            halo_len=1 if g else 0, k=k, keep=True)
        x2, _, miss = compose_from([m], x)
        x = x2 if miss == 1 else f.shard_fixup(sh, x)[0]
        sh.close()
    sseed = streams.MASTER_SEED + 5
    try:
        end, total = seq.certify(d, bounds, claims, lambda lo, hi: streams.splitmix_bytes(sseed, lo, hi - lo), threads=G)
        ok = (end, total) == tuple(final)
    except seq.CertificateError:
        ok = False
    return {"bytes": n, "segments": G, "cores": G, "ok": bool(ok), "seconds": round(time.perf_counter() - t0, 1),
            "method": "GPU-claimed segment starts, oracle loop per segment on its own core (induction)"}


# ----------------------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c5", choices=["c1", "c2", "c3", "c4", "c5"])
    ap.add_argument("--k-override", type=int, default=0, help="k for c1-c4 (c5 uses --k)")
    ap.add_argument("--ac-states", type=int, default=1024, help="c3: minimum Aho-Corasick states (1024 / 4096)")
    ap.add_argument("--n-states", type=int, default=8)
    ap.add_argument("--image", "--m", dest="m", type=int, default=2,
                    help="C5: |image(c)| of the random DFA (--image under torchrun: --m is ambiguous there)")
    ap.add_argument("--k", type=int, default=2)
    ap.add_argument("--size-gib", type=float, default=0.0, help="input size (default: the config's)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-certify", action="store_true", help="skip the full-length certificate (C5)")
    ap.add_argument("--variant", type=int, default=-1)
    ap.add_argument("--offset", type=int, default=0,
                    help="start the input this many bytes past a 32-byte boundary (unaligned-input path, R10)")
    ap.add_argument("--lookback", type=int, default=-1,
                    help="look-back window bytes (R7; -1 = the config's default: c5 0, c1/c4 64, c2/c3 32)")
    ap.add_argument("--chunk", type=int, default=0)
    ap.add_argument("--lb-width", type=int, default=0,
                    help="look-back window walk over the top 4/8/12/16 image states only (0 = the whole image)")
    ap.add_argument("--eager", type=int, default=0,
                    help="eager-completion window bytes (NEXT-3): 0 = library default (128), 1 = off, 32..128")
    ap.add_argument("--tune", action="store_true",
                    help="NEXT-2: fsm_autotune the look-back and eager windows on a prefix sample before timing")
    ap.add_argument("--tune-k", action="store_true", help="with --tune: also choose k in [1, min(16, N)]")
    ap.add_argument("--no-ablation", action="store_true",
                    help="skip the sequential-merge ablation run (Fig. 4a, SURVEY 8.a11)")
    args = ap.parse_args()
    w = make_workload(args)
    w["lookback"] = args.lookback if args.lookback >= 0 else {"c5": 0, "c1": 64, "c4": 64, "c2": 32, "c3": 32}[args.config]
    if args.impl == "reference":
        return run_reference(args, w)

    import torch
    import torch.distributed as dist

    from paper_conf_ppopp_xiaja20_b200 import fsmspec
    from paper_conf_ppopp_xiaja20_b200.dist import run_sharded
    from paper_conf_ppopp_xiaja20_b200.fsmspec import FSM

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # test hook: FSM_BENCH_BACKEND=gloo runs the N > 1 host logic with every rank on GPU 0 (NCCL
    # refuses two ranks on one GPU); the contract run always uses NCCL, one rank per GPU
    backend = os.environ.get("FSM_BENCH_BACKEND", "nccl")
    if backend != "nccl":
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cdev = dev if backend == "nccl" else torch.device("cpu")  # device of the collectives' tensors
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    d = w["dfa"]
    k = w["k"]
    total = w["total"]
    lo = total * rank // world // 32 * 32
    hi = total if rank == world - 1 else total * (rank + 1) // world // 32 * 32
    n = hi - lo
    nsym = n * 8 if w["bits"] else n   # the library counts symbols: bits in bit mode
    off = args.offset
    base = torch.empty(n + 64 + off, dtype=torch.uint8, device=dev)
    buf = base[off:]  # buf.data_ptr() is base + off: unaligned when off % 32 != 0
    halo = torch.zeros(32, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)
    if "data" in w:
        buf[:n] = torch.from_numpy(w["data"][lo:hi]).to(dev)
        if rank:
            halo[0] = int(w["data"][lo - 1])
    else:
        w["fill"](buf.data_ptr(), lo, n, stream.cuda_stream)
        if rank:
            w["fill"](halo.data_ptr(), lo - 1, 1, stream.cuda_stream)
    torch.cuda.synchronize()

    f = FSM.from_dfa(d)
    f.set_stream(stream.cuda_stream)
    lookback = w["lookback"]
    eager = args.eager
    w["eager"] = eager
    f.set_options(variant=args.variant, chunk_bytes=args.chunk, lookback_len=lookback, eager_window=eager,
                  lookback_width=args.lb_width)
    w["width"] = args.lb_width
    tuning = None
    if args.tune:
        # offline, like fsm_create (not timed): the measured cost model picks the windows (and k)
        tuning = f.autotune(buf.data_ptr(), nsym, k_min=0 if args.tune_k else k, k_max=0 if args.tune_k else k)
        k, lookback, eager = tuning["k"], tuning["lookback_len"], tuning["eager_window"]
        w["k"], w["lookback"], w["eager"], w["width"] = k, lookback, eager, tuning["lookback_width"]
        w["name"] = re.sub(r"spec-\d+", f"spec-{k} (tuned)", w["name"])
    res = torch.zeros(4, dtype=torch.int32, device=dev)
    small = total < 4 * 126_000_000
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev) if small else None

    def step():
        if world == 1:
            f.run_spec_k_async(buf.data_ptr(), nsym, k, res.data_ptr())
            return None
        return run_sharded(f, buf.data_ptr(), nsym, halo.data_ptr() if rank else None, k, d.start,
                           device=cdev)

    # parity gate on the bench's own launch configuration: the prefix sample the oracle also times
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    times = []
    with ClockSampler(local) as clk:
        clk.start()
        for _ in range(args.steps):
            if flush is not None:
                flush.zero_()
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            out = step()
            e1.record(stream)
            torch.cuda.synchronize()
            times.append(e0.elapsed_time(e1) / 1e3)
        clk.stop()
    t = torch.tensor([statistics.median(times)], dtype=torch.float64, device=cdev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    step_s = float(t.item())
    st = f.stats() if world == 1 else {}
    if world == 1:
        f.run_spec_k(buf.data_ptr(), nsym, k)
        st = f.stats()
    r = res.cpu().numpy().view(np.uint32)
    final = (int(r[0]), int(r[2]) | (int(r[3]) << 32)) if world == 1 else out

    # ---- e2e through the host-buffer C-ABI entry point (pinned host memory, H2D in the region)
    e2e = None
    if not args.no_e2e:
        try:
            import psutil
            avail = psutil.virtual_memory().available
        except Exception:
            avail = 0
        fits = n * world + (8 << 30) < avail * 0.8  # every rank pins its shard in the same host RAM
        if world > 1:
            flag = torch.tensor([1 if fits else 0], dtype=torch.int32, device=cdev)
            dist.all_reduce(flag, op=dist.ReduceOp.MIN)  # all ranks take the same branch
            fits = bool(flag.item())
        if fits:
            hbuf = torch.empty(n, dtype=torch.uint8, pin_memory=True)
            hview = hbuf.numpy()
            if "data" in w:
                hview[:] = w["data"][lo:hi]
            else:
                w["host"](lo, n, out=hview)
            if world == 1:
                et = []
                for i in range(max(1, min(args.steps, 3)) + 1):
                    torch.cuda.synchronize()
                    t0 = time.perf_counter()
                    got = f.run_spec_k_host(hbuf.data_ptr(), nsym, k)
                    dt = time.perf_counter() - t0
                    if i:
                        et.append(dt)
                assert got == final, (got, final)
                e2e = {"value": round(n / statistics.median(et) / 1e9, 3), "unit": "GB/s",
                       "h2d_bytes_per_step": n, "d2h_bytes_per_step": 16}
            else:
                # N > 1: every rank copies its shard from pinned host memory into its device buffer
                # and runs the sharded path (shard kernel, all-gather, compose, fix-up); the step
                # time is the max over ranks; bytes are whole-job totals like `value`
                et = []
                got = None
                for i in range(max(1, min(args.steps, 3)) + 1):
                    dist.barrier()
                    torch.cuda.synchronize()
                    t0 = time.perf_counter()
                    buf[:n].copy_(hbuf, non_blocking=True)
                    got = step()
                    torch.cuda.synchronize()
                    dt = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=cdev)
                    dist.all_reduce(dt, op=dist.ReduceOp.MAX)
                    if i:
                        et.append(float(dt.item()))
                assert tuple(got) == tuple(out), (got, out)
                e2e = {"value": round(total / statistics.median(et) / 1e9, 3), "unit": "GB/s",
                       "h2d_bytes_per_step": total, "d2h_bytes_per_step": 16 * world,
                       "note": "per rank: pinned shard -> device copy + sharded run; max over ranks"}
            del hbuf
        else:
            e2e = {"value": None, "unit": "GB/s", "h2d_bytes_per_step": total, "d2h_bytes_per_step": 16,
                   "note": f"host RAM {avail / GiB:.0f} GiB too small for {world} x {n / GiB:.0f} GiB pinned buffers"}

    if rank != 0:
        dist.destroy_process_group()
        return
    gbs = total / step_s / 1e9
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except OSError:
        pass
    peak = float(peaks.get("hbm_gbs", 6650.0))
    # per-launch DRAM traffic, LDS utilisation and bank conflicts from the committed ncu capture of
    # the same config (profiles/ncu_metrics.json, written by tools/ncu_metrics.py), scaled per byte
    nm = {}
    try:
        nm = json.load(open(os.path.join(ROOT, "profiles", "ncu_metrics.json"))).get(config_key(args, w), {})
    except (OSError, ValueError):
        pass
    traffic = round(nm["dram_bytes_per_input_byte"] * n) if nm.get("dram_bytes_per_input_byte") else None
    line = {
        "metric": METRIC, "value": round(gbs, 3), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(step_s * 1e3, 4), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": config_json(args, w),
        "roofline": {"bound": "hbm", "achieved": round(n / step_s / 1e9, 3) if world == 1 else round(gbs / world, 3),
                     "peak": peak, "unit": "GB/s", "frac": round((n / step_s / 1e9) / peak, 4),
                     "traffic": traffic, "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy)" if peaks else "fallback"},
        "ncu": ({"source": nm.get("source"), "capture_input_bytes": nm.get("input_bytes"),
                 "dram_bytes_per_input_byte": nm.get("dram_bytes_per_input_byte"), "lds_util": nm.get("lds_util"),
                 "bank_conflicts_per_kib": nm.get("bank_conflicts_per_kib"), "alu_pipe_pct": nm.get("alu_pipe_pct"),
                 "issue_pct": nm.get("issue_pct")} if nm else None),
        "clocks": clk.summary(),
        # one fused kernel per step, plus the look-back window pre-pass when the window is >= 32 bytes
        # (and, for N > 1, a fix-up kernel per shard-boundary miss round)
        "gpu_launches": args.steps * (2 if (lookback or 0) >= 32 else 1),
        "result": {"final_state": final[0], "accept_count": final[1]},
        "stats": {kk: v for kk, v in st.items()},
        "reexec_rate": round(st["reexec_true"] / st["chunks"], 6) if st.get("chunks") else None,
        "e2e": e2e,
    }
    if tuning is not None:
        line["tuning"] = {kk: (round(v, 3) if isinstance(v, float) else v) for kk, v in tuning.items()}
    # achievable HBM read ceiling on the same buffer (read-only streaming kernel)
    if world == 1 and n >= (1 << 30):
        from fsmgen import _native
        sink = torch.zeros(4, dtype=torch.int32, device=dev)
        rs = []
        for i in range(4):
            if flush is not None:
                flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            rc = _native.dev_lib().fsmgen_dev_read_stream(base.data_ptr(), n, sink.data_ptr(),
                                                          torch.cuda.get_device_properties(dev).multi_processor_count,
                                                          stream.cuda_stream)
            e1.record(stream)
            torch.cuda.synchronize()
            if rc == 0 and i:
                rs.append(e0.elapsed_time(e1) / 1e3)
        if rs:
            rgbs = (n // 32 * 32) / statistics.median(rs) / 1e9
            line["roofline"]["read_ceiling"] = {"value": round(rgbs, 1), "unit": "GB/s",
                                                "frac": round((n / step_s / 1e9) / rgbs, 4),
                                                "kernel": "read-only LDG.256 stream over the same input"}
    if not args.no_ablation and world == 1:
        # internal ablation: the paper's sequential merge (Fig. 4a) on the same input and chains
        f.set_options(variant=args.variant, chunk_bytes=args.chunk, merge=fsmspec.FSM_MERGE_SEQUENTIAL,
                      lookback_len=lookback, eager_window=eager)
        f.run_spec_k_async(buf.data_ptr(), nsym, k, res.data_ptr())
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        f.run_spec_k_async(buf.data_ptr(), nsym, k, res.data_ptr())
        e1.record(stream)
        torch.cuda.synchronize()
        ts = e0.elapsed_time(e1) / 1e3
        r2 = res.cpu().numpy().view(np.uint32)
        same = (int(r2[0]), int(r2[2]) | (int(r2[3]) << 32)) == final
        f.set_options(variant=args.variant, chunk_bytes=args.chunk, merge=fsmspec.FSM_MERGE_PARALLEL,
                      lookback_len=lookback, eager_window=eager)
        line["ablation"] = {"sequential_merge_gbs": round(n / ts / 1e9, 3),
                            "parallel_over_sequential": round(ts / step_s, 2), "same_result": same,
                            "paper_v100_context": "2.02-6.74x (P:11, P:53)"}
    if not args.no_cpu and world == 1:
        try:
            all_cores = os.sched_getaffinity(0)
            os.sched_setaffinity(0, {sorted(all_cores)[0]})  # the 1-core oracle baseline
        except (AttributeError, OSError):
            all_cores = None
        cb = cpu_oracle_rate(w, budget_s=12.0)
        if all_cores:
            os.sched_setaffinity(0, all_cores)  # the certificate below uses every core
        # parity on the sampled prefix: the GPU runs the same prefix in the bench's configuration
        gp = f.run_spec_k(buf.data_ptr(), cb["bytes"] * (8 if w["bits"] else 1), k)
        line["cpu_baseline"] = {"value": round(cb["gbs"], 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                                "sample": f"first {cb['bytes']} bytes of the workload ({cb['seconds']:.1f} s)"}
        line["parity_sample"] = {"bytes": cb["bytes"], "ok": gp == cb["result"]}
        line["host_cores"] = os.cpu_count()
        line["cpu_model"] = cpu_model()
        if "host" in w and not args.no_certify:
            line["parity_full"] = certify_full(args, w, f, buf, n, k, final)
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
