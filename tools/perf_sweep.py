"""Quick device-time sweep (not the bench contract): GB/s of fsm_run_spec_k_async over C5-style
inputs for several (N, m, k, variant, chunk) points.  Usage: python tools/perf_sweep.py [GiB]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from fsmgen import dfas, streams  # noqa: E402
from paper_conf_ppopp_xiaja20_b200.fsmspec import FSM  # noqa: E402

gib = float(sys.argv[1]) if len(sys.argv) > 1 else 8
pts = json.loads(sys.argv[2]) if len(sys.argv) > 2 else [
    [8, 1, 1, -1, 0], [8, 2, 2, -1, 0], [8, 2, 1, -1, 0], [4, 2, 2, -1, 0], [16, 2, 2, -1, 0],
    [8, 4, 4, -1, 0], [8, 8, 8, -1, 0], [64, 4, 4, -1, 0], [256, 8, 8, -1, 0], [4096, 8, 8, -1, 0]]
n = int(gib * (1 << 30))
buf = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
streams.splitmix_fill_device(buf.data_ptr(), 1234, 0, n)
res = torch.zeros(4, dtype=torch.int32, device="cuda")
for N, m, k, var, chunk in pts:
    d = dfas.random_dfa(N, m, seed=N * 7 + m)
    f = FSM.from_dfa(d)
    if var >= 0 or chunk:
        f.set_options(variant=var, chunk_bytes=chunk)
    for _ in range(2):
        f.run_spec_k_async(buf.data_ptr(), n, k, res.data_ptr())
    torch.cuda.synchronize()
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        f.run_spec_k_async(buf.data_ptr(), n, k, res.data_ptr())
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    f.run_spec_k(buf.data_ptr(), n, k)
    st = f.stats()
    t = min(ts)
    print(json.dumps({"N": N, "m": m, "k": k, "var": st["variant"], "T": st["threads_per_tile"],
                      "chunk": st["chunk_bytes"], "GBps": round(n / t / 1e9, 1), "ms": round(t * 1e3, 3),
                      "reexec": st["reexec_chunks"], "bmiss": st["boundary_misses"]}), flush=True)
    f.close()
