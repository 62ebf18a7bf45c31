"""C1 (1 MiB C-comment text) geometry sweep: device time per run for chunk/threads/lookback/k."""
import itertools
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from fsmgen import dfas, streams  # noqa: E402
from paper_conf_ppopp_xiaja20_b200.fsmspec import FSM  # noqa: E402

d = dfas.c_comment(True)
data = streams.c_source(1 << 20, seed=streams.MASTER_SEED + 1)
x = torch.from_numpy(data).cuda()
res = torch.zeros(4, dtype=torch.int32, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
f = FSM.from_dfa(d)
for k, chunk, T, lb in itertools.product((1, 2), (64, 128, 256, 512, 1024), (64, 128, 256), (0, 32, 64)):
    f.set_options(chunk_bytes=chunk, threads_per_tile=T, lookback_len=lb)
    ts = []
    for i in range(8):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        f.run_spec_k_async(x.data_ptr(), data.size, k, res.data_ptr())
        e1.record()
        torch.cuda.synchronize()
        if i >= 3:
            ts.append(e0.elapsed_time(e1))
    f.run_spec_k(x.data_ptr(), data.size, k)
    st = f.stats()
    print(json.dumps({"k": k, "chunk": chunk, "T": T, "lb": lb, "us": round(min(ts) * 1e3, 1),
                      "GBps": round(data.size / min(ts) / 1e6, 2), "reexec": st["reexec_chunks"],
                      "tiles": st["tiles"]}), flush=True)
