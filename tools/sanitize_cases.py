#!/usr/bin/env python
"""Small runs of every kernel kind for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): the fused kernel split and unsplit for each table variant, the look-back window
pre-pass, Alg. 2 kernels, the multi-FSM kernel, the sequential-merge kernels, the shard fix-up
walk, the head-peeled unaligned path and the debug merge tree.  Each result is checked against the
oracle; the sanitizer's own report is what the run is for.
Usage: compute-sanitizer --tool racecheck python tools/sanitize_cases.py [quick]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from fsmgen import dfas, streams  # noqa: E402
from oracle import seq  # noqa: E402
from paper_conf_ppopp_xiaja20_b200 import fsmspec  # noqa: E402
from paper_conf_ppopp_xiaja20_b200.fsmspec import FSM, run_multi  # noqa: E402

V = {"P4": 0, "P8": 1, "B": 2, "G": 3, "HS": 5, "CL": 6, "N8": 7, "R16": 8, "RG": 9}
L = int(os.environ.get("SAN_BYTES", 1 << 20))


def dev(data, off=0):
    buf = torch.zeros(data.size + off + 64, dtype=torch.uint8, device="cuda")
    buf[off:off + data.size] = torch.from_numpy(np.ascontiguousarray(data))
    return buf


def check(name, got, exp):
    status = "ok" if tuple(got) == tuple(exp) else f"MISMATCH {got} != {exp}"
    print(f"case {name}: {status}", flush=True)


def main():
    torch.cuda.set_device(0)
    cases = [
        ("P4", dfas.random_dfa(4, 2, seed=1), (1, 2)),
        ("N8", dfas.random_dfa(8, 2, seed=2), (1, 2)),
        ("P8", dfas.random_dfa(8, 3, seed=3), (1, 3)),
        ("R16", dfas.random_dfa(16, 3, seed=4), (1, 2)),
        ("B", dfas.random_dfa(64, 4, seed=5), (1, 4)),
        ("RG", dfas.random_dfa(64, 4, seed=5), (1, 4)),
        ("RG", dfas.random_dfa(200, 3, seed=8), (1, 2)),
        ("CL", dfas.html_tokenizer(), (1, 2)),
        ("G", dfas.random_dfa(1000, 3, seed=6), (1, 2)),
        ("HS", dfas.random_dfa(3000, 3, seed=7), (1,)),
    ]
    for var, d, ks in cases:
        data = streams.html_bytes(L, 3) if var == "CL" else streams.splitmix_bytes(11, 0, L)
        exp = seq.run(d, data)
        buf = dev(data)
        with FSM.from_dfa(d) as f:
            for k in ks:
                for lb in (0, 64):  # 64: the look-back window pre-pass (spec_kernel)
                    f.set_options(variant=V[var], lookback_len=lb, chunk_bytes=256)
                    check(f"{var} k={k} lookback={lb}", f.run_spec_k(buf.data_ptr(), L, k), exp)
            f.set_options(variant=V[var], merge=fsmspec.FSM_MERGE_SEQUENTIAL, chunk_bytes=256)
            check(f"{var} sequential merge", f.run_spec_k(buf.data_ptr(), L, ks[-1]), exp)
    # Alg. 2 kernels (K = 12, 16)
    d = dfas.random_dfa(40, 14, seed=8)
    data = streams.splitmix_bytes(12, 0, L)
    buf = dev(data)
    with FSM.from_dfa(d) as f:
        for k in (12, 16):
            f.set_options(variant=V["B"], check=fsmspec.FSM_CHECK_HASH, chunk_bytes=256)
            check(f"B hash k={k}", f.run_spec_k(buf.data_ptr(), L, k), seq.run(d, data))
    # unaligned input (head peel), eager completion on
    d = dfas.random_dfa(8, 3, seed=9)
    data = streams.splitmix_bytes(13, 0, L + 7)
    buf = dev(data, 13)
    with FSM.from_dfa(d) as f:
        check("N8 unaligned", f.run_spec_k(buf.data_ptr() + 13, data.size, 2), seq.run(d, data))
    # multi-FSM kernel
    ds = [dfas.random_dfa(8, 2, seed=20 + i) for i in range(3)]
    data = streams.splitmix_bytes(14, 0, L)
    buf = dev(data)
    fs = [FSM.from_dfa(x) for x in ds]
    got = run_multi(fs, buf.data_ptr(), L, [2, 2, 2])
    for i, x in enumerate(ds):
        check(f"multi {i}", got[i], seq.run(x, data))
    for x in fs:
        x.close()
    # shard run + fix-up walk
    d = dfas.random_dfa(16, 6, seed=21)
    data = streams.splitmix_bytes(15, 0, L)
    buf = dev(data)
    lo = L // 3 // 32 * 32
    with FSM.from_dfa(d) as f:
        m, sh = f.run_shard(buf.data_ptr() + lo, L - lo, halo=buf.data_ptr() + lo - 1, halo_len=1, k=2, keep=True)
        spec = {s for s, _, _ in m.slots()}
        for x in [q for q in range(16) if q not in spec][:3]:
            check(f"fixup from {x}", f.shard_fixup(sh, x), seq.run_from(d, x, data[lo:]))
        sh.close()
    # debug merge tree (Fig. 4)
    d = dfas.c_comment(True)
    data = np.frombuffer(b"/*xxx**/", np.uint8)
    buf = dev(data)
    with FSM.from_dfa(d) as f:
        f.debug_set_spec([[0, 2], [2, 3], [0, 2], [2, 3]], chunk_bytes=2)
        check("fig4 debug", f.run_spec_k(buf.data_ptr(), 8, 2), seq.run(d, data))
        f.debug_get_merge()
    torch.cuda.synchronize()
    print("sanitize cases done", flush=True)


if __name__ == "__main__":
    main()
