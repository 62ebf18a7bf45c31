#!/usr/bin/env python
"""Fig. 5-style state-frequency evidence for hot-state caching (Sec. 4.2; NEXT-1) on the
C3 Snort-style Aho-Corasick DFAs: the CDF of transitions over states sorted by dynamic frequency,
and the share of transitions whose source row the HS variant's *static* in-degree order (the
library's fsm_hot_state_order) would hold in shared memory for H cached rows.
Counts come from a plain visit-counting loop (a throwaway C helper built here); host only.
Usage: state_cdf.py [sample_MiB] > profiles/r02_c3_state_cdf.json"""
import ctypes
import json
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

from fsmgen import dfas, streams  # noqa: E402
from paper_conf_ppopp_xiaja20_b200 import fsmspec  # noqa: E402

SRC = r"""
#include <stdint.h>
void visits(const uint32_t *t, uint32_t q, const uint8_t *x, uint64_t n, uint64_t *cnt) {
    for (uint64_t i = 0; i < n; i++) { cnt[q]++; q = t[(uint64_t)q * 256 + x[i]]; }
}
"""


def main():
    mib = int(sys.argv[1]) if len(sys.argv) > 1 else 256
    d_ = tempfile.mkdtemp()
    open(os.path.join(d_, "v.c"), "w").write(SRC)
    so = os.path.join(d_, "v.so")
    subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", so, os.path.join(d_, "v.c")])
    lib = ctypes.CDLL(so)
    out = {"what": "C3 Aho-Corasick DFAs: CDF of transitions by source state (P:227-233, Fig. 5 analogue)",
           "sample_bytes": mib << 20}
    for min_states in (1024, 4096):
        pats = dfas.snort_patterns(min_states, seed=streams.MASTER_SEED + 3)
        d = dfas.aho_corasick(pats)
        data = streams.ac_payload(mib << 20, streams.MASTER_SEED + 3, pats)
        t = np.ascontiguousarray(d.table, np.uint32)
        cnt = np.zeros(d.n_states, np.uint64)
        lib.visits(ctypes.c_void_p(t.ctypes.data), ctypes.c_uint32(d.start), ctypes.c_void_p(data.ctypes.data),
                   ctypes.c_uint64(data.size), ctypes.c_void_p(cnt.ctypes.data))
        total = float(cnt.sum())
        dyn = np.sort(cnt)[::-1].cumsum() / total
        order = fsmspec.hot_state_order(d.table)
        stat = cnt[np.array(order)].cumsum() / total
        pts = [1, 2, 4, 8, 16, 32, 64, 128, 256, 384, 512, 1024, 2048, 4096]
        out[f"ac_{d.n_states}_states"] = {
            "n_states": d.n_states,
            "dynamic_cdf": {h: round(float(dyn[min(h, d.n_states) - 1]), 5) for h in pts if h <= d.n_states},
            "static_in_degree_order_coverage": {h: round(float(stat[min(h, d.n_states) - 1]), 5)
                                                for h in pts if h <= d.n_states},
            "states_for_95pct": int(np.searchsorted(dyn, 0.95) + 1),
            "paper_context": "RegExp1, 18 states: the 8 most frequent states take ~95 % of transitions (P:233)",
        }
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
