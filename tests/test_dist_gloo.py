"""Multi-process (gloo, CPU) tests of the cross-GPU shard merge host logic:
all-gather of k-slot shard maps, composition from q0, and the fix-up rounds for shard-boundary
misses.  The per-shard device work is replaced by a test double computed with the oracle model
(the GPU path itself is covered by tests/test_gpu_parity.py::test_shard_maps_compose_and_fixup)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from fsmgen import dfas, streams
from oracle import seq, speck
from paper_conf_ppopp_xiaja20_b200 import dist as fdist
from paper_conf_ppopp_xiaja20_b200 import fsmspec
from paper_conf_ppopp_xiaja20_b200.fsmspec import fsm_shard_map


class _Shard:
    def __init__(self, data):
        self.data = data

    def close(self):
        pass


class OracleShardFSM:
    """Test double with the FSM shard API, backed by the oracle model."""

    def __init__(self, d, data):
        self.d, self.data = d, data
        self.fixups = 0

    def run_shard(self, ptr, length, halo=None, halo_len=0, k=1, keep=False):
        lo = ptr
        shard = self.data[lo:lo + length]
        if int(shard.max(initial=0)) >= self.d.alphabet:  # the library's sink rule (reading A14)
            raise fsmspec.SymbolError(fsmspec.FSM_ESYMBOL, "fsm_run_shard")
        starts = [self.d.start] if not halo_len else speck.lookback(self.d.table, int(self.data[lo - 1]), k)
        ends, counts = speck.shard_map(self.d, shard, length, starts)
        m = fsm_shard_map()
        m.k = k
        for s, (st, e, c) in enumerate(zip(starts, ends, counts)):
            m.valid_mask |= 1 << s
            m.start[s], m.end[s], m.count[s] = st, e, c
        return m, (_Shard(shard) if keep else None)

    def shard_fixup(self, shard, x):
        self.fixups += 1
        return seq.run_from(self.d, x, shard.data)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, m, k, L, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    d = dfas.random_dfa(n, m, seed=100 + n + m)
    data = streams.splitmix_bytes(3, 0, L)
    lo = L * rank // world
    hi = L * (rank + 1) // world
    f = OracleShardFSM(d, data)
    res = fdist.run_sharded(f, lo, hi - lo, lo - 1 if rank else None, k, d.start, device=torch.device("cpu"))
    q.put((rank, res, f.fixups))
    dist.destroy_process_group()


@pytest.mark.parametrize("world,n,m,k", [(2, 8, 2, 2), (2, 16, 5, 1), (3, 8, 4, 1), (4, 16, 3, 3)])
def test_run_sharded_gloo(world, n, m, k):
    L = 4000
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, n, m, k, L, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    d = dfas.random_dfa(n, m, seed=100 + n + m)
    exp = seq.run(d, streams.splitmix_bytes(3, 0, L))
    for rank, res, _ in out:
        assert tuple(res) == exp, (rank, res, exp)
    if k >= m:
        assert all(fx == 0 for _, _, fx in out)     # k >= |image(halo)|: no fix-up round


def _map(slots):
    m = fsm_shard_map()
    m.k = len(slots)
    for s, (st, e, c) in enumerate(slots):
        m.valid_mask |= 1 << s
        m.start[s], m.end[s], m.count[s] = st, e, c
    return m


def test_compose_from_in_library():
    """fsm_compose_from (the C-ABI membership check over shard maps) on hand-made maps."""
    maps = [_map([(0, 3, 5)]), _map([(3, 1, 2), (4, 2, 0)]), _map([(1, 0, 7)])]
    assert fsmspec.compose_from(maps, 0) == (0, 14, 3)
    x, t, miss = fsmspec.compose_from([_map([(0, 4, 1)]), _map([(3, 1, 2)]), _map([(1, 0, 7)])], 0)
    assert (x, t, miss) == (4, 1, 1)
    assert fsmspec.compose_from([], 5, 9) == (5, 9, 0)
    big = _map([(2, 2, (1 << 40) + 3)])
    assert fsmspec.compose_from([big, big], 2, 1) == (2, (1 << 41) + 7, 2)   # u64 counts


def _worker_bad(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    d = dfas.c_comment(False)   # 3-symbol alphabet
    data = np.array([0, 1, 2, 2] * 500, np.uint8)
    data[1500] = 9              # out of alphabet, inside rank 1's shard
    L = data.size
    lo, hi = L * rank // world, L * (rank + 1) // world
    try:
        fdist.run_sharded(OracleShardFSM(d, data), lo, hi - lo, lo - 1 if rank else None, 2, d.start,
                          device=torch.device("cpu"))
        q.put((rank, "no error"))
    except fsmspec.SymbolError:
        q.put((rank, "esymbol"))
    dist.destroy_process_group()


def test_run_sharded_reports_out_of_alphabet_on_every_rank():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker_bad, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=120) for _ in ps)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert out == [(0, "esymbol"), (1, "esymbol")]
