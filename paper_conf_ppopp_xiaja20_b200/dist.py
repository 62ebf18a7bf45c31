"""Multi-GPU spec-k: contiguous shards, one all-gather of k-slot shard mappings, compose, fix-up.

SURVEY.md 8.e.  Rank g owns bytes [lo_g, hi_g) of the input plus the look-back byte before it
(the halo).  Each rank runs its shard through the C ABI (fsm_run_shard): shard 0 from q0, shard
g > 0 keyed on S_g = look-back(halo) -- exactly as a chunk is speculated -- producing a
k-slot mapping.  The mappings are all-gathered (the only collective; a few hundred bytes,
latency-bound), every rank composes M_0 x ... x M_{G-1} from q0 with the library's
fsm_compose_from (the membership check of Alg. 1 on shard maps; a miss is not re-executed
speculatively), and the first shard whose true start was not speculated runs the fix-up
(fsm_shard_fixup) and broadcasts its (end, count).  At most G fix-up rounds; zero when
k >= |image(halo)|.  This module only marshals: the composition and every re-execution run in
libfsmspec; torch supplies the process group and device buffers.
"""
from __future__ import annotations

import numpy as np

from .fsmspec import FSM_ESYMBOL, FSM_KMAX, FSM, SymbolError, compose_from, fsm_shard_map

_MAPW = 3 + 3 * FSM_KMAX  # esymbol flag, k, valid_mask, start[16], end[16], count[16]


def _pack(m: fsm_shard_map, esymbol: bool) -> np.ndarray:
    v = np.zeros(_MAPW, np.int64)
    v[0], v[1], v[2] = int(esymbol), m.k, m.valid_mask
    v[3:3 + FSM_KMAX] = list(m.start)
    v[3 + FSM_KMAX:3 + 2 * FSM_KMAX] = list(m.end)
    v[3 + 2 * FSM_KMAX:] = np.array(list(m.count), dtype=np.uint64).view(np.int64)
    return v


def _unpack(v: np.ndarray) -> tuple[bool, fsm_shard_map]:
    m = fsm_shard_map()
    m.k, m.valid_mask = int(v[1]), int(v[2])
    for s in range(FSM_KMAX):
        m.start[s] = int(v[3 + s])
        m.end[s] = int(v[3 + FSM_KMAX + s])
    cnt = v[3 + 2 * FSM_KMAX:].view(np.uint64)
    for s in range(FSM_KMAX):
        m.count[s] = int(cnt[s])
    return bool(v[0]), m


def run_sharded(f: FSM, shard_ptr: int, shard_len: int, halo_ptr: int | None, k: int, q0: int,
                group=None, device=None):
    """Run this rank's shard and complete the cross-GPU merge.  Returns (final_state, count) on
    every rank; raises SymbolError on every rank if any shard held an out-of-alphabet byte.
    ``shard_len`` is in symbols (bits in bit mode; every shard but the last must be a whole number
    of bytes)."""
    import torch
    import torch.distributed as dist

    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    esym = False
    try:
        m, shard = f.run_shard(shard_ptr, shard_len, halo=halo_ptr if rank else None,
                               halo_len=1 if rank else 0, k=k, keep=True)
    except SymbolError:
        m, shard, esym = fsm_shard_map(), None, True
    mine = torch.from_numpy(_pack(m, esym)).to(device)
    if dist.get_backend(group) == "nccl":
        allm = torch.empty(world * _MAPW, dtype=torch.int64, device=device)
        dist.all_gather_into_tensor(allm, mine, group=group)   # the one collective (NVLink/NVSwitch)
        host = allm.cpu().numpy().reshape(world, _MAPW)
    else:  # gloo (CPU tests of this host logic)
        parts = [torch.empty_like(mine) for _ in range(world)]
        dist.all_gather(parts, mine, group=group)
        host = torch.stack(parts).cpu().numpy()
    gathered = [_unpack(host[g]) for g in range(world)]
    if any(e for e, _ in gathered):
        if shard is not None:
            shard.close()
        raise SymbolError(FSM_ESYMBOL, "run_sharded")
    maps = [mp for _, mp in gathered]
    x, total, miss = compose_from(maps, q0, 0)
    fix = torch.zeros(2, dtype=torch.int64, device=device)
    while miss < world:
        if rank == miss:
            e, c = f.shard_fixup(shard, x)
            fix[0], fix[1] = e, np.int64(np.uint64(c).view(np.int64))
        dist.broadcast(fix, src=dist.get_global_rank(group, miss) if group is not None else miss, group=group)
        e, c = fix.cpu().numpy()
        x, total, g = compose_from(maps[miss + 1:], int(e), total + int(np.int64(c).view(np.uint64)))
        miss = miss + 1 + g
    shard.close()
    return x, total
