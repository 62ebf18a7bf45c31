"""Multi-GPU spec-k: contiguous shards, one all-gather of k-slot shard mappings, compose, fix-up.

SURVEY.md 8.e.  Rank g owns bytes [lo_g, hi_g) of the input plus the look-back byte before it
(the halo).  Each rank runs its shard through the C ABI (fsm_run_shard): shard 0 from q0, shard
g > 0 keyed on S_g = look-back(halo) -- exactly as a chunk is speculated -- producing a
k-slot mapping.  The mappings are all-gathered (the only collective; a few hundred bytes,
latency-bound), every rank composes M_0 x ... x M_{G-1} from q0 with the delayed rule (a miss is
not re-executed speculatively), and the first shard whose true start was not speculated
runs the fix-up (fsm_shard_fixup) and broadcasts its (end, count).  At most G fix-up rounds; zero
when k >= |image(halo)|.  Torch is used only for the process group and device buffers.
"""
from __future__ import annotations

import numpy as np

from .fsmspec import FSM_KMAX, FSM, fsm_shard_map

_MAPW = 2 + 3 * FSM_KMAX  # k, valid_mask, start[16], end[16], count[16]


def _pack(m: fsm_shard_map) -> np.ndarray:
    v = np.zeros(_MAPW, np.int64)
    v[0], v[1] = m.k, m.valid_mask
    v[2:2 + FSM_KMAX] = list(m.start)
    v[2 + FSM_KMAX:2 + 2 * FSM_KMAX] = list(m.end)
    v[2 + 2 * FSM_KMAX:] = np.array(list(m.count), dtype=np.uint64).view(np.int64)
    return v


def _unpack(v: np.ndarray) -> list[tuple[int, int, int]]:
    mask = int(v[1])
    cnt = v[2 + 2 * FSM_KMAX:].view(np.uint64)
    return [(int(v[2 + s]), int(v[2 + FSM_KMAX + s]), int(cnt[s])) for s in range(FSM_KMAX) if (mask >> s) & 1]


def compose_from(q0: int, maps: list[list[tuple[int, int, int]]], start_at: int = 0, x: int | None = None,
                 total: int = 0):
    """Fold the gathered shard maps from a known state; returns (state, count, first_miss_or_None)."""
    x = q0 if x is None else x
    for g in range(start_at, len(maps)):
        hit = [(e, c) for s, e, c in maps[g] if s == x]
        if not hit:
            return x, total, g
        x, total = hit[0][0], total + hit[0][1]
    return x, total, None


def run_sharded(f: FSM, shard_ptr: int, shard_len: int, halo_ptr: int | None, k: int, q0: int,
                group=None, device=None):
    """Run this rank's shard and complete the cross-GPU merge.  Returns (final_state, count) on
    every rank.  ``shard_len`` is in symbols (bits in bit mode; every shard but the last must be
    a whole number of bytes)."""
    import torch
    import torch.distributed as dist

    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    m, shard = f.run_shard(shard_ptr, shard_len, halo=halo_ptr if rank else None,
                           halo_len=1 if rank else 0, k=k, keep=True)
    mine = torch.from_numpy(_pack(m)).to(device)
    if dist.get_backend(group) == "nccl":
        allm = torch.empty(world * _MAPW, dtype=torch.int64, device=device)
        dist.all_gather_into_tensor(allm, mine, group=group)   # the one collective (NVLink/NVSwitch)
        host = allm.cpu().numpy().reshape(world, _MAPW)
    else:  # gloo (CPU tests of this host logic)
        parts = [torch.empty_like(mine) for _ in range(world)]
        dist.all_gather(parts, mine, group=group)
        host = torch.stack(parts).cpu().numpy()
    maps = [_unpack(host[g]) for g in range(world)]
    x, total, miss = compose_from(q0, maps)
    fix = torch.zeros(2, dtype=torch.int64, device=device)
    while miss is not None:
        if rank == miss:
            e, c = f.shard_fixup(shard, x)
            fix[0], fix[1] = e, np.int64(np.uint64(c).view(np.int64))
        dist.broadcast(fix, src=dist.get_global_rank(group, miss) if group is not None else miss, group=group)
        e, c = fix.cpu().numpy()
        x, total, miss = compose_from(q0, maps, miss + 1, int(e), total + int(np.int64(c).view(np.uint64)))
    shard.close()
    return x, total
