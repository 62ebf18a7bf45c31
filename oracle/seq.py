"""TEST INFRASTRUCTURE ONLY -- the sequential oracle (Fig. 1c).

run(dfa, data, length)          -> (final_state, accept_count)   C loop, any size
run_py(table, start, F, syms)   -> same, pure Python (tiny cases; pins the C loop)
run_from(...)                   -> from an arbitrary start state (used for shard maps / certificates)
run_splitmix(dfa, seed, length) -> streams the counter-based C5 input through the C loop
certify(...)                    -> multi-core check of claimed segment start states
Definition: q_i = delta(q_{i-1}, x_i), count = |{i in [1, L] : q_i in F}| (readings A3, A4).
"""
from __future__ import annotations

import concurrent.futures as cf
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "fsm_oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")
ESYMBOL = -4


class OracleSymbolError(ValueError):
    """Input contained a symbol >= alphabet (reading A14)."""


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O3", "-shared", "-fPIC", "-o", _SO, _SRC])
    return _SO


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        l = ctypes.CDLL(build())
        l.oracle_run.restype = ctypes.c_int
        l.oracle_run.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p,
                                 ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int,
                                 ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint64)]
        _lib = l
    return _lib


def _arrays(dfa):
    table = np.ascontiguousarray(dfa.table, dtype=np.uint32)
    acc = np.ascontiguousarray(dfa.accept, dtype=np.uint8)
    return table, acc


def run_from(dfa, start: int, data: np.ndarray, length: int | None = None,
             _cache: tuple | None = None) -> tuple[int, int]:
    """Run the plain loop from ``start`` over ``length`` symbols of ``data`` (bits in bit mode)."""
    table, acc = _cache if _cache is not None else _arrays(dfa)
    data = np.ascontiguousarray(data, dtype=np.uint8)
    if length is None:
        length = data.size * 8 if dfa.bit_mode else data.size
    need = (length + 7) // 8 if dfa.bit_mode else length
    assert data.size >= need
    q = ctypes.c_uint32()
    n = ctypes.c_uint64()
    rc = lib().oracle_run(table.ctypes.data, table.shape[1], start, acc.ctypes.data,
                          data.ctypes.data, length, int(dfa.bit_mode), ctypes.byref(q), ctypes.byref(n))
    if rc == ESYMBOL:
        raise OracleSymbolError("symbol outside the alphabet")
    assert rc == 0
    return int(q.value), int(n.value)


def run(dfa, data: np.ndarray, length: int | None = None) -> tuple[int, int]:
    return run_from(dfa, dfa.start, data, length)


def run_py(table, start: int, accept, symbols) -> tuple[int, int]:
    """Pure-Python sequential loop over an explicit symbol sequence (tiny cases only)."""
    q = start
    cnt = 0
    for c in symbols:
        if c >= len(table[q]):
            raise OracleSymbolError("symbol outside the alphabet")
        q = int(table[q][c])
        cnt += 1 if accept[q] else 0
    return q, cnt


def bits_of(data: np.ndarray, n_bits: int) -> list[int]:
    """MSB-first symbol sequence of a packed bitstream (reading A13)."""
    return [int((int(data[i >> 3]) >> (7 - (i & 7))) & 1) for i in range(n_bits)]


def run_splitmix(dfa, seed: int, length: int, start: int | None = None, offset: int = 0,
                 piece: int = 1 << 28) -> tuple[int, int]:
    """Stream bytes [offset, offset+length) of the counter-based generator through the loop,
    piece by piece (the generator regenerates the bytes the GPU side generated in place)."""
    from fsmgen import streams

    q = dfa.start if start is None else start
    cnt = 0
    cache = _arrays(dfa)
    buf = np.empty(min(piece, max(length, 1)), dtype=np.uint8)
    pos = 0
    while pos < length:
        n = min(piece, length - pos)
        streams.splitmix_bytes(seed, offset + pos, n, out=buf)
        q, c = run_from(dfa, q, buf[:n], n, _cache=cache)
        cnt += c
        pos += n
    return q, cnt


def certify(dfa, segments: list[tuple[int, int]], claimed_starts: list[int], fetch,
            threads: int | None = None) -> tuple[int, int]:
    """Certificate check.  ``segments`` = contiguous [lo, hi) byte ranges that
    tile [0, L); ``claimed_starts[i]`` = the state the GPU claims at ``segments[i][0]``;
    ``fetch(lo, hi)`` returns those input bytes.  Each segment runs the plain loop from its claimed
    start on its own core; the check passes only if segment 0 starts at q0 and every segment ends
    where the next one claims to start.  By induction the result equals the sequential oracle."""
    assert segments and segments[0][0] == 0
    if claimed_starts[0] != dfa.start:
        raise AssertionError("segment 0 does not start at q0")
    cache = _arrays(dfa)

    def one(i):
        lo, hi = segments[i]
        return run_from(dfa, claimed_starts[i], fetch(lo, hi), hi - lo, _cache=cache)

    with cf.ThreadPoolExecutor(max_workers=threads or os.cpu_count()) as ex:
        res = list(ex.map(one, range(len(segments))))
    total = 0
    for i, (end, c) in enumerate(res):
        total += c
        if i + 1 < len(segments) and end != claimed_starts[i + 1]:
            raise AssertionError(f"segment {i} ends in {end}, next claims {claimed_starts[i + 1]}")
    return res[-1][0], total
