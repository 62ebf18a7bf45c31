"""TEST INFRASTRUCTURE ONLY -- the sequential oracle (Fig. 1c).

run(dfa, data, length)          -> (final_state, accept_count)   C loop, any size
run_py(table, start, F, syms)   -> same, pure Python (tiny cases; pins the C loop)
run_from(...)                   -> from an arbitrary start state (used for shard maps / certificates)
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


class CertificateError(AssertionError):
    """The GPU-claimed segment start states are not the oracle's."""


def certify(dfa, bounds: list[int], claimed_starts: list[int], fetch, piece: int = 1 << 28,
            threads: int | None = None) -> tuple[int, int]:
    """Certificate check of a long byte-mode run.  ``bounds`` = b_0 = 0 < b_1 <
    ... < b_G = L cut the input into G contiguous segments; ``claimed_starts[g]`` = the state a
    GPU run claims at b_g; ``fetch(lo, hi)`` returns input bytes [lo, hi) (called piece by piece,
    so inputs far larger than host memory stream through).  Every segment runs the plain loop
    (``run_from``) from its claimed start, on its own thread; the check passes only if segment 0
    starts in q0 and every segment ends where the next one claims to start -- then, by induction
    over the segments, the concatenation is the sequential run of Fig. 1c over the whole input and
    the returned (final state, summed count) is the oracle's result.  Raises CertificateError."""
    assert not dfa.bit_mode and len(bounds) == len(claimed_starts) + 1 and bounds[0] == 0
    if claimed_starts[0] != dfa.start:
        raise CertificateError(f"segment 0 claims {claimed_starts[0]}, q0 = {dfa.start}")
    cache = _arrays(dfa)

    def one(g):
        q, total = claimed_starts[g], 0
        for o in range(bounds[g], bounds[g + 1], piece):
            hi = min(o + piece, bounds[g + 1])
            q, c = run_from(dfa, q, fetch(o, hi), hi - o, _cache=cache)
            total += c
        return q, total

    with cf.ThreadPoolExecutor(max_workers=threads or min(len(claimed_starts), os.cpu_count() or 1)) as ex:
        res = list(ex.map(one, range(len(claimed_starts))))
    for g in range(len(res) - 1):
        if res[g][0] != claimed_starts[g + 1]:
            raise CertificateError(f"segment {g} ends in {res[g][0]}, segment {g + 1} claims {claimed_starts[g + 1]}")
    return res[-1][0], sum(c for _, c in res)
