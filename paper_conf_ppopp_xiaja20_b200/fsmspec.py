"""Thin ctypes binding of libfsmspec (include/fsmspec.h) -- argument marshalling only.

Every step of the spec-k path runs in the CUDA kernels behind the C ABI; there is no CPU
fallback: if libfsmspec.so is missing this module raises on import.  Torch is used only to
hand over device pointers and streams (``tensor.data_ptr()``, ``stream.cuda_stream``).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.environ.get("FSMSPEC_SO") or os.path.join(_HERE, "libfsmspec.so")  # override: experiments only

FSM_OK, FSM_EINVAL, FSM_ENOMEM, FSM_ECUDA, FSM_ESYMBOL, FSM_EUNSUPPORTED = 0, -1, -2, -3, -4, -5
FSM_INPUT_BYTES, FSM_INPUT_BITS_MSB = 0, 1
FSM_KMAX = 16
FSM_VARIANT_AUTO, FSM_VARIANT_P4, FSM_VARIANT_P8, FSM_VARIANT_B, FSM_VARIANT_G = -1, 0, 1, 2, 3
FSM_VARIANT_HS, FSM_VARIANT_CL, FSM_VARIANT_N8, FSM_VARIANT_R16, FSM_VARIANT_RG = 5, 6, 7, 8, 9
VARIANT_NAMES = {0: "P4", 1: "P8", 2: "B", 3: "G", 5: "HS", 6: "CL", 7: "N8", 8: "R16", 9: "RG"}
FSM_MERGE_PARALLEL, FSM_MERGE_SEQUENTIAL = 0, 1
FSM_EAGER_OFF = 1
FSM_PRERESOLVE_NONE = 0x80000000
FSM_CHECK_AUTO, FSM_CHECK_NESTED, FSM_CHECK_HASH = 0, 1, 2

# every symbol declared in include/fsmspec.h
EXPORTS = ("fsm_create", "fsm_create_ex", "fsm_destroy", "fsm_strerror", "fsm_set_stream",
           "fsm_run_spec_k", "fsm_run_spec_k_async", "fsm_run_spec_k_host", "fsm_set_options",
           "fsm_get_options", "fsm_get_stats", "fsm_run_shard", "fsm_shard_fixup", "fsm_shard_free",
           "fsm_map_compose", "fsm_compose_from", "fsm_lookback_table", "fsm_version", "fsm_autotune",
           "fsm_run_multi", "fsm_debug_set_spec", "fsm_debug_get_merge", "fsm_hot_state_order")


class fsm_options(ctypes.Structure):
    _fields_ = [("chunk_bytes", ctypes.c_uint32), ("threads_per_tile", ctypes.c_uint32),
                ("variant", ctypes.c_int32), ("merge", ctypes.c_uint32), ("ctas_per_sm", ctypes.c_uint32),
                ("lookback_len", ctypes.c_uint32), ("eager_window", ctypes.c_uint32), ("preresolve", ctypes.c_uint32),
                ("grid_sms", ctypes.c_uint32), ("check", ctypes.c_uint32), ("lookback_width", ctypes.c_uint32)]


class fsm_tuning(ctypes.Structure):
    _fields_ = [("k", ctypes.c_uint32), ("lookback_len", ctypes.c_uint32), ("eager_window", ctypes.c_uint32),
                ("candidates", ctypes.c_uint32), ("sample_len", ctypes.c_uint64), ("best_gbs", ctypes.c_double),
                ("paper_gbs", ctypes.c_double), ("hit_rate", ctypes.c_double), ("variant", ctypes.c_int32),
                ("preresolve", ctypes.c_uint32), ("lookback_width", ctypes.c_uint32), ("chunk_bytes", ctypes.c_uint32)]


class fsm_stats(ctypes.Structure):
    _fields_ = [("chunks", ctypes.c_uint64), ("tiles", ctypes.c_uint64), ("reexec_chunks", ctypes.c_uint64),
                ("reexec_symbols", ctypes.c_uint64), ("boundary_misses", ctypes.c_uint64),
                ("reexec_true", ctypes.c_uint64), ("reexec_true_symbols", ctypes.c_uint64),
                ("reexec_candidate", ctypes.c_uint64), ("reexec_candidate_symbols", ctypes.c_uint64),
                ("eager_resolved", ctypes.c_uint64), ("max_miss_chain", ctypes.c_uint64),
                ("chunk_bytes", ctypes.c_uint32), ("threads_per_tile", ctypes.c_uint32),
                ("variant", ctypes.c_uint32), ("k_slots", ctypes.c_uint32), ("lookback_len", ctypes.c_uint32),
                ("preresolve", ctypes.c_uint32), ("check", ctypes.c_uint32), ("lookback_width", ctypes.c_uint32)]


class fsm_shard_map(ctypes.Structure):
    _fields_ = [("k", ctypes.c_uint32), ("valid_mask", ctypes.c_uint32),
                ("start", ctypes.c_uint32 * FSM_KMAX), ("end", ctypes.c_uint32 * FSM_KMAX),
                ("count", ctypes.c_uint64 * FSM_KMAX)]

    def slots(self):
        return [(int(self.start[s]), int(self.end[s]), int(self.count[s]))
                for s in range(FSM_KMAX) if (self.valid_mask >> s) & 1]


_L6 = ctypes.c_uint32 * FSM_KMAX * 32 * 6


class fsm_debug_merge(ctypes.Structure):
    _fields_ = [("k", ctypes.c_uint32), ("start", _L6), ("end", _L6), ("count", _L6), ("brk", _L6),
                ("identity", ctypes.c_uint32 * 32 * 6)]

    def mapping(self, level: int, lane: int) -> dict:
        """Slot s -> (start, end, count) for valid slots, (start, None, brk) for invalid ones."""
        out = {}
        for s in range(self.k):
            st = int(self.start[level][lane][s])
            if st == 0xFFFFFFFF:
                continue
            b = int(self.brk[level][lane][s])
            out[st] = (int(self.end[level][lane][s]), int(self.count[level][lane][s])) if b == 0xFFFFFFFF else None
        return out


class FsmError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        self.status = status
        super().__init__(f"{what}: {lib().fsm_strerror(status).decode()} ({status})")


class SymbolError(FsmError):
    pass


_lib = None
_P = ctypes.c_void_p
_U32, _U64, _I32 = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32


def lib() -> ctypes.CDLL:
    """Load libfsmspec.so.  Raises if it has not been built -- there is no fallback path."""
    global _lib
    if _lib is None:
        if not os.path.exists(SO_PATH):
            raise ImportError(f"{SO_PATH} is not built; run `python -c 'import __graft_entry__ as g; g.build()'`")
        l = ctypes.CDLL(SO_PATH)
        sig = {
            "fsm_create": (_I32, [_P, _U32, _U32, _U32, _P, ctypes.POINTER(_P)]),
            "fsm_create_ex": (_I32, [_P, _U32, _U32, _U32, _P, _U32, ctypes.POINTER(_P)]),
            "fsm_destroy": (None, [_P]),
            "fsm_strerror": (ctypes.c_char_p, [_I32]),
            "fsm_set_stream": (_I32, [_P, _P]),
            "fsm_run_spec_k": (_I32, [_P, _P, _U64, _U32, ctypes.POINTER(_U32), ctypes.POINTER(_U64)]),
            "fsm_run_spec_k_async": (_I32, [_P, _P, _U64, _U32, _P]),
            "fsm_run_spec_k_host": (_I32, [_P, _P, _U64, _U32, ctypes.POINTER(_U32), ctypes.POINTER(_U64)]),
            "fsm_set_options": (_I32, [_P, ctypes.POINTER(fsm_options)]),
            "fsm_get_options": (_I32, [_P, ctypes.POINTER(fsm_options)]),
            "fsm_get_stats": (_I32, [_P, ctypes.POINTER(fsm_stats)]),
            "fsm_run_shard": (_I32, [_P, _P, _U64, _P, _U32, _U32, ctypes.POINTER(fsm_shard_map),
                                     ctypes.POINTER(_P)]),
            "fsm_shard_fixup": (_I32, [_P, _P, _U32, ctypes.POINTER(_U32), ctypes.POINTER(_U64)]),
            "fsm_shard_free": (None, [_P]),
            "fsm_map_compose": (_I32, [ctypes.POINTER(fsm_shard_map), ctypes.POINTER(fsm_shard_map),
                                       ctypes.POINTER(fsm_shard_map)]),
            "fsm_lookback_table": (_I32, [_P, _U32, _U32, _U32, _P, _P]),
            "fsm_version": (ctypes.c_char_p, []),
            "fsm_hot_state_order": (_I32, [_P, _U32, _U32, _U32, _P]),
            "fsm_compose_from": (_I32, [ctypes.POINTER(fsm_shard_map), _U32, _U32, _U64, ctypes.POINTER(_U32),
                                        ctypes.POINTER(_U64), ctypes.POINTER(_U32)]),
            "fsm_debug_set_spec": (_I32, [_P, _P, _U32, _U32, _U32]),
            "fsm_debug_get_merge": (_I32, [_P, ctypes.POINTER(fsm_debug_merge)]),
            "fsm_run_multi": (_I32, [ctypes.POINTER(_P), _U32, _P, _U64, ctypes.POINTER(_U32), ctypes.POINTER(_U32),
                                     ctypes.POINTER(_U64)]),
            "fsm_autotune": (_I32, [_P, _P, _U64, _U32, _U32, _U64, ctypes.POINTER(fsm_tuning)]),
        }
        for name, (res, args) in sig.items():
            fn = getattr(l, name)
            fn.restype = res
            fn.argtypes = args
        _lib = l
    return _lib


def _check(rc: int, what: str) -> None:
    if rc == FSM_ESYMBOL:
        raise SymbolError(rc, what)
    if rc != FSM_OK:
        raise FsmError(rc, what)


def _ptr(x) -> int:
    """Device or host address of a torch tensor / numpy array / int."""
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return int(x.data_ptr())


def lookback_table(table: np.ndarray, bit_mode: bool = False):
    """fsm_lookback_table (host only): (lb [256, 16] uint16, nimg [256] uint8)."""
    t = np.ascontiguousarray(table, dtype=np.uint32)
    lb = np.zeros((256, FSM_KMAX), np.uint16)
    ni = np.zeros(256, np.uint8)
    _check(lib().fsm_lookback_table(t.ctypes.data, t.shape[0], t.shape[1],
                                    FSM_INPUT_BITS_MSB if bit_mode else FSM_INPUT_BYTES,
                                    lb.ctypes.data, ni.ctypes.data), "fsm_lookback_table")
    return lb, ni


def hot_state_order(table: np.ndarray, bit_mode: bool = False) -> list[int]:
    """fsm_hot_state_order (host only): states by static in-degree, the hot-state caching order."""
    t = np.ascontiguousarray(table, dtype=np.uint32)
    out = np.zeros(t.shape[0], np.uint32)
    _check(lib().fsm_hot_state_order(t.ctypes.data, t.shape[0], t.shape[1],
                                     FSM_INPUT_BITS_MSB if bit_mode else FSM_INPUT_BYTES, out.ctypes.data),
           "fsm_hot_state_order")
    return [int(x) for x in out]


def map_compose(a: fsm_shard_map, b: fsm_shard_map) -> fsm_shard_map:
    out = fsm_shard_map()
    _check(lib().fsm_map_compose(ctypes.byref(a), ctypes.byref(b), ctypes.byref(out)), "fsm_map_compose")
    return out


def compose_from(maps, start_state: int, start_count: int = 0) -> tuple[int, int, int]:
    """fsm_compose_from (host only): follow start_state through the shard maps in order ->
    (state, count, first_miss) with first_miss == len(maps) when every map matched."""
    n = len(maps)
    arr = (fsm_shard_map * max(n, 1))(*maps)
    q, c, g = _U32(), _U64(), _U32()
    _check(lib().fsm_compose_from(arr, n, start_state, start_count, ctypes.byref(q), ctypes.byref(c), ctypes.byref(g)),
           "fsm_compose_from")
    return int(q.value), int(c.value), int(g.value)


class FSM:
    """One handle = one DFA on the current CUDA device (fsm_create_ex)."""

    def __init__(self, table, start: int, accept=None, bit_mode: bool = False):
        t = np.ascontiguousarray(table, dtype=np.uint32)
        self.n_states, self.alphabet = int(t.shape[0]), int(t.shape[1])
        self.bit_mode = bit_mode
        acc = None if accept is None else np.ascontiguousarray(accept, dtype=np.uint8)
        h = _P()
        _check(lib().fsm_create_ex(t.ctypes.data, self.n_states, self.alphabet, start,
                                   acc.ctypes.data if acc is not None else None,
                                   FSM_INPUT_BITS_MSB if bit_mode else FSM_INPUT_BYTES, ctypes.byref(h)),
               "fsm_create")
        self._h = h

    @classmethod
    def from_dfa(cls, dfa) -> "FSM":
        return cls(dfa.table, dfa.start, dfa.accept, dfa.bit_mode)

    def close(self) -> None:
        if getattr(self, "_h", None) and _lib is not None:
            _lib.fsm_destroy(self._h)
        self._h = None

    __del__ = close

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ---------------------------------------------------------------------------- configuration
    def set_stream(self, stream) -> None:
        s = 0 if stream is None else (stream if isinstance(stream, int) else stream.cuda_stream)
        _check(lib().fsm_set_stream(self._h, s), "fsm_set_stream")

    def set_options(self, chunk_bytes: int = 0, threads_per_tile: int = 0, variant: int = FSM_VARIANT_AUTO,
                    merge: int = FSM_MERGE_PARALLEL, ctas_per_sm: int = 0, lookback_len: int = 0,
                    eager_window: int = 0, preresolve: int = 0, grid_sms: int = 0, check: int = 0,
                    lookback_width: int = 0) -> None:
        o = fsm_options(chunk_bytes, threads_per_tile, variant, merge, ctas_per_sm, lookback_len, eager_window,
                        preresolve, grid_sms, check, lookback_width)
        _check(lib().fsm_set_options(self._h, ctypes.byref(o)), "fsm_set_options")

    def options(self) -> dict:
        o = fsm_options()
        _check(lib().fsm_get_options(self._h, ctypes.byref(o)), "fsm_get_options")
        return {n: getattr(o, n) for n, _ in o._fields_}

    def stats(self) -> dict:
        s = fsm_stats()
        _check(lib().fsm_get_stats(self._h, ctypes.byref(s)), "fsm_get_stats")
        return {n: int(getattr(s, n)) for n, _ in s._fields_}

    # ---------------------------------------------------------------------------------- runs
    def run_spec_k(self, inp, length: int, k: int) -> tuple[int, int]:
        """fsm_run_spec_k over a device-resident input (torch CUDA tensor or device address)."""
        q, n = _U32(), _U64()
        _check(lib().fsm_run_spec_k(self._h, _ptr(inp), length, k, ctypes.byref(q), ctypes.byref(n)),
               "fsm_run_spec_k")
        return int(q.value), int(n.value)

    def run_spec_k_async(self, inp, length: int, k: int, dev_result) -> None:
        """fsm_run_spec_k_async: enqueue only; the result lands in ``dev_result`` (16 device bytes)."""
        _check(lib().fsm_run_spec_k_async(self._h, _ptr(inp), length, k, _ptr(dev_result)),
               "fsm_run_spec_k_async")

    def run_spec_k_host(self, host_inp, length: int, k: int) -> tuple[int, int]:
        """fsm_run_spec_k_host: end-to-end over a host buffer (numpy array / pinned tensor)."""
        q, n = _U32(), _U64()
        _check(lib().fsm_run_spec_k_host(self._h, _ptr(host_inp), length, k, ctypes.byref(q), ctypes.byref(n)),
               "fsm_run_spec_k_host")
        return int(q.value), int(n.value)

    def autotune(self, inp, length: int, k_min: int = 0, k_max: int = 0, sample_len: int = 0) -> dict:
        """fsm_autotune (NEXT-2): choose k, look-back window and eager window by timing the kernel on
        a prefix sample; the chosen windows are applied to this handle, the chosen k is returned."""
        t = fsm_tuning()
        _check(lib().fsm_autotune(self._h, _ptr(inp), length, k_min, k_max, sample_len, ctypes.byref(t)), "fsm_autotune")
        return {n: (float(getattr(t, n)) if isinstance(getattr(t, n), float) else int(getattr(t, n)))
                for n, _ in t._fields_}

    def run_shard(self, inp, length: int, halo=None, halo_len: int = 0, k: int = 1, keep: bool = False):
        """fsm_run_shard -> (fsm_shard_map, shard handle or None)."""
        m = fsm_shard_map()
        st = _P()
        _check(lib().fsm_run_shard(self._h, _ptr(inp), length, _ptr(halo) if halo is not None else None,
                                   halo_len, k, ctypes.byref(m), ctypes.byref(st) if keep else None),
               "fsm_run_shard")
        return m, (Shard(st) if keep else None)

    # ------------------------------------------------------------------------- test-only hooks
    def debug_set_spec(self, sets, chunk_bytes: int, k: int = 0) -> None:
        """fsm_debug_set_spec: fixed chunk_bytes geometry; ``sets`` = per-chunk speculated state lists
        (None = look-back as usual; an entry None / missing = no state in that slot)."""
        if sets is None:
            _check(lib().fsm_debug_set_spec(self._h, None, 0, 0, chunk_bytes), "fsm_debug_set_spec")
            return
        k = k or max(len(x) for x in sets)
        a = np.full((len(sets), k), 0xFFFFFFFF, np.uint32)
        for j, x in enumerate(sets):
            for s, v in enumerate(x):
                if v is not None:
                    a[j, s] = v
        _check(lib().fsm_debug_set_spec(self._h, a.ctypes.data, len(sets), k, chunk_bytes), "fsm_debug_set_spec")

    def debug_get_merge(self) -> fsm_debug_merge:
        m = fsm_debug_merge()
        _check(lib().fsm_debug_get_merge(self._h, ctypes.byref(m)), "fsm_debug_get_merge")
        return m

    def shard_fixup(self, shard: "Shard", true_start: int) -> tuple[int, int]:
        q, n = _U32(), _U64()
        _check(lib().fsm_shard_fixup(self._h, shard._h, true_start, ctypes.byref(q), ctypes.byref(n)),
               "fsm_shard_fixup")
        return int(q.value), int(n.value)


class Shard:
    def __init__(self, h):
        self._h = h

    def close(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.fsm_shard_free(self._h)
        self._h = None

    __del__ = close


def run_multi(fsms, inp, length: int, ks) -> list[tuple[int, int]]:
    """fsm_run_multi (NEXT-4): every FSM of ``fsms`` over the same device-resident input, fused per
    (variant, K) group; returns [(final_state, accept_count)] in order."""
    m = len(fsms)
    hs = (_P * m)(*[f._h for f in fsms])
    kk = (_U32 * m)(*ks)
    q = (_U32 * m)()
    n = (_U64 * m)()
    _check(lib().fsm_run_multi(hs, m, _ptr(inp), length, kk, q, n), "fsm_run_multi")
    return [(int(q[i]), int(n[i])) for i in range(m)]
