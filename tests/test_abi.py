"""CPU-side checks of the C-ABI boundary: the library loads, exports every symbol that
include/fsmspec.h declares, and its host-only logic (look-back table, map composition) agrees
with independent definitions.  No compute call needs a GPU here."""
import ctypes
import os
import re

import numpy as np
import pytest

from fsmgen import dfas
from oracle import speck
from paper_conf_ppopp_xiaja20_b200 import fsmspec

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "fsmspec.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(fsm_[a-z_]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    syms = header_symbols()
    assert len(syms) >= 15
    lib = fsmspec.lib()
    for s in syms:
        assert hasattr(lib, s), s
    assert sorted(fsmspec.EXPORTS) == syms


def test_strerror_and_version():
    lib = fsmspec.lib()
    assert lib.fsm_strerror(0) == b"ok"
    assert b"alphabet" in lib.fsm_strerror(fsmspec.FSM_ESYMBOL)
    assert b"sm_100a" in lib.fsm_version()


def test_lookback_fig2(golden):
    # after x only a and c are possible; the paper picks a (reading A5: ties -> smaller id)
    d = dfas.c_comment(expanded=False)
    lb, ni = fsmspec.lookback_table(d.table)
    assert ni[2] == 2 and list(lb[2, :2]) == [0, 2]
    assert lb[2, 2] == 0xFFFF


@pytest.mark.parametrize("seed", range(8))
def test_lookback_matches_model(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 40))
    a = int(rng.integers(1, 257))
    t = rng.integers(0, n, (n, a)).astype(np.uint32)
    lb, ni = fsmspec.lookback_table(t)
    for c in range(256):
        if c < a:
            exp = speck.lookback(t, c, 16)
        else:
            exp = [n]  # bytes outside the alphabet lead to the sink (internal id n, reading A14)
        assert list(lb[c, :ni[c]]) == exp
        assert ni[c] == len(exp)


def test_lookback_bit_mode_widened():
    d = dfas.div7()
    lb, ni = fsmspec.lookback_table(d.table, bit_mode=True)
    # widened byte step of Div7 is a permutation: image = all 7 states, equal preimage counts
    assert all(ni == 7) and all(list(lb[c, :7]) == list(range(7)) for c in range(256))


def test_invalid_arguments_rejected_on_host():
    lib = fsmspec.lib()
    t = np.zeros((2, 2), np.uint32)
    h = ctypes.c_void_p()
    assert lib.fsm_create(t.ctypes.data, 0, 2, 0, None, ctypes.byref(h)) == fsmspec.FSM_EINVAL
    assert lib.fsm_create(t.ctypes.data, 2, 2, 5, None, ctypes.byref(h)) == fsmspec.FSM_EINVAL
    bad = np.array([[0, 7], [1, 1]], np.uint32)
    assert lib.fsm_create(bad.ctypes.data, 2, 2, 0, None, ctypes.byref(h)) == fsmspec.FSM_EINVAL
    assert lib.fsm_create_ex(np.zeros((2, 3), np.uint32).ctypes.data, 2, 3, 0, None, 1,
                             ctypes.byref(h)) == fsmspec.FSM_EINVAL
    assert lib.fsm_lookback_table(t.ctypes.data, 2, 300, 0, None, None) == fsmspec.FSM_EINVAL


def _m(starts, ends, counts, k=None):
    m = fsmspec.fsm_shard_map()
    m.k = k or len(starts)
    for i, (s, e, c) in enumerate(zip(starts, ends, counts)):
        if s is None:
            continue
        m.valid_mask |= 1 << i
        m.start[i], m.end[i], m.count[i] = s, e, c
    return m


def test_map_compose_matches_merge_semantics(golden):
    # Fig. 4 chunks 0 and 1 as shard maps: a->c, c->d then c->c, d->c  =>  a->c, c->c
    a = _m([0, 2], [2, 3], [0, 0])
    b = _m([2, 3], [2, 2], [0, 0])
    r = fsmspec.map_compose(a, b)
    assert r.slots() == [(0, 2, 0), (2, 2, 0)]
    # chunks 2 and 3: a->a(2) has no match in {c, d} -> invalid
    c = _m([0, 2], [0, 3], [2, 0])
    d = _m([2, 3], [0, 0], [1, 1])
    r2 = fsmspec.map_compose(c, d)
    assert r2.slots() == [(2, 0, 1)]
    root = fsmspec.map_compose(r, r2)
    assert root.slots() == [(0, 0, 1), (2, 0, 1)]


@pytest.mark.parametrize("seed", range(20))
def test_map_compose_vs_model_random(seed):
    rng = np.random.default_rng(seed)
    n, k = 8, 4
    maps = []
    for _ in range(3):
        st = [int(x) for x in rng.choice(n, k, replace=False)]
        en = [int(x) for x in rng.integers(0, n, k)]
        cn = [int(x) for x in rng.integers(0, 9, k)]
        maps.append((st, en, cn))
    x = _m(*maps[0])
    y = _m(*maps[1])
    z = _m(*maps[2])
    left = fsmspec.map_compose(fsmspec.map_compose(x, y), z)
    right = fsmspec.map_compose(x, fsmspec.map_compose(y, z))
    assert left.slots() == right.slots()
    ma = speck.Mapping(*maps[0])
    mb = speck.Mapping(*maps[1])
    mm = speck.merge(ma, mb)
    exp = [(s, e, c) for s, e, c in zip(mm.starts, mm.ends, mm.counts) if e is not None]
    assert fsmspec.map_compose(x, y).slots() == exp


def test_variant_enum_matches_header():
    """The binding's variant ids and names are the header's FSM_VARIANT_* enum (one table variant
    per id; RG = 9 is the newest)."""
    txt = open(os.path.join(ROOT, "include", "fsmspec.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    enum = {m.group(1): int(m.group(2)) for m in re.finditer(r"FSM_VARIANT_([A-Z0-9]+)\s*=\s*(-?\d+)", txt)}
    assert enum.pop("AUTO") == fsmspec.FSM_VARIANT_AUTO == -1
    assert {v: k for k, v in enum.items()} == fsmspec.VARIANT_NAMES
    for name, v in enum.items():
        assert getattr(fsmspec, "FSM_VARIANT_" + name) == v


def test_hot_state_order_p5(golden):
    """P5: the static frequency of Fig. 1b is a = c = 4, b = d = 2, so with 6 shared-
    memory entries (two rows of three symbols) the rows of a and c are cached.  The library's own
    hot-state caching order (the HS variant's renumbering) must put a and c first, for the
    3-symbol table and for the 256-column expansion alike."""
    g = golden["c_comment_fig1"]
    names = g["states"]
    for expanded in (False, True):
        d = dfas.c_comment(expanded=expanded)
        order = fsmspec.hot_state_order(d.table)
        rows = 6 // 3                                                       # 6 entries
        assert {names[s] for s in order[:rows]} == set(g["hot_rows_6_entries"]["rows"]), expanded
        assert sorted(order) == list(range(4))
    # in-degree ranking against an independent count on random tables (ties -> smaller id)
    rng = np.random.default_rng(5)
    for _ in range(5):
        t = rng.integers(0, 12, (12, 256)).astype(np.uint32)
        indeg = np.bincount(t.ravel(), minlength=12)
        exp = sorted(range(12), key=lambda s: (-indeg[s], s))
        assert fsmspec.hot_state_order(t) == exp
