"""The paper's worked examples replayed on the CUDA merge, through the
test-only hook fsm_debug_set_spec (fixed tiny chunks, injected speculated sets) and the merge-tree
readback fsm_debug_get_merge, plus the per-run re-execution counters.

* Fig. 2: chunks `/*xx` | `x**/`, spec-1; look-back on `x` guesses a, chunk 1 ends in b,
  the check fails, chunk 1 is re-executed from c; final a; 1 re-execution.
* Fig. 4: four chunks of two bytes, spec-2 with the figure's sets injected;
  merged chunks 0+1 = {a->c, c->c}; merged 2+3 = {c->a, a invalid}; root = {a->a, c->a}; the
  delayed strategy re-executes nothing, nor does the sequential merge (Fig. 4a).
Expected values come from tests/golden/c_comment_fig2_fig4.json (the paper's narrative)."""
import numpy as np
import pytest

from fsmgen import dfas, streams
from oracle import seq, speck

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_ppopp_xiaja20_b200 import fsmspec  # noqa: E402
from paper_conf_ppopp_xiaja20_b200.fsmspec import FSM  # noqa: E402

ST = {"a": 0, "b": 1, "c": 2, "d": 3}
NAME = {v: k for k, v in ST.items()}
VARIANTS = {"P4": 0, "P8": 1, "B": 2, "G": 3, "HS": 5, "CL": 6, "N8": 7, "R16": 8, "RG": 9}


def dev(data: np.ndarray):
    buf = torch.zeros(data.size + 64, dtype=torch.uint8, device="cuda")
    buf[:data.size] = torch.from_numpy(np.ascontiguousarray(data))
    return buf, buf.data_ptr()


def named(m, level, lane):
    """Level/lane mapping of the readback in the golden file's notation."""
    return {NAME[s]: (None if v is None else [NAME[v[0]], v[1]]) for s, v in m.mapping(level, lane).items()}


@pytest.mark.parametrize("var", list(VARIANTS))
def test_fig2_speculation_and_reexecution(golden, var):
    g = golden["c_comment_fig2_fig4"]["P2"]
    d = dfas.c_comment(True)
    data = np.frombuffer("".join(g["chunks"]).encode(), np.uint8)
    with FSM.from_dfa(d) as f:
        f.set_options(variant=VARIANTS[var], eager_window=fsmspec.FSM_EAGER_OFF)
        f.debug_set_spec(None, chunk_bytes=len(g["chunks"][0]))
        buf, ptr = dev(data)
        got = f.run_spec_k(ptr, data.size, 1)
        st = f.stats()
        m = f.debug_get_merge()
    assert got == (ST[g["final"]], 1) == seq.run(d, data)
    assert named(m, 0, 0) == {"a": ["c", 0]}                     # chunk 0 from the known start a
    assert named(m, 0, 1) == {g["guess_chunk1"]: ["b", 3]}       # look-back on x guesses a; ends in b
    assert named(m, 1, 0) == {"a": None}                         # c is not a speculated start: invalid
    assert m.brk[1][0][0] == 1 and m.end[1][0][0] == ST["c"]     # ... when entering chunk 1 in state c
    assert st["reexec_true"] == g["reexec"] and st["reexec_candidate"] == 0
    assert st["reexec_true_symbols"] == 4 and st["max_miss_chain"] == 1


@pytest.mark.parametrize("var", list(VARIANTS))
def test_fig4_merge_tree(golden, var):
    g = golden["c_comment_fig2_fig4"]["P3"]
    d = dfas.c_comment(True)
    data = np.frombuffer("".join(g["chunks"]).encode(), np.uint8)
    sets = [[ST[s] for s in ss] for ss in g["injected_sets"]]
    with FSM.from_dfa(d) as f:
        f.set_options(variant=VARIANTS[var])
        f.debug_set_spec(sets, chunk_bytes=2)
        buf, ptr = dev(data)
        got = f.run_spec_k(ptr, data.size, 2)
        st = f.stats()
        m = f.debug_get_merge()
    assert got == (ST["a"], 1) == seq.run(d, data)
    # level 0: the chunk mappings of Fig. 4, counts with F = {a}
    assert named(m, 0, 0) == {"a": ["c", 0], "c": ["d", 0]}
    assert named(m, 0, 1) == {"c": ["c", 0], "d": ["c", 0]}
    assert named(m, 0, 2) == {"a": ["a", 2], "c": ["d", 0]}
    assert named(m, 0, 3) == {"c": ["a", 1], "d": ["a", 1]}
    # level 1 = the pairwise merges, level 2 = the root (Fig. 4b)
    assert named(m, 1, 0) == g["merged_01"]
    assert named(m, 1, 2) == g["merged_23"]
    a_slot = sets[2].index(ST["a"])
    assert m.brk[1][2][a_slot] == 3 and m.end[1][2][a_slot] == ST["a"]  # invalid entering chunk 3 in a
    assert named(m, 2, 0) == g["root"]
    assert all(m.identity[0][lane] for lane in range(4, 32)) and not any(m.identity[0][:4])
    # P4: the delayed strategy re-executes nothing
    assert st["reexec_chunks"] == golden["c_comment_fig2_fig4"]["P4"]["reexec_delayed"] == 0
    assert st["boundary_misses"] == 0


def test_fig4_sequential_merge_reexecutes_nothing(golden):
    g = golden["c_comment_fig2_fig4"]
    d = dfas.c_comment(True)
    data = np.frombuffer("".join(g["P3"]["chunks"]).encode(), np.uint8)
    sets = [[ST[s] for s in ss] for ss in g["P3"]["injected_sets"]]
    with FSM.from_dfa(d) as f:
        f.set_options(merge=fsmspec.FSM_MERGE_SEQUENTIAL)
        f.debug_set_spec(sets, chunk_bytes=2)
        buf, ptr = dev(data)
        assert f.run_spec_k(ptr, data.size, 2) == (ST["a"], 1)
        assert f.stats()["reexec_chunks"] == g["P4"]["reexec_sequential"]


def test_injected_chunk0_without_true_start_is_resolved():
    """Chunk 0's injected set does not contain q0 = a: the true path misses at chunk 0 and is
    re-executed (a tile-boundary miss of tile 0), the result is still exact."""
    d = dfas.c_comment(True)
    data = np.frombuffer(b"/*xxx**/", np.uint8)
    with FSM.from_dfa(d) as f:
        f.debug_set_spec([[ST["c"], ST["d"]], [ST["c"], ST["d"]], [ST["a"], ST["c"]], [ST["c"], ST["d"]]], chunk_bytes=2)
        buf, ptr = dev(data)
        assert f.run_spec_k(ptr, data.size, 2) == (ST["a"], 1)
        st = f.stats()
    assert st["boundary_misses"] == 1 and st["reexec_true"] >= 1


def test_debug_hook_validates():
    d = dfas.c_comment(True)
    with FSM.from_dfa(d) as f:
        with pytest.raises(fsmspec.FsmError):
            f.debug_set_spec([[0, 0]], chunk_bytes=2)        # duplicated slot (reading A6)
        with pytest.raises(fsmspec.FsmError):
            f.debug_set_spec([[7]], chunk_bytes=2)           # not a state
        f.debug_set_spec([[0], [0]], chunk_bytes=4)
        buf, ptr = dev(np.frombuffer(b"/*xxx**/x", np.uint8))
        with pytest.raises(fsmspec.FsmError):
            f.run_spec_k(ptr, 9, 1)                         # 3 chunks, 2 injected
        f.debug_set_spec(None, 0)                           # cleared: normal geometry again
        assert f.run_spec_k(ptr, 9, 1) == seq.run(d, np.frombuffer(b"/*xxx**/x", np.uint8))


# --------------------------------------------------------------------- per-run counters (a8)
def _true_path_misses(d, data, chunk, k):
    """#chunks whose true start is not in their depth-1 look-back set (A5), chunk 0 = {q0}: what
    the delayed strategy must re-execute, from the oracle loop per chunk."""
    x, miss = d.start, 0
    for j, b in enumerate(range(0, data.size, chunk)):
        if j and x not in speck.lookback(d.table, int(data[b - 1]), k):
            miss += 1
        x = seq.run_from(d, x, data[b:b + chunk])[0]
    return miss


@pytest.mark.parametrize("n,m,k,pre", [(8, 3, 1, 0), (8, 4, 2, 0), (8, 4, 2, fsmspec.FSM_PRERESOLVE_NONE),
                                       (16, 5, 3, 1), (16, 5, 3, 0), (64, 6, 4, 2)])
def test_reexec_true_equals_model_miss_count(n, m, k, pre):
    d = dfas.random_dfa(n, m, seed=300 + n + m)
    data = streams.splitmix_bytes(41 + n, 0, 1 << 20)
    chunk = 256
    with FSM.from_dfa(d) as f:
        f.set_options(chunk_bytes=chunk, eager_window=fsmspec.FSM_EAGER_OFF, preresolve=pre)
        buf, ptr = dev(data)
        assert f.run_spec_k(ptr, data.size, k) == seq.run(d, data)
        st = f.stats()
    assert st["reexec_true"] == _true_path_misses(d, data, chunk, k), st
    assert st["reexec_chunks"] == st["reexec_true"] + st["reexec_candidate"]
    if pre == fsmspec.FSM_PRERESOLVE_NONE:
        assert st["reexec_candidate"] == 0      # only the true path is ever re-executed


def test_stats_are_per_run():
    """Counters describe the most recent call: three async runs on other inputs, then a sync run,
    give the same counters as a fresh handle's single sync run (no leak across runs)."""
    d = dfas.random_dfa(8, 4, seed=77)
    data = streams.splitmix_bytes(77, 0, 3 << 20)
    other = streams.splitmix_bytes(78, 0, 5 << 20)
    with FSM.from_dfa(d) as f:
        f.set_options(eager_window=fsmspec.FSM_EAGER_OFF)
        buf, ptr = dev(data)
        f.run_spec_k(ptr, data.size, 2)
        fresh = f.stats()
    assert fresh["reexec_chunks"] > 0
    with FSM.from_dfa(d) as f:
        f.set_options(eager_window=fsmspec.FSM_EAGER_OFF)
        buf, ptr = dev(data)
        obuf, optr = dev(other)
        res = torch.zeros(4, dtype=torch.int32, device="cuda")
        for _ in range(3):
            f.run_spec_k_async(optr, other.size, 2, res.data_ptr())
        f.run_spec_k(ptr, data.size, 2)
        assert f.stats() == fresh
        # an async run's own counters are readable too
        f.run_spec_k_async(optr, other.size, 2, res.data_ptr())
        a1 = f.stats()
        f.run_spec_k_async(optr, other.size, 2, res.data_ptr())
        assert f.stats() == a1


def test_unaligned_input_peels_one_sector():
    """An unaligned pointer runs from the aligned address below it (chunk 0 = [head, chunk)); the
    result and the re-execution counters do not depend on the offset beyond chunk 0."""
    d = dfas.random_dfa(8, 2, seed=5)
    data = streams.splitmix_bytes(5, 0, (8 << 20) + 77)
    exp = seq.run(d, data)
    for off in (0, 1, 7, 31):
        buf = torch.zeros(data.size + 128, dtype=torch.uint8, device="cuda")
        buf[off:off + data.size] = torch.from_numpy(data)
        with FSM.from_dfa(d) as f:
            for lb in (0, 64):
                f.set_options(lookback_len=lb)
                for k in (1, 2):
                    assert f.run_spec_k(buf.data_ptr() + off, data.size, k) == exp, (off, lb, k)


# --------------------------------------------------------------------- Alg. 2 (hash check) on the GPU
@pytest.mark.parametrize("n,m", [(16, 12), (40, 16), (255, 14)])
@pytest.mark.parametrize("k", [12, 13, 16])
def test_hash_check_matches_nested(n, m, k):
    """Alg. 2 and Alg. 1 give identical results and identical re-execution
    counts for every variant that has the hash form; the run reports which check it used."""
    if k > n:
        pytest.skip("k <= N")
    d = dfas.random_dfa(n, m, seed=500 + n + m)
    data = streams.splitmix_bytes(600 + n, 0, (3 << 20) + 11)
    exp = seq.run(d, data)
    for var in ("B", "G", "R16", "CL", "HS"):
        if var == "R16" and n > 16:  # (byte mode here)
            continue
        with FSM.from_dfa(d) as f:
            buf, ptr = dev(data)
            stats = {}
            for chk in (fsmspec.FSM_CHECK_NESTED, fsmspec.FSM_CHECK_HASH):
                try:
                    f.set_options(variant=VARIANTS[var], check=chk, chunk_bytes=512,
                                  eager_window=fsmspec.FSM_EAGER_OFF)
                except fsmspec.FsmError:
                    break  # the DFA does not fit this variant
                assert f.run_spec_k(ptr, data.size, k) == exp, (var, chk)
                stats[chk] = f.stats()
            if len(stats) == 2:
                a, b = stats[fsmspec.FSM_CHECK_NESTED], stats[fsmspec.FSM_CHECK_HASH]
                assert a["check"] == fsmspec.FSM_CHECK_NESTED
                if b["check"] == fsmspec.FSM_CHECK_HASH:
                    # the chunk-level true-path miss count does not depend on the tile geometry
                    assert a["reexec_true"] == b["reexec_true"], (var, a, b)


def test_hash_check_merge_tree_identical():
    """With injected 12-slot sets on tiny chunks, every level of the warp merge tree read back
    from the GPU is the same under Alg. 1 and Alg. 2 (including invalid slots and where they broke)."""
    d = dfas.random_dfa(16, 14, seed=9)
    rng = np.random.default_rng(4)
    data = rng.integers(0, 256, 64).astype(np.uint8)
    sets = [list(rng.choice(16, 12, replace=False)) for _ in range(32)]
    out = {}
    for chk in (fsmspec.FSM_CHECK_NESTED, fsmspec.FSM_CHECK_HASH):
        with FSM.from_dfa(d) as f:
            f.set_options(variant=VARIANTS["G"], check=chk)
            f.debug_set_spec(sets, chunk_bytes=2)
            buf, ptr = dev(data)
            assert f.run_spec_k(ptr, data.size, 12) == seq.run(d, data)
            assert f.stats()["check"] == chk
            m = f.debug_get_merge()
            out[chk] = [[m.mapping(lv, lane) for lane in range(32)] for lv in range(6)]
            out[chk].append([[int(m.brk[lv][lane][s]) for s in range(16)] for lv in range(6) for lane in range(32)])
    assert out[fsmspec.FSM_CHECK_NESTED] == out[fsmspec.FSM_CHECK_HASH]


# --------------------------------------------------------------------- randomised merge trees vs the CPU model
@pytest.mark.parametrize("seed", range(4))
def test_random_injected_merge_trees(seed):
    """Tiny random DFAs (N <= 4, 2 symbols), random inputs of up to 32 chunks of 1-4 bytes and random
    injected speculated sets (chunk 0's may miss q0): every warp-scan level read back from the GPU
    equals the CPU model's merge (oracle/speck.py, Sec. 3.3) of the same chunks, slot by
    slot and validity included, and the result equals the oracle.  ~400 cases per seed."""
    rng = np.random.default_rng(1000 + seed)
    cases = 0
    while cases < 400:
        n = int(rng.integers(2, 5))
        table = rng.integers(0, n, (n, 2)).astype(np.uint32)
        acc = rng.integers(0, 2, n).astype(np.uint8)
        d = dfas.DFA(table, int(rng.integers(0, n)), acc, False, "tiny")
        c = int(rng.integers(1, 5))
        nch = int(rng.integers(1, 33))
        L = c * (nch - 1) + int(rng.integers(1, c + 1))
        data = rng.integers(0, 2, L).astype(np.uint8)
        k = int(rng.integers(1, n + 1))
        sets = [list(rng.choice(n, int(rng.integers(1, k + 1)), replace=False)) for _ in range(nch)]
        with FSM.from_dfa(d) as f:
            f.set_options(eager_window=fsmspec.FSM_EAGER_OFF)
            f.debug_set_spec([[int(x) for x in s_] for s_ in sets], chunk_bytes=c, k=k)
            buf, ptr = dev(data)
            got = f.run_spec_k(ptr, L, k)
            m = f.debug_get_merge()
        assert got == seq.run(d, data), (seed, cases)
        bounds = [min(j * c, L) for j in range(nch)] + [L]
        maps = speck.local_phase(d, [int(x) for x in data], bounds, sets)
        level = list(maps)
        for lv in range(6):
            for j in range(nch):
                exp = {s: (None if e is None else (e, cnt)) for s, e, cnt in zip(level[j].starts, level[j].ends,
                                                                                   level[j].counts)}
                assert m.mapping(lv, j) == exp, (seed, cases, lv, j)
            step = 1 << lv
            level = [speck.merge(level[j], level[j + step]) if j + step < nch else level[j] for j in range(nch)]
        cases += 1


@pytest.mark.parametrize("k", [1, 2, 3, 5, 7])
def test_div7_reexecution_rate_is_one_minus_k_over_7(k):
    """Div7 on random bits: the widened-byte look-back image is all 7 states with equal
    weight, so a chunk's true start is speculated with probability k/7 and the GPU's true-path
    re-execution rate must approach 1 - k/7; k = 7 (spec-N) never re-executes."""
    d = dfas.div7()
    n_bits = 8 * (32 << 20)
    data = streams.random_bits(n_bits, seed=70 + k)
    with FSM.from_dfa(d) as f:
        f.set_options(eager_window=fsmspec.FSM_EAGER_OFF, chunk_bytes=1024, variant=VARIANTS["P8"])
        buf, ptr = dev(data)
        assert f.run_spec_k(ptr, n_bits, k) == seq.run(d, data, n_bits)
        st = f.stats()
    rate = st["reexec_true"] / (st["chunks"] - 1)
    assert abs(rate - (1 - k / 7)) < 0.01, (k, rate, st)
