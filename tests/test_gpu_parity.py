"""GPU parity: the CUDA path (through the C ABI) against the sequential oracle, bit-exact in the
final state and the accept count, on seeded synthetic DFAs and inputs that span
several tiles and a ragged tail, every table variant, every instantiated k, both merges, the
async / host-buffer / shard entry points, and the edge cases (empty input, unaligned pointers,
bit-mode tails, out-of-alphabet bytes, k = N, k > |image|)."""
import numpy as np
import pytest

from fsmgen import dfas, streams
from oracle import seq, speck

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_ppopp_xiaja20_b200 import fsmspec  # noqa: E402
from paper_conf_ppopp_xiaja20_b200.fsmspec import FSM  # noqa: E402


def dev(data: np.ndarray, offset: int = 0):
    buf = torch.zeros(data.size + offset + 64, dtype=torch.uint8, device="cuda")
    buf[offset:offset + data.size] = torch.from_numpy(np.ascontiguousarray(data))
    return buf, buf.data_ptr() + offset


def gpu_run(dfa, data, length=None, k=1, offset=0, **opt):
    if length is None:
        length = data.size * 8 if dfa.bit_mode else data.size
    with FSM.from_dfa(dfa) as f:
        if opt:
            f.set_options(**opt)
        buf, ptr = dev(data, offset)
        res = f.run_spec_k(ptr, length, k)
        st = f.stats()
        torch.cuda.synchronize()
    return res, st


VARIANTS = {"P4": 0, "P8": 1, "B": 2, "G": 3, "HS": 5, "CL": 6, "N8": 7, "R16": 8, "RG": 9}


def dfa_bits(dfa):
    return bool(dfa.bit_mode)


def fits(dfa, var):
    n = dfa.n_states + (1 if (not dfa.bit_mode and dfa.alphabet < 256) else 0)
    # R16 and CL use region counting (accept-partitioned ids): byte mode only
    return {"P4": n <= 4 and not dfa.bit_mode, "P8": n <= 8,
            "N8": n <= 8 and not dfa.bit_mode, "R16": n <= 16 and not dfa.bit_mode,
            "RG": n <= 256 and not dfa.bit_mode,
            "B": n <= 256, "G": True, "HS": not dfa.bit_mode and n <= 32768,
            "CL": not dfa.bit_mode and _n_classes(dfa) >= 2
            and n * ((_n_classes(dfa) + 1) // 2) * 128 <= 0x10000 - 1024}[var]


def _n_classes(dfa):
    """Distinct byte columns of the byte-level (widened in bit mode) table, as the library counts them."""
    t = dfa.table
    if dfa.bit_mode:
        n = t.shape[0]
        nx = np.zeros((n, 256), np.int64)
        cnt = np.zeros((n, 256), np.int64)
        for s in range(n):
            for c in range(256):
                q, k = s, 0
                for i in range(7, -1, -1):
                    q = int(t[q, (c >> i) & 1])
                    k += int(dfa.accept[q])
                nx[s, c], cnt[s, c] = q, k
        cols = {tuple(nx[:, c]) + tuple(cnt[:, c]) for c in range(256)}
    else:
        full = np.full((t.shape[0] + (1 if t.shape[1] < 256 else 0), 256), t.shape[0], np.int64)
        full[:t.shape[0], :t.shape[1]] = t
        acc = np.concatenate([dfa.accept, [0] * (full.shape[0] - t.shape[0])]).astype(np.int64)
        cols = {tuple(full[:, c]) + tuple(acc[full[:, c]]) for c in range(256)}
    return len(cols)


# --------------------------------------------------------------------- worked example on GPU
@pytest.mark.parametrize("var", ["P4", "P8", "N8", "R16", "B", "G", "HS", "CL"])
@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_fig1_worked_example(var, k):
    d = dfas.c_comment(True)
    data = np.frombuffer(b"/*xxx**/", np.uint8)
    (q, n), _ = gpu_run(d, data, k=k, variant=VARIANTS[var])
    assert (q, n) == (0, 1) == seq.run(d, data)


# --------------------------------------------------------------------- C1-shaped text
@pytest.mark.parametrize("var", ["P4", "P8", "N8", "R16", "B", "G", "HS", "CL"])
@pytest.mark.parametrize("chunk", [0, 64, 96, 4096, 16384])
def test_c_comment_text(var, chunk):
    d = dfas.c_comment(True)
    data = streams.c_source(300_001, seed=streams.MASTER_SEED + 1, comment_frac=0.3)
    exp = seq.run(d, data)
    for k in (1, 2, 4):
        got, st = gpu_run(d, data, k=k, variant=VARIANTS[var], chunk_bytes=chunk)
        assert got == exp, (var, chunk, k, st)


# --------------------------------------------------------------------- random DFAs, all variants, all k
CASES = [(2, 2), (4, 2), (4, 4), (7, 3), (8, 1), (8, 2), (8, 8), (16, 2), (16, 5), (20, 2), (32, 3), (64, 4),
         (100, 4), (255, 8),
         (1000, 3), (4096, 8)]


@pytest.mark.parametrize("n,m", CASES)
def test_random_dfa_parity(n, m):
    d = dfas.random_dfa(n, m, seed=1000 + n * 17 + m)
    length = 1_000_003
    data = streams.splitmix_bytes(5 + n, 0, length)
    exp = seq.run(d, data)
    for var in VARIANTS:
        if not fits(d, var):
            continue
        for k in sorted({1, 2, 3, min(m, 16), min(n, 16), 5, 16} & set(range(1, min(n, 16) + 1))):
            for chunk in (64, 1024, 8192 if dfa_bits(d) else 16384):
                got, st = gpu_run(d, data, k=k, variant=VARIANTS[var], chunk_bytes=chunk)
                assert got == exp, (n, m, var, k, chunk, st)
                if k >= m:
                    assert st["reexec_chunks"] == 0, st  # k >= |image| never re-executes


@pytest.mark.parametrize("length", [0, 1, 2, 31, 32, 33, 63, 64, 65, 4095, 4096, 4097, 65536 * 3 + 7])
@pytest.mark.parametrize("offset", [0, 1, 13, 32])
def test_lengths_and_alignment(length, offset):
    d = dfas.random_dfa(8, 3, seed=42)
    data = streams.splitmix_bytes(77, 0, max(length, 1))[:length]
    exp = seq.run(d, data, length)
    for k in (1, 2, 3):
        got, _ = gpu_run(d, data, length, k=k, offset=offset, chunk_bytes=64)
        assert got == exp, (length, offset, k)


@pytest.mark.parametrize("length", [1 << 20, (64 << 20) + 5, 300 << 20])
def test_default_geometry_power_of_two_chunks(length):
    """pick_geometry's wave model: default chunks are powers of two up to 16 KiB (4 KiB for G),
    results exact at every size."""
    d = dfas.random_dfa(16, 2, seed=77)
    data = streams.splitmix_bytes(78, 0, length)
    exp = seq.run(d, data)
    for var, k, cap in (("R16", 2, 16384), ("G", 1, 4096)):
        got, st = gpu_run(d, data, k=k, variant=VARIANTS[var])
        assert got == exp, (var, length, st)
        c = st["chunk_bytes"]
        assert 64 <= c <= cap and c & (c - 1) == 0, st


def test_chunk_limits():
    """fsm_set_options: chunks up to 16 KiB in byte mode, 8 KiB in bit mode (32-bit tile-window counts)."""
    with FSM.from_dfa(dfas.random_dfa(8, 2, seed=1)) as f:
        f.set_options(chunk_bytes=16384)
        for bad in (16416, 32768, 100):
            with pytest.raises(fsmspec.FsmError):
                f.set_options(chunk_bytes=bad)
    with FSM.from_dfa(dfas.div7()) as f:
        f.set_options(chunk_bytes=8192)
        with pytest.raises(fsmspec.FsmError):
            f.set_options(chunk_bytes=16384)


def test_out_of_alphabet_is_reported():
    d = dfas.c_comment(False)   # 3-symbol alphabet -> internal sink
    good = np.array([0, 1, 2, 2, 1, 0] * 5000, np.uint8)
    assert gpu_run(d, good, k=2)[0] == seq.run(d, good)
    bad = good.copy()
    bad[12345] = 7
    with pytest.raises(fsmspec.SymbolError):
        gpu_run(d, bad, k=2)


# --------------------------------------------------------------------- bit mode (Huffman, Div7)
@pytest.mark.parametrize("n_bits", [0, 1, 3, 8, 13, 4096 * 8 + 5, 1_000_003])
def test_div7_bits(n_bits):
    d = dfas.div7()
    data = streams.random_bits(max(n_bits, 1), seed=n_bits)
    exp = seq.run(d, data, n_bits)
    for k in (1, 3, 7):
        for var in ("P8", "B", "G"):
            got, st = gpu_run(d, data, n_bits, k=k, variant=VARIANTS[var], chunk_bytes=64)
            assert got == exp, (n_bits, k, var)
            if k == 7:
                assert st["reexec_chunks"] == 0   # spec-N


@pytest.mark.parametrize("n,m", [(9, 1), (12, 3), (16, 2), (16, 16)])
@pytest.mark.parametrize("offset", [0, 5])
def test_r16_lane_replicated_bytes(n, m, offset):
    """R16 (N <= 16, lane-replicated byte entries): every k, both merges, look-back windows, eager
    completion, unaligned starts and a ragged tail against the oracle."""
    d = dfas.random_dfa(n, m, seed=7000 + n * 31 + m)
    length = 700_001
    data = streams.splitmix_bytes(900 + n + m, 0, length)
    exp = seq.run(d, data)
    for k in sorted({1, 2, 3, 4, n}):  # k <= N
        for opt in ({}, {"merge": fsmspec.FSM_MERGE_SEQUENTIAL}, {"lookback_len": 64}, {"eager_window": 64},
                    {"chunk_bytes": 96}):
            got, st = gpu_run(d, data, k=k, offset=offset, variant=VARIANTS["R16"], **opt)
            assert got == exp, (n, m, k, opt, st)
            assert st["variant"] == VARIANTS["R16"]


@pytest.mark.parametrize("kind", ["huffman13", "huffman17", "rand12", "rand16"])
def test_bit_mode_9_to_16_states_converging(kind):
    """Bit-mode DFAs with 9-16 states and chains that converge (Huffman decoders with 13 / 17
    symbols, near-permutation random bit DFAs), k >= 2, several chunkings.  A widened byte's count
    (F-visits over 8 bits) depends on the source state, so the region-counting R16 is byte-mode only:
    the library refuses it here and the auto choice (B) must be exact."""
    if kind.startswith("huffman"):
        ns = int(kind[7:])
        w = dfas.zipf_weights(ns, seed=ns)
        d, codes = dfas.huffman(w.tolist())
        n_bits = 2_000_003
        data, _ = streams.huffman_bits(codes, w / w.sum(), n_bits, seed=ns)
    else:
        n = int(kind[4:])
        r = dfas.random_dfa(n, n - 1, seed=31 * n, alphabet=2)
        d = dfas.DFA(r.table, 0, r.accept, True, f"randbits_{n}")
        n_bits = 2_000_003
        data = streams.random_bits(n_bits, seed=n)
    assert 9 <= d.n_states <= 16
    with FSM.from_dfa(d) as f, pytest.raises(fsmspec.FsmError):
        f.set_options(variant=VARIANTS["R16"])
    exp = seq.run(d, data, n_bits)
    for k in (2, 3, 4, 8):
        for chunk in (64, 256, 4096):
            got, st = gpu_run(d, data, n_bits, k=k, chunk_bytes=chunk)
            assert got == exp, (kind, k, chunk, st)
            assert st["variant"] == VARIANTS["B"]


def _accept_dfa(n, m, n_acc, alphabet, seed, ncls=None):
    """A random (n, m) DFA with exactly n_acc accepting states (region-counting edge cases); with
    ncls, its columns are those of a random ncls-symbol DFA under a random byte -> class map."""
    rng = np.random.default_rng(seed)
    if ncls:
        r = dfas.random_dfa(n, m, seed=seed, alphabet=ncls)
        table = np.ascontiguousarray(r.table[:, rng.integers(0, ncls, alphabet)])
    else:
        table = dfas.random_dfa(n, m, seed=seed, alphabet=alphabet).table
    acc = np.zeros(n, np.uint8)
    acc[rng.permutation(n)[:n_acc]] = 1
    return dfas.DFA(table, int(seed % n), acc, False, f"acc_{n}_{n_acc}")


@pytest.mark.parametrize("n,n_acc,alphabet", [(16, 0, 256), (16, 16, 256), (16, 8, 256), (16, 11, 256),
                                               (15, 7, 256), (15, 8, 200), (12, 1, 256), (13, 12, 97),
                                               (38, 5, 256), (38, 33, 256), (30, 15, 120)])
def test_region_counting_partitions(n, n_acc, alphabet):
    """R16 and CL count accepts by the destination id's region (accept-partitioned renumbering,
    host_tables.h renumber_by_accept): F empty, F = Q, balanced partitions, the complement
    orientation (|F| > |Q minus F|), a sink (alphabet < 256) and user start states that move.  Every k,
    chunk sizes with ragged tails, unaligned starts; results in user ids against the oracle."""
    d = _accept_dfa(n, 3, n_acc, alphabet, seed=8000 + 97 * n + n_acc + alphabet, ncls=None if n <= 16 else 20)
    if alphabet < 256:
        rng = np.random.default_rng(n)
        data = rng.integers(0, alphabet, 500_003).astype(np.uint8)
    else:
        data = streams.splitmix_bytes(8100 + n + n_acc, 0, 500_003)
    exp = seq.run(d, data)
    for var in ("R16", "RG", "CL"):
        if not fits(d, var):
            continue
        for k in (1, 2, 3, 4):
            for chunk, offset in ((0, 0), (96, 0), (1024, 7)):
                got, st = gpu_run(d, data, k=k, variant=VARIANTS[var], chunk_bytes=chunk, offset=offset)
                assert got == exp, (var, k, chunk, offset, st)
                assert st["variant"] == VARIANTS[var]


def test_div7_closed_form_on_gpu():
    d = dfas.div7()
    n_bits = 5000
    data = streams.random_bits(n_bits, seed=3)
    bits = "".join(str(b) for b in seq.bits_of(data, n_bits))
    got, _ = gpu_run(d, data, n_bits, k=7)
    assert got[0] == int(bits, 2) % 7


def test_huffman_zipf():
    w = dfas.zipf_weights(256, seed=streams.MASTER_SEED + 2)
    d, codes = dfas.huffman(w.tolist())
    n_bits = 3_000_005
    data, nsym = streams.huffman_bits(codes, w / w.sum(), n_bits, seed=11)
    exp = seq.run(d, data, n_bits)
    assert exp[1] == nsym
    for k in (1, 2, 4):
        for var in ("B", "G"):
            got, st = gpu_run(d, data, n_bits, k=k, variant=VARIANTS[var])
            assert got == exp, (k, var, st)


def test_aho_corasick():
    pats = dfas.snort_patterns(1024, seed=streams.MASTER_SEED + 3)
    d = dfas.aho_corasick(pats)
    rng = np.random.default_rng(3)
    data = rng.integers(0, 256, 2_000_000).astype(np.uint8)
    for _ in range(500):
        p = pats[int(rng.integers(0, len(pats)))]
        pos = int(rng.integers(0, data.size - len(p)))
        data[pos:pos + len(p)] = np.frombuffer(p, np.uint8)
    exp = seq.run(d, data)
    for k in (1, 2, 4):
        for var in ("HS", "G"):
            got, _ = gpu_run(d, data, k=k, variant=VARIANTS[var])
            assert got == exp, (k, var)
    # renumbered handle (hot-state caching): the async result is in user state ids
    with FSM.from_dfa(d) as f:
        buf, ptr = dev(data)
        res = torch.zeros(4, dtype=torch.int32, device="cuda")
        f.run_spec_k_async(ptr, data.size, 2, res.data_ptr())
        r = res.cpu().numpy().view(np.uint32)
        assert (int(r[0]), int(r[2]) | (int(r[3]) << 32)) == exp
        m, sh = f.run_shard(ptr + 1000 * 32, data.size - 1000 * 32, halo=ptr + 1000 * 32 - 1, halo_len=1, k=2,
                            keep=True)
        for s_, e_, c_ in m.slots():
            assert (e_, c_) == seq.run_from(d, s_, data[1000 * 32:])
        q = int(seq.run(d, data[:1000 * 32])[0])
        assert f.shard_fixup(sh, q) == seq.run_from(d, q, data[1000 * 32:])


# --------------------------------------------------------------------- other entry points
def test_sequential_merge_ablation_parity():
    d = dfas.random_dfa(16, 5, seed=9)
    data = streams.splitmix_bytes(9, 0, 2_000_017)
    exp = seq.run(d, data)
    for k in (1, 2, 5):
        got, st = gpu_run(d, data, k=k, merge=fsmspec.FSM_MERGE_SEQUENTIAL)
        assert got == exp, (k, st)
    got, st = gpu_run(dfas.div7(), streams.random_bits(100_000, 1), 100_000, k=3,
                      merge=fsmspec.FSM_MERGE_SEQUENTIAL, chunk_bytes=64)
    assert got == seq.run(dfas.div7(), streams.random_bits(100_000, 1), 100_000)


def test_async_and_host_entry_points():
    d = dfas.random_dfa(8, 2, seed=5)
    data = streams.splitmix_bytes(21, 0, 5_000_000)
    exp = seq.run(d, data)
    with FSM.from_dfa(d) as f:
        buf, ptr = dev(data)
        res = torch.zeros(4, dtype=torch.int32, device="cuda")
        f.run_spec_k_async(ptr, data.size, 2, res.data_ptr())
        r = res.cpu().numpy().view(np.uint32)
        assert (int(r[0]), int(r[2]) | (int(r[3]) << 32)) == exp
        assert f.run_spec_k_host(data, data.size, 2) == exp
        pinned = torch.from_numpy(data).pin_memory()
        assert f.run_spec_k_host(pinned.data_ptr(), data.size, 1) == exp


def test_host_entry_point_multi_piece():
    d = dfas.random_dfa(16, 3, seed=6)
    length = (1 << 28) + 12345   # two 256 MiB pieces chained on the device
    data = np.empty(length, np.uint8)
    streams.splitmix_bytes(31, 0, length, out=data)
    exp = seq.run(d, data)
    with FSM.from_dfa(d) as f:
        assert f.run_spec_k_host(data, length, 3) == exp


# --------------------------------------------------------------------- shards (multi-GPU logic)
@pytest.mark.parametrize("G", [2, 3, 5])
@pytest.mark.parametrize("k", [1, 2])
def test_shard_maps_compose_and_fixup(G, k):
    """Single-GPU emulation of G shards: per-shard maps keyed on the halo's
    look-back set equal the oracle from each start; composing them and fixing up the
    shard-boundary misses gives the oracle result."""
    d = dfas.random_dfa(16, 4, seed=77 + G)
    L = 3_000_000
    data = streams.splitmix_bytes(4 + G, 0, L)
    exp = seq.run(d, data)
    bounds = [L * g // G // 32 * 32 for g in range(G)] + [L]
    buf, base = dev(data)
    with FSM.from_dfa(d) as f:
        maps, shards = [], []
        for g in range(G):
            lo, hi = bounds[g], bounds[g + 1]
            m, st = f.run_shard(base + lo, hi - lo, halo=(base + lo - 1) if g else None,
                                halo_len=1 if g else 0, k=k, keep=True)
            # each slot equals the oracle run from its start
            for s, e, c in m.slots():
                assert (e, c) == seq.run_from(d, s, data[lo:hi]), (g, s)
            if g:
                starts = [s for s, _, _ in m.slots()]
                assert starts == speck.lookback(d.table, int(data[lo - 1]), k)
            maps.append(m)
            shards.append(st)
        x, total = d.start, 0
        for g in range(G):
            hit = [(e, c) for s, e, c in maps[g].slots() if s == x]
            if hit:
                e, c = hit[0]
            else:
                e, c = f.shard_fixup(shards[g], x)
            x, total = e, total + c
        assert (x, total) == exp


@pytest.mark.parametrize("kind", ["rand16_6", "html", "div7", "rand8_3_unaligned"])
def test_shard_fixup_walks_tile_descriptors(kind):
    """SURVEY.md 8.e fix-up: for every true start that the shard did not speculate (k < |image(halo)|),
    fsm_shard_fixup equals the oracle from that start.  For converging DFAs the walk re-executes
    at most one tile (it joins a shard slot's path at the first tile boundary) and costs < 1 % of the
    shard run; for a permutation DFA (Div7, paths never meet) it falls back to the parallel kernel."""
    off = 0
    if kind == "html":
        d, data, k, nsym = dfas.html_tokenizer(), streams.html_bytes(64 << 20, 9), 1, None
    elif kind == "div7":
        d, k = dfas.div7(), 2
        data = streams.random_bits(8 * (16 << 20), 6)
        nsym = 8 * (16 << 20)
    else:
        n, m = int(kind.split("_")[0][4:]), int(kind.split("_")[1])
        d, data, k, nsym = dfas.random_dfa(n, m, seed=n * m), streams.splitmix_bytes(n + m, 0, 64 << 20), 2, None
        if "unaligned" in kind:
            off = 5
    nbytes = data.size
    lo = (nbytes // 3) // 32 * 32 + off
    buf, base = dev(data)
    shard = data[lo:]
    with FSM.from_dfa(d) as f:
        s_sym = (nbytes - lo) * 8 if d.bit_mode else nbytes - lo
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record()
        m, st = f.run_shard(base + lo, s_sym, halo=base + lo - 1, halo_len=1, k=k, keep=True)
        t1.record()
        torch.cuda.synchronize()
        shard_ms = t0.elapsed_time(t1)
        spec = {s for s, _, _ in m.slots()}
        n_int = d.n_states
        misses = [x for x in range(n_int) if x not in spec]
        assert misses, "k < |image(halo)| needed"
        for x in misses[:6]:
            exp = seq.run_from(d, x, shard, s_sym if d.bit_mode else None)
            t0.record()
            got = f.shard_fixup(st, x)
            t1.record()
            torch.cuda.synchronize()
            assert got == exp, (kind, x)
            fst = f.stats()
            if kind != "div7":
                assert fst["reexec_true"] <= 1, fst          # touched at most one tile
                assert t0.elapsed_time(t1) < 0.01 * shard_ms + 0.5, (t0.elapsed_time(t1), shard_ms)
        st.close()


# --------------------------------------------------------------------- look-back windows (R7)
def _wl_cases():
    pats = dfas.snort_patterns(300, seed=8)
    w = dfas.zipf_weights(256, seed=4)
    hd, codes = dfas.huffman(w.tolist())
    hb, _ = streams.huffman_stream(codes, w, 8 * 600_000 + 5, seed=5)
    return [
        ("html", dfas.html_tokenizer(), streams.html_bytes(1_500_000, 3), None),
        ("ccomment", dfas.c_comment(True), streams.c_source(700_001, seed=3, comment_frac=0.4), None),
        ("ac", dfas.aho_corasick(pats), streams.ac_payload(1_200_000, 4, pats), None),
        ("rand", dfas.random_dfa(64, 6, seed=3), streams.splitmix_bytes(12, 0, 1_000_001), None),
        ("huff", hd, hb, 8 * 600_000 + 5),
        ("div7", dfas.div7(), streams.random_bits(8 * 300_000 + 3, 6), 8 * 300_000 + 3),
    ]


@pytest.mark.parametrize("lookback", [32, 64, 256])
def test_lookback_window_parity(lookback):
    for name, d, data, length in _wl_cases():
        exp = seq.run(d, data, length)
        for k in (1, 2):
            for chunk in (64, 2048):
                got, st = gpu_run(d, data, length, k=k, chunk_bytes=chunk, lookback_len=lookback)
                assert got == exp, (name, lookback, k, chunk, st)
                assert st["lookback_len"] == lookback


@pytest.mark.parametrize("width", [4, 8, 12])
def test_lookback_width_parity(width):
    """The window walk over the top 4 / 8 / 12 image states only (fsm_options.lookback_width): exact
    results, the width reported; widths that are not multiples of 4 (or > 16) are rejected."""
    for name, d, data, length in _wl_cases():
        exp = seq.run(d, data, length)
        for k in (1, 3):
            got, st = gpu_run(d, data, length, k=k, chunk_bytes=512, lookback_len=64, lookback_width=width)
            assert got == exp, (name, width, k, st)
            assert st["lookback_width"] == width and st["lookback_len"] == 64
    with FSM.from_dfa(dfas.html_tokenizer()) as f:
        for bad in (2, 5, 20):
            with pytest.raises(fsmspec.FsmError):
                f.set_options(lookback_len=64, lookback_width=bad)


def test_lookback_window_reduces_misses():
    d = dfas.html_tokenizer()
    data = streams.html_bytes(4_000_000, 5)
    _, st1 = gpu_run(d, data, k=2, chunk_bytes=1024)
    _, st64 = gpu_run(d, data, k=2, chunk_bytes=1024, lookback_len=64)
    assert st64["reexec_chunks"] < st1["reexec_chunks"] / 4, (st1, st64)


@pytest.mark.parametrize("lookback", [0, 64])
def test_lookback_seqmerge_and_shards(lookback):
    d = dfas.html_tokenizer()
    data = streams.html_bytes(2_000_000, 8)
    exp = seq.run(d, data)
    got, _ = gpu_run(d, data, k=2, merge=fsmspec.FSM_MERGE_SEQUENTIAL, lookback_len=lookback)
    assert got == exp
    buf, base = dev(data)
    G, L = 3, data.size
    bounds = [L * g // G // 32 * 32 for g in range(G)] + [L]
    with FSM.from_dfa(d) as f:
        f.set_options(lookback_len=lookback)
        x, total = d.start, 0
        for g in range(G):
            lo, hi = bounds[g], bounds[g + 1]
            m, sh = f.run_shard(base + lo, hi - lo, halo=(base + lo - 1) if g else None,
                                halo_len=1 if g else 0, k=2, keep=True)
            for s, e, c in m.slots():
                assert (e, c) == seq.run_from(d, s, data[lo:hi])
            hit = [(e, c) for s, e, c in m.slots() if s == x]
            e, c = hit[0] if hit else f.shard_fixup(sh, x)
            x, total = e, total + c
        assert (x, total) == exp


@pytest.mark.parametrize("lookback", [0, 64])
def test_html_all_variants(lookback):
    d = dfas.html_tokenizer()
    data = streams.html_bytes(2_500_000, 21)
    exp = seq.run(d, data)
    for var in ("CL", "B", "G", "HS"):
        for k in (1, 2, 4):
            got, st = gpu_run(d, data, k=k, variant=VARIANTS[var], lookback_len=lookback)
            assert got == exp, (var, k, lookback, st)


def test_merge_switch_reuses_window_buffers():
    """One handle alternating parallel / sequential merge with the window pre-pass, growing the
    input between calls (the bench's ablation pattern): every result equals the oracle's.  A
    sequential-merge (re)allocation once freed the pre-pass buffer still in use (illegal access)."""
    d = dfas.html_tokenizer()
    data = streams.html_bytes(6_000_000, 33)
    buf, base = dev(data)
    with FSM.from_dfa(d) as f:
        for n in (1_000_000, 3_000_000, 6_000_000):
            exp = seq.run(d, data[:n])
            for merge in (fsmspec.FSM_MERGE_PARALLEL, fsmspec.FSM_MERGE_SEQUENTIAL, fsmspec.FSM_MERGE_PARALLEL):
                f.set_options(lookback_len=64, merge=merge, chunk_bytes=512)
                assert f.run_spec_k(base, n, 2) == exp, (n, merge)
        torch.cuda.synchronize()


@pytest.mark.parametrize("eager", [fsmspec.FSM_EAGER_OFF, 32, 128])
def test_eager_window_settings(eager):
    """Eager completion (NEXT-3) off, short and full: identical results, and switching it off
    cannot reduce the re-execution count (it only ever replaces re-executions)."""
    cases = [("html", dfas.html_tokenizer(), streams.html_bytes(3_000_000, 41), 2),
             ("rand64m4", dfas.random_dfa(64, 4, seed=7), streams.splitmix_bytes(9, 0, 2_000_000), 2)]
    for name, d, data, k in cases:
        exp = seq.run(d, data)
        for lb in (0, 64):
            got, st = gpu_run(d, data, k=k, lookback_len=lb, eager_window=eager, chunk_bytes=1024)
            assert got == exp, (name, eager, lb, st)
            if eager == fsmspec.FSM_EAGER_OFF:
                _, st_on = gpu_run(d, data, k=k, lookback_len=lb, chunk_bytes=1024)
                assert st["reexec_chunks"] >= st_on["reexec_chunks"], (name, lb, st, st_on)


def test_autotune_choice_is_exact_and_not_slower():
    """NEXT-2: fsm_autotune times candidates on a prefix sample and applies the fastest windows; the
    run with the chosen k and options equals the oracle, and the choice is never slower (on the
    sample) than the paper's plain setting it also timed."""
    cases = [("html", dfas.html_tokenizer(), streams.html_bytes(24_000_000, 51), 0, 0),
             ("rand16m2", dfas.random_dfa(16, 2, seed=3), streams.splitmix_bytes(4, 0, 16_000_000), 0, 4),
             ("rand64m4-fixedk", dfas.random_dfa(64, 4, seed=5), streams.splitmix_bytes(6, 0, 8_000_000), 2, 2)]
    for name, d, data, kmin, kmax in cases:
        exp = seq.run(d, data)
        buf, ptr = dev(data)
        with FSM.from_dfa(d) as f:
            t = f.autotune(ptr, data.size, k_min=kmin, k_max=kmax, sample_len=8_000_000)
            assert t["candidates"] >= 3 and 0.0 <= t["hit_rate"] <= 1.0, (name, t)
            assert t["best_gbs"] >= t["paper_gbs"] > 0 or kmin > 1, (name, t)
            if kmin:
                assert t["k"] == kmin
            o = f.options()
            assert o["lookback_len"] == t["lookback_len"] and o["eager_window"] == t["eager_window"]
            assert o["variant"] == t["variant"] and t["variant"] in VARIANTS.values()
            assert f.run_spec_k(ptr, data.size, t["k"]) == exp, (name, t)
        torch.cuda.synchronize()


def test_run_multi_matches_single_runs():
    """NEXT-4: many FSMs over one resident input.  fsm_run_multi fuses DFAs of the same variant and
    K into one launch; every DFA's result equals the oracle, across mixed variants (P4, P8, B, CL,
    HS/G), mixed k, per-handle look-back options and a ragged length."""
    data = streams.html_bytes(5_000_003, 61)
    buf, ptr = dev(data)
    dfa_list = [dfas.html_tokenizer(), dfas.random_dfa(8, 2, seed=1), dfas.random_dfa(8, 3, seed=2),
                dfas.c_comment(True), dfas.random_dfa(16, 2, seed=3), dfas.random_dfa(200, 4, seed=4),
                dfas.random_dfa(8, 2, seed=5), dfas.aho_corasick(dfas.snort_patterns(300, seed=6))]
    ks = [1, 2, 2, 1, 2, 4, 2, 1]
    exp = [seq.run(d, data) for d in dfa_list]
    fs = [FSM.from_dfa(d) for d in dfa_list]
    try:
        fs[0].set_options(lookback_len=64)
        fs[4].set_options(lookback_len=32, eager_window=fsmspec.FSM_EAGER_OFF)
        got = fsmspec.run_multi(fs, ptr, data.size, ks)
        assert got == exp
        # stats describe each handle's own run
        for f in fs:
            assert f.stats()["chunks"] > 0
        # a second call on the same handles (epochs, tickets advance) and a sub-group
        assert fsmspec.run_multi(fs[1:3] + fs[6:7], ptr, 4_000_000, [2, 2, 2]) == \
            [seq.run(d, data[:4_000_000]) for d in (dfa_list[1], dfa_list[2], dfa_list[6])]
        with pytest.raises(fsmspec.FsmError):
            fsmspec.run_multi([fs[1], fs[1]], ptr, data.size, [1, 1])
    finally:
        for f in fs:
            f.close()
        torch.cuda.synchronize()


@pytest.mark.parametrize("k", [6, 8, 12, 16])
def test_html_cl_large_k(k):
    """Large-K CL kernels: the split (epilogue-warp) layout does not fit next to the 146 KiB class
    table for every K, so those launches fall back to the unsplit kernel; both are exact."""
    d = dfas.html_tokenizer()
    data = streams.html_bytes(3_000_001, 71 + k)
    exp = seq.run(d, data)
    for lb in (0, 64):
        got, st = gpu_run(d, data, k=k, variant=VARIANTS["CL"], lookback_len=lb)
        assert got == exp, (k, lb, st)


# --------------------------------------------------------------------- production geometry
FULL_CASES = [("P4", 4, 2), ("N8", 8, 2), ("P8", 8, 3), ("R16", 16, 2), ("B", 64, 4), ("RG", 64, 4), ("RG", 200, 3), ("G", 1000, 3),
              ("HS", 3000, 3), ("CL", 0, 0)]


@pytest.mark.parametrize("var,n,m", FULL_CASES)
def test_full_geometry_parity(var, n, m):
    """Every table variant at the bench's launch geometry (inputs large enough that pick_geometry
    chooses the maximal tile and chunks of several KiB -- up to 16 KiB, 4 KiB for the L2-table
    variants G / HS -- split kernels where the policy splits) against the
    oracle, k = 1 and 2, with the default look-back and eager completion."""
    L = 1280 << 20  # > 148 SMs x 1024 threads x 8 KiB: the maximal tile, two waves of tiles
    if var == "CL":
        d = dfas.html_tokenizer()
        data = streams.html_bytes(L, 21)
    else:
        d = dfas.random_dfa(n, m, seed=900 + n)
        data = streams.splitmix_bytes(31 + n, 0, L)
    exp = seq.run(d, data)
    buf, ptr = dev(data)
    with FSM.from_dfa(d) as f:
        for k in (1, 2):
            f.set_options(variant=VARIANTS[var], lookback_len=64 if var == "CL" else 0)
            assert f.run_spec_k(ptr, L, k) == exp, (var, k)
            st = f.stats()
            assert 2048 <= st["chunk_bytes"] <= (4096 if var in ("G", "HS") else 16384), st
            assert st["threads_per_tile"] >= 224, st
            assert st["variant"] == VARIANTS[var]
