"""Pins for the oracle (oracle/seq.py, oracle/speck.py) against what the paper and mathematics fix.

Every oracle function is pinned to something other than itself:
paper-printed worked examples (tests/golden/*.json with citations), closed forms (Div7), an
independent matrix formulation of the DFA run, brute force on tiny DFAs, generator round trips
(Huffman, Aho-Corasick vs naive search) and algebraic invariants (associativity, k-invariance).
"""
import itertools
import random

import numpy as np
import pytest

from fsmgen import dfas, streams
from oracle import seq, speck

ST = {"a": 0, "b": 1, "c": 2, "d": 3}
NAME = "abcd"


def cc_syms(text: str):
    return [{"/": 0, "*": 1}.get(ch, 2) for ch in text]


# ------------------------------------------------------------------ the Fig. 1 table itself
def test_fig1_table_matches_golden(golden):
    g = golden["c_comment_fig1"]
    d = dfas.c_comment(expanded=False)
    assert d.table.tolist() == g["table"]
    indeg = np.bincount(d.table.ravel(), minlength=4)
    assert [int(x) for x in indeg] == [g["in_degree"][s] for s in "abcd"]
    img = sorted({int(d.table[s, 2]) for s in range(4)})
    assert img == [ST[s] for s in g["image_x"]["states"]]


def test_fig1_expanded_table_consistent():
    d3, d = dfas.c_comment(False), dfas.c_comment(True)
    for byte in range(256):
        assert (d.table[:, byte] == d3.table[:, {0x2F: 0, 0x2A: 1}.get(byte, 2)]).all()


# ------------------------------------------------------------------ P1 and derived mini pins
def test_p1_paper_final_state(golden):
    g = golden["c_comment_fig1"]["P1"]
    d = dfas.c_comment(True)
    data = np.frombuffer(g["input"].encode(), np.uint8)
    q, n = seq.run(d, data)
    assert q == ST[g["final"]]
    assert n == 1                                                                 # reading A4
    q2, n2 = seq.run_py(dfas.c_comment(False).table, 0, d.accept, cc_syms(g["input"]))
    assert (q2, n2) == (q, n)


def test_c_comment_mini_pins_with_traces(golden):
    d3 = dfas.c_comment(False)
    d = dfas.c_comment(True)
    for case in golden["derived_mini_pins"]["c_comment"]:
        syms = cc_syms(case["input"])
        # step-by-step trace through the Fig. 1b table
        q, trace = 0, ""
        for c in syms:
            q = int(d3.table[q, c])
            trace += NAME[q]
        assert trace == case["trace"]
        exp = (ST[case["final"]], case["count"])
        assert seq.run_py(d3.table, 0, d3.accept, syms) == exp
        assert seq.run(d, np.frombuffer(case["input"].encode(), np.uint8)) == exp
        assert seq.run(d3, np.array(syms, np.uint8)) == exp


# ------------------------------------------------------------------ Div7 closed form
def _div7_expect(bits: str):
    v, cnt = 0, 0
    for i in range(len(bits)):
        v = int(bits[: i + 1], 2)
        cnt += v % 7 == 0
    return (int(bits, 2) % 7 if bits else 0), cnt


def test_div7_golden(golden):
    d = dfas.div7()
    for case in golden["derived_mini_pins"]["div7_msb_first"]:
        b = case["bits"]
        assert _div7_expect(b) == (case["final"], case["count"])
        data = np.packbits(np.array([int(ch) for ch in b], np.uint8)) if b else np.zeros(1, np.uint8)
        assert seq.run(d, data, len(b)) == (case["final"], case["count"])


def test_div7_partial_byte_pin():
    # byte 0xE0 with len = 3 bits -> '111' = 7 -> (0, 1); pad bits ignored (reading A13)
    assert seq.run(dfas.div7(), np.array([0xE0], np.uint8), 3) == (0, 1)
    assert seq.run(dfas.div7(), np.array([0xFF], np.uint8), 3) == (0, 1)


@pytest.mark.parametrize("n_bits", [1, 7, 8, 9, 63, 64, 500, 2048])
def test_div7_closed_form_random(n_bits):
    data = streams.random_bits(n_bits, seed=n_bits)
    bits = "".join(str(x) for x in seq.bits_of(data, n_bits))
    final = int(bits, 2) % 7
    # count of prefixes divisible by 7 with Python big ints
    v, cnt = 0, 0
    for ch in bits:
        v = 2 * v + int(ch)
        cnt += v % 7 == 0
    assert seq.run(dfas.div7(), data, n_bits) == (final, cnt)


# ------------------------------------------------------------------ independent matrix formulation
def _matrix_run(table, start, accept, syms):
    """Reference through linear algebra: the state distribution e_q0 propagated by the 0/1
    transition matrices M_c[s, t] = [delta(s, c) == t] (row vector times matrix)."""
    n = table.shape[0]
    mats = []
    for c in range(table.shape[1]):
        m = np.zeros((n, n), dtype=np.int64)
        m[np.arange(n), table[:, c]] = 1
        mats.append(m)
    v = np.zeros(n, dtype=np.int64)
    v[start] = 1
    f = np.asarray(accept, dtype=np.int64)
    cnt = 0
    for c in syms:
        v = v @ mats[c]
        cnt += int(v @ f)
    return int(np.argmax(v)), cnt


@pytest.mark.parametrize("seed", range(12))
def test_oracle_vs_matrix_formulation(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 9))
    a = int(rng.integers(1, 6))
    table = rng.integers(0, n, (n, a)).astype(np.uint32)
    acc = (rng.random(n) < 0.4).astype(np.uint8)
    start = int(rng.integers(0, n))
    syms = rng.integers(0, a, int(rng.integers(0, 200))).astype(np.uint8)
    d = dfas.DFA(table, start, acc)
    exp = _matrix_run(table, start, acc, syms)
    assert seq.run(d, syms) == exp
    assert seq.run_py(table, start, acc, syms.tolist()) == exp


def test_oracle_rejects_out_of_alphabet():
    d = dfas.c_comment(False)
    with pytest.raises(seq.OracleSymbolError):
        seq.run(d, np.array([0, 1, 3], np.uint8))
    with pytest.raises(seq.OracleSymbolError):
        seq.run_py(d.table, 0, d.accept, [0, 5])


# ------------------------------------------------------------------ generators (round trips)
def test_huffman_mini_pin(golden):
    g = golden["derived_mini_pins"]["huffman_mini"]
    d, codes = dfas.huffman(g["weights"])
    assert codes == g["codes"]
    assert d.table.tolist() == g["table"]
    for s in g["streams"]:
        bits = np.array([int(ch) for ch in s["bits"]], np.uint8)
        assert seq.run(d, np.packbits(bits), len(bits)) == (s["final"], s["count"])


def test_huffman_zipf_roundtrip():
    w = dfas.zipf_weights(256, seed=7)
    d, codes = dfas.huffman(w.tolist())
    assert d.n_states == 255                      # states = #symbols - 1 (PAPER.md:266/300 structure)
    p = w / w.sum()
    data, nsym = streams.huffman_bits(codes, p, 200_000, seed=3)
    q, n = seq.run(d, data, 200_000)
    assert n == nsym                              # root visits = complete codewords
    # an uncut stream returns to the root
    nb = sum(len(codes[s]) for s in [1, 2, 3])
    bits = np.array([int(ch) for ch in codes[1] + codes[2] + codes[3]], np.uint8)
    assert seq.run(d, np.packbits(bits), nb) == (0, 3)


def test_aho_corasick_textbook(golden):
    g = golden["derived_mini_pins"]["aho_corasick_textbook"]
    d = dfas.aho_corasick([p.encode() for p in g["patterns"]])
    assert d.n_states == g["n_states"]
    assert seq.run(d, np.frombuffer(g["text"].encode(), np.uint8))[1] == g["count"]


def test_aho_corasick_vs_naive_search():
    pats = dfas.snort_patterns(60, seed=5)
    d = dfas.aho_corasick(pats)
    rng = np.random.default_rng(1)
    text = bytearray(rng.integers(97, 123, 20000).astype(np.uint8).tobytes())
    for _ in range(30):  # plant patterns
        p = pats[int(rng.integers(0, len(pats)))]
        pos = int(rng.integers(0, len(text) - len(p)))
        text[pos:pos + len(p)] = p
    text = bytes(text)
    ends = set()
    for p in pats:
        i = text.find(p)
        while i >= 0:
            ends.add(i + len(p))
            i = text.find(p, i + 1)
    assert seq.run(d, np.frombuffer(text, np.uint8))[1] == len(ends)


@pytest.mark.parametrize("n,m", [(8, 1), (8, 2), (16, 2), (64, 4), (256, 16)])
def test_random_dfa_image_size(n, m):
    d = dfas.random_dfa(n, m, seed=n * 31 + m)
    for c in range(256):
        assert len(set(d.table[:, c].tolist())) == m


def _mod7_bytes_dfa():
    """Byte-mode Div7: state = value of the big-endian byte string so far mod 7, F = {0}."""
    t = np.array([[(256 * s + c) % 7 for c in range(256)] for s in range(7)], np.uint32)
    acc = np.zeros(7, np.uint8)
    acc[0] = 1
    return dfas.DFA(t, 0, acc, False, "mod7_bytes")


@pytest.mark.parametrize("G,piece", [(1, 1 << 28), (5, 64), (9, 1000)])
def test_certify_closed_form(G, piece):
    """seq.certify against the closed form of byte-mode Div7: claims computed with
    Python big ints (int.from_bytes(prefix) % 7) pass and return (value mod 7, #prefixes = 0 mod
    7); a corrupted claim, a wrong segment-0 start, or a claim off by one segment all fail."""
    d = _mod7_bytes_dfa()
    data = np.random.default_rng(G).integers(0, 256, 3001).astype(np.uint8)
    L = data.size
    bounds = [L * g // G for g in range(G)] + [L]
    val = [int.from_bytes(data[:b].tobytes(), "big") % 7 for b in range(L + 1)]
    claims = [val[b] for b in bounds[:-1]]
    exp = (val[L], sum(1 for i in range(1, L + 1) if val[i] == 0))

    def fetch(lo, hi):
        return data[lo:hi]

    assert seq.certify(d, bounds, claims, fetch, piece=piece) == exp
    if G > 1:
        bad = list(claims)
        bad[G // 2] = (bad[G // 2] + 1) % 7
        with pytest.raises(seq.CertificateError):
            seq.certify(d, bounds, bad, fetch, piece=piece)
        shifted = [claims[0]] + [val[b + 1] for b in bounds[1:-1]]
        if shifted != claims:
            with pytest.raises(seq.CertificateError):
                seq.certify(d, bounds, shifted, fetch, piece=piece)
    with pytest.raises(seq.CertificateError):
        seq.certify(d, bounds, [(claims[0] + 3) % 7] + claims[1:], fetch, piece=piece)


def test_splitmix_c_matches_numpy():
    w = streams.splitmix_words(123, 5, 100)
    b = streams.splitmix_bytes(123, 40, 800)
    assert b.tobytes() == w.tobytes()
    b2 = streams.splitmix_bytes(123, 43, 9)
    assert b2.tobytes() == w.tobytes()[3:12]


# ------------------------------------------------------------------ the spec-k CPU model
def test_p2_fig2_speculation(golden):
    g = golden["c_comment_fig2_fig4"]["P2"]
    d = dfas.c_comment(False)
    syms = cc_syms("".join(g["chunks"]))
    data = np.array(syms, np.uint8)
    assert speck.lookback(d.table, 2, 1) == [ST[g["guess_chunk1"]]]
    r = speck.spec_k(d, data, k=1, bounds=[0, 4, 8])
    assert r["maps"][1].starts == [ST["a"]]
    assert r["maps"][1].ends == [ST["b"]]                                          # wrong guess
    assert r["reexec"] == g["reexec"]
    assert r["final"] == ST[g["final"]]


def _fig4(golden, strategy="delayed", check="nested"):
    g = golden["c_comment_fig2_fig4"]["P3"]
    d = dfas.c_comment(False)
    data = np.array(cc_syms("".join(g["chunks"])), np.uint8)
    sets = [[ST[s] for s in ss] for ss in g["injected_sets"]]
    return g, d, speck.spec_k(d, data, k=2, bounds=[0, 2, 4, 6, 8], injected=sets,
                              strategy=strategy, check=check)


def _as_dict(m):
    return {NAME[s]: (None if e is None else [NAME[e], c]) for s, e, c in zip(m.starts, m.ends, m.counts)}


@pytest.mark.parametrize("check", ["nested", "hash"])
def test_p3_fig4_parallel_merge(golden, check):
    g, d, r = _fig4(golden, check=check)
    maps = r["maps"]
    m01 = speck.merge(maps[0], maps[1], check)
    m23 = speck.merge(maps[2], maps[3], check)
    assert _as_dict(m01) == {k: v for k, v in g["merged_01"].items()}
    assert _as_dict(m23) == {k: v for k, v in g["merged_23"].items()}
    root = speck.merge(m01, m23, check)
    assert _as_dict(root) == g["root"]
    # associativity: (((0 x 1) x 2) x 3) gives the same root
    left = speck.merge(speck.merge(speck.merge(maps[0], maps[1], check), maps[2], check), maps[3], check)
    assert _as_dict(left) == g["root"]
    assert (r["final"], r["count"]) == (ST["a"], 1)


def test_p4_fig4_reexecution_counts(golden):
    g = golden["c_comment_fig2_fig4"]["P4"]
    assert _fig4(golden, "delayed")[2]["reexec"] == g["reexec_delayed"]
    assert _fig4(golden, "eager")[2]["reexec"] == g["reexec_eager"]
    assert _fig4(golden, "sequential")[2]["reexec"] == g["reexec_sequential"]


def _random_map(rng, n, k, first):
    starts = rng.sample(range(n), min(k, n))
    ends = [rng.randrange(n) if rng.random() < 0.85 else None for _ in starts]
    return speck.Mapping(starts, ends, [rng.randrange(5) for _ in starts], first, first)


@pytest.mark.parametrize("seed", range(40))
def test_merge_associative_and_checks_agree(seed):
    rng = random.Random(seed)
    n, k = rng.randint(1, 8), rng.randint(1, 5)
    a, b, c = (_random_map(rng, n, k, i) for i in range(3))
    for chk in ("nested", "hash"):
        x = speck.merge(speck.merge(a, b, chk), c, chk)
        y = speck.merge(a, speck.merge(b, c, chk), chk)
        assert (x.ends, x.counts) == (y.ends, y.counts)
    probe = [e for e in a.ends if e is not None] + list(range(n))
    assert speck.check_nested_loop(probe, b.starts) == speck.check_hash(probe, b.starts)


def test_brute_force_model_equals_oracle():
    """All DFAs with N <= 2 and |Sigma| = 2 (every start, every F), all inputs of length <= 6,
    every chunking into <= 3 chunks, k = 1..N; plus random speculated subsets.  Every strategy
    and both checks must equal the sequential oracle (SURVEY.md 8.c.4 brute force)."""
    rng = random.Random(0)
    cases = 0
    for n in (1, 2):
        for flat in itertools.product(range(n), repeat=2 * n):
            table = np.array(flat, np.uint32).reshape(n, 2)
            for start in range(n):
                for fmask in itertools.product((0, 1), repeat=n):
                    d = dfas.DFA(table, start, np.array(fmask, np.uint8))
                    for L in range(0, 7):
                        for bits in itertools.product((0, 1), repeat=L):
                            data = np.array(bits, np.uint8)
                            exp = seq.run_py(table, start, fmask, bits)
                            for nc in range(1, min(3, max(L, 1)) + 1):
                                for k in range(1, n + 1):
                                    for strat in ("delayed", "sequential", "eager"):
                                        r = speck.spec_k(d, data, k=k, n_chunks=nc, strategy=strat)
                                        assert (r["final"], r["count"]) == exp
                                        cases += 1
                                inj = [[start]] + [rng.sample(range(n), rng.randint(1, n))
                                                   for _ in range(nc - 1)]
                                r = speck.spec_k(d, data, k=n, n_chunks=nc, injected=inj, check="hash")
                                assert (r["final"], r["count"]) == exp
    assert cases > 10000


@pytest.mark.parametrize("seed", range(6))
def test_model_random_n3_and_k_invariance(seed):
    rng = np.random.default_rng(seed)
    n = 3
    table = rng.integers(0, n, (n, 2)).astype(np.uint32)
    d = dfas.DFA(table, 0, (rng.random(n) < 0.5).astype(np.uint8))
    data = rng.integers(0, 2, 40).astype(np.uint8)
    exp = seq.run(d, data)
    for k in (1, 2, 3):
        for nc in (1, 3, 8, 40):
            r = speck.spec_k(d, data, k=k, n_chunks=nc)
            assert (r["final"], r["count"]) == exp
            if k == n:
                assert r["reexec"] == 0                          # spec-N never re-executes


def test_k_at_least_image_never_reexecutes():
    d = dfas.random_dfa(16, 3, seed=11)
    data = streams.splitmix_bytes(9, 0, 3000)
    exp = seq.run(d, data)
    r = speck.spec_k(d, data, k=3, n_chunks=50)
    assert (r["final"], r["count"]) == exp and r["reexec"] == 0
    r1 = speck.spec_k(d, data, k=1, n_chunks=50)
    assert (r1["final"], r1["count"]) == exp and r1["reexec"] > 0


def test_div7_hit_rate_linear_in_k():
    """for random bits the speculation success rate is linear in k (-> k/7)."""
    d = dfas.div7()
    data = streams.random_bits(7 * 4000, seed=77)
    n_chunks = 700
    rates = []
    for k in (1, 2, 4, 7):
        r = speck.spec_k(d, data, k=k, n_chunks=n_chunks, length=7 * 4000)
        assert (r["final"], r["count"]) == seq.run(d, data, 7 * 4000)
        rates.append(1 - r["reexec"] / (n_chunks - 1))
    for k, rate in zip((1, 2, 4, 7), rates):
        assert abs(rate - k / 7) < 0.06, (k, rate)
    assert rates[-1] == 1.0


def test_html_tokenizer_structure_and_snippets(golden):
    d = dfas.html_tokenizer()
    assert d.n_states == 38 and d.alphabet == 256          # PAPER.md:269 (38 states)
    assert (d.table[:, 0x80:] == d.table[:, [ord("g")]]).all()   # bytes >= 0x80 act as letters (A17)
    for case in golden["html_snippets"]["cases"]:
        q, n = seq.run(d, np.frombuffer(case["html"].encode(), np.uint8))
        assert (dfas.HTML_STATES[q], n) == (case["final"], case["count"]), case


def test_c_generators_round_trip():
    """Generator pins: the C Huffman encoder's complete-codeword count equals the decoder DFA's
    accept count (root visits); AC payload accept count equals naive multi-pattern search; HTML
    blocks are deterministic per (seed, block)."""
    w = dfas.zipf_weights(256, seed=3)
    d, codes = dfas.huffman(w.tolist())
    n_bits = 8 * 100_000 + 3
    data, nsym = streams.huffman_stream(codes, w, n_bits, seed=9)
    assert seq.run(d, data, n_bits)[1] == nsym
    pats = dfas.snort_patterns(200, seed=4)
    ad = dfas.aho_corasick(pats)
    pay = streams.ac_payload(1 << 18, 5, pats)
    text = pay.tobytes()
    ends = set()
    for p in pats:
        i = text.find(p)
        while i >= 0:
            ends.add(i + len(p))
            i = text.find(p, i + 1)
    assert seq.run(ad, pay)[1] == len(ends) > 0
    h1 = streams.html_bytes(3 << 20, 11)
    h2 = streams.html_bytes(3 << 20, 11)
    assert (h1 == h2).all() and h1[:15].tobytes() == b"<!DOCTYPE html>"
    assert seq.run(dfas.html_tokenizer(), h1)[1] > 10000
