"""Seeded DFA constructions for the workloads.

A DFA is (Q, Sigma, q0, delta, F) (Sec. 2.1).  ``table`` is state-major,
``table[s, c] = delta(s, c)`` (Fig. 1b rows are states; reading A3).
These are workload definitions, not the spec-k method: both the oracle side and the CUDA side
receive the same table as an input.
"""
from __future__ import annotations

import dataclasses
import heapq

import numpy as np

from . import streams


@dataclasses.dataclass
class DFA:
    table: np.ndarray          # (N, A) uint32, state-major
    start: int
    accept: np.ndarray         # (N,) uint8 mask, nonzero = accepting
    bit_mode: bool = False     # input packs 8 MSB-first binary symbols per byte (A13)
    name: str = ""

    @property
    def n_states(self) -> int:
        return int(self.table.shape[0])

    @property
    def alphabet(self) -> int:
        return int(self.table.shape[1])


# ---------------------------------------------------------------------------------------------
# W1: the C-comment FSM of Fig. 1 (table reconstructed in SURVEY.md 8.c.2, reading A1/A2)
A, B, C, D = 0, 1, 2, 3
CC_SYMBOLS = {ord("/"): 0, ord("*"): 1}  # every other byte is 'x' (symbol 2)
_CC3 = np.array([
    #  '/' '*'  x
    [B, A, A],   # a (q0)
    [B, C, A],   # b
    [C, D, C],   # c
    [A, D, C],   # d
], dtype=np.uint32)


def c_comment(expanded: bool = True) -> DFA:
    """Fig. 1 C-comment FSM, F = {a} (A2).  expanded=True gives the 256-column byte table
    ('/' = 0x2F, '*' = 0x2A, every other byte = x); otherwise the 3-symbol table."""
    acc = np.array([1, 0, 0, 0], dtype=np.uint8)
    if not expanded:
        return DFA(_CC3.copy(), A, acc, False, "c_comment3")
    t = np.repeat(_CC3[:, 2:3], 256, axis=1)
    t[:, ord("/")] = _CC3[:, 0]
    t[:, ord("*")] = _CC3[:, 1]
    return DFA(np.ascontiguousarray(t), A, acc, False, "c_comment")


def cc_encode(text: bytes) -> np.ndarray:
    """Map text to the 3-symbol alphabet of the unexpanded C-comment table."""
    return np.array([CC_SYMBOLS.get(b, 2) for b in text], dtype=np.uint8)


# ---------------------------------------------------------------------------------------------
# W6: Div7: s' = (2 s + b) mod 7, q0 = 0, F = {0}, bit alphabet
def div7() -> DFA:
    t = np.array([[(2 * s + b) % 7 for b in (0, 1)] for s in range(7)], dtype=np.uint32)
    acc = np.zeros(7, np.uint8)
    acc[0] = 1
    return DFA(t, 0, acc, True, "div7")


# ---------------------------------------------------------------------------------------------
# W2: Huffman decoder (construction rules = reading A16)
def huffman(weights: list[int]) -> tuple[DFA, list[str]]:
    """Decoder DFA over bits for integer symbol ``weights`` (leaf ids 0..n-1).

    Tree: min-heap on (weight, node id); the first pop becomes the bit-0 child.  States are the
    internal nodes: root = 0, the others numbered in descending creation order.  On bit b an
    internal node moves to its b-child; reaching a leaf emits the symbol and returns to the root.
    F = {root}, so the accept count = number of complete codewords (decoded symbols)."""
    n = len(weights)
    assert n >= 2
    heap = [(int(w), i) for i, w in enumerate(weights)]
    heapq.heapify(heap)
    children: dict[int, tuple[int, int]] = {}
    nxt = n
    while len(heap) > 1:
        w0, c0 = heapq.heappop(heap)
        w1, c1 = heapq.heappop(heap)
        children[nxt] = (c0, c1)
        heapq.heappush(heap, (w0 + w1, nxt))
        nxt += 1
    root = heap[0][1]
    internal = sorted(children, reverse=True)  # descending creation order; root is the last made
    assert internal[0] == root
    sid = {node: i for i, node in enumerate(internal)}
    table = np.zeros((len(internal), 2), dtype=np.uint32)
    for node, (c0, c1) in children.items():
        for b, ch in enumerate((c0, c1)):
            table[sid[node], b] = 0 if ch < n else sid[ch]
    codes = [""] * n

    def walk(node: int, prefix: str) -> None:
        if node < n:
            codes[node] = prefix
            return
        c0, c1 = children[node]
        walk(c0, prefix + "0")
        walk(c1, prefix + "1")

    walk(root, "")
    acc = np.zeros(len(internal), np.uint8)
    acc[0] = 1
    return DFA(table, 0, acc, True, f"huffman{len(internal)}"), codes


def zipf_weights(n_symbols: int, seed: int, s: float = 1.0) -> np.ndarray:
    """C2 source: p_i proportional to 1/rank^s over n_symbols, ranks permuted by the seed.
    Returned as integer weights (deterministic heap ties)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    ranks = rng.permutation(n_symbols) + 1
    w = np.floor((2.0 ** 40) / ranks.astype(np.float64) ** s).astype(np.int64)
    return w


# ---------------------------------------------------------------------------------------------
# W7: Aho-Corasick "Snort-style" DFA
def aho_corasick(patterns: list[bytes]) -> DFA:
    """Full 256-column DFA of the Aho-Corasick automaton; F = nodes with a non-empty output set
    (including outputs inherited through failure links); q0 = root = 0."""
    goto: list[dict[int, int]] = [{}]
    out = [False]
    for p in patterns:
        s = 0
        for ch in p:
            if ch not in goto[s]:
                goto.append({})
                out.append(False)
                goto[s][ch] = len(goto) - 1
            s = goto[s][ch]
        out[s] = True
    n = len(goto)
    fail = [0] * n
    table = np.zeros((n, 256), dtype=np.uint32)
    order = []
    for ch in range(256):
        t = goto[0].get(ch, 0)
        table[0, ch] = t
        if t:
            fail[t] = 0
            order.append(t)
    i = 0
    while i < len(order):
        s = order[i]
        i += 1
        out[s] = out[s] or out[fail[s]]
        for ch in range(256):
            t = goto[s].get(ch)
            if t is None:
                table[s, ch] = table[fail[s], ch]
            else:
                table[s, ch] = t
                fail[t] = int(table[fail[s], ch])
                order.append(t)
    acc = np.array(out, dtype=np.uint8)
    return DFA(table, 0, acc, False, f"aho_corasick{n}")


def snort_patterns(min_states: int, seed: int) -> list[bytes]:
    """Random patterns (length U[4,32], 80 % bytes from a 72-char printable set, 20 % uniform),
    added until the trie has >= min_states nodes."""
    rng = np.random.Generator(np.random.PCG64(seed))
    content = np.frombuffer(b"abcdefghijklmnopqrstuvwxyzABCDEFGHIJKLMNOPQRSTUVWXYZ0123456789"
                            b"/.:=?&%-_ ", dtype=np.uint8)
    pats: list[bytes] = []
    nodes: set[bytes] = {b""}
    while len(nodes) < min_states:
        L = int(rng.integers(4, 33))
        pick = rng.random(L) < 0.8
        b = np.where(pick, content[rng.integers(0, content.size, L)], rng.integers(0, 256, L))
        p = bytes(b.astype(np.uint8))
        pats.append(p)
        for i in range(1, L + 1):
            nodes.add(p[:i])
    return pats


# ---------------------------------------------------------------------------------------------
# W8: random (N, m) DFA with |image(c)| = m exactly for every byte c (config C5)
def random_dfa(n_states: int, m: int, seed: int, alphabet: int = 256) -> DFA:
    assert 1 <= m <= n_states
    rng = np.random.Generator(np.random.PCG64(seed))
    t = np.zeros((n_states, alphabet), dtype=np.uint32)
    for c in range(alphabet):
        img = rng.choice(n_states, size=m, replace=False)
        perm = rng.permutation(n_states)
        col = np.empty(n_states, dtype=np.uint32)
        col[perm[:m]] = img
        if n_states > m:
            col[perm[m:]] = img[rng.integers(0, m, n_states - m)]
        t[:, c] = col
    acc = np.array([streams.word(seed, s) % 4 == 0 for s in range(n_states)], dtype=np.uint8)
    return DFA(t, 0, acc, False, f"random_{n_states}_{m}")


# ---------------------------------------------------------------------------------------------
# W5: HTML tokenizer with exactly 38 states (PAPER.md:269 gives only "38 states, 128 inputs"; the
# FSM itself is our construction, reading A17).  Simplified WHATWG tokenizer; bytes >= 0x80 behave
# as letters.  Accepting states are the token-complete "emit" states, so the accept count is the
# number of tokens: tags, comments, declarations, character references and text runs (a text run
# is counted by the '<' that ends it).
HTML_STATES = [
    "Data", "Text", "TextEmit", "TagOpen", "EndTagOpen", "TagName", "EndTagName", "BeforeAttrName",
    "AttrName", "AfterAttrName", "BeforeAttrValue", "AttrValueDQ", "AttrValueSQ", "AttrValueUnq",
    "AfterAttrValueQuoted", "SelfClosingStart", "TagEmit", "MarkupDeclOpen", "CommentStartDash",
    "CommentStart", "Comment", "CommentEndDash", "CommentEnd", "CommentEmit", "DocD", "DocO", "DocC",
    "DocT", "DocY", "DocP", "DocE", "DoctypeBody", "DoctypeEmit", "CharRef", "CharRefNamed",
    "CharRefNumeric", "CharRefHex", "CharRefEmit"]
HTML_ACCEPT = ("TextEmit", "TagEmit", "CommentEmit", "DoctypeEmit", "CharRefEmit")


def html_tokenizer() -> DFA:
    S = {n: i for i, n in enumerate(HTML_STATES)}
    assert len(S) == 38
    ws = set(b" \t\n\r\f")
    letters = set(range(ord("a"), ord("z") + 1)) | set(range(ord("A"), ord("Z") + 1)) | set(range(0x80, 0x100))
    digits = set(range(ord("0"), ord("9") + 1))
    hexd = digits | set(b"abcdefABCDEF")
    t = np.zeros((38, 256), dtype=np.uint32)

    def setrow(state, default, rules):
        r = t[S[state]]
        r[:] = S[default]
        for chars, dst in rules:
            for c in chars:
                r[c] = S[dst]

    lt, gt, sl, ex, da, eq = ord("<"), ord(">"), ord("/"), ord("!"), ord("-"), ord("=")
    dq, sq, am, hs, sc = ord('"'), ord("'"), ord("&"), ord("#"), ord(";")
    data_rules = [([lt], "TagOpen"), ([am], "CharRef")]
    for st in ("Data", "TagEmit", "CommentEmit", "DoctypeEmit", "CharRefEmit"):
        setrow(st, "Text", data_rules)
    setrow("Text", "Text", [([lt], "TextEmit"), ([am], "CharRef")])
    for st in ("TagOpen", "TextEmit"):
        setrow(st, "Text", [(letters, "TagName"), ([sl], "EndTagOpen"), ([ex], "MarkupDeclOpen"), ([lt], "TagOpen")])
    setrow("EndTagOpen", "Text", [(letters, "EndTagName"), ([gt], "Data")])
    setrow("TagName", "TagName", [(ws, "BeforeAttrName"), ([sl], "SelfClosingStart"), ([gt], "TagEmit")])
    setrow("EndTagName", "EndTagName", [([gt], "TagEmit")])
    setrow("BeforeAttrName", "AttrName", [(ws, "BeforeAttrName"), ([sl], "SelfClosingStart"), ([gt], "TagEmit")])
    setrow("AttrName", "AttrName", [(ws, "AfterAttrName"), ([sl], "SelfClosingStart"), ([eq], "BeforeAttrValue"),
                                    ([gt], "TagEmit")])
    setrow("AfterAttrName", "AttrName", [(ws, "AfterAttrName"), ([sl], "SelfClosingStart"),
                                         ([eq], "BeforeAttrValue"), ([gt], "TagEmit")])
    setrow("BeforeAttrValue", "AttrValueUnq", [(ws, "BeforeAttrValue"), ([dq], "AttrValueDQ"),
                                               ([sq], "AttrValueSQ"), ([gt], "TagEmit")])
    setrow("AttrValueDQ", "AttrValueDQ", [([dq], "AfterAttrValueQuoted")])
    setrow("AttrValueSQ", "AttrValueSQ", [([sq], "AfterAttrValueQuoted")])
    setrow("AttrValueUnq", "AttrValueUnq", [(ws, "BeforeAttrName"), ([gt], "TagEmit")])
    setrow("AfterAttrValueQuoted", "AttrName", [(ws, "BeforeAttrName"), ([sl], "SelfClosingStart"), ([gt], "TagEmit")])
    setrow("SelfClosingStart", "AttrName", [([gt], "TagEmit"), (ws, "BeforeAttrName")])
    setrow("MarkupDeclOpen", "DoctypeBody", [([da], "CommentStartDash"), (b"Dd", "DocD"), ([gt], "DoctypeEmit")])
    setrow("CommentStartDash", "DoctypeBody", [([da], "CommentStart"), ([gt], "DoctypeEmit")])
    setrow("CommentStart", "Comment", [([da], "CommentEndDash"), ([gt], "CommentEmit")])
    setrow("Comment", "Comment", [([da], "CommentEndDash")])
    setrow("CommentEndDash", "Comment", [([da], "CommentEnd")])
    setrow("CommentEnd", "Comment", [([gt], "CommentEmit"), ([da], "CommentEnd")])
    for a, b, nxt in (("DocD", "Oo", "DocO"), ("DocO", "Cc", "DocC"), ("DocC", "Tt", "DocT"),
                      ("DocT", "Yy", "DocY"), ("DocY", "Pp", "DocP"), ("DocP", "Ee", "DocE")):
        setrow(a, "DoctypeBody", [(b.encode(), nxt), ([gt], "DoctypeEmit")])
    setrow("DocE", "DoctypeBody", [([gt], "DoctypeEmit")])
    setrow("DoctypeBody", "DoctypeBody", [([gt], "DoctypeEmit")])
    setrow("CharRef", "Text", [([hs], "CharRefNumeric"), (letters, "CharRefNamed"), ([lt], "TagOpen")])
    setrow("CharRefNamed", "Text", [(letters | digits, "CharRefNamed"), ([sc], "CharRefEmit"), ([lt], "TagOpen")])
    setrow("CharRefNumeric", "Text", [(b"xX", "CharRefHex"), (digits, "CharRefNumeric"), ([sc], "CharRefEmit"),
                                      ([lt], "TagOpen")])
    setrow("CharRefHex", "Text", [(hexd, "CharRefHex"), ([sc], "CharRefEmit"), ([lt], "TagOpen")])
    acc = np.array([1 if n in HTML_ACCEPT else 0 for n in HTML_STATES], dtype=np.uint8)
    return DFA(t, S["Data"], acc, False, "html38")
