"""Seeded synthetic input streams (workload generators; no spec-k arithmetic).

Recipes:
* ``splitmix_bytes``  -- C5: i.i.d. uniform bytes, byte j = byte (j mod 8) of
  mix64(seed + (j//8 + 1) * GOLDEN).  Counter-based: any range can be generated independently,
  on the host (fsmgen.c) or in place in HBM (fsmgen_dev.cu).
* ``c_source``        -- C1: synthetic C-like text with /* ... */ block comments (~20 % of bytes).
* ``random_bits``     -- Div7 test input: i.i.d. bits packed MSB-first.
* ``huffman_bits``    -- C2: i.i.d. symbols from a distribution, Huffman-encoded MSB-first.
Structured generators are block-seeded: block b uses a PCG64 stream seeded with word(seed, b).
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _native

MASTER_SEED = 20200222  # config seed = master + config index
GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)
BLOCK = 1 << 20


def _mix64(z: np.ndarray) -> np.ndarray:
    z = (z ^ (z >> np.uint64(30))) * _C1
    z = (z ^ (z >> np.uint64(27))) * _C2
    return z ^ (z >> np.uint64(31))


def splitmix_words(seed: int, start: int, n: int) -> np.ndarray:
    """Pure-numpy words [start, start+n) of the counter-based stream (reference for the C twin)."""
    with np.errstate(over="ignore"):
        i = np.arange(start, start + n, dtype=np.uint64)
        return _mix64(np.uint64(seed) + (i + np.uint64(1)) * GOLDEN)


def word(seed: int, i: int) -> int:
    return int(_native.host_lib().fsmgen_word(seed & (2**64 - 1), i))


def splitmix_bytes(seed: int, offset: int, length: int, out: np.ndarray | None = None) -> np.ndarray:
    """Stream bytes [offset, offset+length) as a uint8 array (host C fill)."""
    if out is None:
        out = np.empty(length, dtype=np.uint8)
    assert out.dtype == np.uint8 and out.size >= length and out.flags.c_contiguous
    if length:
        _native.host_lib().fsmgen_fill(out.ctypes.data, seed & (2**64 - 1), offset, length)
    return out[:length]


def splitmix_fill_device(ptr: int, seed: int, offset: int, length: int, stream: int = 0) -> None:
    """Fill device memory at ``ptr`` with stream bytes [offset, offset+length) (fsmgen_dev.cu)."""
    rc = _native.dev_lib().fsmgen_dev_fill(ctypes.c_void_p(ptr), seed & (2**64 - 1), offset, length,
                                           ctypes.c_void_p(stream))
    if rc != 0:
        raise RuntimeError(f"fsmgen_dev_fill failed ({rc})")


def _block_rng(seed: int, block: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(word(seed, block)))


def random_bits(n_bits: int, seed: int) -> np.ndarray:
    """Div7 input: n_bits i.i.d. bits, MSB-first in ceil(n_bits/8) bytes; pad bits are zero."""
    nbytes = (n_bits + 7) // 8
    data = splitmix_bytes(seed, 0, nbytes).copy()
    if n_bits % 8:
        data[-1] &= np.uint8((0xFF << (8 - n_bits % 8)) & 0xFF)
    return data


# ----------------------------------------------------------------------------------------------
# C1: synthetic C source with block comments
_IDENT = np.frombuffer(b"abcdefghijklmnopqrstuvwxyz_", dtype=np.uint8)
_DIGIT = np.frombuffer(b"0123456789", dtype=np.uint8)
_OPS = [b"+", b"-", b"=", b";", b"(", b")", b"{", b"}", b",", b"<", b">", b"&", b"|", b"!",
        b"[", b"]", b"*", b"/", b"==", b"->", b"++", b" * ", b" / "]
_BODY = np.frombuffer(b"abcdefghijklmnopqrstuvwxyz     ,.:*/-=", dtype=np.uint8)


def _comment(rng: np.random.Generator) -> bytes:
    n = int(rng.integers(4, 160))
    body = bytearray(_BODY[rng.integers(0, _BODY.size, n)].tobytes())
    # no early terminator inside the body: a '*' is never followed by '/'
    for i in range(len(body) - 1):
        if body[i] == 0x2A and body[i + 1] == 0x2F:
            body[i + 1] = 0x20
    return b"/*" + bytes(body) + b"*/"


def _c_block(rng: np.random.Generator, n: int, comment_frac: float) -> bytes:
    out: list[bytes] = []
    size = 0
    # a comment is ~84 bytes on average and a token ~5: choose the rate so ~comment_frac of
    # the bytes lie inside comments
    p_comment = comment_frac * 5.0 / (84.0 * (1 - comment_frac) + comment_frac * 5.0)
    while size < n:
        r = rng.random()
        if r < p_comment:
            t = _comment(rng)
        elif r < 0.45:
            t = _IDENT[rng.integers(0, _IDENT.size, int(rng.integers(1, 10)))].tobytes()
        elif r < 0.55:
            t = _DIGIT[rng.integers(0, 10, int(rng.integers(1, 5)))].tobytes()
        elif r < 0.80:
            t = _OPS[int(rng.integers(0, len(_OPS)))]
        elif r < 0.93:
            t = b" "
        else:
            t = b"\n" + b"    " * int(rng.integers(0, 3))
        out.append(t)
        size += len(t)
    return b"".join(out)[:n]


def c_source(nbytes: int, seed: int, comment_frac: float = 0.2) -> np.ndarray:
    """C1 input: block-seeded synthetic C text of exactly ``nbytes`` bytes."""
    blocks = []
    for b in range((nbytes + BLOCK - 1) // BLOCK):
        n = min(BLOCK, nbytes - b * BLOCK)
        blocks.append(_c_block(_block_rng(seed, b), n, comment_frac))
    return np.frombuffer(b"".join(blocks), dtype=np.uint8).copy()


# ----------------------------------------------------------------------------------------------
# C2: Huffman-encoded bitstream
def huffman_bits(codes: list[str], probs: np.ndarray, n_bits: int, seed: int) -> tuple[np.ndarray, int]:
    """Encode i.i.d. symbols drawn from ``probs`` with ``codes`` (MSB-first), truncated at exactly
    ``n_bits`` bits.  Returns (packed bytes, number of symbols whose code is complete)."""
    lens = np.array([len(c) for c in codes], dtype=np.int64)
    vals = np.array([int(c, 2) for c in codes], dtype=np.uint64)
    mean = float((probs * lens).sum())
    out_bits = []
    total = 0
    complete = 0
    b = 0
    while total < n_bits:
        rng = _block_rng(seed, b)
        nsym = int((n_bits - total) / mean * 1.05) + 64
        nsym = min(nsym, 1 << 22)
        syms = rng.choice(len(codes), size=nsym, p=probs)
        l = lens[syms]
        v = vals[syms]
        # expand each code to bits, MSB first
        maxl = int(l.max())
        shifts = np.arange(maxl - 1, -1, -1, dtype=np.uint64)
        mat = ((v[:, None] >> shifts[None, :]) & np.uint64(1)).astype(np.uint8)
        keep = np.arange(maxl)[None, :] >= (maxl - l)[:, None]
        bits = mat[keep]
        room = n_bits - total
        if bits.size > room:
            ends = np.cumsum(l)
            complete += int(np.searchsorted(ends, room, side="right"))
            bits = bits[:room]
        else:
            complete += nsym
        out_bits.append(bits)
        total += bits.size
        b += 1
    allbits = np.concatenate(out_bits) if out_bits else np.zeros(0, np.uint8)
    return np.packbits(allbits), complete


# ----------------------------------------------------------------------------------------------
# Large structured inputs through the C generators (block-seeded, generated on all host cores)
def _blocks_parallel(fn, n: int, out: np.ndarray | None = None) -> np.ndarray:
    import concurrent.futures as cf
    import os

    if out is None:
        out = np.empty(n, dtype=np.uint8)
    nb = (n + BLOCK - 1) // BLOCK
    with cf.ThreadPoolExecutor(os.cpu_count()) as ex:
        list(ex.map(lambda b: fn(out[b * BLOCK:], min(BLOCK, n - b * BLOCK), b), range(nb)))
    return out[:n]


def html_bytes(n: int, seed: int, out: np.ndarray | None = None) -> np.ndarray:
    """C4 input: synthetic HTML documents (nested tags from a 40-tag vocabulary, depth <= 8, 0-4
    attributes with double/single/unquoted values, word text runs, ~3 % comments, ~1 % entities,
    one DOCTYPE per document), 1 MiB blocks."""
    lib = _native.host_lib()
    return _blocks_parallel(lambda o, m, b: lib.fsmgen_html_block(o.ctypes.data, m, seed, b), n, out)


def ac_payload(n: int, seed: int, patterns: list[bytes], out: np.ndarray | None = None) -> np.ndarray:
    """C3 input: packet payloads of U[64,1500] bytes, 75 % content-set bytes, 25 % uniform, a
    random pattern planted with probability 1e-3 per position, 1 MiB blocks."""
    lib = _native.host_lib()
    pats = np.frombuffer(b"".join(patterns), dtype=np.uint8).copy()
    offs = np.zeros(len(patterns) + 1, dtype=np.uint32)
    offs[1:] = np.cumsum([len(p) for p in patterns])
    return _blocks_parallel(lambda o, m, b: lib.fsmgen_ac_block(o.ctypes.data, m, seed, b, pats.ctypes.data,
                                                                offs.ctypes.data, len(patterns)), n, out)


def _alias(probs: np.ndarray):
    n = probs.size
    p = probs * n / probs.sum()
    prob = np.zeros(n, np.float64)
    alias = np.zeros(n, np.uint32)
    small = [i for i in range(n) if p[i] < 1.0]
    large = [i for i in range(n) if p[i] >= 1.0]
    while small and large:
        s, l = small.pop(), large.pop()
        prob[s] = p[s]
        alias[s] = l
        p[l] = p[l] + p[s] - 1.0
        (small if p[l] < 1.0 else large).append(l)
    for i in large + small:
        prob[i] = 1.0
        alias[i] = i
    return np.minimum(np.floor(prob * 2.0 ** 32), 2.0 ** 32 - 1).astype(np.uint32), alias


def huffman_stream(codes: list[str], weights: np.ndarray, n_bits: int, seed: int) -> tuple[np.ndarray, int]:
    """C2 input: i.i.d. symbols (alias method over ``weights``) Huffman-encoded MSB-first, cut at
    exactly n_bits bits.  Returns (packed bytes, number of complete codewords)."""
    lib = _native.host_lib()
    prob, alias = _alias(np.asarray(weights, dtype=np.float64))
    code = np.array([int(c, 2) for c in codes], dtype=np.uint32)
    clen = np.array([len(c) for c in codes], dtype=np.uint8)
    out = np.zeros((n_bits + 7) // 8 + 8, dtype=np.uint8)
    nsym = lib.fsmgen_huffman(out.ctypes.data, n_bits, seed, prob.ctypes.data, alias.ctypes.data, len(codes),
                              code.ctypes.data, clen.ctypes.data)
    return out[:(n_bits + 7) // 8], int(nsym)
