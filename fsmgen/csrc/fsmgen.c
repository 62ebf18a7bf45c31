/* fsmgen.c -- seeded, counter-based synthetic input generator (host side).
 *
 * This is a WORKLOAD generator shared by the oracle side and the product side.
 * It holds none of the spec-k method's arithmetic: it only produces bytes.
 *
 * Stream definition:
 *   word(seed, i) = mix64(seed + (i + 1) * GOLDEN)          (SplitMix64 finaliser)
 *   byte j of the stream = byte (j mod 8) of word(seed, j / 8), little-endian.
 * The device twin lives in fsmgen_dev.cu and implements the same formula.
 */
#include <stdint.h>
#include <string.h>

#define GOLDEN 0x9E3779B97F4A7C15ULL

static inline uint64_t mix64(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

uint64_t fsmgen_word(uint64_t seed, uint64_t i) { return mix64(seed + (i + 1) * GOLDEN); }

/* Fill out[0..len) with stream bytes [offset, offset + len). */
void fsmgen_fill(uint8_t *out, uint64_t seed, uint64_t offset, uint64_t len)
{
    uint64_t j = offset, end = offset + len;
    /* head: up to the next word boundary */
    while (j < end && (j & 7)) {
        uint64_t w = fsmgen_word(seed, j >> 3);
        *out++ = (uint8_t)(w >> (8 * (j & 7)));
        j++;
    }
    while (j + 8 <= end) {
        uint64_t w = fsmgen_word(seed, j >> 3);
        memcpy(out, &w, 8); /* little-endian host */
        out += 8;
        j += 8;
    }
    while (j < end) {
        uint64_t w = fsmgen_word(seed, j >> 3);
        *out++ = (uint8_t)(w >> (8 * (j & 7)));
        j++;
    }
}

/* ------------------------------------------------------------------ structured generators ---
 * Block-seeded: block b draws from the SplitMix64 sequence started at word(seed, b); blocks are
 * independent so Python can generate them on all cores.  Workload generators only. */
typedef struct { uint64_t s; } rng_t;
static inline uint64_t rng_next(rng_t *r) { return mix64(r->s += GOLDEN); }
static inline uint32_t rng_below(rng_t *r, uint32_t n) { return (uint32_t)(((rng_next(r) >> 32) * (uint64_t)n) >> 32); }
static inline double rng_unit(rng_t *r) { return (double)(rng_next(r) >> 11) * (1.0 / 9007199254740992.0); }

typedef struct { uint8_t *p; uint64_t n, cap; } sink_t;
static inline void put(sink_t *o, const char *s)
{
    while (*s && o->n < o->cap) o->p[o->n++] = (uint8_t)*s++;
}
static inline void putc_(sink_t *o, char c)
{
    if (o->n < o->cap) o->p[o->n++] = (uint8_t)c;
}

static const char *kTags[40] = {"div", "p", "span", "a", "ul", "li", "h1", "h2", "h3", "table", "tr", "td",
    "img", "br", "em", "strong", "b", "i", "code", "pre", "section", "article", "header", "footer", "nav",
    "main", "form", "input", "button", "label", "select", "option", "small", "sup", "sub", "blockquote",
    "figure", "caption", "dl", "dd"};
static const char *kAttrs[10] = {"class", "id", "href", "src", "title", "alt", "style", "name", "type", "value"};
static const char *kEnt[6] = {"&amp;", "&lt;", "&gt;", "&#65;", "&#x41;", "&nbsp;"};

static void word(sink_t *o, rng_t *r)
{
    uint32_t len = 1 + rng_below(r, 9);
    for (uint32_t i = 0; i < len; i++) putc_(o, (char)('a' + rng_below(r, 26)));
}

static void text_run(sink_t *o, rng_t *r)
{
    uint32_t nw = 1 + rng_below(r, 12);
    for (uint32_t w = 0; w < nw; w++) {
        if (w) putc_(o, ' ');
        if (rng_unit(r) < 0.01) put(o, kEnt[rng_below(r, 6)]);
        else word(o, r);
    }
}

static void element(sink_t *o, rng_t *r, int depth)
{
    if (o->n >= o->cap) return;
    double u = rng_unit(r);
    if (u < 0.03) {  /* comment */
        put(o, "<!-- ");
        text_run(o, r);
        put(o, " -->");
        return;
    }
    if (u < 0.35) { text_run(o, r); return; }
    const char *tag = kTags[rng_below(r, 40)];
    putc_(o, '<');
    put(o, tag);
    uint32_t na = rng_below(r, 5);
    for (uint32_t a = 0; a < na; a++) {
        putc_(o, ' ');
        put(o, kAttrs[rng_below(r, 10)]);
        putc_(o, '=');
        double q = rng_unit(r);
        char qc = q < 0.7 ? '"' : (q < 0.9 ? '\'' : 0);
        if (qc) putc_(o, qc);
        uint32_t nw = qc ? 1 + rng_below(r, 3) : 1;
        for (uint32_t w = 0; w < nw; w++) {
            if (w) putc_(o, ' ');
            word(o, r);
        }
        if (qc) putc_(o, qc);
    }
    if (!strcmp(tag, "img") || !strcmp(tag, "br") || !strcmp(tag, "input")) {
        put(o, rng_unit(r) < 0.5 ? "/>" : ">");
        return;
    }
    putc_(o, '>');
    uint32_t nkids = depth >= 8 ? 0 : rng_below(r, 5);
    for (uint32_t k = 0; k < nkids && o->n < o->cap; k++) element(o, r, depth + 1);
    if (nkids == 0) text_run(o, r);
    put(o, "</");
    put(o, tag);
    putc_(o, '>');
}

/* C4: synthetic HTML documents, exactly n bytes for block `block`. */
void fsmgen_html_block(uint8_t *out, uint64_t n, uint64_t seed, uint64_t block)
{
    rng_t r = {fsmgen_word(seed, block)};
    sink_t o = {out, 0, n};
    while (o.n < n) {
        put(&o, "<!DOCTYPE html>\n<html><head><title>");
        text_run(&o, &r);
        put(&o, "</title></head><body>\n");
        uint32_t ne = 4 + rng_below(&r, 20);
        for (uint32_t e = 0; e < ne && o.n < n; e++) {
            element(&o, &r, 1);
            putc_(&o, '\n');
        }
        put(&o, "</body></html>\n");
    }
}

/* C3: packet payloads (U[64,1500] bytes each, no headers): bytes 75 % from the content set,
 * 25 % uniform; at each position a random pattern is planted with probability 1e-3. */
void fsmgen_ac_block(uint8_t *out, uint64_t n, uint64_t seed, uint64_t block, const uint8_t *pats,
                     const uint32_t *offs, uint32_t npats)
{
    static const char content[] = "abcdefghijklmnopqrstuvwxyzABCDEFGHIJKLMNOPQRSTUVWXYZ0123456789/.:=?&%-_ ";
    const uint32_t nc = (uint32_t)(sizeof(content) - 1);
    rng_t r = {fsmgen_word(seed, block)};
    uint64_t i = 0;
    while (i < n) {
        uint64_t plen = 64 + rng_below(&r, 1437);
        for (uint64_t k = 0; k < plen && i < n; k++, i++) {
            uint64_t z = rng_next(&r);
            out[i] = (z & 3) ? (uint8_t)content[((z >> 8) & 0xFFFFFFFF) % nc] : (uint8_t)(z >> 40);
        }
    }
    if (npats) {
        for (i = 0; i < n; i++) {
            if ((rng_next(&r) >> 11) % 1000 == 0) {
                uint32_t q = rng_below(&r, npats);
                uint32_t a = offs[q], b = offs[q + 1];
                for (uint32_t t = a; t < b && i + (t - a) < n; t++) out[i + (t - a)] = pats[t];
            }
        }
    }
}

/* C2: i.i.d. symbols by the alias method (prob scaled to 2^32, alias index), Huffman-encoded
 * MSB-first into out (zeroed by the caller), stopping at exactly n_bits bits.  Returns the
 * number of symbols whose codeword is complete. */
uint64_t fsmgen_huffman(uint8_t *out, uint64_t n_bits, uint64_t seed, const uint32_t *prob,
                        const uint32_t *alias, uint32_t nsym, const uint32_t *code, const uint8_t *clen)
{
    uint64_t bit = 0, complete = 0, block = 0, in_block = 0, acc = 0;
    uint32_t nacc = 0;  /* bits pending in acc (< 8 after each flush) */
    uint64_t byte = 0;
    rng_t r = {fsmgen_word(seed, 0)};
    while (bit < n_bits) {
        if (in_block == (1u << 20)) {
            r.s = fsmgen_word(seed, ++block);
            in_block = 0;
        }
        in_block++;
        uint64_t z = rng_next(&r);
        uint32_t col = (uint32_t)(((z >> 32) * (uint64_t)nsym) >> 32);
        uint32_t sym = ((uint32_t)z < prob[col]) ? col : alias[col];
        uint32_t l = clen[sym];
        uint64_t c = code[sym];
        if (bit + l > n_bits) { /* truncated codeword: keep its first bits */
            uint32_t keep = (uint32_t)(n_bits - bit);
            c >>= (l - keep);
            l = keep;
        } else {
            complete++;
        }
        acc = (acc << l) | c;
        nacc += l;
        bit += l;
        while (nacc >= 8) {
            out[byte++] = (uint8_t)(acc >> (nacc - 8));
            nacc -= 8;
        }
        acc &= (1ull << nacc) - 1ull;
    }
    if (nacc) out[byte] = (uint8_t)(acc << (8 - nacc));
    return complete;
}
