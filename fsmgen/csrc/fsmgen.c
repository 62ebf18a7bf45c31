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
