// host_tables.h -- host preprocessing at fsm_create: validation, sink state,
// bit-mode widening, the look-back table and the per-variant device table images.
// Pure host code (no CUDA calls) so that it is usable without a GPU.
#pragma once
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <vector>

#include "speck_types.h"

namespace speck {

// The DFA as the kernels see it: 256 byte columns, internal ids (sink appended when alphabet <
// 256 in byte mode), entries next | count where count = accept increments along the step (byte
// mode: F[next]; bit mode: F-visits over the 8 MSB-first bits of the byte).
struct ByteDFA {
    uint32_t n = 0;                 // internal states
    uint32_t sink = 0xFFFFFFFFu;    // internal sink id or none
    std::vector<uint32_t> next;     // [n][256]
    std::vector<uint8_t> inc;       // [n][256] accept increments (0..8)
    std::vector<uint32_t> bittab;   // bit mode: [n][2] next | acc << 16 (tail bits)
};

inline int build_byte_dfa(const uint32_t *table, uint32_t n_states, uint32_t alphabet,
                          const uint8_t *accept, bool bit_mode, ByteDFA &d)
{
    auto acc = [&](uint32_t s) -> uint8_t { return (accept && s < n_states && accept[s]) ? 1 : 0; };
    if (!bit_mode) {
        const bool need_sink = alphabet < 256;
        d.n = n_states + (need_sink ? 1 : 0);
        d.sink = need_sink ? n_states : 0xFFFFFFFFu;
        d.next.assign((size_t)d.n * 256, 0);
        d.inc.assign((size_t)d.n * 256, 0);
        for (uint32_t s = 0; s < d.n; s++)
            for (uint32_t c = 0; c < 256; c++) {
                uint32_t t = (s == d.sink || c >= alphabet) ? d.sink : table[(size_t)s * alphabet + c];
                d.next[(size_t)s * 256 + c] = t;
                d.inc[(size_t)s * 256 + c] = acc(t);
            }
    } else {
        // widening: T8[s][byte] = delta over the 8 bits MSB-first, C8 = F-visits on the way
        d.n = n_states;
        d.next.assign((size_t)d.n * 256, 0);
        d.inc.assign((size_t)d.n * 256, 0);
        d.bittab.assign((size_t)d.n * 2, 0);
        for (uint32_t s = 0; s < d.n; s++) {
            for (uint32_t b = 0; b < 2; b++) {
                uint32_t t = table[(size_t)s * 2 + b];
                d.bittab[(size_t)s * 2 + b] = t | ((uint32_t)acc(t) << 16);
            }
            for (uint32_t c = 0; c < 256; c++) {
                uint32_t q = s, k = 0;
                for (int i = 7; i >= 0; i--) {
                    q = table[(size_t)q * 2 + ((c >> i) & 1)];
                    k += acc(q);
                }
                d.next[(size_t)s * 256 + c] = q;
                d.inc[(size_t)s * 256 + c] = (uint8_t)k;
            }
        }
    }
    return 0;
}

// Renumber the states by `order` (order[new] = old for the n_user user states; the sink, if any,
// keeps the last id): perm[old] = new, inv[new] = old.
inline void apply_order(ByteDFA &d, uint32_t n_user, const std::vector<uint32_t> &order, std::vector<uint32_t> &perm,
                        std::vector<uint32_t> &inv)
{
    perm.assign(d.n, 0);
    inv.assign(d.n, 0);
    for (uint32_t r = 0; r < n_user; r++) {
        perm[order[r]] = r;
        inv[r] = order[r];
    }
    for (uint32_t s = n_user; s < d.n; s++) perm[s] = inv[s] = s;  // the sink
    std::vector<uint32_t> nx(d.next.size());
    std::vector<uint8_t> ic(d.inc.size());
    for (uint32_t s = 0; s < d.n; s++)
        for (uint32_t c = 0; c < 256; c++) {
            nx[(size_t)perm[s] * 256 + c] = perm[d.next[(size_t)s * 256 + c]];
            ic[(size_t)perm[s] * 256 + c] = d.inc[(size_t)s * 256 + c];
        }
    d.next.swap(nx);
    d.inc.swap(ic);
}

// Static-frequency renumbering for hot-state caching (Sec. 4.2): the frequency of a state is its
// in-degree in the transition table ("the frequency of each of states a and c is 4");
// states are renumbered by decreasing frequency (ties: smaller id first) so that the hottest rows
// are the ids [0, H).  The sink (if any) keeps the last id.  perm[old] = new, inv[new] = old.
inline void renumber_by_frequency(ByteDFA &d, uint32_t n_user, std::vector<uint32_t> &perm,
                                  std::vector<uint32_t> &inv)
{
    std::vector<uint64_t> indeg(d.n, 0);
    for (uint32_t s = 0; s < n_user; s++)
        for (uint32_t c = 0; c < 256; c++) indeg[d.next[(size_t)s * 256 + c]]++;
    std::vector<uint32_t> order(n_user);
    for (uint32_t s = 0; s < n_user; s++) order[s] = s;
    std::stable_sort(order.begin(), order.end(),
                     [&](uint32_t a, uint32_t b) { return indeg[a] != indeg[b] ? indeg[a] > indeg[b] : a < b; });
    apply_order(d, n_user, order, perm, inv);
}

// Accept-partitioned renumbering (byte mode; the region-counting variants R16 / CL):
// the larger of F and Q \ F gets the ids [0, nA), the smaller one [nA, n_user), each in user order;
// the sink keeps the last id.  A step's accept increment is then a function of the destination id
// alone -- [q >= nA], or its complement when the high region is Q \ F -- which the kernels take as
// the carry of q + 2^32 - nA, so the table entries carry the bare next state.  The sink's increment
// is unspecified (a path that enters it ends in FSM_ESYMBOL).
inline void renumber_by_accept(ByteDFA &d, uint32_t n_user, const uint8_t *accept, std::vector<uint32_t> &perm,
                               std::vector<uint32_t> &inv, uint32_t &nA, bool &comp)
{
    std::vector<uint32_t> fin, non;
    for (uint32_t s = 0; s < n_user; s++) ((accept && accept[s]) ? fin : non).push_back(s);
    comp = fin.size() > non.size();
    const std::vector<uint32_t> &lo = comp ? fin : non, &hi = comp ? non : fin;
    nA = (uint32_t)lo.size();
    std::vector<uint32_t> order(lo);
    order.insert(order.end(), hi.begin(), hi.end());
    apply_order(d, n_user, order, perm, inv);
}


// HS image: the first `hot` rows as u16 entries next | count << 15 (byte mode, N <= 32768).
inline std::vector<uint8_t> image_hs(const ByteDFA &d, uint32_t hot)
{
    std::vector<uint8_t> img((size_t)hot * 512);
    uint16_t *p = reinterpret_cast<uint16_t *>(img.data());
    for (size_t i = 0; i < (size_t)hot * 256; i++) p[i] = (uint16_t)(d.next[i] | ((uint32_t)d.inc[i] << 15));
    return img;
}

// Byte classes: bytes whose columns are identical (same next state and count for every state).
inline uint32_t byte_classes(const ByteDFA &d, std::vector<uint32_t> &cls, std::vector<uint32_t> &rep)
{
    cls.assign(256, 0);
    rep.clear();
    for (uint32_t c = 0; c < 256; c++) {
        uint32_t found = 0xFFFFFFFFu;
        for (uint32_t k = 0; k < rep.size() && found == 0xFFFFFFFFu; k++) {
            const uint32_t r = rep[k];
            bool same = true;
            for (uint32_t s = 0; s < d.n && same; s++)
                same = d.next[(size_t)s * 256 + c] == d.next[(size_t)s * 256 + r] &&
                       d.inc[(size_t)s * 256 + c] == d.inc[(size_t)s * 256 + r];
            if (same) found = k;
        }
        if (found == 0xFFFFFFFFu) {
            found = (uint32_t)rep.size();
            rep.push_back(c);
        }
        cls[c] = found;
    }
    return (uint32_t)rep.size();
}

// CL image (byte mode, accept-partitioned ids): u32 [256] class id per byte, then per state s and
// slot q < nslot = ceil(ncls / 2) one u32 holding the u16 entries of classes 2q, 2q + 1: R(next) =
// 0x400 + next * nslot * 128, the shared address of the next state's row (speck_kernel.cuh TableCL;
// the kernel checks that dynamic shared memory starts at 0x400).  A padding class is never indexed.
inline uint32_t cl_slots(uint32_t ncls) { return (ncls + 1) >> 1; }
inline std::vector<uint8_t> image_cl(const ByteDFA &d, const std::vector<uint32_t> &cls,
                                     const std::vector<uint32_t> &rep)
{
    const uint32_t nslot = cl_slots((uint32_t)rep.size()), rb = nslot * 128;
    std::vector<uint8_t> img((256 + (size_t)d.n * nslot) * 4);
    uint32_t *p = reinterpret_cast<uint32_t *>(img.data());
    for (uint32_t c = 0; c < 256; c++) p[c] = cls[c];
    for (uint32_t s = 0; s < d.n; s++)
        for (uint32_t q = 0; q < nslot; q++) {
            uint32_t w = 0;
            for (uint32_t h = 0; h < 2; h++) {
                const uint32_t x = 2 * q + h;
                if (x >= rep.size()) continue;
                w |= (0x400u + d.next[(size_t)s * 256 + rep[x]] * rb) << (16 * h);
            }
            p[256 + (size_t)s * nslot + q] = w;
        }
    return img;
}

// Look-back table (reading A5): image of each byte ranked by preimage count, ties -> smaller id.
// The internal sink is not a source: it is only ever entered through an out-of-alphabet byte,
// whose image is then exactly {sink}.
inline void build_lookback(const ByteDFA &d, uint16_t *lb, uint8_t *nimg)
{
    std::vector<uint32_t> pre(d.n);
    std::vector<uint32_t> ids;
    for (uint32_t c = 0; c < 256; c++) {
        std::fill(pre.begin(), pre.end(), 0u);
        for (uint32_t s = 0; s < d.n; s++)
            if (s != d.sink) pre[d.next[(size_t)s * 256 + c]]++;
        ids.clear();
        for (uint32_t q = 0; q < d.n; q++)
            if (pre[q]) ids.push_back(q);
        std::stable_sort(ids.begin(), ids.end(), [&](uint32_t a, uint32_t b) {
            return pre[a] != pre[b] ? pre[a] > pre[b] : a < b;
        });
        uint32_t m = (uint32_t)std::min<size_t>(ids.size(), KMAX);
        nimg[c] = (uint8_t)m;
        for (uint32_t i = 0; i < KMAX; i++) lb[c * KMAX + i] = i < m ? (uint16_t)ids[i] : (uint16_t)0xFFFF;
    }
}

// Variant images (layouts documented in speck_kernel.cuh / DESIGN.md).
// P8: field = next | count << 4 (count 0..8).  P4 (byte mode only): field = next | (4 + count) << 4
// with count 0/1, so the high nibble selects byte 0 or 1 of PRMT's constant operand (speck_kernel.cuh).
inline std::vector<uint8_t> image_packed(const ByteDFA &d, bool wide)
{
    const uint32_t bytes = wide ? 8 : 4;
    std::vector<uint8_t> img(256 * bytes, wide ? 0 : 0x40);
    for (uint32_t c = 0; c < 256; c++)
        for (uint32_t s = 0; s < d.n; s++) {
            const uint32_t nx = d.next[(size_t)s * 256 + c], k = d.inc[(size_t)s * 256 + c];
            img[c * bytes + s] = (uint8_t)(wide ? (nx | (k << 4)) : (nx | ((4 + k) << 4)));
        }
    return img;
}

// N8 (byte mode, N <= 8): per symbol one u32 row of 4-bit fields, field s = next | count << 3.
inline std::vector<uint8_t> image_n8(const ByteDFA &d)
{
    std::vector<uint8_t> img(256 * 4, 0);
    uint32_t *p = reinterpret_cast<uint32_t *>(img.data());
    for (uint32_t c = 0; c < 256; c++)
        for (uint32_t s = 0; s < d.n; s++) {
            const uint32_t nx = d.next[(size_t)s * 256 + c], k = d.inc[(size_t)s * 256 + c];
            p[c] |= (nx | (k << 3)) << (4 * s);
        }
    return img;
}

// R16 (N <= 16, byte mode): byte entries E[s][c] = next (accept-partitioned ids: the count is the
// kernel's region test), row-major (the kernel lane-replicates each u32 of four entries).
inline std::vector<uint8_t> image_r16(const ByteDFA &d)
{
    std::vector<uint8_t> img((size_t)d.n * 256);
    for (size_t i = 0; i < (size_t)d.n * 256; i++) img[i] = (uint8_t)d.next[i];
    return img;
}

inline std::vector<uint8_t> image_b(const ByteDFA &d)
{
    std::vector<uint8_t> img((size_t)d.n * 512);
    uint16_t *p = reinterpret_cast<uint16_t *>(img.data());
    for (size_t i = 0; i < (size_t)d.n * 256; i++) p[i] = (uint16_t)(d.next[i] | ((uint32_t)d.inc[i] << 8));
    return img;
}

inline std::vector<uint8_t> image_g(const ByteDFA &d)
{
    std::vector<uint8_t> img((size_t)d.n * 1024);
    uint32_t *p = reinterpret_cast<uint32_t *>(img.data());
    for (size_t i = 0; i < (size_t)d.n * 256; i++) p[i] = d.next[i] | ((uint32_t)d.inc[i] << 16);
    return img;
}

}  // namespace speck
