// speck_kernel.cuh -- the fused spec-k kernel for sm_100a (B200).
//
// One persistent CTA loop; each iteration takes the next tile from an atomic ticket (dynamic
// tile ids => forward progress without co-residency assumptions) and runs the whole hot path:
//
//   a2  chunking: tile = blockDim.x chunks of p.chunk bytes, one chunk per thread;
//       each thread streams its own chunk with 32-byte LDG.256 (full sectors) -- the paper's
//       coalescing layout transformation realised on the fly, see DESIGN.md.
//   a3  look-back speculation: S_j = top-k of image(x[b_j - 1]) (Alg. 3 l.3 P:207).
//   a4  local processing: k independent lookup chains per chunk (Alg. 3) plus accept
//       counts, k unrolled into registers.
//   a5  warp merge: shuffle suffix scan of chunk mappings with the membership check of Alg. 1
//       (P:121-143); an unmatched ending state marks the slot invalid (delayed re-execution,
//       P:188-190) and records where it broke.
//   a6  block merge: warp aggregates through shared memory, scanned by warp 0.
//   a8  delayed, selective re-execution: only chunks whose (candidate) start was not speculated
//       are re-executed, in lockstep with that chunk's speculated chains, stopping as soon as the
//       re-executed run joins one of them (exact early exit).
//   a7  grid merge: decoupled look-back over per-tile descriptors (replaces the paper's
//       persistent-thread sequential global merge).
//   a9  the last tile writes (final state, accept count) or the shard's k-slot mapping.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "speck_types.h"

namespace speck {

enum { VAR_P4 = 0, VAR_P8 = 1, VAR_B = 2, VAR_G = 3, /* 4: retired (H8) */ VAR_HS = 5, VAR_CL = 6, VAR_N8 = 7, VAR_R16 = 8, VAR_RG = 9 };
constexpr int kThreads = 256;  // auxiliary kernels
// Eager completion (NEXT-3): per chunk, up to kExt image states beyond the speculated ones are run
// in lockstep over the chunk's first kExtWindow bytes; entry = key | slot << 16 | (delta & 0xFFF) << 20.
constexpr int kExt = 4;
constexpr uint32_t kExtWindow = 128;  // bytes of lockstep per chunk; |count delta| <= 8 * 128 fits 12 bits
constexpr uint32_t kExtNone = 0xFFFFu;
constexpr uint32_t kHashSize = 32;
// Early-exit re-execution (R3) runs the chunk's chains in lockstep for at most this many bytes; past
// it (paths that do not meet, e.g. permutation DFAs with k < N) the re-executed path continues alone:
// K + 1 lookups per byte only where a meeting is likely, one afterwards.  Exact either way.
constexpr uint32_t kLockstepWindow = 256;  // Alg. 2 buckets per thread (reading A10: next power of two >= 2k, k <= 16)
// Threads per tile (one chunk per thread) of the fused kernel, by the number of chains K: large
// CTAs keep few tiles in flight (short look-back windows) at one CTA per SM; the register budget
// caps them for large K.
// (K = 2, 3 at 768 threads get 85 registers: the multi-chain prologue spills at 64; measured
// +6 % over 1024 threads for (8, 2, k=2).)
// B / R16 / RG at K = 4 (their chains converge within a few bytes, after which one LDS-bound chain
// per thread remains): 768 threads (80 registers) instead of 512 (128).  The shared-memory tables
// at K = 8, 12: 384 / 320 threads (164 / 168 registers, no spills) instead of 256; K = 16 keeps 256
// (at 288 threads ptxas caps it at 168 registers and spills 1.2 KB).
__host__ __device__ constexpr int max_threads(int K, int var = -1)
{
    return K == 1 ? 1024 : K <= 3 ? 768 : (K == 4 && (var == 2 || var == 8 || var == 9)) ? 768 : K <= 6 ? 512
         : ((var == 2 || var == 6 || var == 8 || var == 9) && K <= 12) ? (K <= 8 ? 384 : 320) : 256;
}
__host__ __device__ constexpr int min_blocks(int) { return 1; }
constexpr uint32_t kPackedTableBytes = 65536;  // 256 symbols x 256-byte lane-replicated rows

// ------------------------------------------------------------------------------- PTX helpers --
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(uint32_t *p, uint32_t v)
{
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

struct Bytes32 {
    uint32_t w[8];
};
// 256-bit non-coherent streaming load (SASS LDG.E.NA.ENL2.256): one full 32-byte sector per lane.
__device__ __forceinline__ Bytes32 ldg256(const uint8_t *p)
{
    Bytes32 r;
    asm volatile("ld.global.nc.L1::no_allocate.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.w[0]), "=r"(r.w[1]), "=r"(r.w[2]), "=r"(r.w[3]), "=r"(r.w[4]), "=r"(r.w[5]),
                   "=r"(r.w[6]), "=r"(r.w[7])
                 : "l"(p));
    return r;
}
// streaming load of 32-byte block i of a chunk
__device__ __forceinline__ Bytes32 ldg_block(const uint8_t *p, uint64_t i) { return ldg256(p + 32 * i); }
__device__ __forceinline__ uint4 ldg128(const uint8_t *p)
{
    return __ldg(reinterpret_cast<const uint4 *>(p));
}

// PTX prmt in its default mode: every selector nibble is used as-is.  CUDA's __byte_perm masks
// the selector with 0x7777 first (an extra LOP3 on the dependency chain); the packed variants
// keep bit 3 of the low nibble zero by construction and ignore result bytes 1-3.
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel)
{
    uint32_t d;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(sel));
    return d;
}

// FMA-pipe integer helpers (IMAD / IMAD.HI).  The hot loop is ALU-pipe bound (PRMT, LOP3,
// IADD3 all issue there); half of the accept-count work is moved to the otherwise idle FMA pipe.
__device__ __forceinline__ uint32_t mad_hi(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm("mad.hi.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
__device__ __forceinline__ uint32_t mad_lo(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}

// Shared-memory loads at a 32-bit shared-window address (the packed tables live at 0x10000 so that
// a single PRMT produces the complete address).
__device__ __forceinline__ uint32_t lds_u32(uint32_t a)
{
    uint32_t v;
    asm("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t a)
{
    uint32_t v;
    asm("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u16(uint32_t a)
{
    uint32_t v;
    asm("ld.shared.u16 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint2 lds_v2(uint32_t a)
{
    uint2 v;
    asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
// acc + [x >= T] with negT = 2^32 - T: the carry out of x + negT, added by a second add (IADD3 and
// IADD3.X, each issued on either integer pipe at full rate; measured tools/pipe_probe: IMAD.HI takes
// 4 cycles per warp per SMSP, an add 1).  The region count of R16 / RG / CL.
__device__ __forceinline__ uint32_t add_ge(uint32_t acc, uint32_t x, uint32_t negT)
{
    uint32_t d;
    asm("{\n\t.reg .u32 t;\n\tadd.cc.u32 t, %1, %2;\n\taddc.u32 %0, %3, 0;\n\t}" : "=r"(d) : "r"(x), "r"(negT), "r"(acc));
    return d;
}
__device__ __forceinline__ uint32_t dp4a_u(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm("dp4a.u32.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
constexpr uint32_t kPackedBase = 0x10000u;  // shared-window address of the packed tables
constexpr uint32_t kSmemWindowBase = 1024u;  // dynamic shared memory starts here (measured: tools/smem_probe)
__host__ __device__ constexpr bool is_packed(int var) { return var == 0 || var == 1 || var == 7; }
// CL: the entry table sits at the start of dynamic smem (shared addresses [0x400, 0x10000): its u16
// entries are shared addresses) and the lane-replicated class map at the fixed shared address
// 0x10000 with a 256-byte stride, so a class-map address is ONE PRMT of the input word
// (0x10000 | byte << 8 | lane * 4, the packed tables' form).
constexpr uint32_t kClMapBase = 0x10000u;
constexpr uint32_t kClMaxTable = kClMapBase - 1024u;  // entry-table bytes that fit below the map
// Offset (from the start of dynamic smem) of the scratch area that follows the table.  Packed
// tables and CL's class map occupy the window [0x10000, 0x20000); everything else goes above the
// table.
__host__ __device__ constexpr uint32_t scratch_offset(int var, uint32_t table_bytes)
{
    return is_packed(var) ? (kPackedBase + 65536u - kSmemWindowBase)
         : var == 6 ? (kClMapBase + 256u * 256u - kSmemWindowBase)
         : ((table_bytes + 15u) & ~15u);
}
__device__ __forceinline__ void check_smem_window(int var, uint32_t need)
{
    if (!is_packed(var) && var != 6) return;
    extern __shared__ __align__(16) uint8_t smem[];
    uint32_t dyn;
    asm("mov.u32 %0, %%dynamic_smem_size;" : "=r"(dyn));
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(smem);
    if (base != kSmemWindowBase || dyn < need) __trap();  // loud: the layout assumption does not hold
}

struct KConst {
    uint32_t k_1e24, k_16, k_512;
    const uint32_t *gtab;  // full u32 table in global memory (HS variant)
    uint32_t hot_rows;     // HS: states [0, hot_rows) have their rows in shared memory
    uint32_t ncls, cl_magic;  // CL: byte classes, ceil(2^32 / ncls)
    uint32_t k_4;             // N8
    uint32_t rc_t, rc_comp;      // region counting (R16, RG, CL; Params)
    uint32_t r_logl;             // RG: log2 of the lanes sharing a table copy
};
__device__ __forceinline__ KConst kconst(const Params &p)
{
    return KConst{p.k_1e24, p.k_16, p.k_512, p.table_g, p.hot_rows, p.ncls, p.cl_magic, p.k_4, p.rc_t, p.rc_comp, p.r_logl};
}

// ------------------------------------------------------------------- table-placement variants --
// Every variant exposes
//   setup(smem, global image, n)       copy / expand the table into shared memory (once per CTA)
//   init(s) / state_of(cur) / count_of(acc)
//   step<K>(w, j, cur, acc)            advance all K chains by byte j of word w (the hot loop)
//   row(c) / apply(row, st, cnt)       single-chain step used by re-execution
// Entries carry the accept increment of the destination state (byte mode 0/1, bit mode 0..8).

// P4/P8: the transition function of symbol c packed into one row of N <= 4 (8) byte fields.
// The row address depends only on the input byte, so it is off the dependency chain; one
// conflict-free LDS.32/LDS.64 serves all K chains, and each chain step is a single PRMT (byte
// select by the current state).  Rows are lane-replicated (lane l reads its own copy) and live at
// shared address 0x10000 + c * 256 + lane * 4|8, so the address is ONE PRMT of the input word:
// byte0 <- lane offset, byte1 <- input byte c, byte2 <- 0x01.
//  P8 field = next | count << 4 (bit mode: count 0..8).
//  P4 field = next | (4 + count) << 4 (byte mode): PRMT's second operand X = 0x4544 turns the
//     high nibble into a selector of X, so result byte 1 = 0x44 + count of the previous step and
//     one DP4A (dot with 0x100) accumulates it; the 0x44 bias is removed at the end.
template <int VAR>
struct TablePacked {
    static constexpr bool kWide = VAR == VAR_P8;
    static constexpr uint32_t kX = 0x4544u;
    uint32_t lanereg;
    __device__ __forceinline__ void setup(uint8_t *, const void *g, uint32_t, const KConst &kc)
    {
        lanereg = kPackedBase | ((threadIdx.x & 31) * (kWide ? 8 : 4));
        if (kWide) {
            const uint2 *rows = static_cast<const uint2 *>(g);
            for (uint32_t i = threadIdx.x; i < 256 * 32; i += blockDim.x) {
                const uint2 v = __ldg(rows + (i >> 5));
                asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(kPackedBase + i * 8), "r"(v.x), "r"(v.y));
            }
        } else {
            const uint32_t *rows = static_cast<const uint32_t *>(g);
            for (uint32_t i = threadIdx.x; i < 256 * 32; i += blockDim.x) {
                const uint32_t v = __ldg(rows + (i >> 5));
                asm volatile("st.shared.u32 [%0], %1;" ::"r"(kPackedBase + (i >> 5) * 256 + (i & 31) * 4), "r"(v));
            }
        }
    }
    __device__ __forceinline__ uint32_t init(uint32_t st) const { return kWide ? st : (st | 0x44444440u); }
    __device__ __forceinline__ uint32_t state_of(uint32_t cur) const { return cur & 0xFu; }
    // P8: acc = count * 16.
    // P4: acc = sum of (0x44 + lagged count) over n steps; the last step's count sits in cur.
    __device__ __forceinline__ uint32_t count_of(uint32_t acc, uint32_t accf, uint32_t cur, uint64_t n) const
    {
        if (kWide) return (acc >> 4) + accf;
        return acc - 0x44u * (uint32_t)n + ((cur >> 4) & 0xFu) - 4u;
    }

    template <int K>
    __device__ __forceinline__ void step(uint32_t w, int j, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                         uint32_t (&accf)[K]) const
    {
        const uint32_t a = prmt(w, lanereg, 0x7604u | (uint32_t(j) << 4));
        if (kWide) {
            const uint2 r = lds_v2(a);
#pragma unroll
            for (int s = 0; s < K; s++) {
                cur[s] = prmt(r.x, r.y, cur[s]);  // the chain: one PRMT per step
                acc[s] += cur[s] & 0xF0u;         // LOP3 + IADD3 (an IMAD.HI would take 4 cycles per warp)
            }
        } else {
            const uint32_t r = lds_u32(a);
#pragma unroll
            for (int s = 0; s < K; s++) {
                cur[s] = prmt(r, kX, cur[s]);
                acc[s] = dp4a_u(cur[s], 0x100u, acc[s]);
            }
        }
    }
    using Row = uint2;
    __device__ __forceinline__ Row row(uint32_t c) const
    {
        const uint32_t a = lanereg + (c << 8);
        if (kWide) return lds_v2(a);
        return make_uint2(lds_u32(a), kX);
    }
    __device__ __forceinline__ uint32_t apply(Row r, uint32_t st, uint32_t &cnt) const
    {
        const uint32_t f = prmt(r.x, r.y, st) & 0xFFu;
        cnt += kWide ? (f >> 4) : ((f >> 4) - 4u);
        return f & 0xFu;
    }
};

// N8: N <= 8, byte mode.  The transition function of symbol c is ONE 32-bit row of eight 4-bit
// fields, field s = next | count << 3, lane-replicated at 0x10000 + c * 256 + lane * 4 (P4's layout,
// so the address is one PRMT of the input word and the load is one conflict-free LDS.32 = one
// wavefront per byte per warp, half of P8's LDS.64).  A chain carries the shift amount 4 * state:
// t = funnel-shift-right(row, cur) in wrap mode (only cur & 31 is used), and the next shift amount
// is t * 4, whose bits 2..4 are t's next-state bits -- the garbage above bit 4 is ignored by the
// next wrap-mode shift.  Chain step: SHF.R.W (ALU) + IMAD (FMA); the count bit = bit 3 of t is
// summed four bytes at a time (step4).
struct TableN8 {
    uint32_t lanereg;
    uint32_t c4;
    __device__ __forceinline__ void setup(uint8_t *, const void *g, uint32_t, const KConst &kc)
    {
        lanereg = kPackedBase | ((threadIdx.x & 31) * 4);
        c4 = kc.k_4;
        const uint32_t *rows = static_cast<const uint32_t *>(g);
        for (uint32_t i = threadIdx.x; i < 256 * 32; i += blockDim.x) {
            const uint32_t v = __ldg(rows + (i >> 5));
            asm volatile("st.shared.u32 [%0], %1;" ::"r"(kPackedBase + (i >> 5) * 256 + (i & 31) * 4), "r"(v));
        }
    }
    __device__ __forceinline__ static uint32_t shr_wrap(uint32_t row, uint32_t sh)
    {
        uint32_t d;
        asm("shf.r.wrap.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(row), "r"(0u), "r"(sh));
        return d;
    }
    __device__ __forceinline__ uint32_t init(uint32_t st) const { return st * 4u; }
    __device__ __forceinline__ uint32_t state_of(uint32_t cur) const { return (cur >> 2) & 7u; }
    // accf counts in units of 32 (the DP4A of bit 5 of v in step4, and the byte tails in step); acc
    // is unused.
    __device__ __forceinline__ uint32_t count_of(uint32_t acc, uint32_t accf, uint32_t, uint64_t) const
    {
        return acc + (accf >> 5);
    }
    template <int K>
    __device__ __forceinline__ void step(uint32_t w, int j, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                         uint32_t (&accf)[K]) const
    {
        const uint32_t r = lds_u32(prmt(w, lanereg, 0x7604u | (uint32_t(j) << 4)));
#pragma unroll
        for (int s = 0; s < K; s++) {
            const uint32_t t = shr_wrap(r, cur[s]);          // field of the current state in bits 0..3
            cur[s] = mad_lo(t, c4, 0u);                      // next shift amount (bits 2..4 valid)
            accf[s] += (t & 8u) << 2;                        // byte tails of step4 chunks: units of 32
        }
    }
    // Four bytes of word w at once: the four rows are loaded up front, and the count of the four
    // steps is taken in one go -- the next shift amounts v = 4t carry the accept bit in bit 5; their
    // low bytes are gathered by two PRMTs into one word, masked, and summed by one DP4A (acc counts
    // in units of 32).  ALU: 4 address PRMT + 4 SHF + 3 PRMT + 1 LOP3; FMA: 4 IMAD + 1 DP4A.
    template <int K>
    __device__ __forceinline__ void step4(uint32_t w, uint32_t (&cur)[K], uint32_t (&acc)[K], uint32_t (&accf2)[K]) const
    {
        uint32_t r[4];
#pragma unroll
        for (int j = 0; j < 4; j++) r[j] = lds_u32(prmt(w, lanereg, 0x7604u | (uint32_t(j) << 4)));
#pragma unroll
        for (int s = 0; s < K; s++) {
            uint32_t v[4];
            uint32_t c = cur[s];
#pragma unroll
            for (int j = 0; j < 4; j++) {
                v[j] = mad_lo(shr_wrap(r[j], c), c4, 0u);
                c = v[j];
            }
            cur[s] = c;
            const uint32_t lo = prmt(v[0], v[1], 0x0040u), hi = prmt(v[2], v[3], 0x0040u);
            acc[s] = dp4a_u(prmt(lo, hi, 0x5410u) & 0x20202020u, 0x01010101u, acc[s]);
        }
    }
    using Row = uint32_t;
    __device__ __forceinline__ Row row(uint32_t c) const { return lds_u32(lanereg + (c << 8)); }
    __device__ __forceinline__ uint32_t apply(Row r, uint32_t st, uint32_t &cnt) const
    {
        const uint32_t f = (r >> (4 * st)) & 0xFu;
        cnt += f >> 3;
        return f & 7u;
    }
};

// B: u16 entries T[s][c] = next | count << 8 in shared memory (N <= 256; 512 B per state).
struct TableB {
    const uint8_t *sm;
    __device__ __forceinline__ void setup(uint8_t *s, const void *g, uint32_t n, const KConst &kc)
    {
        sm = s;
        c512 = kc.k_512;
        const uint4 *src = static_cast<const uint4 *>(g);
        uint4 *dst = reinterpret_cast<uint4 *>(s);
        for (uint32_t i = threadIdx.x; i < n * 32; i += blockDim.x) dst[i] = __ldg(src + i);
    }
    uint32_t c512;
    __device__ __forceinline__ uint32_t init(uint32_t st) const { return st; }
    __device__ __forceinline__ uint32_t state_of(uint32_t cur) const { return cur; }
    // acc counts in units of 256 (at most 8 x 8 KiB x 256 = 2^24 per chunk)
    __device__ __forceinline__ uint32_t count_of(uint32_t acc, uint32_t accf, uint32_t, uint64_t) const { return (acc >> 8) + accf; }
    template <int K>
    __device__ __forceinline__ void step(uint32_t w, int j, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                         uint32_t (&accf)[K]) const
    {
        const uint32_t c2 = j == 0 ? ((w << 1) & 0x1FEu) : ((w >> (8 * j - 1)) & 0x1FEu);
        const uint8_t *base = sm + c2;
#pragma unroll
        for (int s = 0; s < K; s++) {
            // entry = next | count << 8; address = next * 512 + 2c on the FMA pipe (IMAD)
            const uint32_t e = *reinterpret_cast<const uint16_t *>(base + mad_lo(cur[s], c512, 0u));
            cur[s] = e & 0xFFu;
            acc[s] = acc[s] + e - cur[s];  // + 256 * count: one IADD3 (IMAD.HI takes 4 cycles per warp)
        }
    }
    using Row = uint32_t;
    __device__ __forceinline__ Row row(uint32_t c) const { return c << 1; }
    __device__ __forceinline__ uint32_t apply(Row c2, uint32_t st, uint32_t &cnt) const
    {
        const uint32_t e = *reinterpret_cast<const uint16_t *>(sm + (st << 9) + c2);
        cnt += e >> 8;
        return e & 0xFFu;
    }
};

// G: u32 entries T[s][c] = next | count << 16 in global memory (L2-resident), any N <= 65535.
struct TableG {
    const uint32_t *gt;
    __device__ __forceinline__ void setup(uint8_t *, const void *g, uint32_t, const KConst &) { gt = static_cast<const uint32_t *>(g); }
    __device__ __forceinline__ uint32_t init(uint32_t st) const { return st; }
    __device__ __forceinline__ uint32_t state_of(uint32_t cur) const { return cur; }
    __device__ __forceinline__ uint32_t count_of(uint32_t acc, uint32_t accf, uint32_t, uint64_t) const { return acc + accf; }
    template <int K>
    __device__ __forceinline__ void step(uint32_t w, int j, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                         uint32_t (&accf)[K]) const
    {
        const uint32_t c = (w >> (8 * j)) & 0xFFu;
#pragma unroll
        for (int s = 0; s < K; s++) {
            const uint32_t e = __ldg(gt + ((cur[s] << 8) | c));
            accf[s] = mad_hi(e, 1u << 16, accf[s]);  // + (e >> 16)
            cur[s] = e & 0xFFFFu;
        }
    }
    using Row = uint32_t;
    __device__ __forceinline__ Row row(uint32_t c) const { return c; }
    __device__ __forceinline__ uint32_t apply(Row c, uint32_t st, uint32_t &cnt) const
    {
        const uint32_t e = __ldg(gt + ((st << 8) | c));
        cnt += e >> 16;
        return e & 0xFFFFu;
    }
};

// HS: hot-state row caching (Sec. 4.2) for tables that exceed shared
// memory.  States are renumbered at create time by static frequency -- the in-degree in the
// transition table, the paper's scheme -- so the hottest states are ids [0, H).  Their rows
// live in shared memory as u16 entries (next | count << 15, 512 B per row, H up to ~400); the
// other rows are read from the full u32 table in global memory (L2-resident).  The renumbering
// replaces the paper's Hot_States[hash(state)] lookup by one compare.
struct TableHS {
    const uint8_t *sm;
    const uint32_t *gt;
    uint32_t hot;
    __device__ __forceinline__ void setup(uint8_t *s, const void *g, uint32_t, const KConst &kc)
    {
        sm = s;
        gt = kc.gtab;
        hot = kc.hot_rows;
        const uint4 *src = static_cast<const uint4 *>(g);
        uint4 *dst = reinterpret_cast<uint4 *>(s);
        for (uint32_t i = threadIdx.x; i < hot * 32; i += blockDim.x) dst[i] = __ldg(src + i);
    }
    __device__ __forceinline__ uint32_t init(uint32_t st) const { return st; }
    __device__ __forceinline__ uint32_t state_of(uint32_t cur) const { return cur; }
    __device__ __forceinline__ uint32_t count_of(uint32_t acc, uint32_t accf, uint32_t, uint64_t) const { return acc + accf; }
    __device__ __forceinline__ uint32_t lookup(uint32_t st, uint32_t c, uint32_t &cnt) const
    {
        if (st < hot) {
            const uint32_t e = *reinterpret_cast<const uint16_t *>(sm + (st << 9) + (c << 1));
            cnt += e >> 15;
            return e & 0x7FFFu;
        }
        const uint32_t e = __ldg(gt + ((st << 8) | c));
        cnt += e >> 16;
        return e & 0xFFFFu;
    }
    template <int K>
    __device__ __forceinline__ void step(uint32_t w, int j, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                         uint32_t (&accf)[K]) const
    {
        const uint32_t c = (w >> (8 * j)) & 0xFFu;
#pragma unroll
        for (int s = 0; s < K; s++) cur[s] = lookup(cur[s], c, accf[s]);
    }
    using Row = uint32_t;
    __device__ __forceinline__ Row row(uint32_t c) const { return c; }
    __device__ __forceinline__ uint32_t apply(Row c, uint32_t st, uint32_t &cnt) const { return lookup(st, c, cnt); }
};

// CL: byte-class compressed, lane-replicated table (byte-mode DFAs with few distinct byte columns,
// e.g. the HTML tokenizer: 38 states x 24 classes).  Row of state s at R(s) = 0x400 + s * RB
// (RB = ceil(ncls / 2) * 128): the u16 entry (s, class x) of lane l sits at
//   R(s) + (x >> 1) * 128 + l * 4 + (x & 1) * 2
// and holds R(next) -- the chain value IS the next row's address.  Class map: u32 [256][32 lanes]
// at 0x10000 + byte * 256 + lane * 4 = the lane's offset of the byte's class, (x >> 1) * 128 + l * 4
// + (x & 1) * 2.  Every lookup is conflict-free (each lane reads its own bank).  Per byte: PRMT
// (class-map address) + LDS (class offset), off the chain; IADD + LDS.U16 on the chain; two adds for
// the count (region counting on the row address: ids are accept-partitioned, so [next >= nA] =
// [R(next) >= R(nA)] = the carry of R(next) + 2^32 - R(nA)).  Ids are recovered by a multiply-high.
struct TableCL {
    uint32_t cmreg;   // kClMapBase | lane * 4
    uint32_t tbase, rb, idmagic, negT, comp;
    __device__ __forceinline__ void setup(uint8_t *s, const void *g, uint32_t n, const KConst &kc)
    {
        tbase = (uint32_t)__cvta_generic_to_shared(s);  // 0x400 (checked)
        const uint32_t nslot = (kc.ncls + 1) >> 1;
        rb = nslot * 128u;
        idmagic = kc.cl_magic;
        negT = 0u - kc.rc_t;
        comp = kc.rc_comp;
        const uint32_t lane = threadIdx.x & 31;
        cmreg = kClMapBase | (lane * 4);
        const uint32_t *img = static_cast<const uint32_t *>(g);
        for (uint32_t i = threadIdx.x; i < 256 * 32; i += blockDim.x) {
            const uint32_t c = i >> 5, l = i & 31, x = __ldg(img + c);  // image: class id per byte
            const uint32_t v = (x >> 1) * 128u + l * 4u + (x & 1u) * 2u;
            asm volatile("st.shared.u32 [%0], %1;" ::"r"(kClMapBase + c * 256 + l * 4), "r"(v));
        }
        for (uint32_t i = threadIdx.x; i < n * nslot * 32; i += blockDim.x) {
            const uint32_t e = i >> 5, l = i & 31;  // e = s * nslot + slot: two u16 entries
            asm volatile("st.shared.u32 [%0], %1;" ::"r"(tbase + e * 128 + l * 4), "r"(__ldg(img + 256 + e)));
        }
    }
    __device__ __forceinline__ uint32_t init(uint32_t st) const { return tbase + st * rb; }
    __device__ __forceinline__ uint32_t id_of(uint32_t cur) const { return __umulhi(cur - tbase, idmagic); }
    __device__ __forceinline__ uint32_t state_of(uint32_t cur) const { return id_of(cur); }
    // acc: steps into the high region, n steps in all
    __device__ __forceinline__ uint32_t count_of(uint32_t acc, uint32_t accf, uint32_t, uint64_t n) const
    {
        return comp ? (uint32_t)n - (acc + accf) : acc + accf;
    }
    template <int K>
    __device__ __forceinline__ void step(uint32_t w, int j, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                         uint32_t (&accf)[K]) const
    {
        const uint32_t cm = lds_u32(prmt(w, cmreg, 0x7604u | (uint32_t(j) << 4)));  // off the chain
#pragma unroll
        for (int s = 0; s < K; s++) {
            cur[s] = lds_u16(cur[s] + cm);              // R(next)
            accf[s] = add_ge(accf[s], cur[s], negT);    // + [R(next) >= R(nA)]
        }
    }
    using Row = uint32_t;
    __device__ __forceinline__ Row row(uint32_t c) const { return lds_u32(cmreg + (c << 8)); }
    // one step in the chain representation (row address), exact count: the lockstep loops
    __device__ __forceinline__ uint32_t step1(Row cm, uint32_t cur, uint32_t &cnt) const
    {
        const uint32_t e = lds_u16(cur + cm);
        cnt += (uint32_t)(e >= 0u - negT) ^ comp;  // the accept increment (garbage only for the sink)
        return e;
    }
    __device__ __forceinline__ uint32_t apply(Row cm, uint32_t st, uint32_t &cnt) const
    {
        return id_of(step1(cm, init(st), cnt));
    }
};

// R16: N <= 16, byte mode, lane-replicated byte entries E[s][c] = next (accept-partitioned ids,
// region counting).  Lane l owns bank l: the entry (s, c) of lane l sits at shared address
//   tbase + s * 8192 + (c >> 2) * 128 + l * 4 + (c & 3)
// (the four entries of symbols 4q..4q+3 share the lane's word), so every LDS.U8 of a warp is one
// conflict-free wavefront whatever the lanes' states and symbols -- B's u16 table at N = 16 is read at
// random banks (72 % replays).  128 KiB at N = 16.  The symbol part of the address is computed, not
// loaded (two LOP3 per word, two PRMT + one IMAD/LEA per byte, off the chain).  The chain step is
// IMAD (row offset of the bare next state) + LDS.U8, and the count is two adds off the chain (region
// counting: [q >= nA] = the carry of q + 2^32 - nA, host_tables.h renumber_by_accept) -- no ALU-only
// operation on the chain, none for the count.
// RG (GROUPED, N <= 256, auto for 16 < N): the same with G = 32 >> logl copies instead of 32 -- lanes
// 2^logl * g .. 2^logl * (g + 1) - 1 share copy g, which occupies banks of their own, so a warp's
// LDS.U8 costs the worst bank load of 2^logl lanes on 2^logl banks instead of 32 lanes on 32 (B):
//   tbase + s * (8192 >> logl) + (c >> b) * 128 + g * 2^b + (c & (2^b - 1)),   b = 2 + logl,
// G * N * 256 <= 128 KiB (logl = 1: N <= 32, 2: N <= 64, ...).  logl is a run-time parameter.
template <bool GROUPED>
struct TableRep {
    uint32_t lane4;   // the lane's copy offset g * 2^b in every byte
    uint32_t tb;      // shared address of the table (low byte 0; PRMT source of bytes 1..3)
    uint32_t mlo;     // 2^b - 1 in every byte
    uint32_t sstride, cmul, negT, comp;
    __device__ __forceinline__ void setup(uint8_t *s, const void *g, uint32_t n, const KConst &kc)
    {
        tb = (uint32_t)__cvta_generic_to_shared(s);
        if (tb & 0xFFu) __trap();  // the PRMT address form needs a 256-aligned table
        const uint32_t logl = GROUPED ? kc.r_logl : 0u, lane = threadIdx.x & 31;
        lane4 = ((lane >> logl) << (2 + logl)) * 0x01010101u;
        mlo = ((4u << logl) - 1u) * 0x01010101u;
        sstride = (kc.k_512 << 4) >> logl;
        cmul = (kc.k_16 << 1) >> logl;
        negT = 0u - kc.rc_t;
        comp = kc.rc_comp;
        // smem word i: line i >> 5, copy (i & 31) >> logl, word (line << logl) | (i & (2^logl - 1))
        // of the row-major image (u32 [n][64]: entries 4q..4q+3 of row s)
        const uint32_t *img = static_cast<const uint32_t *>(g);
        const uint32_t lm = (1u << logl) - 1u;
        for (uint32_t i = threadIdx.x; i < ((n * 64 * 32) >> logl); i += blockDim.x)
            asm volatile("st.shared.u32 [%0], %1;" ::"r"(tb + i * 4),
                         "r"(__ldg(img + (((i >> 5) << logl) | (i & lm)))));
    }
    __device__ __forceinline__ uint32_t init(uint32_t st) const { return st; }
    __device__ __forceinline__ uint32_t state_of(uint32_t cur) const { return cur; }
    // acc: steps into the high region, n steps in all
    __device__ __forceinline__ uint32_t count_of(uint32_t acc, uint32_t accf, uint32_t, uint64_t n) const
    {
        return comp ? (uint32_t)n - (acc + accf) : acc + accf;
    }
    // symbol part of the address of byte j of w.  R16's odd bytes combine the two halves with a
    // shift-add (LEA, ALU pipe) instead of an IMAD: measured 0-2 % faster than IMADs on every byte,
    // although ncu shows the ALU pipe 82 % busy and the FMA pipe 20 %.
    __device__ __forceinline__ uint32_t sym(uint32_t w, int j) const
    {
        const uint32_t m = GROUPED ? mlo : 0x03030303u;
        const uint32_t lo = (w & m) | lane4, hi = w & ~m;
        const uint32_t h = prmt(hi, 0u, 0x4440u | uint32_t(j)), l = prmt(lo, tb, 0x7650u | uint32_t(j));
        return (!GROUPED && (j & 1)) ? (h << 5) + l : mad_lo(h, cmul, l);
    }
    template <int K>
    __device__ __forceinline__ void step(uint32_t w, int j, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                         uint32_t (&accf)[K]) const
    {
        const uint32_t a = sym(w, j);
#pragma unroll
        for (int s = 0; s < K; s++) {
            cur[s] = lds_u8(mad_lo(cur[s], sstride, a));  // next state
            accf[s] = add_ge(accf[s], cur[s], negT);      // + [next >= nA]
        }
    }
    using Row = uint32_t;
    __device__ __forceinline__ Row row(uint32_t c) const { return sym(c, 0); }
    __device__ __forceinline__ uint32_t apply(Row a, uint32_t st, uint32_t &cnt) const
    {
        const uint32_t e = lds_u8(a + st * sstride);
        cnt += (uint32_t)(e >= 0u - negT) ^ comp;  // the accept increment (garbage only for the sink)
        return e;
    }
};
using TableR16 = TableRep<false>;
using TableRG = TableRep<true>;

template <int VAR> struct TableFor;
template <> struct TableFor<VAR_P4> { using type = TablePacked<VAR_P4>; };
template <> struct TableFor<VAR_P8> { using type = TablePacked<VAR_P8>; };
template <> struct TableFor<VAR_B> { using type = TableB; };
template <> struct TableFor<VAR_G> { using type = TableG; };
template <> struct TableFor<VAR_HS> { using type = TableHS; };
template <> struct TableFor<VAR_CL> { using type = TableCL; };
template <> struct TableFor<VAR_N8> { using type = TableN8; };
template <> struct TableFor<VAR_R16> { using type = TableR16; };
template <> struct TableFor<VAR_RG> { using type = TableRG; };

// --------------------------------------------------------------------- a4: local processing --
template <class TB> struct TableHasStep4 { static constexpr bool value = false; };
// Tables whose chain representation is not the state id but can be stepped one byte at a time
// with an exact count (step1): the lockstep loops run in that representation (equality of two
// chain values is equality of states) and skip the id conversions of apply().
template <class TB> struct TableHasStep1 { static constexpr bool value = false; };
template <> struct TableHasStep1<TableCL> { static constexpr bool value = true; };
template <class TB>
__device__ __forceinline__ uint32_t nat_init(const TB &tb, uint32_t st)
{
    if constexpr (TableHasStep1<TB>::value) return tb.init(st);
    else return st;
}
template <class TB>
__device__ __forceinline__ uint32_t nat_apply(const TB &tb, const typename TB::Row &r, uint32_t x, uint32_t &cnt)
{
    if constexpr (TableHasStep1<TB>::value) return tb.step1(r, x, cnt);
    else return tb.apply(r, x, cnt);
}
template <> struct TableHasStep4<TableN8> { static constexpr bool value = true; };

template <int K, class TB>
__device__ __forceinline__ void process32(const TB &tb, const Bytes32 &x, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                          uint32_t (&accf)[K])
{
    if constexpr (TableHasStep4<TB>::value) {
#pragma unroll
        for (int q = 0; q < 8; q++) tb.template step4<K>(x.w[q], cur, accf, acc);
    } else if constexpr (K <= 4) {
#pragma unroll
        for (int q = 0; q < 8; q++)
#pragma unroll
            for (int j = 0; j < 4; j++) tb.template step<K>(x.w[q], j, cur, acc, accf);
    } else {
        uint32_t w[8];
#pragma unroll
        for (int q = 0; q < 8; q++) w[q] = x.w[q];
#pragma unroll 1
        for (int q = 0; q < 8; q++) {
#pragma unroll
            for (int j = 0; j < 4; j++) tb.template step<K>(w[0], j, cur, acc, accf);
#pragma unroll
            for (int r = 0; r < 7; r++) w[r] = w[r + 1];
        }
    }
}

template <int K, class TB>
__device__ __forceinline__ bool chains_converged(const TB &tb, const uint32_t (&cur)[K])
{
    bool c = true;
#pragma unroll
    for (int s = 1; s < K; s++) c = c && tb.state_of(cur[s]) == tb.state_of(cur[0]);
    return c;
}

// Alg. 3 over bytes [b, e) of the input: 32-byte blocks (one full sector per lane per
// LDG.256) with two blocks in flight, then the ragged tail byte by byte.
// Convergence: two chains that reach the same state stay identical for the rest of the chunk
// (the state-convergence property of [18]).  After every block the warp votes; once all
// chains of every active lane coincide the remainder runs ONE chain and its count increments
// are added to every slot -- bit-identical to running all k chains.  Absent slots start as a copy
// of slot 0 so they never block the vote (their results are ignored).
// Blocks [i, nblk) of 32 bytes with a 3-buffer rotation (2 blocks in flight, no register moves).
// On entry x0 = block i, x1 = block i+1.  With CHECK, returns true as soon as the warp votes
// that all chains coincide; x0/x1 then hold blocks i, i+1 for the continuation.
template <int KK, bool CHECK, class TB>
__device__ __forceinline__ bool run_blocks(const TB &tb, const uint8_t *p, uint64_t &i, uint64_t nblk, Bytes32 &x0,
                                           Bytes32 &x1, uint32_t (&cur)[KK], uint32_t (&acc)[KK],
                                           uint32_t (&accf)[KK])
{
    Bytes32 x2;
    while (i < nblk) {
        if (i + 2 < nblk) x2 = ldg_block(p, i + 2);
        process32<KK>(tb, x0, cur, acc, accf);
        ++i;
        if (CHECK && __all_sync(__activemask(), chains_converged<KK>(tb, cur))) {
            x0 = x1;
            x1 = x2;
            return true;
        }
        if (i >= nblk) break;
        if (i + 2 < nblk) x0 = ldg_block(p, i + 2);
        process32<KK>(tb, x1, cur, acc, accf);
        ++i;
        if (CHECK && __all_sync(__activemask(), chains_converged<KK>(tb, cur))) {
            x1 = x0;
            x0 = x2;
            return true;
        }
        if (i >= nblk) break;
        if (i + 2 < nblk) x1 = ldg_block(p, i + 2);
        process32<KK>(tb, x2, cur, acc, accf);
        ++i;
        if (CHECK && __all_sync(__activemask(), chains_converged<KK>(tb, cur))) {
            x0 = x0;  // blocks i, i+1 already in x0, x1
            return true;
        }
    }
    return false;
}

// Alg. 3 over bytes [b, e) of the input: 32-byte blocks (one full sector per lane per
// LDG.256) with two blocks in flight, then the ragged tail byte by byte.
// Convergence: two chains that reach the same state stay identical for the rest of the chunk
// (the state-convergence property of [18]).  After every block the warp votes; once all
// chains of every active lane coincide the remainder runs ONE chain and its count increments
// are added to every slot -- bit-identical to running all k chains.  Absent slots start as a copy
// of slot 0 so they never block the vote (their results are ignored).
template <int K, class TB>
__device__ __forceinline__ void local_phase(const TB &tb, const uint8_t *__restrict__ in, uint64_t b, uint64_t e,
                                            bool aligned, uint32_t (&cur)[K], uint32_t (&acc)[K],
                                            uint32_t (&accf)[K], uint32_t *stash = nullptr)
{
    if (aligned && (b & 31)) {
        // the peeled head of an unaligned input (chunk 0 starts at in + head): bytes up to the first
        // 32-byte boundary one at a time, then full sectors
        const uint64_t stop = min(e, (b + 31) & ~(uint64_t)31);
        for (; b < stop; b++) tb.template step<K>(__ldg(in + b), 0, cur, acc, accf);
        stash = nullptr;
    }
    const uint8_t *p = in + b;
    const uint64_t n = e - b;
    const uint64_t nblk = aligned ? (n >> 5) : 0;
    uint64_t i = 0;
    bool single = false;
    Bytes32 x0, x1;
    if (nblk) {
        x0 = ldg_block(p, 0);
        if (nblk > 1) x1 = ldg_block(p, 1);
        if (stash) {
            reinterpret_cast<uint4 *>(stash)[0] = make_uint4(x0.w[0], x0.w[1], x0.w[2], x0.w[3]);
            reinterpret_cast<uint4 *>(stash)[1] = make_uint4(x0.w[4], x0.w[5], x0.w[6], x0.w[7]);
        }
        single = run_blocks<K, (K > 1)>(tb, p, i, nblk, x0, x1, cur, acc, accf);
    }
    if constexpr (K > 1) {
        if (single) {
            uint32_t c1[1] = {cur[0]}, a1[1] = {0u}, f1[1] = {0u};
            run_blocks<1, false>(tb, p, i, nblk, x0, x1, c1, a1, f1);
            for (uint64_t t = nblk << 5; t < n; t++) tb.template step<1>(__ldg(p + t), 0, c1, a1, f1);
#pragma unroll
            for (int s = 0; s < K; s++) {
                cur[s] = c1[0];
                acc[s] += a1[0];
                accf[s] += f1[0];
            }
            return;
        }
    }
    for (uint64_t t = nblk << 5; t < n; t++) {
        const uint32_t c = __ldg(p + t);
        tb.template step<K>(c, 0, cur, acc, accf);
    }
}


// ----------------------------------------------------------------- a3: look-back speculation --
// Candidate start states of the chunk starting at byte b, ranked.  Depth 1 (lookback < 32): the
// image of the preceding byte ranked by preimage count (A5; host table LB).  Window
// (lookback = Lw >= 32, multiple of 32): the image of x[b-Lw-1] is run through the Lw bytes
// before the chunk and the reached states are ranked by multiplicity (how many image states
// reach each), ties to the smaller id -- the same rule one level deeper (reading R7).  If the
// window would reach before the start of a known-start run, the single exact state is used.
// Returns S (top k, NOSTATE-padded), X (the next kExt candidates, for eager completion).
template <int K, class TB>
__device__ __forceinline__ void speculate(const TB &tb, const Params &p, uint64_t b, bool first_chunk, bool empty,
                                          uint32_t start_state, uint32_t (&S)[K], uint32_t (&X)[kExt])
{
#pragma unroll
    for (int s = 0; s < K; s++) S[s] = NOSTATE;
#pragma unroll
    for (int q = 0; q < kExt; q++) X[q] = NOSTATE;
    if (empty) return;
    if (first_chunk && !p.keyed && !p.spec_all) {
        S[0] = start_state;
        return;
    }
    const uint32_t ksel = p.k;
    if (p.spec) {  // ranked candidates from the look-back pre-pass (spec_kernel.cuh)
        const uint16_t *c = p.spec + (b / p.chunk) * p.spec_stride;
#pragma unroll
        for (int s = 0; s < K; s++)
            if ((uint32_t)s < ksel) {
                const uint32_t v = __ldg(c + s);
                S[s] = v == 0xFFFFu ? NOSTATE : v;
            }
#pragma unroll
        for (int q = 0; q < kExt; q++) {
            const uint32_t v = __ldg(c + ksel + q);
            X[q] = v == 0xFFFFu ? NOSTATE : v;
        }
        return;
    }
    const uint32_t c = first_chunk ? p.halo_byte : (uint32_t)__ldg(p.in + b - 1);
    const uint32_t ni = __ldg(p.nimg + c);
#pragma unroll
    for (int s = 0; s < K; s++)
        if ((uint32_t)s < min(ni, ksel)) S[s] = (uint32_t)__ldg(p.lb + c * KMAX + s);
#pragma unroll
    for (int q = 0; q < kExt; q++)
        if (ksel + q < ni) X[q] = (uint32_t)__ldg(p.lb + c * KMAX + ksel + q);
}

// --------------------------------------------------------- a5/a6: composition of mappings --
// (L x R)[s]: a complete slot of L whose end state is a speculated start of R continues with R's
// slot (which may itself be broken further on) and adds counts -- the membership check of
// Alg. 1, all K compares unrolled into predicated selects (k is a compile-time
// constant).  No match: the slot breaks at R's first chunk.
// With `ext` (the eager-completion entries of R's first chunk, in smem) a state that is not a
// speculated start of R but was run to convergence with one of R's chains continues as that slot,
// corrected by the count difference up to the meeting point -- exact, and no break.
template <int K>
__device__ __forceinline__ void compose(uint32_t (&eob)[K], uint32_t (&cnt)[K], const uint32_t (&Sr)[K],
                                        const uint32_t (&eobr)[K], const uint32_t (&cntr)[K], uint32_t first_r,
                                        const uint32_t *ext = nullptr)
{
#pragma unroll
    for (int s = 0; s < K; s++) {
        const uint32_t x = eob[s];
        if ((x >> 16) == COMPLETE) {
            const uint32_t st = x & 0xFFFFu;
            uint32_t ne = st | (first_r << 16), nc = 0;
            bool hit = false;
#pragma unroll
            for (int j = 0; j < K; j++)
                if (Sr[j] == st) {
                    ne = eobr[j];
                    nc = cntr[j];
                    hit = true;
                }
            if (!hit && ext) {
                const uint32_t *ex = ext + first_r * kExt;
#pragma unroll
                for (int q = 0; q < kExt; q++) {
                    const uint32_t v = ex[q];
                    if ((v & 0xFFFFu) == st) {
                        const uint32_t l = (v >> 16) & 0xFu;
                        const int32_t delta = (int32_t)v >> 20;
#pragma unroll
                        for (int j = 0; j < K; j++)
                            if ((uint32_t)j == l) {
                                ne = eobr[j];
                                nc = cntr[j] + (uint32_t)delta;
                            }
                    }
                }
            }
            eob[s] = ne;
            cnt[s] += nc;
        }
    }
}

// Alg. 2: the hash implementation of the runtime check, which the paper uses for large
// k (k > 12, footnote P:200) because Alg. 1 costs O(k^2).  B200 form: instead of dynamically
// indexed per-thread arrays (which the paper notes spill to local memory), every thread owns
// one column of a shared-memory table -- word (row * T + tid), so a warp's accesses are conflict-free:
//   rows 0 .. kHashSize-1   hash_init_states: bucket h holds (slot << 16 | start), open addressing
//                           (linear probing) in place of fixed-capacity chains; HASH_SIZE = 32 = the
//                           next power of two >= 2k for 8 < k <= 16 and hash = s mod HASH_SIZE (A10)
//   rows 32 .. 32+K-1       hash_end_states of the thread's current mapping (eob per slot)
//   rows 32+K .. 32+2K-1    its counts
// Step 1 (lines 7-12) is built once per scan from the thread's own start set (a lane's mapping is
// always keyed on its own first chunk's starts); before each scan level the lane publishes its
// current ends and counts, and step 2 (lines 14-28) probes the RIGHT lane's column: O(k) per slot
// set, no shuffles of the right mapping and no k x k compare network.  Results are identical to
// Alg. 1 (the same matches; starts are distinct, reading A6).
constexpr uint32_t kHashEmpty = 0xFFFFFFFFu;
template <int K>
__device__ __forceinline__ void hash_build(uint32_t *hs, uint32_t T, uint32_t tid, const uint32_t (&S)[K])
{
#pragma unroll
    for (uint32_t h = 0; h < kHashSize; h++) hs[h * T + tid] = kHashEmpty;
#pragma unroll
    for (int j = 0; j < K; j++)
        if (S[j] != NOSTATE) {
            uint32_t h = S[j] & (kHashSize - 1);
            while (hs[h * T + tid] != kHashEmpty) h = (h + 1) & (kHashSize - 1);
            hs[h * T + tid] = ((uint32_t)j << 16) | S[j];
        }
}
template <int K>
__device__ __forceinline__ void hash_publish(uint32_t *hs, uint32_t T, uint32_t tid, const uint32_t (&eob)[K],
                                             const uint32_t (&cnt)[K])
{
#pragma unroll
    for (int s = 0; s < K; s++) {
        hs[(kHashSize + s) * T + tid] = eob[s];
        hs[(kHashSize + K + s) * T + tid] = cnt[s];
    }
}
// (L x R)[s] with R published in column rt (Alg. 2 step 2); same semantics as compose().
template <int K>
__device__ __forceinline__ void compose_hash(uint32_t (&eob)[K], uint32_t (&cnt)[K], const uint32_t *hs, uint32_t T,
                                             uint32_t rt, uint32_t first_r, const uint32_t *ext)
{
#pragma unroll
    for (int s = 0; s < K; s++) {
        const uint32_t x = eob[s];
        if ((x >> 16) == COMPLETE) {
            const uint32_t st = x & 0xFFFFu;
            uint32_t h = st & (kHashSize - 1), j = 0xFFFFFFFFu;
            for (;;) {  // at most K occupied buckets of 2K: terminates at an empty one
                const uint32_t e = hs[h * T + rt];
                if (e == kHashEmpty) break;
                if ((e & 0xFFFFu) == st) {
                    j = e >> 16;
                    break;
                }
                h = (h + 1) & (kHashSize - 1);
            }
            uint32_t ne = st | (first_r << 16), nc = 0;
            if (j != 0xFFFFFFFFu) {
                ne = hs[(kHashSize + j) * T + rt];
                nc = hs[(kHashSize + K + j) * T + rt];
            } else if (ext) {
                const uint32_t *ex = ext + first_r * kExt;
#pragma unroll
                for (int q = 0; q < kExt; q++) {
                    const uint32_t v = ex[q];
                    if ((v & 0xFFFFu) == st) {
                        const uint32_t l = (v >> 16) & 0xFu;
                        ne = hs[(kHashSize + l) * T + rt];
                        nc = hs[(kHashSize + K + l) * T + rt] + (uint32_t)((int32_t)v >> 20);
                    }
                }
            }
            eob[s] = ne;
            cnt[s] += nc;
        }
    }
}

// Test hook (fsm_debug_get_merge): the lane's mapping after scan level `level` (0 = the chunk's own).
template <int K>
__device__ __forceinline__ void dbg_record(uint4 *dbg, int level, const uint32_t (&S)[K], const uint32_t (&eob)[K],
                                           const uint32_t (&cnt)[K], bool ident)
{
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int s = 0; s < K; s++) dbg[(level * 32 + lane) * KMAX + s] = make_uint4(S[s], eob[s], cnt[s], ident ? 1u : 0u);
}

// Warp-level suffix scan (Kogge-Stone over shuffles): afterwards lane i holds the mapping of
// elements [i, 32) keyed on its own start set.  first0 = chunk index of lane 0's element, step =
// chunk distance between lanes.  Level d composes lane i with lane i + d, so lane 0 after d = 1 is
// M_0 x M_1, lane 2 is M_2 x M_3, and lane 0 after d = 2 is (M_0 x M_1) x (M_2 x M_3): the merge tree
// of Fig. 4b.  dbg (test hook, normally null) records every level.
template <int K, bool HASH = false>
__device__ __forceinline__ void warp_suffix_scan(uint32_t (&S)[K], uint32_t (&eob)[K], uint32_t (&cnt)[K], bool &ident,
                                                 uint32_t first0, uint32_t step, const uint32_t *ext = nullptr,
                                                 uint4 *dbg = nullptr, uint32_t *hs = nullptr)
{
    const int lane = threadIdx.x & 31;
    if (dbg) dbg_record<K>(dbg, 0, S, eob, cnt, ident);
    if constexpr (HASH) {
        const uint32_t T = blockDim.x, tid = threadIdx.x;
        hash_build<K>(hs, T, tid, S);
#pragma unroll
        for (int d = 1, level = 1; d < 32; d <<= 1, level++) {
            const bool ir = __shfl_down_sync(0xFFFFFFFFu, (int)ident, d) != 0;
            hash_publish<K>(hs, T, tid, eob, cnt);
            __syncwarp();
            if (lane + d < 32 && !ir && !ident) compose_hash<K>(eob, cnt, hs, T, tid + d, first0 + (lane + d) * step, ext);
            __syncwarp();
            if (dbg) dbg_record<K>(dbg, level, S, eob, cnt, ident);
        }
        return;
    }
#pragma unroll
    for (int d = 1, level = 1; d < 32; d <<= 1, level++) {
        uint32_t Sr[K], er[K], cr[K];
#pragma unroll
        for (int s = 0; s < K; s++) {
            Sr[s] = __shfl_down_sync(0xFFFFFFFFu, S[s], d);
            er[s] = __shfl_down_sync(0xFFFFFFFFu, eob[s], d);
            cr[s] = __shfl_down_sync(0xFFFFFFFFu, cnt[s], d);
        }
        const bool ir = __shfl_down_sync(0xFFFFFFFFu, (int)ident, d) != 0;
        if (lane + d < 32 && !ir && !ident) compose<K>(eob, cnt, Sr, er, cr, first0 + (lane + d) * step, ext);
        if (dbg) dbg_record<K>(dbg, level, S, eob, cnt, ident);
    }
}

// ----------------------------------------------------------------- shared-memory layout ----
// Split mode (dedicated epilogue warp): the tile state the epilogue reads (qe, qc, sj, ext) is
// double-buffered -- buffer b at offset b * buf -- and there is no stash (re-execution and eager
// completion read the chunk's first bytes from L2 instead).
struct Layout {
    uint32_t qe, qc, sj, ws, we, wc, wi, misc, stash, ext, hs, total, buf;
    __host__ __device__ Layout(uint32_t T, uint32_t K, uint32_t start, bool split = false, bool hash = false)
    {
        uint32_t o = start;
        // Alg. 2 scratch: one column per thread of kHashSize buckets + K end states + K counts
        hs = o;
        if (hash) o += T * (kHashSize + 2 * K) * 4;
        qe = o;  o += T * K * 4;
        qc = o;  o += T * K * 4;
        sj = o;  o += T * K * 2;
        o = (o + 15) & ~15u;
        if (split) {
            ext = o; o += T * kExt * 4;
            buf = o - qe;
            o += buf;
            stash = 0;
        }
        ws = o;  o += 32 * K * 4;
        we = o;  o += 32 * K * 4;
        wc = o;  o += 32 * K * 4;
        wi = o;  o += 32 * 4;
        misc = o; o += 16;
        if (!split) {
            stash = o; o += T * 32;
            ext = o; o += T * kExt * 4;
            buf = 0;
        }
        total = o;
    }
};

// Named barriers of the split kernel: 1 = worker warps; 2, 3 = tile state of buffer 0 / 1 handed to
// the epilogue warp; 4, 5 = buffer 0 / 1 free again.
__device__ __forceinline__ void named_sync(uint32_t id, uint32_t n)
{
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ void named_arrive(uint32_t id, uint32_t n)
{
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}
// Which fused kernels run split (measured on B200, 4 GiB inputs, split vs unsplit): the CL variant
// (HTML, k = 1: +13 %, its serial re-executions dominate the epilogue) and the multi-chain kernels
// of the shared-memory variants (P4 / P8 / B, K >= 2: +6..15 %).  K = 1 kernels of P8 / B / G / HS
// lose more from the missing 32nd worker warp and stash than they gain (-4..-8 %): unsplit.
// A launch runs split only if this policy says so AND the double-buffered layout fits in shared
// memory (large-K CL kernels next to a 150 KiB table do not).
__host__ __device__ constexpr bool split_kernel(int var, int K)
{
    return var == 6 /* CL */ || ((var == 0 || var == 1 || var == 2 || var == 7 || var == 8 || var == 9) /* P4 P8 B N8 R16 RG */ && K >= 2);
}

// Per-tile context used by re-execution and the epilogue.
struct TileCtx {
    const uint8_t *in;
    uint64_t len;
    uint64_t tile_base;
    uint32_t head;      // chunk 0 of the run starts at in + head (peeled unaligned input)
    uint32_t chunk;
    uint32_t nch;       // non-empty chunks in this tile (>= 1)
    bool aligned;
    const uint32_t *Qe, *Qc;
    const uint16_t *Sj;
    const uint32_t *stash;  // first 32 bytes of every chunk (valid when aligned and >= 32 bytes)
    const uint32_t *ext;    // eager-completion entries, kExt per chunk
};

// Look up an eager-completion entry of chunk c for state st: returns the slot (or -1) and delta.
__device__ __forceinline__ int ext_lookup(const uint32_t *ext, uint32_t c, uint32_t st, int32_t &delta)
{
    const uint32_t *ex = ext + c * kExt;
#pragma unroll
    for (int q = 0; q < kExt; q++) {
        const uint32_t v = ex[q];
        if ((v & 0xFFFFu) == st) {
            delta = (int32_t)v >> 20;
            return (int)((v >> 16) & 0xFu);
        }
    }
    return -1;
}

// a8: resolve a broken slot.  The run is in state `st` when entering chunk c of the tile, with
// count n so far.  Re-execute chunk c from st in lockstep with the chunk's speculated chains
// ("re-execute the next chunk with states[s]"); the moment the re-executed state equals a
// speculated chain's state both runs coincide for the rest of the chunk, so the result is exact:
// (that chain's path, n + cnt_x(p) - cnt_l(p) + its count).  Otherwise continue at chunk c+1.
// The work done is tallied in rc (chunks, bytes, longest run of consecutive re-executed chunks,
// eager-entry completions); the caller attributes it to the true or a candidate path.
template <int K, class TB>
__device__ void resolve(const TB &tb, const TileCtx &t, uint32_t st, uint32_t c, uint32_t n, uint32_t &out_st,
                        uint32_t &out_n, ReCount &rc)
{
    uint32_t chain = 0, last_c = 0xFFFFFFFFu;
    for (;;) {
        {   // eager completion already ran this state into one of the chunk's chains
            int32_t dl;
            const int l = ext_lookup(t.ext, c, st, dl);
            if (l >= 0) {
                rc.eager++;
                if (c == 0 && rc.chunks == 0) rc.join0 = (uint32_t)l;
                n += (uint32_t)dl + t.Qc[c * K + l];
                const uint32_t x = t.Qe[c * K + l];
                if ((x >> 16) == COMPLETE) {
                    out_st = x & 0xFFFFu;
                    out_n = n;
                    return;
                }
                st = x & 0xFFFFu;
                c = x >> 16;
                continue;
            }
        }
        const uint64_t b = max(t.tile_base + (uint64_t)c * t.chunk, (uint64_t)t.head);
        const uint64_t e = min(t.tile_base + (uint64_t)(c + 1) * t.chunk, t.len);
        uint32_t y[K], cy[K];
        bool pres[K];
#pragma unroll
        for (int l = 0; l < K; l++) {
            const uint32_t sv = t.Sj[c * K + l];
            pres[l] = sv != 0xFFFFu;
            y[l] = nat_init(tb, pres[l] ? sv : 0u);
            cy[l] = 0;
        }
        uint32_t cx = 0, cyc = 0;
        int conv = -1;
        uint64_t pos = b;
        const uint64_t wend = min(e, b + kLockstepWindow);
        uint32_t sn = nat_init(tb, st);  // the re-executed path in the chain representation
        auto one = [&](uint32_t byte) {
            const typename TB::Row r = tb.row(byte);
            sn = nat_apply(tb, r, sn, cx);
#pragma unroll
            for (int l = 0; l < K; l++) y[l] = nat_apply(tb, r, y[l], cy[l]);
#pragma unroll
            for (int l = 0; l < K; l++)
                if (pres[l] && conv < 0 && y[l] == sn) {
                    conv = l;
                    cyc = cy[l];
                }
        };
        if (t.stash && t.aligned && (b & 31) == 0 && e - b >= 32) {
            // the chunk's first 32 bytes were stashed in smem by its owner during the local phase:
            // the usual early exit never touches global memory
#pragma unroll 1
            for (int q = 0; q < 32 && conv < 0; q++) {
                one((t.stash[c * 8 + (q >> 2)] >> (8 * (q & 3))) & 0xFFu);
                pos++;
            }
        }
        if (t.aligned) {
            while (conv < 0 && (pos & 15) && pos < wend) {
                one(__ldg(t.in + pos));
                pos++;
            }
            while (conv < 0 && pos + 16 <= wend) {
                const uint4 v = ldg128(t.in + pos);
                uint32_t used = 0;
#pragma unroll 1
                for (int q = 0; q < 16 && conv < 0; q++) {
                    const uint32_t wq = q < 8 ? (q < 4 ? v.x : v.y) : (q < 12 ? v.z : v.w);
                    one((wq >> (8 * (q & 3))) & 0xFFu);
                    used++;
                }
                pos += used;
            }
        }
        while (conv < 0 && pos < wend) {
            one(__ldg(t.in + pos));
            pos++;
        }
        if (conv < 0 && pos < e) {  // past the lockstep window: the re-executed path alone
            if (t.aligned) {
                for (; (pos & 15) && pos < e; pos++) sn = nat_apply(tb, tb.row(__ldg(t.in + pos)), sn, cx);
                for (; pos + 16 <= e; pos += 16) {
                    const uint4 v = ldg128(t.in + pos);
                    const uint32_t w4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                    for (int q = 0; q < 16; q++) sn = nat_apply(tb, tb.row((w4[q >> 2] >> (8 * (q & 3))) & 0xFFu), sn, cx);
                }
            }
            for (; pos < e; pos++) sn = nat_apply(tb, tb.row(__ldg(t.in + pos)), sn, cx);
        }
        if constexpr (TableHasStep1<TB>::value) st = tb.state_of(sn);
        else st = sn;
        chain = c == last_c + 1 ? chain + 1 : 1;
        last_c = c;
        rc.chunks++;
        rc.bytes += (uint32_t)(pos - b);
        rc.chain = max(rc.chain, chain);
        uint32_t x;
        if (conv >= 0) {
            if (c == 0 && rc.chunks == 1) rc.join0 = (uint32_t)conv;
            n += cx - cyc + t.Qc[c * K + conv];
            x = t.Qe[c * K + conv];
        } else {
            n += cx;
            if (c + 1 >= t.nch) {
                out_st = st;
                out_n = n;
                return;
            }
            x = st | ((c + 1) << 16);
#pragma unroll
            for (int l = 0; l < K; l++)
                if (t.Sj[(c + 1) * K + l] == st) {
                    x = t.Qe[(c + 1) * K + l];
                    n += t.Qc[(c + 1) * K + l];
                }
        }
        if ((x >> 16) == COMPLETE) {
            out_st = x & 0xFFFFu;
            out_n = n;
            return;
        }
        st = x & 0xFFFFu;
        c = x >> 16;
    }
}

__device__ __forceinline__ void add_stats(DevStats *S, const ReCount &rc, bool true_path)
{
    if (!rc.chunks && !rc.eager) return;
    if (true_path) {
        if (rc.chunks) {
            atomicAdd(&S->reexec_true, (unsigned long long)rc.chunks);
            atomicAdd(&S->reexec_true_bytes, (unsigned long long)rc.bytes);
            atomicMax(&S->max_miss_chain, (unsigned long long)rc.chain);
        }
        if (rc.eager) atomicAdd(&S->eager_resolved, (unsigned long long)rc.eager);
    } else if (rc.chunks) {
        atomicAdd(&S->reexec_cand, (unsigned long long)rc.chunks);
        atomicAdd(&S->reexec_cand_bytes, (unsigned long long)rc.bytes);
    }
}

// a7-a9 for one tile, run by one full warp once the tile's suffix mappings Qe/Qc (keyed on the
// chunks' speculated starts Sj) are in shared memory: pre-resolution of the tile aggregate's broken
// slots (R5, the top p.preresolve tile-start candidates), publication of A, decoupled look-back,
// own inclusive prefix P (resolving the true path's broken slot if it was left unresolved), and the
// result.
template <int K, bool HASH, class TB>
__device__ __forceinline__ void tile_epilogue(const TB &tb, const Params &p, uint32_t tile, uint64_t tile_base,
                                              uint32_t nch_max, uint32_t *Qe, uint32_t *Qc, const uint16_t *Sj,
                                              const uint32_t *stash, const uint32_t *Ext, uint32_t start_state,
                                              unsigned long long start_count, uint32_t ksel, uint32_t *hs)
{
    const int lane = threadIdx.x & 31;
    TileCtx t;
    t.in = p.in;
    t.len = p.len;
    t.tile_base = tile_base;
    t.head = p.head;
    t.chunk = p.chunk;
    {
        const uint64_t rem = p.len > tile_base ? p.len - tile_base : 0;
        const uint64_t nch = (rem + p.chunk - 1) / p.chunk;
        t.nch = (uint32_t)(nch < 1 ? 1 : (nch > nch_max ? nch_max : nch));
    }
    t.aligned = p.aligned != 0;
    t.Qe = Qe;
    t.Qc = Qc;
    t.Sj = Sj;
    t.stash = stash;
    t.ext = Ext;

    // a8 (tile candidates, R5): resolve the broken slots of the tile aggregate Q_0 for the top
    // p.preresolve speculated tile starts, so that a successor's look-back can pass through them
    // without waiting for this tile's P.  The other slots are published broken (lazy): they are
    // resolved only if the true path turns out to enter this tile in them.
    ReCount rc5{0, 0, 0, 0, 0xFFFFu};
    uint32_t qe = lane < K ? Qe[lane] : 0u, qc = lane < K ? Qc[lane] : 0u;  // own-prefix source
    if (lane < K && (uint32_t)lane < p.preresolve) {
        if ((qe >> 16) < ABSENT) {
            uint32_t st, n;
            resolve<K>(tb, t, qe & 0xFFFFu, qe >> 16, qc, st, n, rc5);
            qe = st | (COMPLETE << 16);
            qc = n;
            Qe[lane] = qe;  // a later tile-boundary re-execution that joins this slot reuses it
            Qc[lane] = qc;
        }
    }
    __syncwarp();

    // a7: publish the aggregate A_b (slot = {start, end, count, broken})
    TileDesc *D = p.desc + tile;
    if (lane < K) {
        const uint32_t sv = Sj[lane];
        const bool broken = (qe >> 16) != COMPLETE;
        D->aslot[lane] = make_uint4(sv == 0xFFFFu ? NOSTATE : sv, qe & 0xFFFFu, qc, broken ? 1u : 0u);
    }
    __threadfence();
    __syncwarp();
    const uint32_t ep = p.epoch << 2;
    if (lane == 0) st_release(&D->flag, ep | ST_A);

    // a7: decoupled look-back -> exclusive prefix E (lane s holds shard slot s).
    // (1) walk back 32 descriptors at a time to the nearest inclusive prefix P_m.
    uint32_t Es = 0;
    unsigned long long Ec = 0;
    bool Ev = false;
    int64_t m;
    {
        int64_t base = (int64_t)tile - 1;
        for (;;) {
            const int64_t tt = base - lane;
            uint32_t st = ST_P;
            if (tt >= 0) {
                const uint32_t f = ld_acquire(&p.desc[tt].flag);
                st = (f & ~3u) == ep ? (f & 3u) : (uint32_t)ST_X;
            }
            const unsigned pm = __ballot_sync(0xFFFFFFFFu, st == ST_P);
            const unsigned xm = __ballot_sync(0xFFFFFFFFu, st == ST_X);
            const int fp = pm ? __ffs(pm) - 1 : 32;
            const unsigned before = fp >= 32 ? 0xFFFFFFFFu : ((1u << fp) - 1u);
            if (xm & before) {
                __nanosleep(64);
                continue;
            }
            if (fp < 32) {
                m = base - fp;
                break;
            }
            base -= 32;
        }
    }
    auto load_P = [&](int64_t tt) {
        const TileDesc *Dt = p.desc + tt;
        while (ld_acquire(&Dt->flag) != (ep | ST_P)) __nanosleep(64);
        const uint32_t pmask = __ldcg(&Dt->pmask);
        Ev = lane < KMAX && ((pmask >> lane) & 1u);
        if (lane < KMAX) {
            Es = __ldcg(&Dt->pstate[lane]);
            Ec = __ldcg(&Dt->pcnt[lane]);
        }
    };
    if (m < 0) {
        if (!p.keyed) {
            Ev = lane == 0;
            Es = start_state;
            Ec = start_count;
        } else {
            const uint32_t c = p.halo_byte;
            const uint32_t ni = min((uint32_t)__ldg(p.nimg + c), ksel);
            Ev = (uint32_t)lane < ni;
            Es = Ev ? (uint32_t)__ldg(p.lb + c * KMAX + lane) : 0u;
            Ec = 0;
        }
    } else {
        load_P(m);
    }
    // (2) apply the aggregates A_{m+1} .. A_{b-1}, 32 per step: every lane loads one tile's
    // aggregate in parallel, a warp suffix scan composes the 32 mappings (the same operator as
    // the chunk merge), and the composed window is applied to E.  A slot that breaks inside the
    // window (a tile-boundary miss, or a slot a tile published unresolved) is taken from that
    // tile's P, and the walk continues after it.
    for (int64_t nx = m + 1; nx < (int64_t)tile;) {
        const int64_t tt = nx + lane;
        uint32_t S2[K], e2[K], c2[K];
        bool id2 = tt >= (int64_t)tile;
        if (!id2) {
            const TileDesc *Dt = p.desc + tt;
            while ((ld_acquire(&Dt->flag) & ~3u) != ep) __nanosleep(32);
#pragma unroll
            for (int l = 0; l < K; l++) {
                const uint4 v = __ldcg(&Dt->aslot[l]);
                S2[l] = v.x;
                e2[l] = v.x == NOSTATE ? (ABSENT << 16) : (v.y | ((v.w ? (uint32_t)lane : COMPLETE) << 16));
                c2[l] = v.z;
            }
        } else {
#pragma unroll
            for (int l = 0; l < K; l++) S2[l] = NOSTATE, e2[l] = ABSENT << 16, c2[l] = 0;
        }
        warp_suffix_scan<K, HASH>(S2, e2, c2, id2, 0, 1, nullptr, nullptr, hs);
        int brk = 32;
        {
            uint32_t ne = 0, nc = 0;
            bool found = false;
#pragma unroll
            for (int l = 0; l < K; l++) {
                const uint32_t sl = __shfl_sync(0xFFFFFFFFu, S2[l], 0);
                const uint32_t el = __shfl_sync(0xFFFFFFFFu, e2[l], 0);
                const uint32_t cl = __shfl_sync(0xFFFFFFFFu, c2[l], 0);
                if (Ev && sl == Es) {
                    ne = el;
                    nc = cl;
                    found = true;
                }
            }
            if (Ev) {
                if (!found) brk = 0;
                else if ((ne >> 16) != COMPLETE) brk = (int)(ne >> 16);
                else {
                    Es = ne & 0xFFFFu;
                    Ec += nc;
                }
            }
        }
        const int mb = __reduce_min_sync(0xFFFFFFFFu, brk);
        if (mb < 32) {
            load_P(nx + mb);  // E := P of the tile where a slot broke (it resolves its own true path)
            nx = nx + mb + 1;
        } else {
            nx += 32;
        }
    }

    // own inclusive prefix P_b = E then A_b.  A tile-boundary miss (E's state is no speculated tile
    // start) resolves through chunk 0; a hit on a slot left unresolved resolves from its break.
    uint32_t Ps = 0;
    unsigned long long Pc = 0;
    ReCount rct{0, 0, 0, 0, 0xFFFFu};
    // the slot values live in lanes 0..K-1: fetch the hit slot's (qe, qc) with a full-warp shuffle
    int hit = -1;
    if (Ev) {
#pragma unroll
        for (int l = 0; l < K; l++)
            if (hit < 0 && Sj[l] == Es) hit = l;
    }
    const uint32_t hq = __shfl_sync(0xFFFFFFFFu, qe, hit < 0 ? 0 : hit);
    const uint32_t hc = __shfl_sync(0xFFFFFFFFu, qc, hit < 0 ? 0 : hit);
    if (Ev) {
        if (hit >= 0 && (hq >> 16) == COMPLETE) {
            Ps = hq & 0xFFFFu;
            Pc = Ec + hc;
        } else {
            uint32_t st, n;
            if (hit >= 0) resolve<K>(tb, t, hq & 0xFFFFu, hq >> 16, hc, st, n, rct);  // lazy R5 slot
            else resolve<K>(tb, t, Es, 0, 0, st, n, rct);                               // tile-boundary miss
            Ps = st;
            Pc = Ec + n;
            if (hit < 0) atomicAdd(&p.stats->boundary_misses, 1ull);
        }
    }
    const unsigned vmask = __ballot_sync(0xFFFFFFFFu, Ev);
    if (lane < KMAX) {
        D->pstate[lane] = Ps;
        D->pcnt[lane] = Pc;
    }
    if (lane == 0) D->pmask = vmask;
    __threadfence();
    __syncwarp();
    if (lane == 0) st_release(&D->flag, ep | ST_P);

    // counters: a pre-resolved slot is on the true path iff some valid prefix slot entered the
    // tile in its speculated start, or a tile-boundary re-execution joined it in chunk 0 (keyed
    // mode: every shard slot's path is needed)
    add_stats(p.stats, rct, true);
    if (__any_sync(0xFFFFFFFFu, rc5.chunks | rc5.eager)) {
        const uint32_t mine = lane < K ? (uint32_t)Sj[lane] : 0xFFFFFFFEu;
        bool needed = false;
#pragma unroll
        for (int q = 0; q < KMAX; q++) {
            const uint32_t eq = __shfl_sync(0xFFFFFFFFu, Es, q);
            const bool vq = __shfl_sync(0xFFFFFFFFu, (int)Ev, q) != 0;
            const uint32_t jq = __shfl_sync(0xFFFFFFFFu, rct.join0, q);
            needed = needed || (vq && (eq == mine || jq == (uint32_t)lane));
        }
        add_stats(p.stats, rc5, needed);
    }

    // a9: the last tile writes the result (bit-mode tail applied here)
    if (tile == p.ntiles - 1) {
        uint32_t x = Ps;
        unsigned long long cc = Pc;
        if (Ev && p.tail_bits) {
            const uint32_t tail_byte = __ldg(p.in + p.len);
            for (uint32_t i = 0; i < p.tail_bits; i++) {
                const uint32_t bit = (tail_byte >> (7 - i)) & 1u;
                const uint32_t en = __ldg(p.bittab + x * 2 + bit);
                x = en & 0xFFFFu;
                cc += en >> 16;
            }
        }
        DevResult *R = p.result;
        if (!p.keyed) {
            if (lane == 0) {
                R->final_state = x;  // internal id (chains pieces on the device)
                R->status = 0;
                R->count = cc;
                if (p.user_out) {
                    p.user_out[0] = p.inv ? __ldg(p.inv + x) : x;
                    p.user_out[1] = 0;
                    p.user_out[2] = (uint32_t)cc;
                    p.user_out[3] = (uint32_t)(cc >> 32);
                }
            }
        } else {
            const uint32_t c = p.halo_byte;
            const uint32_t ni = min((uint32_t)__ldg(p.nimg + c), ksel);
            if (lane < KMAX) {
                R->start[lane] = (uint32_t)lane < ni ? (uint32_t)__ldg(p.lb + c * KMAX + lane) : NOSTATE;
                R->end[lane] = x;
                R->mcount[lane] = cc;
            }
            if (lane == 0) {
                R->valid_mask = vmask;
                R->k = ksel;
                R->status = 0;
            }
        }
    }
}

// ------------------------------------------------------------------------------- the kernel --
// The body serves two kernels.  speck_kernel: one DFA, parameters in the kernel parameter space.
// speck_multi_kernel (NEXT-4, many FSMs over one resident input): M DFAs of the same
// table variant and K share one persistent grid and one ticket counter; ticket t is tile t / M of
// DFA t % M, so the M CTAs that run the same input tile for different DFAs run at about the same
// time and the tile is read from HBM once and from L2 M - 1 times.  Each DFA keeps its own
// descriptors (its own decoupled look-back), result and counters (pm[d]); a CTA reloads the table
// image into shared memory when its ticket switches DFA.
// SPLIT (speck_kernel with FSM_SPLIT): the last warp of the CTA is a dedicated epilogue warp; the
// other warps (T - 32 chunks per tile) hand each tile's state over in one of two buffers and go
// straight on to the next tile, so the serial epilogue (pre-resolution re-executions, look-back)
// overlaps the next tile's local phase instead of idling the SM at a barrier.
template <int K, int VAR, bool MULTI, bool SPLIT = false, bool HASH = false>
__device__ __forceinline__ void speck_body(const Params &p0, const Params *__restrict__ pm, uint32_t M)
{
    static_assert(!(MULTI && SPLIT), "multi-FSM runs use the unsplit body");
    static_assert(!HASH || K > 8, "Alg. 2 is instantiated for large k only (P:200)");
    using TB = typename TableFor<VAR>::type;
    extern __shared__ __align__(16) uint8_t smem[];  // no static shared memory: see kSmemWindowBase

    const uint32_t T = blockDim.x;
    const uint32_t TW = SPLIT ? T - 32 : T;  // chunks per tile
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, W = TW >> 5;
    const uint32_t j = threadIdx.x;

    // MULTI: p0.table_bytes is the group's largest table image, so one layout serves every DFA
    const Layout L(T, K, scratch_offset(VAR, p0.table_bytes), SPLIT, HASH);
    uint32_t *const hs = reinterpret_cast<uint32_t *>(smem + L.hs);  // Alg. 2 columns (HASH only)
    check_smem_window(VAR, L.total);
    TB tb;
    if (!MULTI) tb.setup(smem, p0.table, p0.n_states, kconst(p0));
    uint32_t *Qe = reinterpret_cast<uint32_t *>(smem + L.qe);
    uint32_t *Qc = reinterpret_cast<uint32_t *>(smem + L.qc);
    uint16_t *Sj = reinterpret_cast<uint16_t *>(smem + L.sj);
    uint32_t *wS = reinterpret_cast<uint32_t *>(smem + L.ws);
    uint32_t *wE = reinterpret_cast<uint32_t *>(smem + L.we);
    uint32_t *wC = reinterpret_cast<uint32_t *>(smem + L.wc);
    uint32_t *wI = reinterpret_cast<uint32_t *>(smem + L.wi);
    uint32_t &s_tile = *reinterpret_cast<uint32_t *>(smem + L.misc);
    uint32_t *Ext = reinterpret_cast<uint32_t *>(smem + L.ext);
    const uint32_t ntickets = MULTI ? p0.ntiles * M : p0.ntiles;
    uint32_t loaded = 0xFFFFFFFFu;  // MULTI: DFA whose table image is in shared memory
    uint32_t *s_tiles = &s_tile;    // SPLIT: one ticket slot per buffer

    if (SPLIT) __syncthreads();  // table setup done (every thread, before the roles split)
    if (SPLIT && warp == W) {
        // ---- the epilogue warp: tiles in ticket order, buffers alternating
        const uint32_t start_state = p0.start_dev ? p0.start_dev->final_state : p0.start_state;
        const unsigned long long start_count = p0.start_dev ? p0.start_dev->count : 0ull;
        named_arrive(4, T);
        named_arrive(5, T);
        for (uint32_t it = 0;; it++) {
            const uint32_t bb = it & 1u;
            named_sync(2 + bb, T);
            const uint32_t tile = s_tiles[bb];
            if (tile >= p0.ntiles) break;
            const uint32_t o = bb * L.buf;
            tile_epilogue<K, HASH>(tb, p0, tile, (uint64_t)tile * TW * p0.chunk, TW,
                                   reinterpret_cast<uint32_t *>(smem + L.qe + o), reinterpret_cast<uint32_t *>(smem + L.qc + o),
                                   reinterpret_cast<const uint16_t *>(smem + L.sj + o), nullptr,
                                   reinterpret_cast<const uint32_t *>(smem + L.ext + o), start_state, start_count, p0.k, hs);
            __syncwarp();
            named_arrive(4 + bb, T);
        }
        return;
    }

    for (uint32_t it = 0;; it++) {
        const uint32_t bb = SPLIT ? (it & 1u) : 0u;
        if (SPLIT) {
            named_sync(4 + bb, T);  // buffer bb free: the epilogue is done with tile it - 2
            if (threadIdx.x == 0) s_tiles[bb] = atomicAdd(p0.ticket, 1u) - p0.ticket_base;
            named_sync(1, TW);
            Qe = reinterpret_cast<uint32_t *>(smem + L.qe + bb * L.buf);
            Qc = reinterpret_cast<uint32_t *>(smem + L.qc + bb * L.buf);
            Sj = reinterpret_cast<uint16_t *>(smem + L.sj + bb * L.buf);
            Ext = reinterpret_cast<uint32_t *>(smem + L.ext + bb * L.buf);
        } else {
            __syncthreads();  // smem reuse across tiles; also orders the table setup
            if (threadIdx.x == 0) s_tile = atomicAdd(p0.ticket, 1u) - p0.ticket_base;
            __syncthreads();
        }
        const uint32_t ticket = s_tiles[bb];
        if (ticket >= ntickets) {
            if (SPLIT) named_arrive(2 + bb, T);  // tells the epilogue warp to stop
            break;
        }
        const uint32_t dfa = MULTI ? ticket % M : 0u;
        const uint32_t tile = MULTI ? ticket / M : ticket;
        const Params &p = MULTI ? pm[dfa] : p0;
        if (MULTI && dfa != loaded) {  // block-uniform
            tb.setup(smem, p.table, p.n_states, kconst(p));
            loaded = dfa;
            __syncthreads();
        }
        const uint32_t start_state = p.start_dev ? p.start_dev->final_state : p.start_state;
        const unsigned long long start_count = p.start_dev ? p.start_dev->count : 0ull;
        const uint32_t ksel = p.k;

        const uint64_t tile_base = (uint64_t)tile * TW * p.chunk;
        const uint64_t b0 = tile_base + (uint64_t)j * p.chunk;
        const uint64_t b = max(b0, (uint64_t)p.head);  // chunk 0 starts at the peeled head
        const bool first_chunk = tile == 0 && j == 0;
        const bool empty = b >= p.len && !first_chunk;
        const uint64_t e = b >= p.len ? b : min(b0 + p.chunk, p.len);

        // ---- a3: speculated start set (+ eager-completion candidates)
        uint32_t S[K], Xc[kExt];
        speculate<K>(tb, p, b, first_chunk, empty, start_state, S, Xc);

        // ---- a4: local processing
        uint32_t cur[K], acc[K], accf[K];
#pragma unroll
        for (int s = 0; s < K; s++) {
            cur[s] = tb.init(S[s] == NOSTATE ? (S[0] == NOSTATE ? 0u : S[0]) : S[s]);
            acc[s] = 0;
            accf[s] = 0;
        }
        uint32_t *const stash_j = SPLIT ? nullptr : reinterpret_cast<uint32_t *>(smem + L.stash) + j * 8;
        if (!empty && e > b) local_phase<K>(tb, p.in, b, e, p.aligned != 0, cur, acc, accf, stash_j);
        uint32_t eob[K], cnt[K];
#pragma unroll
        for (int s = 0; s < K; s++) {
            eob[s] = S[s] == NOSTATE ? (ABSENT << 16) : (tb.state_of(cur[s]) | (COMPLETE << 16));
            cnt[s] = tb.count_of(acc[s], accf[s], cur[s], empty ? 0 : e - b);
        }

        // ---- NEXT-3 eager completion (bounded): the next image states of the look-back symbol
        // beyond the k speculated ones run in lockstep with the k chains over the stashed first
        // 32 bytes; a state that meets a chain is recorded as (state, slot, count delta).
        {
            uint32_t ent[kExt];
#pragma unroll
            for (int q = 0; q < kExt; q++) ent[q] = kExtNone;
            if (p.eager_window && p.aligned && (b & 31) == 0 && !empty && e - b >= 32 && Xc[0] != NOSTATE) {
                uint32_t y[K], cy[K], u[kExt], cu[kExt];
                bool live[kExt];
#pragma unroll
                for (int l = 0; l < K; l++) {
                    y[l] = nat_init(tb, S[l] == NOSTATE ? 0u : S[l]);
                    cy[l] = 0;
                }
                int nlive = 0;
#pragma unroll
                for (int q = 0; q < kExt; q++) {
                    live[q] = Xc[q] != NOSTATE;
                    u[q] = nat_init(tb, live[q] ? Xc[q] : 0u);
                    cu[q] = 0;
                    nlive += live[q];
                }
                // window: the stashed first 32 bytes, then up to kExtWindow bytes from global (L2)
                const uint32_t wlen = (uint32_t)((e - b) < p.eager_window ? (e - b) : p.eager_window) & ~31u;
#pragma unroll 1
                for (uint32_t blk = 0; blk < wlen && nlive > 0; blk += 32) {
                    Bytes32 xb;
                    if (blk == 0 && stash_j) {
#pragma unroll
                        for (int q = 0; q < 8; q++) xb.w[q] = stash_j[q];
                    } else {
                        xb = ldg256(p.in + b + blk);
                    }
#pragma unroll 1
                    for (int pos = 0; pos < 32 && nlive > 0; pos++) {
                        const uint32_t byte = (xb.w[pos >> 2] >> (8 * (pos & 3))) & 0xFFu;
                        const typename TB::Row r = tb.row(byte);
#pragma unroll
                        for (int l = 0; l < K; l++) y[l] = nat_apply(tb, r, y[l], cy[l]);
#pragma unroll
                        for (int q = 0; q < kExt; q++) {
                            if (!live[q]) continue;
                            u[q] = nat_apply(tb, r, u[q], cu[q]);
#pragma unroll
                            for (int l = 0; l < K; l++)
                                if (live[q] && S[l] != NOSTATE && y[l] == u[q]) {
                                    live[q] = false;
                                    nlive--;
                                    ent[q] = Xc[q] | ((uint32_t)l << 16) | (((cu[q] - cy[l]) & 0xFFFu) << 20);
                                }
                        }
                    }
                }
            }
#pragma unroll
            for (int q = 0; q < kExt; q++) Ext[j * kExt + q] = ent[q];
        }
        bool ident = empty;

        // ---- a5: warp stage (chunks warp*32 .. warp*32+31)
        __syncwarp();  // the lanes' eager-completion entries are read by the scan
        warp_suffix_scan<K, HASH>(S, eob, cnt, ident, (uint32_t)warp * 32, 1, Ext,
                                  (p.dbg && tile == 0 && warp == 0) ? p.dbg : nullptr, hs);

        // ---- a6: block stage
        if (lane == 0) {
#pragma unroll
            for (int s = 0; s < K; s++) {
                wS[warp * K + s] = S[s];
                wE[warp * K + s] = eob[s];
                wC[warp * K + s] = cnt[s];
            }
            wI[warp] = ident;
        }
        if (SPLIT) named_sync(1, TW); else __syncthreads();
        if (warp == 0) {
            uint32_t S2[K], e2[K], c2[K];
            bool id2 = true;
            if (lane < W) {
#pragma unroll
                for (int s = 0; s < K; s++) {
                    S2[s] = wS[lane * K + s];
                    e2[s] = wE[lane * K + s];
                    c2[s] = wC[lane * K + s];
                }
                id2 = wI[lane] != 0;
            } else {
#pragma unroll
                for (int s = 0; s < K; s++) S2[s] = NOSTATE, e2[s] = ABSENT << 16, c2[s] = 0;
            }
            warp_suffix_scan<K, HASH>(S2, e2, c2, id2, 0, 32, Ext, nullptr, hs);
            __syncwarp();
            if (lane < W) {
#pragma unroll
                for (int s = 0; s < K; s++) {
                    wE[lane * K + s] = e2[s];
                    wC[lane * K + s] = c2[s];
                }
            }
        }
        if (SPLIT) named_sync(1, TW); else __syncthreads();
        if (warp + 1 < W && !ident && wI[warp + 1] == 0) {
            uint32_t Sr[K], er[K], cr[K];
#pragma unroll
            for (int s = 0; s < K; s++) {
                Sr[s] = wS[(warp + 1) * K + s];
                er[s] = wE[(warp + 1) * K + s];
                cr[s] = wC[(warp + 1) * K + s];
            }
            compose<K>(eob, cnt, Sr, er, cr, (uint32_t)(warp + 1) * 32, Ext);
        }
#pragma unroll
        for (int s = 0; s < K; s++) {
            Qe[j * K + s] = eob[s];
            Qc[j * K + s] = cnt[s];
            Sj[j * K + s] = (uint16_t)(S[s] == NOSTATE ? 0xFFFFu : S[s]);
        }
        if (SPLIT) {
            named_arrive(2 + bb, T);  // hand the tile over to the epilogue warp
            continue;
        }
        __syncthreads();

        if (warp != 0) continue;

        // ================= warp 0: tile epilogue (pre-resolution, look-back, publication) =====
        tile_epilogue<K, HASH>(tb, p, tile, tile_base, TW, Qe, Qc, Sj, reinterpret_cast<const uint32_t *>(smem + L.stash),
                               Ext, start_state, start_count, ksel, hs);
    }
}

// SPLIT is chosen per launch by the host: split_kernel(VAR, K) and the double-buffered layout fits.
template <int K, int VAR, bool SPLIT, bool HASH = false>
__global__ void __launch_bounds__(max_threads(K, VAR), min_blocks(K)) speck_kernel(Params p)
{
    speck_body<K, VAR, false, SPLIT, HASH>(p, nullptr, 1);
}

template <int K, int VAR>
__global__ void __launch_bounds__(max_threads(K, VAR), min_blocks(K))
    speck_multi_kernel(Params g, const Params *__restrict__ pm, uint32_t M)
{
    speck_body<K, VAR, true>(g, pm, M);
}

}  // namespace speck
