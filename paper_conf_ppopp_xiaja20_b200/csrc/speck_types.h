// speck_types.h -- structures shared by the host side (fsmspec.cu) and the kernels (speck_kernel.cuh).
#pragma once
#include <cstdint>

namespace speck {

constexpr int KMAX = 16;

// ---- slot encoding inside a mapping (the merge element) ---------------------------------------
// eob = state | brk << 16:  brk == COMPLETE : the run of this slot reaches the end of the range
//                           brk == ABSENT   : the slot holds no speculated state (|image| < k)
//                           otherwise       : the run breaks (no speculated match) when entering
//                                             chunk `brk` of the tile in state `state` -- the
//                                             paper's "invalid" slot plus where it broke.
constexpr uint32_t COMPLETE = 0xFFFFu;
constexpr uint32_t ABSENT = 0xFFFEu;
constexpr uint32_t NOSTATE = 0xFFFFu;  // start-set sentinel: never equal to a state id

enum Status : uint32_t { ST_X = 0, ST_A = 1, ST_P = 2 };

// One descriptor per tile for the decoupled look-back.  The flag carries the
// run epoch so descriptors never need clearing between runs.  A payload: the tile's aggregate
// mapping keyed on its first chunk's start set.  P payload: the inclusive prefix -- a mapping
// keyed on the shard's start set (one slot in known-start mode).
struct __align__(128) TileDesc {
    uint32_t flag;                 // epoch << 2 | Status
    uint32_t pmask;                // P: valid slots
    uint32_t pad[2];
    uint4 aslot[KMAX];             // A: {start (NOSTATE = absent), end, count within tile, broken}
                                   //    broken != 0: the slot's run breaks inside the tile (lazy R5):
                                   //    a successor whose path enters it waits for this tile's P
    uint32_t pstate[KMAX];         // P: state after this tile, per shard slot
    unsigned long long pcnt[KMAX]; // P: count up to and including this tile, per shard slot
};

// Re-execution counters of one run (reset by the host at the start of every API call).  A8: only
// chunks whose true start was not speculated should be re-executed; re-executions made for a
// tile-start candidate that turns out not to be on the true path (R5 pre-resolution) are counted
// apart.  In keyed (shard) mode every valid shard slot's path counts as "true".
struct DevStats {
    unsigned long long reexec_true;        // chunk re-executions on the true path
    unsigned long long reexec_true_bytes;  // bytes they consumed (early exit on convergence)
    unsigned long long reexec_cand;        // re-executions on tile-start candidate paths that were not taken
    unsigned long long reexec_cand_bytes;
    unsigned long long boundary_misses;    // tile-boundary misses (true start not a speculated tile start)
    unsigned long long eager_resolved;     // true-path misses completed from an eager-completion entry
    unsigned long long max_miss_chain;     // longest run of consecutive re-executed chunks on the true path
    unsigned long long pad;
};

// Per-slot re-execution tally of one resolve() call.
struct ReCount {
    uint32_t chunks, bytes, chain, eager;
    uint32_t join0;  // slot of chunk 0 that a re-execution starting at chunk 0 joined (0xFFFF = none)
};

// Result area written by the last tile.
struct DevResult {
    uint32_t final_state;   // known-start mode
    uint32_t status;
    unsigned long long count;
    // keyed mode: the shard map
    uint32_t valid_mask;
    uint32_t k;
    uint32_t start[KMAX];
    uint32_t end[KMAX];
    unsigned long long mcount[KMAX];
};

struct Params {
    const uint8_t *in;             // input bytes of this run (bit mode: packed bytes)
    uint64_t len;                  // whole bytes processed by the tiles
    uint32_t chunk;                // bytes per chunk (multiple of 32)
    uint32_t ntiles;
    uint32_t k;                    // speculated states in use (<= template K)
    uint32_t lookback;             // look-back window in bytes (0/1: the preceding byte only)
    const uint16_t *spec;          // window look-back: ranked candidates per chunk (spec_kernel), or null
    uint32_t spec_stride;          // candidates per chunk in `spec` (k + kExt)
    uint32_t aligned;              // `in` is 32-byte aligned (always, but for tiny debug chunks)
    uint32_t head;                 // the caller's input starts at in + head (0..31): an unaligned
                                   // input is run from the aligned address below it, chunk 0 being
                                   // [head, chunk); every position is relative to `in`, len included
    const void *table;             // variant image in global memory
    uint32_t n_states;             // internal states (incl. sink)
    uint32_t table_bytes;          // bytes of the shared-memory table image (0 for G)
    const uint16_t *lb;            // look-back table [256][KMAX]
    const uint8_t *nimg;           // min(|image(c)|, KMAX)
    TileDesc *desc;
    uint32_t *ticket;
    uint32_t ticket_base;
    uint32_t epoch;
    // start of the run
    uint32_t keyed;                // 0: known start; 1: keyed on S_g = LB[halo]
    uint32_t start_state;          // known start (ignored if start_dev)
    const DevResult *start_dev;    // optional: known start (final_state, count) from a previous piece
    uint32_t halo_byte;            // keyed mode
    // bit-mode tail (applied by the last tile)
    uint32_t tail_bits;            // the byte holding them is in[len]
    const uint32_t *bittab;        // [n_states][2]: next | acc << 16
    DevResult *result;
    DevStats *stats;
    // constants passed at run time so that ptxas cannot strength-reduce the FMA-pipe IMADs into
    // ALU-pipe shifts (the hot loop balances the two pipes): 1 << 24, 16, 512
    uint32_t k_1e24, k_16, k_512;
    const uint32_t *table_g;       // full u32 table (HS variant's cold rows)
    uint32_t hot_rows;             // HS variant: rows cached in shared memory
    const uint32_t *inv;           // internal -> user state ids (renumbered handles), or null
    uint32_t ncls, cl_magic;       // CL variant: byte classes and ceil(2^32 / row bytes) (state ids)
    uint32_t *user_out;            // optional: the last tile also writes {user state, 0, count lo, hi} here
    uint32_t eager_window;         // NEXT-3 eager completion: bytes of lockstep per chunk (0 = off)
    uint32_t k_4;                  // N8 variant: FMA-pipe constant 4, see k_1e24 above
    uint32_t preresolve;           // R5: tile-start slots (in rank order) resolved before publishing A
    uint32_t spec_all;             // test hook: `spec` also overrides chunk 0 of a known-start run
    uint4 *dbg;                    // test hook: warp-scan levels of tile 0, warp 0 ([6][32][KMAX]), or null
    // region counting (byte mode, accept-partitioned ids, host_tables.h renumber_by_accept): the
    // accept increment of a step into state q is [q >= nA] (R16, RG: rc_t = nA) or [R(q) >= R(nA)]
    // (CL's row addresses: rc_t = R(nA)); rc_comp: the high region is the NON-accepting one
    // (count = steps - that).
    uint32_t rc_t, rc_comp;
    uint32_t r_logl;               // RG variant: log2 of the lanes that share one table copy
    uint32_t lb_width;             // window look-back: image states run through the window (4..16)
};

}  // namespace speck
