// fixup_kernel.cuh -- shard-boundary fix-up: the shard's true start x was not in its
// speculated set S_g, so the shard map has no slot for it.  The delayed strategy re-executes
// only where x's own path is not covered; here the coverage is what the keyed run left behind in
// the tile descriptors (copied when the shard ran):
//   A_t  the aggregate of tile t keyed on its chunk-0 speculated starts (complete or broken slots)
//   P_t  the inclusive prefix after tile t of every valid shard slot's path
// One warp walks x's path tile by tile:
//   (1) at the start of tile t > 0, if x's state equals P_{t-1}[s] for a valid shard slot s, x's path
//       has joined slot s's path: the result is slot s's (end, count) corrected by the counts
//       (exact; done);
//   (2) else if the state is a speculated start of tile t with a complete aggregate slot, jump over
//       the tile with it;
//   (3) else re-execute tile t from its start: lane l < K runs A_t's chain l, the last lane runs x's
//       path, in lockstep byte by byte (the warp-parallel form of R3); when x's state equals a
//       chain whose aggregate slot is complete, both paths coincide to the tile's end, so x leaves
//       the tile with that slot's end and count + cnt_x(p) - cnt_l(p).
// Usually (1) holds at the end of tile 0: the fix-up touches one tile for a few bytes.  The walk
// stops after `limit` re-executed bytes (paths that never meet, e.g. permutation DFAs with k < N) and
// reports where it is; the host then runs the rest of the shard from that state with the parallel
// known-start kernel.
#pragma once
#include "speck_kernel.cuh"

namespace speck {

struct FixParams {
    const uint8_t *in;         // shard input (caller's pointer)
    uint64_t len;              // whole bytes of the shard
    uint32_t head;             // the keyed run's peeled head (tile t covers [t*tb - head, (t+1)*tb - head))
    uint64_t tile_bytes;       // bytes per tile of the keyed run (kernel coordinates)
    uint32_t ntiles;
    uint64_t limit;            // re-executed bytes to try before handing back to the host
    const TileDesc *desc;      // the keyed run's descriptors (copied at fsm_run_shard)
    const void *table;
    uint32_t n_states;
    uint32_t x;                // true start (internal id)
    uint32_t k;                // shard slots
    uint32_t kslots;           // aggregate slots per descriptor (the keyed run's instantiated K)
    uint32_t valid_mask;
    uint32_t end[KMAX];        // shard map (internal ids) and counts
    unsigned long long count[KMAX];
    uint32_t tail_bits;        // bit mode: trailing bits after the last whole byte (in[len])
    const uint32_t *bittab;
    unsigned long long *out;   // [0] = done, [1] = state, [2] = count, [3] = re-executed bytes, [4] = resume tile
    DevStats *stats;
    KConst kc;
};

template <int VAR>
__global__ void __launch_bounds__(kThreads) fixup_kernel(FixParams f)
{
    using TB = typename TableFor<VAR>::type;
    extern __shared__ __align__(16) uint8_t smem[];
    check_smem_window(VAR, scratch_offset(VAR, 0));
    TB tb;
    tb.setup(smem, f.table, f.n_states, f.kc);
    __syncthreads();
    if (threadIdx.x >= 32) return;
    const int lane = threadIdx.x;
    uint32_t y = f.x;
    unsigned long long cy = 0, rebytes = 0, retiles = 0;
    uint32_t t = 0;
    bool done = false;
    for (; t < f.ntiles && !done; t++) {
        const TileDesc &D = f.desc[t];
        if (t > 0) {  // (1) joined a shard slot's path at the tile boundary?
            const TileDesc &Pd = f.desc[t - 1];
            const bool v = lane < KMAX && ((f.valid_mask >> lane) & 1u) && ((Pd.pmask >> lane) & 1u) &&
                           Pd.pstate[lane] == y;
            const unsigned m = __ballot_sync(0xFFFFFFFFu, v);
            if (m) {
                const int s = __ffs(m) - 1;
                unsigned long long e = 0, c = 0, pc = 0;
#pragma unroll
                for (int l = 0; l < KMAX; l++)
                    if (l == s) {
                        e = f.end[l];
                        c = f.count[l];
                    }
                pc = Pd.pcnt[s];
                y = (uint32_t)e;
                cy += c - pc;
                done = true;
                break;
            }
        }
        // (2) pass through the tile with a complete aggregate slot
        uint4 a = make_uint4(NOSTATE, 0u, 0u, 1u);
        if ((uint32_t)lane < f.kslots) a = D.aslot[lane];  // slots >= K of a descriptor are stale
        const bool have = (uint32_t)lane < f.kslots && a.x != NOSTATE;
        const unsigned hm = __ballot_sync(0xFFFFFFFFu, have && a.w == 0u && a.x == y);
        if (hm) {
            const int l = __ffs(hm) - 1;
            y = __shfl_sync(0xFFFFFFFFu, a.y, l);
            cy += __shfl_sync(0xFFFFFFFFu, a.z, l);
            continue;
        }
        // (3) lockstep re-execution of tile t: lanes l < KMAX run the aggregate's chains, lane 31 runs y
        if (rebytes >= f.limit) break;
        const int64_t lo = max((int64_t)t * (int64_t)f.tile_bytes - (int64_t)f.head, (int64_t)0);
        const int64_t hi = min((int64_t)(t + 1) * (int64_t)f.tile_bytes - (int64_t)f.head, (int64_t)f.len);
        uint32_t st = lane == 31 ? y : (have ? a.x : 0u), cnt = 0;
        const bool chain = have && a.w == 0u;  // a chain whose aggregate slot is complete
        int64_t pos = lo;
        int conv = -1;
        retiles++;
        while (pos < hi) {
            const typename TB::Row r = tb.row(__ldg(f.in + pos));
            st = tb.apply(r, st, cnt);
            pos++;
            const uint32_t ys = __shfl_sync(0xFFFFFFFFu, st, 31);
            const unsigned cm = __ballot_sync(0xFFFFFFFFu, chain && st == ys);
            if (cm) {
                conv = __ffs(cm) - 1;
                break;
            }
        }
        rebytes += (unsigned long long)(pos - lo);
        const uint32_t cx = __shfl_sync(0xFFFFFFFFu, cnt, 31);
        if (conv >= 0) {
            const uint32_t cl = __shfl_sync(0xFFFFFFFFu, cnt, conv);
            y = __shfl_sync(0xFFFFFFFFu, a.y, conv);
            cy += (unsigned long long)cx - cl + __shfl_sync(0xFFFFFFFFu, a.z, conv);
        } else {
            y = __shfl_sync(0xFFFFFFFFu, st, 31);
            cy += cx;
        }
    }
    if (!done && t >= f.ntiles) {  // walked the whole shard: apply the bit-mode tail
        for (uint32_t i = 0; i < f.tail_bits; i++) {
            const uint32_t en = __ldg(f.bittab + y * 2 + ((__ldg(f.in + f.len) >> (7 - i)) & 1u));
            y = en & 0xFFFFu;
            cy += en >> 16;
        }
        done = true;
    }
    if (lane == 0) {
        f.out[0] = done ? 1ull : 0ull;
        f.out[1] = y;
        f.out[2] = cy;
        f.out[3] = rebytes;
        f.out[4] = t;
        if (retiles) {
            atomicAdd(&f.stats->reexec_true, retiles);
            atomicAdd(&f.stats->reexec_true_bytes, rebytes);
        }
    }
}

}  // namespace speck
