// fixup_kernel.cuh -- shard-boundary fix-up: the shard's true start x was not in
// its speculated set S_g.  One thread re-executes from the shard start in lockstep with the k
// speculated chains and stops when x's run equals one of them; from there both runs coincide,
// so the shard result for x is that slot's (end, count) corrected by the counts up to the meeting
// point (exact).  If no meeting happens within `limit` bytes the host re-runs the whole shard in
// known-start mode with the parallel kernel.
#pragma once
#include "speck_kernel.cuh"

namespace speck {

struct FixParams {
    const uint8_t *in;
    uint64_t len;          // whole bytes of the shard
    uint64_t limit;        // bytes to try before giving up
    const void *table;
    uint32_t n_states;
    uint32_t x;            // true start
    uint32_t k;
    uint32_t valid_mask;
    uint32_t start[KMAX];
    uint32_t end[KMAX];
    unsigned long long count[KMAX];
    unsigned long long *out;   // [0] = converged flag, [1] = end, [2] = count, [3] = bytes consumed
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
    if (threadIdx.x != 0) return;
    uint32_t y[KMAX], cy[KMAX];
    bool pres[KMAX];
#pragma unroll
    for (int l = 0; l < KMAX; l++) {
        pres[l] = (uint32_t)l < f.k && ((f.valid_mask >> l) & 1u);
        y[l] = pres[l] ? f.start[l] : 0u;
        cy[l] = 0;
    }
    uint32_t st = f.x, cx = 0, cyc = 0;
    int conv = -1;
    const uint64_t lim = min(f.len, f.limit);
    uint64_t pos = 0;
    while (conv < 0 && pos < lim) {
        const uint32_t byte = __ldg(f.in + pos);
        const typename TB::Row r = tb.row(byte);
        st = tb.apply(r, st, cx);
#pragma unroll
        for (int l = 0; l < KMAX; l++)
            if (pres[l]) y[l] = tb.apply(r, y[l], cy[l]);
#pragma unroll
        for (int l = 0; l < KMAX; l++)
            if (pres[l] && conv < 0 && y[l] == st) {
                conv = l;
                cyc = cy[l];
            }
        pos++;
    }
    if (conv >= 0) {
        unsigned long long e = 0, c = 0;
#pragma unroll
        for (int l = 0; l < KMAX; l++)
            if (l == conv) {
                e = f.end[l];
                c = f.count[l];
            }
        f.out[0] = 1;
        f.out[1] = e;
        f.out[2] = c + cx - cyc;
    } else {
        f.out[0] = 0;
    }
    f.out[3] = pos;
}

}  // namespace speck
