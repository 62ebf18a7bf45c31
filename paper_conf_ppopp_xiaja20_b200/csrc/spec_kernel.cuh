// spec_kernel.cuh -- a3 look-back speculation with a window (reading R7), as a pre-pass.
//
// For every chunk (start byte b): the image of x[b-Lw-1] (the host look-back table; its top
// lb_width states by preimage count when the option narrows the walk) is run
// through the Lw bytes x[b-Lw .. b) and the reached states are ranked by multiplicity (how many
// image states reach each), ties to the smaller (user) id; the top k + kExt distinct states are written
// to spec[chunk][0 .. k + kExt) (0xFFFF = none).  Chunks whose window would reach before the start
// of a known-start run get the single exact state; keyed runs and short prefixes fall back to the
// depth-1 look-back.  One thread per chunk; the fused kernel then only reads its chunk's list.
// Kept out of the fused kernel so its 16-chain working set does not raise the hot loop's register
// allocation.
#pragma once
#include "speck_kernel.cuh"

namespace speck {

constexpr int kSpecThreads = 1024;  // one CTA per SM when the table image fills shared memory

template <int VAR>
__global__ void __launch_bounds__(kSpecThreads) spec_kernel(Params p, uint16_t *__restrict__ spec)
{
    using TB = typename TableFor<VAR>::type;
    extern __shared__ __align__(16) uint8_t smem[];
    check_smem_window(VAR, scratch_offset(VAR, p.table_bytes));
    TB tb;
    tb.setup(smem, p.table, p.n_states, kconst(p));
    __syncthreads();
    const uint64_t nch = p.len == 0 ? 1 : (p.len + p.chunk - 1) / p.chunk;
    const uint32_t ksel = p.k, stride = p.spec_stride, Lw = p.lookback;
    const uint32_t start_state = p.start_dev ? p.start_dev->final_state : p.start_state;
    for (uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; g < nch; g += (uint64_t)gridDim.x * blockDim.x) {
        uint16_t *out = spec + g * stride;
        const uint64_t b = max(g * p.chunk, (uint64_t)p.head);
        uint32_t written = 0;
        if (g == 0 && !p.keyed) {
            out[written++] = (uint16_t)start_state;
        } else if (b >= Lw + 1 + p.head && p.aligned) {
            const uint32_t c0 = __ldg(p.in + b - Lw - 1);
            const uint32_t ni = min((uint32_t)__ldg(p.nimg + c0), p.lb_width);  // the top lb_width (A5 rank)
            // the image chains run in the table variant's own hot-loop form (its step(), on groups of
            // 4 chains, only as many groups as the image has states); ids are recovered at the end
            uint32_t cur[KMAX / 4][4], acc[KMAX / 4][4], accf[KMAX / 4][4];
#pragma unroll
            for (int q0 = 0; q0 < KMAX / 4; q0++)
#pragma unroll
                for (int i = 0; i < 4; i++) {
                    const int ii = q0 * 4 + i;
                    cur[q0][i] = tb.init((uint32_t)__ldg(p.lb + c0 * KMAX + ((uint32_t)ii < ni ? ii : 0)));
                    acc[q0][i] = accf[q0][i] = 0;
                }
            // the next window block is in flight while this one is stepped (one HBM latency per
            // window instead of one per 32 bytes)
            Bytes32 xn = ldg256(p.in + b - Lw);
            for (uint32_t o = 0; o < Lw; o += 32) {
                const Bytes32 x = xn;
                if (o + 32 < Lw) xn = ldg256(p.in + b - Lw + o + 32);
#pragma unroll
                for (int q = 0; q < 8; q++) {
#pragma unroll
                    for (int j = 0; j < 4; j++)
#pragma unroll
                        for (int q0 = 0; q0 < KMAX / 4; q0++)
                            if ((uint32_t)(q0 * 4) < ni) tb.template step<4>(x.w[q], j, cur[q0], acc[q0], accf[q0]);
                }
            }
            uint32_t y[KMAX];
#pragma unroll
            for (int q0 = 0; q0 < KMAX / 4; q0++)
#pragma unroll
                for (int i = 0; i < 4; i++) y[q0 * 4 + i] = tb.state_of(cur[q0][i]);
            uint32_t mult[KMAX];
#pragma unroll
            for (int i = 0; i < KMAX; i++) {
                uint32_t m = 0;
#pragma unroll
                for (int j = 0; j < KMAX; j++) m += ((uint32_t)j < ni && y[j] == y[i]) ? 1u : 0u;
                mult[i] = (uint32_t)i < ni ? m : 0u;
            }
            // ties go to the smaller USER id (as in the host look-back table, reading A5)
            uint32_t uy[KMAX];
#pragma unroll
            for (int i = 0; i < KMAX; i++) uy[i] = p.inv ? __ldg(p.inv + y[i]) : y[i];
            // selection: repeatedly take the best remaining (multiplicity desc, user id asc)
            for (; written < stride; written++) {
                uint32_t bm = 0, bs = NOSTATE, bu = 0xFFFFFFFFu;
#pragma unroll
                for (int i = 0; i < KMAX; i++)
                    if (mult[i] > bm || (mult[i] == bm && mult[i] && uy[i] < bu)) {
                        bm = mult[i];
                        bs = y[i];
                        bu = uy[i];
                    }
                if (!bm) break;
#pragma unroll
                for (int i = 0; i < KMAX; i++)
                    if (y[i] == bs) mult[i] = 0;
                out[written] = (uint16_t)bs;
            }
        } else if (!p.keyed && b <= Lw + p.head) {
            // the window would reach the start of a known-start run: the exact state (at most Lw
            // bytes from the start)
            uint32_t st = start_state, dummy = 0;
            for (uint64_t t = p.head; t < b; t++) st = tb.apply(tb.row(__ldg(p.in + t)), st, dummy);
            out[written++] = (uint16_t)st;
        } else {
            const uint32_t c = g == 0 ? p.halo_byte : (uint32_t)__ldg(p.in + b - 1);
            const uint32_t ni = min((uint32_t)__ldg(p.nimg + c), stride);
            for (; written < ni; written++) out[written] = __ldg(p.lb + c * KMAX + written);
        }
        // the first k entries are the speculated set, the rest eager-completion candidates
        (void)ksel;
        for (; written < stride; written++) out[written] = 0xFFFFu;
    }
}

}  // namespace speck
