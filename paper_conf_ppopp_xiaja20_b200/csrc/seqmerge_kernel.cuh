// seqmerge_kernel.cuh -- the sequential-merge ablation (Fig. 4a).
//
// Same local phase as the parallel path (Alg. 3, same chunking and look-back), but every chunk
// writes its k-slot mapping to global memory and ONE thread then walks the chunks in order with
// the true state: a speculated match takes the chunk's ending state, otherwise the chunk is
// re-executed from the true state (same exact early-exit re-execution as the parallel path, so
// the two differ only in the merge).  The walking CTA prefetches the next batch of mappings into
// shared memory so the walk is bound by shared-memory latency, not HBM latency.  This is the
// merge the paper shows to be the scalability bottleneck.
#pragma once
#include "speck_kernel.cuh"

namespace speck {

struct SeqBuf {
    uint16_t *S;   // [nchunks][K]
    uint32_t *E;   // [nchunks][K]
    uint32_t *C;   // [nchunks][K]
};

template <int K, int VAR>
__global__ void __launch_bounds__(kThreads) seq_local_kernel(Params p, SeqBuf sb)
{
    using TB = typename TableFor<VAR>::type;
    extern __shared__ __align__(16) uint8_t smem[];
    check_smem_window(VAR, scratch_offset(VAR, p.table_bytes));
    TB tb;
    tb.setup(smem, p.table, p.n_states, kconst(p));
    __syncthreads();
    const uint64_t nch = p.len == 0 ? 1 : (p.len + p.chunk - 1) / p.chunk;
    const uint32_t start_state = p.start_dev ? p.start_dev->final_state : p.start_state;
    for (uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; g < nch; g += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t b = max(g * p.chunk, (uint64_t)p.head), e = min((g + 1) * p.chunk, p.len);
        uint32_t S[K], Xc[kExt];
        speculate<K>(tb, p, b, g == 0, false, start_state, S, Xc);
        uint32_t cur[K], acc[K], accf[K];
#pragma unroll
        for (int s = 0; s < K; s++) {
            cur[s] = tb.init(S[s] == NOSTATE ? (S[0] == NOSTATE ? 0u : S[0]) : S[s]);
            acc[s] = 0;
            accf[s] = 0;
        }
        if (e > b) local_phase<K>(tb, p.in, b, e, p.aligned != 0, cur, acc, accf);
#pragma unroll
        for (int s = 0; s < K; s++) {
            sb.S[g * K + s] = (uint16_t)(S[s] == NOSTATE ? 0xFFFFu : S[s]);
            sb.E[g * K + s] = tb.state_of(cur[s]);
            sb.C[g * K + s] = tb.count_of(acc[s], accf[s], cur[s], e - b);
        }
    }
}

template <int K, int VAR>
__global__ void __launch_bounds__(kThreads) seq_walk_kernel(Params p, SeqBuf sb)
{
    using TB = typename TableFor<VAR>::type;
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t T = blockDim.x;
    const uint32_t tb_bytes = scratch_offset(VAR, p.table_bytes);
    check_smem_window(VAR, tb_bytes + (uint32_t)(2 * T * K * 2 + 16 + 2 * 2 * T * K * 4));
    TB tb;
    tb.setup(smem, p.table, p.n_states, kconst(p));
    // double-buffered batches of T mappings
    uint16_t *bS = reinterpret_cast<uint16_t *>(smem + tb_bytes);            // [2][T][K]
    uint32_t *bE = reinterpret_cast<uint32_t *>(smem + tb_bytes + 2 * T * K * 2 + 16);
    uint32_t *bC = bE + 2 * T * K;
    const uint64_t nch = p.len == 0 ? 1 : (p.len + p.chunk - 1) / p.chunk;
    const uint64_t nbatch = (nch + T - 1) / T;
    auto load = [&](uint64_t batch, int buf) {
        const uint64_t g0 = batch * T;
        for (uint32_t i = threadIdx.x - 1; i < T * K; i += T - 1) {  // threads 1..T-1
            const uint64_t g = g0 + i / K;
            if (g < nch) {
                bS[buf * T * K + i] = sb.S[g0 * K + i];
                bE[buf * T * K + i] = sb.E[g0 * K + i];
                bC[buf * T * K + i] = sb.C[g0 * K + i];
            }
        }
    };
    load(0, 0);
    __syncthreads();
    uint32_t x = p.start_dev ? p.start_dev->final_state : p.start_state;
    unsigned long long total = p.start_dev ? p.start_dev->count : 0ull;
    unsigned long long reexec = 0, rebytes = 0, maxchain = 0, chain = 0;
    for (uint64_t batch = 0; batch < nbatch; batch++) {
        const int buf = batch & 1;
        if (threadIdx.x != 0) {
            if (batch + 1 < nbatch) load(batch + 1, buf ^ 1);
        } else {
            const uint64_t g0 = batch * T;
            const uint32_t n = (uint32_t)((nch - g0) < T ? (nch - g0) : T);
            for (uint32_t i = 0; i < n; i++) {
                const uint16_t *Sg = bS + buf * T * K + i * K;
                int hit = -1;
#pragma unroll
                for (int l = 0; l < K; l++)
                    if (Sg[l] == x) hit = l;
                if (hit >= 0) {
                    total += bC[buf * T * K + i * K + hit];
                    x = bE[buf * T * K + i * K + hit];
                    chain = 0;
                    continue;
                }
                // re-execute the chunk from the true state (Fig. 4a), early exit on convergence
                const uint64_t b = max((g0 + i) * p.chunk, (uint64_t)p.head), e = min((g0 + i + 1) * p.chunk, p.len);
                uint32_t y[K], cy[K];
                bool pres[K];
#pragma unroll
                for (int l = 0; l < K; l++) {
                    pres[l] = Sg[l] != 0xFFFFu;
                    y[l] = pres[l] ? Sg[l] : 0u;
                    cy[l] = 0;
                }
                uint32_t cx = 0, cyc = 0;
                int conv = -1;
                uint64_t pos = b;
                const uint64_t wend = min(e, b + kLockstepWindow);
                while (conv < 0 && pos < wend) {
                    const typename TB::Row r = tb.row(__ldg(p.in + pos));
                    x = tb.apply(r, x, cx);
#pragma unroll
                    for (int l = 0; l < K; l++) y[l] = tb.apply(r, y[l], cy[l]);
#pragma unroll
                    for (int l = 0; l < K; l++)
                        if (pres[l] && conv < 0 && y[l] == x) {
                            conv = l;
                            cyc = cy[l];
                        }
                    pos++;
                }
                for (; conv < 0 && pos < e; pos++) x = tb.apply(tb.row(__ldg(p.in + pos)), x, cx);  // alone
                reexec++;
                rebytes += pos - b;
                chain++;  // consecutive re-executed chunks (reset by a speculated hit)
                maxchain = chain > maxchain ? chain : maxchain;
                if (conv >= 0) {
                    total += (unsigned long long)cx - cyc + bC[buf * T * K + i * K + conv];
                    x = bE[buf * T * K + i * K + conv];
                } else {
                    total += cx;
                }
            }
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        const uint32_t tail_byte = p.tail_bits ? __ldg(p.in + p.len) : 0u;
        for (uint32_t i = 0; i < p.tail_bits; i++) {
            const uint32_t en = __ldg(p.bittab + x * 2 + ((tail_byte >> (7 - i)) & 1u));
            x = en & 0xFFFFu;
            total += en >> 16;
        }
        p.result->final_state = x;
        p.result->status = 0;
        p.result->count = total;
        if (p.user_out) {
            p.user_out[0] = p.inv ? __ldg(p.inv + x) : x;
            p.user_out[1] = 0;
            p.user_out[2] = (uint32_t)total;
            p.user_out[3] = (uint32_t)(total >> 32);
        }
        atomicAdd(&p.stats->reexec_true, reexec);  // the walker follows the true path only
        atomicAdd(&p.stats->reexec_true_bytes, rebytes);
        atomicMax(&p.stats->max_miss_chain, maxchain);
    }
}

inline size_t seq_walk_smem(uint32_t T, int K, int var, uint32_t table_bytes)
{
    return scratch_offset(var, table_bytes) + 2 * T * K * 2 + 16 + 2 * 2 * T * K * 4;
}

}  // namespace speck
