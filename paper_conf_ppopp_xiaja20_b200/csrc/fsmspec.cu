// fsmspec.cu -- libfsmspec: the C ABI of include/fsmspec.h over the sm_100a kernels.
//
// Host responsibilities only: validation, preprocessing at create (host_tables.h), geometry,
// kernel dispatch, result/stat transfer.  Every step of the hot path runs in the kernels of
// speck_kernel.cuh / fixup_kernel.cuh / seqmerge_kernel.cuh; there is no CPU fallback.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>

#include "../../include/fsmspec.h"
#include "fixup_kernel.cuh"
#include "host_tables.h"
#include "seqmerge_kernel.cuh"
#include "spec_kernel.cuh"
#include "speck_kernel.cuh"

using namespace speck;

// ------------------------------------------------------------------ kernel instantiations ----
// k is a compile-time constant; a run with k uses the smallest instantiated K >= k and
// marks the extra slots absent (kernels_inst.cuh instantiates the same list).
static const int kKs[] = {1, 2, 3, 4, 6, 8, 12, 16};
constexpr int kNumKs = 8;

typedef void (*KernelFn)(Params);
typedef void (*FixFn)(FixParams);
typedef void (*SeqLocalFn)(Params, SeqBuf);
typedef void (*SeqWalkFn)(Params, SeqBuf);
typedef void (*SpecFn)(Params, uint16_t *);
typedef void (*MultiFn)(Params, const Params *, uint32_t);

// Kernel instantiations live in one translation unit per table variant (kernels_*.cu, compiled in
// parallel); each exports these accessors.
#define FSM_DECLARE_VARIANT(NAME)                                   \
    KernelFn get_kernel_##NAME(int K, bool split, bool hash);       \
    MultiFn get_multi_##NAME(int K);                                \
    FixFn get_fix_##NAME();                                         \
    void get_seq_##NAME(int K, SeqLocalFn &l, SeqWalkFn &w);       \
    SpecFn get_spec_##NAME();
FSM_DECLARE_VARIANT(p4)
FSM_DECLARE_VARIANT(p8)
FSM_DECLARE_VARIANT(b)
FSM_DECLARE_VARIANT(g)
FSM_DECLARE_VARIANT(hs)
FSM_DECLARE_VARIANT(cl)
FSM_DECLARE_VARIANT(n8)
FSM_DECLARE_VARIANT(r16)
FSM_DECLARE_VARIANT(rg)

static KernelFn get_kernel(int var, int K, bool split, bool hash)
{
    switch (var) {
    case VAR_P4: return get_kernel_p4(K, split, hash);
    case VAR_P8: return get_kernel_p8(K, split, hash);
    case VAR_HS: return get_kernel_hs(K, split, hash);
    case VAR_CL: return get_kernel_cl(K, split, hash);
    case VAR_N8: return get_kernel_n8(K, split, hash);
    case VAR_R16: return get_kernel_r16(K, split, hash);
    case VAR_RG: return get_kernel_rg(K, split, hash);
    case VAR_B: return get_kernel_b(K, split, hash);
    default: return get_kernel_g(K, split, hash);
    }
}
static MultiFn get_multi(int var, int K)
{
    switch (var) {
    case VAR_P4: return get_multi_p4(K);
    case VAR_P8: return get_multi_p8(K);
    case VAR_HS: return get_multi_hs(K);
    case VAR_CL: return get_multi_cl(K);
    case VAR_N8: return get_multi_n8(K);
    case VAR_R16: return get_multi_r16(K);
    case VAR_RG: return get_multi_rg(K);
    case VAR_B: return get_multi_b(K);
    default: return get_multi_g(K);
    }
}
static FixFn get_fix(int var)
{
    switch (var) {
    case VAR_P4: return get_fix_p4();
    case VAR_P8: return get_fix_p8();
    case VAR_HS: return get_fix_hs();
    case VAR_CL: return get_fix_cl();
    case VAR_N8: return get_fix_n8();
    case VAR_R16: return get_fix_r16();
    case VAR_RG: return get_fix_rg();
    case VAR_B: return get_fix_b();
    default: return get_fix_g();
    }
}
static SpecFn get_spec(int var)
{
    switch (var) {
    case VAR_P4: return get_spec_p4();
    case VAR_P8: return get_spec_p8();
    case VAR_HS: return get_spec_hs();
    case VAR_CL: return get_spec_cl();
    case VAR_N8: return get_spec_n8();
    case VAR_R16: return get_spec_r16();
    case VAR_RG: return get_spec_rg();
    case VAR_B: return get_spec_b();
    default: return get_spec_g();
    }
}
static void get_seq(int var, int K, SeqLocalFn &l, SeqWalkFn &w)
{
    switch (var) {
    case VAR_P4: get_seq_p4(K, l, w); break;
    case VAR_P8: get_seq_p8(K, l, w); break;
    case VAR_HS: get_seq_hs(K, l, w); break;
    case VAR_CL: get_seq_cl(K, l, w); break;
    case VAR_N8: get_seq_n8(K, l, w); break;
    case VAR_R16: get_seq_r16(K, l, w); break;
    case VAR_RG: get_seq_rg(K, l, w); break;
    case VAR_B: get_seq_b(K, l, w); break;
    default: get_seq_g(K, l, w); break;
    }
}

static int kslots(uint32_t k)
{
    for (int i = 0; i < kNumKs; i++)
        if (kKs[i] >= (int)k) return kKs[i];
    return 16;
}

// ------------------------------------------------------------------------------ the handle ----
struct fsm {
    int device = 0;
    int num_sms = 148;
    cudaStream_t stream = nullptr;
    cudaStream_t copy_stream = nullptr;
    uint32_t n_user = 0, alphabet = 0, start = 0, mode = 0;
    ByteDFA dfa;
    int auto_variant = VAR_G;
    bool permutation = false;  // every in-alphabet symbol permutes the states: paths never meet
    fsm_options opt{};
    // device tables
    void *d_img[10] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
    uint32_t img_bytes[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
    uint32_t ncls = 0, cl_magic = 0;  // CL variant
    uint32_t rc_comp = 0;                // region counting (byte mode, accept-partitioned ids)
    uint32_t r_logl = 0;                 // RG: log2 of the lanes sharing one table copy
    uint32_t rc_nA = 0, cl_rc_t = 0;     // ids [0, nA) count 0 (1 if rc_comp); CL: R(nA), the row address
    // static-frequency renumbering (hot-state caching): user <-> internal ids
    bool renumbered = false;
    std::vector<uint32_t> perm, inv;
    uint32_t *d_inv = nullptr;
    uint32_t hot_rows = 0;
    uint32_t start_int = 0;
    uint16_t *d_lb = nullptr;
    uint8_t *d_nimg = nullptr;
    uint32_t *d_bittab = nullptr;
    // run state
    TileDesc *d_desc = nullptr;
    size_t desc_cap = 0;
    uint32_t *d_ticket = nullptr;
    uint32_t ticket_base = 0;
    uint32_t epoch = 0;
    DevResult *d_result = nullptr;   // [0] = run result, [1] = scratch for chained pieces
    DevStats *d_stats = nullptr;
    DevResult *h_result = nullptr;   // pinned
    DevStats *h_stats = nullptr;     // pinned
    unsigned long long *d_fix = nullptr;
    // e2e staging
    uint8_t *d_stage[2] = {nullptr, nullptr};
    size_t stage_bytes = 0;
    cudaEvent_t ev_copied[2] = {nullptr, nullptr}, ev_used[2] = {nullptr, nullptr};
    // look-back window pre-pass output
    uint16_t *d_spec = nullptr;
    size_t spec_cap = 0;
    // multi-FSM groups led by this handle: per-DFA Params in device memory
    Params *d_multi = nullptr;
    size_t multi_cap = 0;
    // sequential-merge ablation buffers
    SeqBuf seq{};
    size_t seq_cap = 0;
    // geometry / configuration of the most recent run (the counters are read from d_stats)
    fsm_stats last{};
    uint32_t last_head = 0;  // peeled head of the most recent run (kernel coordinates)
    // test hook (fsm_debug_set_spec): fixed chunk bytes, injected sets, merge-tree readback
    uint32_t dbg_chunk = 0, dbg_n = 0, dbg_k = 0;
    uint16_t *d_dbg_spec = nullptr;
    uint4 *d_dbg = nullptr;
    // hex lookback for host queries
    std::vector<uint16_t> lb;
    std::vector<uint8_t> nimg;
};

struct fsm_shard {
    const uint8_t *input = nullptr;
    uint64_t len = 0;          // symbols
    uint32_t k = 0;
    int variant = 0;           // the table variant the shard ran with (the fix-up uses the same)
    fsm_shard_map map{};
    // keyed runs: the tile descriptors (aggregates A_t, prefixes P_t) the fix-up walks
    TileDesc *d_desc = nullptr;
    uint32_t ntiles = 0, head = 0, kslots = 0;
    uint64_t tile_bytes = 0;
};

#define CK(x)                                                  \
    do {                                                       \
        cudaError_t _e = (x);                                  \
        if (_e != cudaSuccess) return cuda_status(_e);         \
    } while (0)

static int cuda_status(cudaError_t e)
{
    if (e == cudaErrorMemoryAllocation) return FSM_ENOMEM;
    if (getenv("FSM_DEBUG")) fprintf(stderr, "fsmspec: CUDA error %s\n", cudaGetErrorString(e));
    return FSM_ECUDA;
}

extern "C" const char *fsm_strerror(int status)
{
    switch (status) {
    case FSM_OK: return "ok";
    case FSM_EINVAL: return "invalid argument";
    case FSM_ENOMEM: return "out of memory";
    case FSM_ECUDA: return "CUDA error";
    case FSM_ESYMBOL: return "input symbol outside the alphabet";
    case FSM_EUNSUPPORTED: return "unsupported device (sm_100 required)";
    default: return "unknown status";
    }
}

extern "C" const char *fsm_version(void) { return "fsmspec 0.1 (sm_100a)"; }

extern "C" int fsm_lookback_table(const uint32_t *table, uint32_t n_states, uint32_t alphabet, uint32_t input_mode,
                                  uint16_t *lb_out, uint8_t *nimg_out)
{
    if (!table || !lb_out || !nimg_out || n_states == 0 || alphabet == 0 || alphabet > 256) return FSM_EINVAL;
    if (input_mode == FSM_INPUT_BITS_MSB && alphabet != 2) return FSM_EINVAL;
    for (size_t i = 0; i < (size_t)n_states * alphabet; i++)
        if (table[i] >= n_states) return FSM_EINVAL;
    ByteDFA d;
    build_byte_dfa(table, n_states, alphabet, nullptr, input_mode == FSM_INPUT_BITS_MSB, d);
    build_lookback(d, lb_out, nimg_out);
    return FSM_OK;
}

extern "C" int fsm_hot_state_order(const uint32_t *table, uint32_t n_states, uint32_t alphabet, uint32_t input_mode,
                                   uint32_t *order_out)
{
    if (!table || !order_out || n_states == 0 || alphabet == 0 || alphabet > 256) return FSM_EINVAL;
    if (input_mode == FSM_INPUT_BITS_MSB && alphabet != 2) return FSM_EINVAL;
    for (size_t i = 0; i < (size_t)n_states * alphabet; i++)
        if (table[i] >= n_states) return FSM_EINVAL;
    ByteDFA d;
    build_byte_dfa(table, n_states, alphabet, nullptr, input_mode == FSM_INPUT_BITS_MSB, d);
    std::vector<uint32_t> perm, inv;
    renumber_by_frequency(d, n_states, perm, inv);
    for (uint32_t r = 0; r < n_states; r++) order_out[r] = inv[r];
    return FSM_OK;
}

static void free_all(fsm *f)
{
    for (int i = 0; i < 10; i++) cudaFree(f->d_img[i]);
    cudaFree(f->d_inv);
    cudaFree(f->d_lb);
    cudaFree(f->d_nimg);
    cudaFree(f->d_bittab);
    cudaFree(f->d_desc);
    cudaFree(f->d_ticket);
    cudaFree(f->d_result);
    cudaFree(f->d_stats);
    cudaFree(f->d_fix);
    cudaFree(f->d_stage[0]);
    cudaFree(f->d_stage[1]);
    cudaFree(f->d_spec);
    cudaFree(f->d_multi);
    cudaFree(f->d_dbg_spec);
    cudaFree(f->d_dbg);
    cudaFree(f->seq.S);
    cudaFree(f->seq.E);
    cudaFree(f->seq.C);
    if (f->h_result) cudaFreeHost(f->h_result);
    if (f->h_stats) cudaFreeHost(f->h_stats);
    for (int i = 0; i < 2; i++) {
        if (f->ev_copied[i]) cudaEventDestroy(f->ev_copied[i]);
        if (f->ev_used[i]) cudaEventDestroy(f->ev_used[i]);
    }
    if (f->copy_stream) cudaStreamDestroy(f->copy_stream);
}

template <class T>
static int upload(T **dptr, const void *src, size_t bytes)
{
    void *p = nullptr;
    CK(cudaMalloc(&p, bytes ? bytes : 16));
    if (bytes) CK(cudaMemcpy(p, src, bytes, cudaMemcpyHostToDevice));
    *dptr = static_cast<T *>(p);
    return FSM_OK;
}

extern "C" int fsm_create_ex(const uint32_t *table, uint32_t n_states, uint32_t alphabet, uint32_t start,
                             const uint8_t *accept_mask, uint32_t input_mode, fsm_t **out)
{
    if (!table || !out || n_states == 0 || n_states > 65535 || alphabet == 0 || alphabet > 256 || start >= n_states)
        return FSM_EINVAL;
    if (input_mode != FSM_INPUT_BYTES && input_mode != FSM_INPUT_BITS_MSB) return FSM_EINVAL;
    const bool bits = input_mode == FSM_INPUT_BITS_MSB;
    if (bits && alphabet != 2) return FSM_EINVAL;
    if (!bits && alphabet < 256 && n_states >= 65535) return FSM_EINVAL;  // the sink needs an id < 0xFFFF
    for (size_t i = 0; i < (size_t)n_states * alphabet; i++)
        if (table[i] >= n_states) return FSM_EINVAL;

    int dev = 0;
    CK(cudaGetDevice(&dev));
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, dev));
    if (prop.major != 10) return FSM_EUNSUPPORTED;

    fsm *f = new (std::nothrow) fsm();
    if (!f) return FSM_ENOMEM;
    f->device = dev;
    f->num_sms = prop.multiProcessorCount;
    f->n_user = n_states;
    f->alphabet = alphabet;
    f->start = start;
    f->mode = input_mode;
    build_byte_dfa(table, n_states, alphabet, accept_mask, bits, f->dfa);
    f->start_int = start;
    // the look-back table ranks in user ids (reading A5: ties -> the smaller user id), then is
    // mapped to the internal ids below
    f->lb.resize(256 * KMAX);
    f->nimg.resize(256);
    build_lookback(f->dfa, f->lb.data(), f->nimg.data());
    if (!bits && f->dfa.n > 256 && f->dfa.n <= 32768) {
        // tables beyond shared memory: hot-state caching needs hot rows = small ids (Sec. 4.2)
        renumber_by_frequency(f->dfa, n_states, f->perm, f->inv);
        f->renumbered = true;
    } else if (!bits && f->dfa.n <= 256) {
        // region counting (R16, CL): accept increments become a function of the destination id
        uint32_t nA = 0;
        bool comp = false;
        renumber_by_accept(f->dfa, n_states, accept_mask, f->perm, f->inv, nA, comp);
        f->renumbered = true;
        f->rc_nA = nA;
        f->rc_comp = comp ? 1u : 0u;
    }
    if (f->renumbered) {
        f->start_int = f->perm[start];
        for (auto &v : f->lb)
            if (v != 0xFFFFu) v = (uint16_t)f->perm[v];
    }
    {   // paths of a DFA whose every symbol is a bijection never converge (R5 default below)
        bool perm = true;
        const uint32_t ncols = bits ? 256u : alphabet;
        std::vector<uint8_t> seen(f->dfa.n);
        for (uint32_t c = 0; c < ncols && perm; c++) {
            std::fill(seen.begin(), seen.end(), 0);
            for (uint32_t s = 0; s < n_states && perm; s++) {
                const uint32_t t = f->dfa.next[(size_t)s * 256 + c];
                if (t >= n_states || seen[t]) perm = false;
                else seen[t] = 1;
            }
        }
        f->permutation = perm;
    }
    const uint32_t n = f->dfa.n;
    // N > 256: the u32 table in L2 with the L1 acting as a hardware hot-row cache (G) measured faster
    // up to ~2K states (1027-state AC: 1.12 vs 0.98 TB/s); beyond that explicit hot-state caching in
    // shared memory wins (4121-state AC: 0.90 vs 0.76 TB/s).  Both use the frequency renumbering.
    // N <= 8 in byte mode: N8 (4-bit fields, one LDS.32 per byte, batched DP4A counts) measured
    // +15..28 % over P8 (LDS.64-bound) on (8, m, k) DFAs; P4 stays ahead for N <= 4; bit mode has
    // up to 8 accepts per byte, which N8's 1-bit count field cannot hold, so it keeps P8.
    // 8 < N <= 16: R16 (lane-replicated byte entries, conflict-free LDS.U8) measured +23..38 % over B
    // (random-bank LDS.U16): (16, 2, k=2) 2265 -> 3034, (16, 1, k=1) 2341 -> 3224 GB/s.
    // 16 < N <= 256 in byte mode: RG (R16's layout in fewer copies, bank-conflict degree of 2^logl
    // lanes instead of 32) measured +2..24 % over B: (24, 2) 2254 -> 2752, (32, 3) 2186 -> 2685,
    // (64, 4) 1908 -> 2180, (255, 2) 2225 -> 2270 GB/s.
    f->auto_variant = (n <= 4 && !bits) ? VAR_P4 : (n <= 8 && !bits) ? VAR_N8 : n <= 8 ? VAR_P8 : (n <= 16 && !bits) ? VAR_R16
                    : (n <= 256 && !bits) ? VAR_RG : n <= 256 ? VAR_B
                    : (f->renumbered && n > 2048) ? VAR_HS : VAR_G;
    f->opt.chunk_bytes = 0;
    f->opt.threads_per_tile = 0;  // auto: max_threads(K)
    f->opt.variant = FSM_VARIANT_AUTO;
    f->opt.merge = FSM_MERGE_PARALLEL;
    f->opt.ctas_per_sm = 0;

    int rc = FSM_OK;
    auto fail = [&](int r) {
        free_all(f);
        delete f;
        return r;
    };
    // every variant the DFA fits, so that tests can force any of them
    if (n <= 4 && !bits) {  // P4's count encoding is byte-mode only (count 0/1)
        auto img = image_packed(f->dfa, false);
        if ((rc = upload(&f->d_img[VAR_P4], img.data(), img.size()))) return fail(rc);
        f->img_bytes[VAR_P4] = 0;  // packed tables live in a fixed shared-window slot (scratch_offset)
    }
    if (n <= 8 && !bits) {  // N8's count bit is byte-mode only
        auto img = image_n8(f->dfa);
        if ((rc = upload(&f->d_img[VAR_N8], img.data(), img.size()))) return fail(rc);
        f->img_bytes[VAR_N8] = 0;
    }
    if (n <= 8) {
        auto img = image_packed(f->dfa, true);
        if ((rc = upload(&f->d_img[VAR_P8], img.data(), img.size()))) return fail(rc);
        f->img_bytes[VAR_P8] = 0;
    }
    if (n <= 16 && !bits) {  // region counting: byte mode only (accept-partitioned ids)
        auto img = image_r16(f->dfa);
        if ((rc = upload(&f->d_img[VAR_R16], img.data(), img.size()))) return fail(rc);
        f->img_bytes[VAR_R16] = n * 8192u;  // lane-replicated in shared memory
    }
    if (n <= 256 && !bits) {  // RG: 32 >> logl copies of the R16 layout, <= 128 KiB (logl = 0: R16's)
        uint32_t logl = 0;
        while ((n << 13) >> logl > (128u << 10)) logl++;
        auto img = image_r16(f->dfa);
        if ((rc = upload(&f->d_img[VAR_RG], img.data(), img.size()))) return fail(rc);
        f->img_bytes[VAR_RG] = (n * 8192u) >> logl;
        f->r_logl = logl;
    }
    if (n <= 256) {
        auto img = image_b(f->dfa);
        if ((rc = upload(&f->d_img[VAR_B], img.data(), img.size()))) return fail(rc);
        f->img_bytes[VAR_B] = (uint32_t)img.size();
    }
    {
        auto img = image_g(f->dfa);
        if ((rc = upload(&f->d_img[VAR_G], img.data(), img.size()))) return fail(rc);
        f->img_bytes[VAR_G] = 0;
    }
    if (!bits && f->dfa.n <= 32768) {
        // hot rows: as many u16 rows (512 B each) as fit next to the kernel's scratch
        f->hot_rows = std::min<uint32_t>(f->dfa.n, 384);
        auto img = image_hs(f->dfa, f->hot_rows);
        if ((rc = upload(&f->d_img[VAR_HS], img.data(), img.size()))) return fail(rc);
        f->img_bytes[VAR_HS] = (uint32_t)img.size();
    }
    if (!bits) {
        // CL: byte classes + lane-replicated class-compressed table when it fits below the class map
        // (u16 entries = row addresses, so the whole table must lie below shared address 0x10000)
        std::vector<uint32_t> cls, rep;
        const uint32_t nc = byte_classes(f->dfa, cls, rep), rb = cl_slots(nc) * 128;
        if (nc >= 2 && (uint64_t)f->dfa.n * rb <= kClMaxTable) {
            auto img = image_cl(f->dfa, cls, rep);
            if ((rc = upload(&f->d_img[VAR_CL], img.data(), img.size()))) return fail(rc);
            f->img_bytes[VAR_CL] = f->dfa.n * rb;
            f->ncls = nc;
            f->cl_magic = (uint32_t)((((uint64_t)1 << 32) + rb - 1) / rb);  // id = (R - 0x400) / rb
            f->cl_rc_t = 0x400u + f->rc_nA * rb;                            // R(nA)
            if (f->auto_variant == VAR_B || f->auto_variant == VAR_RG) f->auto_variant = VAR_CL;
        }
    }
    if (f->renumbered && (rc = upload(&f->d_inv, f->inv.data(), f->inv.size() * 4))) return fail(rc);
    if ((rc = upload(&f->d_lb, f->lb.data(), f->lb.size() * 2))) return fail(rc);
    if ((rc = upload(&f->d_nimg, f->nimg.data(), f->nimg.size()))) return fail(rc);
    if (bits && (rc = upload(&f->d_bittab, f->dfa.bittab.data(), f->dfa.bittab.size() * 4))) return fail(rc);
    {
        cudaError_t e;
        if ((e = cudaMalloc(&f->d_ticket, 64)) != cudaSuccess) return fail(cuda_status(e));
        if ((e = cudaMemset(f->d_ticket, 0, 64)) != cudaSuccess) return fail(cuda_status(e));
        if ((e = cudaMalloc(&f->d_result, 2 * sizeof(DevResult))) != cudaSuccess) return fail(cuda_status(e));
        if ((e = cudaMemset(f->d_result, 0, 2 * sizeof(DevResult))) != cudaSuccess) return fail(cuda_status(e));
        if ((e = cudaMalloc(&f->d_stats, sizeof(DevStats))) != cudaSuccess) return fail(cuda_status(e));
        if ((e = cudaMemset(f->d_stats, 0, sizeof(DevStats))) != cudaSuccess) return fail(cuda_status(e));
        if ((e = cudaMalloc(&f->d_fix, 64)) != cudaSuccess) return fail(cuda_status(e));
        if ((e = cudaMallocHost(&f->h_result, sizeof(DevResult) + sizeof(DevStats))) != cudaSuccess)
            return fail(cuda_status(e));
        f->h_stats = nullptr;
    }
    *out = f;
    return FSM_OK;
}

extern "C" int fsm_create(const uint32_t *table, uint32_t n_states, uint32_t alphabet, uint32_t start,
                          const uint8_t *accept_mask, fsm_t **out)
{
    return fsm_create_ex(table, n_states, alphabet, start, accept_mask, FSM_INPUT_BYTES, out);
}

extern "C" void fsm_destroy(fsm_t *f)
{
    if (!f) return;
    cudaStreamSynchronize(f->stream);
    free_all(f);
    delete f;
}

extern "C" int fsm_set_stream(fsm_t *f, void *s)
{
    if (!f) return FSM_EINVAL;
    f->stream = (cudaStream_t)s;
    return FSM_OK;
}

extern "C" int fsm_set_options(fsm_t *f, const fsm_options *o)
{
    if (!f || !o) return FSM_EINVAL;
    // chunk <= 8 KiB (16 KiB in byte mode) keeps 32-tile look-back windows of counts inside 32 bits
    // (up to 8 accepts per byte in bit mode, 1 in byte mode)
    const uint32_t max_chunk = f->mode == FSM_INPUT_BITS_MSB ? 8192u : 16384u;
    if (o->chunk_bytes && (o->chunk_bytes % 32 || o->chunk_bytes > max_chunk)) return FSM_EINVAL;
    if (o->threads_per_tile && (o->threads_per_tile % 32 || o->threads_per_tile < 32 || o->threads_per_tile > 1024))
        return FSM_EINVAL;
    if (o->variant < FSM_VARIANT_AUTO || o->variant > FSM_VARIANT_RG) return FSM_EINVAL;
    if (o->variant != FSM_VARIANT_AUTO && !f->d_img[o->variant]) return FSM_EINVAL;  // too large, or retired (4)  // table too large for it
    if (o->merge > FSM_MERGE_SEQUENTIAL) return FSM_EINVAL;
    if (o->lookback_len > 1 && (o->lookback_len % 32 || o->lookback_len > 1024)) return FSM_EINVAL;
    if (o->eager_window > FSM_EAGER_OFF && (o->eager_window % 32 || o->eager_window > kExtWindow)) return FSM_EINVAL;
    if (o->preresolve > FSM_KMAX && o->preresolve != FSM_PRERESOLVE_NONE) return FSM_EINVAL;
    if (o->check > FSM_CHECK_HASH) return FSM_EINVAL;
    if (o->lookback_width % 4 || o->lookback_width > FSM_KMAX) return FSM_EINVAL;
    f->opt.chunk_bytes = o->chunk_bytes;            // 0 = adaptive
    f->opt.threads_per_tile = o->threads_per_tile;  // 0 = auto
    f->opt.variant = o->variant;
    f->opt.merge = o->merge;
    f->opt.ctas_per_sm = o->ctas_per_sm;
    f->opt.grid_sms = o->grid_sms;
    f->opt.check = o->check;
    f->opt.lookback_width = o->lookback_width;
    f->opt.lookback_len = o->lookback_len;
    f->opt.eager_window = o->eager_window;
    f->opt.preresolve = o->preresolve;
    return FSM_OK;
}

extern "C" int fsm_get_options(const fsm_t *f, fsm_options *o)
{
    if (!f || !o) return FSM_EINVAL;
    *o = f->opt;
    return FSM_OK;
}

extern "C" int fsm_get_stats(const fsm_t *f, fsm_stats *s)
{
    if (!f || !s) return FSM_EINVAL;
    DevStats h{};
    CK(cudaMemcpyAsync(&h, f->d_stats, sizeof(DevStats), cudaMemcpyDeviceToHost, f->stream));
    CK(cudaStreamSynchronize(f->stream));
    fsm_stats r = f->last;
    r.reexec_true = h.reexec_true;
    r.reexec_true_symbols = h.reexec_true_bytes;
    r.reexec_candidate = h.reexec_cand;
    r.reexec_candidate_symbols = h.reexec_cand_bytes;
    r.reexec_chunks = h.reexec_true + h.reexec_cand;
    r.reexec_symbols = h.reexec_true_bytes + h.reexec_cand_bytes;
    r.boundary_misses = h.boundary_misses;
    r.eager_resolved = h.eager_resolved;
    r.max_miss_chain = h.max_miss_chain;
    *s = r;
    return FSM_OK;
}

// ----------------------------------------------------------------------------------- runs ----
struct RunSpec {
    uint32_t *user_out;    // async API: user-visible result written by the kernel (may be null)
    const uint8_t *in;
    uint64_t len_sym;      // symbols
    uint32_t k;
    bool keyed;
    uint32_t halo_byte;
    uint32_t start_state;
    const DevResult *start_dev;
    DevResult *result;
    int force_variant;     // -1 = handle options
    uint32_t merge;
    uint64_t geom_len_bytes = 0;  // geometry as for a run of this many bytes (0 = len): tuning samples
    uint32_t force_T = 0, force_chunk = 0;  // multi-FSM groups: one geometry for every DFA
    bool multi = false;                     // launched by the multi-FSM kernel (never split)
    bool accumulate = false;                // keep the counters of the call's earlier launches
};

constexpr int kMultiMaxK = 8;  // fused multi-FSM kernels are instantiated for K <= 8
// FSM_CHECK_AUTO: Alg. 2 for K >= 12 when its per-thread columns fit next to the table at the full
// tile size, else Alg. 1 (measured on B200: the hash form wins where the tile keeps
// its size, e.g. 64-state B k = 16 +12 %, and loses where the tile must halve, e.g. HTML CL -26 %)
constexpr bool kHashAuto = true;
// R5 default (fsm_options.preresolve = 0), measured: the top-ranked tile-start
// candidate only -- except for DFAs whose paths never meet (every symbol a permutation), where a
// lazily resolved candidate costs a whole-chunk re-execution chain on the look-back's critical
// path, so every candidate is pre-resolved in parallel.
static uint32_t preresolve_of(const fsm *f)
{
    const uint32_t v = f->opt.preresolve;
    if (v == 0) return f->permutation ? (uint32_t)FSM_KMAX : 1u;
    return v == FSM_PRERESOLVE_NONE ? 0u : v;
}

// Chunks per tile: a split kernel (split_kernel(var, K)) gives the CTA's last warp to the epilogue.
static uint32_t tile_chunks(uint32_t T, bool split) { return split ? T - 32 : T; }
constexpr uint32_t kMaxSmem = 232448u;  // dynamic shared memory per CTA on sm_100 (227 KiB)

static int variant_of(const fsm *f, int force, uint32_t k = 1)
{
    if (force >= 0) return force;
    if (f->opt.variant != FSM_VARIANT_AUTO) return f->opt.variant;
    (void)k;
    return f->auto_variant;
}

// Geometry: T chunks per tile (CTA threads), chunk bytes.  Large inputs: the largest CTA the
// register budget allows for K and 16 KiB chunks (8 KiB in bit mode, 4 KiB for G / HS).  Small
// inputs: shrink the CTA, then the chunk, so that every SM still gets a tile.
static void pick_geometry(const fsm *f, uint64_t len_bytes, int K, int var, uint32_t &T, uint32_t &chunk)
{
    const uint32_t tmax = (uint32_t)max_threads(K, var);
    T = f->opt.threads_per_tile ? std::min<uint32_t>(f->opt.threads_per_tile, tmax) : tmax;
    if (!f->opt.threads_per_tile)
        while (T > 128 && len_bytes < (uint64_t)f->num_sms * T * 4096) T = std::max(128u, (T >> 1) & ~31u);
    if (f->opt.chunk_bytes) {
        chunk = f->opt.chunk_bytes;
        return;
    }
    // Power-of-two chunks up to 16 KiB in byte mode, 8 KiB in bit mode (the counts' 32-bit range, see
    // fsm_set_options) and 4 KiB for the L2-table variants G / HS, chosen by a wave
    // model: a persistent grid of one CTA per SM takes tiles dynamically, so a run costs about
    // ceil(tiles / SMs) x (chunk + a per-chunk overhead of ~K KiB-equivalents: speculation, the K-chain
    // prologue, the window walk, the merge; C4 k = 4: 16 KiB 1832 vs 8 KiB 1439 GB/s).  Measured on 8 GiB against 4 KiB: C4 k = 1 2590 -> 2992, (64, 4, k = 4)
    // 2349 -> 2534, (16, 2, k = 2) 3467 -> 3578 GB/s; C3 (G) 1191 at 4 KiB vs 1058 at 8 KiB.
    // Chunks that are not powers of two measured 2-25 % slower (7328 B: C4 2225 GB/s).  16 KiB
    // against 8 KiB on 8 GiB: C4 2987 -> 3190, (64, 4, k = 4) 2535 -> 2634, (8, 2, k = 2) 4391 -> 4481.
    const uint64_t cap = (var == VAR_G || var == VAR_HS) ? 4096 : f->mode == FSM_INPUT_BITS_MSB ? 8192 : 16384;
    const uint64_t te = split_kernel(var, K) && T >= 64 ? T - 32 : T;  // chunks per tile
    uint64_t best = 0, best_cost = ~0ull;
    for (uint64_t c = cap; c >= 64; c >>= 1) {
        const uint64_t tiles = std::max<uint64_t>(1, (len_bytes + te * c - 1) / (te * c));
        const uint64_t cost = (tiles + f->num_sms - 1) / f->num_sms * (c + 1024ull * K);
        if (cost < best_cost) {
            best = c;
            best_cost = cost;
        }
    }
    chunk = (uint32_t)best;
}

static int ensure_desc(fsm *f, size_t ntiles)
{
    if (ntiles <= f->desc_cap) return FSM_OK;
    size_t cap = std::max<size_t>(ntiles, 1024);
    cudaStreamSynchronize(f->stream);
    cudaFree(f->d_desc);
    f->d_desc = nullptr;
    f->desc_cap = 0;
    CK(cudaMalloc(&f->d_desc, cap * sizeof(TileDesc)));
    CK(cudaMemset(f->d_desc, 0, cap * sizeof(TileDesc)));
    f->desc_cap = cap;
    return FSM_OK;
}

static int launch_seq(fsm *f, Params p, int var, int K, uint32_t T);
// SMs the persistent grids are spread over (fsm_options.grid_sms; the a11 grid-size sweep)
static uint64_t grid_sms(const fsm *f)
{
    return f->opt.grid_sms ? std::min<uint64_t>(f->opt.grid_sms, (uint64_t)f->num_sms) : (uint64_t)f->num_sms;
}
constexpr size_t kDbgBytes = (size_t)6 * 32 * KMAX * sizeof(uint4);  // fsm_debug_get_merge levels

// Everything of a run but the fused kernel's launch: variant, geometry, Params, the look-back
// pre-pass (launched here), descriptors.  Shared by single runs and multi-FSM groups.
struct Prepared {
    Params p;
    int var, K;
    uint32_t T;
    size_t smem;
    bool split;
    bool hash;  // Alg. 2 runtime check (K >= 12)
};

// Alg. 1 vs Alg. 2 (fsm_options.check = FSM_CHECK_AUTO): see DESIGN.md "a5"
static bool hash_wanted(const fsm *f, int K)
{
    if (K < 12) return false;
    if (f->opt.check == FSM_CHECK_HASH) return true;
    if (f->opt.check == FSM_CHECK_NESTED) return false;
    return kHashAuto;
}

static int prepare_run(fsm *f, const RunSpec &r, Prepared &out)
{
    const int var = variant_of(f, r.force_variant, r.k);
    const int K = kslots(r.k);
    const bool bits = f->mode == FSM_INPUT_BITS_MSB;
    const uint64_t ulen_bytes = bits ? r.len_sym / 8 : r.len_sym;
    // An unaligned input is run from the 32-byte-aligned address below it: chunk 0 is [head, chunk)
    // and every kernel position is relative to that address, so every other chunk starts on a full
    // sector (one peeled partial sector instead of a byte-at-a-time run).  Debug geometries with
    // tiny chunks on an unaligned input keep the byte path instead.
    uint32_t head = (uint32_t)((uintptr_t)r.in & 31);
    bool aligned = true;
    if (head && f->dbg_chunk && !r.multi && f->dbg_chunk < 64) {
        head = 0;
        aligned = false;
    }
    const uint64_t len_bytes = ulen_bytes + head;  // kernel coordinates
    uint32_t T = 0, chunk = 0;
    pick_geometry(f, r.geom_len_bytes ? std::max(r.geom_len_bytes, ulen_bytes) : ulen_bytes, K, var, T, chunk);
    if (r.force_T) T = r.force_T;
    if (r.force_chunk) chunk = r.force_chunk;
    const bool dbg = f->dbg_chunk != 0 && !r.multi;
    if (dbg) {  // test hook: the fixed tiny geometry of fsm_debug_set_spec (one warp of chunks per tile)
        chunk = f->dbg_chunk;
        T = 32;
        if (f->dbg_n) {
            const uint64_t nch = len_bytes == 0 ? 1 : (len_bytes + chunk - 1) / chunk;
            if (nch != f->dbg_n || r.k != f->dbg_k || r.keyed || head) return FSM_EINVAL;
        }
    }
    if (r.merge == FSM_MERGE_SEQUENTIAL) T = std::min<uint32_t>(T, kThreads);
    if (split_kernel(var, K) && T < 64) T = 64;  // at least one worker warp besides the epilogue warp
    bool split = split_kernel(var, K) && !r.multi && r.merge == FSM_MERGE_PARALLEL;
    bool hash = hash_wanted(f, K) && !r.multi && r.merge == FSM_MERGE_PARALLEL;
    if (hash) split = false;  // Alg. 2 kernels are instantiated unsplit
    {
        const uint32_t tb = var == VAR_HS ? 0u : f->img_bytes[var];
        if (hash && !f->opt.threads_per_tile && f->opt.check == FSM_CHECK_HASH) {
            // Alg. 2 requested: halve the tile until its per-thread columns fit next to the table
            while (T > 64 && Layout(T, K, scratch_offset(var, tb), false, true).total > kMaxSmem)
                T = std::max(64u, (T >> 1) & ~31u);  // whole warps (max_threads need not be a power of two)
        }
        if (hash && Layout(T, K, scratch_offset(var, tb), false, true).total > kMaxSmem) hash = false;  // Alg. 1
        if (split)  // the double-buffered layout must fit next to the table (HS sizes its hot rows after)
            split = Layout(T, K, scratch_offset(var, tb), true, hash).total <= kMaxSmem;
    }
    const uint64_t tile_bytes = (uint64_t)tile_chunks(T, split) * chunk;
    uint64_t ntiles64 = (len_bytes + tile_bytes - 1) / tile_bytes;
    if (ntiles64 == 0) ntiles64 = 1;
    if (ntiles64 > 0x7FFFFFFFull) return FSM_EINVAL;
    const uint32_t ntiles = (uint32_t)ntiles64;
    int rc;

    Params p{};
    p.in = r.in - head;
    p.head = head;
    p.len = len_bytes;
    p.chunk = chunk;
    p.ntiles = ntiles;
    p.k = r.k;
    p.lookback = f->opt.lookback_len > 1 ? f->opt.lookback_len : 0;
    p.lb_width = f->opt.lookback_width ? f->opt.lookback_width : KMAX;
    p.eager_window = f->opt.eager_window == 0 ? kExtWindow : f->opt.eager_window == FSM_EAGER_OFF ? 0u : f->opt.eager_window;
    p.preresolve = preresolve_of(f);
    if (dbg && f->dbg_n) {
        p.lookback = 0;
        p.eager_window = 0;
        p.spec = f->d_dbg_spec;
        p.spec_stride = r.k + kExt;
        p.spec_all = 1;
    }
    if (dbg) {
        p.dbg = f->d_dbg;
        CK(cudaMemsetAsync(f->d_dbg, 0xFF, kDbgBytes, f->stream));
    }
    p.aligned = aligned ? 1u : 0u;
    p.table = f->d_img[var];
    p.n_states = f->dfa.n;
    p.table_bytes = f->img_bytes[var];
    p.lb = f->d_lb;
    p.nimg = f->d_nimg;
    p.keyed = r.keyed;
    p.start_state = r.start_state;
    p.start_dev = r.start_dev;
    p.halo_byte = r.halo_byte;
    p.tail_bits = bits ? (uint32_t)(r.len_sym & 7) : 0;
    p.bittab = f->d_bittab;
    p.result = r.result;
    p.stats = f->d_stats;
    p.ticket = f->d_ticket;
    p.k_1e24 = 1u << 24;
    p.k_16 = 16;
    p.k_512 = 512;
    p.k_4 = 4;
    p.table_g = static_cast<const uint32_t *>(f->d_img[VAR_G]);
    p.hot_rows = f->hot_rows;
    p.inv = f->d_inv;
    p.user_out = r.user_out;
    p.ncls = f->ncls;
    p.cl_magic = f->cl_magic;
    p.rc_t = var == VAR_CL ? f->cl_rc_t : f->rc_nA;
    p.rc_comp = f->rc_comp;
    p.r_logl = f->r_logl;

    if (var == VAR_HS) {
        // as many hot rows as fit next to this launch's scratch (227 KB per CTA)
        const uint32_t scratch = Layout(T, K, 0, split, hash).total;
        const uint32_t avail = scratch < kMaxSmem ? kMaxSmem - scratch : 0u;
        const uint32_t hot = std::min<uint32_t>(f->hot_rows, avail / 512);
        p.hot_rows = hot;
        p.table_bytes = hot * 512;
    }
    const size_t smem = Layout(T, K, scratch_offset(var, p.table_bytes), split, hash).total;

    if (p.lookback >= 32) {
        // a3 pre-pass: ranked look-back candidates per chunk (spec_kernel.cuh)
        const uint64_t nch = len_bytes == 0 ? 1 : (len_bytes + chunk - 1) / chunk;
        p.spec_stride = (uint32_t)r.k + kExt;
        const size_t need = nch * p.spec_stride;
        if (need > f->spec_cap) {
            cudaStreamSynchronize(f->stream);
            cudaFree(f->d_spec);
            f->d_spec = nullptr;
            f->spec_cap = 0;
            CK(cudaMalloc(&f->d_spec, need * 2));
            f->spec_cap = need;
        }
        SpecFn sf = get_spec(var);
        const size_t smem_s = std::max<size_t>(16, scratch_offset(var, p.table_bytes));
        CK(cudaFuncSetAttribute((const void *)sf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_s));
        int occ_s = 0;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_s, sf, kSpecThreads, smem_s));
        const uint64_t blocks = std::min<uint64_t>((nch + kSpecThreads - 1) / kSpecThreads,
                                                   (uint64_t)std::max(occ_s, 1) * f->num_sms);
        sf<<<(uint32_t)blocks, kSpecThreads, smem_s, f->stream>>>(p, f->d_spec);
        CK(cudaGetLastError());
        p.spec = f->d_spec;
    }

    out.p = p;
    out.var = var;
    out.K = K;
    out.T = T;
    out.smem = smem;
    out.split = split;
    out.hash = hash;
    if (r.merge == FSM_MERGE_SEQUENTIAL) return FSM_OK;
    if ((rc = ensure_desc(f, ntiles))) return rc;
    out.p.desc = f->d_desc;
    f->epoch = (f->epoch + 1) & 0x3FFFFFFFu;
    if (f->epoch == 0) f->epoch = 1;
    out.p.epoch = f->epoch;
    f->last.chunks = (len_bytes + chunk - 1) / chunk;
    f->last.tiles = ntiles;
    f->last.chunk_bytes = chunk;
    f->last.threads_per_tile = tile_chunks(T, split);
    f->last.variant = var;
    f->last.k_slots = K;
    f->last.lookback_len = p.lookback;
    f->last.lookback_width = p.lookback >= 32 ? p.lb_width : 0;
    f->last.preresolve = p.preresolve;
    f->last_head = head;
    f->last.check = hash ? FSM_CHECK_HASH : FSM_CHECK_NESTED;
    return FSM_OK;
}

static int launch_run(fsm *f, const RunSpec &r)
{
    if (!r.accumulate) CK(cudaMemsetAsync(f->d_stats, 0, sizeof(DevStats), f->stream));  // per-call counters
    Prepared pr;
    int rc = prepare_run(f, r, pr);
    if (rc) return rc;
    Params p = pr.p;
    const int var = pr.var, K = pr.K;
    const uint32_t T = pr.T;
    const size_t smem = pr.smem;
    if (r.merge == FSM_MERGE_SEQUENTIAL) {
        if (r.keyed) return FSM_EINVAL;
        return launch_seq(f, p, var, K, T);
    }

    KernelFn fn = get_kernel(var, K, pr.split, pr.hash);
    CK(cudaFuncSetAttribute((const void *)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, (int)T, smem));
    if (occ < 1) return FSM_EINVAL;
    if (f->opt.ctas_per_sm) occ = std::min<int>(occ, (int)f->opt.ctas_per_sm);
    const uint32_t ntiles = p.ntiles;
    const uint32_t grid = (uint32_t)std::min<uint64_t>(ntiles, (uint64_t)occ * grid_sms(f));
    p.ticket_base = f->ticket_base;
    fn<<<grid, T, smem, f->stream>>>(p);
    CK(cudaGetLastError());
    f->ticket_base += ntiles + grid;  // every CTA takes one ticket past the end
    return FSM_OK;
}

// Sequential-merge ablation (Fig. 4a): local kernel over all chunks, then one walking CTA.
static int launch_seq(fsm *f, Params p, int var, int K, uint32_t T)
{
    const uint64_t nch = p.len == 0 ? 1 : (p.len + p.chunk - 1) / p.chunk;
    if (nch * K > f->seq_cap) {
        cudaStreamSynchronize(f->stream);
        cudaFree(f->seq.S);
        cudaFree(f->seq.E);
        cudaFree(f->seq.C);
        f->seq = SeqBuf{};
        f->seq_cap = 0;
        CK(cudaMalloc(&f->seq.S, nch * K * 2));
        CK(cudaMalloc(&f->seq.E, nch * K * 4));
        CK(cudaMalloc(&f->seq.C, nch * K * 4));
        f->seq_cap = nch * K;
    }
    SeqLocalFn lf;
    SeqWalkFn wf;
    get_seq(var, K, lf, wf);
    const size_t smem_l = scratch_offset(var, p.table_bytes);
    CK(cudaFuncSetAttribute((const void *)lf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)std::max<size_t>(smem_l, 16)));
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, lf, (int)T, std::max<size_t>(smem_l, 16)));
    const uint64_t blocks = std::min<uint64_t>((nch + T - 1) / T, (uint64_t)std::max(occ, 1) * grid_sms(f));
    lf<<<(uint32_t)blocks, T, std::max<size_t>(smem_l, 16), f->stream>>>(p, f->seq);
    CK(cudaGetLastError());
    const size_t smem_w = seq_walk_smem(T, K, var, p.table_bytes);
    CK(cudaFuncSetAttribute((const void *)wf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_w));
    wf<<<1, T, smem_w, f->stream>>>(p, f->seq);
    CK(cudaGetLastError());
    f->last.chunks = nch;
    f->last.tiles = 0;
    f->last.chunk_bytes = p.chunk;
    f->last.threads_per_tile = T;
    f->last.variant = var;
    f->last.k_slots = K;
    f->last.lookback_len = p.lookback;
    return FSM_OK;
}

static int check_run_args(const fsm *f, const uint8_t *input, uint64_t len, uint32_t k)
{
    if (!f) return FSM_EINVAL;
    if (k < 1 || k > FSM_KMAX || k > f->n_user) return FSM_EINVAL;
    if (len > 0 && !input) return FSM_EINVAL;
    return FSM_OK;
}

// Read the result of the run just enqueued (one small D2H).
static int finish_sync(fsm *f, const DevResult *dres)
{
    CK(cudaMemcpyAsync(f->h_result, dres, sizeof(DevResult), cudaMemcpyDeviceToHost, f->stream));
    CK(cudaStreamSynchronize(f->stream));
    return FSM_OK;
}

static bool is_sink(const fsm *f, uint32_t s) { return f->dfa.sink != 0xFFFFFFFFu && s == f->dfa.sink; }
static uint32_t to_user(const fsm *f, uint32_t s) { return f->renumbered && s < f->inv.size() ? f->inv[s] : s; }
static uint32_t to_int(const fsm *f, uint32_t s) { return f->renumbered && s < f->perm.size() ? f->perm[s] : s; }

extern "C" int fsm_run_spec_k_async(fsm_t *f, const uint8_t *input, uint64_t len, uint32_t k, fsm_result *dev_result)
{
    int rc = check_run_args(f, input, len, k);
    if (rc) return rc;
    if (!dev_result) return FSM_EINVAL;
    RunSpec r{reinterpret_cast<uint32_t *>(dev_result), input, len, k, false, 0, f->start_int, nullptr, f->d_result,
              -1, f->opt.merge};
    return launch_run(f, r);  // the last tile writes the user-visible result into dev_result
}

extern "C" int fsm_run_spec_k(fsm_t *f, const uint8_t *input, uint64_t len, uint32_t k, uint32_t *final_state,
                              uint64_t *accept_count)
{
    int rc = check_run_args(f, input, len, k);
    if (rc) return rc;
    if (!final_state || !accept_count) return FSM_EINVAL;
    RunSpec r{nullptr, input, len, k, false, 0, f->start_int, nullptr, f->d_result, -1, f->opt.merge};
    if ((rc = launch_run(f, r))) return rc;
    if ((rc = finish_sync(f, f->d_result))) return rc;
    if (is_sink(f, f->h_result->final_state)) return FSM_ESYMBOL;
    *final_state = to_user(f, f->h_result->final_state);
    *accept_count = f->h_result->count;
    return FSM_OK;
}

// End-to-end over a host buffer: pieces copied H2D on a copy stream into two staging buffers,
// each piece's kernel chained to the previous piece's result on the device.
extern "C" int fsm_run_spec_k_host(fsm_t *f, const uint8_t *host_input, uint64_t len, uint32_t k,
                                   uint32_t *final_state, uint64_t *accept_count)
{
    int rc = check_run_args(f, host_input, len, k);
    if (rc) return rc;
    if (!final_state || !accept_count) return FSM_EINVAL;
    const bool bits = f->mode == FSM_INPUT_BITS_MSB;
    const uint64_t nbytes = bits ? (len + 7) / 8 : len;
    const size_t piece = (size_t)1 << 28;  // 256 MiB
    if (!f->d_stage[0]) {
        CK(cudaMalloc(&f->d_stage[0], piece + 64));
        CK(cudaMalloc(&f->d_stage[1], piece + 64));
        for (int i = 0; i < 2; i++) {
            CK(cudaEventCreateWithFlags(&f->ev_copied[i], cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&f->ev_used[i], cudaEventDisableTiming));
        }
        CK(cudaStreamCreateWithFlags(&f->copy_stream, cudaStreamNonBlocking));
        f->stage_bytes = piece;
    }
    // the stage buffers may still be read by a previous call's kernels
    for (int i = 0; i < 2; i++) CK(cudaEventRecord(f->ev_used[i], f->stream));
    const uint64_t npieces = nbytes == 0 ? 1 : (nbytes + piece - 1) / piece;
    uint64_t chunks = 0, tiles = 0;
    for (uint64_t pi = 0; pi < npieces; pi++) {
        const int sb = (int)(pi & 1);
        const uint64_t off = pi * piece;
        const uint64_t nb = std::min<uint64_t>(piece, nbytes - std::min(nbytes, off));
        CK(cudaStreamWaitEvent(f->copy_stream, f->ev_used[sb], 0));
        if (nb) CK(cudaMemcpyAsync(f->d_stage[sb], host_input + off, nb, cudaMemcpyHostToDevice, f->copy_stream));
        CK(cudaEventRecord(f->ev_copied[sb], f->copy_stream));
        CK(cudaStreamWaitEvent(f->stream, f->ev_copied[sb], 0));
        uint64_t sym = bits ? std::min<uint64_t>(len - off * 8, (uint64_t)nb * 8) : nb;
        // chain: piece pi starts from piece pi-1's result (d_result[0]); it writes to d_result[pi&1 ^ ...]
        DevResult *res = f->d_result + ((pi + 1) & 1);
        const DevResult *prev = pi == 0 ? nullptr : f->d_result + (pi & 1);
        RunSpec r{nullptr, f->d_stage[sb], sym, k, false, 0, f->start_int, prev, res, -1, FSM_MERGE_PARALLEL};
        r.accumulate = pi > 0;  // the call's counters sum over its pieces
        if ((rc = launch_run(f, r))) return rc;
        CK(cudaEventRecord(f->ev_used[sb], f->stream));
        chunks += f->last.chunks;
        tiles += f->last.tiles;
    }
    const DevResult *fin = f->d_result + (npieces & 1);
    if ((rc = finish_sync(f, fin))) return rc;
    f->last.chunks = chunks;
    f->last.tiles = tiles;
    if (is_sink(f, f->h_result->final_state)) return FSM_ESYMBOL;
    *final_state = to_user(f, f->h_result->final_state);
    *accept_count = f->h_result->count;
    return FSM_OK;
}

// ------------------------------------------------------------------------------- shards ----
extern "C" int fsm_run_shard(fsm_t *f, const uint8_t *input, uint64_t len, const uint8_t *halo, uint32_t halo_len,
                             uint32_t k, fsm_shard_map *out, fsm_shard_t **state)
{
    int rc = check_run_args(f, input, len, k);
    if (rc) return rc;
    if (!out || (halo_len > 0 && !halo)) return FSM_EINVAL;
    uint32_t hb = 0;
    const bool keyed = halo_len > 0;
    if (keyed) {
        uint8_t h = 0;
        CK(cudaMemcpyAsync(&h, halo + halo_len - 1, 1, cudaMemcpyDeviceToHost, f->stream));
        CK(cudaStreamSynchronize(f->stream));
        hb = h;
    }
    RunSpec r{nullptr, input, len, k, keyed, hb, f->start_int, nullptr, f->d_result, -1, FSM_MERGE_PARALLEL};
    if ((rc = launch_run(f, r))) return rc;
    if ((rc = finish_sync(f, f->d_result))) return rc;
    const DevResult *hr = f->h_result;
    // an out-of-alphabet byte maps every state to the absorbing sink: every path ends there
    if (!keyed && is_sink(f, hr->final_state)) return FSM_ESYMBOL;
    if (keyed)
        for (int s = 0; s < KMAX; s++)
            if (((hr->valid_mask >> s) & 1u) && is_sink(f, hr->end[s])) return FSM_ESYMBOL;
    fsm_shard_map m{};
    m.k = k;
    if (!keyed) {
        m.valid_mask = 1;
        m.start[0] = f->start;
        m.end[0] = to_user(f, hr->final_state);
        m.count[0] = hr->count;
    } else {
        m.valid_mask = hr->valid_mask & ((1u << KMAX) - 1);
        for (int s = 0; s < KMAX; s++) {
            const bool v = (m.valid_mask >> s) & 1u;
            m.start[s] = v ? to_user(f, hr->start[s]) : hr->start[s];
            m.end[s] = v ? to_user(f, hr->end[s]) : hr->end[s];
            m.count[s] = hr->mcount[s];
        }
    }
    *out = m;
    if (state) {
        fsm_shard *st = new (std::nothrow) fsm_shard();
        if (!st) return FSM_ENOMEM;
        st->input = input;
        st->len = len;
        st->k = k;
        st->variant = (int)f->last.variant;
        st->map = m;
        if (keyed && f->last.tiles) {
            st->ntiles = (uint32_t)f->last.tiles;
            st->tile_bytes = (uint64_t)f->last.threads_per_tile * f->last.chunk_bytes;
            st->head = f->last_head;
            st->kslots = f->last.k_slots;
            if (cudaMalloc(&st->d_desc, st->ntiles * sizeof(TileDesc)) != cudaSuccess ||
                cudaMemcpyAsync(st->d_desc, f->d_desc, st->ntiles * sizeof(TileDesc), cudaMemcpyDeviceToDevice,
                                f->stream) != cudaSuccess ||
                cudaStreamSynchronize(f->stream) != cudaSuccess) {
                fsm_shard_free(st);
                return FSM_ECUDA;
            }
        }
        *state = st;
    }
    return FSM_OK;
}

extern "C" int fsm_shard_fixup(fsm_t *f, fsm_shard_t *st, uint32_t true_start, uint32_t *end, uint64_t *count)
{
    if (!f || !st || !end || !count || true_start >= f->n_user) return FSM_EINVAL;
    for (int s = 0; s < KMAX; s++)
        if (((st->map.valid_mask >> s) & 1u) && st->map.start[s] == true_start) {
            *end = st->map.end[s];
            *count = st->map.count[s];
            return FSM_OK;
        }
    CK(cudaMemsetAsync(f->d_stats, 0, sizeof(DevStats), f->stream));  // the fix-up's own counters
    const bool bits = f->mode == FSM_INPUT_BITS_MSB;
    const uint64_t whole = bits ? st->len / 8 : st->len;
    const int var = st->variant;
    uint32_t y = to_int(f, true_start);
    uint64_t cy = 0, resume_byte = 0;
    if (st->d_desc && st->ntiles) {
        // walk x's path over the keyed run's tile descriptors (fixup_kernel.cuh)
        FixParams fp{};
        fp.in = st->input;
        fp.len = whole;
        fp.head = st->head;
        fp.tile_bytes = st->tile_bytes;
        fp.ntiles = st->ntiles;
        fp.limit = (uint64_t)1 << 20;
        fp.desc = st->d_desc;
        fp.table = f->d_img[var];
        fp.n_states = f->dfa.n;
        fp.x = y;
        fp.k = st->map.k;
        fp.kslots = st->kslots;
        fp.valid_mask = st->map.valid_mask;
        for (int s = 0; s < KMAX; s++) {
            const bool v = (st->map.valid_mask >> s) & 1u;
            fp.end[s] = v ? to_int(f, st->map.end[s]) : st->map.end[s];
            fp.count[s] = st->map.count[s];
        }
        fp.tail_bits = bits ? (uint32_t)(st->len & 7) : 0u;
        fp.bittab = f->d_bittab;
        fp.out = f->d_fix;
        fp.stats = f->d_stats;
        fp.kc = KConst{1u << 24, 16, 512, static_cast<const uint32_t *>(f->d_img[VAR_G]), f->hot_rows, f->ncls,
                       f->cl_magic, 4, var == VAR_CL ? f->cl_rc_t : f->rc_nA, f->rc_comp,
                       f->r_logl};
        FixFn fn = get_fix(var);
        const size_t smem = std::max<uint32_t>(16, scratch_offset(var, f->img_bytes[var]));
        CK(cudaFuncSetAttribute((const void *)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        fn<<<1, kThreads, smem, f->stream>>>(fp);
        CK(cudaGetLastError());
        unsigned long long h[5];
        CK(cudaMemcpyAsync(h, f->d_fix, sizeof(h), cudaMemcpyDeviceToHost, f->stream));
        CK(cudaStreamSynchronize(f->stream));
        if (h[0]) {
            *end = to_user(f, (uint32_t)h[1]);
            *count = h[2];
            return FSM_OK;
        }
        y = (uint32_t)h[1];
        cy = h[2];
        const uint64_t t = h[4];
        resume_byte = t * st->tile_bytes > st->head ? std::min<uint64_t>(t * st->tile_bytes - st->head, whole) : 0;
    }
    // the paths did not meet within the walk's budget: run the rest of the shard from the state
    // reached with the parallel known-start kernel (exact)
    const uint64_t rest = st->len - (bits ? resume_byte * 8 : resume_byte);
    RunSpec r{nullptr, st->input + resume_byte, rest, st->k, false, 0, y, nullptr, f->d_result, var, FSM_MERGE_PARALLEL};
    r.accumulate = true;
    int rc = launch_run(f, r);
    if (rc) return rc;
    if ((rc = finish_sync(f, f->d_result))) return rc;
    *end = to_user(f, f->h_result->final_state);
    *count = f->h_result->count + cy;
    return FSM_OK;
}

extern "C" void fsm_shard_free(fsm_shard_t *st)
{
    if (!st) return;
    cudaFree(st->d_desc);
    delete st;
}

// ---------------------------------------------------------------------------- test hooks ----
extern "C" int fsm_debug_set_spec(fsm_t *f, const uint32_t *sets, uint32_t n_chunks, uint32_t k, uint32_t chunk_bytes)
{
    if (!f) return FSM_EINVAL;
    if (chunk_bytes == 0) {
        f->dbg_chunk = f->dbg_n = f->dbg_k = 0;
        return FSM_OK;
    }
    if (chunk_bytes > 8192) return FSM_EINVAL;
    if (sets) {
        if (n_chunks == 0 || k < 1 || k > FSM_KMAX || k > f->n_user) return FSM_EINVAL;
        const uint32_t stride = k + kExt;
        std::vector<uint16_t> h((size_t)n_chunks * stride, 0xFFFFu);
        for (uint32_t j = 0; j < n_chunks; j++)
            for (uint32_t s = 0; s < k; s++) {
                const uint32_t v = sets[(size_t)j * k + s];
                if (v == 0xFFFFFFFFu) continue;
                if (v >= f->n_user) return FSM_EINVAL;
                for (uint32_t q = 0; q < s; q++)
                    if (sets[(size_t)j * k + q] == v) return FSM_EINVAL;  // reading A6: never duplicated
                h[(size_t)j * stride + s] = (uint16_t)to_int(f, v);
            }
        cudaStreamSynchronize(f->stream);
        cudaFree(f->d_dbg_spec);
        f->d_dbg_spec = nullptr;
        int rc = upload(&f->d_dbg_spec, h.data(), h.size() * 2);
        if (rc) return rc;
    }
    if (!f->d_dbg) CK(cudaMalloc(&f->d_dbg, kDbgBytes));
    f->dbg_chunk = chunk_bytes;
    f->dbg_n = sets ? n_chunks : 0;
    f->dbg_k = sets ? k : 0;
    return FSM_OK;
}

extern "C" int fsm_debug_get_merge(const fsm_t *f, fsm_debug_merge *out)
{
    if (!f || !out || !f->d_dbg) return FSM_EINVAL;
    std::vector<uint4> h(kDbgBytes / sizeof(uint4));
    CK(cudaStreamSynchronize(f->stream));
    CK(cudaMemcpy(h.data(), f->d_dbg, kDbgBytes, cudaMemcpyDeviceToHost));
    const uint32_t K = f->last.k_slots;
    out->k = K;
    for (int l = 0; l < 6; l++)
        for (int lane = 0; lane < 32; lane++) {
            out->identity[l][lane] = h[(size_t)(l * 32 + lane) * KMAX].w == 1u;
            for (uint32_t s = 0; s < (uint32_t)KMAX; s++) {
                const uint4 v = h[(size_t)(l * 32 + lane) * KMAX + s];
                const uint32_t code = v.y >> 16, st = v.y & 0xFFFFu;
                const bool have = s < K && v.x != NOSTATE && v.x != 0xFFFFFFFFu;
                out->start[l][lane][s] = have ? to_user(f, v.x) : 0xFFFFFFFFu;
                out->count[l][lane][s] = have ? v.z : 0u;
                if (!have || code == ABSENT) {
                    out->brk[l][lane][s] = 0xFFFFFFFEu;
                    out->end[l][lane][s] = 0xFFFFFFFFu;
                } else {
                    out->brk[l][lane][s] = code == COMPLETE ? 0xFFFFFFFFu : code;
                    out->end[l][lane][s] = to_user(f, st);
                }
            }
        }
    return FSM_OK;
}

extern "C" int fsm_map_compose(const fsm_shard_map *a, const fsm_shard_map *b, fsm_shard_map *out)
{
    if (!a || !b || !out) return FSM_EINVAL;
    fsm_shard_map r = *a;
    r.valid_mask = 0;
    for (int s = 0; s < KMAX; s++) {
        if (!((a->valid_mask >> s) & 1u)) continue;
        for (int j = 0; j < KMAX; j++)
            if (((b->valid_mask >> j) & 1u) && b->start[j] == a->end[s]) {
                r.end[s] = b->end[j];
                r.count[s] = a->count[s] + b->count[j];
                r.valid_mask |= 1u << s;
                break;
            }
    }
    *out = r;
    return FSM_OK;
}

extern "C" int fsm_compose_from(const fsm_shard_map *maps, uint32_t n, uint32_t start_state, uint64_t start_count,
                                uint32_t *state, uint64_t *count, uint32_t *first_miss)
{
    if (!state || !count || !first_miss || (n > 0 && !maps)) return FSM_EINVAL;
    uint32_t x = start_state;
    uint64_t c = start_count;
    uint32_t g = 0;
    for (; g < n; g++) {
        const fsm_shard_map &m = maps[g];
        int hit = -1;
        for (int s = 0; s < KMAX && hit < 0; s++)
            if (((m.valid_mask >> s) & 1u) && m.start[s] == x) hit = s;
        if (hit < 0) break;
        x = m.end[hit];
        c += m.count[hit];
    }
    *state = x;
    *count = c;
    *first_miss = g;
    return FSM_OK;
}

// ------------------------------------------------------------------ NEXT-2: autotuning -------
// Staged measured search (include/fsmspec.h): the cost of a candidate is its median sampled time.
namespace {
struct TuneCand {
    uint32_t k, lookback, eager;
    int32_t variant = FSM_VARIANT_AUTO;
    uint32_t preresolve = 0;
    uint32_t width = 0;
    uint32_t chunk = 0;  // 0 = the geometry's choice
    uint32_t used_chunk = 0;
    double ms = 0, hit = 0;
};
}  // namespace

static int time_candidate(fsm *f, const uint8_t *in, uint64_t len, uint64_t geom_len, TuneCand &c, cudaEvent_t e0,
                          cudaEvent_t e1)
{
    fsm_options o = f->opt;
    o.lookback_len = c.lookback;
    o.eager_window = c.eager;
    o.variant = c.variant;
    o.preresolve = c.preresolve;
    o.lookback_width = c.width;
    o.chunk_bytes = c.chunk;
    o.merge = FSM_MERGE_PARALLEL;
    int rc = fsm_set_options(f, &o);
    if (rc) return rc;
    // warm-up run, synchronous: also yields the sampled success rate
    RunSpec r{nullptr, in, len, c.k, false, 0, f->start_int, nullptr, f->d_result, -1, FSM_MERGE_PARALLEL, geom_len};
    if ((rc = launch_run(f, r))) return rc;
    if ((rc = finish_sync(f, f->d_result))) return rc;
    fsm_stats st;
    if ((rc = fsm_get_stats(f, &st))) return rc;
    c.hit = st.chunks ? 1.0 - (double)st.reexec_true / (double)st.chunks : 1.0;
    c.used_chunk = st.chunk_bytes;
    float t[3];
    for (int i = 0; i < 3; i++) {
        CK(cudaEventRecord(e0, f->stream));
        if ((rc = launch_run(f, r))) return rc;
        CK(cudaEventRecord(e1, f->stream));
        CK(cudaEventSynchronize(e1));
        CK(cudaEventElapsedTime(&t[i], e0, e1));
    }
    std::sort(t, t + 3);
    c.ms = t[1];
    return FSM_OK;
}

extern "C" int fsm_autotune(fsm_t *f, const uint8_t *input, uint64_t len, uint32_t k_min, uint32_t k_max,
                            uint64_t sample_len, fsm_tuning *out)
{
    if (!f || !out || (len > 0 && !input)) return FSM_EINVAL;
    const uint32_t kcap = std::min<uint32_t>(FSM_KMAX, f->n_user);
    if (k_max == 0 || k_max > kcap) k_max = kcap;
    if (k_min == 0) k_min = 1;
    if (k_min > k_max) return FSM_EINVAL;
    const bool bits = f->mode == FSM_INPUT_BITS_MSB;
    const uint64_t sym_per_byte = bits ? 8 : 1;
    // default sample: 4 GiB -- several waves of full-size tiles over every SM (a 2 GiB prefix of C4
    // ranked window 256 above 128, which is 3 % faster on the 8 GiB run), run with the
    // geometry (chunk, tile) of the full input so that the sampled cost is the full run's per byte
    if (sample_len == 0) sample_len = ((uint64_t)4 << 30) * sym_per_byte;
    const uint64_t n = std::min(len, sample_len);
    const fsm_options saved = f->opt;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    std::vector<TuneCand> tried;
    int rc = FSM_OK;
    auto run = [&](uint32_t k, uint32_t lb, uint32_t eg, int32_t var = -2, uint32_t pre = 0, uint32_t w = 0,
                   uint32_t ch = 0) -> int {
        if (var == -2) var = saved.variant;  // stages 1-2: the handle's own variant choice
        if (ch == 0) ch = saved.chunk_bytes;
        for (const TuneCand &c : tried)
            if (c.k == k && c.lookback == lb && c.eager == eg && c.variant == var && c.preresolve == pre && c.width == w &&
                c.chunk == ch)
                return FSM_OK;
        TuneCand c{k, lb, eg, var, pre, w, ch};
        int r = time_candidate(f, input, n, len / sym_per_byte, c, e0, e1);
        if (r == FSM_OK) tried.push_back(c);
        return r;
    };
    // stage 1: every instantiated k with the default window and with the paper's setting
    std::vector<uint32_t> ks;
    for (int i = 0; i < kNumKs; i++)
        if ((uint32_t)kKs[i] >= k_min && (uint32_t)kKs[i] <= k_max) ks.push_back((uint32_t)kKs[i]);
    if (ks.empty() || ks[0] != k_min) ks.insert(ks.begin(), k_min);
    if (ks.back() != k_max) ks.push_back(k_max);
    for (uint32_t k : ks) {
        if ((rc = run(k, 64, 0))) break;
        if ((rc = run(k, 0, FSM_EAGER_OFF))) break;
    }
    // stage 2: windows x eager for the two fastest k
    if (rc == FSM_OK) {
        std::vector<TuneCand> s1 = tried;
        std::sort(s1.begin(), s1.end(), [](const TuneCand &a, const TuneCand &b) { return a.ms < b.ms; });
        std::vector<uint32_t> best_k;
        for (const TuneCand &c : s1)
            if (best_k.size() < 2 && std::find(best_k.begin(), best_k.end(), c.k) == best_k.end()) best_k.push_back(c.k);
        static const uint32_t lbs[] = {0, 32, 64, 128, 256};
        for (uint32_t k : best_k)
            for (uint32_t lb : lbs)
                for (uint32_t eg : {FSM_EAGER_OFF, 0u})
                    if (rc == FSM_OK) rc = run(k, lb, eg);
    }
    // stage 2b: the window walk over the top 4 / 8 image states only (R7 width) at the best windowed setting
    if (rc == FSM_OK) {
        const TuneCand *b = nullptr;
        for (const TuneCand &c : tried)
            if (c.lookback >= 32 && (!b || c.ms < b->ms)) b = &c;
        if (b) {
            const TuneCand bw = *b;
            for (uint32_t w : {4u, 8u})
                if (rc == FSM_OK) rc = run(bw.k, bw.lookback, bw.eager, bw.variant, 0, w);
        }
    }
    if (rc == FSM_OK) rc = run(1, 0, FSM_EAGER_OFF);  // the paper's plain spec-1, for reference
    // stage 3: every table variant the DFA fits, at the best (k, window, eager) so far
    if (rc == FSM_OK) {
        const TuneCand *b = nullptr;
        for (const TuneCand &c : tried)
            if (c.k >= k_min && c.k <= k_max && (!b || c.ms < b->ms)) b = &c;
        const TuneCand best_so_far = *b;
        const int base = saved.variant != FSM_VARIANT_AUTO ? saved.variant : f->auto_variant;  // what stages 1-2 ran
        for (int v = 0; v < 10 && rc == FSM_OK; v++)
            if (f->d_img[v] && v != base)
                rc = run(best_so_far.k, best_so_far.lookback, best_so_far.eager, v, 0, best_so_far.width);
    }
    // stage 4: R5 pre-resolution (top-1 vs every candidate) at the best setting so far
    if (rc == FSM_OK) {
        const TuneCand *b = nullptr;
        for (const TuneCand &c : tried)
            if (c.k >= k_min && c.k <= k_max && (!b || c.ms < b->ms)) b = &c;
        const TuneCand bb = *b;
        if (bb.k > 1)
            for (uint32_t pre : {1u, (uint32_t)FSM_KMAX})
                if (rc == FSM_OK) rc = run(bb.k, bb.lookback, bb.eager, bb.variant, pre, bb.width);
    }
    // stage 5: chunk size (half and double the geometry's choice) at the best setting so far, when the
    // caller left it adaptive and the sample is the whole input (a prefix has other tile waves: it
    // measured 16 KiB chunks 15 % slow on a 2 GiB prefix of C4 that are 16 % fast on the 8 GiB run)
    if (rc == FSM_OK && saved.chunk_bytes == 0 && n == len) {
        const TuneCand *b = nullptr;
        for (const TuneCand &c : tried)
            if (c.k >= k_min && c.k <= k_max && (!b || c.ms < b->ms)) b = &c;
        const TuneCand bb = *b;
        const uint32_t cmax = bits ? 8192u : 16384u;
        for (uint32_t ch : {bb.used_chunk / 2, bb.used_chunk * 2})
            if (rc == FSM_OK && ch >= 64 && ch % 32 == 0 && ch <= cmax)
                rc = run(bb.k, bb.lookback, bb.eager, bb.variant, bb.preresolve, bb.width, ch);
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    f->opt = saved;
    if (rc) return rc;
    const TuneCand *best = nullptr;  // the paper's reference point may lie outside [k_min, k_max]
    for (const TuneCand &c : tried)
        if (c.k >= k_min && c.k <= k_max && (!best || c.ms < best->ms)) best = &c;
    const double bytes = (double)n / (double)sym_per_byte;
    double paper_ms = 0;
    for (const TuneCand &c : tried)
        if (c.k == 1 && c.lookback == 0 && c.eager == FSM_EAGER_OFF) paper_ms = c.ms;
    out->k = best->k;
    out->lookback_len = best->lookback;
    out->eager_window = best->eager == 0 ? kExtWindow : best->eager;
    out->candidates = (uint32_t)tried.size();
    out->sample_len = n;
    out->best_gbs = best->ms > 0 ? bytes / (best->ms * 1e6) : 0.0;
    out->paper_gbs = paper_ms > 0 ? bytes / (paper_ms * 1e6) : 0.0;
    out->hit_rate = best->hit;
    out->variant = best->variant != FSM_VARIANT_AUTO ? best->variant
                 : saved.variant != FSM_VARIANT_AUTO ? saved.variant : f->auto_variant;
    out->preresolve = best->preresolve;
    out->lookback_width = best->width;
    out->chunk_bytes = best->chunk;
    f->opt.lookback_width = best->width;
    f->opt.chunk_bytes = best->chunk;
    f->opt.lookback_len = best->lookback;
    f->opt.eager_window = out->eager_window;
    f->opt.variant = out->variant;
    f->opt.preresolve = best->preresolve;
    return FSM_OK;
}

// --------------------------------------------------------- NEXT-4: many FSMs, one input ------
// DFAs are grouped by (table variant, K); each group is one fused launch (speck_multi_kernel) led
// by fsms[0]: its stream, ticket counter and Params buffer.  Every handle keeps its own
// descriptors, result and counters.
extern "C" int fsm_run_multi(fsm_t *const *fsms, uint32_t m, const uint8_t *input, uint64_t len, const uint32_t *k,
                             uint32_t *final_states, uint64_t *accept_counts)
{
    if (!fsms || m == 0 || m > FSM_MULTI_MAX || !k || !final_states || !accept_counts) return FSM_EINVAL;
    fsm *lead = fsms[0];
    for (uint32_t i = 0; i < m; i++) {
        int rc = check_run_args(fsms[i], input, len, k[i]);
        if (rc) return rc;
        if (fsms[i]->mode != lead->mode || fsms[i]->device != lead->device) return FSM_EINVAL;
        for (uint32_t j = 0; j < i; j++)
            if (fsms[j] == fsms[i]) return FSM_EINVAL;  // one result slot per handle
    }
    const bool bits = lead->mode == FSM_INPUT_BITS_MSB;
    const uint64_t len_bytes = bits ? len / 8 : len;
    // every handle runs on the leader's stream for this call
    std::vector<cudaStream_t> saved(m);
    for (uint32_t i = 0; i < m; i++) {
        saved[i] = fsms[i]->stream;
        fsms[i]->stream = lead->stream;
    }
    auto restore = [&]() {
        for (uint32_t i = 0; i < m; i++) fsms[i]->stream = saved[i];
    };
    if (lead->multi_cap < m) {
        cudaStreamSynchronize(lead->stream);
        cudaFree(lead->d_multi);
        lead->d_multi = nullptr;
        lead->multi_cap = 0;
        if (cudaMalloc(&lead->d_multi, m * sizeof(Params)) != cudaSuccess) {
            restore();
            return FSM_ECUDA;
        }
        lead->multi_cap = m;
    }
    for (uint32_t i = 0; i < m; i++)  // per-call counters of every handle
        if (cudaMemsetAsync(fsms[i]->d_stats, 0, sizeof(DevStats), lead->stream) != cudaSuccess) {
            restore();
            return FSM_ECUDA;
        }
    std::vector<int> group_of(m, -1);
    std::vector<Params> hp(m);
    int rc = FSM_OK;
    uint32_t base = 0;
    for (uint32_t i = 0; i < m && rc == FSM_OK; i++) {
        if (group_of[i] >= 0) continue;
        const int var = variant_of(fsms[i], -1, k[i]);
        const int K = kslots(k[i]);
        std::vector<uint32_t> g;
        for (uint32_t j = i; j < m; j++)
            if (group_of[j] < 0 && variant_of(fsms[j], -1, k[j]) == var && kslots(k[j]) == K) {
                group_of[j] = (int)i;
                g.push_back(j);
            }
        if (K > kMultiMaxK) {  // fused multi-FSM kernels exist for K <= 8: one launch per DFA here
            for (uint32_t j : g) {
                RunSpec r{nullptr, input, len, k[j], false, 0, fsms[j]->start_int, nullptr, fsms[j]->d_result, -1,
                          FSM_MERGE_PARALLEL};
                r.accumulate = true;
                if ((rc = launch_run(fsms[j], r))) break;
            }
            continue;
        }
        uint32_t T = 0, chunk = 0;
        pick_geometry(fsms[i], len_bytes, K, var, T, chunk);
        size_t smem = 0;
        uint32_t tbytes = 0;
        for (uint32_t n = 0; n < g.size() && rc == FSM_OK; n++) {
            fsm *f = fsms[g[n]];
            RunSpec r{nullptr, input, len, k[g[n]], false, 0, f->start_int, nullptr, f->d_result, var,
                      FSM_MERGE_PARALLEL, 0, T, chunk, true};
            Prepared pr;
            if ((rc = prepare_run(f, r, pr))) break;
            hp[base + n] = pr.p;
            smem = std::max(smem, pr.smem);
            tbytes = std::max(tbytes, pr.p.table_bytes);
        }
        if (rc) break;
        const uint32_t M = (uint32_t)g.size();
        Params gp = hp[base];
        gp.table_bytes = tbytes;
        if ((uint64_t)gp.ntiles * M > 0x7FFFFFFFull) {
            rc = FSM_EINVAL;
            break;
        }
        if (cudaMemcpyAsync(lead->d_multi + base, hp.data() + base, M * sizeof(Params), cudaMemcpyHostToDevice,
                            lead->stream) != cudaSuccess) {
            rc = FSM_ECUDA;
            break;
        }
        MultiFn fn = get_multi(var, K);
        int occ = 0;
        if (cudaFuncSetAttribute((const void *)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess ||
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, (int)T, smem) != cudaSuccess || occ < 1) {
            rc = FSM_ECUDA;
            break;
        }
        if (lead->opt.ctas_per_sm) occ = std::min<int>(occ, (int)lead->opt.ctas_per_sm);
        const uint64_t ntickets = (uint64_t)gp.ntiles * M;
        const uint32_t grid = (uint32_t)std::min<uint64_t>(ntickets, (uint64_t)occ * grid_sms(lead));
        gp.ticket = lead->d_ticket;
        gp.ticket_base = lead->ticket_base;
        fn<<<grid, T, smem, lead->stream>>>(gp, lead->d_multi + base, M);
        if (cudaGetLastError() != cudaSuccess) {
            rc = FSM_ECUDA;
            break;
        }
        lead->ticket_base += (uint32_t)ntickets + grid;
        base += M;
    }
    bool esym = false;
    for (uint32_t i = 0; i < m && rc == FSM_OK; i++) {
        fsm *f = fsms[i];
        if ((rc = finish_sync(f, f->d_result))) break;
        if (is_sink(f, f->h_result->final_state)) esym = true;
        final_states[i] = to_user(f, f->h_result->final_state);
        accept_counts[i] = f->h_result->count;
    }
    restore();
    if (rc) return rc;
    return esym ? FSM_ESYMBOL : FSM_OK;
}
