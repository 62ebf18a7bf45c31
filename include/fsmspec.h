/* fsmspec.h -- C ABI of libfsmspec: spec-k speculative FSM execution with parallel merge on B200.
 *
 * Method: Xia, Jiang & Agrawal, "Scaling Out Speculative Execution of Finite-State Machines with
 * Parallel Merge", PPoPP'20.  P:n = PAPER.md line n.
 *   - problem statement: a DFA (Q, Sigma, q0, delta, F) run over a long input      P:61 (Sec. 2.1)
 *   - Table 1 vocabulary: num_states N, num_guess k, num_inputs, num_item, num_thread
 *   - spec-k: k = 1 speculative, k = N enumerative, otherwise enumerative speculation
 *   - local processing of k speculated start states per chunk (Alg. 3)
 *   - runtime membership check (Alg. 1 nested loop / Alg. 2 hash)
 *   - parallel merge with delayed re-execution (invalid marking)
 * Result = (q_L, |{i in [1, L] : q_i in F}|): the final state and the accept-position count
 * (readings A4 and A21); it is bit-exact and independent of k, geometry,
 * look-back policy and number of GPUs.
 *
 * Conventions
 *   - Every function returns FSM_OK (0) or a negative status; out-parameters are written only
 *     on FSM_OK.  Sticky CUDA errors are reported as FSM_ECUDA and not cleared.
 *   - A handle is bound to the CUDA device that is current at fsm_create; calls on a handle
 *     must be made with that device current.  One handle must not be used concurrently from two
 *     host threads.
 *   - "device pointer" = memory on the handle's device (cudaMalloc / torch CUDA tensor).
 *     Input buffers are borrowed for the duration of the call (the async call: until the
 *     stream work completes).  The caller keeps ownership of everything it passes in.
 */
#ifndef FSMSPEC_H
#define FSMSPEC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct fsm fsm_t;

enum {
    FSM_OK = 0,
    FSM_EINVAL = -1,       /* invalid argument (see each call) */
    FSM_ENOMEM = -2,       /* device or host allocation failed */
    FSM_ECUDA = -3,        /* any CUDA runtime failure */
    FSM_ESYMBOL = -4,      /* the input contained a byte >= alphabet (reading A14) */
    FSM_EUNSUPPORTED = -5  /* current device is not sm_100 */
};

enum { FSM_INPUT_BYTES = 0, FSM_INPUT_BITS_MSB = 1 };

#define FSM_KMAX 16

/* Table-placement variants; FSM_VARIANT_AUTO picks by state count. */
enum {
    FSM_VARIANT_AUTO = -1,
    FSM_VARIANT_P4 = 0,  /* N <= 4 (byte mode): packed 4 x u8 row per symbol, lane-replicated smem, PRMT chain */
    FSM_VARIANT_P8 = 1,  /* N <= 8:   packed 8 x u8 row per symbol, lane-replicated smem, PRMT chain */
    FSM_VARIANT_B = 2,   /* N <= 256: u16 entries (next | count << 8) in shared memory            */
    FSM_VARIANT_G = 3,   /* any N:    u32 entries (next | count << 16) in global memory / L2      */
    /* 4 is retired (H8: half rows, one LDS.32 per chain step -- measured slower than P8 and N8) */
    FSM_VARIANT_HS = 5,  /* byte mode, N <= 32768: hot-state row caching (Sec. 4.2): the most frequent
                            states' rows in shared memory (u16), the rest from the u32 table in L2 */
    FSM_VARIANT_CL = 6,  /* byte mode, N x ceil(byte-classes / 2) <= 504: class-compressed, lane-replicated u16
                            table whose entries are the next row's shared address, one PRMT + LDS for the class,
                            IADD + conflict-free LDS.U16 per chain step (e.g. the HTML tokenizer)       */
    FSM_VARIANT_N8 = 7,  /* N <= 8 (byte mode): one u32 row of eight 4-bit fields per symbol, lane-replicated
                            smem (one LDS.32 per byte), chain = wrap-mode funnel shift + IMAD          */
    FSM_VARIANT_R16 = 8, /* N <= 16 (byte mode): byte entries (bare next state), lane-replicated so that lane
                            l reads bank l (128 KiB smem at N = 16), IMAD + conflict-free LDS.U8 per chain
                            step.  R16 and CL count accepts by region: byte-mode handles renumber their
                            states internally so that F (or its complement) is the top id range; results,
                            maps and debug readbacks are always in the caller's ids                   */
    FSM_VARIANT_RG = 9   /* N <= 256 (byte mode): R16's layout in 32 >> logl copies (lanes 2^logl g ..
                            share copy g, which owns banks of its own; logl = smallest with the table
                            <= 128 KiB): a warp's LDS.U8 costs the worst bank load of 2^logl lanes     */
};

/* Merge strategies: the paper's parallel merge (default) and its sequential-merge baseline
 * (Fig. 4a; the internal ablation of SURVEY.md 8.a11). */
enum { FSM_MERGE_PARALLEL = 0, FSM_MERGE_SEQUENTIAL = 1 };

/* fsm_create: build a handle for the DFA on the current device.
 *   table       host pointer, n_states * alphabet entries, state-major:
 *               delta(s, c) = table[s * alphabet + c] (Fig. 1b rows are states, P:229/P:235;
 *               reading A3).  Copied; the caller keeps it.
 *   n_states    N, 1 .. 65535.
 *   alphabet    1 .. 256 symbols; input bytes >= alphabet drive an internal absorbing sink
 *               state and make the run return FSM_ESYMBOL.
 *   start       q0 < n_states.
 *   accept_mask host pointer to n_states bytes (nonzero = in F) or NULL for F = {}.  Copied.
 *   out         receives the handle.
 * Errors: FSM_EINVAL (n_states or alphabet out of range, start or any entry >= n_states,
 * NULL table/out), FSM_EUNSUPPORTED (device is not sm_100), FSM_ENOMEM, FSM_ECUDA. */
int fsm_create(const uint32_t *table, uint32_t n_states, uint32_t alphabet, uint32_t start,
               const uint8_t *accept_mask, fsm_t **out);

/* As fsm_create; input_mode FSM_INPUT_BITS_MSB (requires alphabet == 2) reads the input as a
 * packed bitstream, 8 symbols per byte, MSB first (Huffman decoding P:288, Div7 P:360; reading
 * A13).  Lengths are then in bits. */
int fsm_create_ex(const uint32_t *table, uint32_t n_states, uint32_t alphabet, uint32_t start,
                  const uint8_t *accept_mask, uint32_t input_mode, fsm_t **out);

/* Release all device and host resources of the handle.  NULL is a no-op. */
void fsm_destroy(fsm_t *f);

/* Static string for a status code. */
const char *fsm_strerror(int status);

/* Stream the handle's work is enqueued on (a cudaStream_t); NULL = legacy default stream. */
int fsm_set_stream(fsm_t *f, void *cuda_stream);

/* fsm_run_spec_k: run spec-k over a device-resident input and return the result on the host.
 *   input   device pointer to the input (bytes; packed bits in bit mode); may be NULL iff len = 0.
 *           Any alignment is accepted; 32-byte-aligned inputs take the vectorised path.
 *   len     number of symbols (bytes; bits in bit mode).  len = 0 returns (start, 0).
 *   k       number of speculated states per chunk, 1 <= k <= min(FSM_KMAX, n_states).
 * Blocks until the result is on the host.  Errors: FSM_EINVAL, FSM_ESYMBOL, FSM_ECUDA. */
int fsm_run_spec_k(fsm_t *f, const uint8_t *input, uint64_t len, uint32_t k,
                   uint32_t *final_state, uint64_t *accept_count);

/* Result record written to device memory by the asynchronous call. */
typedef struct {
    uint32_t final_state;   /* == n_states means an out-of-alphabet byte was seen */
    uint32_t status;        /* 0 */
    uint64_t accept_count;
} fsm_result;

/* fsm_run_spec_k_async: as fsm_run_spec_k, but only enqueues the work on the handle's stream; the
 * kernel writes an fsm_result to `dev_result` (device pointer, 8-byte aligned).  No host
 * synchronisation.  `final_state == n_states` signals FSM_ESYMBOL (when alphabet < 256). */
int fsm_run_spec_k_async(fsm_t *f, const uint8_t *input, uint64_t len, uint32_t k,
                         fsm_result *dev_result);

/* fsm_run_spec_k_host: end-to-end form over a HOST buffer (pinned or pageable).  The library
 * copies the input to the device in pieces on a copy stream and overlaps each piece's copy with
 * the previous piece's kernel; pieces are chained on the device (the end state and count of piece
 * p seed piece p+1).  Same arguments, result and errors as fsm_run_spec_k. */
int fsm_run_spec_k_host(fsm_t *f, const uint8_t *host_input, uint64_t len, uint32_t k,
                        uint32_t *final_state, uint64_t *accept_count);

/* Tuning knobs; zero fields keep the current value.  Applied to subsequent runs. */
typedef struct {
    uint32_t chunk_bytes;       /* bytes per chunk (per thread), multiple of 32, <= 16384 (8192 in bit
                                   mode); 0 = adaptive (power-of-two chunks by a wave model) */
    uint32_t threads_per_tile;  /* chunks per tile (CTA size), 64 .. 1024, multiple of 32 */
    int32_t variant;            /* FSM_VARIANT_*; FSM_VARIANT_AUTO = by state count */
    uint32_t merge;             /* FSM_MERGE_* */
    uint32_t ctas_per_sm;       /* cap on resident CTAs per SM for the persistent grid; 0 = max */
    uint32_t lookback_len;      /* look-back: 0 or 1 = the byte before the chunk; 32..1024 (multiple
                                   of 32) = run the image of the byte before a window of that many bytes
                                   through the window and rank the reached states by multiplicity */
    uint32_t eager_window;      /* NEXT-3 eager completion: per chunk, the next look-back
                                   candidates beyond the k speculated ones run in lockstep with the chains
                                   over the chunk's first eager_window bytes, recording where they meet a
                                   chain.  0 = default (128), FSM_EAGER_OFF = off, else 32..128 in steps
                                   of 32.  Results are identical either way; only the re-execution work
                                   changes. */
    uint32_t preresolve;        /* delayed re-execution across tiles: a tile publishes its
                                   aggregate mapping (one slot per speculated tile start) for the
                                   decoupled look-back; the broken slots of the top `preresolve` start
                                   candidates (rank order) are re-executed before publishing, so a
                                   successor passes through them without waiting; the others are
                                   published invalid and re-executed only if the true path enters the
                                   tile in them.  0 = default: the top candidate only, or every
                                   candidate when every symbol permutes the states (paths never meet,
                                   so a lazily resolved candidate is a whole-chunk re-execution chain);
                                   1..FSM_KMAX = top n (n >= k: every slot); FSM_PRERESOLVE_NONE = only
                                   the true path is ever re-executed.  Identical results. */
    uint32_t grid_sms;          /* SMs the persistent grids use (0 = all): the grid-size sweep of the
                                   sequential- vs parallel-merge ablation (Figs. 7-11 vary the number of
                                   thread blocks) */
    uint32_t check;             /* runtime membership check of the merge: FSM_CHECK_AUTO (default),
                                   FSM_CHECK_NESTED = Alg. 1 (O(k^2)), FSM_CHECK_HASH = Alg. 2
                                   (O(k), per-thread shared-memory buckets); the hash form is
                                   built for k > 8 (instantiated K = 12, 16) and falls back to Alg. 1
                                   where its scratch does not fit next to the table.  Identical results. */
    uint32_t lookback_width;    /* look-back window walk (lookback_len >= 32): only the top lookback_width
                                   states of the image (by preimage count, A5) are run through the window
                                   and ranked; 0 = default (the whole image, up to FSM_KMAX), else 4, 8,
                                   12 or 16.  Only the speculation (and so the re-execution work) changes. */
} fsm_options;

#define FSM_EAGER_OFF 1u
#define FSM_PRERESOLVE_NONE 0x80000000u
enum { FSM_CHECK_AUTO = 0, FSM_CHECK_NESTED = 1, FSM_CHECK_HASH = 2 };

int fsm_set_options(fsm_t *f, const fsm_options *opt);
int fsm_get_options(const fsm_t *f, fsm_options *opt);

/* Counters of the most recent run call on this handle (synchronous or asynchronous; every run
 * call resets them, fsm_run_spec_k_host sums its pieces).  Re-execution rate = reexec_true /
 * chunks.  "True path" = the run of the actual start state (keyed shard runs:
 * of every valid shard slot); a8 allows re-execution only there.  Candidate-path
 * re-executions are the optional pre-resolution of tile-start candidates (fsm_options.preresolve)
 * that turned out not to be taken. */
typedef struct {
    uint64_t chunks;            /* chunks processed (one thread each) */
    uint64_t tiles;             /* tiles (CTAs' work units) */
    uint64_t reexec_chunks;     /* all chunk re-executions = reexec_true + reexec_candidate */
    uint64_t reexec_symbols;    /* bytes consumed by them (early exit on convergence) */
    uint64_t boundary_misses;   /* tile-boundary misses: true tile start not speculated */
    uint64_t reexec_true;       /* chunk re-executions on the true path */
    uint64_t reexec_true_symbols;
    uint64_t reexec_candidate;  /* chunk re-executions on tile-start candidate paths not taken */
    uint64_t reexec_candidate_symbols;
    uint64_t eager_resolved;    /* true-path misses completed from an eager-completion entry (NEXT-3) */
    uint64_t max_miss_chain;    /* longest run of consecutive re-executed chunks on the true path */
    uint32_t chunk_bytes, threads_per_tile, variant, k_slots, lookback_len, preresolve;
    uint32_t check;             /* FSM_CHECK_NESTED or FSM_CHECK_HASH: the check the run used */
    uint32_t lookback_width;    /* image states the look-back window walk ran (0: no window walk) */
} fsm_stats;

/* Synchronises the handle's stream (the counters live on the device). */
int fsm_get_stats(const fsm_t *f, fsm_stats *s);

/* ---------------------------------------------------------------- shard level (multi-GPU) ---
 * A shard is a contiguous piece [lo, hi) of a longer input.  Shard 0 starts in
 * q0; shard g > 0 speculates its start from the look-back byte just before it (the halo) and
 * returns a k-slot mapping keyed on that speculated set, exactly as a chunk does. */
typedef struct {
    uint32_t k;                     /* slots in use */
    uint32_t valid_mask;            /* bit s set = slot s holds a start state */
    uint32_t start[FSM_KMAX];
    uint32_t end[FSM_KMAX];
    uint64_t count[FSM_KMAX];
} fsm_shard_map;

typedef struct fsm_shard fsm_shard_t;  /* per-shard state kept for a later fix-up */

/* fsm_run_shard: run one shard.  An out-of-alphabet byte inside the shard drives every path into
 * the sink, so it is reported as FSM_ESYMBOL here (no map is written).
 *   input, len  device pointer and length (bytes, or bits in bit mode; bit-mode shards must start
 *               on a byte boundary, i.e. every shard but the last has len % 8 == 0).
 *   halo        device pointer to the halo_len bytes immediately before the shard, or NULL with
 *               halo_len = 0 for shard 0 (start = q0).  Only the last halo byte is used.
 *   out         receives the mapping; state (optional) receives a handle for fsm_shard_fixup,
 *               which borrows `input` until fsm_shard_free.
 * Errors: FSM_EINVAL, FSM_ESYMBOL, FSM_ECUDA, FSM_ENOMEM. */
int fsm_run_shard(fsm_t *f, const uint8_t *input, uint64_t len, const uint8_t *halo,
                  uint32_t halo_len, uint32_t k, fsm_shard_map *out, fsm_shard_t **state);

/* fsm_shard_fixup: the shard's true start state turned out not to be speculated (a shard-boundary
 * miss).  Re-executes from the shard start in lockstep with the speculated chains and stops when
 * it joins one (exact); falls back to a full parallel re-run of the shard from `true_start`. */
int fsm_shard_fixup(fsm_t *f, fsm_shard_t *state, uint32_t true_start, uint32_t *end,
                    uint64_t *count);

void fsm_shard_free(fsm_shard_t *state);  /* NULL is a no-op */

/* fsm_map_compose: host-only, pure.  out = a followed by b, keyed on a's starts: a slot of a
 * whose end is a start of b continues with b's end and adds counts; otherwise it becomes invalid
 * (delayed strategy).  out may alias a or b. */
int fsm_map_compose(const fsm_shard_map *a, const fsm_shard_map *b, fsm_shard_map *out);

/* fsm_compose_from: host-only, pure.  Follows the state `start_state` (count `start_count`) through
 * maps[0 .. n) in order -- at each map, the valid slot whose start equals the current state gives
 * the next state and adds its count (the membership check of Alg. 1, applied to shard
 * maps, SURVEY.md 8.e "Compose").  Stops at the first map with no such slot: *first_miss = its
 * index (that shard's true start was not speculated; the caller runs fsm_shard_fixup there and
 * continues from map first_miss + 1), or n when every map matched.  *state / *count are the state
 * and count before maps[*first_miss] (after the last map when *first_miss == n).
 * Errors: FSM_EINVAL (NULL pointers with n > 0). */
int fsm_compose_from(const fsm_shard_map *maps, uint32_t n, uint32_t start_state, uint64_t start_count,
                     uint32_t *state, uint64_t *count, uint32_t *first_miss);

/* ------------------------------------------------------------- NEXT-2: k / look-back tuning ---
 * The paper leaves the choice of k to the user and names a cost model for it as future work
 * (Figs. 12-13, show the best k differs by FSM and input).  fsm_autotune picks
 * k, the look-back window (reading R7) and the eager-completion window (NEXT-3) for one
 * DFA and input by timing the real kernel on a prefix sample of the input -- a measured cost
 * model: every candidate's cost is its own sampled time, which already includes its sampled
 * re-execution (miss) rate.  The search is staged: (1) every instantiated k in [k_min, k_max] with the
 * default window (64 bytes, eager on) and with the paper's depth-1 look-back (eager off); (2) for
 * the two fastest k, look-back windows {0, 32, 64, 128, 256} x eager {off, 128}; (3) for the chosen
 * setting, every table variant the DFA fits (the by-size default is a heuristic: e.g. a random
 * 1024-state DFA runs faster with hot-state caching, a 1027-state Aho-Corasick DFA without); (4) for
 * k > 1, pre-resolution of the top tile-start candidate vs every candidate (fsm_options.preresolve).
 *   input, len   device pointer and length (symbols) of the input the runs will process
 *   k_min, k_max smallest / largest k to consider (0 = 1 / min(FSM_KMAX, n_states); k_min = k_max
 *                tunes only the windows for that k)
 *   sample_len   symbols timed per candidate (0 = min(len, 4 GiB)); the prefix is used, run with the
 *                chunk and tile geometry of the full length so its cost per byte is the full run's
 *   out          the choice and its evidence; the chosen lookback_len / eager_window / variant are
 *                also written into the handle's options (the caller passes out->k to the runs)
 * Results of runs are identical under every setting; only speed changes.  Synchronises the
 * handle's stream.  Errors: FSM_EINVAL, FSM_ECUDA. */
typedef struct {
    uint32_t k;                 /* chosen k */
    uint32_t lookback_len;      /* chosen look-back window (0 = depth-1 look-back) */
    uint32_t eager_window;      /* chosen eager-completion window (FSM_EAGER_OFF = off) */
    uint32_t candidates;        /* configurations timed */
    uint64_t sample_len;        /* symbols per timed run */
    double best_gbs;            /* sample bytes / median time of the chosen configuration */
    double paper_gbs;           /* same for the paper's plain setting: k = 1, depth-1 look-back, no eager */
    double hit_rate;            /* 1 - re-executed chunks / chunks, chosen configuration */
    int32_t variant;            /* chosen table variant (FSM_VARIANT_*), applied to the options */
    uint32_t preresolve;        /* chosen fsm_options.preresolve (0 = the default policy), applied */
    uint32_t lookback_width;    /* chosen fsm_options.lookback_width (0 = the whole image), applied */
    uint32_t chunk_bytes;       /* chosen fsm_options.chunk_bytes (0 = adaptive), applied; tuned only
                                   when the handle's chunk_bytes was adaptive */
} fsm_tuning;

int fsm_autotune(fsm_t *f, const uint8_t *input, uint64_t len, uint32_t k_min, uint32_t k_max,
                 uint64_t sample_len, fsm_tuning *out);

/* -------------------------------------------------- NEXT-4: many FSMs over one resident input ---
 * The network-intrusion case the paper uses to justify amortised layout work: M
 * DFAs scan the same input.  fsm_run_multi computes, for each DFA i, exactly what
 * fsm_run_spec_k(fsms[i], input, len, k[i]) computes, in fused launches: DFAs with the same table
 * variant and instantiated K share one persistent grid, whose CTAs take (tile, DFA) pairs in
 * tile-major order so that the input is read from HBM about once per group (the other DFAs hit
 * the tile in L2).  Each handle's own options (look-back, eager window) apply; the chunk and tile
 * geometry are the first handle of each group's.  DFAs run with k > 8 are not fused (one launch
 * each, same results).
 *   fsms, m        1 <= m <= FSM_MULTI_MAX distinct handles, same input mode and device; the work is
 *                  enqueued on fsms[0]'s stream
 *   input, len     as fsm_run_spec_k (one input for all)
 *   k              m values, each valid for its handle
 *   final_states, accept_counts   m results each (user state ids)
 * Blocks until the results are on the host; each handle's fsm_get_stats describes its own run.
 * Errors: FSM_EINVAL, FSM_ECUDA; FSM_ESYMBOL if any DFA saw an out-of-alphabet byte (results are
 * still written; that DFA's final state is then n_states). */
#define FSM_MULTI_MAX 64u
int fsm_run_multi(fsm_t *const *fsms, uint32_t m, const uint8_t *input, uint64_t len, const uint32_t *k,
                  uint32_t *final_states, uint64_t *accept_counts);

/* ----------------------------------------------------------------------- host-only helpers ---
 * fsm_lookback_table: the look-back speculation table the library builds at fsm_create (host
 * code, no GPU needed).  For every input byte c: the image {delta(s, c)} (bit mode: of the
 * 8-bit widened step) ranked by preimage count descending, ties to the smaller id (P:71,
 * reading A5).  lb_out: 256 * FSM_KMAX uint16 (0xFFFF = unused), nimg_out: 256 bytes =
 * min(|image|, FSM_KMAX).  States are internal ids (the sink, if any, is id n_states). */
int fsm_lookback_table(const uint32_t *table, uint32_t n_states, uint32_t alphabet,
                       uint32_t input_mode, uint16_t *lb_out, uint8_t *nimg_out);

/* ---------------------------------------------------------------------- test-only hooks ---
 * Used by tests to replay the paper's worked examples on the CUDA merge (Fig. 2; Fig. 4,
 * P:103-105; SURVEY.md 8.b "Python layer" and 8.c.3 P2-P4).  Not for production use.
 *
 * fsm_debug_set_spec: fix the geometry of the following runs on f to chunks of `chunk_bytes` bytes
 * (1 .. 8192, any value) in tiles of 32 chunks, and -- if `sets` is not NULL -- inject the
 * speculated start sets: sets[j * k + s] = slot s of chunk j (user state ids, 0xFFFFFFFF = no
 * state), for chunks 0 .. n_chunks-1, chunk 0 included (this overrides reading A7's S_0 = {q0};
 * the true start must then be one of chunk 0's slots or is resolved by re-execution like any
 * miss).  Runs must have exactly n_chunks chunks and the same k.  The look-back window and eager
 * completion are off while injected.  chunk_bytes = 0 clears everything.
 * Errors: FSM_EINVAL (k out of range, a state >= n_states, n_chunks = 0 with sets). */
int fsm_debug_set_spec(fsm_t *f, const uint32_t *sets, uint32_t n_chunks, uint32_t k, uint32_t chunk_bytes);

/* The merge tree of tile 0, warp 0 of the most recent run made under fsm_debug_set_spec: level 0 =
 * each chunk's own mapping M_j (lane j), level l = lane j's mapping after the l-th warp-scan level,
 * i.e. M_j x ... x M_{j + 2^l - 1} (Fig. 4b: level 1 lane 0 = chunks 0+1, lane 2 = chunks 2+3,
 * level 2 lane 0 = the root).  Slot s of lane j at level l: start = speculated start of chunk j
 * (0xFFFFFFFF = none); valid = the slot's run passed every membership check so far;
 * end / count = the state reached and F-visits (meaningful when valid; when invalid, end = the
 * state at the chunk where the check failed and brk = that chunk's index).  States in user ids. */
typedef struct {
    uint32_t k;                              /* slots per mapping (the run's instantiated K) */
    uint32_t start[6][32][FSM_KMAX];
    uint32_t end[6][32][FSM_KMAX];
    uint32_t count[6][32][FSM_KMAX];
    uint32_t brk[6][32][FSM_KMAX];           /* 0xFFFFFFFF = valid; 0xFFFFFFFE = no state */
    uint32_t identity[6][32];                /* lane held no chunk (past the end of the input) */
} fsm_debug_merge;

int fsm_debug_get_merge(const fsm_t *f, fsm_debug_merge *out);

/* fsm_hot_state_order: the static frequency order of hot-state caching (Sec. 4.2; NEXT-1),
 * host only: user state ids sorted by in-degree in the byte-level transition table (bit mode: the
 * widened table) descending, ties to the smaller id.  The HS variant keeps the rows of a prefix of
 * this order in shared memory.  order_out: n_states entries.  Errors: FSM_EINVAL. */
int fsm_hot_state_order(const uint32_t *table, uint32_t n_states, uint32_t alphabet, uint32_t input_mode,
                        uint32_t *order_out);

/* Library version string. */
const char *fsm_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FSMSPEC_H */
