/*
 * abs.h — C ABI of the B200-native Adaptive Bulk Search (ABS) hot path.
 *
 * Method: Yasudo, Nakano, Ito, Tatekawa, Katsuki, Yazane, Inaba, "Adaptive
 * Bulk Search: Solving Quadratic Unconstrained Binary Optimization Problems
 * on Multiple GPUs", ICPP 2020.  Citations "P:Lnnn" are line numbers of
 * /root/reference/PAPER.md; "reading Cnn" refers to DESIGN.md §Readings.
 *
 * Problem: given an n x n symmetric int16 weight matrix W, find an
 * n-bit vector X minimising E(X) = X^T W X = sum_{i,j} W_ij x_i x_j (Eq.(1)).
 *
 * Conventions shared by every call:
 *   - Bit vectors: bit i of X is bit (i & 31) of uint32 word (i >> 5); a vector
 *     has words(n) = ceil(n / 32) words; on input bits >= n are ignored, on
 *     output they are 0.
 *   - Energies are int64 (P:L519 prints -33,115,098,990 > 2^31); per-bit
 *     deltas Delta_i(X) = E(flip_i X) - E(X) (Eq.(11)) are int32,
 *     exact for n <= 32768 (reading C12).
 *   - Every call returns ABS_OK (0) or a negative ABS_E* code; no C++
 *     exception crosses the ABI.  A context is NOT thread-safe: one caller
 *     thread per context.  The library owns its CUDA streams, device memory
 *     and (async mode) its host GA thread.
 *   - "Host" pointers are ordinary CPU memory owned by the caller; the
 *     library copies what it needs before returning.  Calls whose names end
 *     in _dev take CUDA device pointers on the context's device.
 *   - There is no CPU fallback: a context can only be created on a CUDA
 *     device of compute capability 10.0 (B200, sm_100a); otherwise
 *     abs_create returns ABS_ECUDA.
 */
#ifndef ABS_H
#define ABS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define ABS_API __attribute__((visibility("default")))
#else
#define ABS_API
#endif

#define ABS_OK 0
#define ABS_EINVAL (-1)   /* bad argument (n out of range, W not symmetric, NULL, ...) */
#define ABS_ENOMEM (-2)   /* host or device allocation failed */
#define ABS_ECUDA (-3)    /* CUDA runtime error or no sm_100 device */
#define ABS_ENCCL (-4)    /* reserved for the multi-GPU elite exchange; the
                           * library itself makes no NCCL call: the exchange runs in the
                           * caller's process group (dist.py, torch.distributed over NCCL),
                           * which reports its own errors */
#define ABS_ESTATE (-5)   /* call not valid in the current state */
#define ABS_EEMPTY (-6)   /* no finite-energy solution in the pool yet */
#define ABS_ERANGE (-7)   /* a Delta left the int32 range (cannot happen for n <= 32768) */

#define ABS_N_MAX 32768   /* 32k bits, P:L23 / P:L416 */
#define ABS_LADDER_MAX 32

/* Search modes. */
#define ABS_MODE_LOCKSTEP 0 /* deterministic: every search runs one round per
                             * step, the host inserts all results in global
                             * search-id order, then generates the next
                             * targets.  Bit-exact with
                             * the oracle. */
#define ABS_MODE_ASYNC 1    /* the paper's system (Fig. 5): a
                             * persistent kernel and a host GA thread exchange
                             * targets and results through pinned buffers
                             * without synchronising. */

/* Local-search policies ("any policy, including a greedy algorithm
 * and SA"; reading E2). */
#define ABS_POLICY_WINDOW 0 /* Fig. 2 / P:L305: argmin over a sliding window of l bits */
#define ABS_POLICY_SA 1     /* Eq.(7) / Alg. 1: random bit, accepted if dE <= 0, else
                             * with p = exp(-dE/(k_B t)) = 2^(-dE/tau), k_B t = tau/ln 2,
                             * as the exact Q32 integer P = floor(2^32 p) (reading E2);
                             * proposals from Philox4x32-10, key = seed, counter =
                             * (lo32(c), hi32(c), global search id, 'SAPL'), c = the
                             * search's proposal count (persists across rounds);
                             * k = out[0] mod n, accepted iff out[1] < P(dE, tau).
                             * local_flips counts proposals. */

typedef struct abs_config {
    int32_t searches;       /* searches run by this context (per GPU); 0 -> one wave:
                             * abs_device_searches(n, device) (148 at n = 32768) */
    int32_t search_offset;  /* global id of this context's first search
                             * (multi-GPU partitioning) */
    int64_t local_flips;    /* L: forced flips of the local search per round
                             * ("fixed number of flips"); 0 -> n (reading C8) */
    int32_t pool_size;      /* m: solutions kept by the host GA; 0 -> 64 */
    int32_t ladder_len;     /* window lengths l ("temperature"):      */
    int32_t ladder[ABS_LADDER_MAX]; /* search s uses ladder[s mod ladder_len];
                             * ladder_len 0 -> {4,8,..,min(256,n/4)} (reading C7) */
    uint64_t seed;          /* Philox key for the pool and GA draws */
    int32_t p_cross;        /* per-mille; <0 -> 450 (reading C10) */
    int32_t p_mut;          /* per-mille; <0 -> 450; copy = 1000 - p_cross - p_mut */
    int32_t mut_max;        /* mutation flips 1 + (u mod mut_max) bits; 0 -> max(1, n/32) */
    int32_t mode;           /* ABS_MODE_LOCKSTEP or ABS_MODE_ASYNC */
    int32_t external_merge; /* lockstep only: 1 = do NOT insert this context's
                             * results into its pool; the caller inserts the
                             * results of all ranks with abs_pool_insert (in
                             * global search-id order) before the next step */
    int32_t device;         /* CUDA device ordinal; -1 -> current device */
    int32_t trace;          /* async only: 1 = record, per round, the target the
                             * search used and its (B, E_B) (abs_trace_*), so a
                             * run can be replayed exactly; costs host memory */
    int32_t policy;         /* ABS_POLICY_WINDOW (default) or ABS_POLICY_SA */
    int32_t sa_tau_min;     /* SA temperatures ("a different temperature for each */
    int32_t sa_tau_max;     /* search"): search s (global id) at level     */
    int32_t sa_levels;      /* j = s mod K has tau = min + (max-min) j / (K-1)
                             * (integer division); 0 -> min = max(1, max_ij |W_ij|),
                             * max = min, K = 1 */
    int32_t reserved[3];    /* must be 0 */
} abs_config;

typedef struct abs_stats {
    int64_t flips;            /* flips done by all searches (straight + local) */
    int64_t straight_flips;   /* of which straight-search flips (Alg. 5) */
    int64_t evaluated;        /* searched solutions = flips * n */
    int64_t rounds;           /* completed rounds (device Steps 2-5), all searches */
    double search_seconds;    /* device time inside abs_search (CUDA events) */
    int64_t pool_inserted;    /* accepted pool insertions */
    int32_t n;
    int32_t n_pad;            /* padded length used on device (multiple of 1024) */
    int32_t searches;
    int32_t threads_per_search;
    int64_t steps;            /* abs_search steps completed */
    int64_t h2d_bytes;        /* bytes copied host->device by the library */
    int64_t d2h_bytes;        /* bytes copied device->host by the library */
    int64_t kernel_launches;  /* kernels launched by the library */
    double step_seconds;      /* device time (CUDA events on the library stream)
                               * from entry to exit of every abs_search call,
                               * host GA gaps included */
    int64_t round_kernel_launches; /* launches of the search (round) kernel */
    double init_seconds;      /* device time of the last batched initialisation
                               * (abs_energy / abs_energy_dev / abs_seed_pool;
                               * CUDA events around its kernels) */
} abs_stats;

typedef struct abs_ctx abs_ctx;

/* Fill *cfg with defaults (all fields 0 / -1 as documented above). */
ABS_API void abs_config_init(abs_config *cfg);

/* Create a context for an instance.  W: host, row-major n x n
 * int16, must be symmetric (W_ij = W_ji) else ABS_EINVAL; copied,
 * caller keeps ownership.  1 <= n <= 32768.  cfg may be NULL (defaults).
 * Every search starts from the zero vector with E = 0 and Delta_i = W_ii
 * (device Step 1).  The pool starts as m Philox random bit
 * vectors with E = +infinity (host Step 1). */
ABS_API int abs_create(abs_ctx **out, int32_t n, const int16_t *W, const abs_config *cfg);

/* As abs_create, but W is a device pointer (row-major n x n int16) on the
 * configured device; it is copied, the caller keeps ownership. */
ABS_API int abs_create_dev(abs_ctx **out, int32_t n, const int16_t *W_dev, const abs_config *cfg);

/* Seed the host pool.  X == NULL: re-draw the Philox random pool with E =
 * +infinity.  Otherwise X is `count` host bit vectors; their
 * energies are computed ON THE DEVICE by the batched initialisation kernel
 * (the host never computes an energy) and they are inserted with the
 * pool rule (abs_pool_insert).  Valid before or between abs_search calls. */
ABS_API int abs_seed_pool(abs_ctx *c, const uint32_t *X, int32_t count);

/* Run `steps` steps (steps >= 0); blocks until done.
 *   lockstep: each step = host GA generates one target per search from the
 *     pool, every search runs one round — read target, reset best,
 *     straight search C -> T, L window-policy local flips, emit (B, E_B)
 *     (device Steps 2-5) — then the results are inserted in
 *     search-id order (unless external_merge).
 *   async: the persistent kernel runs until steps * searches more rounds
 *     have been emitted in total; the host GA thread inserts results and
 *     writes new targets while it runs.  When all searches are
 *     resident each runs at its own pace (rounds per search may differ);
 *     otherwise every search does exactly `steps` rounds. */
ABS_API int abs_search(abs_ctx *c, int64_t steps);

/* Best solution found so far: the host keeps the pool sorted by energy,
 * E(X_0) < E(X_1) < ..., so this is pool[0].  X_out: host,
 * words(n) words; *E_out: host.  ABS_EEMPTY if no finite energy exists yet. */
ABS_API int abs_best(const abs_ctx *c, uint32_t *X_out, int64_t *E_out);

/* Counters since create (abs_stats above): flips, and searched solutions =
 * flips * n, the paper's search-rate accounting (every flip evaluates all n
 * neighbours in O(1) each); device seconds by CUDA events. */
ABS_API int abs_stats_get(const abs_ctx *c, abs_stats *s);

/* Top-k finite pool entries (ascending energy).  X_out: k*words(n) words,
 * E_out: k.  *count_out = number written (<= k). */
ABS_API int abs_pool_get(const abs_ctx *c, int32_t k, uint32_t *X_out, int64_t *E_out, int32_t *count_out);

/* Insert `count` (X, E) pairs in the given order with the pool rule
 * (P:L359): binary search on E; rejected if an entry with the same
 * energy exists (reading C10) or E is not better than the worst entry;
 * otherwise inserted in order and the worst entry dropped.  E must be the
 * true energy of X (it is not recomputed).  *inserted_out may be NULL. */
ABS_API int abs_pool_insert(abs_ctx *c, const uint32_t *X, const int64_t *E, int32_t count, int32_t *inserted_out);

/* Batched initialisation: for `count` host bit vectors compute
 * E (Eq.(1)) and, if delta_out != NULL, all Delta_i (Eq.(13)) on the
 * device.  E_out: count int64; delta_out: count*n int32 (row-major). */
ABS_API int abs_energy(abs_ctx *c, const uint32_t *X, int32_t count, int64_t *E_out, int32_t *delta_out);

/* Engines of the batched initialisation. */
#define ABS_INIT_AUTO 0 /* the tensor-core engine */
#define ABS_INIT_ALU 1  /* plain integer kernel: conditional row adds, W read once per 16 solutions */
#define ABS_INIT_MMA 2  /* tensor cores: S = X Wz^T as two exact int8 GEMMs,
                         * W = 256 hi + lo (hi s8, lo u8), tcgen05.mma kind::i8 with int32
                         * TMEM accumulators; the int8 planes of W (2 n_pad^2 bytes) are
                         * built on first use and kept with the context */

/* Batched initialisation on DEVICE buffers (same operation as abs_energy,
 * Eq.(1) and Eq.(13)): X_dev = count bit vectors of
 * words(n) uint32 each (ABI bit order; bits >= n ignored), E_dev = count
 * int64 (overwritten), delta_dev = count*n int32 row-major or NULL.  All
 * pointers are device memory of the context's device, owned by the caller.
 * Blocking; results are exact in every engine.  ABS_EINVAL for bad
 * arguments or engine, ABS_ENOMEM if the planes / staging cannot be
 * allocated, ABS_ECUDA on a CUDA error. */
ABS_API int abs_energy_dev(abs_ctx *c, const uint32_t *X_dev, int32_t count, int64_t *E_dev, int32_t *delta_dev,
                           int32_t engine);

/* Lockstep: the (B, E_B) every local search emitted in the last step, in
 * local search order.  B_out: searches*words(n) words, EB_out: searches. */
ABS_API int abs_round_results(const abs_ctx *c, uint32_t *B_out, int64_t *EB_out);

/* Lockstep: the targets T the searches used in the last step. */
ABS_API int abs_round_targets(const abs_ctx *c, uint32_t *T_out);

/* Async trace (cfg.trace = 1): number of recorded rounds. */
ABS_API int abs_trace_count(const abs_ctx *c, int64_t *count);

/* Async trace entry i (arrival order): local search index, round number,
 * the target T the round used (words(n)), and its (B, E_B).  Any output may
 * be NULL. */
ABS_API int abs_trace_get(const abs_ctx *c, int64_t i, int32_t *s_out, int32_t *round_out, uint32_t *T_out,
                          uint32_t *B_out, int64_t *EB_out);

/* Per-search state (debug / parity): current solution C (words(n)), Delta
 * (n int32), E, window offset a, window length l, FNV-1a-64 hash of the flip
 * sequence (h = (h ^ k) * 0x100000001b3 from 0xcbf29ce484222325), flips.
 * Any output pointer may be NULL.  `s` is the local search index. */
ABS_API int abs_search_state(const abs_ctx *c, int32_t s, uint32_t *X_out, int32_t *delta_out, int64_t *E_out,
                     int32_t *a_out, int32_t *l_out, uint64_t *hash_out, int64_t *flips_out);

/* Stops the host GA thread (the host side of the system),
 * frees the context's device and pinned host memory.  c may be NULL. */
ABS_API void abs_destroy(abs_ctx *c);

ABS_API const char *abs_strerror(int rc);

/* Human-readable detail of the last error returned on the calling thread
 * (never NULL; "" if none). */
ABS_API const char *abs_last_error(void);

/* Diagnostics: per-search, per-warp cycle accounting of the lockstep round
 * kernel ([searches][32][24] int64; [0..5] local flips: window selection,
 * row wait, row update, publish/bookkeeping, barrier, tail; [6] local flips;
 * [8..14] the same for straight flips; the rest reserved).  Only in a
 * library built with -DABS_TIMING; otherwise ABS_EINVAL. */
ABS_API int abs_debug_timing(const abs_ctx *c, long long *out);

/* Ising front end.  The Ising Hamiltonian
 *     H(S) = -sum_{i<j} J_ij s_i s_j - sum_i h_i s_i,   s_i in {-1,+1}
 * maps to a QUBO (each bit is a spin, value 0/1 instead of -1/+1) by
 * s_i = 2 x_i - 1, so that H(S) = E(X) + offset with E of Eq.(1):
 *     W_ij = -2 J_ij (i != j),  W_ii = 2 sum_{j!=i} J_ij - 2 h_i,
 *     offset = sum_i h_i - sum_{i<j} J_ij.
 * Host-only (no GPU).  J: n x n int32 row-major, only i < j is read (J_ij for
 * the pair); h: n int32.  W_out: n x n int16 (symmetric), *offset_out int64.
 * ABS_ERANGE if some W entry leaves int16; ABS_EINVAL for bad arguments. */
ABS_API int abs_ising_to_qubo(int32_t n, const int32_t *J, const int32_t *h, int16_t *W_out, int64_t *offset_out);

/* Inverse map, exact in integers: J2_out = 2 J (n x n, zero diagonal,
 * symmetric), h2_out = 2 h (n), *offset2_out = 2 * offset, with
 * J_ij = -W_ij / 2, h_i = -(sum_j W_ij) / 2, offset = sum h - sum_{i<j} J.
 * Host-only.  Any output may be NULL. */
ABS_API int abs_qubo_to_ising(int32_t n, const int16_t *W, int32_t *J2_out, int32_t *h2_out, int64_t *offset2_out);

/* Number of searches whose CTAs are co-resident on `device` for an
 * n-bit instance (SMs x resident round-kernel CTAs per SM): the search
 * count that fills the GPU in one wave ("blocks ... run in
 * parallel").  Needs a visible CUDA device (ABS_ECUDA otherwise). */
ABS_API int abs_device_searches(int32_t n, int32_t device, int32_t *out);

/* Synthetic random QUBO instance (the paper's random benchmark, P:L468:
 * "uniform random" weights) generated directly in device memory, so each
 * rank of a multi-GPU run builds its replica of W (2 GiB at n = 32768)
 * without staging it through host memory.  W_dev: n*n int16,
 * row-major, device memory of `device` (-1: current), owned by the caller;
 * overwritten with a symmetric W whose upper triangle (i <= j) is
 *   W_ij = int16 half (j & 1) of word ((j >> 1) & 3) of
 *          Philox4x32-10(key = (lo32 seed, hi32 seed), counter = (i, j >> 3, 0x52514243, 0))
 * (i.i.d. uniform over all 65536 values) and W_ji = W_ij.  Blocking.
 * ABS_EINVAL for n outside [1, 32768] or W_dev == NULL, ABS_ECUDA on a CUDA error. */
ABS_API int abs_random_qubo_dev(int32_t n, uint64_t seed, int16_t *W_dev, int32_t device);

/* Library version string. */
ABS_API const char *abs_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ABS_H */
