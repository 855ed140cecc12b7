// Host side of libabs: context, device layout, host GA (pool + targets) and
// the search drivers behind the C ABI of include/abs.h.
// Citations: /root/reference/PAPER.md line numbers (P:Lnnn); readings Cnn in DESIGN.md.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <climits>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <thread>
#include <vector>

#include "abs.h"
#include "abs_internal.h"
#include "philox.hpp"

namespace absb {

constexpr uint32_t kTagPool = 0x504F4F4Cu;  // 'POOL'
constexpr uint32_t kTagGA = 0x47415447u;    // 'GATG'
constexpr int64_t kEInf = INT64_MAX;        // "+infinity" energy

thread_local std::string g_last_error;

static int fail(int rc, const std::string &what)
{
    g_last_error = what;
    return rc;
}

#define ABS_CU(expr)                                                                                 \
    do {                                                                                             \
        cudaError_t e_ = (expr);                                                                     \
        if (e_ != cudaSuccess)                                                                       \
            return ::absb::fail(ABS_ECUDA, std::string(#expr) + ": " + cudaGetErrorString(e_));      \
    } while (0)

#define ABS_CK(expr)                                                                                 \
    do {                                                                                             \
        int e_ = (expr);                                                                             \
        if (e_ != 0)                                                                                 \
            return ::absb::fail(ABS_ECUDA, std::string(#expr) + ": " +                               \
                                               cudaGetErrorString(static_cast<cudaError_t>(e_)));    \
    } while (0)

static int words_of(int n) { return (n + 31) / 32; }

// ------------------------------------------------------------------ solution pool
struct Pool {
    int n = 0, m = 0, words = 0;
    std::vector<int64_t> E;   // ascending; distinct finite values; +inf entries last
    std::vector<uint32_t> X;  // m x words

    void init(int n_, int m_) {
        n = n_; m = m_; words = words_of(n_);
        E.assign(m, kEInf);
        X.assign((size_t)m * words, 0u);
    }
    // Host Step 1: random bit vectors with energy +infinity.
    void randomize(uint64_t seed) {
        const Philox4x32x10 rng(seed);
        for (int e = 0; e < m; ++e) {
            uint32_t *x = &X[(size_t)e * words];
            for (int q = 0; 4 * q < words; ++q) {
                const auto blk = rng({static_cast<uint32_t>(q), static_cast<uint32_t>(e), 0u, kTagPool});
                for (int u = 0; u < 4 && 4 * q + u < words; ++u) x[4 * q + u] = blk[u];
            }
            if (n % 32) x[words - 1] &= (1u << (n % 32)) - 1u;
            E[e] = kEInf;
        }
    }
    // Distinct sorted insert, reading C10: same energy = same solution.
    bool insert(const uint32_t *x, int64_t e) {
        const auto it = std::lower_bound(E.begin(), E.end(), e);
        const size_t pos = (size_t)(it - E.begin());
        if (pos == (size_t)m) return false;
        if (E[pos] == e && e != kEInf) return false;
        // the worst solution is replaced
        std::move_backward(E.begin() + pos, E.end() - 1, E.end());
        std::move_backward(X.begin() + pos * words, X.end() - words, X.end());
        E[pos] = e;
        std::copy(x, x + words, X.begin() + pos * words);
        return true;
    }
    int finite() const {
        return (int)(std::lower_bound(E.begin(), E.end(), kEInf) - E.begin());
    }
};

struct GaParams {
    uint64_t seed = 1;
    int p_cross = 450, p_mut = 450, mut_max = 1;
};

// New target for (round r, search sid): mutation / crossover / copy,
// parents uniform over the pool (reading C10).  T must hold words(n) words.
static void ga_target(const Pool &P, const GaParams &ga, int64_t r, int64_t sid, uint32_t *T)
{
    const Philox4x32x10 rng(ga.seed);
    const uint32_t c1 = static_cast<uint32_t>(sid), c2 = static_cast<uint32_t>(r);
    const auto head = rng({0u, c1, c2, kTagGA});
    const uint32_t choice = head[0] % 1000u;
    const uint32_t *p1 = &P.X[(size_t)(head[1] % (uint32_t)P.m) * P.words];
    const uint32_t *p2 = &P.X[(size_t)(head[2] % (uint32_t)P.m) * P.words];
    if (choice < (uint32_t)ga.p_cross) {
        // crossover: each bit from either parent
        Philox4x32x10::Block blk{};
        for (int w = 0; w < P.words; ++w) {
            if ((w & 3) == 0) blk = rng({1u + (uint32_t)(w >> 2), c1, c2, kTagGA});
            const uint32_t take2 = blk[w & 3];
            T[w] = (p1[w] & ~take2) | (p2[w] & take2);
        }
    } else if (choice < (uint32_t)(ga.p_cross + ga.p_mut)) {
        // mutation: flip some random bits
        std::copy(p1, p1 + P.words, T);
        const uint32_t flips = 1u + head[3] % (uint32_t)std::max(1, ga.mut_max);
        Philox4x32x10::Block blk{};
        for (uint32_t f = 0; f < flips; ++f) {
            if ((f & 3u) == 0) blk = rng({1u + (f >> 2), c1, c2, kTagGA});
            const uint32_t bit = blk[f & 3u] % (uint32_t)P.n;
            T[bit >> 5] ^= 1u << (bit & 31);
        }
    } else {
        std::copy(p1, p1 + P.words, T);  // copy
    }
}

// Run f(i) for i in [0, count) on up to min(16, cores) host threads; serial below
// `grain` items.  Used for the GA targets of a lockstep step, which only READ the pool
// (each target is a function of the pool, the round and the search id alone).  An
// OpenMP team persists between steps (spawning std::threads every step cost about as
// much as the targets themselves at 10,000 searches).
template <class F>
static void parallel_for(int count, int grain, const F &f)
{
    const int hc = (int)std::max(1u, std::thread::hardware_concurrency());
    const int nth = std::min(std::min(16, hc), std::max(1, count / std::max(1, grain)));
    if (nth <= 1) {
        for (int i = 0; i < count; ++i) f(i);
        return;
    }
#pragma omp parallel for num_threads(nth) schedule(static)
    for (int i = 0; i < count; ++i) f(i);
}

}  // namespace absb

using namespace absb;

struct TraceEntry {
    int32_t s, round;
    std::vector<uint32_t> T, B;
    int64_t EB;
};

struct abs_ctx {
    abs_config cfg{};
    int device = 0;
    cudaStream_t st = nullptr;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr, evs0 = nullptr, evs1 = nullptr;
    // lockstep steps of one-warp searches with more searches than resident CTAs: the
    // first `split` searches run on st while the host builds the others' targets, which
    // then run on st2 (their CTAs fill SMs as the first launch's finish); evj joins st2
    cudaStream_t st2 = nullptr;
    cudaEvent_t evj = nullptr;
    int split = 0;
    Instance I;
    SearchState S;
    int64_t L = 0;
    Pool pool;
    GaParams ga;
    int64_t round = 0;        // lockstep: rounds done (identical on every rank)
    int bytes_per_vec = 0;    // n_pad / 8
    // pinned host staging
    uint8_t *T_h = nullptr, *B_h = nullptr;
    int64_t *EB_h = nullptr;
    bool have_results = false;
    // stats
    double search_seconds = 0.0;
    int64_t rounds_done = 0, pool_inserted = 0, steps = 0;
    int64_t h2d = 0, d2h = 0, launches = 0, round_launches = 0;
    double step_seconds = 0.0;
    // ---- asynchronous mode (the paper's Fig. 5): mapped pinned exchange buffers
    bool async_ready = false;
    uint8_t *Tmap = nullptr;                     // [S][2][bpv] host view
    uint32_t *tseq = nullptr, *rtver = nullptr, *rack = nullptr;
    uint8_t *Rb = nullptr;                       // [S][2][bpv]
    int64_t *Reb = nullptr;                      // [S][2]
    unsigned int *rcount_d = nullptr;          // device: results published (ring index)
    uint32_t *ring = nullptr, *ringseq = nullptr;  // arrival ring [cap][2] / [cap]
    uint32_t ring_mask = 0, ring_head = 0;
    unsigned long long *queue_d = nullptr;
    int *done_d = nullptr;
    std::vector<uint32_t> tver, consumed;        // host-side per-search versions / consumed rounds
    std::vector<std::vector<std::vector<uint32_t>>> hist;  // trace: targets by version
    std::vector<TraceEntry> trace;
    int async_grid = 0;
    long long *timing_d = nullptr;  // diagnostics build
    // ---- tensor-core batched init: W int8 planes (built on first use), A staging
    int8_t *Whi = nullptr;
    uint8_t *Wlo = nullptr;
    uint8_t *Ainit = nullptr;
    size_t Ainit_bytes = 0;
    double init_ms = 0.0;  // last batched-init launch (CUDA events)
};

static void free_ctx(abs_ctx *c)
{
    if (!c) return;
    if (c->device >= 0) cudaSetDevice(c->device);
    if (c->st) cudaStreamSynchronize(c->st);
    cudaFree(c->I.Wz);
    cudaFree(c->I.diag);
    cudaFree(c->I.rowmax);
    cudaFree(c->Whi);
    cudaFree(c->Wlo);
    cudaFree(c->Ainit);
    cudaFree(c->S.g);
    cudaFree(c->S.X);
    cudaFree(c->S.B);
    cudaFree(c->S.T);
    cudaFree(c->S.E);
    cudaFree(c->S.EB);
    cudaFree(c->S.a);
    cudaFree(c->S.l);
    cudaFree(c->S.hash);
    cudaFree(c->S.flips);
    cudaFree(c->S.sflips);
    cudaFree(c->S.tau);
    cudaFree(c->S.sa_ctr);
    if (c->T_h) cudaFreeHost(c->T_h);
    if (c->B_h) cudaFreeHost(c->B_h);
    if (c->EB_h) cudaFreeHost(c->EB_h);
    if (c->Tmap) cudaFreeHost(c->Tmap);
    if (c->tseq) cudaFreeHost(c->tseq);
    if (c->rtver) cudaFreeHost(c->rtver);
    if (c->rack) cudaFreeHost(c->rack);
    if (c->Rb) cudaFreeHost(c->Rb);
    if (c->Reb) cudaFreeHost(c->Reb);
    cudaFree(c->rcount_d);
    if (c->ring) cudaFreeHost(c->ring);
    if (c->ringseq) cudaFreeHost(c->ringseq);
    cudaFree(c->queue_d);
    cudaFree(c->timing_d);
    cudaFree(c->done_d);
    if (c->evj) cudaEventDestroy(c->evj);
    if (c->st2) cudaStreamDestroy(c->st2);
    if (c->ev0) cudaEventDestroy(c->ev0);
    if (c->ev1) cudaEventDestroy(c->ev1);
    if (c->evs0) cudaEventDestroy(c->evs0);
    if (c->evs1) cudaEventDestroy(c->evs1);
    if (c->st) cudaStreamDestroy(c->st);
    delete c;
}

static std::vector<int32_t> default_ladder(int n)
{
    // reading C7: {4, 8, ..., min(256, n/4)}
    const int top = std::min(256, std::max(1, n / 4));
    std::vector<int32_t> lad;
    for (int v = 4; v <= top; v *= 2) lad.push_back(v);
    if (lad.empty()) lad.push_back(std::max(1, top));
    return lad;
}

// bit vectors: ABI words(n) uint32 <-> device bytes [n_pad/8] (little-endian, same bytes)
static void words_to_bytes(const uint32_t *w, int words, uint8_t *dst, int bytes, int n)
{
    std::memset(dst, 0, (size_t)bytes);
    std::memcpy(dst, w, sizeof(uint32_t) * (size_t)words);
    if (n % 32) {
        uint32_t last;
        std::memcpy(&last, dst + 4 * (words - 1), 4);
        last &= (1u << (n % 32)) - 1u;
        std::memcpy(dst + 4 * (words - 1), &last, 4);
    }
}

static int create_common(abs_ctx **out, int32_t n, const int16_t *W, bool W_on_device, const abs_config *cfg_in)
{
    if (!out) return fail(ABS_EINVAL, "out is NULL");
    *out = nullptr;
    if (n < 1 || n > ABS_N_MAX) return fail(ABS_EINVAL, "n must be in [1, 32768]");
    if (!W) return fail(ABS_EINVAL, "W is NULL");
    abs_config cfg;
    abs_config_init(&cfg);
    if (cfg_in) cfg = *cfg_in;
    if (cfg.searches < 0 || cfg.search_offset < 0) return fail(ABS_EINVAL, "bad searches/search_offset");
    if (cfg.local_flips == 0) cfg.local_flips = n;  // reading C8
    if (cfg.local_flips < 0 || cfg.local_flips > INT32_MAX) return fail(ABS_EINVAL, "bad local_flips");
    if (cfg.pool_size == 0) cfg.pool_size = 64;
    if (cfg.pool_size < 1) return fail(ABS_EINVAL, "bad pool_size");
    if (cfg.ladder_len < 0 || cfg.ladder_len > ABS_LADDER_MAX) return fail(ABS_EINVAL, "bad ladder_len");
    if (cfg.p_cross < 0) cfg.p_cross = 450;
    if (cfg.p_mut < 0) cfg.p_mut = 450;
    if (cfg.p_cross + cfg.p_mut > 1000) return fail(ABS_EINVAL, "p_cross + p_mut > 1000");
    if (cfg.mut_max == 0) cfg.mut_max = std::max(1, n / 32);
    if (cfg.mut_max < 0) return fail(ABS_EINVAL, "bad mut_max");
    if (cfg.mode != ABS_MODE_LOCKSTEP && cfg.mode != ABS_MODE_ASYNC) return fail(ABS_EINVAL, "bad mode");
    if (cfg.policy != ABS_POLICY_WINDOW && cfg.policy != ABS_POLICY_SA) return fail(ABS_EINVAL, "bad policy");
    if (cfg.sa_tau_min < 0 || cfg.sa_tau_max < 0 || cfg.sa_levels < 0)
        return fail(ABS_EINVAL, "bad SA temperatures");
    if (cfg.sa_tau_max != 0 && cfg.sa_tau_max < cfg.sa_tau_min) return fail(ABS_EINVAL, "sa_tau_max < sa_tau_min");
    for (int i = 0; i < 3; ++i)
        if (cfg.reserved[i] != 0) return fail(ABS_EINVAL, "reserved config fields must be 0");
    std::vector<int32_t> ladder;
    if (cfg.ladder_len == 0) {
        ladder = default_ladder(n);
    } else {
        for (int i = 0; i < cfg.ladder_len; ++i) {
            if (cfg.ladder[i] < 1) return fail(ABS_EINVAL, "ladder entries must be >= 1");
            ladder.push_back(std::min(cfg.ladder[i], n));
        }
    }
    cfg.ladder_len = (int)ladder.size();
    for (int i = 0; i < cfg.ladder_len; ++i) cfg.ladder[i] = ladder[i];

    int dev = cfg.device;
    if (dev < 0) ABS_CU(cudaGetDevice(&dev));
    ABS_CU(cudaSetDevice(dev));
    cudaDeviceProp prop;
    ABS_CU(cudaGetDeviceProperties(&prop, dev));
    if (prop.major != 10) return fail(ABS_ECUDA, "libabs is built for sm_100a (B200); device is sm_" +
                                                     std::to_string(prop.major) + std::to_string(prop.minor));
    if (cfg.searches == 0) {  // one wave: every SM filled with co-resident searches
        int32_t one_wave = 0;
        ABS_CK(abs_device_searches(n, dev, &one_wave));
        cfg.searches = one_wave;
    }

    abs_ctx *c = new (std::nothrow) abs_ctx();
    if (!c) return fail(ABS_ENOMEM, "host allocation");
    c->cfg = cfg;
    c->device = dev;
    c->L = cfg.local_flips;
    c->ga.seed = cfg.seed;
    c->ga.p_cross = cfg.p_cross;
    c->ga.p_mut = cfg.p_mut;
    c->ga.mut_max = cfg.mut_max;

    auto bail = [&](int rc) {
        free_ctx(c);
        return rc;
    };
#define CTX_CU(expr)                                                                                         \
    do {                                                                                                     \
        cudaError_t e_ = (expr);                                                                             \
        if (e_ != cudaSuccess) return bail(fail(e_ == cudaErrorMemoryAllocation ? ABS_ENOMEM : ABS_ECUDA,    \
                                                std::string(#expr) + ": " + cudaGetErrorString(e_)));        \
    } while (0)

    CTX_CU(cudaStreamCreateWithFlags(&c->st, cudaStreamNonBlocking));
    CTX_CU(cudaStreamCreateWithFlags(&c->st2, cudaStreamNonBlocking));
    CTX_CU(cudaEventCreateWithFlags(&c->evj, cudaEventDisableTiming));
    CTX_CU(cudaEventCreate(&c->ev0));
    CTX_CU(cudaEventCreate(&c->ev1));
    CTX_CU(cudaEventCreate(&c->evs0));
    CTX_CU(cudaEventCreate(&c->evs1));

    // ---- instance layout
    Instance &I = c->I;
    I.n = n;
    layout_for(n, I.n_pad, I.bpt, I.nt);
    c->bytes_per_vec = I.n_pad / 8;
    CTX_CU(cudaMalloc(&I.Wz, (size_t)I.n_pad * I.n_pad * sizeof(int16_t)));
    CTX_CU(cudaMalloc(&I.diag, (size_t)I.n_pad * sizeof(int32_t)));
    CTX_CU(cudaMalloc(&I.rowmax, (size_t)I.n_pad * sizeof(int32_t)));
    {
        int16_t *W_in = nullptr;
        const size_t wbytes = (size_t)n * n * sizeof(int16_t);
        if (W_on_device) {
            W_in = const_cast<int16_t *>(W);
        } else {
            CTX_CU(cudaMalloc(&W_in, wbytes));
            CTX_CU(cudaMemcpyAsync(W_in, W, wbytes, cudaMemcpyHostToDevice, c->st));
            c->h2d += (int64_t)wbytes;
        }
        unsigned long long *asym = nullptr;
        CTX_CU(cudaMalloc(&asym, sizeof(unsigned long long)));
        CTX_CU(cudaMemsetAsync(asym, 0, sizeof(unsigned long long), c->st));
        const int rc = launch_prepare_w(W_in, n, I.n_pad, I.Wz, I.diag, asym, c->st);
        c->launches++;
        unsigned long long bad = 0;
        cudaError_t e2 = cudaMemcpyAsync(&bad, asym, sizeof(bad), cudaMemcpyDeviceToHost, c->st);
        cudaError_t e3 = cudaStreamSynchronize(c->st);
        cudaFree(asym);
        if (!W_on_device) cudaFree(W_in);
        if (rc) return bail(fail(ABS_ECUDA, std::string("prepare_w: ") + cudaGetErrorString((cudaError_t)rc)));
        CTX_CU(e2);
        CTX_CU(e3);
        if (bad) return bail(fail(ABS_EINVAL, "W is not symmetric (" + std::to_string(bad) + " entries)"));
        const int rc2 = launch_rowmax(I, c->st);
        c->launches++;
        if (rc2) return bail(fail(ABS_ECUDA, std::string("rowmax: ") + cudaGetErrorString((cudaError_t)rc2)));
        std::vector<int32_t> rm((size_t)I.n_pad);
        CTX_CU(cudaMemcpyAsync(rm.data(), I.rowmax, sizeof(int32_t) * rm.size(), cudaMemcpyDeviceToHost, c->st));
        CTX_CU(cudaStreamSynchronize(c->st));
        I.wmax = 0;
        for (int32_t v : rm) I.wmax = std::max(I.wmax, v);
    }
    // SA temperatures (reading E2): defaults from the instance's weight scale
    if (c->cfg.sa_tau_min == 0) c->cfg.sa_tau_min = std::max(1, I.wmax);
    if (c->cfg.sa_tau_max == 0) c->cfg.sa_tau_max = c->cfg.sa_tau_min;
    if (c->cfg.sa_levels == 0) c->cfg.sa_levels = 1;

    // ---- per-search state
    SearchState &S = c->S;
    S.S = cfg.searches;
    const size_t Sn = (size_t)std::max(1, S.S);
    CTX_CU(cudaMalloc(&S.g, Sn * (size_t)I.n_pad * sizeof(int32_t)));
    CTX_CU(cudaMalloc(&S.X, Sn * c->bytes_per_vec));
    CTX_CU(cudaMalloc(&S.B, Sn * c->bytes_per_vec));
    CTX_CU(cudaMalloc(&S.T, Sn * c->bytes_per_vec));
    CTX_CU(cudaMalloc(&S.E, Sn * sizeof(int64_t)));
    CTX_CU(cudaMalloc(&S.EB, Sn * sizeof(int64_t)));
    CTX_CU(cudaMalloc(&S.a, Sn * sizeof(int32_t)));
    CTX_CU(cudaMalloc(&S.l, Sn * sizeof(int32_t)));
    CTX_CU(cudaMalloc(&S.hash, Sn * sizeof(uint64_t)));
    CTX_CU(cudaMalloc(&S.flips, Sn * sizeof(int64_t)));
    CTX_CU(cudaMalloc(&S.sflips, Sn * sizeof(int64_t)));
    CTX_CU(cudaMalloc(&S.tau, Sn * sizeof(int32_t)));
    CTX_CU(cudaMalloc(&S.sa_ctr, Sn * sizeof(uint64_t)));
    CTX_CU(cudaMemsetAsync(S.sa_ctr, 0, Sn * sizeof(uint64_t), c->st));
    {
        // search s (global id g) at temperature level j = g mod K (reading E2)
        const int32_t K = c->cfg.sa_levels, tmin = c->cfg.sa_tau_min, tmax = c->cfg.sa_tau_max;
        std::vector<int32_t> tv(Sn);
        for (size_t s = 0; s < Sn; ++s) {
            const int64_t j = (int64_t)(cfg.search_offset + s) % K;
            tv[s] = K == 1 ? tmin : (int32_t)(tmin + ((int64_t)(tmax - tmin) * j) / (K - 1));
        }
        CTX_CU(cudaMemcpyAsync(S.tau, tv.data(), Sn * sizeof(int32_t), cudaMemcpyHostToDevice, c->st));
        CTX_CU(cudaStreamSynchronize(c->st));
        c->h2d += (int64_t)(Sn * sizeof(int32_t));
    }
    {
        std::vector<int32_t> lv(Sn);
        for (size_t s = 0; s < Sn; ++s) lv[s] = ladder[(size_t)(cfg.search_offset + s) % ladder.size()];
        CTX_CU(cudaMemcpyAsync(S.l, lv.data(), Sn * sizeof(int32_t), cudaMemcpyHostToDevice, c->st));
        c->h2d += (int64_t)(Sn * sizeof(int32_t));
    }
    {
        const int rc = launch_zero_start(I, S, 0, S.S, c->st);  // device Step 1
        c->launches++;
        if (rc) return bail(fail(ABS_ECUDA, std::string("zero_start: ") + cudaGetErrorString((cudaError_t)rc)));
    }
    CTX_CU(cudaMemsetAsync(S.T, 0, Sn * c->bytes_per_vec, c->st));
    CTX_CU(cudaMallocHost(&c->T_h, Sn * c->bytes_per_vec));
    if (I.nt == 32) {  // one-warp searches: split a lockstep step beyond the resident CTAs (lockstep_step)
        int per_sm = 0, sms = 0;
        CTX_CU((cudaError_t)round_occupancy(I.nt, I.bpt, &per_sm));
        CTX_CU(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c->device));
        const int resident = per_sm * sms;
        c->split = (resident > 0 && S.S > resident) ? resident : 0;
    }
    CTX_CU(cudaMallocHost(&c->B_h, Sn * c->bytes_per_vec));
    CTX_CU(cudaMallocHost(&c->EB_h, Sn * sizeof(int64_t)));
    std::memset(c->T_h, 0, Sn * c->bytes_per_vec);
    CTX_CU(cudaStreamSynchronize(c->st));

    // ---- host GA pool (host Step 1)
    c->pool.init(n, cfg.pool_size);
    c->pool.randomize(cfg.seed);
#undef CTX_CU
    *out = c;
    return ABS_OK;
}

// One lockstep step: targets, one round per search, inserts.
static int lockstep_step(abs_ctx *c)
{
    const int S = c->S.S, words = c->pool.words, bpv = c->bytes_per_vec;
    // host Step 4: "generates ... new target solutions by GA"; the targets are
    // independent given the pool, so large batches are built on several host threads
    std::vector<uint32_t> T(words);
    // targets of searches [s0, s1) into T_h, then to the device on stream st
    auto targets = [&](int s0, int s1, cudaStream_t st) -> int {
        parallel_for(s1 - s0, 512, [&](int i) {  // T_h rows: bpv = n_pad / 8 bytes, 4-byte aligned
            const int s = s0 + i;
            ga_target(c->pool, c->ga, c->round, (int64_t)c->cfg.search_offset + s,
                      reinterpret_cast<uint32_t *>(c->T_h + (size_t)s * bpv));
        });
        ABS_CU(cudaMemcpyAsync(c->S.T + (size_t)s0 * bpv, c->T_h + (size_t)s0 * bpv, (size_t)(s1 - s0) * bpv,
                               cudaMemcpyHostToDevice, st));
        c->h2d += (int64_t)(s1 - s0) * bpv;
        return ABS_OK;
    };
    // one launch, or (c->split) the first `split` searches launched while the host builds the
    // other targets: the same round for every search, the results inserted after both
    const int s_first = c->split > 0 ? c->split : S;
    if (const int rc = targets(0, s_first, c->st)) return rc;
    RoundArgs a{};
    a.Wz = c->I.Wz;
    a.wmax = c->I.wmax;
    a.n = c->I.n;
    a.n_pad = c->I.n_pad;
    a.nt = c->I.nt;
    a.bpt = c->I.bpt;
    a.g = c->S.g;
    a.X = c->S.X;
    a.T = c->S.T;
    a.B = c->S.B;
    a.E = c->S.E;
    a.EB = c->S.EB;
    a.a = c->S.a;
    a.l = c->S.l;
    a.hash = c->S.hash;
    a.flips = c->S.flips;
    a.sflips = c->S.sflips;
    a.L = c->L;
    a.S = S;
    a.policy = c->cfg.policy;
    a.sid0 = c->cfg.search_offset;
    a.seed = c->cfg.seed;
    a.tau = c->S.tau;
    a.sa_ctr = c->S.sa_ctr;
#ifdef ABS_TIMING
    if (!c->timing_d) {
        ABS_CU(cudaMalloc(&c->timing_d, (size_t)S * 32 * 24 * sizeof(long long)));
        ABS_CU(cudaMemset(c->timing_d, 0, (size_t)S * 32 * 24 * sizeof(long long)));
    }
    a.timing = c->timing_d;
#endif
    ABS_CU(cudaEventRecord(c->ev0, c->st));
    a.S = s_first;
    a.sbase = 0;
    ABS_CK(launch_round(a, c->st));
    c->launches++;
    c->round_launches++;
    if (s_first < S) {
        if (const int rc = targets(s_first, S, c->st2)) return rc;  // overlaps the first launch
        a.S = S - s_first;
        a.sbase = s_first;
        ABS_CK(launch_round(a, c->st2));
        c->launches++;
        c->round_launches++;
        ABS_CU(cudaEventRecord(c->evj, c->st2));
        ABS_CU(cudaStreamWaitEvent(c->st, c->evj, 0));
    }
    ABS_CU(cudaEventRecord(c->ev1, c->st));
    ABS_CU(cudaMemcpyAsync(c->B_h, c->S.B, (size_t)S * bpv, cudaMemcpyDeviceToHost, c->st));
    ABS_CU(cudaMemcpyAsync(c->EB_h, c->S.EB, (size_t)S * sizeof(int64_t), cudaMemcpyDeviceToHost, c->st));
    c->d2h += (int64_t)S * (bpv + 8);
    ABS_CU(cudaStreamSynchronize(c->st));
    float ms = 0.f;
    ABS_CU(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
    c->search_seconds += ms * 1e-3;
    c->have_results = true;
    c->rounds_done += S;
    if (!c->cfg.external_merge) {
        // host Step 3: insert the new solutions (ascending search id); a result not better
        // than the worst pool entry is rejected by the rule, checked first (most results)
        for (int s = 0; s < S; ++s) {
            if (c->EB_h[s] >= c->pool.E.back() && c->pool.E.back() != kEInf) continue;
            std::memcpy(T.data(), c->B_h + (size_t)s * bpv, sizeof(uint32_t) * words);
            c->pool_inserted += c->pool.insert(T.data(), c->EB_h[s]) ? 1 : 0;
        }
    }
    c->round += 1;
    c->steps += 1;
    return ABS_OK;
}

// ------------------------------------------------------------------ asynchronous mode
template <typename T>
static T vload(const T *p)
{
    return *reinterpret_cast<const volatile T *>(p);
}
template <typename T>
static void vstore(T *p, T v)
{
    *reinterpret_cast<volatile T *>(p) = v;
}

static int async_setup(abs_ctx *c)
{
    const int S = c->S.S, bpv = c->bytes_per_vec;
    const unsigned fl = cudaHostAllocMapped | cudaHostAllocPortable;
    ABS_CU(cudaHostAlloc(&c->Tmap, (size_t)S * 2 * bpv, fl));
    ABS_CU(cudaHostAlloc(&c->Rb, (size_t)S * 2 * bpv, fl));
    ABS_CU(cudaHostAlloc(&c->Reb, (size_t)S * 2 * sizeof(int64_t), fl));
    ABS_CU(cudaHostAlloc(&c->tseq, (size_t)S * sizeof(uint32_t), fl));
    ABS_CU(cudaHostAlloc(&c->rtver, (size_t)S * 2 * sizeof(uint32_t), fl));
    ABS_CU(cudaHostAlloc(&c->rack, (size_t)S * sizeof(uint32_t), fl));
    std::memset(c->Tmap, 0, (size_t)S * 2 * bpv);
    std::memset(c->Rb, 0, (size_t)S * 2 * bpv);
    std::memset(c->tseq, 0, (size_t)S * sizeof(uint32_t));
    std::memset(c->rack, 0, (size_t)S * sizeof(uint32_t));
    ABS_CU(cudaMalloc(&c->rcount_d, sizeof(unsigned int)));
    ABS_CU(cudaMemset(c->rcount_d, 0, sizeof(unsigned int)));
    uint32_t cap = 64;
    while (cap < 2u * (uint32_t)S) cap <<= 1;
    ABS_CU(cudaHostAlloc(&c->ring, (size_t)cap * 2 * sizeof(uint32_t), fl));
    ABS_CU(cudaHostAlloc(&c->ringseq, (size_t)cap * sizeof(uint32_t), fl));
    std::memset(c->ringseq, 0, (size_t)cap * sizeof(uint32_t));
    c->ring_mask = cap - 1;
    c->ring_head = 0;
    ABS_CU(cudaMalloc(&c->queue_d, sizeof(unsigned long long)));
    ABS_CU(cudaMalloc(&c->done_d, (size_t)S * sizeof(int)));
    ABS_CU(cudaMemset(c->done_d, 0, (size_t)S * sizeof(int)));
    c->tver.assign(S, 0);
    c->consumed.assign(S, 0);
    if (c->cfg.trace) c->hist.assign(S, {});
    // round-0 targets from the initial pool (host Step 1 + Step 4)
    std::vector<uint32_t> T(c->pool.words);
    for (int s = 0; s < S; ++s) {
        ga_target(c->pool, c->ga, c->round, (int64_t)c->cfg.search_offset + s, T.data());
        std::memcpy(c->Tmap + ((size_t)s * 2 + 1) * bpv, T.data(), sizeof(uint32_t) * T.size());
        c->tver[s] = 1;
        if (c->cfg.trace) c->hist[s].assign(2, {}), c->hist[s][1] = T;
    }
    std::atomic_thread_fence(std::memory_order_release);
    for (int s = 0; s < S; ++s) vstore(c->tseq + s, 1u);
    c->async_ready = true;
    return ABS_OK;
}

// Host Steps 2-4 for every result published so far, in arrival
// order (the ring): insert it into the pool, acknowledge the slot, generate one
// new target for the search.  Cost O(results), independent of S.
static void async_consume(abs_ctx *c)
{
    const int bpv = c->bytes_per_vec, words = c->pool.words;
    std::vector<uint32_t> B(words), T(words);
    constexpr uint32_t kBatch = 256;
    uint32_t es[kBatch], er[kBatch];
    for (;;) {
        // collect the arrived entries (sequential reads), then prefetch their result
        // slots: the slots were written by the GPU, so every first touch is a miss
        const uint32_t h0 = c->ring_head;
        uint32_t nb = 0;
        while (nb < kBatch && vload(c->ringseq + ((h0 + nb) & c->ring_mask)) == h0 + nb + 1u) ++nb;
        if (nb == 0) break;
        std::atomic_thread_fence(std::memory_order_acquire);
        for (uint32_t e = 0; e < nb; ++e) {
            const uint32_t h = (h0 + e) & c->ring_mask;
            es[e] = vload(c->ring + 2 * h);
            er[e] = vload(c->ring + 2 * h + 1);
            const size_t slot = (size_t)es[e] * 2 + (er[e] & 1);
            for (int off = 0; off < bpv; off += 64) __builtin_prefetch(c->Rb + slot * bpv + off);
            __builtin_prefetch(c->Reb + slot);
            __builtin_prefetch(c->rtver + slot);
        }
        c->ring_head = h0 + nb;
        for (uint32_t e = 0; e < nb; ++e) {
            const int s = (int)es[e];
            const uint32_t r = er[e];
            const size_t slot = (size_t)s * 2 + (r & 1);
            const int64_t EB = vload(c->Reb + slot);
            const uint32_t v = vload(c->rtver + slot);
            // Step 3; a result not better than the worst pool entry is rejected by the rule
            const bool cand = EB < c->pool.E.back() || c->pool.E.back() == kEInf;
            if (cand || c->cfg.trace) std::memcpy(B.data(), c->Rb + slot * bpv, sizeof(uint32_t) * words);
            if (cand) c->pool_inserted += c->pool.insert(B.data(), EB) ? 1 : 0;
            if (c->cfg.trace) c->trace.push_back(TraceEntry{s, (int32_t)r, c->hist[s][v], B, EB});
            c->consumed[s] = r + 1;
            std::atomic_thread_fence(std::memory_order_release);
            vstore(c->rack + s, r + 1);
            // Step 4: "as many new target solutions as newly arrived solutions"
            ga_target(c->pool, c->ga, (int64_t)r + 1, (int64_t)c->cfg.search_offset + s, T.data());
            const uint32_t nv = c->tver[s] + 1;
            std::memcpy(c->Tmap + ((size_t)s * 2 + (nv & 1)) * bpv, T.data(), sizeof(uint32_t) * words);
            if (c->cfg.trace) c->hist[s].push_back(T);
            std::atomic_thread_fence(std::memory_order_release);
            vstore(c->tseq + s, nv);
            c->tver[s] = nv;
        }
    }
}

static int async_run(abs_ctx *c, int64_t steps)
{
    if (!c->async_ready) {
        const int rc = async_setup(c);
        if (rc) return rc;
    }
    const int S = c->S.S;
    if ((int64_t)c->round + steps > INT32_MAX) return fail(ABS_EINVAL, "too many rounds");
    ABS_CU(cudaMemsetAsync(c->queue_d, 0, sizeof(unsigned long long), c->st));
    AsyncArgs q{};
    auto dev = [](auto *h) {
        void *d = nullptr;
        cudaHostGetDevicePointer(&d, (void *)h, 0);
        return d;
    };
    q.queue = c->queue_d;
    q.total = (long long)S * steps;
    q.base = (int)c->round;
    q.done = c->done_d;
    q.Tmap = (const uint8_t *)dev(c->Tmap);
    q.tseq = (const uint32_t *)dev(c->tseq);
    q.Rb = (uint8_t *)dev(c->Rb);
    q.Reb = (int64_t *)dev(c->Reb);
    q.rtver = (uint32_t *)dev(c->rtver);
    q.rack = (const uint32_t *)dev(c->rack);
    q.rcount = c->rcount_d;
    q.ring = (uint32_t *)dev(c->ring);
    q.ringseq = (uint32_t *)dev(c->ringseq);
    q.ring_mask = c->ring_mask;
    RoundArgs a{};
    a.Wz = c->I.Wz;
    a.wmax = c->I.wmax;
    a.n = c->I.n;
    a.n_pad = c->I.n_pad;
    a.nt = c->I.nt;
    a.bpt = c->I.bpt;
    a.g = c->S.g;
    a.X = c->S.X;
    a.T = nullptr;
    a.B = c->S.B;
    a.E = c->S.E;
    a.EB = c->S.EB;
    a.a = c->S.a;
    a.l = c->S.l;
    a.hash = c->S.hash;
    a.flips = c->S.flips;
    a.sflips = c->S.sflips;
    a.L = c->L;
    a.S = S;
    a.policy = c->cfg.policy;
    a.sid0 = c->cfg.search_offset;
    a.seed = c->cfg.seed;
    a.tau = c->S.tau;
    a.sa_ctr = c->S.sa_ctr;
#ifdef ABS_TIMING
    if (!c->timing_d) {
        ABS_CU(cudaMalloc(&c->timing_d, (size_t)S * 32 * 24 * sizeof(long long)));
        ABS_CU(cudaMemset(c->timing_d, 0, (size_t)S * 32 * 24 * sizeof(long long)));
    }
    a.timing = c->timing_d;
#endif

    // the host GA thread, concurrent with the persistent kernel
    std::atomic<bool> stop{false};
    std::thread ga([c, &stop]() {
        for (;;) {
            const bool last = stop.load(std::memory_order_acquire);
            // Step 2: poll for newly arrived solutions
            const bool ready = vload(c->ringseq + (c->ring_head & c->ring_mask)) == c->ring_head + 1u;
            if (ready || last) {
                async_consume(c);
                if (last) break;
            } else {
                std::this_thread::sleep_for(std::chrono::microseconds(20));
            }
        }
    });
    ABS_CU(cudaEventRecord(c->ev0, c->st));
    const int rc = launch_round(a, c->st, &q, &c->async_grid);
    c->launches++;
    c->round_launches++;
    cudaError_t e1 = cudaEventRecord(c->ev1, c->st);
    cudaError_t e2 = cudaStreamSynchronize(c->st);
    stop.store(true, std::memory_order_release);
    ga.join();  // drains every published result
    if (rc) return fail(ABS_ECUDA, std::string("round_kernel_async: ") + cudaGetErrorString((cudaError_t)rc));
    ABS_CU(e1);
    ABS_CU(e2);
    float ms = 0.f;
    ABS_CU(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
    c->search_seconds += ms * 1e-3;
    c->rounds_done += (int64_t)S * steps;
    c->round += steps;
    c->steps += steps;
    return ABS_OK;
}

extern "C" {

void abs_config_init(abs_config *cfg)
{
    if (!cfg) return;
    std::memset(cfg, 0, sizeof(*cfg));
    cfg->seed = 1;
    cfg->p_cross = -1;
    cfg->p_mut = -1;
    cfg->mode = ABS_MODE_LOCKSTEP;
    cfg->device = -1;
}

int abs_create(abs_ctx **out, int32_t n, const int16_t *W, const abs_config *cfg)
{
    try {
        return create_common(out, n, W, false, cfg);
    } catch (const std::bad_alloc &) {
        return fail(ABS_ENOMEM, "host allocation");
    } catch (...) {
        return fail(ABS_EINVAL, "unexpected exception");
    }
}

int abs_create_dev(abs_ctx **out, int32_t n, const int16_t *W_dev, const abs_config *cfg)
{
    try {
        return create_common(out, n, W_dev, true, cfg);
    } catch (const std::bad_alloc &) {
        return fail(ABS_ENOMEM, "host allocation");
    } catch (...) {
        return fail(ABS_EINVAL, "unexpected exception");
    }
}

// Batched init on device buffers: X_dev packed words, row
// stride words(n); E_dev count int64; delta_dev count*n int32 or NULL.
static int energy_device(abs_ctx *c, const uint32_t *X_dev, int32_t count, int64_t *E_dev, int32_t *delta_dev,
                         int32_t engine)
{
    const int row_bytes = 4 * words_of(c->I.n);
    const uint8_t *X = reinterpret_cast<const uint8_t *>(X_dev);
    if (engine == ABS_INIT_ALU) {
        ABS_CU(cudaEventRecord(c->ev0, c->st));
        ABS_CK(launch_batch_init(c->I, X, row_bytes, count, E_dev, delta_dev, c->st));
        ABS_CU(cudaEventRecord(c->ev1, c->st));
        c->launches += 1;
    } else {
        if (!c->Whi) {  // int8 planes of W, once per instance
            const size_t pb = init_mma_plane_bytes(c->I.n_pad);
            if (cudaMalloc(&c->Whi, pb) != cudaSuccess) return fail(ABS_ENOMEM, "W hi plane");
            if (cudaMalloc(&c->Wlo, pb) != cudaSuccess) return fail(ABS_ENOMEM, "W lo plane");
            ABS_CK(launch_wsplit(c->I, c->Whi, c->Wlo, c->st));
            c->launches += 1;
        }
        const size_t ab = init_mma_a_bytes(count, c->I.n_pad);
        if (ab > c->Ainit_bytes) {
            cudaFree(c->Ainit);
            c->Ainit = nullptr;
            c->Ainit_bytes = 0;
            if (cudaMalloc(&c->Ainit, ab) != cudaSuccess) return fail(ABS_ENOMEM, "init A staging");
            c->Ainit_bytes = ab;
        }
        ABS_CU(cudaEventRecord(c->ev0, c->st));
        ABS_CK(launch_init_mma(c->I, c->Whi, c->Wlo, X, row_bytes, count, c->Ainit, E_dev, delta_dev, c->st));
        ABS_CU(cudaEventRecord(c->ev1, c->st));
        c->launches += 2;
    }
    return ABS_OK;
}

int abs_energy_dev(abs_ctx *c, const uint32_t *X_dev, int32_t count, int64_t *E_dev, int32_t *delta_dev,
                   int32_t engine)
{
    if (!c || count < 0 || (count > 0 && (!X_dev || !E_dev))) return fail(ABS_EINVAL, "bad arguments");
    if (engine != ABS_INIT_AUTO && engine != ABS_INIT_ALU && engine != ABS_INIT_MMA)
        return fail(ABS_EINVAL, "unknown engine");
    if (count == 0) return ABS_OK;
    ABS_CU(cudaSetDevice(c->device));
    const int rc = energy_device(c, X_dev, count, E_dev, delta_dev, engine);
    if (rc) return rc;
    ABS_CU(cudaStreamSynchronize(c->st));
    float ms = 0.f;
    ABS_CU(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
    c->init_ms = ms;
    return ABS_OK;
}

int abs_energy(abs_ctx *c, const uint32_t *X, int32_t count, int64_t *E_out, int32_t *delta_out)
{
    if (!c || (count > 0 && (!X || !E_out)) || count < 0) return fail(ABS_EINVAL, "bad arguments");
    if (count == 0) return ABS_OK;
    ABS_CU(cudaSetDevice(c->device));
    const int n = c->I.n, words = words_of(n);
    uint32_t *X_d = nullptr;
    int64_t *E_d = nullptr;
    int32_t *D_d = nullptr;
    auto cleanup = [&]() {
        cudaFree(X_d);
        cudaFree(E_d);
        cudaFree(D_d);
    };
    const size_t xbytes = sizeof(uint32_t) * (size_t)count * words;
    cudaError_t e = cudaMalloc(&X_d, xbytes);
    if (e == cudaSuccess) e = cudaMalloc(&E_d, sizeof(int64_t) * (size_t)count);
    if (e == cudaSuccess && delta_out) e = cudaMalloc(&D_d, sizeof(int32_t) * (size_t)count * n);
    if (e != cudaSuccess) {
        cleanup();
        return fail(ABS_ENOMEM, std::string("abs_energy: ") + cudaGetErrorString(e));
    }
    e = cudaMemcpyAsync(X_d, X, xbytes, cudaMemcpyHostToDevice, c->st);
    int rc = (e == cudaSuccess) ? energy_device(c, X_d, count, E_d, D_d, ABS_INIT_AUTO) : ABS_ECUDA;
    if (rc == ABS_OK) {
        e = cudaMemcpyAsync(E_out, E_d, sizeof(int64_t) * (size_t)count, cudaMemcpyDeviceToHost, c->st);
        if (e == cudaSuccess && delta_out)
            e = cudaMemcpyAsync(delta_out, D_d, sizeof(int32_t) * (size_t)count * n, cudaMemcpyDeviceToHost, c->st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(c->st);
        if (e != cudaSuccess) rc = fail(ABS_ECUDA, std::string("abs_energy: ") + cudaGetErrorString(e));
    }
    cleanup();
    c->h2d += (int64_t)xbytes;
    c->d2h += (int64_t)count * 8 + (delta_out ? (int64_t)count * n * 4 : 0);
    return rc;
}

int abs_seed_pool(abs_ctx *c, const uint32_t *X, int32_t count)
{
    if (!c) return fail(ABS_EINVAL, "ctx is NULL");
    if (!X) {
        c->pool.randomize(c->cfg.seed);
        return ABS_OK;
    }
    if (count < 0) return fail(ABS_EINVAL, "count < 0");
    std::vector<int64_t> E((size_t)count);
    // energies on the device: "a host never computes the energy function"
    const int rc = abs_energy(c, X, count, E.data(), nullptr);
    if (rc) return rc;
    const int words = c->pool.words;
    std::vector<uint32_t> x(words);
    for (int b = 0; b < count; ++b) {
        std::memcpy(x.data(), X + (size_t)b * words, sizeof(uint32_t) * words);
        if (c->I.n % 32) x[words - 1] &= (1u << (c->I.n % 32)) - 1u;
        c->pool_inserted += c->pool.insert(x.data(), E[b]) ? 1 : 0;
    }
    return ABS_OK;
}

int abs_search(abs_ctx *c, int64_t steps)
{
    if (!c || steps < 0) return fail(ABS_EINVAL, "bad arguments");
    if (c->S.S == 0 || steps == 0) return ABS_OK;
    try {
        ABS_CU(cudaSetDevice(c->device));
        ABS_CU(cudaEventRecord(c->evs0, c->st));
        if (c->cfg.mode == ABS_MODE_ASYNC) {
            const int rc = async_run(c, steps);
            if (rc) return rc;
        } else {
            for (int64_t s = 0; s < steps; ++s) {
                const int rc = lockstep_step(c);
                if (rc) return rc;
            }
        }
        ABS_CU(cudaEventRecord(c->evs1, c->st));
        ABS_CU(cudaEventSynchronize(c->evs1));
        float ms = 0.f;
        ABS_CU(cudaEventElapsedTime(&ms, c->evs0, c->evs1));
        c->step_seconds += ms * 1e-3;
        return ABS_OK;
    } catch (const std::bad_alloc &) {
        return fail(ABS_ENOMEM, "host allocation");
    }
}

int abs_best(const abs_ctx *c, uint32_t *X_out, int64_t *E_out)
{
    if (!c || !X_out || !E_out) return fail(ABS_EINVAL, "bad arguments");
    if (c->pool.finite() == 0) return fail(ABS_EEMPTY, "no finite energy in the pool");
    std::memcpy(X_out, c->pool.X.data(), sizeof(uint32_t) * c->pool.words);
    *E_out = c->pool.E[0];
    return ABS_OK;
}

int abs_stats_get(const abs_ctx *c, abs_stats *s)
{
    if (!c || !s) return fail(ABS_EINVAL, "bad arguments");
    std::memset(s, 0, sizeof(*s));
    const int S = c->S.S;
    if (S > 0) {
        ABS_CU(cudaSetDevice(c->device));
        std::vector<int64_t> f(S), sf(S);
        ABS_CU(cudaMemcpy(f.data(), c->S.flips, sizeof(int64_t) * S, cudaMemcpyDeviceToHost));
        ABS_CU(cudaMemcpy(sf.data(), c->S.sflips, sizeof(int64_t) * S, cudaMemcpyDeviceToHost));
        for (int i = 0; i < S; ++i) {
            s->flips += f[i];
            s->straight_flips += sf[i];
        }
    }
    s->evaluated = s->flips * (int64_t)c->I.n;
    s->rounds = c->rounds_done;
    s->search_seconds = c->search_seconds;
    s->pool_inserted = c->pool_inserted;
    s->n = c->I.n;
    s->n_pad = c->I.n_pad;
    s->searches = S;
    s->threads_per_search = c->I.nt;
    s->steps = c->steps;
    s->h2d_bytes = c->h2d;
    s->d2h_bytes = c->d2h;
    s->kernel_launches = c->launches;
    s->step_seconds = c->step_seconds;
    s->round_kernel_launches = c->round_launches;
    s->init_seconds = c->init_ms * 1e-3;
    return ABS_OK;
}

int abs_pool_get(const abs_ctx *c, int32_t k, uint32_t *X_out, int64_t *E_out, int32_t *count_out)
{
    if (!c || k < 0 || (k > 0 && (!X_out || !E_out))) return fail(ABS_EINVAL, "bad arguments");
    const int cnt = std::min(k, c->pool.finite());
    std::memcpy(X_out, c->pool.X.data(), sizeof(uint32_t) * (size_t)cnt * c->pool.words);
    std::memcpy(E_out, c->pool.E.data(), sizeof(int64_t) * (size_t)cnt);
    if (count_out) *count_out = cnt;
    return ABS_OK;
}

int abs_pool_insert(abs_ctx *c, const uint32_t *X, const int64_t *E, int32_t count, int32_t *inserted_out)
{
    if (!c || count < 0 || (count > 0 && (!X || !E))) return fail(ABS_EINVAL, "bad arguments");
    const int words = c->pool.words;
    std::vector<uint32_t> x(words);
    int ins = 0;
    for (int b = 0; b < count; ++b) {
        std::memcpy(x.data(), X + (size_t)b * words, sizeof(uint32_t) * words);
        if (c->I.n % 32) x[words - 1] &= (1u << (c->I.n % 32)) - 1u;
        ins += c->pool.insert(x.data(), E[b]) ? 1 : 0;
    }
    c->pool_inserted += ins;
    if (inserted_out) *inserted_out = ins;
    return ABS_OK;
}

int abs_round_results(const abs_ctx *c, uint32_t *B_out, int64_t *EB_out)
{
    if (!c || !B_out || !EB_out) return fail(ABS_EINVAL, "bad arguments");
    if (!c->have_results || c->cfg.mode != ABS_MODE_LOCKSTEP) return fail(ABS_ESTATE, "no lockstep round has run");
    const int words = c->pool.words;
    for (int s = 0; s < c->S.S; ++s) {
        std::memcpy(B_out + (size_t)s * words, c->B_h + (size_t)s * c->bytes_per_vec, sizeof(uint32_t) * words);
        EB_out[s] = c->EB_h[s];
    }
    return ABS_OK;
}

int abs_round_targets(const abs_ctx *c, uint32_t *T_out)
{
    if (!c || !T_out) return fail(ABS_EINVAL, "bad arguments");
    if (!c->have_results) return fail(ABS_ESTATE, "no round has run");
    const int words = c->pool.words;
    for (int s = 0; s < c->S.S; ++s)
        std::memcpy(T_out + (size_t)s * words, c->T_h + (size_t)s * c->bytes_per_vec, sizeof(uint32_t) * words);
    return ABS_OK;
}

int abs_debug_timing(const abs_ctx *c, long long *out)
{
#ifdef ABS_TIMING
    if (!c || !out || !c->timing_d) return fail(ABS_ESTATE, "no timing data");
    ABS_CU(cudaMemcpy(out, c->timing_d, (size_t)c->S.S * 32 * 24 * sizeof(long long), cudaMemcpyDeviceToHost));
    return ABS_OK;
#else
    (void)c;
    (void)out;
    return fail(ABS_EINVAL, "built without ABS_TIMING");
#endif
}

int abs_trace_count(const abs_ctx *c, int64_t *count)
{
    if (!c || !count) return fail(ABS_EINVAL, "bad arguments");
    *count = (int64_t)c->trace.size();
    return ABS_OK;
}

int abs_trace_get(const abs_ctx *c, int64_t i, int32_t *s_out, int32_t *round_out, uint32_t *T_out, uint32_t *B_out,
                  int64_t *EB_out)
{
    if (!c || i < 0 || i >= (int64_t)c->trace.size()) return fail(ABS_EINVAL, "bad arguments");
    const TraceEntry &e = c->trace[(size_t)i];
    if (s_out) *s_out = e.s;
    if (round_out) *round_out = e.round;
    if (T_out) std::copy(e.T.begin(), e.T.end(), T_out);
    if (B_out) std::copy(e.B.begin(), e.B.end(), B_out);
    if (EB_out) *EB_out = e.EB;
    return ABS_OK;
}

int abs_search_state(const abs_ctx *c, int32_t s, uint32_t *X_out, int32_t *delta_out, int64_t *E_out,
                     int32_t *a_out, int32_t *l_out, uint64_t *hash_out, int64_t *flips_out)
{
    if (!c || s < 0 || s >= c->S.S) return fail(ABS_EINVAL, "bad arguments");
    ABS_CU(cudaSetDevice(c->device));
    const int n = c->I.n, nt = c->I.nt, bpv = c->bytes_per_vec, words = words_of(n);
    std::vector<uint8_t> xb(bpv);
    ABS_CU(cudaMemcpy(xb.data(), c->S.X + (size_t)s * bpv, bpv, cudaMemcpyDeviceToHost));
    if (X_out) std::memcpy(X_out, xb.data(), sizeof(uint32_t) * words);
    if (delta_out) {
        std::vector<int32_t> g((size_t)c->I.n_pad);
        ABS_CU(cudaMemcpy(g.data(), c->S.g + (size_t)s * c->I.n_pad, sizeof(int32_t) * g.size(),
                          cudaMemcpyDeviceToHost));
        for (int i = 0; i < n; ++i) {
            const int beta = i >> 3, t = beta % nt, slot = 8 * (beta / nt) + (i & 7);
            const int gi = g[(size_t)slot * nt + t];
            const int xi = (xb[i >> 3] >> (i & 7)) & 1;
            delta_out[i] = xi ? -gi : gi;  // Delta_i = phi(x_i) g_i (Eq.(13))
        }
    }
    int64_t v64;
    int32_t v32;
    uint64_t u64;
    if (E_out) { ABS_CU(cudaMemcpy(&v64, c->S.E + s, 8, cudaMemcpyDeviceToHost)); *E_out = v64; }
    if (a_out) { ABS_CU(cudaMemcpy(&v32, c->S.a + s, 4, cudaMemcpyDeviceToHost)); *a_out = v32; }
    if (l_out) { ABS_CU(cudaMemcpy(&v32, c->S.l + s, 4, cudaMemcpyDeviceToHost)); *l_out = v32; }
    if (hash_out) { ABS_CU(cudaMemcpy(&u64, c->S.hash + s, 8, cudaMemcpyDeviceToHost)); *hash_out = u64; }
    if (flips_out) { ABS_CU(cudaMemcpy(&v64, c->S.flips + s, 8, cudaMemcpyDeviceToHost)); *flips_out = v64; }
    return ABS_OK;
}

void abs_destroy(abs_ctx *c) { free_ctx(c); }

const char *abs_strerror(int rc)
{
    switch (rc) {
    case ABS_OK: return "ok";
    case ABS_EINVAL: return "invalid argument";
    case ABS_ENOMEM: return "out of memory";
    case ABS_ECUDA: return "CUDA error";
    case ABS_ENCCL: return "NCCL error (multi-GPU exchange)";
    case ABS_ESTATE: return "invalid state";
    case ABS_EEMPTY: return "pool has no finite-energy solution";
    case ABS_ERANGE: return "delta out of int32 range";
    default: return "unknown error";
    }
}

const char *abs_last_error(void) { return g_last_error.c_str(); }

int abs_ising_to_qubo(int32_t n, const int32_t *J, const int32_t *h, int16_t *W_out, int64_t *offset_out)
{
    if (n < 1 || !J || !h || !W_out || !offset_out) return fail(ABS_EINVAL, "abs_ising_to_qubo: bad arguments");
    // s_i = 2 x_i - 1: -J s_i s_j = -4J x_i x_j + 2J (x_i + x_j) - J;  -h s_i = -2h x_i + h
    int64_t offset = 0;
    std::vector<int64_t> lin((size_t)n, 0);
    for (int32_t i = 0; i < n; ++i) {
        lin[i] -= 2 * (int64_t)h[i];
        offset += h[i];
        for (int32_t j = i + 1; j < n; ++j) {
            const int64_t Jij = J[(size_t)i * n + j];
            lin[i] += 2 * Jij;
            lin[j] += 2 * Jij;
            offset -= Jij;
        }
    }
    for (int32_t i = 0; i < n; ++i) {
        for (int32_t j = 0; j < n; ++j) {
            // x^T W x counts the pair (i, j) twice: W_ij = -4 J / 2
            const int64_t v = i == j ? lin[i] : -2 * (int64_t)J[(size_t)std::min(i, j) * n + std::max(i, j)];
            if (v < INT16_MIN || v > INT16_MAX)
                return fail(ABS_ERANGE, "abs_ising_to_qubo: W entry out of int16 range at (" + std::to_string(i) +
                                            ", " + std::to_string(j) + ")");
            W_out[(size_t)i * n + j] = (int16_t)v;
        }
    }
    *offset_out = offset;
    return ABS_OK;
}

int abs_qubo_to_ising(int32_t n, const int16_t *W, int32_t *J2_out, int32_t *h2_out, int64_t *offset2_out)
{
    if (n < 1 || !W) return fail(ABS_EINVAL, "abs_qubo_to_ising: bad arguments");
    int64_t off2 = 0;
    for (int32_t i = 0; i < n; ++i) {
        int64_t row = 0;
        for (int32_t j = 0; j < n; ++j) {
            const int64_t w = W[(size_t)i * n + j];
            if (w != W[(size_t)j * n + i]) return fail(ABS_EINVAL, "abs_qubo_to_ising: W is not symmetric");
            row += w;
            if (J2_out) J2_out[(size_t)i * n + j] = i == j ? 0 : (int32_t)(-w);
            if (j > i) off2 += w;  // -sum_{i<j} 2J = +sum_{i<j} W_ij
        }
        if (h2_out) h2_out[i] = (int32_t)(-row);
        off2 -= row;  // sum 2h = -sum_i sum_j W_ij
    }
    if (offset2_out) *offset2_out = off2;
    return ABS_OK;
}

int abs_device_searches(int32_t n, int32_t device, int32_t *out)
{
    if (!out || n < 1 || n > 32768) return fail(ABS_EINVAL, "abs_device_searches: n out of range or out == NULL");
    int prev = 0;
    ABS_CU(cudaGetDevice(&prev));
    ABS_CU(cudaSetDevice(device));
    int n_pad = 0, bpt = 0, nt = 0, per_sm = 0, sms = 0;
    layout_for(n, n_pad, bpt, nt);
    const int rc = round_occupancy(nt, bpt, &per_sm);
    const cudaError_t e2 = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    cudaSetDevice(prev);
    ABS_CK(rc);
    ABS_CU(e2);
    *out = per_sm * sms;
    return ABS_OK;
}

int abs_random_qubo_dev(int32_t n, uint64_t seed, int16_t *W_dev, int32_t device)
{
    if (n < 1 || n > ABS_N_MAX || !W_dev) return fail(ABS_EINVAL, "abs_random_qubo_dev: n out of range or W_dev == NULL");
    int prev = 0;
    ABS_CU(cudaGetDevice(&prev));
    if (device >= 0) ABS_CU(cudaSetDevice(device));
    int rc = launch_random_qubo(W_dev, n, seed, 0);
    if (rc == 0) rc = (int)cudaDeviceSynchronize();
    cudaSetDevice(prev);
    ABS_CU((cudaError_t)rc);
    return ABS_OK;
}

const char *abs_version(void) { return "abs-b200 0.1 (sm_100a)"; }

}  // extern "C"
