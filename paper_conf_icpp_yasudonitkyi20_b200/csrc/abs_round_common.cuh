// Shared pieces of the ABS round kernels (multi-warp searches: abs_round.cu;
// one-warp searches: abs_round_warp.cu): the SA acceptance (Eq.(7)), Philox,
// and the lockstep / asynchronous kernel shells around a round implementation
// R (R::init_barriers, R::run).  Citations: /root/reference/PAPER.md (P:Lnnn).
#pragma once
#include <algorithm>
#include <climits>
#include <cstdint>

#include "abs_internal.h"
#include "ptx.cuh"

// Diagnostics build (-DABS_TIMING): per-warp cycle accounting of the flip loop.
#ifdef ABS_TIMING
#define ABS_T(x) x
#else
#define ABS_T(x)
#endif

namespace absb {
namespace {

constexpr unsigned kFullMask = 0xffffffffu;

template <int kP>
struct MaskOf;
template <>
struct MaskOf<32> {
    using T = uint32_t;
};
template <>
struct MaskOf<64> {
    using T = uint64_t;
};

constexpr uint32_t kTagSA = 0x5341504Cu;  // 'SAPL'
// SA proposals evaluated per barrier by the multi-warp searches (at most; the batch
// adapts, Round::sa_next), <= 32 (one lane per proposal): each batch pays a CTA barrier;
// 32 measured +9.5% at n = 32k and +1.5% at n = 10,000 over 8.  One-warp searches
// (WarpRound::sa_next) always evaluate 32 at once against their shared-memory state mirror.
#ifndef ABS_SA_BATCH_MULTI
#define ABS_SA_BATCH_MULTI 32
#endif
constexpr int kSaBatchMulti = ABS_SA_BATCH_MULTI;
static_assert(kSaBatchMulti >= 1 && kSaBatchMulti <= 32, "one lane per proposal");

// Philox4x32-10 (Salmon et al., SC'11), the library's device copy (the oracle
// has its own; both are pinned by the Random123 known-answer vectors).
__device__ __forceinline__ void philox4x32_10(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, uint32_t k0,
                                              uint32_t k1, uint32_t (&o)[4])
{
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
        const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
        c0 = hi1 ^ c1 ^ k0;
        c1 = lo1;
        c2 = hi0 ^ c3 ^ k1;
        c3 = lo0;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    o[0] = c0;
    o[1] = c1;
    o[2] = c2;
    o[3] = c3;
}

// Exact unsigned 32-bit division by a divisor fixed for a round (n for the SA bit
// draw, tau for the acceptance exponent): Granlund-Montgomery round-up multiply,
// q = (t + ((x - t) >> s1)) >> s2 with t = umulhi(m, x), for every x < 2^32, d >= 1
// (tests/test_udiv.py checks the same arithmetic on the host).
struct UDiv {
    uint32_t d, m, s1, s2;
};
__host__ __device__ inline UDiv make_udiv(uint32_t d)
{
    uint32_t l = 0;  // ceil(log2 d)
    while (l < 32 && (1ull << l) < d) ++l;
    UDiv r;
    r.d = d;
    r.m = (uint32_t)((((1ull << l) - d) << 32) / d + 1);
    r.s1 = l < 1 ? l : 1;
    r.s2 = l > 1 ? l - 1 : 0;
    return r;
}
__device__ __forceinline__ uint32_t udiv(uint32_t x, const UDiv &v)
{
    const uint32_t t = __umulhi(v.m, x);
    return (t + ((x - t) >> v.s1)) >> v.s2;
}
__device__ __forceinline__ uint32_t umod(uint32_t x, const UDiv &v) { return x - udiv(x, v) * v.d; }

// SA acceptance (Eq.(7), reading E2): an uphill move dE > 0 is
// accepted with p = exp(-dE/(k_B t)), k_B t = tau / ln 2, i.e. p = 2^(-dE/tau);
// the decision is u < P for a uniform uint32 u and the Q32 integer
// P = floor(2^32 p), computed exactly in integers:
//   2^(-dE/tau) = 2^(-q) e^(-x),  q = dE div tau,  x = ln2 (dE mod tau) / tau,
//   e^(-x) by its Taylor series in Q63 (terms vanish by k = 19 since x < ln 2).
constexpr uint64_t kLn2Q64 = 0xB17217F7D1CF79ABull;  // floor(ln 2 * 2^64)

__device__ __noinline__ uint64_t sa_threshold_exact(int dE, int tau)
{
    const uint32_t ut = (uint32_t)tau;
    const uint32_t q = (uint32_t)dE / ut;
    const uint32_t r = (uint32_t)dE - q * ut;
    if (q > 32) return 0;
    // F = floor(r 2^64 / tau), Q64, by two 64/32-bit long-division steps (r < tau < 2^31)
    const uint64_t n1 = (uint64_t)r << 32;
    const uint64_t h = n1 / ut;
    const uint64_t n2 = (n1 - h * ut) << 32;
    const uint64_t F = (h << 32) | (n2 / ut);
    const uint64_t x = __umul64hi(F, kLn2Q64);  // ln2 r / tau, Q64
    uint64_t term = 1ull << 63, y = 1ull << 63;  // Q63
#pragma unroll
    for (int k = 1; k <= 20; ++k) {
        term = __umul64hi(term, x) / (uint64_t)k;  // x^k / k!
        y = (k & 1) ? y - term : y + term;
    }
    return y >> (31 + q);  // 2^32 2^(-q) y / 2^63
}

// floor((2^64 - 1) / (2 tau)): sa_accept's reciprocal of the chord denominator, once per round
__device__ __forceinline__ uint64_t sa_inv2tau(int tau) { return ~0ull / (2ull * (uint32_t)tau); }

// u < P(dE, tau), deciding most draws without P: the chord C of 2^(-x) between
// the integer exponents q and q+1 lies above the convex 2^(-x) and at most 6.2%
// above it, so P <= C and P > 15 C / 16 - 1 (reading E2); only a
// draw inside that band computes P.  C is taken through the reciprocal inv2tau
// (no division per draw): C' = floor(prod inv2tau / 2^64) lies in [C - 2, C],
// and the band is widened by 2 to match.
__device__ __forceinline__ bool sa_accept(int dE, int tau, uint64_t inv2tau, uint32_t u)
{
    if (dE <= 0) return true;
    const uint32_t q = (uint32_t)dE / (uint32_t)tau;
    if (q > 32) return false;
    const uint32_t r = (uint32_t)dE - q * (uint32_t)tau;
    const uint64_t prod = (1ull << (32 - q)) * (2ull * (uint32_t)tau - r);  // < 2^64
    const long long C = (long long)__umul64hi(prod, inv2tau);
    if ((long long)u >= C + 18) return false;
    if ((long long)u < C - (C >> 4) - 16) return true;
    return (uint64_t)u < sa_threshold_exact(dE, tau);
}

// sa_accept without its exact step: 1 accept, 0 reject, 2 undecided (u inside the
// chord band; the caller decides it with sa_threshold_exact).
__device__ __forceinline__ int sa_accept_fast(int dE, int tau, uint64_t inv2tau, uint32_t u)
{
    if (dE <= 0) return 1;
    const uint32_t q = (uint32_t)dE / (uint32_t)tau;
    if (q > 32) return 0;
    const uint32_t r = (uint32_t)dE - q * (uint32_t)tau;
    const uint64_t prod = (1ull << (32 - q)) * (2ull * (uint32_t)tau - r);  // < 2^64
    const long long C = (long long)__umul64hi(prod, inv2tau);
    if ((long long)u >= C + 18) return 0;
    if ((long long)u < C - (C >> 4) - 16) return 1;
    return 2;
}

// The same two with the round's divisor of tau precomputed (one-warp kernels).
__device__ __forceinline__ bool sa_accept(int dE, const UDiv &dt, uint64_t inv2tau, uint32_t u)
{
    if (dE <= 0) return true;
    const uint32_t q = udiv((uint32_t)dE, dt);
    if (q > 32) return false;
    const uint32_t r = (uint32_t)dE - q * dt.d;
    const uint64_t prod = (1ull << (32 - q)) * (2ull * dt.d - r);  // < 2^64
    const long long C = (long long)__umul64hi(prod, inv2tau);
    if ((long long)u >= C + 18) return false;
    if ((long long)u < C - (C >> 4) - 16) return true;
    return (uint64_t)u < sa_threshold_exact(dE, (int)dt.d);
}
__device__ __forceinline__ int sa_accept_fast(int dE, const UDiv &dt, uint64_t inv2tau, uint32_t u)
{
    if (dE <= 0) return 1;
    const uint32_t q = udiv((uint32_t)dE, dt);
    if (q > 32) return 0;
    const uint32_t r = (uint32_t)dE - q * dt.d;
    const uint64_t prod = (1ull << (32 - q)) * (2ull * dt.d - r);  // < 2^64
    const long long C = (long long)__umul64hi(prod, inv2tau);
    if ((long long)u >= C + 18) return 0;
    if ((long long)u < C - (C >> 4) - 16) return 1;
    return 2;
}



template <class R, int kThreads, int kMinBlocks>
__global__ void __launch_bounds__(kThreads, kMinBlocks) round_kernel(const RoundArgs A)
{
    extern __shared__ __align__(128) unsigned char smem[];
    const int sid = blockIdx.x + A.sbase;
    const size_t bpv = (size_t)A.n_pad / 8;
    int fbase = 0;
    R::init_barriers(smem);
    uint8_t *const B0 = A.B + sid * bpv;
    int64_t *const EB0 = A.EB + sid;
    R::run(
        A, smem, sid, A.T + sid * bpv,
        [=](uint8_t *&Bp, int64_t *&EBp) {
            Bp = B0;
            EBp = EB0;
        },
        fbase);
}

// ---------------------------------------------------------------- asynchronous mode
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(uint32_t *p, uint32_t v)
{
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ int ld_acquire_gpu(const int *p)
{
    int v;
    asm volatile("ld.acquire.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_gpu(int *p, int v)
{
    asm volatile("st.release.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// The paper's device loop (Steps 2-5 repeated) as a persistent
// kernel.  When every search fits on the GPU (S <= resident CTAs) CTA b owns
// search b and draws round tickets from a shared budget, so each search runs
// at its own pace ("each CUDA block operates asynchronously");
// otherwise CTAs take (search, round) items from a queue.  A round reads the
// search's latest target from mapped host memory (Step 2; a stale target is
// reused, reading C11) and publishes (B, E_B) to mapped host memory with a
// system-scope release and appends (search, round) to an arrival ring the host
// GA polls.
// Host and device never synchronise directly.
template <class R, int kThreads, int kMinBlocks>
__global__ void __launch_bounds__(kThreads, kMinBlocks) round_kernel_async(const RoundArgs A, const AsyncArgs Q)
{
    extern __shared__ __align__(128) unsigned char smem[];
    // the current work item, kept in shared memory so that nothing of it stays
    // live in registers across the flip loop
    __shared__ long long item;
    __shared__ int cur_s, cur_r, r_own;
    __shared__ uint32_t tver;
    const size_t bpv = (size_t)A.n_pad / 8;
    constexpr bool multi = kThreads > 32;
    int fbase = 0;
    R::init_barriers(smem);
    if (threadIdx.x == 0) r_own = Q.owned ? ld_acquire_gpu(Q.done + blockIdx.x) : 0;
    for (;;) {
        if (threadIdx.x == 0) {
            const long long q = (long long)atomicAdd(Q.queue, 1ull);
            item = q;
            if (q < Q.total) {
                const int s = Q.owned ? (int)blockIdx.x : (int)(q % A.S);
                const int r = Q.owned ? r_own++ : Q.base + (int)(q / A.S);
                ABS_T(const long long w0 = clock64();)
                if (!Q.owned)
                    while (ld_acquire_gpu(Q.done + s) != r) __nanosleep(256);  // round r-1 of s finished
                ABS_T(const long long w1 = clock64();)
                // the result slot of round r (double-buffered) must have been consumed by the host
                while ((int)ld_acquire_sys(Q.rack + s) < r - 1) __nanosleep(1024);
                ABS_T(const long long w2 = clock64();)
                tver = ld_acquire_sys(Q.tseq + s);  // latest published target version
                cur_s = s;
                cur_r = r;
                ABS_T(if (A.timing) {
                    unsigned long long *tm = (unsigned long long *)&A.timing[((size_t)s * 32) * 24];
                    atomicAdd(tm + 16, (unsigned long long)(w1 - w0));
                    atomicAdd(tm + 17, (unsigned long long)(w2 - w1));
                    atomicAdd(tm + 18, (unsigned long long)(clock64() - w2));
                    atomicAdd(tm + 20, 1ull);
                })
            }
        }
        if (multi) __syncthreads();
        else __syncwarp();
        if (item >= Q.total) break;
        R::run(
            A, smem, cur_s, Q.Tmap + ((size_t)cur_s * 2 + (tver & 1)) * bpv,
            [&](uint8_t *&Bp, int64_t *&EBp) {
                const int s = cur_s, r = cur_r;
                Bp = Q.Rb + ((size_t)s * 2 + (r & 1)) * bpv;
                EBp = Q.Reb + (size_t)s * 2 + (r & 1);
            },
            fbase);
        if (threadIdx.x == 0) Q.rtver[(size_t)cur_s * 2 + (cur_r & 1)] = tver;
        __threadfence_system();  // B, E_B and the target version reach host memory ...
        if (multi) __syncthreads();
        else __syncwarp();
        if (threadIdx.x == 0) {
            ABS_T(const long long p0 = clock64();)
            const int s = cur_s, r = cur_r;
            // arrival ring: the host GA drains results in this order.  The
            // index comes from a DEVICE counter: a system-scope atomic on host memory
            // serialises every CTA over PCIe (~1M results/s for the whole GPU)
            const uint32_t idx = atomicAdd(Q.rcount, 1u);
            Q.ring[2 * (idx & Q.ring_mask)] = (uint32_t)s;
            Q.ring[2 * (idx & Q.ring_mask) + 1] = (uint32_t)r;
            st_release_sys(Q.ringseq + (idx & Q.ring_mask), idx + 1u);  // ... before the ring entry
            st_release_gpu(Q.done + s, r + 1);
            ABS_T(if (A.timing) atomicAdd((unsigned long long *)&A.timing[((size_t)s * 32) * 24 + 19],
                                          (unsigned long long)(clock64() - p0));)
        }
    }
}


// One launch of the round kernel of implementation R: lockstep (q == NULL, one CTA
// per search) or the persistent async kernel (grid = resident CTAs, at most S).
template <class R, int kThreads, int kMinBlocks>
int launch_kernel(const RoundArgs &a, cudaStream_t st, size_t smem, const AsyncArgs *q, int *grid_out)
{
    if (!q) {
        auto k = round_kernel<R, kThreads, kMinBlocks>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k<<<a.S, a.nt, smem, st>>>(a);
        return (int)cudaGetLastError();
    }
    auto k = round_kernel_async<R, kThreads, kMinBlocks>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int per_sm = 0, dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, a.nt, smem);
    const int grid = (int)std::min<long long>((long long)a.S, (long long)std::max(1, per_sm) * sms);
    if (grid_out) *grid_out = grid;
    AsyncArgs q2 = *q;
    q2.owned = grid >= a.S ? 1 : 0;
    k<<<grid, a.nt, smem, st>>>(a, q2);
    return (int)cudaGetLastError();
}

template <class R, int kThreads, int kMinBlocks>
int occupancy_of(int nt, size_t smem, int *per_sm)
{
    auto k = round_kernel<R, kThreads, kMinBlocks>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    return (int)cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k, nt, smem);
}

}  // namespace
}  // namespace absb
