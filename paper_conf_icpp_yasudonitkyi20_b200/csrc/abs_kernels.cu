// sm_100a kernels of the ABS hot path.  Citations: /root/reference/PAPER.md
// line numbers (P:Lnnn); readings Cnn are listed in DESIGN.md.
//
// One search = one CTA of NT threads (NT = n_pad / 32, a multiple of 32), 32
// bits per thread (the paper's "p bits per thread", fixed at 32 here).
// The per-bit state lives in registers for the whole round: the field
//   g_i = 2 * sum_{j != i} W_ij x_j + W_ii        so that Delta_i = phi(x_i) g_i  (Eq.(13))
// which turns the flip update Eq.(16) into a sign-free row add:
//   g_i += 2 phi(x_k) W_ik  for i != k  (g_k unchanged; Wz has a zero diagonal,
//   so the full-row add leaves g_k alone without a branch).
// The row W_k* is staged into shared memory by cp.async.bulk (TMA bulk copy,
// SASS UBLKCP) in four chunks, one per byte-group, each with its own mbarrier,
// so compute on chunk j overlaps the arrival of chunk j+1.
#include <climits>
#include <cstdint>

#include "abs_internal.h"

namespace absb {
namespace {

constexpr uint64_t kFnvOffset = 0xcbf29ce484222325ull;
constexpr uint64_t kFnvPrime = 0x100000001b3ull;
constexpr unsigned kFull = 0xffffffffu;

// ------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void fence_mbar_init()
{
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

// TMA bulk copy global -> shared, completion signalled on an mbarrier.
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar)
{
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity)
{
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

// ------------------------------------------------------------------ search helpers
// Delta_i = phi(x_i) * g_i (Eq.(3): phi(0) = +1, phi(1) = -1)
__device__ __forceinline__ int readout(int g, uint32_t xm, int s)
{
    return ((xm >> s) & 1u) ? -g : g;
}

// global bit index of slot s of thread t
__device__ __forceinline__ int slot_index(int t, int nt, int s)
{
    return 8 * (t + nt * (s >> 3)) + (s & 7);
}

// bits [lo, hi) of the byte-group starting at element `base`, as an 8-bit mask
__device__ __forceinline__ uint32_t range8(int base, int lo, int hi)
{
    const int e0 = max(lo - base, 0);
    const int e1 = min(hi - base, 8);
    if (e1 <= e0) return 0u;
    return ((1u << e1) - 1u) & ~((1u << e0) - 1u);
}

// Window {(a + j) mod n : 0 <= j < l} (Fig. 2) restricted to the 32
// slots of thread t, as a slot mask.
__device__ __forceinline__ uint32_t window_mask(int a, int l, int n, int t, int nt)
{
    const int hi1 = min(a + l, n);
    const int hi2 = a + l - n;  // wrapped part [0, hi2) when > 0
    uint32_t cm = 0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const int base = 8 * (t + nt * j);
        uint32_t m = 0;
        if (base + 8 > a && base < hi1) m |= range8(base, a, hi1);
        if (hi2 > 0 && base < hi2) m |= range8(base, 0, hi2);
        cm |= m << (8 * j);
    }
    return cm;
}

// Lowest-index argmin of Delta over the slots in `cm` (ascending slot order
// is ascending bit index within a thread).  ci2 = 2 * index + x_index, or
// INT_MAX when cm selects nothing.
__device__ __forceinline__ void candidates(const int (&g)[32], uint32_t xm, uint32_t cm, int t, int nt, int &cv,
                                           int &ci2)
{
    cv = INT_MAX;
    int cs = -1;
#pragma unroll
    for (int s = 0; s < 32; ++s) {
        const int d = readout(g[s], xm, s);
        if (((cm >> s) & 1u) && d < cv) {
            cv = d;
            cs = s;
        }
    }
    ci2 = cs < 0 ? INT_MAX : 2 * slot_index(t, nt, cs) + (int)((xm >> cs) & 1u);
}

struct Red {
    int v;  // min Delta over all bits (neighbour tracking)
    int c;  // min Delta over the candidate set (straight: mismatches, local: window)
    int i;  // 2 * (lowest index attaining c) + x_that_index
};

// CTA-wide reduction; every thread receives the result.  Lowest index wins
// ties (reading C5).  Two alternating smem slots -> one barrier per call.
template <bool kSingleWarp>
__device__ __forceinline__ Red block_reduce(Red r, Red *sred, int &rb, int lane, int warp, int nw)
{
    // sred points at Red[2][32]
    Red w;
    w.v = __reduce_min_sync(kFull, r.v);
    w.c = __reduce_min_sync(kFull, r.c);
    w.i = __reduce_min_sync(kFull, r.c == w.c ? r.i : INT_MAX);
    if (kSingleWarp) return w;
    Red *buf = sred + (rb & 1) * 32;
    ++rb;
    if (lane == 0) buf[warp] = w;
    __syncthreads();
    Red x;
    if (lane < nw) {
        x = buf[lane];
    } else {
        x.v = INT_MAX;
        x.c = INT_MAX;
        x.i = INT_MAX;
    }
    w.v = __reduce_min_sync(kFull, x.v);
    w.c = __reduce_min_sync(kFull, x.c);
    w.i = __reduce_min_sync(kFull, x.c == w.c ? x.i : INT_MAX);
    return w;
}

template <bool kSingleWarp>
__device__ __forceinline__ bool block_any(bool p)
{
    if (kSingleWarp) return __any_sync(kFull, p);
    return __syncthreads_or(p) != 0;
}

// ------------------------------------------------------------------ round kernel
// Per-CTA scratch in shared memory (after the row buffer).
struct RoundSmem {
    uint64_t bar[4];     // one mbarrier per row chunk
    Red red[2][32];      // block_reduce slots
    uint64_t hash;       // thread 0 only
    long long nflip, nstraight;
};

// Update g with row k (chunks arrive via TMA), read out Delta, min over all
// bits and (straight phase) the lowest-index argmin over mismatches.
template <bool kStraight>
__device__ __forceinline__ void flip_elems(int (&g)[32], uint32_t xm, uint32_t mism, const uint4 *sW4,
                                           uint64_t *bar, uint32_t parity, int c, int t, int nt, int &vmin,
                                           int &cv, int &cs)
{
    vmin = INT_MAX;
    cv = INT_MAX;
    cs = -1;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        mbar_wait(&bar[j], parity);
        const uint4 w4 = sW4[t + nt * j];
        const uint32_t wv[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int s0 = 8 * j + 2 * q;
            const int wlo = (int)(short)(wv[q] & 0xffffu);
            const int whi = ((int)wv[q]) >> 16;
            g[s0] += c * wlo;  // Eq.(16) in field form
            g[s0 + 1] += c * whi;
            const int d0 = readout(g[s0], xm, s0);
            const int d1 = readout(g[s0 + 1], xm, s0 + 1);
            vmin = min(vmin, min(d0, d1));  // all n neighbours evaluated (Eq.(5))
            if (kStraight) {
                if (((mism >> s0) & 1u) && d0 < cv) {
                    cv = d0;
                    cs = s0;
                }
                if (((mism >> (s0 + 1)) & 1u) && d1 < cv) {
                    cv = d1;
                    cs = s0 + 1;
                }
            }
        }
    }
}

// One CTA runs one round (device Steps 2-5) of search blockIdx.x.
template <int kMaxThreads, int kMinBlocks, bool kSingleWarp>
__global__ void __launch_bounds__(kMaxThreads, kMinBlocks) round_kernel(const RoundArgs A)
{
    extern __shared__ __align__(128) unsigned char smem[];
    const int nt = kSingleWarp ? 32 : A.nt;
    const int t = threadIdx.x;
    const int lane = t & 31, warp = t >> 5, nw = nt >> 5;
    const int sid = blockIdx.x;

    const uint4 *sW4 = reinterpret_cast<const uint4 *>(smem);
    RoundSmem *sm = reinterpret_cast<RoundSmem *>(smem + 64 * nt);
    uint32_t *stm = reinterpret_cast<uint32_t *>(smem + 64 * nt + sizeof(RoundSmem));  // [nt] target bits
    uint32_t *sbm = stm + nt;                                                          // [nt] best bits

    if (t == 0) {
#pragma unroll
        for (int j = 0; j < 4; ++j) mbar_init(&sm->bar[j], 1);
        fence_mbar_init();
        sm->hash = A.hash[sid];
        sm->nflip = 0;
        sm->nstraight = 0;
    }

    // ---- load the search state (registers for the whole round)
    int g[32];
    {
        const int32_t *gs = A.g + (size_t)sid * 32 * nt;
#pragma unroll
        for (int s = 0; s < 32; ++s) g[s] = gs[(size_t)s * nt + t];
    }
    uint32_t xm = 0;
    {
        const uint8_t *Xs = A.X + (size_t)sid * 4 * nt;
        const uint8_t *Ts = A.T + (size_t)sid * 4 * nt;
        uint32_t tm = 0;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            xm |= (uint32_t)Xs[t + nt * j] << (8 * j);
            tm |= (uint32_t)Ts[t + nt * j] << (8 * j);  // Step 2: read target T
        }
        stm[t] = tm;
        sbm[t] = xm;  // Step 3, reading C4: B = C ...
    }
    int64_t E = A.E[sid];
    int64_t EB = E;  // ... and E_B = E(C) (Alg. 5)
    int a = A.a[sid];
    const int l = A.l[sid];
    int left = (int)A.L;
    int rb = 0;
    uint32_t parity = 0;
    if (!kSingleWarp) __syncthreads();  // barrier init + smem state visible
    else __syncwarp();

    bool straight = block_any<kSingleWarp>(xm != stm[t]);
    Red r;
    {
        // first selection of the round
        int cv, ci2;
        const uint32_t cm = straight ? (xm ^ stm[t]) : window_mask(a, l, A.n, t, nt);
        candidates(g, xm, cm, t, nt, cv, ci2);
        r = block_reduce<kSingleWarp>(Red{INT_MAX, cv, ci2}, sm->red[0], rb, lane, warp, nw);
    }
    bool have = straight || left > 0;

    while (have) {
        const int k = r.i >> 1;
        // ---- flip k (Alg. 4 lines P:L328-336 / Alg. 5 lines P:L371-376)
        if (t == 0) {
            const uint32_t chunk = 16u * (uint32_t)nt;
            const char *src = reinterpret_cast<const char *>(A.Wz) + (size_t)k * (size_t)A.n_pad * 2;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                mbar_arrive_expect_tx(&sm->bar[j], chunk);
                bulk_g2s(smem + (size_t)chunk * j, src + (size_t)chunk * j, chunk, &sm->bar[j]);
            }
            sm->hash = (sm->hash ^ (uint64_t)(uint32_t)k) * kFnvPrime;
            sm->nflip += 1;
            if (straight) sm->nstraight += 1;
        }
        const int c = (r.i & 1) ? -2 : 2;  // 2 phi(x_k) with the pre-flip bit (Eq.(16))
        E += r.c;                           // E(X) <- E(X) + d_k
        {
            const int beta = k >> 3;
            if (t == beta % nt) xm ^= 1u << (8 * (beta / nt) + (k & 7));  // x_k <- 1 - x_k
        }
        int vmin, cv, cs, ci2;
        if (straight) {
            flip_elems<true>(g, xm, xm ^ stm[t], sW4, sm->bar, parity, c, t, nt, vmin, cv, cs);
            ci2 = cs < 0 ? INT_MAX : 2 * slot_index(t, nt, cs) + (int)((xm >> cs) & 1u);
        } else {
            flip_elems<false>(g, xm, 0u, sW4, sm->bar, parity, c, t, nt, vmin, cv, cs);
            a = (int)(((int64_t)a + l) % A.n);  // offset <- (a + l) mod n
            const uint32_t cm = window_mask(a, l, A.n, t, nt);
            if (__any_sync(kFull, cm != 0u)) {
                candidates(g, xm, cm, t, nt, cv, ci2);
            } else {
                cv = INT_MAX;
                ci2 = INT_MAX;
            }
        }
        parity ^= 1u;
        r = block_reduce<kSingleWarp>(Red{vmin, cv, ci2}, sm->red[0], rb, lane, warp, nw);

        // ---- neighbour tracking (reading C2): cand = E' + min(0, m)
        {
            const int m = r.v;
            const int64_t cand = E + (m < 0 ? (int64_t)m : 0);
            if (cand < EB) {  // uniform across the CTA
                uint32_t bm = xm;
                if (m < 0) {
                    int ii = INT_MAX;
#pragma unroll
                    for (int s = 31; s >= 0; --s)
                        if (readout(g[s], xm, s) == m) ii = slot_index(t, nt, s);
                    const Red q = block_reduce<kSingleWarp>(Red{INT_MAX, 0, ii}, sm->red[0], rb, lane, warp, nw);
                    const int beta = q.i >> 3;
                    if (t == beta % nt) bm ^= 1u << (8 * (beta / nt) + (q.i & 7));
                }
                sbm[t] = bm;
                EB = cand;
            }
        }

        if (!straight) {
            if (--left <= 0) break;
        } else if (r.i == INT_MAX) {
            // X = T: the straight search is over; local search from T (Step 4b)
            straight = false;
            if (left <= 0) break;
            int cv2, ci22;
            candidates(g, xm, window_mask(a, l, A.n, t, nt), t, nt, cv2, ci22);
            r = block_reduce<kSingleWarp>(Red{INT_MAX, cv2, ci22}, sm->red[0], rb, lane, warp, nw);
        }
    }

    // ---- Step 5: store (B, E_B) and the state C' for the next round
    {
        int32_t *gs = A.g + (size_t)sid * 32 * nt;
#pragma unroll
        for (int s = 0; s < 32; ++s) gs[(size_t)s * nt + t] = g[s];
        uint8_t *Xs = A.X + (size_t)sid * 4 * nt;
        uint8_t *Bs = A.B + (size_t)sid * 4 * nt;
        const uint32_t bm = sbm[t];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            Xs[t + nt * j] = (uint8_t)(xm >> (8 * j));
            Bs[t + nt * j] = (uint8_t)(bm >> (8 * j));
        }
        if (t == 0) {
            A.E[sid] = E;
            A.EB[sid] = EB;
            A.a[sid] = a;
            A.hash[sid] = sm->hash;
            A.flips[sid] += sm->nflip;
            A.sflips[sid] += sm->nstraight;
        }
    }
}

// ------------------------------------------------------------------ setup kernels
// Wz = W with zero diagonal padded to n_pad x n_pad; diag = W_ii; counts
// asymmetric entries (W must be symmetric).
__global__ void prepare_w_kernel(const int16_t *__restrict__ W, int n, int n_pad, int16_t *__restrict__ Wz,
                                 int32_t *__restrict__ diag, unsigned long long *asym)
{
    __shared__ int16_t ta[32][33];
    __shared__ int16_t tb[32][33];
    const int bx = blockIdx.x * 32, by = blockIdx.y * 32;
    const int tx = threadIdx.x, ty = threadIdx.y;
    for (int r = ty; r < 32; r += 8) {
        const int row = by + r, col = bx + tx;
        ta[r][tx] = (row < n && col < n) ? W[(size_t)row * n + col] : (int16_t)0;
        const int row2 = bx + r, col2 = by + tx;  // transposed block
        tb[r][tx] = (row2 < n && col2 < n) ? W[(size_t)row2 * n + col2] : (int16_t)0;
    }
    __syncthreads();
    unsigned long long bad = 0;
    for (int r = ty; r < 32; r += 8) {
        const int row = by + r, col = bx + tx;
        const int16_t v = ta[r][tx];
        if (v != tb[tx][r]) ++bad;
        Wz[(size_t)row * n_pad + col] = (row == col) ? (int16_t)0 : v;
        if (row == col) diag[row] = (row < n) ? (int32_t)v : 0;
    }
    if (bad) atomicAdd(asym, bad);
}

// Device Step 1: C = 0, E = 0, Delta_i = W_ii (g_i = W_ii).
__global__ void zero_start_kernel(int n, int nt, const int32_t *__restrict__ diag, int32_t *g, uint8_t *X,
                                  uint8_t *B, int64_t *E, int64_t *EB, int32_t *a, uint64_t *hash, int64_t *flips,
                                  int64_t *sflips, int s0)
{
    const int sid = s0 + blockIdx.x;
    const int t = threadIdx.x;
    int32_t *gs = g + (size_t)sid * 32 * nt;
    for (int s = 0; s < 32; ++s) {
        const int i = slot_index(t, nt, s);
        gs[(size_t)s * nt + t] = (i < n) ? diag[i] : INT_MAX;  // pads are never candidates nor minima
    }
    for (int j = 0; j < 4; ++j) {
        X[(size_t)sid * 4 * nt + t + nt * j] = 0;
        B[(size_t)sid * 4 * nt + t + nt * j] = 0;
    }
    if (t == 0) {
        E[sid] = 0;
        EB[sid] = 0;
        a[sid] = 0;  // reading C6
        hash[sid] = kFnvOffset;
        flips[sid] = 0;
        sflips[sid] = 0;
    }
}

// Batched initialisation.  Thread = column i, 16 solutions per
// CTA row of the grid.  y_b = Wz x_b (Wz zero-diagonal), then
//   g_i = 2 y_i + W_ii,  Delta_i = phi(x_i) g_i   (Eq.(13))
//   E = sum_i x_i (y_i + W_ii)                    (Eq.(1))
constexpr int kInitB = 16;
constexpr int kInitT = 256;
__global__ void __launch_bounds__(kInitT) batch_init_kernel(const int16_t *__restrict__ Wz,
                                                            const int32_t *__restrict__ diag, int n, int n_pad,
                                                            const uint8_t *__restrict__ X, int count,
                                                            int64_t *__restrict__ Eout, int32_t *__restrict__ delta)
{
    extern __shared__ uint32_t sx[];  // [kInitB][n_pad/32]
    __shared__ long long red[kInitB][kInitT / 32];
    const int words = n_pad / 32;
    const int b0 = blockIdx.y * kInitB;
    const int i = blockIdx.x * kInitT + threadIdx.x;
    for (int q = threadIdx.x; q < kInitB * words; q += kInitT) {
        const int b = q / words, w = q % words;
        uint32_t v = 0;
        if (b0 + b < count) {
            const uint8_t *xb = X + (size_t)(b0 + b) * (n_pad / 8) + 4 * w;
            v = (uint32_t)xb[0] | ((uint32_t)xb[1] << 8) | ((uint32_t)xb[2] << 16) | ((uint32_t)xb[3] << 24);
        }
        sx[b * words + w] = v;
    }
    __syncthreads();
    int acc[kInitB];
#pragma unroll
    for (int b = 0; b < kInitB; ++b) acc[b] = 0;
    for (int w = 0; w < words; ++w) {
        uint32_t xw[kInitB];
        uint32_t any = 0;
#pragma unroll
        for (int b = 0; b < kInitB; ++b) {
            xw[b] = sx[b * words + w];
            any |= xw[b];
        }
        if (!any) continue;
        for (int jj = 0; jj < 32; ++jj) {
            const int j = w * 32 + jj;
            const int v = Wz[(size_t)j * n_pad + i];  // column i of row j == W_ij (symmetric)
#pragma unroll
            for (int b = 0; b < kInitB; ++b)
                if ((xw[b] >> jj) & 1u) acc[b] += v;
        }
    }
    const int di = diag[i];
    const uint32_t *xi_w = sx + (i >> 5);
#pragma unroll
    for (int b = 0; b < kInitB; ++b) {
        const int xi = (int)((xi_w[b * words] >> (i & 31)) & 1u);
        const int gi = 2 * acc[b] + di;
        if (delta && i < n && b0 + b < count) delta[(size_t)(b0 + b) * n + i] = xi ? -gi : gi;
        long long e = xi ? (long long)acc[b] + di : 0;
        for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(kFull, e, o);
        if ((threadIdx.x & 31) == 0) red[b][threadIdx.x >> 5] = e;
    }
    __syncthreads();
    if (threadIdx.x < kInitB && b0 + (int)threadIdx.x < count) {
        long long e = 0;
        for (int w = 0; w < kInitT / 32; ++w) e += red[threadIdx.x][w];
        atomicAdd(reinterpret_cast<unsigned long long *>(Eout + b0 + threadIdx.x), (unsigned long long)e);
    }
}

}  // namespace

// ------------------------------------------------------------------ launchers
size_t round_smem_bytes(int32_t nt)
{
    return (size_t)64 * nt + sizeof(RoundSmem) + 2 * sizeof(uint32_t) * (size_t)nt;
}

int launch_prepare_w(const int16_t *W_in, int32_t n, int32_t n_pad, int16_t *Wz, int32_t *diag,
                     unsigned long long *asym_count, cudaStream_t st)
{
    dim3 grid(n_pad / 32, n_pad / 32), block(32, 8);
    prepare_w_kernel<<<grid, block, 0, st>>>(W_in, n, n_pad, Wz, diag, asym_count);
    return (int)cudaGetLastError();
}

int launch_zero_start(const Instance &I, SearchState &S, int32_t s0, int32_t s1, cudaStream_t st)
{
    if (s1 <= s0) return 0;
    zero_start_kernel<<<s1 - s0, I.nt, 0, st>>>(I.n, I.nt, I.diag, S.g, S.X, S.B, S.E, S.EB, S.a, S.hash, S.flips,
                                                 S.sflips, s0);
    return (int)cudaGetLastError();
}

int launch_round(const RoundArgs &a, cudaStream_t st)
{
    const size_t smem = round_smem_bytes(a.nt);
    if (a.nt == 32) {
        auto k = round_kernel<32, 32, true>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k<<<a.S, 32, smem, st>>>(a);
    } else {
        auto k = round_kernel<1024, 1, false>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k<<<a.S, a.nt, smem, st>>>(a);
    }
    return (int)cudaGetLastError();
}

int launch_batch_init(const Instance &I, const uint8_t *X, int32_t count, int64_t *E, int32_t *delta,
                      cudaStream_t st)
{
    if (count <= 0) return 0;
    cudaMemsetAsync(E, 0, sizeof(int64_t) * (size_t)count, st);
    dim3 grid(I.n_pad / kInitT, (count + kInitB - 1) / kInitB);
    const size_t smem = (size_t)kInitB * (I.n_pad / 32) * sizeof(uint32_t);
    cudaFuncSetAttribute(batch_init_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    batch_init_kernel<<<grid, kInitT, smem, st>>>(I.Wz, I.diag, I.n, I.n_pad, X, count, E, delta);
    return (int)cudaGetLastError();
}

}  // namespace absb
