// The ABS search kernel for sm_100a: one CTA runs one round (device Steps
// 2-5) of one search.  Citations: /root/reference/PAPER.md line
// numbers (P:Lnnn); readings Cnn are listed in DESIGN.md.
//
// Layout.  A search of n <= n_pad = 32*NT bits is held by NT threads, 32 bits
// each (the paper's "p bits per thread"): thread t owns the byte-groups
// beta = t + NT*j (j = 0..3), i.e. bits 8*beta .. 8*beta+7, in register slots
// s = 8j + e.  Per bit the registers hold the field
//     g_i = 2 sum_{j != i} W_ij x_j + W_ii,   Delta_i = phi(x_i) g_i   (Eq.(13)),
// so the flip update Eq.(16) is a sign-free row add g_i += 2 phi(x_k) W_ik
// (W is stored with a zero diagonal, so g_k is untouched).  x bits live in one
// register per thread.
//
// Memory.  Row k of W (2*n_pad bytes) is copied into shared memory by
// cp.async.bulk (TMA, SASS UBLKCP) in four chunks, one per byte-group j, each
// signalling its own mbarrier.  Two row buffers: while flip f consumes row
// k_f, row k_{f+1} is already in flight.
//
// Window-first prefetch (local phase, l <= kWinMax).  The next flip k_{f+1}
// depends only on the window W_{f+1} = {(a_{f+1} + r) mod n : r < l}
// (Fig. 2).  During flip f-1 the owners of W_{f+1}'s bits publish
// Delta_i(X_f) and x_i(X_f) to shared memory; at the start of flip f warp 0
// applies row k_f to those l values only, takes the lowest-index argmin and
// issues the TMA for row k_{f+1} immediately -- the row fetch overlaps the
// processing of row k_f instead of following it.
#include <climits>
#include <cstdint>

#include "abs_internal.h"
#include "ptx.cuh"

namespace absb {
namespace {

constexpr uint64_t kFnvPrime = 0x100000001b3ull;
constexpr unsigned kFull = 0xffffffffu;
constexpr int kWinMax = 256;  // largest l served by the prefetch path (ladder max, reading C7)

// Delta_i = phi(x_i) * g_i (Eq.(3): phi(0) = +1, phi(1) = -1)
__device__ __forceinline__ int readout(int g, uint32_t xm, int s)
{
    return ((xm >> s) & 1u) ? -g : g;
}

__device__ __forceinline__ int slot_index(int t, int nt, int s)
{
    return 8 * (t + nt * (s >> 3)) + (s & 7);
}

__device__ __forceinline__ int sext16(uint32_t w)
{
    return (int)(short)(w & 0xffffu);
}

// bits [lo, hi) of the byte-group starting at element `base`, as an 8-bit mask
__device__ __forceinline__ uint32_t range8(int base, int lo, int hi)
{
    const int e0 = max(lo - base, 0);
    const int e1 = min(hi - base, 8);
    if (e1 <= e0) return 0u;
    return ((1u << e1) - 1u) & ~((1u << e0) - 1u);
}

// Slots of thread t inside the window {(a + r) mod n : r < l} (Fig. 2).
__device__ __forceinline__ uint32_t window_mask(int a, int l, int n, int t, int nt)
{
    const int end = a + l;          // exclusive; > n when the window wraps (reading C6)
    const int hi1 = min(end, n);
    const int hi2 = end - n;        // wrapped part [0, hi2)
    uint32_t cm = 0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const int base = 8 * (t + nt * j);
        const bool h1 = (base + 8 > a) && (base < hi1);
        const bool h2 = base < hi2;
        if (h1 | h2) {
            uint32_t m = 0;
            if (h1) m |= range8(base, a, hi1);
            if (h2) m |= range8(base, 0, hi2);
            cm |= m << (8 * j);
        }
    }
    return cm;
}

struct Red {
    int v;  // min Delta over all bits (neighbour tracking)
    int c;  // min Delta over the candidate set
    int i;  // 2 * (lowest index attaining c) + x_index (INT_MAX if unknown / none)
};

// CTA-wide min reduction (three keys); all threads get the result.  Lowest
// index wins ties (reading C5).  Alternating slots -> one barrier per call.
template <bool kMulti>
__device__ __forceinline__ Red block_reduce(Red r, Red (*sred)[32], int &rb, int lane, int warp, int nw)
{
    Red w;
    w.v = __reduce_min_sync(kFull, r.v);
    w.c = __reduce_min_sync(kFull, r.c);
    w.i = __reduce_min_sync(kFull, r.c == w.c ? r.i : INT_MAX);
    if (!kMulti) {
        __syncwarp();  // orders lane 0's shared-memory bookkeeping before the other lanes read it
        return w;
    }
    Red *buf = sred[rb & 1];
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

template <bool kMulti>
__device__ __forceinline__ bool block_any(bool p)
{
    if (!kMulti) return __any_sync(kFull, p);
    return __syncthreads_or(p) != 0;
}

// Register pressure: in the 1024-thread kernel, slots 24..31 (byte-group 3)
// live in shared memory between uses ([2][nt] int4, conflict-free).  Volatile
// PTX so the compiler cannot forward the stored values and keep them live.
__device__ __forceinline__ void hi_load(int (&g)[32], const int4 *sgh, int t, int nt)
{
    asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(g[24]), "=r"(g[25]), "=r"(g[26]), "=r"(g[27])
                 : "r"(smem_u32(sgh + t)));
    asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(g[28]), "=r"(g[29]), "=r"(g[30]), "=r"(g[31])
                 : "r"(smem_u32(sgh + nt + t)));
}

__device__ __forceinline__ void hi_store(const int (&g)[32], int4 *sgh, int t, int nt)
{
    asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(smem_u32(sgh + t)), "r"(g[24]), "r"(g[25]),
                 "r"(g[26]), "r"(g[27])
                 : "memory");
    asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(smem_u32(sgh + nt + t)), "r"(g[28]), "r"(g[29]),
                 "r"(g[30]), "r"(g[31])
                 : "memory");
}

// Lowest-index argmin over the slots in `cm`; ci2 = 2*index + x (INT_MAX if none).
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

// 2*index + x of the lowest slot in `cm` whose Delta equals v (INT_MAX if none).
__device__ __forceinline__ int lowest_equal(const int (&g)[32], uint32_t xm, uint32_t cm, int v, int t, int nt)
{
    int r = INT_MAX;
#pragma unroll
    for (int s = 0; s < 32; ++s) {
        const bool hit = ((cm >> s) & 1u) && readout(g[s], xm, s) == v;
        if (hit && r == INT_MAX) r = 2 * slot_index(t, nt, s) + (int)((xm >> s) & 1u);
    }
    return r;
}

// Byte-group j (0..3) of bit i: i >> 3 = t + nt*j with t < nt (no division).
__device__ __forceinline__ int group_of(int i, int nt)
{
    const int beta = i >> 3;
    return (beta >= nt) + (beta >= 2 * nt) + (beta >= 3 * nt);
}

// Row update for one flip: g += c * W_k* over the 32 slots (Eq.(16), field
// form), then, unless kMode == kUpdate, the n neighbour deltas (Eq.(5)):
// min over all bits (vmin) and, kMode == kStraight, over the mismatches (cmin).
enum { kUpdate = 0, kMin = 1, kStraight = 2 };
template <int kMode, bool kHi>
__device__ __forceinline__ void process_row(int (&g)[32], uint32_t xm, uint32_t mism, const uint4 *row4,
                                            uint64_t *bars, uint32_t par, int c, int t, int nt, int &vmin,
                                            int &cmin, int4 *sgh)
{
    vmin = INT_MAX;
    cmin = INT_MAX;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        if (kHi && j == 3) hi_load(g, sgh, t, nt);
        mbar_wait(&bars[j], par);
        const uint4 w4 = row4[t + nt * j];
        const uint32_t wv[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int s0 = 8 * j + 2 * q;
            g[s0] += c * sext16(wv[q]);
            g[s0 + 1] += c * (((int)wv[q]) >> 16);
            if (kMode != kUpdate) {
                const int d0 = readout(g[s0], xm, s0);
                const int d1 = readout(g[s0 + 1], xm, s0 + 1);
                vmin = min(vmin, min(d0, d1));
                if (kMode == kStraight) {
                    const int m0 = ((mism >> s0) & 1u) ? d0 : INT_MAX;
                    const int m1 = ((mism >> (s0 + 1)) & 1u) ? d1 : INT_MAX;
                    cmin = min(cmin, min(m0, m1));
                }
            }
        }
        if (kHi && j == 3) hi_store(g, sgh, t, nt);
    }
}

// Smem bookkeeping of a CTA (after the two row buffers).
struct RoundSmem {
    uint64_t bar[2][4];   // [row buffer][chunk]
    Red red[2][32];
    int sel[2][4];        // window warp -> all: next (k, Delta_k, x_k, exact_next), by flip parity
    int thr[2];           // improvement threshold min(E_B - E(X'), ...) clamped to int32, by flip parity
    long long E, EB, LB;  // E(X), E_B, lower bound on min_i Delta_i(X): thread 0 only
    uint64_t hash;        // thread 0 only
    long long nflip, nstraight;
};
struct WindowSmem {       // published Delta / x of the next window, by flip parity
    int d[2][kWinMax];
    uint8_t x[2][kWinMax];
};

__device__ __forceinline__ void issue_row(const RoundArgs &A, int k, unsigned char *buf, uint64_t *bars, int nt)
{
    const uint32_t chunk = 16u * (uint32_t)nt;
    const char *src = reinterpret_cast<const char *>(A.Wz) + (size_t)k * (size_t)A.n_pad * 2;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        mbar_arrive_expect_tx(&bars[j], chunk);
        bulk_g2s(buf + (size_t)chunk * j, src + (size_t)chunk * j, chunk, &bars[j]);
    }
}

// Owners of the bits of window {(a2 + r) mod n : r < l} publish Delta and x.
__device__ __forceinline__ void publish_window(int (&g)[32], uint32_t xm, int a2, int l, int n, int t, int nt,
                                               int *wd, uint8_t *wx, const int4 *sgh)
{
    // window bytes: [b0, b1] and, when the window wraps (reading C6), [0, b2]
    const int end = a2 + l;
    const int b0 = a2 >> 3;
    const int b1 = (min(end, n) - 1) >> 3;
    const int b2 = end > n ? ((end - n - 1) >> 3) : -1;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const int beta = t + nt * j;
        if ((unsigned)(beta - b0) <= (unsigned)(b1 - b0) || beta <= b2) {
            if (j == 3 && sgh) hi_load(g, sgh, t, nt);
            const int base = 8 * beta;
#pragma unroll
            for (int e = 0; e < 8; ++e) {
                const int i = base + e;
                int r = i - a2;
                if (r < 0) r += n;
                if (i < n && r < l) {
                    wd[r] = readout(g[8 * j + e], xm, 8 * j + e);
                    wx[r] = (uint8_t)((xm >> (8 * j + e)) & 1u);
                }
            }
        }
    }
}

template <bool kMulti, int kNT>
__global__ void __launch_bounds__(kMulti ? 1024 : 32, kMulti ? 1 : 32) round_kernel(const RoundArgs A)
{
    extern __shared__ __align__(128) unsigned char smem[];
    const int nt = kNT ? kNT : (kMulti ? A.nt : 32);  // compile-time for the common sizes
    const int n = A.n;
    const int t = threadIdx.x;
    const int lane = t & 31, warp = t >> 5, nw = nt >> 5;
    const int sid = blockIdx.x;
    const size_t rowb = (size_t)64 * nt;  // bytes of one padded row

    unsigned char *rowbuf = smem;  // [2][rowb]
    RoundSmem *sm = reinterpret_cast<RoundSmem *>(smem + 2 * rowb);
    uint32_t *stm = reinterpret_cast<uint32_t *>(smem + 2 * rowb + sizeof(RoundSmem));  // [nt] target bits
    uint32_t *sbm = stm + nt;                                                          // [nt] best bits
    WindowSmem *win = reinterpret_cast<WindowSmem *>(sbm + nt);                         // kMulti only
    int4 *sgh = reinterpret_cast<int4 *>((reinterpret_cast<uintptr_t>(win + 1) + 15) & ~uintptr_t(15));  // [2][nt]

    if (t == 0) {
#pragma unroll
        for (int b = 0; b < 2; ++b)
#pragma unroll
            for (int j = 0; j < 4; ++j) mbar_init(&sm->bar[b][j], 1);
        fence_mbar_init();
        sm->hash = A.hash[sid];
        sm->nflip = 0;
        sm->nstraight = 0;
        sm->E = A.E[sid];
        sm->EB = sm->E;  // Step 3, reading C4: E_B = E(C) (Alg. 5) ...
        // Lower bound on min_i Delta_i(X) (lazy neighbour tracking, prefetch
        // path): after flipping k, min_i Delta_i(X') >= min(LB - 2*rowmax_k,
        // -Delta_k(X)) (Eq.(16), Eq.(6)); if E(X') + min(0, LB) >= E_B no
        // neighbour of X' can improve B and the n readouts may be skipped
        // without changing any result.  Tightened to the exact minimum after
        // every CTA reduction.
        sm->LB = INT64_MIN / 4;
    }

    // ---- load the search state (registers for the whole round)
    int g[32];
    {
        const int32_t *gs = A.g + (size_t)sid * 32 * nt;
#pragma unroll
        for (int s = 0; s < 32; ++s) g[s] = gs[(size_t)s * nt + t];
        if (kMulti) hi_store(g, sgh, t, nt);
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
        sbm[t] = xm;  // ... and B = C
    }
    int a = A.a[sid];
    const int l = A.l[sid];
    const bool pre = kMulti && l <= kWinMax;
    int left = (int)A.L;
    int rb = 0;
    if (kMulti) __syncthreads();
    else __syncwarp();

    // ---- first selection of the round
    bool straight = block_any<kMulti>(xm != stm[t]);
    int k, dk, xk;
    {
        int cv, ci2;
        const uint32_t cm = straight ? (xm ^ stm[t]) : window_mask(a, l, n, t, nt);
        if (kMulti) hi_load(g, sgh, t, nt);
        candidates(g, xm, cm, t, nt, cv, ci2);
        if (pre && !straight) {
            int a2 = a + l;
            if (a2 >= n) a2 -= n;
            publish_window(g, xm, a2, l, n, t, nt, win->d[0], win->x[0], sgh);
        }
        const Red r = block_reduce<kMulti>(Red{INT_MAX, cv, ci2}, sm->red, rb, lane, warp, nw);
        k = r.i >> 1;
        xk = r.i & 1;
        dk = r.c;
    }
    bool exact = true;  // compute the n neighbour deltas of this flip exactly
    int rk = 0;         // thread 0: rowmax of the row being flipped
    if (t == 0) {
        rk = __ldg(A.rowmax + k);
        issue_row(A, k, rowbuf, sm->bar[0], nt);
    }

    for (int f = 0;; ++f) {
        const int b = f & 1;
        const uint32_t par = (uint32_t)(f >> 1) & 1u;
        unsigned char *row = rowbuf + rowb * b;

        // ---- window-first selection of the next flip (warp 0), prefetch its row
        int rk_next = 0;
        if (pre && !straight && left > 1 && warp == 0) {
            int a1 = a + l;
            if (a1 >= n) a1 -= n;
            {
                // wait for the chunks of row k_f that hold the window's bits
                const int end = a1 + l - 1;
                const int c0 = group_of(a1, nt);
                const int c1 = group_of(min(end, n - 1), nt);
                for (int cc = c0; cc <= c1; ++cc) mbar_wait(&sm->bar[b][cc], par);
                if (end >= n) {
                    const int c2 = group_of(end - n, nt);
                    for (int cc = 0; cc <= c2; ++cc) mbar_wait(&sm->bar[b][cc], par);
                }
            }
            const int *wd = win->d[b];
            const uint8_t *wx = win->x[b];
            const short *rw = reinterpret_cast<const short *>(row);
            int bv = INT_MAX, bi = INT_MAX, bx = 0;
            // l <= kWinMax = 8 * 32: a lane's loads are issued in two batches of four
#pragma unroll
            for (int h = 0; h < kWinMax / 128; ++h) {
                int dd[4], ww[4], xx[4], ii[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int r = lane + 32 * (4 * h + q);
                    int i = a1 + r;
                    if (i >= n) i -= n;
                    ii[q] = i;
                    dd[q] = 0;
                    xx[q] = 0;
                    ww[q] = 0;
                    if (r < l) {
                        dd[q] = wd[r];
                        xx[q] = wx[r];
                        ww[q] = rw[i];
                    }
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    if (lane + 32 * (4 * h + q) < l) {
                        const int i = ii[q];
                        int d = dd[q];
                        int xn = xx[q];
                        if (i == k) {
                            d = -d;  // Eq.(6), k = i
                            xn ^= 1;
                        } else {
                            d += (xx[q] == xk) ? 2 * ww[q] : -2 * ww[q];  // Eq.(16)
                        }
                        if (d < bv || (d == bv && i < bi)) {
                            bv = d;
                            bi = i;
                            bx = xn;
                        }
                    }
                }
            }
            const int mv = __reduce_min_sync(kFull, bv);
            const int mi = __reduce_min_sync(kFull, bv == mv ? 2 * bi + bx : INT_MAX);
            if (lane == 0) {
                issue_row(A, mi >> 1, rowbuf + rowb * (b ^ 1), sm->bar[b ^ 1], nt);
                sm->sel[b][0] = mi >> 1;
                sm->sel[b][1] = mv;
                sm->sel[b][2] = mi & 1;
                rk_next = __ldg(A.rowmax + (mi >> 1));  // consumed after the row update
            }
        }

        // ---- flip k (Alg. 4 lines P:L328-336 / Alg. 5 lines P:L371-376)
        const int c = xk ? -2 : 2;  // 2 phi(x_k), pre-flip bit (Eq.(16))
        {
            const int j = group_of(k, nt);
            if (t == (k >> 3) - nt * j) xm ^= 1u << (8 * j + (k & 7));  // x_k <- 1 - x_k
        }
        int vmin, cmin;
        const uint4 *row4 = reinterpret_cast<const uint4 *>(row);
        uint32_t mism = 0;
        if (straight) {
            mism = xm ^ stm[t];
            process_row<kStraight, kMulti>(g, xm, mism, row4, sm->bar[b], par, c, t, nt, vmin, cmin, sgh);
        } else {
            if (exact) process_row<kMin, kMulti>(g, xm, 0u, row4, sm->bar[b], par, c, t, nt, vmin, cmin, sgh);
            else process_row<kUpdate, kMulti>(g, xm, 0u, row4, sm->bar[b], par, c, t, nt, vmin, cmin, sgh);
            a += l;  // offset <- (a + l) mod n
            if (a >= n) a -= n;
        }
        int ci2 = INT_MAX;
        if (!straight) {
            if (pre) {
                int a2 = a + l;
                if (a2 >= n) a2 -= n;
                publish_window(g, xm, a2, l, n, t, nt, win->d[b ^ 1], win->x[b ^ 1], sgh);
            } else {
                const uint32_t cm = window_mask(a, l, n, t, nt);
                if (__any_sync(kFull, cm != 0u)) {
                    if (kMulti) hi_load(g, sgh, t, nt);
                    candidates(g, xm, cm, t, nt, cmin, ci2);
                }
            }
        }
        // ---- thread 0: E(X') = E(X) + d_k, the bound LB, the improvement
        // threshold, and (prefetch path) whether the next flip must be exact
        if (t == 0) {
            sm->hash = (sm->hash ^ (uint64_t)(uint32_t)k) * kFnvPrime;
            sm->nflip += 1;
            if (straight) sm->nstraight += 1;
            const long long E1 = sm->E + dk;
            const long long LB1 = min(sm->LB - 2 * (long long)rk, -(long long)dk);
            const long long EB = sm->EB;
            sm->E = E1;
            sm->LB = LB1;
            // cand = E(X') + min(0, m) < E_B  <=>  min(0, m) < E_B - E(X')   (<= 2^31 - 32768
            // because E_B <= E(X); clamped below at INT_MIN, where it can never hold)
            sm->thr[b] = (int)max(EB - E1, (long long)INT_MIN);
            if (pre && !straight && left > 1) {
                // E_B may still drop in this flip: the current (larger) E_B only makes
                // the test more conservative
                const int dk1 = sm->sel[b][1];
                const long long LB2 = min(LB1 - 2 * (long long)rk_next, -(long long)dk1);
                sm->sel[b][3] = (E1 + dk1 + min(LB2, 0LL) < EB) ? 1 : 0;
            }
        }
        Red r1;
        if (exact) {
            r1 = block_reduce<kMulti>(Red{vmin, cmin, ci2}, sm->red, rb, lane, warp, nw);
        } else {
            __syncthreads();  // row buffer b free; sel[b], thr[b] and the window published
            r1 = Red{INT_MAX, INT_MAX, INT_MAX};
        }

        // ---- neighbour tracking (reading C2) and, straight phase, the argmin index
        const bool improve = exact && min(r1.v, 0) < sm->thr[b];  // uniform
        if (t == 0 && exact) {
            sm->LB = r1.v;
            if (improve) sm->EB = sm->E + min(r1.v, 0);
        }
        const bool sidx = straight && r1.c != INT_MAX;
        if (improve || sidx) {
            int it = INT_MAX, is = INT_MAX;
            if (kMulti) hi_load(g, sgh, t, nt);
            if (improve && r1.v < 0 && vmin == r1.v) it = lowest_equal(g, xm, 0xffffffffu, r1.v, t, nt);
            if (sidx && cmin == r1.c) is = lowest_equal(g, xm, mism, r1.c, t, nt);
            const Red r2 = block_reduce<kMulti>(Red{it, is, is}, sm->red, rb, lane, warp, nw);
            if (improve) {
                uint32_t bm = xm;
                if (r1.v < 0) {
                    const int istar = r2.v >> 1;
                    const int j = group_of(istar, nt);
                    if (t == (istar >> 3) - nt * j) bm ^= 1u << (8 * j + (istar & 7));
                }
                sbm[t] = bm;
            }
            if (sidx) {
                k = r2.c >> 1;
                xk = r2.c & 1;
                dk = r1.c;
            }
        }

        // ---- next flip
        if (!straight) {
            if (--left <= 0) break;
            if (pre) {
                k = sm->sel[b][0];
                dk = sm->sel[b][1];
                xk = sm->sel[b][2];
                exact = sm->sel[b][3] != 0;
                rk = rk_next;
                continue;  // row already in flight
            }
            k = r1.i >> 1;
            xk = r1.i & 1;
            dk = r1.c;
        } else if (!sidx) {
            // X = T: the straight search is over; local search from T (Step 4b)
            straight = false;
            if (left <= 0) break;
            int cv, cj;
            if (kMulti) hi_load(g, sgh, t, nt);
            candidates(g, xm, window_mask(a, l, n, t, nt), t, nt, cv, cj);
            if (pre) {
                int a2 = a + l;
                if (a2 >= n) a2 -= n;
                publish_window(g, xm, a2, l, n, t, nt, win->d[b ^ 1], win->x[b ^ 1], sgh);
            }
            const Red r = block_reduce<kMulti>(Red{INT_MAX, cv, cj}, sm->red, rb, lane, warp, nw);
            k = r.i >> 1;
            xk = r.i & 1;
            dk = r.c;
            exact = true;
        }
        if (t == 0) {
            rk = __ldg(A.rowmax + k);
            issue_row(A, k, rowbuf + rowb * (b ^ 1), sm->bar[b ^ 1], nt);
        }
    }

    // ---- Step 5: store (B, E_B) and the state C' for the next round
    if (kMulti) __syncthreads();
    else __syncwarp();
    {
        if (kMulti) hi_load(g, sgh, t, nt);
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
            A.E[sid] = sm->E;
            A.EB[sid] = sm->EB;
            A.a[sid] = a;
            A.hash[sid] = sm->hash;
            A.flips[sid] += sm->nflip;
            A.sflips[sid] += sm->nstraight;
        }
    }
}

}  // namespace

size_t round_smem_bytes(int32_t nt)
{
    size_t s = 2 * (size_t)64 * nt + sizeof(RoundSmem) + 2 * sizeof(uint32_t) * (size_t)nt;
    if (nt > 32) s += sizeof(WindowSmem) + 16 + 2 * sizeof(int4) * (size_t)nt;
    return s;
}

int launch_round(const RoundArgs &a, cudaStream_t st)
{
    const size_t smem = round_smem_bytes(a.nt);
    if (a.nt == 32) {
        auto k = round_kernel<false, 32>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k<<<a.S, 32, smem, st>>>(a);
    } else if (a.nt == 1024) {
        auto k = round_kernel<true, 1024>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k<<<a.S, 1024, smem, st>>>(a);
    } else {
        auto k = round_kernel<true, 0>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k<<<a.S, a.nt, smem, st>>>(a);
    }
    return (int)cudaGetLastError();
}

}  // namespace absb
