// The ABS search kernel for sm_100a: one CTA runs one round (device Steps
// 2-5) of one search.  Citations: /root/reference/PAPER.md line
// numbers (P:Lnnn); readings Cnn are listed in DESIGN.md.
//
// Layout.  A search of n <= n_pad = P*NT bits is held by NT threads, P bits
// each (the paper's "p bits per thread"; P = 64 and NT = 512 at
// n = 32k): thread t owns the byte-groups beta = t + NT*j (j < P/8), i.e. bits
// 8*beta .. 8*beta+7, in register slots s = 8j + e.  Per bit it holds the field
//     g_i = 2 sum_{j != i} W_ij x_j + W_ii,   Delta_i = phi(x_i) g_i   (Eq.(13)),
// so the flip update Eq.(16) is a sign-free row add g_i += 2 phi(x_k) W_ik
// (W is stored with a zero diagonal, so g_k is untouched); x is a P-bit mask.
//
// Memory.  Row k of W (2*n_pad bytes) is copied into shared memory by
// cp.async.bulk (TMA, SASS UBLKCP) in P/8 chunks, one per byte-group, each
// completing its own mbarrier.  Two row buffers: while flip f consumes row
// k_f, row k_{f+1} is already in flight.
//
// Window-first prefetch (local phase, l <= kWinMax).  The next flip k_{f+1}
// depends only on the window W_{f+1} = {(a_{f+1} + r) mod n : r < l}
// (Fig. 2).  During flip f-1 the owners of W_{f+1}'s bits publish
// Delta_i(X_f) and x_i(X_f) to shared memory; at the start of flip f the last warp
// applies row k_f to those l values only, takes the lowest-index argmin and
// issues the TMA for row k_{f+1} at once: the row fetch overlaps the processing
// of row k_f instead of following it.
//
// Lazy neighbour tracking.  Every flip evaluates all n neighbours (Eq.(5)) in
// the paper's accounting; B only changes when E(X') + min_i Delta_i(X') < E_B.
// A rigorous lower bound LB on min_i Delta_i is carried along (each flip moves
// every Delta_i, i != k, by at most 2*max_i|W_ik|, and Delta_k becomes
// -Delta_k), and a flip whose bound already rules out an improvement skips the
// n readouts; the result (B, E_B) is identical by construction.
#include <algorithm>
#include <climits>
#include <cstdint>

#include "abs_round_common.cuh"

namespace absb {
namespace {

constexpr uint64_t kFnvPrime = 0x100000001b3ull;
constexpr unsigned kFull = 0xffffffffu;
constexpr int kWinMax = 256;
// bulk copies (and mbarriers) per W row: 1, or 2 half rows (the controller starts the
// window-first selection when the half holding the window lands).  Measured: 2 for the
// n = 32768 variant (+1.7%), 1 elsewhere (2 cost TSP n = 10,000 8%).
#ifndef ABS_ROW_CHUNKS_32K
#define ABS_ROW_CHUNKS_32K 2
#endif
#ifndef ABS_ROW_CHUNKS
#define ABS_ROW_CHUNKS 1
#endif


struct Red {
    int v;  // min Delta over all bits (neighbour tracking)
    int c;  // min Delta over the candidate set
    int i;  // 2 * (lowest index attaining c) + x_index (INT_MAX if unknown / none)
};

// Shared-memory bookkeeping of a CTA (at offset 0; kB = the SA batch cap).
template <int kB>
struct RoundSmemT {
    uint64_t bar[2][2];   // [row buffer][half row]
    Red red[2][32];
    int4 sel[2];          // window warp -> all: next (k, Delta_k, x_k, exact_next), by flip parity
    int thr[2];           // improvement threshold E_B - E(X') clamped to int32, by flip parity
    long long E, EB, LB;  // E(X), E_B, lower bound on min_i Delta_i(X): thread 0 only
    unsigned long long hash;
    long long nflip, nstraight;
    unsigned long long sa_ctr;  // SA: proposals drawn (Philox counter); thread 0 writes
    int sa_tau;                 // SA: this search's temperature
    unsigned long long sa_inv;  // SA: sa_inv2tau(sa_tau)
    UDiv sa_dn, sa_dt;          // SA: exact division by n (bit draw) and by tau (exponent), per round
    int sa_pk[64];              // SA proposal cache: bit and draw of proposal pcb + i (sa_next)
    uint32_t sa_po[64];
    int sa_d[2][kB], sa_x[2][kB];  // SA: Delta_k / x_k of a batch of proposals, by batch parity
    int sa_k[2][kB];               // SA: the batch's proposed bits ...
    uint32_t sa_o[2][kB];          // ... and their acceptance draws
    int4 sa_e;                  // SA early decision of this flip: (k, Delta_k, x_k, proposals consumed)
    int sa_ex[2];               // SA: lazy test of the early-accepted next flip (1: exact), by flip parity
    long long sa_lz[2][3];      // SA: E(X'), E_B, bound LB after this flip's tracking, by flip parity
    int snext[2];               // straight phase: 2k + x of the next flip, from its owner thread
#ifdef ABS_TIMING
    long long tacc[32][24];  // [warp][local 0-6 | straight 8-14 | selection sub-phases 16-20]
#endif
};
struct WindowSmem {  // published Delta / x of the next window, by flip parity
    int d[2][kWinMax];
    uint8_t x[2][kWinMax];
};

template <int kP, int kMaxT, int kNT, bool kSA>
struct Round {
    static_assert(kMaxT > 32, "searches of one warp (n <= 2048) run WarpRound (abs_round_warp.cu)");
    static constexpr int G = kP / 8;  // byte-groups per thread
    static constexpr int kRowChunks = kNT == 512 ? ABS_ROW_CHUNKS_32K : ABS_ROW_CHUNKS;
    static constexpr int kSaBatch = kSaBatchMulti;
    using RoundSmem = RoundSmemT<kSaBatch>;
    static constexpr bool kSaEarly = kSA;  // SA early decision (run())
    using M = typename MaskOf<kP>::T;

    // ---------------------------------------------------------------- small helpers
    // Delta_i = phi(x_i) * g_i (Eq.(3): phi(0) = +1, phi(1) = -1)
    static __device__ __forceinline__ int readout(int g, M xm, int s)
    {
        return ((xm >> s) & 1u) ? -g : g;
    }
    static __device__ __forceinline__ uint32_t bit(M xm, int s) { return (uint32_t)((xm >> s) & 1u); }
    static __device__ __forceinline__ int slot_index(int t, int nt, int s) { return 8 * (t + nt * (s >> 3)) + (s & 7); }
    // byte-group j of bit i (i >> 3 = t + nt*j, t < nt)
    static __device__ __forceinline__ int group_of(int i, int nt)
    {
        const int beta = i >> 3;
        if constexpr (kNT != 0) return beta / kNT;
        int j = 0;
#pragma unroll
        for (int m = 1; m < G; ++m) j += (beta >= m * nt);
        return j;
    }
    // g[s] for a slot s uniform across the active threads (a binary tree over compile-time slots)
    template <int LO, int HI>
    static __device__ __forceinline__ int get_slot(const int (&g)[kP], int s)
    {
        if constexpr (HI - LO == 1) {
            return g[LO];
        } else {
            constexpr int MID = (LO + HI) / 2;
            return s < MID ? get_slot<LO, MID>(g, s) : get_slot<MID, HI>(g, s);
        }
    }
    static __device__ __forceinline__ int sext16(uint32_t w) { return (int)(short)(w & 0xffffu); }

    // bits [lo, hi) of the byte-group starting at element `base`, as an 8-bit mask
    static __device__ __forceinline__ uint32_t range8(int base, int lo, int hi)
    {
        const int e0 = max(lo - base, 0);
        const int e1 = min(hi - base, 8);
        if (e1 <= e0) return 0u;
        return ((1u << e1) - 1u) & ~((1u << e0) - 1u);
    }

    // Slots of thread t inside the window {(a + r) mod n : r < l} (Fig. 2).
    static __device__ __forceinline__ M window_mask(int a, int l, int n, int t, int nt)
    {
        const int end = a + l;  // exclusive; > n when the window wraps (reading C6)
        const int hi1 = min(end, n);
        const int hi2 = end - n;
        M cm = 0;
#pragma unroll
        for (int j = 0; j < G; ++j) {
            const int base = 8 * (t + nt * j);
            const bool h1 = (base + 8 > a) && (base < hi1);
            const bool h2 = base < hi2;
            if (h1 | h2) {
                uint32_t m = 0;
                if (h1) m |= range8(base, a, hi1);
                if (h2) m |= range8(base, 0, hi2);
                cm |= (M)m << (8 * j);
            }
        }
        return cm;
    }

    // Lowest-index argmin over the slots in `cm`; ci2 = 2*index + x (INT_MAX if none).
    static __device__ __forceinline__ void candidates(const int (&g)[kP], M xm, M cm, int t, int nt, int &cv,
                                                      int &ci2)
    {
        cv = INT_MAX;
        int cs = -1;
#pragma unroll
        for (int s = 0; s < kP; ++s) {
            const int d = readout(g[s], xm, s);
            if (bit(cm, s) && d < cv) {
                cv = d;
                cs = s;
            }
        }
        ci2 = cs < 0 ? INT_MAX : 2 * slot_index(t, nt, cs) + (int)bit(xm, cs);
    }

    // Window argmin over {(a + r) mod n : r < l} (Fig. 2) in the mask form
    // (measured faster than a byte-group scan at n = 32k).
    static __device__ __forceinline__ void window_candidates(const int (&g)[kP], M xm, int a, int l, int n, int t,
                                                             int nt, int &cv, int &ci2)
    {
        const M cm = window_mask(a, l, n, t, nt);
        cv = INT_MAX;
        ci2 = INT_MAX;
        if (__any_sync(kFull, cm != 0)) candidates(g, xm, cm, t, nt, cv, ci2);
    }

    // 2*index + x of the lowest slot in `cm` whose Delta equals v (INT_MAX if none).
    static __device__ __forceinline__ int lowest_equal(const int (&g)[kP], M xm, M cm, int v, int t, int nt)
    {
        int r = INT_MAX;
#pragma unroll
        for (int s = 0; s < kP; ++s) {
            const bool hit = bit(cm, s) && readout(g[s], xm, s) == v;
            if (hit && r == INT_MAX) r = 2 * slot_index(t, nt, s) + (int)bit(xm, s);
        }
        return r;
    }

    // CTA-wide min reduction (three keys); all threads get the result.  Lowest
    // index wins ties (reading C5).  Alternating slots -> one barrier per call.
    static __device__ __forceinline__ Red block_reduce(Red r, Red (*sred)[32], int &rb, int lane, int warp, int nw)
    {
        Red w;
        w.v = __reduce_min_sync(kFull, r.v);
        w.c = __reduce_min_sync(kFull, r.c);
        w.i = __reduce_min_sync(kFull, r.c == w.c ? r.i : INT_MAX);
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

    static __device__ __forceinline__ bool block_any(bool p) { return __syncthreads_or(p) != 0; }

    static __device__ __forceinline__ void sync() { __syncthreads(); }

    enum { kUpdate = 0, kMin = 1, kStraight = 2 };

    // Row update for one flip: g += c * W_k* over the P slots (Eq.(16), field
    // form), then, unless kMode == kUpdate, the n neighbour deltas (Eq.(5)):
    // min over all bits (vmin) and, kMode == kStraight, over the mismatches (cmin);
    // cj: the first of this thread's byte-groups holding cmin.
    template <int kMode>
    static __device__ __forceinline__ void process_row(int (&g)[kP], M xm, M mism, const uint4 *row4, uint64_t *bars,
                                                       uint32_t par, int c, int t, int nt, int &vmin, int &cmin,
                                                       int &cj)
    {
        const int cb = c & 0xff;  // c = +-2 as a signed byte
        vmin = INT_MAX;
        int vmin2 = INT_MAX;  // odd groups: two independent min chains (shorter dependency chain)
        cmin = INT_MAX;
        cj = 0;  // kStraight: first byte-group holding cmin (lowest index, reading C5)
#pragma unroll
        for (int j = 0; j < G; ++j) {
            int gmin = INT_MAX;
            if (kRowChunks == 2 ? (j % (G / 2) == 0) : (j == 0)) mbar_wait(&bars[kRowChunks == 2 ? j / (G / 2) : 0], par);
            const uint4 w4 = row4[t + nt * j];
            const uint32_t wv[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int s0 = 8 * j + 2 * q;
                // g += c * W_ik for the two int16 of one word: one 2-way int16 x int8
                // dot product each (IDP.2A on the FMA pipe; no sign-extension on the ALU
                // pipe), with c in byte 0 (low half) or byte 1 (high half) of cb
                g[s0] = __dp2a_lo((int)wv[q], cb, g[s0]);
                g[s0 + 1] = __dp2a_lo((int)wv[q], cb << 8, g[s0 + 1]);
                if (kMode != kUpdate) {
                    const int d0 = readout(g[s0], xm, s0);
                    const int d1 = readout(g[s0 + 1], xm, s0 + 1);
                    if (j & 1) vmin2 = min(vmin2, min(d0, d1));
                    else vmin = min(vmin, min(d0, d1));
                    if (kMode == kStraight) {
                        const int m0 = bit(mism, s0) ? d0 : INT_MAX;
                        const int m1 = bit(mism, s0 + 1) ? d1 : INT_MAX;
                        gmin = min(gmin, min(m0, m1));
                    }
                }
            }
            if (kMode == kStraight && gmin < cmin) {
                cmin = gmin;
                cj = j;
            }
        }
        vmin = min(vmin, vmin2);
    }

    // 2*index + x of the lowest mismatch slot of byte-group jsel whose Delta
    // equals v (INT_MAX if none): the straight phase's argmin index (Alg. 5),
    // scanning 8 slots instead of P.
    static __device__ __forceinline__ int lowest_equal_group(const int (&g)[kP], M xm, M cm, int v, int jsel, int t,
                                                             int nt)
    {
        int r = INT_MAX;
#pragma unroll
        for (int j = 0; j < G; ++j) {
            if (j != jsel) continue;
#pragma unroll
            for (int e = 7; e >= 0; --e) {
                const int s = 8 * j + e;
                if (bit(cm, s) && readout(g[s], xm, s) == v) r = 2 * slot_index(t, nt, s) + (int)bit(xm, s);
            }
        }
        return r;
    }

    static __device__ __forceinline__ void issue_row(const RoundArgs &A, int k, unsigned char *buf, uint64_t *bars,
                                                     int nt)
    {
        const uint32_t half = 8u * G * (uint32_t)nt;  // bytes of G/2 byte-groups = n_pad bytes
        // row stride 2 n_pad bytes; a compile-time constant when NT is (n = 32k: a shift)
        const size_t stride = kNT ? (size_t)2 * kP * kNT : (size_t)A.n_pad * 2;
        const char *src = reinterpret_cast<const char *>(A.Wz) + (size_t)k * stride;
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            if (kRowChunks == 1) {
                if (h == 0) {
                    mbar_arrive_expect_tx(&bars[0], 2 * half);
                    bulk_g2s(buf, src, 2 * half, &bars[0]);
                }
            } else {
                mbar_arrive_expect_tx(&bars[h], half);
                bulk_g2s(buf + (size_t)half * h, src + (size_t)half * h, half, &bars[h]);
            }
        }
    }

    // Owners of the bits of window {(a2 + r) mod n : r < l} publish Delta and x.
    static __device__ __forceinline__ void publish_window(const int (&g)[kP], M xm, int a2, int l, int n, int t,
                                                          int nt, int *wd, uint8_t *wx)
    {
        // window bytes: [b0, b1] and, when the window wraps (reading C6), [0, b2]
        const int end = a2 + l;
        const int b0 = a2 >> 3;
        const int b1 = (min(end, n) - 1) >> 3;
        const int b2 = end > n ? ((end - n - 1) >> 3) : -1;
        if constexpr (kNT != 0 && (kNT & (kNT - 1)) == 0 && kNT > kWinMax / 8) {
            // window spans < kNT bytes: thread t holds at most one byte of [b0, b1]
            // (beta = b0 + ((t - b0) mod kNT)) and, if wrapped, byte t of [0, b2]
            const int dlt = (t - b0) & (kNT - 1);
            const int jw = dlt <= b1 - b0 ? (b0 + dlt) / kNT : -1;
            const int jz = t <= b2 ? 0 : -1;
            if (jw < 0 && jz < 0) return;
        }
#pragma unroll
        for (int j = 0; j < G; ++j) {
            const int beta = t + nt * j;
            if ((unsigned)(beta - b0) <= (unsigned)(b1 - b0) || beta <= b2) {
                const int base = 8 * beta;
#pragma unroll
                for (int e = 0; e < 8; ++e) {
                    const int i = base + e;
                    int r = i - a2;
                    if (r < 0) r += n;
                    if (i < n && r < l) {
                        wd[r] = readout(g[8 * j + e], xm, 8 * j + e);
                        wx[r] = (uint8_t)bit(xm, 8 * j + e);
                    }
                }
            }
        }
    }

    // SA policy (Alg. 1 + Eq.(7), reading E2): draw proposals until one is
    // accepted or the round's proposal budget `left` is spent.  Proposals are
    // evaluated in batches against the current state: lane q of every warp
    // draws proposal c + q (Philox), the owners of the proposed bits broadcast
    // Delta_k and x_k through shared memory (one barrier per batch), and lane q
    // decides proposal q.  The first accepted one is taken; the proposals after
    // it are discarded and drawn again after the flip, so the sequence of
    // decisions is exactly the one-at-a-time sequence (rejections do not change
    // the state).  The batch size bsz adapts to the acceptance rate (uniform
    // across the CTA): doubled after a batch without acceptance, halved when
    // the first proposal of a batch is accepted.  Returns false when nothing
    // was accepted.
    // The proposals of the accepted batch after the accepted one (lo_n of them,
    // from index lo_q of slot lo_s) are left in shared memory for the next
    // flip's early decision; cadd counts proposals that decision consumed.
    static __device__ __forceinline__ bool sa_next(const RoundArgs &A, RoundSmem *sm, const int (&g)[kP], M xm,
                                                   int sid, int n, int t, int nt, int &left, int &k, int &dk, int &xk,
                                                   int &bsz, int &cadd, int &lo_n, int &lo_s, int &lo_q, uint32_t &pcb)
    {
        lo_n = 0;
        if (left <= 0) {  // budget spent (by the early decision): only thread 0 touches sa_ctr
            if (t == 0) sm->sa_ctr += (unsigned long long)cadd;
            cadd = 0;
            return false;
        }
        // thread 0 wrote sa_ctr before the last barrier; the batch loop below runs at least
        // once, so its barrier orders every thread's read here before thread 0's write below
        unsigned long long c = sm->sa_ctr + (unsigned long long)cadd;
        cadd = 0;
        const uint64_t inv2tau = sm->sa_inv;
        const int lane = t & 31;
        bool acc = false;
        int sb = 0;  // batch slot parity (a barrier separates this call from the previous one)
        while (left > 0) {
            const int nb = min(left, bsz);
            // proposals are drawn 64 at a time into a shared cache (two warps, one Philox per
            // thread; proposals depend only on their counter), instead of by every warp per batch;
            // pcb (the cache's first counter, low 32 bits) is kept by every thread in a register
            if ((uint32_t)c - pcb + (uint32_t)nb > 64u) {
                if (t < 64) {
                    uint32_t o[4];
                    const unsigned long long cq = c + (unsigned long long)t;
                    philox4x32_10((uint32_t)cq, (uint32_t)(cq >> 32), (uint32_t)(A.sid0 + sid), kTagSA,
                                  (uint32_t)A.seed, (uint32_t)(A.seed >> 32), o);
                    sm->sa_pk[t] = (int)umod(o[0], sm->sa_dn);  // "randomly select a bit" (Alg. 1): o0 mod n
                    sm->sa_po[t] = o[1];
                }
                pcb = (uint32_t)c;
                sync();
            }
            const int off = (int)((uint32_t)c - pcb);
            int kq = 0;
            uint32_t o1 = 0;
            if (lane < nb) {
                kq = sm->sa_pk[off + lane];
                o1 = sm->sa_po[off + lane];
                if (t < 32) {
                    sm->sa_k[sb][lane] = kq;
                    sm->sa_o[sb][lane] = o1;
                }
            }
            // multi-warp: each warp walks only the proposals whose owner thread is one of
            // its lanes, about nb / warps of them instead of nb (random32k SA +6%, tsp100
            // +3%; one warp owns them all, and the ballot measured -2% on MaxCut there)
            unsigned mine;
            {
                const int own = lane < nb ? (kq >> 3) - nt * group_of(kq, nt) : -1;
                mine = __ballot_sync(kFull, lane < nb && (own >> 5) == (t >> 5));
            }
            while (mine) {
                const int q = __ffs(mine) - 1;
                mine &= mine - 1;
                const int kk = __shfl_sync(kFull, kq, q);
                const int j = group_of(kk, nt);
                if (t == (kk >> 3) - nt * j) {
                    const int e = kk & 7;
                    const int v = get_slot<0, kP>(g, 8 * j + e);  // uniform slot: a branch tree, not 64 selects
                    sm->sa_d[sb][q] = readout(v, xm, 8 * j + e);
                    sm->sa_x[sb][q] = (int)bit(xm, 8 * j + e);
                }
            }
            sync();
            int d = 0, x = 0;
            bool ok = false;
            if (lane < nb) {
                d = sm->sa_d[sb][lane];
                x = sm->sa_x[sb][lane];
                ok = sa_accept(d, sm->sa_dt, inv2tau, o1);  // Eq.(7)
            }
            const unsigned m = __ballot_sync(kFull, ok);
            if (m) {
                const int q = __ffs(m) - 1;  // the first accepted proposal
                if (q == 0) bsz = max(1, bsz >> 1);
                k = __shfl_sync(kFull, kq, q);
                dk = __shfl_sync(kFull, d, q);
                xk = __shfl_sync(kFull, x, q);
                left -= q + 1;
                c += (unsigned long long)(q + 1);
                lo_n = nb - q - 1;
                lo_s = sb;
                lo_q = q + 1;
                acc = true;
                break;
            }
            left -= nb;
            c += (unsigned long long)nb;
            sb ^= 1;
            bsz = min(2 * bsz, kSaBatch);
        }
        if (t == 0) sm->sa_ctr = c;
        return acc;
    }

    // Window-first selection of the next local flip by the controller warp (the last
    // warp): applies row k_f (buffer b) to the published Delta(X_f) of window
    // W_{f+1} = {(a + l + r) mod n : r < l}, takes the lowest-index argmin
    // (reading C5), issues the TMA of row k_{f+1} into buffer b ^ 1 and leaves
    // (k_{f+1}, Delta, x, 1) in sel[b].
    static __device__ __forceinline__ void window_first(const RoundArgs &A, RoundSmem *sm, const WindowSmem *win,
                                                        unsigned char *rowbuf, size_t rowb, int b, uint32_t par,
                                                        int a, int l, int n, int xk, int lane, int warp, int nt,
                                                        long long tc0)
    {
        (void)warp;
        (void)tc0;
        const unsigned char *row = rowbuf + rowb * b;
        int a1 = a + l;
        if (a1 >= n) a1 -= n;
        {
            // wait for the half rows of row k_f that hold the window's bits
            const int end = a1 + l - 1;
            const int h0 = group_of(a1, nt) / (G / 2);
            const int h1 = (end >= n) ? 1 : group_of(end, nt) / (G / 2);
            if (kRowChunks == 1) {
                mbar_wait(&sm->bar[b][0], par);
            } else {
                if (end >= n || h0 == 0) mbar_wait(&sm->bar[b][0], par);
                if (h1 == 1) mbar_wait(&sm->bar[b][1], par);
            }
        }
        ABS_T(const long long ts1 = clock64();)
        const int *wd = win->d[b];
        const uint8_t *wx = win->x[b];
        const short *rw = reinterpret_cast<const short *>(row);
        // key = (Delta_i(X_{f+1}) << 32) | (2i + x_i): its minimum is the
        // lowest-index argmin (reading C5) and carries x_i along
        long long best = LLONG_MAX;
        // l <= kWinMax = 8 * 32: a lane's loads are issued in batches of four;
        // batches wholly beyond l are skipped (warp-uniform)
#pragma unroll
        for (int h = 0; h < kWinMax / 128; ++h) {
            if (h > 0 && 128 * h >= l) break;
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
            // k_f is not in this window (windows are disjoint: l <= kWinMax <= n/8 here),
            // so every entry moves by Eq.(16); the four keys are reduced as a tree
            long long kq[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int d = dd[q] + ww[q] * (2 - 4 * (xx[q] ^ xk));  // Eq.(16)
                kq[q] = (lane + 32 * (4 * h + q) < l)
                            ? (long long)(((unsigned long long)(unsigned)d << 32) | (unsigned)(2 * ii[q] + xx[q]))
                            : LLONG_MAX;
            }
            best = min(best, min(min(kq[0], kq[1]), min(kq[2], kq[3])));
        }
        const int bv = (int)(best >> 32);
        ABS_T(const long long ts2 = clock64();)
        const int mv = __reduce_min_sync(kFull, bv);
        const int mi = __reduce_min_sync(kFull, bv == mv ? (int)(unsigned)best : INT_MAX);
        ABS_T(const long long ts3 = clock64();)
        // the warp is converged here: one elected lane issues (no per-lane loop
        // around the bulk copy's uniform operands)
        if (elect_one()) issue_row(A, mi >> 1, rowbuf + rowb * (b ^ 1), sm->bar[b ^ 1], nt);
        if (lane == 0) sm->sel[b] = make_int4(mi >> 1, mv, mi & 1, 1);
        ABS_T(if (lane == 0) {
            const long long ts4 = clock64();
            sm->tacc[warp][16] += ts1 - tc0;  // wait for row k_f's window half
            sm->tacc[warp][17] += ts2 - ts1;  // window arithmetic
            sm->tacc[warp][18] += ts3 - ts2;  // two warp reductions
            sm->tacc[warp][19] += ts4 - ts3;  // TMA issue + sel
            sm->tacc[warp][20] += 1;
        })
    }

    // The hot loop of the window policy at n > 2048: consecutive NON-exact local flips
    // with the window-first prefetch.  The general flip body of run() with the
    // straight, SA and exact-tracking branches compiled out, so each warp issues
    // little besides its row update (Eq.(16)).  Entered at the start of flip f with
    // row k_f in flight; returns at the start of the first flip that is exact or
    // has no local successor (left <= 1), in the state the general body expects.
    static __device__ __forceinline__ void fast_local(const RoundArgs &A, RoundSmem *sm, WindowSmem *win,
                                                      unsigned char *rowbuf, size_t rowb, int (&g)[kP], M &xm,
                                                      int &a, int l, int n, int t, int nt, int lane, int warp, int nw,
                                                      int ctl, int &left, int &k, int &dk, int &xk, bool &exact,
                                                      int &f, int fbase)
    {
        const long long wmax2 = 2 * (long long)A.wmax;
        while (!exact && left > 1) {
            const int b = (fbase + f) & 1;
            const uint32_t par = (uint32_t)((fbase + f) >> 1) & 1u;
            if (warp == nw - 1) window_first(A, sm, win, rowbuf, rowb, b, par, a, l, n, xk, lane, warp, nt, 0);
            const int c = xk ? -2 : 2;  // 2 phi(x_k), pre-flip bit (Eq.(16))
            {
                const int j = group_of(k, nt);
                if (t == (k >> 3) - nt * j) xm ^= (M)1 << (8 * j + (k & 7));  // x_k <- 1 - x_k
            }
            int vmin, cmin, cj;
            process_row<kUpdate>(g, xm, 0, reinterpret_cast<const uint4 *>(rowbuf + rowb * b), sm->bar[b], par, c, t,
                                 nt, vmin, cmin, cj);
            a += l;  // offset <- (a + l) mod n
            if (a >= n) a -= n;
            int a2 = a + l;
            if (a2 >= n) a2 -= n;
            publish_window(g, xm, a2, l, n, t, nt, win->d[b ^ 1], win->x[b ^ 1]);
            if (t == ctl) {  // E(X') = E(X) + d_k, the bound LB, lazy tracking of flip f+1
                sm->hash = (sm->hash ^ (uint64_t)(uint32_t)k) * kFnvPrime;
                sm->nflip += 1;
                const long long E1 = sm->E + dk;
                const long long LB1 = min(sm->LB - wmax2, -(long long)dk);
                sm->E = E1;
                sm->LB = LB1;
                const int dk1 = sm->sel[b].y;
                const long long LB2 = min(LB1 - wmax2, -(long long)dk1);
                sm->sel[b].w = (E1 + dk1 + min(LB2, 0LL) < sm->EB) ? 1 : 0;
            }
            __syncthreads();  // row buffer b free; sel[b] and the window published
            --left;
            const int4 sv = sm->sel[b];
            k = sv.x;
            dk = sv.y;
            xk = sv.z;
            exact = sv.w != 0;
            ++f;
        }
    }

    static __device__ __forceinline__ void init_barriers(unsigned char *smem)
    {
        RoundSmem *sm = reinterpret_cast<RoundSmem *>(smem);
        if (threadIdx.x == 0) {
#pragma unroll
            for (int b = 0; b < 2; ++b)
#pragma unroll
                for (int h = 0; h < 2; ++h) mbar_init(&sm->bar[b][h], 1);
            fence_mbar_init();
        }
        // made visible by the first barrier of run()
    }

    // ---------------------------------------------------------------- the round
    // One round of search `sid`: target bits from Ts; (B, E_B) go to the
    // pointers out(Bs, EBp) yields at the end of the round (evaluated late so
    // that no output address stays live across the flip loop).
    // fbase counts the rows this CTA has consumed before (row buffer and mbarrier
    // phase of flip f are those of use fbase + f); the barriers are initialised
    // once per launch by init_barriers().
    template <class Out>
    static __device__ __forceinline__ void run(const RoundArgs &A, unsigned char *smem, int sid, const uint8_t *Ts,
                                               const Out &out, int &fbase)
    {
        const int nt = kNT ? kNT : A.nt;
        const int n = A.n;
        const int t = threadIdx.x;
        const int lane = t & 31, warp = t >> 5, nw = nt >> 5;
        // the controller: lane 0 of the LAST warp, which the warp schedulers favour
        // (highest warp id first) -- its serial work is on every flip's critical path
        const int ctl = nt - 32;
        const size_t rowb = (size_t)2 * kP * nt;  // bytes of one padded row (2 * n_pad)

        RoundSmem *sm = reinterpret_cast<RoundSmem *>(smem);
        WindowSmem *win = reinterpret_cast<WindowSmem *>(smem + sizeof(RoundSmem));
        M *stm = reinterpret_cast<M *>(smem + sizeof(RoundSmem) + sizeof(WindowSmem));
        M *sbm = stm + nt;
        unsigned char *rowbuf =
            smem + ((sizeof(RoundSmem) + sizeof(WindowSmem) + 2 * sizeof(M) * nt + 127) & ~size_t(127));

        if (t == 0) {
            sm->hash = A.hash[sid];
            sm->nflip = 0;
            sm->nstraight = 0;
            sm->E = A.E[sid];
            sm->EB = sm->E;  // Step 3, reading C4: E_B = E(C) (Alg. 5) ...
            sm->LB = INT64_MIN / 4;
            sm->sa_ctr = A.policy == 1 ? A.sa_ctr[sid] : 0ull;
            sm->sa_tau = A.policy == 1 ? A.tau[sid] : 1;
            sm->sa_inv = sa_inv2tau(sm->sa_tau);
            sm->sa_dn = make_udiv((uint32_t)A.n);
            sm->sa_dt = make_udiv((uint32_t)sm->sa_tau);
        }

        // ---- the search state (registers for the whole round)
        int g[kP];
        {
            const int32_t *gs = A.g + (size_t)sid * kP * nt;
#pragma unroll
            for (int s = 0; s < kP; ++s) g[s] = gs[(size_t)s * nt + t];
        }
        M xm = 0;
        {
            const uint8_t *Xs = A.X + (size_t)sid * G * nt;
            M tm = 0;
#pragma unroll
            for (int j = 0; j < G; ++j) {
                xm |= (M)Xs[t + nt * j] << (8 * j);
                tm |= (M)Ts[t + nt * j] << (8 * j);  // Step 2: read target T
            }
            stm[t] = tm;
            sbm[t] = xm;  // ... and B = C
        }
        int a = A.a[sid];
        const int l = A.l[sid];
        constexpr bool sa = kSA;  // ABS_POLICY_SA: a separate kernel instantiation
        const bool pre = l <= kWinMax && !sa;
        int left = (int)A.L;
        int sa_bsz = 1;  // SA: proposals per batch (sa_next)
        int sa_cadd = 0, sa_lon = 0, sa_los = 0, sa_loq = 0;  // SA: early decision bookkeeping (sa_next)
        uint32_t sa_pcb = (uint32_t)A.sa_ctr[sid] - 1000u;        // SA: proposal cache base (empty)
        int rb = 0;
        sync();

        // ---- first selection of the round
        bool straight = block_any(xm != stm[t]);
        int k = 0, dk = 0, xk = 0;
        bool have = true;  // a first flip exists (SA may accept nothing)
        if (sa && !straight) {
            have = sa_next(A, sm, g, xm, sid, n, t, nt, left, k, dk, xk, sa_bsz, sa_cadd, sa_lon, sa_los, sa_loq, sa_pcb);
        } else {
            int cv, ci2;
            {  // one inlined scan (code size of the flip loop)
                const M cm = straight ? (M)(xm ^ stm[t]) : window_mask(a, l, n, t, nt);
                candidates(g, xm, cm, t, nt, cv, ci2);
            }
            if (pre && !straight) {
                int a2 = a + l;
                if (a2 >= n) a2 -= n;
                publish_window(g, xm, a2, l, n, t, nt, win->d[fbase & 1], win->x[fbase & 1]);
            }
            const Red r = block_reduce(Red{INT_MAX, cv, ci2}, sm->red, rb, lane, warp, nw);
            k = r.i >> 1;
            xk = r.i & 1;
            dk = r.c;
        }
        bool exact = true;  // compute the n neighbour deltas of this flip exactly
        if (have && t == ctl) issue_row(A, k, rowbuf + rowb * (fbase & 1), sm->bar[fbase & 1], nt);

        int f = 0;
        ABS_T(if (lane == 0) for (int q = 0; q < 24; ++q) sm->tacc[warp][q] = 0;)
        for (; have; ++f) {
#ifndef ABS_TIMING
            if constexpr (!kSA) {
                if (pre && !straight)
                    fast_local(A, sm, win, rowbuf, rowb, g, xm, a, l, n, t, nt, lane, warp, nw, ctl, left, k, dk, xk,
                               exact, f, fbase);
            }
#endif
            const int b = (fbase + f) & 1;
            const uint32_t par = (uint32_t)((fbase + f) >> 1) & 1u;
            unsigned char *row = rowbuf + rowb * b;
            ABS_T(long long tc0 = clock64(); const int to = straight ? 8 : 0;)

            // ---- window-first selection of the next flip (the last warp, the controller), prefetch its row
            if (pre && !straight && left > 1 && warp == nw - 1)
                window_first(A, sm, win, rowbuf, rowb, b, par, a, l, n, xk, lane, warp, nt, ABS_T(tc0) + 0);

            // ---- SA early decision (the SA analogue of the window-first selection): the
            // proposals left over from the batch that accepted k_f were drawn already;
            // their Delta(X_{f+1}) needs one entry of row k_f each (Eq.(16)), so the
            // controller decides them as soon as row k_f lands and, on an acceptance,
            // issues the next row before the update.  Same decisions, in the same
            // order, as one at a time (rejections do not change the state).
            const int sa_cnt = (kSaEarly && !straight) ? min(sa_lon, left) : 0;  // uniform
            if (sa_cnt > 0 && warp == nw - 1) {
                mbar_wait(&sm->bar[b][0], par);
                if (kRowChunks == 2) mbar_wait(&sm->bar[b][1], par);
                int kk = 0, d = 0, xn = 0;
                bool ok = false;
                if (lane < sa_cnt) {
                    const int q = sa_loq + lane;
                    kk = sm->sa_k[sa_los][q];
                    const uint32_t o1 = sm->sa_o[sa_los][q];
                    const int d0 = sm->sa_d[sa_los][q];
                    const int x0 = sm->sa_x[sa_los][q];
                    if (kk == k) {  // Eq.(6): Delta_k(X') = -Delta_k(X)
                        d = -d0;
                        xn = x0 ^ 1;
                    } else {
                        d = d0 + reinterpret_cast<const short *>(row)[kk] * (2 - 4 * (x0 ^ xk));
                        xn = x0;
                    }
                    ok = sa_accept(d, sm->sa_dt, sm->sa_inv, o1);  // Eq.(7)
                }
                const unsigned m = __ballot_sync(kFull, ok);
                const int j = m ? __ffs(m) - 1 : -1;
                const int kn = __shfl_sync(kFull, kk, max(j, 0));
                const int dn = __shfl_sync(kFull, d, max(j, 0));
                const int xnn = __shfl_sync(kFull, xn, max(j, 0));
                if (j >= 0 && elect_one()) issue_row(A, kn, rowbuf + rowb * (b ^ 1), sm->bar[b ^ 1], nt);
                if (lane == 0) sm->sa_e = make_int4(j >= 0 ? kn : -1, dn, xnn, j >= 0 ? j + 1 : sa_cnt);
            }

            ABS_T(long long tc1 = clock64(); mbar_wait(&sm->bar[b][0], par); long long tc2 = clock64();)
            // ---- flip k (Alg. 4 lines P:L328-336 / Alg. 5 lines P:L371-376)
            const int c = xk ? -2 : 2;  // 2 phi(x_k), pre-flip bit (Eq.(16))
            {
                const int j = group_of(k, nt);
                if (t == (k >> 3) - nt * j) xm ^= (M)1 << (8 * j + (k & 7));  // x_k <- 1 - x_k
            }
            int vmin, cmin, cj;
            const uint4 *row4 = reinterpret_cast<const uint4 *>(row);
            M mism = 0;
            if (straight) {
                mism = xm ^ stm[t];
                process_row<kStraight>(g, xm, mism, row4, sm->bar[b], par, c, t, nt, vmin, cmin, cj);
            } else {
                if (exact) process_row<kMin>(g, xm, 0, row4, sm->bar[b], par, c, t, nt, vmin, cmin, cj);
                else process_row<kUpdate>(g, xm, 0, row4, sm->bar[b], par, c, t, nt, vmin, cmin, cj);
                if (!sa) {
                    a += l;  // offset <- (a + l) mod n
                    if (a >= n) a -= n;
                }
            }
            ABS_T(long long tc3 = clock64();)
            // straight phase: the byte-group beta = t + nt * cj of this thread's first
            // minimum; the CTA minimum of (cmin, beta) names the owner of the lowest-index
            // argmin over the mismatches (i = 8 beta + e, reading C5)
            int ci2 = (straight && cmin != INT_MAX) ? t + nt * cj : INT_MAX;
            if (!straight) {
                if (pre) {
                    int a2 = a + l;
                    if (a2 >= n) a2 -= n;
                    publish_window(g, xm, a2, l, n, t, nt, win->d[b ^ 1], win->x[b ^ 1]);
                } else if (!sa) {
                    window_candidates(g, xm, a, l, n, t, nt, cmin, ci2);
                }
            }

            // ---- thread 0: E(X') = E(X) + d_k, the bound LB, the improvement
            // threshold, and (prefetch path) whether the next flip must be exact
            if (t == ctl) {
                sm->hash = (sm->hash ^ (uint64_t)(uint32_t)k) * kFnvPrime;
                sm->nflip += 1;
                if (straight) sm->nstraight += 1;
                const long long E1 = sm->E + dk;
                const long long LB1 = min(sm->LB - 2 * (long long)A.wmax, -(long long)dk);
                const long long EB = sm->EB;
                sm->E = E1;
                sm->LB = LB1;
                // cand = E(X') + min(0, m) < E_B  <=>  min(0, m) < E_B - E(X')   (<= 2^31 - 32768
                // because E_B <= E(X); clamped below at INT_MIN, where it can never hold)
                sm->thr[b] = (int)max(EB - E1, (long long)INT_MIN);
                if (pre && !straight && left > 1) {
                    // E_B may still drop in this flip: the current (larger) E_B only makes
                    // the test more conservative
                    const int dk1 = sm->sel[b].y;
                    const long long LB2 = min(LB1 - 2 * (long long)A.wmax, -(long long)dk1);
                    sm->sel[b].w = (E1 + dk1 + min(LB2, 0LL) < EB) ? 1 : 0;
                }
                if (sa && !straight && sa_cnt > 0) {
                    // SA lazy tracking, early-accepted next flip: the same test (this thread wrote
                    // sa_e in the early decision above)
                    const int4 e = sm->sa_e;
                    if (e.x >= 0) {
                        const long long LB2 = min(LB1 - 2 * (long long)A.wmax, -(long long)e.y);
                        sm->sa_ex[b] = (E1 + e.y + min(LB2, 0LL) < EB) ? 1 : 0;
                    }
                }
            }

            ABS_T(long long tc4 = clock64();)
            Red r1;
            if (exact) {
                r1 = block_reduce(Red{vmin, cmin, ci2}, sm->red, rb, lane, warp, nw);
            } else {
                sync();  // row buffer b free; sel[b], thr[b] and the window published
                r1 = Red{INT_MAX, INT_MAX, INT_MAX};
            }

            ABS_T(long long tc5 = clock64();)
            // ---- neighbour tracking (reading C2) and, straight phase, the argmin index
            const bool improve = exact && min(r1.v, 0) < sm->thr[b];  // uniform
            if (t == ctl && exact) {
                sm->LB = r1.v;
                if (improve) sm->EB = sm->E + min(r1.v, 0);
            }
            if (sa && t == ctl) {  // for the lazy test after sa_next (read after its barrier)
                sm->sa_lz[b][0] = sm->E;
                sm->sa_lz[b][1] = sm->EB;
                sm->sa_lz[b][2] = sm->LB;
            }
            const bool sidx = straight && r1.c != INT_MAX;
            int snext = 0;
            if (sidx) {
                // The owner of byte-group beta finds the index in its 8 slots, publishes it
                // (its warp arrives on named barrier 1, the other warps wait there) and
                // issues the TMA for the next row: no second CTA reduction on the chain.
                const int beta = r1.i;
                const int jb = group_of(8 * beta, nt);
                const int owner = beta - nt * jb;
                if (warp == (owner >> 5)) {
                    if (t == owner) {
                        snext = lowest_equal_group(g, xm, mism, r1.c, jb, t, nt);
                        sm->snext[b] = snext;
                    }
                    snext = __shfl_sync(kFull, snext, owner & 31);
                    named_arrive(1, nt);
                    if (t == owner) issue_row(A, snext >> 1, rowbuf + rowb * (b ^ 1), sm->bar[b ^ 1], nt);
                } else {
                    named_sync(1, nt);
                    snext = sm->snext[b];
                }
            }
            ABS_T(if (lane == 0 && straight) { sm->tacc[warp][7] += improve; sm->tacc[warp][15] += improve && r1.v < 0; })
            if (improve) {
                M bm = xm;
                if (r1.v < 0) {  // B = X' with its best neighbour flipped (reading C2)
                    const int it = (vmin == r1.v) ? lowest_equal(g, xm, ~(M)0, r1.v, t, nt) : INT_MAX;
                    const Red r2 = block_reduce(Red{it, INT_MAX, INT_MAX}, sm->red, rb, lane, warp, nw);
                    const int istar = r2.v >> 1;
                    const int j = group_of(istar, nt);
                    if (t == (istar >> 3) - nt * j) bm ^= (M)1 << (8 * j + (istar & 7));
                }
                sbm[t] = bm;
            }
            if (sidx) {
                k = snext >> 1;
                xk = snext & 1;
                dk = r1.c;
            }

            // ---- next flip
            if (!straight && sa) {
                if (sa_cnt > 0) {  // this flip's early decision (written before the end-of-flip barrier)
                    const int4 e = sm->sa_e;
                    left -= e.w;
                    sa_cadd += e.w;
                    sa_lon = 0;
                    if (e.x >= 0) {  // accepted: its row is in flight
                        k = e.x;
                        dk = e.y;
                        xk = e.z;
                        exact = sm->sa_ex[b] != 0;  // lazy tracking (written before this flip's barrier)
                        continue;
                    }
                }
                if (!sa_next(A, sm, g, xm, sid, n, t, nt, left, k, dk, xk, sa_bsz, sa_cadd, sa_lon, sa_los, sa_loq, sa_pcb)) break;
                {
                    // lazy tracking of the next flip: exact only if E(X'') + min(0, bound on
                    // min Delta(X'')) can beat E_B (sa_lz[b] written before sa_next's barrier)
                    const long long LB2 = min(sm->sa_lz[b][2] - 2 * (long long)A.wmax, -(long long)dk);
                    exact = sm->sa_lz[b][0] + dk + min(LB2, 0LL) < sm->sa_lz[b][1];
                }
            } else if (!straight) {
                if (--left <= 0) break;
                if (pre) {
                    const int4 sv = sm->sel[b];
                    k = sv.x;
                    dk = sv.y;
                    xk = sv.z;
                    exact = sv.w != 0;
                    ABS_T(if (lane == 0) {
                        const long long tc6 = clock64();
                        sm->tacc[warp][to + 0] += tc1 - tc0;
                        sm->tacc[warp][to + 1] += tc2 - tc1;
                        sm->tacc[warp][to + 2] += tc3 - tc2;
                        sm->tacc[warp][to + 3] += tc4 - tc3;
                        sm->tacc[warp][to + 4] += tc5 - tc4;
                        sm->tacc[warp][to + 5] += tc6 - tc5;
                        sm->tacc[warp][to + 6] += 1;
                    })
                    continue;  // row already in flight
                }
                k = r1.i >> 1;
                xk = r1.i & 1;
                dk = r1.c;
            } else if (!sidx) {
                // X = T: the straight search is over; local search from T (Step 4b)
                straight = false;
                if (left <= 0) break;
                if (sa) {
                    if (!sa_next(A, sm, g, xm, sid, n, t, nt, left, k, dk, xk, sa_bsz, sa_cadd, sa_lon, sa_los, sa_loq, sa_pcb)) break;
                    exact = true;
                    if (t == ctl) issue_row(A, k, rowbuf + rowb * (b ^ 1), sm->bar[b ^ 1], nt);
                    continue;
                }
                int cv, cj;
                candidates(g, xm, window_mask(a, l, n, t, nt), t, nt, cv, cj);
                if (pre) {
                    int a2 = a + l;
                    if (a2 >= n) a2 -= n;
                    publish_window(g, xm, a2, l, n, t, nt, win->d[b ^ 1], win->x[b ^ 1]);
                }
                const Red r = block_reduce(Red{INT_MAX, cv, cj}, sm->red, rb, lane, warp, nw);
                k = r.i >> 1;
                xk = r.i & 1;
                dk = r.c;
                exact = true;
            }
            if (t == ctl && !sidx) issue_row(A, k, rowbuf + rowb * (b ^ 1), sm->bar[b ^ 1], nt);
            ABS_T(if (lane == 0) {
                const long long tc6 = clock64();
                sm->tacc[warp][to + 0] += tc1 - tc0;  // window selection (control warp)
                sm->tacc[warp][to + 1] += tc2 - tc1;  // wait for the row
                sm->tacc[warp][to + 2] += tc3 - tc2;  // row update
                sm->tacc[warp][to + 3] += tc4 - tc3;  // publish + bookkeeping
                sm->tacc[warp][to + 4] += tc5 - tc4;  // reduction / barrier
                sm->tacc[warp][to + 5] += tc6 - tc5;  // tracking + next selection
                sm->tacc[warp][to + 6] += 1;
            })
        }

        if (have) fbase += f + 1;  // rows consumed in this round (no row left in flight)
        ABS_T(if (lane == 0 && A.timing) for (int q = 0; q < 24; ++q)
                  atomicAdd((unsigned long long *)&A.timing[((size_t)sid * 32 + warp) * 24 + q],
                            (unsigned long long)sm->tacc[warp][q]);)

        // ---- Step 5: store (B, E_B) and the state C' for the next round
        sync();
        {
            int32_t *gs = A.g + (size_t)sid * kP * nt;
#pragma unroll
            for (int s = 0; s < kP; ++s) gs[(size_t)s * nt + t] = g[s];
            uint8_t *Xs = A.X + (size_t)sid * G * nt;
            const M bm = sbm[t];
            uint8_t *Bs_out;
            int64_t *EB_out;
            out(Bs_out, EB_out);
#pragma unroll
            for (int j = 0; j < G; ++j) {
                Xs[t + nt * j] = (uint8_t)(xm >> (8 * j));
                Bs_out[t + nt * j] = (uint8_t)(bm >> (8 * j));
            }
            if (t == 0) {
                A.E[sid] = sm->E;
                A.EB[sid] = sm->EB;
                *EB_out = sm->EB;
                A.a[sid] = a;
                A.hash[sid] = sm->hash;
                A.flips[sid] += sm->nflip;
                if (sa) A.sa_ctr[sid] = sm->sa_ctr;
                A.sflips[sid] += sm->nstraight;
            }
        }
    }
};

// resident CTAs per SM the register budget is sized for (launch bounds)
constexpr int min_blocks(int p, int max_t) { return max_t == 32 ? (p == 32 ? 32 : 16) : (max_t == 128 ? 6 : 1); }

template <int kP, int kMaxT, int kNT, bool kSA>
int launch_policy(const RoundArgs &a, cudaStream_t st, size_t smem, const AsyncArgs *q, int *grid_out)
{
    return launch_kernel<Round<kP, kMaxT, kNT, kSA>, kMaxT, min_blocks(kP, kMaxT)>(a, st, smem, q, grid_out);
}

}  // namespace

size_t round_smem_bytes(int32_t nt, int32_t bpt)
{
    if (nt == 32) return round_warp_smem_bytes(32 * bpt);  // one-warp searches: abs_round_warp.cu
    const size_t msz = bpt == 64 ? 8 : 4;
    size_t s = sizeof(RoundSmemT<kSaBatchMulti>) + sizeof(WindowSmem) + 2 * msz * (size_t)nt;
    s = (s + 127) & ~size_t(127);
    return s + 2 * (size_t)2 * bpt * nt;  // two row buffers of 2 * n_pad bytes
}

template <int kP, int kMaxT, int kNT>
int launch_variant(const RoundArgs &a, cudaStream_t st, size_t smem, const AsyncArgs *q, int *grid_out)
{
    if (a.policy == 1) return launch_policy<kP, kMaxT, kNT, true>(a, st, smem, q, grid_out);
    return launch_policy<kP, kMaxT, kNT, false>(a, st, smem, q, grid_out);
}

template <int kP, int kMaxT, int kNT>
int occupancy_variant(int nt, size_t smem, int *per_sm)
{
    return occupancy_of<Round<kP, kMaxT, kNT, false>, kMaxT, min_blocks(kP, kMaxT)>(nt, smem, per_sm);
}

int round_occupancy(int32_t nt, int32_t bpt, int *per_sm)
{
    if (nt == 32) return round_warp_occupancy(bpt, per_sm);  // one-warp searches: abs_round_warp.cu
    const size_t smem = round_smem_bytes(nt, bpt);
    if (bpt == 32) {
        return occupancy_variant<32, 128, 0>(nt, smem, per_sm);
    }
    if (nt == 512) return occupancy_variant<64, 512, 512>(nt, smem, per_sm);
    if (nt == 160) return occupancy_variant<64, 512, 160>(nt, smem, per_sm);  // n_pad = 10240 (TSP, 100 cities)
    return occupancy_variant<64, 512, 0>(nt, smem, per_sm);
}

int launch_round(const RoundArgs &a, cudaStream_t st, const AsyncArgs *q, int *grid_out)
{
    if (a.nt == 32) return launch_round_warp(a, st, q, grid_out);  // one-warp searches: abs_round_warp.cu
    const size_t smem = round_smem_bytes(a.nt, a.bpt);
    if (a.bpt == 32) {
        return launch_variant<32, 128, 0>(a, st, smem, q, grid_out);  // nt = 96
    }
    if (a.nt == 512) return launch_variant<64, 512, 512>(a, st, smem, q, grid_out);  // n_pad = 32768
    if (a.nt == 160) return launch_variant<64, 512, 160>(a, st, smem, q, grid_out);  // n_pad = 10240 (TSP, 100 cities)
    return launch_variant<64, 512, 0>(a, st, smem, q, grid_out);
}

}  // namespace absb
