// The ABS round for searches held by ONE warp (n <= 2048: n_pad = 1024 with
// 32 bits per lane, n_pad = 2048 with 64): device Steps 2-5 of
// one search per CTA.  Citations: /root/reference/PAPER.md (P:Lnnn); readings
// Cnn / D / E are listed in DESIGN.md.
//
// The multi-warp kernel (abs_round.cu) is bound by the W-row stream; this one
// is bound by instruction issue and latency (W is L2-resident, 24 CTAs per SM), so its
// state is laid out to make every per-flip step as few warp instructions as
// possible:
//
//  * Keys instead of fields.  Lane t owns the byte-groups beta = t + 32 j
//    (bits 8 beta .. 8 beta + 7, register slots s = 8 j + e) and holds, per
//    bit i, the KEY  D_s = Delta_i * 2^kShift + (s mod 2^kShift)  (kShift = 5
//    for 32 slots, 4 for 64).  |Delta_i| <= 32768 (2n - 1) < 2^(31-kShift)
//    for n <= 2048 (reading C12), so the key is an int32, its order is the
//    order of (Delta_i, slot), and ONE integer min over keys is the
//    lowest-index argmin of Delta (reading C5) -- no readout, no index
//    bookkeeping, no masks of equal values.
//  * The flip update (Eq.(16)) Delta_i += 2 W_ik phi(x_i) phi(x_k) becomes
//    D_s += W_ik * (2^(kShift+1) phi(x_i)) * phi(x_k): one IDP.2A per bit, the
//    per-bit factor taken from a packed multiplier register per pair of slots
//    (byte 0: slot 2p, byte 3: slot 2p+1; dp2a.lo / dp2a.hi select them), the
//    sign phi(x_k) applied by one XOR per pair on flips of a set bit.
//  * Delta_k -> -Delta_k (Eq.(6)) is D_k -> 2 (s mod 2^kShift) - D_k.
//  * Bookkeeping (E, E_B, the lazy bound LB, the flip hash) lives in
//    registers of every lane (warp-uniform values): no shared-memory round
//    trips, no barriers.
//
// Global state stays in the field form of abs_internal.h (g, X bytes); it is
// converted at the start and end of each round.
#include "abs_round_common.cuh"

namespace absb {
namespace {

constexpr uint64_t kFnvPrimeW = 0x100000001b3ull;

template <int kP, bool kSA>
struct WarpRound {
    static constexpr int G = kP / 8;                      // byte-groups per lane
    static constexpr int kShift = kP == 32 ? 5 : 4;      // key = Delta * 2^kShift + slot code
    static constexpr int kBlk = 1 << kShift;             // slots per key block (code range)
    static constexpr int kNB = kP / kBlk;                // key blocks per lane (1 or 4)
    static constexpr uint32_t kPos = 2u << kShift;       // multiplier byte of phi(x_i) = +1
    static constexpr uint32_t kTog = kPos ^ (256u - kPos);  // XOR turning +m into -m in a byte
    static constexpr uint32_t kTogPair = kTog | (kTog << 24);
    static constexpr int kSaBatch = kSaBatchOne;
    using M = typename MaskOf<kP>::T;

    struct Smem {
        uint64_t bar[2];  // row buffer b completes on bar[b]
    };
    static constexpr size_t kHeader = 128;

    static __host__ __device__ size_t smem_bytes(int n_pad) { return kHeader + 2 * (size_t)2 * n_pad; }

    static __device__ __forceinline__ void init_barriers(unsigned char *smem)
    {
        Smem *sm = reinterpret_cast<Smem *>(smem);
        if (threadIdx.x == 0) {
            mbar_init(&sm->bar[0], 1);
            mbar_init(&sm->bar[1], 1);
            fence_mbar_init();
        }
        __syncwarp();
    }

    // ---------------------------------------------------------------- helpers
    static __device__ __forceinline__ int code_of(int s) { return s & (kBlk - 1); }
    // bit index of slot s of lane t
    static __device__ __forceinline__ int index_of(int t, int s) { return 8 * (t + 32 * (s >> 3)) + (s & 7); }
    // slot of bit i in its owner lane ((i >> 3) & 31)
    static __device__ __forceinline__ int slot_of(int i) { return ((i >> 8) << 3) | (i & 7); }
    static __device__ __forceinline__ int lane_of(int i) { return (i >> 3) & 31; }

    // bits [lo, hi) of the byte-group starting at bit `base`, as an 8-bit mask
    static __device__ __forceinline__ uint32_t range8(int base, int lo, int hi)
    {
        const int e0 = min(max(lo - base, 0), 8);
        const int e1 = min(max(hi - base, 0), 8);
        return (0xffu >> (8 - e1)) & ~(0xffu >> (8 - e0)) & 0xffu;
    }

    // Eq.(6) for the owner of bit k: Delta_k -> -Delta_k, x_k -> 1 - x_k (slot s,
    // warp-uniform; a binary search over compile-time slots, nothing indexed
    // dynamically).
    template <int LO, int HI>
    static __device__ __forceinline__ void flip_slot(int (&D)[kP], uint32_t (&SG)[kP / 2], int s, bool own)
    {
        if constexpr (HI - LO == 1) {
            if (own) {
                D[LO] = 2 * code_of(LO) - D[LO];
                SG[LO >> 1] ^= (LO & 1) ? (kTog << 24) : kTog;
            }
        } else {
            constexpr int MID = (LO + HI) / 2;
            if (s < MID) flip_slot<LO, MID>(D, SG, s, own);
            else flip_slot<MID, HI>(D, SG, s, own);
        }
    }

    // D[s] (warp-uniform s)
    template <int LO, int HI>
    static __device__ __forceinline__ int get_slot(const int (&D)[kP], int s)
    {
        if constexpr (HI - LO == 1) {
            return D[LO];
        } else {
            constexpr int MID = (LO + HI) / 2;
            return s < MID ? get_slot<LO, MID>(D, s) : get_slot<MID, HI>(D, s);
        }
    }

    // Lane result of an argmin: key K of the best slot and its key block b.
    // Combines per-block minima in ascending block order: within a block the key
    // orders (Delta, slot); across blocks a later block wins only with a
    // strictly smaller Delta (lower index wins ties, reading C5).
    static __device__ __forceinline__ void combine(int &K, int &b, int k2, int b2)
    {
        if (kNB == 1) {
            K = min(K, k2);
        } else if ((k2 >> kShift) < (K >> kShift)) {
            K = k2;
            b = b2;
        }
    }

    // Warp argmin from each lane's (K, b): (k, Delta_k, x_k), lowest index on ties.
    static __device__ __forceinline__ void select(int K, int b, M xm, int t, int &k, int &dk, int &xk)
    {
        const int v = K >> kShift;  // Delta (K = INT_MAX: no candidate, larger than any Delta)
        const int mv = __reduce_min_sync(kFullMask, v);
        const int s = b * kBlk + code_of(K);
        const int c2 = (K != INT_MAX && v == mv) ? 2 * index_of(t, s) + (int)((xm >> s) & 1u) : INT_MAX;
        const int mi = __reduce_min_sync(kFullMask, c2);
        k = mi >> 1;
        xk = mi & 1;
        dk = mv;
    }

    enum { kUpd = 0, kUpdMin = 1, kUpdStraight = 2, kStraightOnly = 3 };

    // One pass over the lane's slots.  kUpd*: the flip update with row k (Eq.(16));
    // then, kUpdMin / kUpdStraight: vmin = min key over all bits (neighbour
    // tracking, Eq.(5)); kUpdStraight / kStraightOnly: (cK, cb) = lowest-index
    // argmin key over the mismatches `mism` (Alg. 5).
    template <int kMode, bool kX1>
    static __device__ __forceinline__ void pass(int (&D)[kP], const uint32_t (&SG)[kP / 2], const uint4 *row4, int t,
                                                M mism, int &vmin, int &cK, int &cb)
    {
        vmin = INT_MAX;
        cK = INT_MAX;
        cb = 0;
        int bk = INT_MAX;  // current block's masked minimum
#pragma unroll
        for (int j = 0; j < G; ++j) {
            if (kMode != kStraightOnly) {
                const uint4 w = row4[t + 32 * j];
                const uint32_t wv[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const uint32_t sg = kX1 ? (SG[4 * j + q] ^ kTogPair) : SG[4 * j + q];
                    D[8 * j + 2 * q] = __dp2a_lo((int)wv[q], (int)sg, D[8 * j + 2 * q]);
                    D[8 * j + 2 * q + 1] = __dp2a_hi((int)wv[q], (int)sg, D[8 * j + 2 * q + 1]);
                }
            }
            if (kMode == kUpdMin || kMode == kUpdStraight) {
#pragma unroll
                for (int e = 0; e < 8; ++e) vmin = min(vmin, D[8 * j + e]);
            }
            if (kMode == kUpdStraight || kMode == kStraightOnly) {
#pragma unroll
                for (int e = 0; e < 8; ++e) bk = min(bk, ((mism >> (8 * j + e)) & 1u) ? D[8 * j + e] : INT_MAX);
                if (((8 * (j + 1)) & (kBlk - 1)) == 0) {  // end of a key block
                    combine(cK, cb, bk, (8 * j) >> kShift);
                    bk = INT_MAX;
                }
            }
        }
    }

    // Lane part of the window argmin over {(a + r) mod n : r < l} (Fig. 2, P:L305;
    // reading C6): only the byte-groups j the window touches (warp-uniform).
    static __device__ __forceinline__ void window(const int (&D)[kP], int a, int l, int n, int t, int &K, int &b)
    {
        const int end = a + l;  // exclusive; > n when the window wraps
        const int hi1 = min(end, n);
        const int hi2 = end - n;
        const int jA = a >> 8, jB = (hi1 - 1) >> 8;
        const int jW = hi2 > 0 ? (hi2 - 1) >> 8 : -1;
        K = INT_MAX;
        b = 0;
        int bk = INT_MAX;
#pragma unroll
        for (int j = 0; j < G; ++j) {
            const bool touched = (j >= jA && j <= jB) || j <= jW;
            if (touched) {
                const int base = 8 * (t + 32 * j);
                const uint32_t m = range8(base, a, hi1) | range8(base, 0, hi2);
#pragma unroll
                for (int e = 0; e < 8; ++e) bk = min(bk, ((m >> e) & 1u) ? D[8 * j + e] : INT_MAX);
            }
            if (((8 * (j + 1)) & (kBlk - 1)) == 0) {
                if (bk != INT_MAX) combine(K, b, bk, (8 * j) >> kShift);
                bk = INT_MAX;
            }
        }
    }

    // Lowest bit index i* with Delta_i* == m (neighbour tracking, reading C2):
    // only on improving flips.
    static __device__ __forceinline__ int lowest_equal(const int (&D)[kP], int m, int t)
    {
        int r = INT_MAX;
#pragma unroll
        for (int bb = kNB - 1; bb >= 0; --bb) {
            int mk = INT_MAX;
#pragma unroll
            for (int s = 0; s < kBlk; ++s) mk = min(mk, D[bb * kBlk + s]);
            if ((mk >> kShift) == m && mk != INT_MAX) r = index_of(t, bb * kBlk + code_of(mk));
        }
        return __reduce_min_sync(kFullMask, r);
    }

    static __device__ __forceinline__ void issue_row(const RoundArgs &A, int k, unsigned char *buf, uint64_t *bar)
    {
        const uint32_t bytes = (uint32_t)(2 * kP * 32);  // 2 n_pad
        mbar_arrive_expect_tx(bar, bytes);
        bulk_g2s(buf, reinterpret_cast<const char *>(A.Wz) + (size_t)k * bytes, bytes, bar);
    }

    // SA policy (Alg. 1 + Eq.(7), reading E2): proposals from the search's
    // Philox stream in batches of bsz (lane q draws proposal c + q); each
    // proposal's Delta_k and x_k come from its owner lane; lane q decides
    // proposal q; the first acceptance is taken and the proposals after it are
    // drawn again after the flip, so the decisions are the one-at-a-time ones
    // (rejections do not change the state).  Returns false when the budget
    // `left` is spent without an acceptance.
    static __device__ __forceinline__ bool sa_next(const RoundArgs &A, int sid, const int (&D)[kP], M xm, int n, int t,
                                                   int tau, uint64_t inv2tau, unsigned long long &c, int &left, int &bsz,
                                                   int &k, int &dk, int &xk)
    {
        const uint32_t k0 = (uint32_t)A.seed, k1 = (uint32_t)(A.seed >> 32);
        while (left > 0) {
            const int nb = min(left, bsz);
            int kq = 0;
            uint32_t o1 = 0;
            if (t < nb) {
                uint32_t o[4];
                const unsigned long long cq = c + (unsigned long long)t;
                philox4x32_10((uint32_t)cq, (uint32_t)(cq >> 32), (uint32_t)(A.sid0 + sid), kTagSA, k0, k1, o);
                kq = (int)(o[0] % (uint32_t)n);  // "randomly select a bit" (Alg. 1)
                o1 = o[1];
            }
            int dq = 0, xq = 0;
            for (int q = 0; q < nb; ++q) {
                const int kk = __shfl_sync(kFullMask, kq, q);
                const int s = slot_of(kk);
                const int v = get_slot<0, kP>(D, s);
                const int own = lane_of(kk);
                const int d = __shfl_sync(kFullMask, v >> kShift, own);
                const int x = __shfl_sync(kFullMask, (int)((xm >> s) & 1u), own);
                if (t == q) {
                    dq = d;
                    xq = x;
                }
            }
            const bool ok = t < nb && sa_accept(dq, tau, inv2tau, o1);  // Eq.(7)
            const unsigned m = __ballot_sync(kFullMask, ok);
            if (m) {
                const int q = __ffs(m) - 1;  // the first accepted proposal
                if (q == 0) bsz = max(1, bsz >> 1);
                k = __shfl_sync(kFullMask, kq, q);
                dk = __shfl_sync(kFullMask, dq, q);
                xk = __shfl_sync(kFullMask, xq, q);
                left -= q + 1;
                c += (unsigned long long)(q + 1);
                return true;
            }
            left -= nb;
            c += (unsigned long long)nb;
            bsz = min(2 * bsz, kSaBatch);
        }
        return false;
    }

    // ---------------------------------------------------------------- the round
    template <class Out>
    static __device__ __forceinline__ void run(const RoundArgs &A, unsigned char *smem, int sid, const uint8_t *Ts,
                                               const Out &out, int &fbase)
    {
        Smem *sm = reinterpret_cast<Smem *>(smem);
        unsigned char *rowbuf = smem + kHeader;
        constexpr size_t kRowB = (size_t)2 * kP * 32;
        const int n = A.n;
        const int t = threadIdx.x;

        // ---- state: keys, multipliers, bits (Step 2: target T)
        int D[kP];
        uint32_t SG[kP / 2];
        M xm = 0, tm = 0;
        {
            const uint8_t *Xs = A.X + (size_t)sid * G * 32;
#pragma unroll
            for (int j = 0; j < G; ++j) {
                xm |= (M)Xs[t + 32 * j] << (8 * j);
                tm |= (M)Ts[t + 32 * j] << (8 * j);
            }
            const int32_t *gs = A.g + (size_t)sid * kP * 32;
#pragma unroll
            for (int s = 0; s < kP; ++s) {
                const int g = gs[(size_t)s * 32 + t];
                const bool x = (xm >> s) & 1u;
                D[s] = index_of(t, s) < n ? ((x ? -g : g) << kShift) + code_of(s) : INT_MAX;  // Delta = phi(x) g
            }
#pragma unroll
            for (int p = 0; p < kP / 2; ++p) {
                const uint32_t m0 = ((xm >> (2 * p)) & 1u) ? 256u - kPos : kPos;
                const uint32_t m1 = ((xm >> (2 * p + 1)) & 1u) ? 256u - kPos : kPos;
                SG[p] = m0 | (m1 << 24);
            }
        }
        M bm = xm;  // Step 3, reading C4: B = C ...
        long long E = A.E[sid];
        long long EB = E;  // ... E_B = E(C) (Alg. 5)
        // 32-bit bookkeeping of the lazy tracking: R = E_B - E(X) (<= 0) kept >= -2^30 (clamping
        // it up only makes the test below more often true: conservative), and the lower bound
        // LB on min_i Delta_i; kNoLB (unknown, or below -2^30) forces the next flip exact
        constexpr int kRFloor = -(1 << 30), kNoLB = INT_MIN;
        int R = 0, LB = kNoLB;
        unsigned long long hash = A.hash[sid];
        int nflip = 0, nstraight = 0;
        int a = A.a[sid];
        const int l = A.l[sid];
        const int wmax2 = 2 * A.wmax;
        int left = (int)A.L;
        const int tau = kSA ? A.tau[sid] : 1;
        const uint64_t inv2tau = kSA ? sa_inv2tau(tau) : 0ull;
        unsigned long long sa_c = kSA ? A.sa_ctr[sid] : 0ull;
        int sa_bsz = 1;

        // ---- first selection of the round
        bool straight = __any_sync(kFullMask, xm != tm);
        int k = 0, dk = 0, xk = 0;
        bool have = true;
        if (straight) {
            int vmin, cK, cb;
            pass<kStraightOnly, false>(D, SG, nullptr, t, xm ^ tm, vmin, cK, cb);
            select(cK, cb, xm, t, k, dk, xk);
        } else if (kSA) {
            have = sa_next(A, sid, D, xm, n, t, tau, inv2tau, sa_c, left, sa_bsz, k, dk, xk);
        } else if (left > 0) {
            int K, b;
            window(D, a, l, n, t, K, b);
            select(K, b, xm, t, k, dk, xk);
        } else {
            have = false;
        }
        bool exact = true;  // compute the n neighbour deltas of this flip exactly
        if (have && t == 0) issue_row(A, k, rowbuf + kRowB * (fbase & 1), &sm->bar[fbase & 1]);

        int f = 0;
        while (have) {
            const int b = (fbase + f) & 1;
            const uint32_t par = (uint32_t)((fbase + f) >> 1) & 1u;
            ++f;
            mbar_wait(&sm->bar[b], par);
            const uint4 *row4 = reinterpret_cast<const uint4 *>(rowbuf + kRowB * b);

            // ---- flip k (Alg. 4 lines P:L328-336 / Alg. 5 lines P:L371-376)
            flip_slot<0, kP>(D, SG, slot_of(k), lane_of(k) == t);
            if (lane_of(k) == t) xm ^= (M)1 << slot_of(k);
            int vmin = INT_MAX, cK = INT_MAX, cb = 0;
            if (straight) {
                if (xk) pass<kUpdStraight, true>(D, SG, row4, t, xm ^ tm, vmin, cK, cb);
                else pass<kUpdStraight, false>(D, SG, row4, t, xm ^ tm, vmin, cK, cb);
            } else if (exact) {
                if (xk) pass<kUpdMin, true>(D, SG, row4, t, 0, vmin, cK, cb);
                else pass<kUpdMin, false>(D, SG, row4, t, 0, vmin, cK, cb);
            } else {
                if (xk) pass<kUpd, true>(D, SG, row4, t, 0, vmin, cK, cb);
                else pass<kUpd, false>(D, SG, row4, t, 0, vmin, cK, cb);
            }
            __syncwarp();  // every lane is done with row buffer b before it is refilled

            // ---- E(X') = E(X) + d_k; trajectory hash (reading D3); the bound LB
            E += dk;
            R = max(R - dk, kRFloor);
            hash = (hash ^ (unsigned long long)(uint32_t)k) * kFnvPrimeW;
            ++nflip;
            nstraight += straight;
            // Eq.(16) moves Delta_i by <= 2 wmax, Eq.(6) maps Delta_k to -Delta_k
            LB = (LB == kNoLB || LB - wmax2 < kRFloor) ? kNoLB : min(LB - wmax2, -dk);

            // ---- neighbour tracking (reading C2): cand = E(X') + min(0, min_i Delta_i(X'))
            if (straight || exact) {
                const int m = __reduce_min_sync(kFullMask, vmin >> kShift);
                LB = m;
                R = (int)max(EB - E, (long long)kRFloor);  // exact again (R only bounds the lazy test)
                if (E + min(m, 0) < EB) {  // the improvement test itself in int64
                    EB = E + min(m, 0);
                    R = min(m, 0);
                    bm = xm;
                    if (m < 0) {  // B = X' with its best neighbour flipped
                        const int istar = lowest_equal(D, m, t);
                        if (lane_of(istar) == t) bm ^= (M)1 << slot_of(istar);
                    }
                }
            }

            // ---- next flip
            if (straight) {
                if (__any_sync(kFullMask, cK != INT_MAX)) {
                    select(cK, cb, xm, t, k, dk, xk);  // Alg. 5: argmin over the remaining mismatches
                    exact = true;
                } else {
                    // X = T: the straight search is over; local search from T (Step 4b)
                    straight = false;
                    if (left <= 0) break;
                    if (kSA) {
                        if (!sa_next(A, sid, D, xm, n, t, tau, inv2tau, sa_c, left, sa_bsz, k, dk, xk)) break;
                    } else {
                        int K, bb;
                        window(D, a, l, n, t, K, bb);
                        select(K, bb, xm, t, k, dk, xk);
                    }
                    exact = true;
                }
            } else {
                if (kSA) {
                    if (!sa_next(A, sid, D, xm, n, t, tau, inv2tau, sa_c, left, sa_bsz, k, dk, xk)) break;
                } else {
                    a += l;  // offset <- (a + l) mod n
                    if (a >= n) a -= n;
                    if (--left <= 0) break;
                    int K, bb;
                    window(D, a, l, n, t, K, bb);
                    select(K, bb, xm, t, k, dk, xk);
                }
                // lazy tracking: exact only if E(X'') + min(0, bound on min Delta(X'')) can beat E_B
                if (LB == kNoLB || LB - wmax2 < kRFloor) {
                    exact = true;
                } else {
                    const int LB2 = min(LB - wmax2, -dk);
                    exact = dk + min(LB2, 0) < R;
                }
            }
            if (t == 0) issue_row(A, k, rowbuf + kRowB * (b ^ 1), &sm->bar[b ^ 1]);
        }
        fbase += f;  // rows consumed in this round (none left in flight)

        // ---- Step 5: store (B, E_B) and the state C' for the next round
        {
            int32_t *gs = A.g + (size_t)sid * kP * 32;
#pragma unroll
            for (int s = 0; s < kP; ++s) {
                const int dl = D[s] >> kShift;
                gs[(size_t)s * 32 + t] = D[s] == INT_MAX ? INT_MAX : (((xm >> s) & 1u) ? -dl : dl);
            }
            uint8_t *Xs = A.X + (size_t)sid * G * 32;
            uint8_t *Bs_out;
            int64_t *EB_out;
            out(Bs_out, EB_out);
#pragma unroll
            for (int j = 0; j < G; ++j) {
                Xs[t + 32 * j] = (uint8_t)(xm >> (8 * j));
                Bs_out[t + 32 * j] = (uint8_t)(bm >> (8 * j));
            }
            if (t == 0) {
                A.E[sid] = E;
                A.EB[sid] = EB;
                *EB_out = EB;
                A.a[sid] = a;
                A.hash[sid] = hash;
                A.flips[sid] += nflip;
                if (kSA) A.sa_ctr[sid] = sa_c;
                A.sflips[sid] += nstraight;
            }
        }
        __syncwarp();
    }
};

template <int kP, bool kSA>
int launch_p(const RoundArgs &a, cudaStream_t st, const AsyncArgs *q, int *grid_out)
{
    using R = WarpRound<kP, kSA>;
    return launch_kernel<R, 32, kP == 32 ? 24 : 16>(a, st, R::smem_bytes(a.n_pad), q, grid_out);
}

}  // namespace

size_t round_warp_smem_bytes(int32_t n_pad) { return WarpRound<32, false>::smem_bytes(n_pad); }

int round_warp_occupancy(int32_t bpt, int *per_sm)
{
    if (bpt == 32) return occupancy_of<WarpRound<32, false>, 32, 24>(32, WarpRound<32, false>::smem_bytes(1024), per_sm);
    return occupancy_of<WarpRound<64, false>, 32, 16>(32, WarpRound<64, false>::smem_bytes(2048), per_sm);
}

int launch_round_warp(const RoundArgs &a, cudaStream_t st, const AsyncArgs *q, int *grid_out)
{
    if (a.bpt == 32) return a.policy == 1 ? launch_p<32, true>(a, st, q, grid_out) : launch_p<32, false>(a, st, q, grid_out);
    return a.policy == 1 ? launch_p<64, true>(a, st, q, grid_out) : launch_p<64, false>(a, st, q, grid_out);
}

}  // namespace absb
