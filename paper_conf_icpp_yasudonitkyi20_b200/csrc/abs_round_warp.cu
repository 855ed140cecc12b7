// The ABS round for searches held by ONE warp (n <= 2048: n_pad = 1024 with
// 32 bits per lane, n_pad = 2048 with 64): device Steps 2-5 of
// one search per CTA.  Citations: /root/reference/PAPER.md (P:Lnnn); readings
// Cnn / D / E are listed in DESIGN.md.
//
// The multi-warp kernel (abs_round.cu) is bound by the W-row stream; this one
// is bound by instruction issue and latency (W is L2-resident, 32 CTAs per SM for 32 bits per lane, 16 for 64), so its
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
//    per-bit factor taken from a packed multiplier word per pair of slots
//    (byte 0: slot 2p, byte 3: slot 2p+1; dp2a.lo / dp2a.hi select them), the
//    sign phi(x_k) applied by one XOR per pair on flips of a set bit.  The
//    window kernels keep the multiplier words in shared memory (Sg), read next
//    to the row, so a search fits 64 registers.
//  * Delta_k -> -Delta_k (Eq.(6)) is D_k -> 2 (s mod 2^kShift) - D_k.
//  * Bookkeeping (E, E_B, the lazy bound LB, the flip hash) lives in
//    registers of every lane (warp-uniform values): no shared-memory round
//    trips, no barriers.
//  * The window argmin touches only the byte-group the window lies in (a
//    uniform branch tree; whole-byte minima when the window is byte-aligned).
//  * One row buffer in shared memory: the next row is issued only after the
//    warp has consumed the current one (its selection needs the updated keys).
//  * SA: proposals one at a time from registers, or 32 at once against a
//    state mirror in shared memory (sa_next).
//
// Global state stays in the field form of abs_internal.h (g, X bytes); it is
// converted at the start and end of each round.
#include <type_traits>

#include "abs_round_common.cuh"

namespace absb {
namespace {

constexpr uint64_t kFnvPrimeW = 0x100000001b3ull;

#ifndef ABS_SA_SINGLE_TRIES
#define ABS_SA_SINGLE_TRIES 1
#endif
#ifndef ABS_WARP_BUFS
#define ABS_WARP_BUFS 1
#endif
// Resident CTAs (one search each) per SM the register budget is sized for: window
// policy 32 -> 64 registers per thread (32 bits per lane; fits with the multipliers in
// shared memory, kSgSmem), 16 -> 128 (64 bits per lane); the SA kernels (Philox and the
// acceptance arithmetic on top, multipliers in registers) 20 -> 96 and 14 -> 128.
// Measured (A/B, 1 B200): with the multipliers in registers, window 20 / 28 / 32 per SM
// -5% / -2% / -14% against 24 at n = 1024 (28 and 32 spill); with them in shared memory 32
// per SM +4.5% (no spill) and 28 -7%; for 64 bits per lane 16 +4.6%, 20 -12%; SA 20 / 14
// +2-5% over 24 / 16.
#ifndef ABS_WARP_MINB32
#define ABS_WARP_MINB32 32
#endif
#ifndef ABS_WARP_MINB64
#define ABS_WARP_MINB64 16
#endif
#ifndef ABS_WARP_MINB32_SA
#define ABS_WARP_MINB32_SA 20
#endif
#ifndef ABS_WARP_MINB64_SA
#define ABS_WARP_MINB64_SA 14
#endif
constexpr int kMinB32 = ABS_WARP_MINB32, kMinB64 = ABS_WARP_MINB64;
constexpr int kMinB32SA = ABS_WARP_MINB32_SA, kMinB64SA = ABS_WARP_MINB64_SA;
#ifndef ABS_SG_SMEM
#define ABS_SG_SMEM 1
#endif
#ifndef ABS_WIN_TREE64
#define ABS_WIN_TREE64 1
#endif

template <int kP, bool kSA>
struct WarpRound {
    static constexpr int G = kP / 8;                      // byte-groups per lane
    static constexpr int kShift = kP == 32 ? 5 : 4;      // key = Delta * 2^kShift + slot code
    static constexpr int kBlk = 1 << kShift;             // slots per key block (code range)
    static constexpr int kNB = kP / kBlk;                // key blocks per lane (1 or 4)
    static constexpr uint32_t kPos = 2u << kShift;       // multiplier byte of phi(x_i) = +1
    static constexpr uint32_t kTog = kPos ^ (256u - kPos);  // XOR turning +m into -m in a byte
    static constexpr uint32_t kTogPair = kTog | (kTog << 24);
    using M = typename MaskOf<kP>::T;
    // window(): the one-group branch tree (A/B switch for 64 bits per lane: -7% with the multipliers
    // in registers, +1.3% since they are in shared memory)
    static constexpr bool kWinTree = kP == 32 || ABS_WIN_TREE64;
    static constexpr int kSaSingleTries = ABS_SA_SINGLE_TRIES;
    // the multipliers (SG) in shared memory instead of registers (window kernels; A/B switch)
    static constexpr bool kSgSmem = ABS_SG_SMEM && !kSA;

    struct Smem {
        uint64_t bar[2];  // row buffer b completes on bar[b]
    };
    static constexpr size_t kHeader = 128;
    // Row buffers: two (double-buffered by flip parity) for the window policy.  The SA
    // kernel uses one (the next row is issued only after the warp has consumed the current
    // one) and spends the bytes on a MIRROR of the state in shared memory -- every lane's
    // keys (chunk c = slots 4c..4c+3 of lane t at ((c * 32 + t) * 16) and x bits -- so the
    // owner of any proposed bit is one shared load away (sa_next).
    static constexpr int kBufs = ABS_WARP_BUFS;
    static constexpr uint32_t kRowB = 2u * kP * 32;  // one row: 2 n_pad bytes
    static constexpr size_t kMirOff = kHeader + (size_t)kBufs * kRowB;
    static constexpr size_t kMirX = kMirOff + (size_t)kP * 32 * 4;

    static constexpr size_t kSgOff = kSA ? kMirX + 32 * sizeof(M) : kMirOff;  // SG chunks (kSgSmem)
    static __host__ __device__ size_t smem_bytes(int n_pad)
    {
        (void)n_pad;  // n_pad = 32 kP
        return kSgOff + (kSgSmem ? (size_t)kP / 2 * 32 * 4 : 0);
    }

    // The packed multipliers of a lane: 16 (32) registers, or chunks of four in shared memory
    // (pairs 4c..4c+3 of lane t at kSgOff + (c * 32 + t) * 16, conflict-free).
    struct SgReg {
        uint32_t v[kP / 2];
        __device__ __forceinline__ uint4 chunk(int c) const
        {
            return make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
        }
        __device__ __forceinline__ void tog(int p, uint32_t m) { v[p] ^= m; }
        __device__ __forceinline__ void set(int p, uint32_t m) { v[p] = m; }
    };
    struct SgSmem {
        uint32_t a;  // this lane's chunk 0
        __device__ __forceinline__ uint4 chunk(int c) const { return lds128(a + 512u * c); }
        __device__ __forceinline__ void tog(int p, uint32_t m)
        {
            const uint32_t ad = a + 512u * (p >> 2) + 4u * (p & 3);
            sts32(ad, lds32(ad) ^ m);
        }
        __device__ __forceinline__ void set(int p, uint32_t m) { sts32(a + 512u * (p >> 2) + 4u * (p & 3), m); }
    };
    using Sg = typename std::conditional<kSgSmem, SgSmem, SgReg>::type;

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
    static __device__ __forceinline__ int popc_m(M x)
    {
        if constexpr (sizeof(M) == 8) return __popcll(x);
        else return __popc(x);
    }

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
    static __device__ __forceinline__ void flip_slot(int (&D)[kP], Sg &SG, int s, bool own)
    {
        if constexpr (HI - LO == 1) {
            if (own) {
                D[LO] = 2 * code_of(LO) - D[LO];
                SG.tog(LO >> 1, (LO & 1) ? (kTog << 24) : kTog);
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
    static __device__ __forceinline__ void pass(int (&D)[kP], const Sg &SG, uint32_t rowl, M mism,
                                                int &vmin, int &cK, int &cb)
    {
        vmin = INT_MAX;
        cK = INT_MAX;
        cb = 0;
        int bk = INT_MAX;  // current block's masked minimum
#pragma unroll
        for (int j = 0; j < G; ++j) {
            if (kMode != kStraightOnly) {
                const uint4 w = lds128(rowl + 512u * j);  // rowl: this lane's 16 bytes of byte-group 0
                const uint32_t wv[4] = {w.x, w.y, w.z, w.w};
                const uint4 m4 = SG.chunk(j);
                const uint32_t mv[4] = {m4.x, m4.y, m4.z, m4.w};
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const uint32_t sg = kX1 ? (mv[q] ^ kTogPair) : mv[q];
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

    static __device__ __forceinline__ int min8(const int *d)
    {
        return min(min(min(d[0], d[1]), min(d[2], d[3])), min(min(d[4], d[5]), min(d[6], d[7])));
    }

    // Lane part of a window inside byte-group j (warp-uniform), reached by a uniform
    // branch tree over the groups.  Aligned (byte-aligned window): K = min of the lane's 8
    // keys of group j if its byte is inside (`in`), else INT_MAX.  Masked: K = min over the
    // lane's bits of group j in the window [a, end) (beta: the lane's byte of group j).
    template <int LO, int HI>
    static __device__ __forceinline__ void win_aligned(const int (&D)[kP], int j, bool in, int &K)
    {
        if constexpr (HI - LO == 1) {
            K = in ? min8(&D[8 * LO]) : INT_MAX;
        } else {
            constexpr int MID = (LO + HI) / 2;
            if (j < MID) win_aligned<LO, MID>(D, j, in, K);
            else win_aligned<MID, HI>(D, j, in, K);
        }
    }
    template <int LO, int HI>
    static __device__ __forceinline__ void win_masked(const int (&D)[kP], int j, int beta, int a, int end, int &K)
    {
        if constexpr (HI - LO == 1) {
            const uint32_t m = range8(8 * beta, a, end);
            int bk = INT_MAX;
#pragma unroll
            for (int e = 0; e < 8; ++e) bk = min(bk, ((m >> e) & 1u) ? D[8 * LO + e] : INT_MAX);
            K = bk;
        } else {
            constexpr int MID = (LO + HI) / 2;
            if (j < MID) win_masked<LO, MID>(D, j, beta, a, end, K);
            else win_masked<MID, HI>(D, j, beta, a, end, K);
        }
    }

    // Lane part of the window argmin over {(a + r) mod n : r < l} (Fig. 2, P:L305;
    // reading C6): only the byte-groups j the window touches (warp-uniform).
    static __device__ __forceinline__ void window(const int (&D)[kP], int a, int l, int n, int t, int &K, int &b)
    {
        const int end = a + l;  // exclusive; > n when the window wraps
        if (kWinTree && end <= n && (a >> 8) == ((end - 1) >> 8)) {
            // The common case: the window lies in ONE byte-group j0 (no wrap, l <= 256 within
            // a 256-bit group), so only that group's 8 keys per lane are read, reached by a
            // uniform branch tree (no per-group tests).
            const int j0 = a >> 8;
            const int beta = t + 32 * j0;  // this lane's byte of group j0
            if (((a | l) & 7) == 0) win_aligned<0, G>(D, j0, (unsigned)(beta - (a >> 3)) < (unsigned)(l >> 3), K);
            else win_masked<0, G>(D, j0, beta, a, end, K);
            b = (8 * j0) >> kShift;
            return;
        }
        if (((a | l) & 7) == 0 && end <= n) {
            // Byte-aligned window without wrap over several groups: a lane holds whole bytes of
            // it, so a touched byte-group contributes the min of its 8 keys or nothing.
            const int b0 = a >> 3, nb = l >> 3;  // window bytes [b0, b0 + nb)
            const int j0 = a >> 8, j1 = (end - 1) >> 8;
            K = INT_MAX;
            b = 0;
            int bk = INT_MAX;
#pragma unroll
            for (int j = 0; j < G; ++j) {
                if (j >= j0 && j <= j1) {
                    const int gm = min8(&D[8 * j]);
                    if ((unsigned)(t + 32 * j - b0) < (unsigned)nb) bk = min(bk, gm);
                }
                if (((8 * (j + 1)) & (kBlk - 1)) == 0) {
                    if (bk != INT_MAX) combine(K, b, bk, (8 * j) >> kShift);
                    bk = INT_MAX;
                }
            }
            return;
        }
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

    // Row k of W into the row buffer at shared address buf, completing on the
    // mbarrier at shared address bar (one lane).
    static __device__ __forceinline__ void issue_row(const RoundArgs &A, int k, uint32_t buf, uint32_t bar)
    {
        const uint32_t bytes = (uint32_t)(2 * kP * 32);  // 2 n_pad
        mbar_arrive_expect_tx_a(bar, bytes);
        bulk_g2s_a(buf, reinterpret_cast<const char *>(A.Wz) + (size_t)k * bytes, bytes, bar);
    }

    // The state mirror the SA proposals read (smem_bytes): keys and x bits of every lane.
    static __device__ __forceinline__ void mirror(unsigned char *smem, const int (&D)[kP], M xm, int t)
    {
        uint4 *mk = reinterpret_cast<uint4 *>(smem + kMirOff);
#pragma unroll
        for (int c = 0; c < kP / 4; ++c)
            mk[c * 32 + t] = make_uint4((uint32_t)D[4 * c], (uint32_t)D[4 * c + 1], (uint32_t)D[4 * c + 2],
                                        (uint32_t)D[4 * c + 3]);
        reinterpret_cast<M *>(smem + kMirX)[t] = xm;
    }

    // SA policy (Alg. 1 + Eq.(7), reading E2): the next accepted proposal from
    // the search's Philox stream (proposal c draws bit k = o0 mod n and the
    // uniform o1), in one of two modes:
    //  * single (`one`): proposal c alone, Delta_k and x_k fetched from the owner
    //    lane's registers (uniform slot tree + shuffles) -- cheapest when
    //    acceptances are frequent;
    //  * batch: 32 proposals at once, lane q drawing and deciding proposal c + q
    //    against the state mirror in shared memory (Delta_k and x_k of every
    //    proposal one shared load away), written at most once per flip (`mir`).
    // kSaSingleTries rejections in single mode switch to batch mode, an acceptance
    // of the first proposal of a batch back.  Either way the first acceptance is taken
    // and the proposals after it are drawn again after the flip, so the decisions
    // are the one-at-a-time ones (rejections do not change the state).  Returns
    // false when the budget `left` is spent without an acceptance.
    // The proposal cache of sa_next: lane q holds the draw of proposal pc + q (bit pk =
    // o0 mod n, uniform po = o1); proposals depend only on their counter (Philox), so
    // the cache stays valid across flips.
    struct SaCache {
        unsigned long long pc;
        int pk;
        uint32_t po;
    };
    static __device__ __forceinline__ void sa_fill(const RoundArgs &A, int sid, const UDiv &dn, int t,
                                                   unsigned long long c0, SaCache &pr)
    {
        uint32_t o[4];
        const unsigned long long cq = c0 + (unsigned long long)t;
        philox4x32_10((uint32_t)cq, (uint32_t)(cq >> 32), (uint32_t)(A.sid0 + sid), kTagSA, (uint32_t)A.seed,
                      (uint32_t)(A.seed >> 32), o);
        pr.pc = c0;
        pr.pk = (int)umod(o[0], dn);  // "randomly select a bit" (Alg. 1): o0 mod n
        pr.po = o[1];
    }

    static __device__ __forceinline__ bool sa_next(const RoundArgs &A, int sid, unsigned char *smem, const int (&D)[kP],
                                                   M xm, const UDiv &dn, int t, const UDiv &dt, uint64_t inv2tau,
                                                   unsigned long long &c, SaCache &pr, int &left, bool &one,
                                                   bool &mir, int &k, int &dk, int &xk)
    {
        const int *mk = reinterpret_cast<const int *>(smem + kMirOff);
        const M *mx = reinterpret_cast<const M *>(smem + kMirX);
        int miss = 0;  // single-mode rejections in this call
        while (left > 0) {
            if (one) {
                if (c - pr.pc >= 32ull) sa_fill(A, sid, dn, t, c, pr);
                const int q = (int)(c - pr.pc);
                const int kk = __shfl_sync(kFullMask, pr.pk, q);
                const uint32_t u = __shfl_sync(kFullMask, pr.po, q);
                const int s = slot_of(kk), own = lane_of(kk);
                const int v = get_slot<0, kP>(D, s);
                const int d = __shfl_sync(kFullMask, v >> kShift, own);
                const int x = __shfl_sync(kFullMask, (int)((xm >> s) & 1u), own);
                --left;
                ++c;
                if (sa_accept(d, dt, inv2tau, u)) {  // Eq.(7)
                    k = kk;
                    dk = d;
                    xk = x;
                    return true;
                }
                if (++miss >= kSaSingleTries) one = false;
                continue;
            }
            if (!mir) {
                mirror(smem, D, xm, t);
                __syncwarp();
                mir = true;
            }
            if (c - pr.pc > 16ull) sa_fill(A, sid, dn, t, c, pr);  // fewer than 16 cached: a full batch
            const int q0 = (int)(c - pr.pc);                        // lane of proposal c
            const int nb = min(left, 32 - q0);
            int dq = 0, xq = 0, dec = 0;
            if (t >= q0 && t < q0 + nb) {
                const int s = slot_of(pr.pk), own = lane_of(pr.pk);
                dq = mk[((s >> 2) * 32 + own) * 4 + (s & 3)] >> kShift;
                xq = (int)((mx[own] >> s) & 1u);
                dec = sa_accept_fast(dq, dt, inv2tau, pr.po);  // Eq.(7), most draws decided here
            }
            const unsigned acc = __ballot_sync(kFullMask, dec == 1);
            unsigned unk = __ballot_sync(kFullMask, dec == 2);
            // the first proposal that accepts: walk the candidates in order; an undecided one
            // (u inside the chord band) is settled exactly by its own lane, only when every
            // proposal before it has rejected (the later ones do not matter)
            int ql = -1;
            while (acc | unk) {
                const int c1 = __ffs(acc | unk) - 1;
                if ((acc >> c1) & 1u) {
                    ql = c1;
                    break;
                }
                const bool ex = t == c1 && (uint64_t)pr.po < sa_threshold_exact(dq, (int)dt.d);
                if (__any_sync(kFullMask, ex)) {
                    ql = c1;
                    break;
                }
                unk &= unk - 1;  // c1 rejects
            }
            if (ql >= 0) {
                const int q = ql - q0;  // proposals before the accepted one in this batch
                one = q == 0;
                k = __shfl_sync(kFullMask, pr.pk, ql);
                dk = __shfl_sync(kFullMask, dq, ql);
                xk = __shfl_sync(kFullMask, xq, ql);
                left -= q + 1;
                c += (unsigned long long)(q + 1);
                return true;
            }
            left -= nb;
            c += (unsigned long long)nb;
        }
        return false;
    }

    // ---------------------------------------------------------------- the round
    template <class Out>
    static __device__ __forceinline__ void run(const RoundArgs &A, unsigned char *smem, int sid, const uint8_t *Ts,
                                               const Out &out, int &fbase)
    {
        const int n = A.n;
        const int t = threadIdx.x;
        // shared-window addresses: barrier b at sbase + 8 b, row buffer b at sbase + kHeader + kRowB b
        const uint32_t sbase = smem_u32(smem);

        // ---- state: keys, multipliers, bits (Step 2: target T)
        int D[kP];
        Sg SG;
        if constexpr (kSgSmem) SG.a = sbase + (uint32_t)kSgOff + 16u * t;
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
                SG.set(p, m0 | (m1 << 24));
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
        // the straight phase makes exactly Hamming(C, T) flips (Alg. 5), each reducing it by one
        const int nstraight = __reduce_add_sync(kFullMask, (unsigned)popc_m(xm ^ tm));
        int a = A.a[sid];
        const int l = A.l[sid];
        const int wmax2 = 2 * A.wmax;
        int left = (int)A.L;
        const int tau = kSA ? A.tau[sid] : 1;
        const uint64_t inv2tau = kSA ? sa_inv2tau(tau) : 0ull;
        unsigned long long sa_c = kSA ? A.sa_ctr[sid] : 0ull;
        bool sa_one = true, sa_mir = false;  // SA: single-proposal mode; mirror holds the state
        const UDiv sa_dn = make_udiv(kSA ? (uint32_t)n : 1u), sa_dt = make_udiv(kSA ? (uint32_t)tau : 1u);  // SA divisors
        SaCache sa_pr{sa_c - 64, 0, 0u};  // SA: proposal cache, empty (sa_c - pc >= 32)

        // ---- first selection of the round
        bool straight = __any_sync(kFullMask, xm != tm);
        int k = 0, dk = 0, xk = 0;
        bool have = true;
        if (straight) {
            int vmin, cK, cb;
            pass<kStraightOnly, false>(D, SG, 0u, xm ^ tm, vmin, cK, cb);
            select(cK, cb, xm, t, k, dk, xk);
        } else if (kSA) {
            have = sa_next(A, sid, smem, D, xm, sa_dn, t, sa_dt, inv2tau, sa_c, sa_pr, left, sa_one, sa_mir, k, dk, xk);
        } else if (left > 0) {
            int K, b;
            window(D, a, l, n, t, K, b);
            select(K, b, xm, t, k, dk, xk);
        } else {
            have = false;
        }
        bool exact = true;  // compute the n neighbour deltas of this flip exactly
        if (have && elect_one())
            issue_row(A, k, sbase + kHeader + kRowB * (kBufs == 2 ? fbase & 1 : 0), sbase + 8 * (kBufs == 2 ? fbase & 1 : 0));

        int f = 0;
        while (have) {
            // buffer b of this flip and the phase parity of its barrier
            const int b = kBufs == 2 ? (fbase + f) & 1 : 0;
            const uint32_t par = (uint32_t)((fbase + f) >> (kBufs == 2 ? 1 : 0)) & 1u;
            ++f;
            mbar_wait_a(sbase + 8 * b, par);
            const uint32_t rowl = sbase + kHeader + kRowB * b + 16 * t;

            // ---- flip k (Alg. 4 lines P:L328-336 / Alg. 5 lines P:L371-376)
            flip_slot<0, kP>(D, SG, slot_of(k), lane_of(k) == t);
            if (lane_of(k) == t) xm ^= (M)1 << slot_of(k);
            int vmin = INT_MAX, cK = INT_MAX, cb = 0;
            if (straight) {
                if (xk) pass<kUpdStraight, true>(D, SG, rowl, xm ^ tm, vmin, cK, cb);
                else pass<kUpdStraight, false>(D, SG, rowl, xm ^ tm, vmin, cK, cb);
            } else if (exact) {
                if (xk) pass<kUpdMin, true>(D, SG, rowl, 0, vmin, cK, cb);
                else pass<kUpdMin, false>(D, SG, rowl, 0, vmin, cK, cb);
            } else {
                if (xk) pass<kUpd, true>(D, SG, rowl, 0, vmin, cK, cb);
                else pass<kUpd, false>(D, SG, rowl, 0, vmin, cK, cb);
            }
            __syncwarp();  // every lane is done with row buffer b before it is refilled
            sa_mir = false;  // SA: the mirror is stale after the flip

            // ---- E(X') = E(X) + d_k; trajectory hash (reading D3); the bound LB
            E += dk;
            R = max(R - dk, kRFloor);
            hash = (hash ^ (unsigned long long)(uint32_t)k) * kFnvPrimeW;
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
                        if (!sa_next(A, sid, smem, D, xm, sa_dn, t, sa_dt, inv2tau, sa_c, sa_pr, left, sa_one, sa_mir, k, dk, xk)) break;
                    } else {
                        int K, bb;
                        window(D, a, l, n, t, K, bb);
                        select(K, bb, xm, t, k, dk, xk);
                    }
                    exact = true;
                }
            } else {
                if (kSA) {
                    if (!sa_next(A, sid, smem, D, xm, sa_dn, t, sa_dt, inv2tau, sa_c, sa_pr, left, sa_one, sa_mir, k, dk, xk)) break;
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
            if (elect_one()) issue_row(A, k, sbase + kHeader + kRowB * (kBufs == 2 ? b ^ 1 : 0), sbase + 8 * (kBufs == 2 ? b ^ 1 : 0));
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
                A.flips[sid] += f;  // one row per flip
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
    return launch_kernel<R, 32, kP == 32 ? (kSA ? kMinB32SA : kMinB32) : (kSA ? kMinB64SA : kMinB64)>(a, st, R::smem_bytes(a.n_pad), q,
                                                                                                 grid_out);
}

}  // namespace

size_t round_warp_smem_bytes(int32_t n_pad) { return WarpRound<32, false>::smem_bytes(n_pad); }

int round_warp_occupancy(int32_t bpt, int *per_sm)
{
    if (bpt == 32) return occupancy_of<WarpRound<32, false>, 32, kMinB32>(32, WarpRound<32, false>::smem_bytes(1024), per_sm);
    return occupancy_of<WarpRound<64, false>, 32, kMinB64>(32, WarpRound<64, false>::smem_bytes(2048), per_sm);
}

int launch_round_warp(const RoundArgs &a, cudaStream_t st, const AsyncArgs *q, int *grid_out)
{
    if (a.bpt == 32) return a.policy == 1 ? launch_p<32, true>(a, st, q, grid_out) : launch_p<32, false>(a, st, q, grid_out);
    return a.policy == 1 ? launch_p<64, true>(a, st, q, grid_out) : launch_p<64, false>(a, st, q, grid_out);
}

}  // namespace absb
