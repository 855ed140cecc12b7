// Tensor-core batched initialisation for
// sm_100a: tcgen05.mma kind::i8 with TMEM accumulators.
//
// For a batch of solutions X (count x n bits) the fields of Eq.(13)
// need  S_bi = sum_{j != i} W_ij x_bj,  i.e. the dense integer
// contraction  S = X * Wz^T  (Wz = W with zero diagonal; W symmetric).
// It is M = count, N = n, K = n with A = X in {0,1} (u8) -- a GEMM, so it runs
// on the 5th-generation tensor cores.  There is no int16 MMA; W is split
// exactly into two int8 planes,
//     W = 256 * hi + lo,   hi = W >> 8 in [-128, 127] (s8),  lo = W & 255 (u8),
// and two MMAs accumulate  Acc_hi = X * hi^T  (u8 x s8)  and
// Acc_lo = X * lo^T  (u8 x u8)  in int32 TMEM columns.  Every sum is exact:
// |Acc_hi| <= 128 n <= 2^22, Acc_lo <= 255 n < 2^23, |S| <= 32768 n = 2^30.
// The epilogue reads TMEM back with tcgen05.ld and forms, per (b, i),
//     S = 256 Acc_hi + Acc_lo,  g = 2 S + W_ii,  Delta = phi(x_i) g   (Eq.(13))
//     E_b += x_i (S + W_ii)                                            (Eq.(1))
// with E accumulated in int64.
//
// Operands are stored in HBM already in the UMMA "no-swizzle K-major"
// canonical layout, one 16 KiB block per (128-row tile, 128-byte K slab):
// core matrix (8 rows x 16 bytes, 128 contiguous bytes) (g, c) of a block
// sits at g * 1024 + c * 128, so one cp.async.bulk (TMA bulk copy) per
// operand per stage lands the tile in shared memory in the layout the smem
// descriptor names (LBO = 128 B between K-adjacent cores, SBO = 1024 B
// between 8-row groups).  W's planes are built once per instance; X is
// expanded from packed bits per call.
//
// CTA = one 128 (solutions) x 128 (field indices) output tile, 4 warps:
// warp 0 lane 0 = TMA producer, warp 1 lane 0 = MMA issuer (tcgen05.mma is
// issued by one thread for the whole CTA), all 4 warps = epilogue (warp w
// owns TMEM lanes 32w..32w+31 = solutions).  2-stage smem ring (48 KiB per
// stage), 256 TMEM columns, 2 CTAs per SM so one CTA's epilogue overlaps the
// other's main loop.  The grid is M-fastest: CTAs resident at the same time
// share the same W tiles through L2.
#include <cstdint>

#include "abs_internal.h"
#include "ptx.cuh"

namespace absb {
namespace {

constexpr int kBM = 128;             // solutions per tile (UMMA M)
constexpr int kBN = 128;             // field indices per tile (UMMA N)
constexpr int kBK = 128;             // K bytes per stage (4 UMMA K=32 steps)
constexpr int kUK = 32;              // UMMA K for kind::i8
constexpr int kTile = kBM * kBK;     // 16 KiB per operand tile
constexpr int kStages = 2;
constexpr int kStageBytes = 3 * kTile;  // A, B_hi, B_lo
constexpr int kThreads = 128;
constexpr uint32_t kTmemCols = 256;  // [0,128): Acc_hi, [128,256): Acc_lo

// ---- tcgen05 helpers (inline PTX) -------------------------------------------
// Shared-memory matrix descriptor, SWIZZLE_NONE, K-major.
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr)
{
    uint64_t d = (uint64_t)((saddr >> 4) & 0x3FFFu);  // start address
    d |= (uint64_t)((128u >> 4) & 0x3FFFu) << 16;      // LBO: K-adjacent core matrices
    d |= (uint64_t)((1024u >> 4) & 0x3FFFu) << 32;     // SBO: adjacent 8-row groups
    d |= (uint64_t)1 << 46;                            // descriptor version (sm_100)
    return d;                                          // base offset 0, layout SWIZZLE_NONE
}

// Instruction descriptor kind::i8: D s32, A u8 (x), B s8 (hi) or u8 (lo),
// both K-major, N = 128, M = 128.
__host__ __device__ constexpr uint32_t idesc_i8(bool b_signed)
{
    return (2u << 4)                         // D format: s32
           | (0u << 7)                       // A: unsigned 8-bit
           | ((b_signed ? 1u : 0u) << 10)    // B: signed / unsigned 8-bit
           | ((uint32_t)(kBN >> 3) << 17)    // N >> 3
           | ((uint32_t)(kBM >> 4) << 24);   // M >> 4
}

__device__ __forceinline__ void mma_i8(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t accum)
{
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(da), "l"(db), "r"(idesc), "r"(accum)
        : "memory");
}

// The mbarrier tracks completion of every tcgen05 op this thread issued.
__device__ __forceinline__ void mma_commit(uint64_t *bar)
{
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// 32 lanes x 32 consecutive 32-bit columns -> 32 registers per thread.
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32])
{
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}

__device__ __forceinline__ void tmem_ld_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// ---- operand preparation ----------------------------------------------------
// W planes: Wz [n_pad][n_pad] int16 (zero diagonal) -> hi (s8), lo (u8), each
// [n_pad/128 row tiles][n_pad/128 K slabs][16 KiB block].  One thread per
// 16-byte chunk (row i, K bytes j0 .. j0+15).
__global__ void wsplit_kernel(const int16_t *__restrict__ Wz, int n_pad, int8_t *__restrict__ hi,
                              uint8_t *__restrict__ lo)
{
    const int kb = n_pad / kBK;
    const long long chunks = (long long)n_pad * (n_pad / 16);
    for (long long q = blockIdx.x * (long long)blockDim.x + threadIdx.x; q < chunks;
         q += (long long)gridDim.x * blockDim.x) {
        const long long blk = q >> 10;  // 1024 chunks per block
        const int w = (int)(q & 1023);
        const int core = w >> 3, rr = w & 7;
        const int r = (core >> 3) * 8 + rr, c = core & 7;
        const int tile_r = (int)(blk / kb), slab = (int)(blk % kb);
        const int i = tile_r * kBM + r, j0 = slab * kBK + c * 16;
        const int4 *src = reinterpret_cast<const int4 *>(Wz + (size_t)i * n_pad + j0);
        const int4 v0 = src[0], v1 = src[1];
        const uint32_t wv[8] = {(uint32_t)v0.x, (uint32_t)v0.y, (uint32_t)v0.z, (uint32_t)v0.w,
                                (uint32_t)v1.x, (uint32_t)v1.y, (uint32_t)v1.z, (uint32_t)v1.w};
        uint32_t h[4], l[4];
#pragma unroll
        for (int p = 0; p < 4; ++p) {
            // two int16 per word: element 2p' (low half) and 2p'+1 (high half)
            const uint32_t a = wv[2 * p], b = wv[2 * p + 1];
            // lo bytes = low byte of each int16, hi bytes = high byte (arithmetic >> 8 keeps the sign bits)
            l[p] = (a & 0xFFu) | ((a >> 8) & 0xFF00u) | ((b & 0xFFu) << 16) | ((b & 0xFF0000u) << 8);
            h[p] = ((a >> 8) & 0xFFu) | ((a >> 16) & 0xFF00u) | (((b >> 8) & 0xFFu) << 16) | ((b >> 24) << 24);
        }
        const size_t o = (size_t)blk * kTile + (size_t)w * 16;
        *reinterpret_cast<uint4 *>(hi + o) = make_uint4(h[0], h[1], h[2], h[3]);
        *reinterpret_cast<uint4 *>(lo + o) = make_uint4(l[0], l[1], l[2], l[3]);
    }
}

// X: packed bits, row b at X + b * row_bytes (bit j = byte j>>3, bit j&7),
// bits >= n ignored -> A = [m_tiles][n_pad/128][16 KiB] of bytes 0/1, rows
// >= count zero.
__global__ void xexpand_kernel(const uint8_t *__restrict__ X, int row_bytes, int count, int n, int n_pad, int m_tiles,
                               uint8_t *__restrict__ A)
{
    const int kb = n_pad / kBK;
    const long long chunks = (long long)m_tiles * kb * 1024;
    for (long long q = blockIdx.x * (long long)blockDim.x + threadIdx.x; q < chunks;
         q += (long long)gridDim.x * blockDim.x) {
        const long long blk = q >> 10;
        const int w = (int)(q & 1023);
        const int core = w >> 3, rr = w & 7;
        const int r = (core >> 3) * 8 + rr, c = core & 7;
        const int mt = (int)(blk / kb), slab = (int)(blk % kb);
        const int b = mt * kBM + r, j0 = slab * kBK + c * 16;
        uint32_t bits = 0;
        if (b < count && j0 < n) {
            const uint8_t *xb = X + (size_t)b * row_bytes;
            const int nb = (n + 7) >> 3;  // bytes that hold bits < n
            const int byte0 = j0 >> 3;
            bits = (uint32_t)xb[byte0] | (byte0 + 1 < nb ? (uint32_t)xb[byte0 + 1] << 8 : 0u);
            if (n - j0 < 16) bits &= (1u << (n - j0)) - 1u;
        }
        uint32_t o[4];
#pragma unroll
        for (int p = 0; p < 4; ++p) {
            const uint32_t nib = (bits >> (4 * p)) & 0xFu;
            o[p] = (nib & 1u) | ((nib & 2u) << 7) | ((nib & 4u) << 14) | ((nib & 8u) << 21);
        }
        *reinterpret_cast<uint4 *>(A + (size_t)blk * kTile + (size_t)w * 16) = make_uint4(o[0], o[1], o[2], o[3]);
    }
}

// ---- the tensor-core kernel -------------------------------------------------
__global__ void __launch_bounds__(kThreads, 2)
    init_mma_kernel(const uint8_t *__restrict__ A, const int8_t *__restrict__ Bhi, const uint8_t *__restrict__ Blo,
                    const int32_t *__restrict__ diag, const uint8_t *__restrict__ X, int row_bytes, int count, int n,
                    int n_pad, int64_t *__restrict__ Eout, int32_t *__restrict__ delta)
{
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
    __shared__ __align__(8) uint64_t full_bar[kStages], empty_bar[kStages], acc_bar;
    __shared__ uint32_t tmem_base_s;
    __shared__ int32_t diag_s[kBN];

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int mt = blockIdx.x, nt = blockIdx.y;
    const int kb = n_pad / kBK;
    const int m0 = mt * kBM, n0 = nt * kBN;

    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&full_bar[s], 1);
            mbar_init(&empty_bar[s], 1);
        }
        mbar_init(&acc_bar, 1);
        fence_mbar_init();
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_s)),
                     "r"(kTmemCols)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    diag_s[threadIdx.x] = diag[n0 + threadIdx.x];
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tmem_base_s;

    if (warp == 0 && lane == 0) {
        // TMA producer: three bulk copies per stage (A tile, hi tile, lo tile)
        const uint8_t *a_src = A + (size_t)mt * kb * kTile;
        const int8_t *h_src = Bhi + (size_t)nt * kb * kTile;
        const uint8_t *l_src = Blo + (size_t)nt * kb * kTile;
        for (int k = 0; k < kb; ++k) {
            const int s = k % kStages;
            mbar_wait(&empty_bar[s], ((k / kStages) & 1) ^ 1);
            uint8_t *st = smem + s * kStageBytes;
            mbar_arrive_expect_tx(&full_bar[s], kStageBytes);
            bulk_g2s(st, a_src + (size_t)k * kTile, kTile, &full_bar[s]);
            bulk_g2s(st + kTile, h_src + (size_t)k * kTile, kTile, &full_bar[s]);
            bulk_g2s(st + 2 * kTile, l_src + (size_t)k * kTile, kTile, &full_bar[s]);
        }
    } else if (warp == 1 && lane == 0) {
        // MMA issuer: one thread issues every tcgen05.mma of the CTA
        constexpr uint32_t id_hi = idesc_i8(true), id_lo = idesc_i8(false);
        for (int k = 0; k < kb; ++k) {
            const int s = k % kStages;
            mbar_wait(&full_bar[s], (k / kStages) & 1);
            tc_fence_after();
            const uint32_t sa = smem_u32(smem + s * kStageBytes);
#pragma unroll
            for (int u = 0; u < kBK / kUK; ++u) {
                // one K=32 step covers two K-adjacent core matrices: +256 B
                const uint64_t da = sdesc(sa + u * 256);
                const uint64_t dh = sdesc(sa + kTile + u * 256);
                const uint64_t dl = sdesc(sa + 2 * kTile + u * 256);
                const uint32_t acc = (k > 0 || u > 0) ? 1u : 0u;
                mma_i8(tmem, da, dh, id_hi, acc);
                mma_i8(tmem + kBN, da, dl, id_lo, acc);
            }
            mma_commit(&empty_bar[s]);  // smem slot free once these MMAs completed
        }
        mma_commit(&acc_bar);  // accumulators complete
    }
    __syncwarp();

    // ---- epilogue: TMEM -> registers -> (Delta, E) ----
    mbar_wait(&acc_bar, 0);
    tc_fence_after();
    const int r = warp * 32 + lane;  // TMEM lane = tile row = solution
    const int b = m0 + r;
    const bool bvalid = b < count;
    uint32_t xw[4] = {0u, 0u, 0u, 0u};
    if (bvalid) {
        const uint8_t *xb = X + (size_t)b * row_bytes + (n0 >> 3);
        const int nbytes = min(16, ((n + 7) >> 3) - (n0 >> 3));
#pragma unroll
        for (int q = 0; q < 16; ++q)
            if (q < nbytes) xw[q >> 2] |= (uint32_t)xb[q] << (8 * (q & 3));
        const int rem = n - n0;  // mask bits >= n
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int lo_bit = 32 * q;
            if (rem <= lo_bit) xw[q] = 0u;
            else if (rem < lo_bit + 32) xw[q] &= (1u << (rem - lo_bit)) - 1u;
        }
    }
    // the pipeline smem is free now (every MMA completed): reuse for the transpose
    int32_t *stage = reinterpret_cast<int32_t *>(smem) + warp * (32 * 33);
    long long e = 0;
    const uint32_t trow = tmem + ((uint32_t)(warp * 32) << 16);
#pragma unroll 1
    for (int q = 0; q < kBN / 32; ++q) {
        uint32_t h[32], l[32];
        tmem_ld32(trow + q * 32, h);
        tmem_ld32(trow + kBN + q * 32, l);
        tmem_ld_wait();
        const uint32_t xq = q == 0 ? xw[0] : q == 1 ? xw[1] : q == 2 ? xw[2] : xw[3];
#pragma unroll
        for (int j = 0; j < 32; ++j) {
            const int s = 256 * (int)h[j] + (int)l[j];
            const int d = diag_s[q * 32 + j];
            const int x = (int)((xq >> j) & 1u);
            const int g = 2 * s + d;
            stage[lane * 33 + j] = x ? -g : g;
            e += x ? (long long)(s + d) : 0ll;
        }
        __syncwarp();
        if (delta) {
            const int i = n0 + q * 32 + lane;
            for (int rr = 0; rr < 32; ++rr) {
                const int bb = m0 + warp * 32 + rr;
                if (bb < count && i < n) delta[(size_t)bb * n + i] = stage[rr * 33 + lane];
            }
        }
        __syncwarp();
    }
    if (bvalid) atomicAdd(reinterpret_cast<unsigned long long *>(Eout + b), (unsigned long long)e);

    tc_fence_before();
    __syncthreads();
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols) : "memory");
}

}  // namespace

size_t init_mma_plane_bytes(int32_t n_pad) { return (size_t)n_pad * n_pad; }

int launch_wsplit(const Instance &I, int8_t *hi, uint8_t *lo, cudaStream_t st)
{
    wsplit_kernel<<<148 * 8, 256, 0, st>>>(I.Wz, I.n_pad, hi, lo);
    return (int)cudaGetLastError();
}

size_t init_mma_a_bytes(int32_t count, int32_t n_pad)
{
    const size_t m_tiles = (size_t)(count + kBM - 1) / kBM;
    return m_tiles * kBM * (size_t)n_pad;
}

int launch_init_mma(const Instance &I, const int8_t *hi, const uint8_t *lo, const uint8_t *X, int32_t row_bytes,
                    int32_t count, uint8_t *A, int64_t *E, int32_t *delta, cudaStream_t st)
{
    if (count <= 0) return 0;
    const int m_tiles = (count + kBM - 1) / kBM;
    cudaError_t e = cudaMemsetAsync(E, 0, sizeof(int64_t) * (size_t)count, st);
    if (e != cudaSuccess) return (int)e;
    xexpand_kernel<<<148 * 8, 256, 0, st>>>(X, row_bytes, count, I.n, I.n_pad, m_tiles, A);
    if ((e = cudaGetLastError()) != cudaSuccess) return (int)e;
    const int smem = kStages * kStageBytes + 1024;
    e = cudaFuncSetAttribute(init_mma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return (int)e;
    dim3 grid(m_tiles, I.n_pad / kBN);
    init_mma_kernel<<<grid, kThreads, smem, st>>>(A, hi, lo, I.diag, X, row_bytes, count, I.n, I.n_pad, E, delta);
    return (int)cudaGetLastError();
}

}  // namespace absb
