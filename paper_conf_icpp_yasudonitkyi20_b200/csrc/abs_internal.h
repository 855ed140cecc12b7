// Internal declarations shared by the host library (abs_host.cpp) and the
// sm_100a kernels (abs_round.cu, abs_setup.cu, abs_init_mma.cu).  Not part of
// the ABI.
#pragma once
#include <cstddef>
#include <cstdint>

#include <cuda_runtime.h>

namespace absb {

// Every search is held by NT threads (a multiple of 32) with P bits each,
// n_pad = P * NT >= n: P = 32 for n <= 1024 (one warp) and n_pad = 3072;
// P = 64 otherwise (one warp at n_pad = 2048; 512 threads x 128 registers at
// n = 32k).  Threads hold their P fields in registers.
inline void layout_for(int n, int &n_pad, int &bpt, int &nt)
{
    const int p1 = ((n + 1023) / 1024) * 1024;
    if (p1 == 1024 || p1 == 3072) {
        bpt = 32;
        n_pad = p1;
    } else {
        bpt = 64;
        n_pad = ((n + 2047) / 2048) * 2048;
    }
    nt = n_pad / bpt;
}

// Device layout of one instance:
//   Wz   int16 [n_pad][n_pad]  W with ZERO diagonal, rows/cols >= n zero
//   diag int32 [n_pad]         W_ii (0 for i >= n)
// Element i of a search is owned by thread t = (i >> 3) % NT, slot
// s = 8 * ((i >> 3) / NT) + (i & 7): thread t holds the P/8 byte-groups
// beta = t + NT * j (j < P/8) of the bit vector, i.e. bits 8*beta .. 8*beta+7.
struct Instance {
    int32_t n = 0, n_pad = 0, nt = 0, bpt = 32;
    int16_t *Wz = nullptr;
    int32_t *diag = nullptr;
    int32_t *rowmax = nullptr;  // [n_pad] max_i |W_ik| (i != k)
    int32_t wmax = 32768;       // max_{i != k} |W_ik|: one flip moves any Delta_i by at most 2*wmax
};

// Per-search state, structure of arrays (index = local search id).
//   g     int32 [S][P][NT]   field g_i = 2 sum_{j != i} W_ij x_j + W_ii, so
//                           Delta_i = phi(x_i) * g_i (Eq.(13)); pads INT32_MAX
//   X,B,T uint8 [S][n_pad/8] bit vectors as little-endian bytes
struct SearchState {
    int32_t S = 0;
    int32_t *g = nullptr;
    uint8_t *X = nullptr, *B = nullptr, *T = nullptr;
    int64_t *E = nullptr, *EB = nullptr;
    int32_t *a = nullptr, *l = nullptr;
    uint64_t *hash = nullptr;
    int64_t *flips = nullptr, *sflips = nullptr;
    int32_t *tau = nullptr;         // SA temperature per search
    uint64_t *sa_ctr = nullptr;     // SA proposals drawn per search (Philox counter)
};

struct RoundArgs {
    const int16_t *Wz;
    int32_t wmax;
    int32_t n, n_pad, nt, bpt;
    int32_t *g;
    uint8_t *X;
    const uint8_t *T;
    uint8_t *B;
    int64_t *E, *EB;
    int32_t *a;
    const int32_t *l;
    uint64_t *hash;
    int64_t *flips, *sflips;
    int64_t L;
    int32_t S;
    int32_t sbase;           // lockstep: search id of CTA 0 (a launch may cover searches [sbase, sbase + S))
    int32_t policy;          // ABS_POLICY_WINDOW / ABS_POLICY_SA
    int32_t sid0;            // global id of search 0 (Philox counter word)
    uint64_t seed;           // Philox key
    const int32_t *tau;      // SA temperature per search
    uint64_t *sa_ctr;        // SA proposal counter per search
    long long *timing;  // diagnostics build only: [S][32][8] cycle accumulators
};

// Asynchronous mode (ABS_MODE_ASYNC): work queue and the host<->device
// exchange buffers (mapped pinned host memory, device pointers).
struct AsyncArgs {
    unsigned long long *queue;  // device: next work item (search, round) = (q % S, base + q / S)
    long long total;            // rounds of this launch, all searches together = S * steps
    int base;                   // shared queue: rounds every search had completed before this launch
    int owned;                  // 1: CTA b owns search b and draws round tickets (S <= resident CTAs)
    int *done;                  // device [S]: rounds completed per search
    const uint8_t *Tmap;        // mapped [S][2][n_pad/8]: double-buffered targets
    const uint32_t *tseq;       // mapped [S]: latest target version (slot = version & 1)
    uint8_t *Rb;                // mapped [S][2][n_pad/8]: B of round r in slot r & 1
    int64_t *Reb;               // mapped [S][2]: E_B
    uint32_t *rtver;            // mapped [S][2]: target version the round used
    const uint32_t *rack;       // mapped [S]: rounds consumed by the host
    unsigned int *rcount;       // device: total results published; draws the ring index
    uint32_t *ring;             // mapped [ring_mask + 1][2]: (search, round) in arrival order
    uint32_t *ringseq;          // mapped [ring_mask + 1]: entry idx valid when ringseq[idx & mask] == idx + 1
    uint32_t ring_mask;         // capacity - 1; capacity >= 2 S (at most 2 unconsumed results per search)
};

// Launchers (return cudaError_t as int).
int launch_prepare_w(const int16_t *W_in, int32_t n, int32_t n_pad, int16_t *Wz, int32_t *diag,
                     unsigned long long *asym_count, cudaStream_t st);
int launch_rowmax(const Instance &I, cudaStream_t st);
// synthetic random QUBO n x n (row-major, dense) into W (abs_random_qubo_dev)
int launch_random_qubo(int16_t *W, int32_t n, uint64_t seed, cudaStream_t st);
int launch_zero_start(const Instance &I, SearchState &S, int32_t s0, int32_t s1, cudaStream_t st);
// q == nullptr: lockstep round (one CTA per search); otherwise the persistent
// asynchronous kernel (grid = min(S, resident CTAs), *grid_out).
int launch_round(const RoundArgs &a, cudaStream_t st, const AsyncArgs *q = nullptr, int *grid_out = nullptr);
// Batched init, ALU kernel: X packed bits, row b at X + b * row_bytes
// (row_bytes a multiple of 4; bits >= n ignored) -> E [count], and either
// Delta int32 [count][n] (plain layout) or nothing.
int launch_batch_init(const Instance &I, const uint8_t *X, int32_t row_bytes, int32_t count, int64_t *E,
                      int32_t *delta, cudaStream_t st);
// Batched init on the tensor cores (abs_init_mma.cu): W split once
// into int8 planes hi / lo (n_pad * n_pad bytes each, UMMA block layout), X
// expanded per call into A (init_mma_a_bytes), then tcgen05.mma kind::i8.
size_t init_mma_plane_bytes(int32_t n_pad);
size_t init_mma_a_bytes(int32_t count, int32_t n_pad);
int launch_wsplit(const Instance &I, int8_t *hi, uint8_t *lo, cudaStream_t st);
int launch_init_mma(const Instance &I, const int8_t *hi, const uint8_t *lo, const uint8_t *X, int32_t row_bytes,
                    int32_t count, uint8_t *A, int64_t *E, int32_t *delta, cudaStream_t st);
size_t round_smem_bytes(int32_t nt, int32_t bpt);
// one-warp searches (nt == 32, n <= 2048): abs_round_warp.cu
size_t round_warp_smem_bytes(int32_t n_pad);
int round_warp_occupancy(int32_t bpt, int *per_sm);
int launch_round_warp(const RoundArgs &a, cudaStream_t st, const AsyncArgs *q, int *grid_out);
// CTAs of the round kernel for layout (nt, bpt) resident per SM (cudaError_t).
int round_occupancy(int32_t nt, int32_t bpt, int *per_sm);

}  // namespace absb
