// Internal declarations shared by the host library (abs_host.cpp) and the
// sm_100a kernels (abs_kernels.cu).  Not part of the ABI.
#pragma once
#include <cstddef>
#include <cstdint>

#include <cuda_runtime.h>

namespace absb {

// Every search keeps P = 32 bits per thread (one uint32 of x bits per thread)
// and NT threads per search (a multiple of 32, <= 1024), so n_pad = 32 * NT.
constexpr int kBitsPerThread = 32;
constexpr int kMaxThreads = 1024;

// Device layout of one instance:
//   Wz   int16 [n_pad][n_pad]  W with ZERO diagonal, rows/cols >= n zero
//   diag int32 [n_pad]         W_ii (0 for i >= n)
// Element i of a search is owned by thread t = (i >> 3) % NT, slot
// s = 8 * ((i >> 3) / NT) + (i & 7): thread t holds the 4 byte-groups
// beta = t + NT * j (j = 0..3) of the bit vector, i.e. bits 8*beta .. 8*beta+7.
struct Instance {
    int32_t n = 0, n_pad = 0, nt = 0;
    int16_t *Wz = nullptr;
    int32_t *diag = nullptr;
    int32_t *rowmax = nullptr;  // [n_pad] max_i |W_ik| (i != k): bound on one flip's change of any Delta
};

// Per-search state, structure of arrays (index = local search id).
//   g     int32 [S][32][NT]  field g_i = 2 sum_{j != i} W_ij x_j + W_ii, so
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
};

struct RoundArgs {
    const int16_t *Wz;
    const int32_t *rowmax;
    int32_t n, n_pad, nt;
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
};

// Launchers (return cudaError_t as int).
int launch_prepare_w(const int16_t *W_in, int32_t n, int32_t n_pad, int16_t *Wz, int32_t *diag,
                     unsigned long long *asym_count, cudaStream_t st);
int launch_rowmax(const Instance &I, cudaStream_t st);
int launch_zero_start(const Instance &I, SearchState &S, int32_t s0, int32_t s1, cudaStream_t st);
int launch_round(const RoundArgs &a, cudaStream_t st);
// Batched init: X bytes [count][n_pad/8] -> E [count], and either
// Delta int32 [count][n] (plain layout) or nothing.
int launch_batch_init(const Instance &I, const uint8_t *X, int32_t count, int64_t *E, int32_t *delta,
                      cudaStream_t st);
size_t round_smem_bytes(int32_t nt);

}  // namespace absb
