// Probe for the n = 32k round kernel's memory pattern WITH its compute: one
// 512-thread CTA per SM streams random 64 KiB rows of a 2 GiB int16 matrix into
// a ring of shared-memory buffers by TMA (cp.async.bulk), `depth` rows in flight
// while the CTA consumes the oldest: every thread reads its 128 bytes with
// LDS.128 and applies them to 64 register fields with IDP.2A (the flip update),
// then one __syncthreads frees the buffer.  Question answered: does a second
// row in flight still raise the delivered bandwidth when the SM also does the
// update (DESIGN.md §9 item 2)?  One JSON line per configuration.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c) : "memory"); }
__device__ __forceinline__ void expect_tx(uint64_t *b, uint32_t n) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void bulk(void *d, const void *s, uint32_t n, uint64_t *b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(d)), "l"(s), "r"(n), "r"(smem_u32(b)) : "memory"); }
__device__ __forceinline__ void wait(uint64_t *b, uint32_t p) {
    asm volatile("{\n\t.reg .pred q;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%0], %1;\n\t@!q bra W_%=;\n\t}" ::"r"(smem_u32(b)), "r"(p) : "memory"); }

template <int kWork>
__global__ void __launch_bounds__(512, 1) probe(const int16_t *W, int n, int rows, int depth, int *sink)
{
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t *bar = reinterpret_cast<uint64_t *>(sm);
    unsigned char *buf = sm + 128;
    const size_t rowb = (size_t)n * 2;
    const int t = threadIdx.x;
    if (t == 0) {
        for (int d = 0; d < depth; ++d) mbar_init(&bar[d], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    int g[64];
#pragma unroll
    for (int s = 0; s < 64; ++s) g[s] = t + s;
    uint32_t h = 0x9E3779B9u * (blockIdx.x + 1);
    auto issue = [&](int i) {
        h = h * 1664525u + 1013904223u;
        const int k = (int)(h % (uint32_t)n);
        const int d = i % depth;
        expect_tx(&bar[d], (uint32_t)rowb);
        bulk(buf + rowb * d, reinterpret_cast<const char *>(W) + rowb * k, (uint32_t)rowb, &bar[d]);
    };
    if (t == 0)
        for (int i = 0; i < depth && i < rows; ++i) issue(i);
    for (int i = 0; i < rows; ++i) {
        const int d = i % depth;
        wait(&bar[d], (uint32_t)((i / depth) & 1));
        const uint4 *r4 = reinterpret_cast<const uint4 *>(buf + rowb * d);
        const int cb = (i & 1) ? -2 : 2;
        if (kWork == 0) g[0] += (int)r4[t].x;  // touch only
#pragma unroll
        for (int j = 0; j < (kWork ? 8 : 0); ++j) {
            const uint4 w = r4[t + 512 * j];
            const uint32_t wv[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                g[8 * j + 2 * q] = __dp2a_lo((int)wv[q], cb & 0xff, g[8 * j + 2 * q]);
                g[8 * j + 2 * q + 1] = __dp2a_lo((int)wv[q], (cb & 0xff) << 8, g[8 * j + 2 * q + 1]);
                if (kWork > 1) {  // readout + min work of an exact flip
                    g[8 * j + 2 * q] = min(g[8 * j + 2 * q], g[8 * j + 2 * q + 1] ^ 5);
                }
            }
        }
        __syncthreads();  // buffer d free
        if (t == 0 && i + depth < rows) issue(i + depth);
    }
    int s = 0;
#pragma unroll
    for (int q = 0; q < 64; ++q) s ^= g[q];
    if (s == 0x12345678) sink[0] = s;
}

int main()
{
    const int n = 32768;
    int16_t *W;
    int *sink;
    cudaMalloc(&W, (size_t)n * n * 2);
    cudaMemset(W, 1, (size_t)n * n * 2);
    cudaMalloc(&sink, 8);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int rows = 400;
    for (int work : {0, 1, 2})
        for (int depth : {1, 2, 3}) {
            const size_t smem = 128 + (size_t)depth * n * 2;
            auto k = work == 0 ? probe<0> : work == 1 ? probe<1> : probe<2>;
            cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            k<<<sms, 512, smem>>>(W, n, 8, depth, sink);
            cudaEventRecord(e0);
            k<<<sms, 512, smem>>>(W, n, rows, depth, sink);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms = 0;
            cudaEventElapsedTime(&ms, e0, e1);
            const double bytes = (double)sms * rows * n * 2;
            printf("{\"probe\": \"row_compute\", \"work\": %d, \"depth\": %d, \"GBps\": %.1f, \"cycles_per_row_at_1.9GHz\": %.0f, \"err\": \"%s\"}\n",
                   work, depth, bytes / ms / 1e6, ms * 1e-3 / rows * 1.9e9, cudaGetErrorString(cudaGetLastError()));
        }
    return 0;
}
