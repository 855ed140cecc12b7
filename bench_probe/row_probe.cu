// L0 probe: achievable bandwidth of the round kernel's
// memory pattern -- each CTA streams whole random rows of a 2 GiB int16 matrix
// into shared memory with cp.async.bulk (TMA), `depth` rows in flight, no
// compute.  Prints one JSON line per configuration.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c) : "memory"); }
__device__ __forceinline__ void expect_tx(uint64_t *b, uint32_t n) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void bulk(void *d, const void *s, uint32_t n, uint64_t *b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(d)), "l"(s), "r"(n), "r"(smem_u32(b)) : "memory"); }
__device__ __forceinline__ void wait(uint64_t *b, uint32_t p) {
    asm volatile("{\n\t.reg .pred q;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%0], %1;\n\t@!q bra W_%=;\n\t}" ::"r"(smem_u32(b)), "r"(p) : "memory"); }

__global__ void probe(const int16_t *W, int n, int rows, int depth, int chunks, unsigned long long *sink)
{
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t *bar = reinterpret_cast<uint64_t *>(sm);
    unsigned char *buf = sm + 128;
    const size_t rowb = (size_t)n * 2;
    if (threadIdx.x == 0) {
        for (int d = 0; d < depth; ++d) mbar_init(&bar[d], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    unsigned long long acc = 0;
    uint32_t h = 0x9E3779B9u * (blockIdx.x + 1);
    auto issue = [&](int i) {
        h = h * 1664525u + 1013904223u;
        const int k = (int)(h % (uint32_t)n);
        const int d = i % depth;
        expect_tx(&bar[d], (uint32_t)rowb);
        const uint32_t c = (uint32_t)(rowb / chunks);
        for (int q = 0; q < chunks; ++q)
            bulk(buf + rowb * d + (size_t)c * q, reinterpret_cast<const char *>(W) + rowb * k + (size_t)c * q, c, &bar[d]);
    };
    if (threadIdx.x == 0)
        for (int i = 0; i < depth && i < rows; ++i) issue(i);
    for (int i = 0; i < rows; ++i) {
        const int d = i % depth;
        wait(&bar[d], (uint32_t)((i / depth) & 1));
        acc += buf[rowb * d + threadIdx.x * 16];  // touch the data
        __syncthreads();                          // buffer d free
        if (threadIdx.x == 0 && i + depth < rows) issue(i + depth);
    }
    if (threadIdx.x == 0) atomicAdd(sink, acc);
}

int main()
{
    const int n = 32768;
    int16_t *W;
    unsigned long long *sink;
    cudaMalloc(&W, (size_t)n * n * 2);
    cudaMemset(W, 1, (size_t)n * n * 2);
    cudaMalloc(&sink, 8);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int rows = 200;
    for (int depth : {1, 2, 3})
        for (int chunks : {1, 2, 8})
            for (int per_sm : {1, 2}) {
                if (per_sm * depth * 64 > 200) continue;
                const size_t smem = 128 + (size_t)depth * n * 2;
                cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
                const int grid = sms * per_sm;
                probe<<<grid, 128, smem>>>(W, n, 8, depth, chunks, sink);  // warm-up
                cudaEventRecord(e0);
                probe<<<grid, 128, smem>>>(W, n, rows, depth, chunks, sink);
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                float ms = 0;
                cudaEventElapsedTime(&ms, e0, e1);
                const double bytes = (double)grid * rows * n * 2;
                printf("{\"depth\": %d, \"chunks\": %d, \"ctas_per_sm\": %d, \"GBps\": %.1f, \"err\": \"%s\"}\n", depth,
                       chunks, per_sm, bytes / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
            }
    return 0;
}
