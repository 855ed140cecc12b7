// Denominators of the small-n roofline: for n <= ~8k
// W is L2-resident and the round kernel is bound either by reading random W
// rows from L2 or by the integer pipes (one add per bit per flip).
//  (1) L2 random-row read bandwidth: every CTA streams random rows of an
//      n x n int16 matrix (n = 1024 / 2048 / 10240: 2 / 4 / 20 KiB rows) into
//      shared memory with cp.async.bulk (as the round kernel does), depth rows
//      in flight, CTAs per SM as the one-warp kernel runs them.
//  (2) integer issue rate: lanes per clock per SM of independent IADD3 (ALU
//      pipe), IDP.2A / IMAD (FMA pipe) and an even mix of both, from clock64()
//      cycle counts (clock-independent).
// Prints one JSON line per configuration.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c) : "memory"); }
__device__ __forceinline__ void expect_tx(uint64_t *b, uint32_t n) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void bulk(void *d, const void *s, uint32_t n, uint64_t *b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(d)), "l"(s), "r"(n), "r"(smem_u32(b)) : "memory"); }
__device__ __forceinline__ void wait(uint64_t *b, uint32_t p) {
    asm volatile("{\n\t.reg .pred q;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%0], %1;\n\t@!q bra W_%=;\n\t}" ::"r"(smem_u32(b)), "r"(p) : "memory"); }

__global__ void rows_probe(const int16_t *W, int n, int rows, int depth, unsigned long long *sink)
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
        bulk(buf + rowb * d, reinterpret_cast<const char *>(W) + rowb * k, (uint32_t)rowb, &bar[d]);
    };
    if (threadIdx.x == 0)
        for (int i = 0; i < depth && i < rows; ++i) issue(i);
    for (int i = 0; i < rows; ++i) {
        const int d = i % depth;
        wait(&bar[d], (uint32_t)((i / depth) & 1));
        acc += buf[rowb * d + (threadIdx.x * 16) % rowb];
        __syncthreads();
        if (threadIdx.x == 0 && i + depth < rows) issue(i + depth);
    }
    if (threadIdx.x == 0) atomicAdd(sink, acc);
}

// kind 0: IADD3 (ALU pipe); 1: IDP.2A (FMA pipe); 2: IMAD (FMA pipe); 3: IADD3 + IDP.2A alternating
template <int kKind>
__global__ void int_probe(int iters, int *out, long long *cycles)
{
    int a[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) a[q] = threadIdx.x * 7 + q;
    const int b = out[0] | 1, c = out[1] | 3;
    __syncthreads();
    const long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int q = 0; q < 16; ++q) {
            if (kKind == 0 || (kKind == 3 && (q & 1))) {
                asm volatile("add.s32 %0, %0, %1;" : "+r"(a[q]) : "r"(b));
            } else if (kKind == 1 || kKind == 3) {
                a[q] = __dp2a_lo(b, c, a[q]);
            } else {
                asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(a[q]) : "r"(b), "r"(c));
            }
        }
    }
    __syncthreads();
    const long long t1 = clock64();
    int s = 0;
#pragma unroll
    for (int q = 0; q < 16; ++q) s ^= a[q];
    if (s == 0x7fffffff) out[2] = s;
    if (threadIdx.x == 0) atomicMax((unsigned long long *)&cycles[blockIdx.x], (unsigned long long)(t1 - t0));
}

int main()
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long *sink;
    cudaMalloc(&sink, 8);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int n : {1024, 2048, 10240}) {
        int16_t *W;
        cudaMalloc(&W, (size_t)n * n * 2);
        cudaMemset(W, 1, (size_t)n * n * 2);
        for (int threads : {32, 128})
            for (int per_sm : {1, 4, 8, 16, 32})
                for (int depth : {1, 2}) {
                    const size_t smem = 128 + (size_t)depth * n * 2;
                    if (smem * per_sm > 200 * 1024 || threads * per_sm > 2048) continue;
                    cudaFuncSetAttribute(rows_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
                    const int grid = sms * per_sm;
                    const int rows = 4000;
                    rows_probe<<<grid, threads, smem>>>(W, n, 50, depth, sink);  // warm-up (L2 fill)
                    cudaEventRecord(e0);
                    rows_probe<<<grid, threads, smem>>>(W, n, rows, depth, sink);
                    cudaEventRecord(e1);
                    cudaEventSynchronize(e1);
                    float ms = 0;
                    cudaEventElapsedTime(&ms, e0, e1);
                    printf("{\"probe\": \"l2_rows\", \"n\": %d, \"row_bytes\": %d, \"threads\": %d, \"ctas_per_sm\": %d, "
                           "\"depth\": %d, \"GBps\": %.1f, \"err\": \"%s\"}\n",
                           n, 2 * n, threads, per_sm, depth, (double)grid * rows * n * 2 / ms / 1e6,
                           cudaGetErrorString(cudaGetLastError()));
                }
        cudaFree(W);
    }
    int *out;
    long long *cyc;
    cudaMalloc(&out, 16);
    cudaMemset(out, 0, 16);
    const int ctas = sms * 4, threads = 512, iters = 4096;
    cudaMalloc(&cyc, sizeof(long long) * ctas);
    const char *names[4] = {"IADD3 (ALU)", "IDP.2A (FMA)", "IMAD (FMA)", "IADD3+IDP.2A"};
    for (int kind = 0; kind < 4; ++kind) {
        for (int rep = 0; rep < 2; ++rep) {
            cudaMemset(cyc, 0, sizeof(long long) * ctas);
            cudaEventRecord(e0);
            if (kind == 0) int_probe<0><<<ctas, threads>>>(iters, out, cyc);
            if (kind == 1) int_probe<1><<<ctas, threads>>>(iters, out, cyc);
            if (kind == 2) int_probe<2><<<ctas, threads>>>(iters, out, cyc);
            if (kind == 3) int_probe<3><<<ctas, threads>>>(iters, out, cyc);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms = 0;
            cudaEventElapsedTime(&ms, e0, e1);
            long long hc[4096];
            cudaMemcpy(hc, cyc, sizeof(long long) * ctas, cudaMemcpyDeviceToHost);
            long long mx = 0;
            for (int i = 0; i < ctas; ++i) mx = hc[i] > mx ? hc[i] : mx;
            const double ops_per_sm = 4.0 * threads * iters * 16;  // 4 CTAs per SM
            if (rep == 1)
                printf("{\"probe\": \"int32\", \"op\": \"%s\", \"lanes_per_clk_per_sm\": %.1f, \"Tops\": %.2f, "
                       "\"implied_mhz\": %.0f, \"err\": \"%s\"}\n",
                       names[kind], ops_per_sm / (double)mx, ops_per_sm * sms / ms / 1e9,
                       (double)mx / ms / 1e3, cudaGetErrorString(cudaGetLastError()));
        }
    }
    return 0;
}
