// bulk_band.cu -- standalone probe (not part of libsat): pure-DMA copies of an
// n x n int32 matrix with 1-D TMA bulk copies (cp.async.bulk), (a) flat over
// contiguous pieces of P bytes, (b) band-major: a unit is TH rows x U chunks
// of C columns, each chunk loaded as TH row pieces of 4C bytes into an S-slot
// ring and stored back the same way.  Which piece size / geometry keeps HBM
// at the bulk-copy ceiling?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bulk_band bulk_band.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void bar_wait(uint64_t* b, uint32_t ph) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
                     : "=r"(ok) : "r"(smem_u32(b)), "r"(ph) : "memory");
}
__device__ __forceinline__ void ld_bulk(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void st_bulk(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" :: "l"(dst), "r"(smem_u32(src)), "r"(bytes) : "memory");
}

// unit = TH rows x (U chunks of C cols) of an n-col matrix; tickets band-major
template <int TH, int C, int S>
__global__ void band_bulk(const uint32_t* in, uint32_t* out, int n, int U, int units, unsigned long long* ticket) {
    extern __shared__ __align__(128) uint8_t sm[];
    constexpr uint32_t CH = uint32_t(TH) * C * 4;
    uint64_t* full = reinterpret_cast<uint64_t*>(sm + size_t(S) * CH);
    if (threadIdx.x != 0) return;
    for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&full[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
    const int upr = n / (C * U);
    uint32_t g = 0;       // chunk counter (slots)
    for (;;) {
        const int unit = (int)atomicAdd(ticket, 1ull);
        if (unit >= units) break;
        const int band = unit / upr, k0 = (unit % upr) * U;
        const size_t r0 = size_t(band) * TH;
        for (int k = 0; k < U + S - 1; ++k) {
            const int j = k - (S - 1);
            if (j >= 0) {
                const uint32_t it = g + j;
                const int s = it % S;
                bar_wait(&full[s], (it / S) & 1);
                for (int r = 0; r < TH; ++r)
                    st_bulk(out + (r0 + r) * n + size_t(k0 + j) * C, sm + size_t(s) * CH + size_t(r) * C * 4, C * 4);
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
            if (k < U) {
                const uint32_t it = g + k;
                const int s = it % S;
                asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
                asm volatile("{\n.reg .b64 st;\nmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}" :: "r"(smem_u32(&full[s])), "r"(CH) : "memory");
                for (int r = 0; r < TH; ++r)
                    ld_bulk(sm + size_t(s) * CH + size_t(r) * C * 4, in + (r0 + r) * n + size_t(k0 + k) * C, C * 4, &full[s]);
            }
        }
        g += U;
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

static uint8_t* flushbuf;
template <typename F>
static void timeit(const char* name, F f, double bytes) {
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    float best = 1e9, sum = 0;
    const int reps = 10;
    for (int r = 0; r < reps + 2; ++r) {
        cudaMemsetAsync(flushbuf, r, size_t(512) << 20);
        cudaEventRecord(a);
        f();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r >= 2) { best = std::min(best, ms); sum += ms; }
    }
    cudaError_t e = cudaGetLastError();
    printf("%-44s best %.4f ms %.0f GB/s  avg %.4f ms %.0f GB/s %s\n", name, best, bytes / best / 1e6, sum / reps,
           bytes / (sum / reps) / 1e6, e ? cudaGetErrorString(e) : "");
}

int sms, n;
uint32_t *gin, *gout;
unsigned long long* ticket;

template <int TH, int C, int S>
void run(int U, int per_sm) {
    auto k = band_bulk<TH, C, S>;
    const int smem = S * TH * C * 4 + S * 8 + 16;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const int units = (n / TH) * (n / (C * U));
    const int grid = std::min(units, per_sm * sms);
    char nm[160];
    snprintf(nm, sizeof nm, "band TH=%d C=%d S=%d U=%d units=%d grid=%d", TH, C, S, U, units, grid);
    timeit(nm, [&] { cudaMemsetAsync(ticket, 0, 8); k<<<grid, 32, smem>>>(gin, gout, n, U, units, ticket); },
           2.0 * n * n * 4);
}

int main(int argc, char** argv) {
    n = argc > 1 ? atoi(argv[1]) : 16384;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t bytes = size_t(n) * n * 4;
    cudaMalloc(&gin, bytes); cudaMalloc(&gout, bytes);
    cudaMalloc(&flushbuf, size_t(512) << 20);
    cudaMemset(gin, 1, bytes);
    cudaMalloc(&ticket, 8);
    const int nc = n / 128;
    timeit("cudaMemcpyAsync D2D", [&] { cudaMemcpyAsync(gout, gin, bytes, cudaMemcpyDeviceToDevice); }, 2.0 * bytes);
    // flat contiguous pieces: a "band" of 1 row, chunk = piece
    run<1, 8192, 6>(n / 8192, 1);        // 32 KB pieces, ticket per row
    run<1, 2048, 12>(n / 2048, 1);       // 8 KB pieces
    run<1, 512, 24>(n / 512, 1);         // 2 KB
    run<1, 128, 48>(n / 128, 1);         // 512 B pieces, one row per unit
    // band geometries (TH rows x C cols chunks, whole bands or segments)
    run<128, 128, 3>(nc, 1);             // today's band kernel: 128 x 512 B
    run<128, 128, 3>(nc / 8, 1);
    run<64, 256, 3>(nc / 2, 1);
    run<64, 256, 3>(nc / 16, 1);
    run<32, 512, 3>(nc / 4, 1);
    run<32, 512, 3>(nc / 32, 1);
    run<16, 1024, 3>(nc / 8, 1);
    run<16, 1024, 3>(nc / 64, 1);
    run<8, 2048, 3>(nc / 16, 1);
    run<64, 128, 6>(nc, 1);
    run<64, 128, 3>(nc, 2);
    run<32, 128, 6>(nc, 2);
    return 0;
}
