// band_geom.cu -- standalone probe (not part of libsat): the band kernel's
// data movement without its arithmetic, for chunk geometries TH rows x C
// columns.  Loads: 1-D bulk copies, one per row piece (4C bytes), issued by
// the 32 lanes of a producer warp into an S-slot ring (mbarrier tx); stores:
// W consumer warps read the slot (LDS.128) and write with STG.128 streaming
// (as the band kernel's finish()), or the producer bulk-stores the slot back
// (pure DMA).  Units: whole bands, or segments of U chunks in segment-major
// order (the band kernel's ticket order).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o band_geom band_geom.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void bar_init(uint64_t* b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(b)), "r"(c)); }
__device__ __forceinline__ void bar_wait(uint64_t* b, uint32_t ph) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
                     : "=r"(ok) : "r"(smem_u32(b)), "r"(ph) : "memory");
}
__device__ __forceinline__ void bar_arrive(uint64_t* b) { asm volatile("{\n.reg .b64 s;\nmbarrier.arrive.shared::cta.b64 s, [%0];\n}" :: "r"(smem_u32(b)) : "memory"); }
__device__ __forceinline__ void bar_expect(uint64_t* b, uint32_t bytes) {
    asm volatile("{\n.reg .b64 st;\nmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}" :: "r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void ld_bulk(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_bulk(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" :: "l"(dst), "r"(smem_u32(src)), "r"(bytes) : "memory");
}

// MODE 0: consumers STG; MODE 1: pure DMA (producer lanes bulk-store)
template <int TH, int C, int S, int W, int MODE>
__global__ void __launch_bounds__((W + 1) * 32) band_geom(const uint32_t* in, uint32_t* out, int n, int U, int nseg,
                                                         int units, unsigned long long* ticket) {
    extern __shared__ __align__(128) uint8_t sm[];
    constexpr uint32_t CH = uint32_t(TH) * C * 4;
    uint32_t* tiles = reinterpret_cast<uint32_t*>(sm);
    uint64_t* full = reinterpret_cast<uint64_t*>(sm + size_t(S) * CH);
    uint64_t* empty = full + S;
    int* s_unit = reinterpret_cast<int*>(empty + S);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { bar_init(&full[s], 1); bar_init(&empty[s], W * 32); }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const int nb = n / TH;
    uint32_t g = 0;
    for (;;) {
        if (threadIdx.x == 0) *s_unit = (int)atomicAdd(ticket, 1ull);
        __syncthreads();
        const int unit = *s_unit;
        __syncthreads();
        if (unit >= units) break;
        const int seg = unit / nb, band = unit % nb;           // segment-major
        const int k0 = seg * U;
        const size_t r0 = size_t(band) * TH;
        if (warp == W) {
            if (MODE == 0) {
                for (int k = 0; k < U; ++k) {
                    const uint32_t it = g + k;
                    const int s = it % S;
                    if (it >= S) bar_wait(&empty[s], ((it / S) & 1) ^ 1);
                    if (lane == 0) bar_expect(&full[s], CH);
                    __syncwarp();
                    for (int r = lane; r < TH; r += 32)
                        ld_bulk(tiles + size_t(s) * TH * C + size_t(r) * C, in + (r0 + r) * n + size_t(k0 + k) * C, C * 4,
                                &full[s], pol);
                }
            } else {
                for (int k = 0; k < U + S - 1; ++k) {
                    const int j = k - (S - 1);
                    if (j >= 0) {
                        const uint32_t it = g + j;
                        const int s = it % S;
                        bar_wait(&full[s], (it / S) & 1);
                        for (int r = lane; r < TH; r += 32)
                            st_bulk(out + (r0 + r) * n + size_t(k0 + j) * C, tiles + size_t(s) * TH * C + size_t(r) * C, C * 4);
                        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                    }
                    if (k < U) {
                        const uint32_t it = g + k;
                        const int s = it % S;
                        asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
                        __syncwarp();
                        if (lane == 0) bar_expect(&full[s], CH);
                        __syncwarp();
                        for (int r = lane; r < TH; r += 32)
                            ld_bulk(tiles + size_t(s) * TH * C + size_t(r) * C, in + (r0 + r) * n + size_t(k0 + k) * C, C * 4,
                                    &full[s], pol);
                    }
                }
                asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            }
        } else if (MODE == 0) {
            // consumer warp w: rows w, w+W, ...; lane owns 16-B vectors
            for (int k = 0; k < U; ++k) {
                const uint32_t it = g + k;
                const int s = it % S;
                bar_wait(&full[s], (it / S) & 1);
                constexpr int VPR = C / 4;                     // 16-B vectors per row
                constexpr int V = TH * VPR / (W * 32);         // per thread
                uint4 v[V];
#pragma unroll
                for (int i = 0; i < V; ++i) {
                    const int q = (i * W + warp) * 32 + lane;  // vector index in the chunk
                    v[i] = reinterpret_cast<const uint4*>(tiles + size_t(s) * TH * C)[q];
                }
                bar_arrive(&empty[s]);
#pragma unroll
                for (int i = 0; i < V; ++i) {
                    const int q = (i * W + warp) * 32 + lane;
                    const int r = q / VPR, c4 = q % VPR;
                    __stcs(reinterpret_cast<uint4*>(out + (r0 + r) * n + size_t(k0 + k) * C) + c4, v[i]);
                }
            }
        }
        g += U;
    }
    if (MODE == 1 && warp == W) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

static uint8_t* flushbuf;
template <typename F>
static void timeit(const char* name, F f, double bytes) {
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    float best = 1e9, sum = 0;
    const int reps = 8;
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
    printf("%-52s best %.4f ms %.0f GB/s  avg %.4f ms %.0f GB/s %s\n", name, best, bytes / best / 1e6, sum / reps,
           bytes / (sum / reps) / 1e6, e ? cudaGetErrorString(e) : "");
}

int sms, n;
uint32_t *gin, *gout;
unsigned long long* ticket;

template <int TH, int C, int S, int W, int MODE>
void run(int nseg) {
    auto k = band_geom<TH, C, S, W, MODE>;
    const int smem = S * TH * C * 4 + 2 * S * 8 + 16;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, (W + 1) * 32, smem);
    const int nc = n / C, U = nc / nseg;
    const int units = (n / TH) * nseg;
    const int grid = std::min(units, occ * sms);
    char nm[200];
    snprintf(nm, sizeof nm, "TH=%3d C=%4d S=%d W=%2d %s seg=%3d units=%5d grid=%4d", TH, C, S, W, MODE ? "dma" : "stg", nseg,
             units, grid);
    timeit(nm, [&] { cudaMemsetAsync(ticket, 0, 8); k<<<grid, (W + 1) * 32, smem>>>(gin, gout, n, U, nseg, units, ticket); },
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
    timeit("cudaMemcpyAsync D2D", [&] { cudaMemcpyAsync(gout, gin, bytes, cudaMemcpyDeviceToDevice); }, 2.0 * bytes);
    const int big = n >= 32768 ? 4 : 1;
    for (int seg : {1, 4 * big, 16 * big}) {
        run<128, 128, 3, 16, 0>(seg);
        run<128, 128, 3, 16, 1>(seg);
        run<64, 256, 3, 16, 0>(seg);
        run<64, 256, 3, 16, 1>(seg);
        run<32, 512, 3, 16, 0>(seg);
        run<32, 512, 3, 16, 1>(seg);
        run<16, 1024, 3, 16, 0>(seg);
        run<16, 1024, 3, 16, 1>(seg);
        run<32, 256, 3, 8, 0>(seg);    // 2 CTAs/SM
        run<64, 128, 3, 8, 0>(seg);    // 2 CTAs/SM (512-B rows)
    }
    return 0;
}
