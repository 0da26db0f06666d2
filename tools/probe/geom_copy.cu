// geom_copy.cu -- standalone probe (not part of libsat): which band-major
// access geometry moves an n x n int32 matrix at copy speed on this GPU?
// Copies (in -> out) with the band kernel's traffic pattern minus its scan:
// units of H rows x (U chunks of C columns), handed out by an atomic ticket,
// loaded by TMA boxes into an S-slot smem ring, stored either by the consumer
// warps (LDS + STG.128 streaming) or by TMA bulk-tensor stores from the slot.
// Also a flat grid-stride uint4 copy as the reference.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o geom_copy geom_copy.cu
#include <cuda.h>
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c));
}
__device__ __forceinline__ bool mbar_try(uint64_t* b, uint32_t ph) {
    uint32_t ok;
    asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
                 : "=r"(ok) : "r"(smem_u32(b)), "r"(ph) : "memory");
    return ok;
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t ph) { while (!mbar_try(b, ph)) {} }
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("{\n.reg .b64 s;\nmbarrier.arrive.shared::cta.b64 s, [%0];\n}" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint64_t* b, uint32_t bytes) {
    asm volatile("{\n.reg .b64 s;\nmbarrier.arrive.expect_tx.shared::cta.b64 s, [%0], %1;\n}" ::"r"(smem_u32(b)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ uint64_t pol_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void tma_ld(void* dst, const CUtensorMap* m, uint64_t* bar, int c0, int c1, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, %3}], [%4], %5;"
        ::"r"(smem_u32(dst)), "l"((uint64_t)m), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void tma_st(const CUtensorMap* m, const void* src, int c0, int c1, uint64_t pol) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%2, %3}], [%1], %4;"
                 ::"l"((uint64_t)m), "r"(smem_u32(src)), "r"(c0), "r"(c1), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }

// optional per-unit trace (argv[2] == "t"): [unit][2] = start / end globaltimer
__device__ unsigned long long* d_tr = nullptr;
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// MODE 0: consumers LDS + STG.cs; MODE 1: producer TMA-stores each landed slot (pure DMA)
template <int H, int C, int S, int W, int MODE, bool STRIP = false>
__global__ void __launch_bounds__((W + 1) * 32) band_copy(const __grid_constant__ CUtensorMap tin,
                                                          const __grid_constant__ CUtensorMap tout, uint32_t* out,
                                                          int n, int U, unsigned long long* ticket, int units) {
    extern __shared__ __align__(1024) uint8_t sm[];
    constexpr int TILE = H * C;
    uint32_t* tiles = (uint32_t*)sm;
    uint64_t* full = (uint64_t*)(sm + size_t(S) * TILE * 4);
    uint64_t* empty = full + S;
    int* s_unit = (int*)(empty + S);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], W * 32); }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const int upr = n / (C * U);          // units per band
    uint32_t g = 0;
    const uint64_t pol = pol_first();
    for (;;) {
        if (threadIdx.x == 0) *s_unit = (int)atomicAdd(ticket, 1ull);
        __syncthreads();
        const int unit = *s_unit;
        __syncthreads();
        if (unit >= units) break;
        if (d_tr && threadIdx.x == 0) {
            unsigned int smid;
            asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
            d_tr[2 * unit] = (gtimer() & 0xFFFFFFFFFFFFull) | (uint64_t(smid) << 56);
        }
        // band-major: unit = (band, chunk range), chunk k at (cols (k0+k)*C, rows band*H)
        // strip-major: unit = (row segment, strip), chunk k at (cols strip*C, rows (k0+k)*H)
        const int spr = n / (H * U);            // row segments per strip (STRIP)
        const int band = STRIP ? 0 : unit / upr, k0 = STRIP ? (unit / (n / C)) * U : (unit % upr) * U;
        const int strip = STRIP ? unit % (n / C) : 0;
        (void)spr;
        if (warp == W) {
            if (lane == 0 && MODE == 0) {
                for (int k = 0; k < U; ++k) {
                    const uint32_t it = g + k;
                    const int s = it % S;
                    if (it >= S) mbar_wait(&empty[s], ((it / S) & 1) ^ 1);
                    mbar_expect(&full[s], TILE * 4);
                    for (int b = 0; b < C / 128; ++b)
                        tma_ld(tiles + size_t(s) * TILE + b * 128 * H, &tin, &full[s],
                               STRIP ? strip * C + b * 128 : (k0 + k) * C + b * 128, STRIP ? (k0 + k) * H : band * H,
                               pol);
                }
            } else if (lane == 0) {
                // pure DMA: S-1 loads in flight, each landed slot stored by TMA,
                // one store group outstanding before its slot is reloaded
                for (int k = 0; k < U + S - 1; ++k) {
                    const int j = k - (S - 1);
                    if (j >= 0) {
                        const uint32_t itj = g + j;
                        const int sj = itj % S;
                        mbar_wait(&full[sj], (itj / S) & 1);
                        for (int b = 0; b < C / 128; ++b)
                            tma_st(&tout, tiles + size_t(sj) * TILE + b * 128 * H, (k0 + j) * C + b * 128, band * H, pol);
                        bulk_commit();
                    }
                    if (k < U) {
                        const uint32_t it = g + k;
                        const int s = it % S;
                        bulk_wait_read<1>();
                        mbar_expect(&full[s], TILE * 4);
                        for (int b = 0; b < C / 128; ++b)
                            tma_ld(tiles + size_t(s) * TILE + b * 128 * H, &tin, &full[s], (k0 + k) * C + b * 128,
                                   band * H, pol);
                    }
                }
            }
        } else if (MODE == 0) {
            for (int k = 0; k < U; ++k) {
                const uint32_t it = g + k;
                const int s = it % S;
                mbar_wait(&full[s], (it / S) & 1);
                constexpr int V = TILE / 4 / (W * 32);
                uint4 v[V];
#pragma unroll
                for (int i = 0; i < V; ++i) {
                    const int q = (i * W + warp) * 32 + lane;
                    v[i] = ((const uint4*)(tiles + size_t(s) * TILE))[q];
                }
                mbar_arrive(&empty[s]);
#pragma unroll
                for (int i = 0; i < V; ++i) {
                    const int q = (i * W + warp) * 32 + lane;
                    const int b = q / (32 * H), rem = q % (32 * H), r = rem / 32, c4 = rem % 32;
                    if (STRIP)
                        __stcs((uint4*)(out + size_t((k0 + k) * H + r) * n + strip * C + b * 128 + c4 * 4), v[i]);
                    else
                        __stcs((uint4*)(out + size_t(band * H + r) * n + (k0 + k) * C + b * 128 + c4 * 4), v[i]);
                }
            }
        }
        if (d_tr && MODE == 0 && warp == 0 && lane == 0) d_tr[2 * unit + 1] = gtimer();
        g += U;
    }
    if (MODE == 1 && warp == W && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// The same pipelined TMA-load ring with a 1-CTA-per-SM persistent grid but
// loads issued in "waves": the band kernel's geometry with every SM busy.
__global__ void flat_copy(const uint4* __restrict__ in, uint4* __restrict__ out, size_t n4) {
    size_t i = size_t(blockIdx.x) * blockDim.x + threadIdx.x;
    const size_t st = size_t(gridDim.x) * blockDim.x;
    for (; i + 3 * st < n4; i += 4 * st) {
        uint4 a = __ldcs(in + i), b = __ldcs(in + i + st), c = __ldcs(in + i + 2 * st), d = __ldcs(in + i + 3 * st);
        __stcs(out + i, a); __stcs(out + i + st, b); __stcs(out + i + 2 * st, c); __stcs(out + i + 3 * st, d);
    }
    for (; i < n4; i += st) __stcs(out + i, __ldcs(in + i));
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeFn enc;
static int sms;
static uint8_t* flushbuf;

static float timed(void (*launch)(void*), void* ctx, int reps, float* avg) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e9, sum = 0;
    for (int r = 0; r < reps + 2; ++r) {
        cudaMemsetAsync(flushbuf, r, size_t(512) << 20);
        cudaEventRecord(a);
        launch(ctx);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r >= 2) { best = std::min(best, ms); sum += ms; }
    }
    *avg = sum / reps;
    return best;
}

struct Ctx {
    void (*fn)(Ctx*);
    CUtensorMap ti, to;
    uint32_t *in, *out;
    int n, U, units, grid, smem, threads;
    unsigned long long* ticket;
};

template <int H, int C, int S, int W, int MODE, bool STRIP = false>
void run(int n, uint32_t* in, uint32_t* out, int U, int occ_force, const char* tag) {
    Ctx c;
    c.n = n; c.in = in; c.out = out; c.U = U;
    cuuint64_t dims[2] = {(cuuint64_t)n, (cuuint64_t)n}, str[1] = {(cuuint64_t)n * 4};
    cuuint32_t box[2] = {128, H}, es[2] = {1, 1};
    enc(&c.ti, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, in, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    enc(&c.to, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, out, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    c.smem = int(size_t(S) * H * C * 4 + 2 * S * 8 + 16);
    c.threads = (W + 1) * 32;
    auto k = band_copy<H, C, S, W, MODE, STRIP>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, c.smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, c.threads, c.smem);
    if (occ_force) occ = std::min(occ, occ_force);
    cudaMalloc(&c.ticket, 8);
    c.units = (n / H) * (n / (C * U));
    c.grid = std::min(c.units, occ * sms);
    auto launch = [](void* p) {
        Ctx& c = *(Ctx*)p;
        cudaMemsetAsync(c.ticket, 0, 8);
        band_copy<H, C, S, W, MODE, STRIP><<<c.grid, c.threads, c.smem>>>(c.ti, c.to, c.out, c.n, c.U, c.ticket, c.units);
    };
    float avg, best = timed(launch, &c, 10, &avg);
    cudaError_t e = cudaGetLastError();
    printf("%-10s H=%3d C=%4d U=%4d S=%d W=%2d mode=%d occ=%d grid=%4d units=%5d smem=%6d best %.4f ms %.0f GB/s avg %.4f ms %.0f GB/s %s\n",
           tag, H, C, U, S, W, MODE, occ, c.grid, c.units, c.smem, best, 2.0 * n * n * 4 / best / 1e6, avg,
           2.0 * n * n * 4 / avg / 1e6, e ? cudaGetErrorString(e) : "");
    cudaFree(c.ticket);
}

int main(int argc, char** argv) {
    int n = argc > 1 ? atoi(argv[1]) : 16384;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    void* fn;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    enc = (EncodeFn)fn;
    uint32_t *in, *out;
    cudaMalloc(&in, size_t(n) * n * 4);
    cudaMalloc(&out, size_t(n) * n * 4);
    cudaMalloc(&flushbuf, size_t(512) << 20);
    cudaMemset(in, 1, size_t(n) * n * 4);
    // flat reference copies
    for (int mult : {1, 2, 4, 8}) {
        struct F { uint32_t *in, *out; size_t n4; int grid; } f{in, out, size_t(n) * n / 4, sms * mult};
        auto launch = [](void* p) { F& f = *(F*)p; flat_copy<<<f.grid, 512>>>((const uint4*)f.in, (uint4*)f.out, f.n4); };
        float avg, best = timed(launch, &f, 10, &avg);
        printf("flat       grid=%4d x 512  best %.4f ms %.0f GB/s avg %.4f ms %.0f GB/s\n", f.grid, best,
               2.0 * n * n * 4 / best / 1e6, avg, 2.0 * n * n * 4 / avg / 1e6);
    }
    if (argc > 2 && argv[2][0] == 't') {
        // per-band start / end times of the band-kernel geometry copy (one
        // wave of whole 128-row bands): do lower bands finish later?
        unsigned long long* tr;
        const int units = n / 128;
        cudaMalloc(&tr, size_t(units) * 16);
        cudaMemcpyToSymbol(d_tr, &tr, sizeof(tr));
        run<128, 128, 3, 16, 0>(n, in, out, n / 128, 1, "band128t");
        std::vector<unsigned long long> h(size_t(units) * 2);
        cudaMemcpy(h.data(), tr, h.size() * 8, cudaMemcpyDeviceToHost);
        unsigned long long t0 = ~0ull;
        const unsigned long long M = 0xFFFFFFFFFFFFull;
        for (int u = 0; u < units; ++u) t0 = std::min(t0, h[2 * u] & M);
        printf("band smid end_us (last timed launch)\n");
        for (int u = 0; u < units; ++u)
            printf("T %d %d %.1f\n", u, int(h[2 * u] >> 56), ((h[2 * u + 1] & M) - t0) / 1e3);
        return 0;
    }
    if (argc > 2 && argv[2][0] == 's') {
        // small matrices (one wave of bands, argv[2] = "s"): ring depth / box
        // geometry at TH 32 and 16, band-major and strip-major
        run<32, 256, 4, 8, 0>(n, in, out, n / 256, 1, "b32c256s4");
        run<32, 256, 6, 8, 0>(n, in, out, n / 256, 1, "b32c256s6");
        run<32, 512, 3, 8, 0>(n, in, out, n / 512, 1, "b32c512s3");
        run<32, 128, 8, 8, 0>(n, in, out, n / 128, 1, "b32c128s8");
        run<32, 256, 3, 4, 0>(n, in, out, n / 256, 2, "b32c256s3o2");
        run<16, 512, 6, 8, 0>(n, in, out, n / 512, 1, "b16c512s6");
        run<16, 512, 3, 8, 0>(n, in, out, n / 512, 2, "b16c512s3o2");
        run<32, 256, 4, 8, 0>(n, in, out, n / 1024, 1, "b32c256u4");
        run<32, 128, 4, 8, 0, true>(n, in, out, n / 256, 1, "strip32u16");
        run<32, 128, 6, 8, 0, true>(n, in, out, n / 128, 1, "strip32s4");
        return 0;
    }
    const int nc = n / 128;
    const int nr = n / 128;   // 128-row chunks per strip
    run<128, 128, 3, 16, 0>(n, in, out, nc, 1, "band128");
    run<128, 128, 3, 16, 0, true>(n, in, out, nr, 1, "strip128");
    run<128, 128, 3, 16, 0, true>(n, in, out, nr / 4, 1, "strip128s4");
    run<128, 128, 3, 16, 0, true>(n, in, out, nr / 16, 1, "strip128s16");
    run<64, 128, 3, 8, 0, true>(n, in, out, n / 64, 2, "strip64");
    run<128, 128, 3, 16, 1, true>(n, in, out, nr, 1, "strip128dma");
    run<64, 128, 4, 4, 1>(n, in, out, nc / 16, 2, "band64d");
    return 0;
}
