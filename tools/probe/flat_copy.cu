// flat_copy.cu -- standalone probe (not part of libsat): the HBM copy ceiling
// reachable from SM-issued traffic vs cudaMemcpyAsync D2D (what torch copy_
// calls), for an n x n int32 matrix.  Variants: grid-stride uint4 copies with
// different cache hints and loads in flight, and a 1-D TMA bulk copy
// (cp.async.bulk global->smem->global) over per-CTA contiguous pieces.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o flat_copy flat_copy.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int HINT, int UNR>
__global__ void gs_copy(const uint4* __restrict__ in, uint4* __restrict__ out, size_t n4) {
    size_t i = size_t(blockIdx.x) * blockDim.x + threadIdx.x;
    const size_t st = size_t(gridDim.x) * blockDim.x;
    for (; i + (UNR - 1) * st < n4; i += UNR * st) {
        uint4 v[UNR];
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            if (HINT == 0) v[u] = in[i + u * st];
            else if (HINT == 1) v[u] = __ldcs(in + i + u * st);
            else {
                const uint4* p = in + i + u * st;
                asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(p));
            }
        }
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            if (HINT == 0) out[i + u * st] = v[u];
            else __stcs(out + i + u * st, v[u]);
        }
    }
    for (; i < n4; i += st) out[i] = in[i];
}

// block-contiguous: CTA b copies [b*per, (b+1)*per) in a grid-stride-free walk
template <int UNR>
__global__ void blk_copy(const uint4* __restrict__ in, uint4* __restrict__ out, size_t n4, size_t per) {
    const size_t b0 = size_t(blockIdx.x) * per, b1 = min(n4, b0 + per);
    for (size_t i = b0 + threadIdx.x; i < b1; i += UNR * blockDim.x) {
        uint4 v[UNR];
#pragma unroll
        for (int u = 0; u < UNR; ++u) if (i + u * blockDim.x < b1) v[u] = __ldcs(in + i + u * blockDim.x);
#pragma unroll
        for (int u = 0; u < UNR; ++u) if (i + u * blockDim.x < b1) __stcs(out + i + u * blockDim.x, v[u]);
    }
}

// 1-D TMA bulk copy: one elected thread per CTA, S slots of PIECE bytes
template <int S, int PIECE>
__global__ void bulk_copy(const uint8_t* in, uint8_t* out, size_t bytes, unsigned long long* ticket) {
    extern __shared__ __align__(128) uint8_t sm[];
    uint64_t* full = reinterpret_cast<uint64_t*>(sm + S * PIECE);
    __shared__ long long s_piece[S];
    if (threadIdx.x != 0) return;
    for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&full[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
    const long long npieces = (long long)(bytes / PIECE);
    long long k = 0, done = 0;   // loads issued, stores issued
    uint32_t ph[S] = {};
    // prime
    auto issue = [&](int s) {
        const long long pc = (long long)atomicAdd(ticket, 1ull);
        s_piece[s] = pc;
        if (pc >= npieces) return false;
        asm volatile("{\n.reg .b64 st;\nmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}" :: "r"(smem_u32(&full[s])), "r"(PIECE) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     :: "r"(smem_u32(sm + s * PIECE)), "l"(in + pc * PIECE), "r"(PIECE), "r"(smem_u32(&full[s])) : "memory");
        return true;
    };
    bool live[S];
    for (int s = 0; s < S; ++s) live[s] = issue(s);
    for (int it = 0;; ++it) {
        const int s = it % S;
        if (!live[s]) break;
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
                         : "=r"(ok) : "r"(smem_u32(&full[s])), "r"(ph[s]) : "memory");
        ph[s] ^= 1;
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                     :: "l"(out + s_piece[s] * PIECE), "r"(smem_u32(sm + s * PIECE)), "r"(PIECE) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        live[s] = issue(s);
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
    printf("%-34s best %.4f ms %.0f GB/s  avg %.4f ms %.0f GB/s %s\n", name, best, bytes / best / 1e6, sum / reps,
           bytes / (sum / reps) / 1e6, e ? cudaGetErrorString(e) : "");
}

int main(int argc, char** argv) {
    const size_t n = argc > 1 ? atoll(argv[1]) : 16384;
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t bytes = n * n * 4, n4 = bytes / 16;
    uint8_t *in, *out;
    cudaMalloc(&in, bytes); cudaMalloc(&out, bytes);
    cudaMalloc(&flushbuf, size_t(512) << 20);
    cudaMemset(in, 1, bytes);
    unsigned long long* ticket;
    cudaMalloc(&ticket, 8);
    const double B = 2.0 * bytes;
    char nm[128];
    timeit("cudaMemcpyAsync D2D", [&] { cudaMemcpyAsync(out, in, bytes, cudaMemcpyDeviceToDevice); }, B);
    for (int g : {1, 2, 4, 8, 16}) {
        snprintf(nm, sizeof nm, "gs plain u4 grid %d x 512", g * sms);
        timeit(nm, [&] { gs_copy<0, 4><<<g * sms, 512>>>((const uint4*)in, (uint4*)out, n4); }, B);
    }
    for (int g : {1, 4, 16}) {
        snprintf(nm, sizeof nm, "gs cs u8 grid %d x 512", g * sms);
        timeit(nm, [&] { gs_copy<1, 8><<<g * sms, 512>>>((const uint4*)in, (uint4*)out, n4); }, B);
        snprintf(nm, sizeof nm, "gs nc256 u4 grid %d x 512", g * sms);
        timeit(nm, [&] { gs_copy<2, 4><<<g * sms, 512>>>((const uint4*)in, (uint4*)out, n4); }, B);
    }
    for (int g : {1, 4, 16}) {
        const size_t per = (n4 + g * sms - 1) / (g * sms);
        snprintf(nm, sizeof nm, "blk u4 grid %d x 512", g * sms);
        timeit(nm, [&] { blk_copy<4><<<g * sms, 512>>>((const uint4*)in, (uint4*)out, n4, per); }, B);
    }
    {
        auto k = bulk_copy<6, 32768>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 6 * 32768 + 64);
        timeit("bulk 6x32K 1 CTA/SM", [&] { cudaMemsetAsync(ticket, 0, 8); k<<<sms, 32, 6 * 32768 + 64>>>(in, out, bytes, ticket); }, B);
        auto k2 = bulk_copy<3, 32768>;
        cudaFuncSetAttribute(k2, cudaFuncAttributeMaxDynamicSharedMemorySize, 3 * 32768 + 64);
        timeit("bulk 3x32K 2 CTA/SM", [&] { cudaMemsetAsync(ticket, 0, 8); k2<<<2 * sms, 32, 3 * 32768 + 64>>>(in, out, bytes, ticket); }, B);
        auto k3 = bulk_copy<12, 16384>;
        cudaFuncSetAttribute(k3, cudaFuncAttributeMaxDynamicSharedMemorySize, 12 * 16384 + 128);
        timeit("bulk 12x16K 1 CTA/SM", [&] { cudaMemsetAsync(ticket, 0, 8); k3<<<sms, 32, 12 * 16384 + 128>>>(in, out, bytes, ticket); }, B);
    }
    return 0;
}
