// sat_device.cuh -- sm_100a device primitives for libsat (PTX wrappers).
//
// mbarrier / TMA (cp.async.bulk.tensor) / bulk-group / proxy fences, relaxed
// gpu-scope 64-bit descriptor loads and stores, and the per-row warp scan used
// by every SAT kernel.  Nothing here is shared with the CPU oracle.
#pragma once
#include <cstdint>
#include <type_traits>
#include <cuda.h>

namespace sat {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ------------------------------------------------------------- mbarrier
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n\t}"
                 :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n\t}"
                 :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred p;\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
                 "selp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
}
__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// Watchdog for every spin in libsat: a wait that exceeds kSpinLimitNs is a
// protocol bug (no legitimate wait lasts that long), so the kernel traps and
// the call surfaces as SAT_ERR_CUDA instead of hanging the GPU.
constexpr unsigned long long kSpinLimitNs = 4000000000ull;   // 4 s

// Debug: when set (sat_debug_diag_enable), a spin that passes half the limit
// records {what, extra, block, warp} in host-mapped memory before the trap, so
// a protocol deadlock can be read back after the launch fails.
__device__ unsigned int* g_sat_diag = nullptr;

#ifndef SAT_DEBUG
#define SAT_DEBUG 0      // 1: per-chunk event traces and per-warp progress marks (tools/ only)
#endif
constexpr bool kDebug = SAT_DEBUG != 0;

// progress marks (debug builds only): per (block, warp) the last {unit, step,
// mark} in host-mapped memory (`diag` comes from the kernel parameters, not
// from g_sat_diag: a global load per mark would stall the compute warps)
__device__ __forceinline__ void diag_mark(unsigned int* diag, uint32_t unit, uint32_t step, uint32_t mark) {
    if constexpr (kDebug) {
        if (diag != nullptr && (threadIdx.x & 31) == 0) {
            volatile unsigned int* d = diag + 4096u * 32u * 4u + (blockIdx.x * 32u + (threadIdx.x >> 5)) * 4u;
            d[0] = unit; d[1] = step; d[2] = 0xC0DE0000u | mark; d[3] = blockIdx.x;
        }
    }
}

struct SpinGuard {
    unsigned long long t0 = 0;
    unsigned n = 0;
    bool logged = false;
    uint32_t what = 0, extra = 0;
    __device__ __forceinline__ SpinGuard() {}
    __device__ __forceinline__ SpinGuard(uint32_t w, uint32_t e) : what(w), extra(e) {}
    __device__ __forceinline__ void tick() {
        if ((++n & 1023u) == 0) {
            const unsigned long long t = globaltimer_ns();
            if (t0 == 0) {
                t0 = t;
            } else if (t - t0 > kSpinLimitNs) {
                __trap();
            } else if (t - t0 > kSpinLimitNs / 2 && g_sat_diag != nullptr && !logged) {
                logged = true;
                volatile unsigned int* d = g_sat_diag + (blockIdx.x * 32u + (threadIdx.x >> 5)) * 4u;
                d[0] = what; d[1] = extra; d[2] = 0xC0DE0000u | blockIdx.x; d[3] = threadIdx.x;
                __threadfence_system();
            }
        }
    }
};

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    if (mbar_try_wait(bar, parity)) return;
    SpinGuard guard(smem_u32(bar), parity);
    while (!mbar_try_wait(bar, parity)) guard.tick();
}

// ------------------------------------------------------------- clusters / DSMEM
__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
// shared::cluster address of the same smem location in CTA `rank`
__device__ __forceinline__ uint32_t mapa(uint32_t saddr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
    return r;
}
__device__ __forceinline__ void st_cluster_v4(uint32_t raddr, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    asm volatile("st.shared::cluster.v4.b32 [%0], {%1, %2, %3, %4};" :: "r"(raddr), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
}
__device__ __forceinline__ uint4 ld_cluster_v4(uint32_t raddr) {
    uint4 v;
    asm volatile("ld.shared::cluster.v4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(raddr) : "memory");
    return v;
}
__device__ __forceinline__ void st_cluster_u64(uint32_t raddr, unsigned long long v) {
    asm volatile("st.shared::cluster.u64 [%0], %1;" :: "r"(raddr), "l"(v) : "memory");
}
// arrive on an mbarrier in another CTA of the cluster (release at cluster scope)
__device__ __forceinline__ void mbar_arrive_remote(uint32_t raddr) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" :: "r"(raddr) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait_cluster(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred p;\n\t"
                 "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\t"
                 "selp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
    if (mbar_try_wait_cluster(bar, parity)) return;
    SpinGuard guard(smem_u32(bar) | 0x40000000u, parity);
    while (!mbar_try_wait_cluster(bar, parity)) guard.tick();
}
// every thread of every CTA of the cluster (non-.aligned: lanes may arrive
// from divergent paths)
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release;\n\tbarrier.cluster.wait.acquire;" ::: "memory");
}

// ------------------------------------------------------------- TMA
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* m) {
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(m)) : "memory");
}
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* m, uint64_t* bar,
                                            int c0, int c1, int c2, uint64_t policy) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%2, %3, %4}], [%5], %6;"
        :: "r"(smem_u32(dst)), "l"(reinterpret_cast<uint64_t>(m)), "r"(c0), "r"(c1), "r"(c2),
           "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}
// 1-D bulk copy global -> shared (contiguous `bytes`, a multiple of 16, both
// addresses 16-B aligned), completing tx bytes on `bar`
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                          uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1], %2, [%3], %4;"
        :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}
// HBM -> L2 only (no shared memory, no barrier): raises the bytes in flight
// per SM beyond the shared-memory ring
__device__ __forceinline__ void tma_prefetch_3d(const CUtensorMap* m, int c0, int c1, int c2) {
    asm volatile("cp.async.bulk.prefetch.tensor.3d.L2.global.tile [%0, {%1, %2, %3}];"
                 :: "l"(reinterpret_cast<uint64_t>(m)), "r"(c0), "r"(c1), "r"(c2) : "memory");
}
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* m, const void* src,
                                             int c0, int c1, int c2, uint64_t policy) {
    asm volatile(
        "cp.async.bulk.tensor.3d.global.shared::cta.bulk_group.L2::cache_hint"
        " [%0, {%2, %3, %4}], [%1], %5;"
        :: "l"(reinterpret_cast<uint64_t>(m)), "r"(smem_u32(src)), "r"(c0), "r"(c1), "r"(c2),
           "l"(policy)
        : "memory");
}
__device__ __forceinline__ void bulk_commit() {
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(N) : "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait() {
    asm volatile("cp.async.bulk.wait_group %0;" :: "n"(N) : "memory");
}
// generic-proxy smem writes -> visible to the async proxy (TMA store reads)
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// ------------------------------------------------------------- descriptors
// A descriptor word is (tag << 32) | value-bits, written and read as whole
// 64-bit words at gpu scope, so a reader never needs a separate flag/fence:
// every word validates itself.
__device__ __forceinline__ void st_relaxed_v2(uint64_t* p, uint64_t a, uint64_t b) {
    asm volatile("st.relaxed.gpu.global.v2.b64 [%0], {%1, %2};" :: "l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void ld_relaxed_v2(const uint64_t* p, uint64_t& a, uint64_t& b) {
    asm volatile("ld.relaxed.gpu.global.v2.b64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// ------------------------------------------------------------- arithmetic
// int32 SATs are computed in uint32 (mod 2^32); float32 in IEEE fp32 adds;
// float64 (the paper's precision) in IEEE fp64 adds.
template <typename T> __device__ __forceinline__ uint32_t to_bits(T v);
template <> __device__ __forceinline__ uint32_t to_bits<uint32_t>(uint32_t v) { return v; }
template <> __device__ __forceinline__ uint32_t to_bits<float>(float v) { return __float_as_uint(v); }
template <typename T> __device__ __forceinline__ T from_bits(uint32_t v);
template <> __device__ __forceinline__ uint32_t from_bits<uint32_t>(uint32_t v) { return v; }
template <> __device__ __forceinline__ float from_bits<float>(uint32_t v) { return __uint_as_float(v); }

// 32-bit words per element (1 for int32/float32, 2 for float64) and the
// conversions between an element and its words (low word first).
template <typename T> struct Words { static constexpr int N = int(sizeof(T) / 4); };
template <typename T>
__device__ __forceinline__ void to_words(T v, uint32_t* w) {
    if constexpr (sizeof(T) == 8) {
        w[0] = uint32_t(__double2loint(v));
        w[1] = uint32_t(__double2hiint(v));
    } else {
        w[0] = to_bits<T>(v);
    }
}
template <typename T>
__device__ __forceinline__ T from_words(const uint32_t* w) {
    if constexpr (sizeof(T) == 8) return __hiloint2double(int(w[1]), int(w[0]));
    else return from_bits<T>(w[0]);
}

// N consecutive 32-bit words (N*4 B, naturally aligned) with the widest
// vector accesses: generic (shared or global) load / store, read-only global
// load, streaming (evict-first) global store.
template <int N>
__device__ __forceinline__ void ld_words(const void* p, uint32_t (&w)[N]) {
    if constexpr (N % 4 == 0) {
#pragma unroll
        for (int k = 0; k < N / 4; ++k) {
            const uint4 u = reinterpret_cast<const uint4*>(p)[k];
            w[4 * k] = u.x; w[4 * k + 1] = u.y; w[4 * k + 2] = u.z; w[4 * k + 3] = u.w;
        }
    } else if constexpr (N == 2) {
        const uint2 u = *reinterpret_cast<const uint2*>(p);
        w[0] = u.x; w[1] = u.y;
    } else {
        static_assert(N == 1, "1, 2 or 4k words");
        w[0] = *reinterpret_cast<const uint32_t*>(p);
    }
}
template <int N>
__device__ __forceinline__ void st_words(void* p, const uint32_t (&w)[N]) {
    if constexpr (N % 4 == 0) {
#pragma unroll
        for (int k = 0; k < N / 4; ++k)
            reinterpret_cast<uint4*>(p)[k] = make_uint4(w[4 * k], w[4 * k + 1], w[4 * k + 2], w[4 * k + 3]);
    } else if constexpr (N == 2) {
        *reinterpret_cast<uint2*>(p) = make_uint2(w[0], w[1]);
    } else {
        static_assert(N == 1, "1, 2 or 4k words");
        *reinterpret_cast<uint32_t*>(p) = w[0];
    }
}
template <int N>
__device__ __forceinline__ void ldg_words(const void* p, uint32_t (&w)[N]) {
    static_assert(N % 4 == 0, "16-B vectors");
#pragma unroll
    for (int k = 0; k < N / 4; ++k) {
        const uint4 u = __ldg(reinterpret_cast<const uint4*>(p) + k);
        w[4 * k] = u.x; w[4 * k + 1] = u.y; w[4 * k + 2] = u.z; w[4 * k + 3] = u.w;
    }
}
template <int N>
__device__ __forceinline__ void stcs_words(void* p, const uint32_t (&w)[N]) {
    static_assert(N % 4 == 0, "16-B vectors");
#pragma unroll
    for (int k = 0; k < N / 4; ++k)
        __stcs(reinterpret_cast<uint4*>(p) + k, make_uint4(w[4 * k], w[4 * k + 1], w[4 * k + 2], w[4 * k + 3]));
}

// K consecutive elements <-> their words
template <typename T, int K>
__device__ __forceinline__ void pack(const T (&v)[K], uint32_t (&w)[K * Words<T>::N]) {
#pragma unroll
    for (int i = 0; i < K; ++i) to_words<T>(v[i], w + i * Words<T>::N);
}
template <typename T, int K>
__device__ __forceinline__ void unpack(const uint32_t (&w)[K * Words<T>::N], T (&v)[K]) {
#pragma unroll
    for (int i = 0; i < K; ++i) v[i] = from_words<T>(w + i * Words<T>::N);
}
// 4 consecutive elements by 16-B vector loads (read-only path)
template <typename T>
__device__ __forceinline__ void ldg4(const T* p, T (&e)[4]) {
    uint32_t w[4 * Words<T>::N];
    ldg_words<4 * Words<T>::N>(p, w);
    unpack<T, 4>(w, e);
}

// Inclusive warp scan of x (lane order).  Kogge-Stone with shfl.up.
template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T x, int lane) {
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, x, d);
        if (lane >= d) x += y;
    }
    return x;
}

}  // namespace sat
