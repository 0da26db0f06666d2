// sat_band.cuh -- the band kernel: single-pass SAT with decoupled look-back.
//
// This is the B200 realisation of the paper's 1R1W SAT algorithm
// (Sec. VI, Theorem 6; Fig. 11): every element is read
// once and written once.  The paper runs 2n/w-1 kernel launches, one per block
// anti-diagonal, and recovers each block's carries (C, R, S) from its
// neighbours' final SAT edges after the launch barrier.  Here ONE launch does
// everything:
//   * a CTA takes a band of TH rows (ticket order = band order, so every band
//     it waits on is held by a running or finished CTA) and walks it left to
//     right in TH x 128 chunks; a producer warp streams the chunks into an
//     S-slot shared-memory ring with TMA (cp.async.bulk.tensor);
//   * the horizontal carry (the paper's R) is the per-row running sum L held
//     in registers by the warp that owns the row;
//   * the vertical carry (the paper's C and S, i.e. the SAT row above the
//     band) comes from a decoupled look-back over self-validating descriptor
//     words: each (band, chunk) publishes the bottom row of its band-local SAT
//     as an "aggregate", then -- once it knows the SAT row above -- the final
//     SAT bottom row as "inclusive".  The look-back reads a
//     window of LBW bands per round trip;
//   * inside a chunk, Step 3-1/3-2 of 2R1W become: the compute
//     warps' local() = row scans with L + column prefix down the warp's R
//     rows; the result is parked in tensor memory (tcgen05.st) and the smem
//     slot is released at once; NCW control warps do the look-backs and turn
//     the carries into one add vector per warp (SAT row above the band +
//     bottom rows of the warps above); DT-1 chunks later the compute warp
//     takes its values back (tcgen05.ld), adds, and writes them to HBM with
//     coalesced 16-B stores.  The look-back latency is thus hidden by DT
//     chunks parked in TMEM instead of occupying the smem ring.
//
// The same kernel, with MODE/TopSrc switches, is the column pass and row pass
// of 2R2W, Step 3 of 2R1W with external carries
// and the 1R1W band (C) of (1+r)R1W.
//
// Roles (warps): 0..W-1 compute (R rows each), W..W+NCW-1 control
// (descriptors and look-back, in NCW/NS groups of NS warps that split a
// chunk's columns; group g owns the chunks k = g mod NCW/NS), W+NCW =
// producer (TMA loads, one elected lane).
#pragma once
#include "sat_common.h"
#include "sat_device.cuh"

namespace sat {

// The EPL consecutive elements a lane owns in a chunk row (16 B for 4-byte
// types at 128-column chunks and for float64 at 64-column chunks; 32 B for
// float64 at 128 columns), moved as whole vectors.
template <typename T, int N>
struct Vec { T e[N]; };

template <typename T, int N>
__device__ __forceinline__ void vec_words(const Vec<T, N>& v, uint32_t (&w)[N * Words<T>::N]) {
    pack<T, N>(v.e, w);
}
template <typename T, int N>
__device__ __forceinline__ Vec<T, N> ldsv(const T* p) {
    uint32_t w[N * Words<T>::N];
    ld_words<N * Words<T>::N>(p, w);
    Vec<T, N> v;
    unpack<T, N>(w, v.e);
    return v;
}
template <typename T, int N>
__device__ __forceinline__ void stsv(T* p, const Vec<T, N>& v) {
    uint32_t w[N * Words<T>::N];
    vec_words(v, w);
    st_words<N * Words<T>::N>(p, w);
}
// streaming store (evict-first: the SAT is not re-read by this kernel)
template <typename T, int N>
__device__ __forceinline__ void stgv(T* p, const Vec<T, N>& v) {
    uint32_t w[N * Words<T>::N];
    vec_words(v, w);
    stcs_words<N * Words<T>::N>(p, w);
}
template <typename T, int N>
__device__ __forceinline__ void addv(Vec<T, N>& a, const Vec<T, N>& b) {
#pragma unroll
    for (int i = 0; i < N; ++i) a.e[i] += b.e[i];
}
template <typename T, int N>
__device__ __forceinline__ Vec<T, N> zerov() {
    Vec<T, N> v;
#pragma unroll
    for (int i = 0; i < N; ++i) v.e[i] = T(0);
    return v;
}

// Input element -> arithmetic element for the lane's N consecutive columns
// in shared memory: the same type, or a narrower input widened on load (uint8
// pixels -> uint32 sums, the classic integral image; float32 -> float64 sums,
// an accurate float integral image).  DESIGN.md Sec. 4.8.
template <typename T, typename TI, int N>
__device__ __forceinline__ Vec<T, N> ldsv_in(const TI* p) {
    if constexpr (std::is_same<T, TI>::value) {
        return ldsv<T, N>(p);
    } else if constexpr (sizeof(TI) == 1) {
        static_assert(N == 4, "uint8 input: 4 pixels per lane");
        const uint32_t w = *reinterpret_cast<const uint32_t*>(p);
        return Vec<T, N>{{T(w & 255u), T((w >> 8) & 255u), T((w >> 16) & 255u), T(w >> 24)}};
    } else {
        const Vec<TI, N> a = ldsv<TI, N>(p);
        Vec<T, N> v;
#pragma unroll
        for (int i = 0; i < N; ++i) v.e[i] = T(a.e[i]);
        return v;
    }
}

// Shared-memory footprint of one configuration.
template <typename T, int R, int W, int S, int DT, int SUB, typename TI = T, int TWK = TW>
struct BandSmem {
    static constexpr int TH = R * W;
    static constexpr int XS = DT;                    // carry slots: one per parked chunk
    static constexpr size_t tile_elems = size_t(TH) * TWK;           // one TWK-column chunk
    static constexpr size_t slot_elems = tile_elems * SUB;           // one ring slot
    static constexpr size_t tiles = S * slot_elems * sizeof(TI);     // the ring holds input elements
    static constexpr size_t xbuf = size_t(XS) * W * TWK * sizeof(T);
    // + unit queue: ufull[2], uempty[2]
    static constexpr size_t nbars = 2 * S + 2 * XS + 4;
    // + s_unit[2], s_tmem, and per compute warp the (band, chunk) of each
    // parked chunk (finish() may run after the chunk's unit ended)
    static constexpr size_t bars = nbars * sizeof(uint64_t) + 32 + size_t(W) * DT * 8;
    static constexpr size_t total = tiles + xbuf + bars;
};

__device__ __forceinline__ uint32_t band_tag(unsigned long long base, int gb) {
    return uint32_t((base + (unsigned long long)gb) & 0x3FFFFFFFull) << 2;
}

// CPL consecutive columns (4, 2 or 1) as one shared-memory vector access.
template <typename T, int CPL>
__device__ __forceinline__ void lds_cols(const T* p, T (&v)[CPL]) {
    uint32_t w[CPL * Words<T>::N];
    ld_words<CPL * Words<T>::N>(p, w);
    unpack<T, CPL>(w, v);
}
template <typename T, int CPL>
__device__ __forceinline__ void sts_cols(T* p, const T (&v)[CPL]) {
    uint32_t w[CPL * Words<T>::N];
    pack<T, CPL>(v, w);
    st_words<CPL * Words<T>::N>(p, w);
}

// Descriptor words (tag << 32 | 32 value bits): NW consecutive words, each
// single-copy atomic at gpu scope (a float64 value is two words, low first).
template <int NW>
__device__ __forceinline__ void load_words(const uint64_t* q, uint64_t (&w)[NW]) {
    if constexpr (NW % 2 == 0) {
#pragma unroll
        for (int k = 0; k < NW; k += 2) ld_relaxed_v2(q + k, w[k], w[k + 1]);
    } else {
        static_assert(NW == 1, "1 or 2k words");
        asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(w[0]) : "l"(q) : "memory");
    }
}
template <typename T, int CPL>
__device__ __forceinline__ void publish_words(uint64_t* my, uint32_t tag, const T (&v)[CPL]) {
    constexpr int NW = CPL * Words<T>::N;
    const uint64_t hi = uint64_t(tag) << 32;
    uint32_t w[NW];
    pack<T, CPL>(v, w);
    if constexpr (NW % 2 == 0) {
#pragma unroll
        for (int k = 0; k < NW; k += 2) st_relaxed_v2(my + k, hi | w[k], hi | w[k + 1]);
    } else {
        asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" :: "l"(my), "l"(hi | w[0]) : "memory");
    }
}

// Row-wise inclusive prefix-sums of R rows of a chunk (lane owns N
// consecutive columns), continuing from the running row sums L, which are
// advanced to the end of the chunk.  Rows are interleaved step by step so the
// shuffles of different rows overlap.
template <typename T, int R, int N>
__device__ __forceinline__ void row_scan(Vec<T, N> (&v)[R], T (&L)[R], int lane) {
    T inc[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
#pragma unroll
        for (int i = 1; i < N; ++i) v[r].e[i] += v[r].e[i - 1];
        inc[r] = v[r].e[N - 1];
    }
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const T y = __shfl_up_sync(0xffffffffu, inc[r], d);
            if (lane >= d) inc[r] += y;
        }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
        T exc;
        if constexpr (std::is_same<T, uint32_t>::value) {
            exc = inc[r] - v[r].e[N - 1];          // exact in Z/2^32
        } else {
            exc = __shfl_up_sync(0xffffffffu, inc[r], 1);
            if (lane == 0) exc = T(0);
        }
        const T off = L[r] + exc;
#pragma unroll
        for (int i = 0; i < N; ++i) v[r].e[i] += off;
        L[r] += __shfl_sync(0xffffffffu, inc[r], 31);
    }
}

// ---------------------------------------------------------------- TMEM
// The band-local results of a chunk wait for their look-back in tensor memory
// (256 KB per SM, otherwise idle in a scan): each compute thread parks its
// R x 4 values in its own TMEM lane with one tcgen05.st and takes them back
// with one tcgen05.ld when the carries are known.  This keeps the look-back
// latency out of the shared-memory ring, which then only has to cover the
// HBM load latency.
template <int N>
__device__ __forceinline__ void tmem_st(uint32_t taddr, const uint32_t (&r)[N]);
template <int N>
__device__ __forceinline__ void tmem_ld(uint32_t taddr, uint32_t (&r)[N]);

template <>
__device__ __forceinline__ void tmem_st<8>(uint32_t t, const uint32_t (&r)[8]) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
                 :: "r"(t), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]),
                    "r"(r[6]), "r"(r[7]) : "memory");
}
template <>
__device__ __forceinline__ void tmem_ld<8>(uint32_t t, uint32_t (&r)[8]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]),
                   "=r"(r[6]), "=r"(r[7]) : "r"(t) : "memory");
}
template <>
__device__ __forceinline__ void tmem_st<16>(uint32_t t, const uint32_t (&r)[16]) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,"
                 "%9,%10,%11,%12,%13,%14,%15,%16};"
                 :: "r"(t), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]),
                    "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]),
                    "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]) : "memory");
}
template <>
__device__ __forceinline__ void tmem_ld<16>(uint32_t t, uint32_t (&r)[16]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,"
                 "%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]),
                   "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]),
                   "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]) : "r"(t) : "memory");
}
template <>
__device__ __forceinline__ void tmem_st<32>(uint32_t t, const uint32_t (&r)[32]) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,"
                 "%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,"
                 "%27,%28,%29,%30,%31,%32};"
                 :: "r"(t), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]),
                    "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]),
                    "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]),
                    "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]),
                    "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]),
                    "r"(r[30]), "r"(r[31]) : "memory");
}
template <>
__device__ __forceinline__ void tmem_ld<32>(uint32_t t, uint32_t (&r)[32]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,"
                 "%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,"
                 "%28,%29,%30,%31}, [%32];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]),
                   "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]),
                   "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]),
                   "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
                   "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]),
                   "=r"(r[30]), "=r"(r[31]) : "r"(t) : "memory");
}
template <>
__device__ __forceinline__ void tmem_st<64>(uint32_t t, const uint32_t (&r)[64]) {
    // two x32 stores into adjacent column ranges
    uint32_t a[32], b[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) { a[i] = r[i]; b[i] = r[32 + i]; }
    tmem_st<32>(t, a);
    tmem_st<32>(t + 32, b);
}
template <>
__device__ __forceinline__ void tmem_ld<64>(uint32_t t, uint32_t (&r)[64]) {
    uint32_t a[32], b[32];
    tmem_ld<32>(t, a);
    tmem_ld<32>(t + 32, b);
#pragma unroll
    for (int i = 0; i < 32; ++i) { r[i] = a[i]; r[32 + i] = b[i]; }
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tmem_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// TMEM columns per CTA for W compute warps holding DT chunks of R x EPL
// elements of NWE 32-bit words each.
template <int R, int W, int DT, int NWE = 1, int EPL = 4>
struct TmemCols {
    static constexpr int per_chunk = EPL * R * NWE;
    static constexpr int per_warp = DT * per_chunk;
    static constexpr int need = per_warp * ((W + 3) / 4);       // warps w, w+4, .. share lanes
    static constexpr int alloc = need <= 32 ? 32 : need <= 64 ? 64 : need <= 128 ? 128
                                 : need <= 256 ? 256 : 512;
    static_assert(need <= 512, "TMEM holds at most 512 columns");
};

// ---------------------------------------------------------------- column-sum seed
// (sharded mode; sat_common.h ColSeed).  Waits for the producers' flags when
// the vectors live in a peer-exchange mailbox (sat_xchg.cuh).
__device__ __forceinline__ void colseed_wait(const ColSeed& cs) {
    if (cs.flags == nullptr) return;
    for (int q = 0; q < cs.n; ++q) {
        uint64_t v;
        asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(cs.flags + q) : "memory");
        if (v >= cs.epoch) continue;
        SpinGuard guard(0x18000000u | uint32_t(q), uint32_t(cs.epoch));
        do {
            __nanosleep(128);
            guard.tick();
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(cs.flags + q) : "memory");
        } while (v < cs.epoch);
    }
}
// sum_{q < n} vec_q[c .. c+N-1] in q order (columns >= cols read as 0);
// volatile loads: the vectors may have been written over NVLink by another GPU
template <typename T, int N>
__device__ __forceinline__ Vec<T, N> colseedv(const ColSeed& cs, int64_t c, int64_t cols) {
    Vec<T, N> s = zerov<T, N>();
    for (int q = 0; q < cs.n; ++q) {
        const volatile T* v = reinterpret_cast<const volatile T*>(
            reinterpret_cast<const uint8_t*>(cs.base) + int64_t(q) * cs.stride);
#pragma unroll
        for (int i = 0; i < N; ++i)
            if (c + i < cols) s.e[i] += v[c + i];
    }
    return s;
}

template <typename T, int R, int W, int S, int DT, int SUB, int NCW, int NS, int MODE, bool TMA, int MINB,
          int LBW_ = 0, typename TI = T, int TWK = TW>
__global__ void __launch_bounds__((W + NCW + 1) * 32, MINB)
sat_band_kernel(const __grid_constant__ CUtensorMap tm_in,
                const BandParams p)
{
    constexpr int TH = R * W;
    constexpr int EPL = TWK / 32;  // elements per lane in a chunk row
    static_assert(TWK % 32 == 0 && EPL * sizeof(T) >= 16, "a lane moves at least 16 B per chunk row");
    constexpr int CW = W;          // first control warp
    constexpr int PW = W + NCW;    // producer warp
    constexpr uint32_t TILE_BYTES = uint32_t(TH) * TWK * sizeof(TI);
    using SM = BandSmem<T, R, W, S, DT, SUB, TI, TWK>;
    static_assert(std::is_same<T, TI>::value || MODE == MODE_SAT, "widening input: 1R1W only");
    constexpr int NWE = Words<T>::N;             // 32-bit words per element
    using TC = TmemCols<R, W, DT, NWE, EPL>;
    constexpr int XS = SM::XS;
    constexpr bool HOLD = (MODE != MODE_ROW);    // chunks wait for a vertical carry
    // A control warp waits on colr[] of chunk k only after finishing chunk
    // k-NCW, which implies local(k-XS) completed iff NCW <= XS; otherwise the
    // parity wait could pass on a stale phase.
    static_assert(NCW % NS == 0 && (NS == 1 || NS == 2 || NS == 4), "control warps split columns 1, 2 or 4 ways");
    static_assert(NCW / NS <= XS, "more control groups than carry slots");

    extern __shared__ __align__(1024) uint8_t smem[];
    TI* tiles = reinterpret_cast<TI*>(smem);
    T* xbuf = reinterpret_cast<T*>(smem + SM::tiles);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + SM::tiles + SM::xbuf);
    uint64_t* full = bars;              // [S]  TMA load landed (tx count)
    uint64_t* empty = bars + S;         // [S]  every compute warp read the slot
    uint64_t* colr = bars + 2 * S;      // [XS] every compute warp published its bottom row
    uint64_t* topr = bars + 2 * S + XS; // [XS] the control warp wrote the add vectors
    // unit queue: the producer warp takes the next ticket
    // as soon as it has issued the last load of the current unit and posts it
    // in s_unit[u & 1] (ufull); the other warps read it and release the entry
    // (uempty), so the next unit's loads overlap the current unit's last
    // look-backs and stores
    uint64_t* ufull = bars + 2 * S + 2 * XS;
    uint64_t* uempty = ufull + 2;
    long long* s_unit = reinterpret_cast<long long*>(bars + SM::nbars);
    uint32_t* s_tmem = reinterpret_cast<uint32_t*>(s_unit + 2);
    int2* meta = reinterpret_cast<int2*>(s_unit + 4);   // [W][DT]

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], W * 32);
        }
        for (int u = 0; u < 2; ++u) {
            mbar_init(&ufull[u], 1);
            mbar_init(&uempty[u], W + NCW);      // lane 0 of every non-producer warp
        }
        for (int x = 0; x < XS; ++x) {
            mbar_init(&colr[x], W * 32);
            mbar_init(&topr[x], 32 * NS);
        }
        fence_mbar_init();
    }
    if (HOLD && warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(smem_u32(s_tmem)), "r"(TC::alloc) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    if (TMA && warp == PW && lane == 0) prefetch_tmap(&tm_in);
    tmem_fence_before();
    __syncthreads();
    tmem_fence_after();
    const uint32_t tmem_base = HOLD ? *s_tmem : 0u;
    // Programmatic dependent launch: everything above is CTA-local and may
    // overlap the previous kernel's tail; global memory from here on (a
    // no-op when launched without the attribute)
    asm volatile("griddepcontrol.wait;" ::: "memory");
    // ticket/tag base: the host's counter, or (CUDA-graph capture, DESIGN.md
    // Sec. 4) the value sat_epoch_kernel wrote just before this launch
    const unsigned long long kbase = p.base_dev ? __ldcg(p.base_dev) : p.base;

    const int64_t img_elems = p.rows * p.cols;
    const int desc_w = p.nc * TWK;
    const int64_t lx_stride = int64_t(p.total_bands) * TH;
    uint32_t g = 0;                              // CTA-local chunk counter (carry / TMEM slots)
    uint32_t gq = 0;                             // CTA-local ring-slot counter (SUB chunks per slot)
    // compute warps: this warp's rows in a band, TMEM lanes (32*(warp%4) ..)
    // and column range, parked-chunk metadata
    const int rbase = warp * R;
    const uint32_t tm_warp = tmem_base + ((uint32_t(32 * (warp & 3))) << 16)
                             + uint32_t((warp >> 2) * TC::per_warp);
    int2* wmeta = meta + (warp < W ? warp : 0) * DT;
    // finish(it) of the CTA-global chunk stream: + (SAT row above the band +
    // bottom rows of the warps above), from the add vector the control warp
    // left in xbuf, then the 1W.  Runs DT-1 chunks after local(it) -- across
    // unit boundaries, so the look-back of a unit's last chunks overlaps the
    // next unit's first chunks instead of stalling the compute warps.
    auto finish_it = [&](uint32_t it) {
        const int2 md = wmeta[it % DT];
        const int fgb = md.x, fJ = md.y;
        const int fimg = fgb / p.nb;
        const int frow0 = (fgb - fimg * p.nb) * TH;
        T* fout = reinterpret_cast<T*>(p.out) + int64_t(fimg) * (p.rows * p.cols);
        mbar_wait(&topr[it % XS], (it / XS) & 1);
        if constexpr (kDebug) {
            if (p.trace != nullptr && warp == 0 && lane == 0)
                p.trace[(int64_t(fgb) * p.nc + fJ) * 8 + 6] = globaltimer();
        }
        const Vec<T, EPL> add = ldsv<T, EPL>(xbuf + (size_t(it % XS) * W + warp) * TWK + EPL * lane);
        uint32_t u[TC::per_chunk];
        tmem_wait_st();
        tmem_ld<TC::per_chunk>(tm_warp + uint32_t((it % DT) * TC::per_chunk), u);
        tmem_wait_ld();
        const int64_t c = int64_t(fJ) * TWK + EPL * lane;
#pragma unroll
        for (int r = 0; r < R; ++r) {
            Vec<T, EPL> v;
#pragma unroll
            for (int i = 0; i < EPL; ++i) v.e[i] = from_words<T>(u + (EPL * r + i) * NWE);
            addv(v, add);
            const int64_t row = frow0 + rbase + r;
            if (row < p.rows) {
                if constexpr (TMA) {
                    if (c < p.cols) stgv(fout + row * p.cols + c, v);
                } else {
#pragma unroll
                    for (int i = 0; i < EPL; ++i)
                        if (c + i < p.cols) fout[row * p.cols + c + i] = v.e[i];
                }
            }
        }
        if constexpr (kDebug) {
            if (p.trace != nullptr && warp == 0 && lane == 0)
                p.trace[(int64_t(fgb) * p.nc + fJ) * 8 + 3] = globaltimer();
        }
    };

    for (uint32_t useq = 0;; ++useq) {
        long long unit;
        {
            const uint32_t qs = useq & 1u, qph = (useq >> 1) & 1u;
            if (warp == PW) {
                if (lane == 0) {
                    if (useq >= 2) mbar_wait(&uempty[qs], qph ^ 1u);   // every warp read unit useq-2
                    s_unit[qs] = (long long)(atomicAdd(p.ticket, 1ull) - kbase);
                    mbar_arrive(&ufull[qs]);
                }
                __syncwarp();
                mbar_wait(&ufull[qs], qph);
            } else {
                mbar_wait(&ufull[qs], qph);
            }
            unit = s_unit[qs];
            __syncwarp();
            if (warp != PW && lane == 0) mbar_arrive(&uempty[qs]);
        }
        diag_mark(p.diag, uint32_t(unit), 0, 1);
        if (unit < 0) __trap();                       // ticket accounting out of sync: never silently
        if (unit >= p.total_units) break;

        int gb, j0, j1;
        int seg = 0;                                   // band segment (p.nseg > 1)
        if (p.tile_units) {
            // ranges of tile_units chunks of a band's region (external
            // carries: the row carry at the range start comes from Lx)
            const int per = (p.nc + p.tile_units - 1) / p.tile_units;
            gb = int(unit / per);
            const int sr = int(unit % per);
            int r0, r1;
            region_range(p.region, p.tA, p.nb, p.nc, gb % p.nb, r0, r1);
            j0 = min(r1, r0 + sr * p.tile_units);
            j1 = min(r1, j0 + p.tile_units);
        } else if (p.nseg > 1) {
            if (p.order != nullptr) {
                const int2 u = __ldg(p.order + unit);
                seg = u.x;
                gb = u.y;
            } else {
                seg = int(unit / p.total_bands);
                gb = int(unit - (long long)seg * p.total_bands);
            }
            j0 = seg * p.segc;
            j1 = min(p.nc, j0 + p.segc);
        } else {
            gb = int(unit);
            region_range(p.region, p.tA, p.nb, p.nc, gb % p.nb, j0, j1);
        }
        const int img = gb / p.nb;
        const int band = gb - img * p.nb;
        const int nch = j1 - j0;
        const int row0 = band * TH;
        const bool traced = kDebug && p.trace != nullptr;
        (void)traced;

        if (warp < W) {
            // ================= compute warps =================
            // column-sum seed: added to the strip's first row (warp 0, row 0)
            const bool seeded = p.cseed.n > 0 && gb == 0 && warp == 0;
            if (seeded) colseed_wait(p.cseed);
            T L[R];
#pragma unroll
            for (int r = 0; r < R; ++r) L[r] = T(0);
            if (p.Lx != nullptr) {
                const T* lx = reinterpret_cast<const T*>(p.Lx) + int64_t(j0) * lx_stride
                              + int64_t(gb) * TH + rbase;
#pragma unroll
                for (int r = 0; r < R; ++r) L[r] = lx[r];
            }
            if (seg > 0) {
                // row carry from segment seg-1 of this band (an earlier ticket,
                // normally long finished): lane r < R polls row rbase + r
                const uint32_t want = band_tag(kbase, (seg - 1) * p.total_bands + gb) | 3u;
                const bool mine = lane < R * NWE;        // word `lane` of this warp's rows
                const uint64_t* q = p.Lseg + (int64_t(gb) * TH + rbase) * NWE + (mine ? lane : 0);
                uint64_t wv;
                asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(wv) : "l"(q) : "memory");
                if (__any_sync(0xffffffffu, mine && uint32_t(wv >> 32) != want)) {
                    SpinGuard guard(0x20000000u | uint32_t(gb), uint32_t(seg));
                    while (__any_sync(0xffffffffu, mine && uint32_t(wv >> 32) != want)) {
                        __nanosleep(64);
                        guard.tick();
                        asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(wv) : "l"(q) : "memory");
                    }
                }
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    uint32_t w[NWE];
#pragma unroll
                    for (int k = 0; k < NWE; ++k) w[k] = __shfl_sync(0xffffffffu, uint32_t(wv), r * NWE + k);
                    L[r] = from_words<T>(w);
                }
            }
            const TI* gin = reinterpret_cast<const TI*>(p.in) + int64_t(img) * img_elems;
            T* gout = reinterpret_cast<T*>(p.out) + int64_t(img) * img_elems;

            // store R rows of 4 values to the output (16-B vectors on the TMA
            // path, where cols % 4 == 0; guarded scalars otherwise)
            auto store_rows = [&](const Vec<T, EPL> (&v)[R], int k) {
                const int64_t c = int64_t(j0 + k) * TWK + EPL * lane;
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    const int64_t row = row0 + rbase + r;
                    if (row < p.rows) {
                        if constexpr (TMA) {
                            if (c < p.cols) stgv(gout + row * p.cols + c, v[r]);
                        } else {
#pragma unroll
                            for (int i = 0; i < EPL; ++i)
                                if (c + i < p.cols) gout[row * p.cols + c + i] = v[r].e[i];
                        }
                    }
                }
            };

            // local(k): row scans with L, column prefix down this warp's rows;
            // park the result in TMEM, warp bottom row into xbuf
            auto local = [&](int k) {
                const uint32_t it = g + k;
                Vec<T, EPL> v[R];
                Vec<T, EPL> sd;
                if (seeded) sd = colseedv<T, EPL>(p.cseed, int64_t(j0 + k) * TWK + EPL * lane, p.cols);
                if constexpr (TMA) {
                    const uint32_t q = gq + uint32_t(k / SUB);     // ring slot of chunk k
                    const int s = q % S;
                    if (k % SUB == 0) mbar_wait(&full[s], (q / S) & 1);
                    if constexpr (kDebug) {
                        if (traced && warp == 0 && lane == 0)
                        {
                            p.trace[(int64_t(gb) * p.nc + j0 + k) * 8 + 0] = globaltimer();
                            uint32_t smid, nsm;
                            asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
                            asm volatile("mov.u32 %0, %%nsmid;" : "=r"(nsm));
                            p.trace[(int64_t(gb) * p.nc + j0 + k) * 8 + 7] = (uint64_t(blockIdx.x) << 32) | smid;
                        }
                    }
                    {
                        const TI* t = tiles + size_t(s) * SM::slot_elems + size_t(k % SUB) * SM::tile_elems
                                      + size_t(rbase) * TWK + EPL * lane;
#pragma unroll
                        for (int r = 0; r < R; ++r) v[r] = ldsv_in<T, TI, EPL>(t + r * TWK);
                    }
                    if (k % SUB == SUB - 1 || k == nch - 1) {
                        // release the slot to the next TMA write only once the
                        // generic-proxy reads have landed in registers (the
                        // asm consumes them) and are ordered before the async
                        // proxy: without this, a quick refill overtook the LDS
                        // (seen as corrupted rows with 4 compute warps)
#pragma unroll
                        for (int r = 0; r < R; ++r) {
                            uint32_t w[EPL * NWE];
                            vec_words(v[r], w);
#pragma unroll
                            for (int k = 0; k < EPL * NWE; ++k) asm volatile("" :: "r"(w[k]));
                        }
                        fence_proxy_async_smem();
                        mbar_arrive(&empty[s]);
                    }
                } else {
                    const int64_t c = int64_t(j0 + k) * TWK + EPL * lane;
#pragma unroll
                    for (int r = 0; r < R; ++r) {
                        const int64_t row = row0 + rbase + r;
#pragma unroll
                        for (int i = 0; i < EPL; ++i)
                            v[r].e[i] = (row < p.rows && c + i < p.cols) ? T(gin[row * p.cols + c + i]) : T(0);
                    }
                }
                if (seeded) addv(v[0], sd);
                if constexpr (MODE != MODE_COL) row_scan<T, R, EPL>(v, L, lane);
                if constexpr (!HOLD) {
                    store_rows(v, k);                    // the row pass is final
                } else {
#pragma unroll
                    for (int r = 1; r < R; ++r) addv(v[r], v[r - 1]);
                    uint32_t u[TC::per_chunk];
#pragma unroll
                    for (int r = 0; r < R; ++r)
#pragma unroll
                        for (int i = 0; i < EPL; ++i) to_words<T>(v[r].e[i], u + (EPL * r + i) * NWE);
                    tmem_st<TC::per_chunk>(tm_warp + uint32_t((it % DT) * TC::per_chunk), u);
                    stsv(xbuf + (size_t(it % XS) * W + warp) * TWK + EPL * lane, v[R - 1]);
                    if (lane == 0) wmeta[it % DT] = make_int2(gb, j0 + k);
                    mbar_arrive(&colr[it % XS]);
                }
            };
            if constexpr (!HOLD) {
                for (int k = 0; k < nch; ++k) local(k);
            } else {
                for (int k = 0; k < nch; ++k) {
                    local(k);
                    diag_mark(p.diag, uint32_t(unit), uint32_t(k), 2);
                    if (g + k >= uint32_t(DT - 1)) finish_it(g + k - (DT - 1));
                    diag_mark(p.diag, uint32_t(unit), uint32_t(k), 3);
                }
            }
            if (seeded && p.cseed.acks != nullptr) {
                // every seed vector this unit needed has been read (the values
                // are in the stored results); the last band-0 unit (segments)
                // acknowledges to the producers (sat_xchg.cuh)
                __syncwarp();
                if (lane == 0) {
                    __threadfence();
                    const unsigned int n = atomicAdd(p.cseed.done, 1u);
                    if (n + 1 == unsigned(p.nseg > 1 ? p.nseg : 1)) {
                        *p.cseed.done = 0u;
#pragma unroll 1
                        for (int q = 0; q < p.cseed.n; ++q)
                            asm volatile("st.release.sys.global.u64 [%0], %1;"
                                         :: "l"(p.cseed.acks[q]), "l"(uint64_t(p.cseed.epoch)) : "memory");
                    }
                }
            }
            if (p.nseg > 1 && seg + 1 < p.nseg && lane < R * NWE) {
                // hand the row carry to segment seg+1 of this band (word `lane`)
                uint32_t wl[R * NWE];
                pack<T, R>(L, wl);
                uint32_t mine = wl[0];
#pragma unroll
                for (int k = 1; k < R * NWE; ++k) if (lane == k) mine = wl[k];
                const uint64_t w = (uint64_t(band_tag(kbase, seg * p.total_bands + gb) | 3u) << 32) | mine;
                asm volatile("st.relaxed.gpu.global.b64 [%0], %1;"
                             :: "l"(p.Lseg + (int64_t(gb) * TH + rbase) * NWE + lane), "l"(w) : "memory");
            }
            if (p.Lb != nullptr && !p.tile_units && lane == 0) {
                T* lb = reinterpret_cast<T*>(p.Lb) + int64_t(gb) * TH + rbase;
#pragma unroll
                for (int r = 0; r < R; ++r) lb[r] = L[r];
            }
        } else if (warp < PW) {
            // ================= control warps: descriptors + look-back =================
            // NCW warps form G = NCW/NS groups; group g owns the chunks
            // k = g mod G and its NS warps split the 128 columns (CPL per
            // lane), so one round trip reads LBW = 16/CPL bands' words in the
            // same 32 registers per lane.
            if constexpr (HOLD) {
                constexpr int CPL = EPL / NS;
                constexpr int G = NCW / NS;
                constexpr int NW = CPL * NWE;                  // descriptor words per band
                constexpr int LBW = LBW_ > 0 ? LBW_ : (16 / NW > 0 ? 16 / NW : 1);   // bands per round trip
                const int cw = warp - CW;
                const int grp = cw / NS;
                const int cl = (cw % NS) * (TWK / NS) + lane * CPL;  // column within the chunk
                const uint32_t tagbase = band_tag(kbase, gb);
                const bool lookback = (p.top_src == TOP_LOOKBACK);
                const bool publish = lookback && band + 1 < p.nb;   // the last band is never read
                const T* gout = reinterpret_cast<const T*>(p.out) + int64_t(img) * img_elems;
                // group grp owns the CTA-global chunks it = g + k with it = grp
                // (mod G), across unit boundaries: consecutive chunks of a
                // group are exactly G <= XS apart, so its parity waits on
                // colr[] can never pass on a stale phase (with the unit queue
                // the next unit starts before every group finished this one)
                for (int k = int((uint32_t(grp) + uint32_t(G) - g % uint32_t(G)) % uint32_t(G)); k < nch; k += G) {
                    const uint32_t it = g + k;
                    const int J = j0 + k;
                    const int c0 = J * TWK + cl;
                    T* xb = xbuf + size_t(it % XS) * W * TWK + cl;
                    mbar_wait(&colr[it % XS], (it / XS) & 1);
                    if constexpr (kDebug) {
                        if (traced && cw == grp * NS && lane == 0)
                            p.trace[(int64_t(gb) * p.nc + J) * 8 + 1] = globaltimer();
                    }
                    T agg[CPL];
                    lds_cols<T, CPL>(xb, agg);
#pragma unroll
                    for (int w2 = 1; w2 < W; ++w2) {
                        T b[CPL];
                        lds_cols<T, CPL>(xb + w2 * TWK, b);
#pragma unroll
                        for (int i = 0; i < CPL; ++i) agg[i] += b[i];
                    }
                    uint64_t* my = p.desc + (int64_t(gb) * desc_w + c0) * NWE;
                    if (p.jitter && lookback) {
                        uint32_t h = (uint32_t(gb) * 2654435761u) ^ (uint32_t(J) * 40503u) ^ (uint32_t(cl) * 97u);
                        h ^= h >> 13; h *= 0x5bd1e995u; h ^= h >> 15;
                        __nanosleep(h % (uint32_t)p.jitter);
                    }
                    T top[CPL];
#pragma unroll
                    for (int i = 0; i < CPL; ++i) top[i] = T(0);
                    unsigned long long hops = 0, polls = 0;
                    if (publish && band > 0) publish_words<T, CPL>(my, tagbase | 1u, agg);
                    if (!lookback) {
                        lds_cols<T, CPL>(reinterpret_cast<const T*>(p.TopX) + int64_t(gb) * desc_w + c0, top);
                    } else if (band == 0) {
                        if (p.seed_kind != SEED_NONE && img == 0) {
                            // the SAT row just above the matrix (seeded mode)
                            const T* sd = reinterpret_cast<const T*>(p.seed);
#pragma unroll
                            for (int i = 0; i < CPL; ++i) top[i] = (c0 + i < p.cols) ? sd[c0 + i] : T(0);
                        }
                    } else {
                        // decoupled look-back over bands band-1, band-2, ...,
                        // LBW descriptor rows per round trip: adds the SAT row
                        // above this band to top.  Hierarchical (p.hg > 0,
                        // DESIGN.md Sec. 4.13): band by band only down to the
                        // first band g0 of this band's group, then one group
                        // word per group above (phase 2 below)
                        constexpr uint32_t kAll = (1u << CPL) - 1u;
                        uint32_t pend = kAll;
                        const int g0 = p.hg > 0 ? band - band % p.hg : 0;
                        int kb = band - 1;
                        SpinGuard guard(0x80000000u | uint32_t(J), uint32_t(gb));
                        while (pend && kb >= g0) {
                            uint64_t wv[LBW][NW];
#pragma unroll
                            for (int q = 0; q < LBW; ++q) {
                                const int b2 = kb - q;
                                if (b2 >= g0) {
                                    load_words<NW>(p.desc + ((int64_t(gb) - (band - b2)) * desc_w + c0) * NWE, wv[q]);
                                } else {
#pragma unroll
                                    for (int i = 0; i < NW; ++i) wv[q][i] = 0;
                                }
                            }
                            bool stalled = false;
#pragma unroll
                            for (int q = 0; q < LBW; ++q) {
                                if (!pend || stalled) break;
                                const int b2 = kb - q;
                                if (b2 < g0) break;
                                if (p.region == REG_C && b2 + J < p.tA) {
                                    // tile (b2, J) belongs to (A): its final SAT row is in `out`
                                    const int64_t row = int64_t(b2 + 1) * TH - 1;
#pragma unroll
                                    for (int i = 0; i < CPL; ++i)
                                        if ((pend >> i) & 1u)
                                            top[i] += (c0 + i < p.cols) ? gout[row * p.cols + c0 + i] : T(0);
                                    pend = 0;
                                    break;
                                }
                                const uint32_t tk = band_tag(kbase, gb - (band - b2));
                                bool ready = true;
#pragma unroll
                                for (int i = 0; i < NW; ++i) {
                                    const uint32_t t = uint32_t(wv[q][i] >> 32);
                                    ready = ready && ((t & ~3u) == tk) && (t & 3u);
                                }
                                // the words of one float64 value must come from the
                                // same publication (aggregate and inclusive share a slot)
#pragma unroll
                                for (int i = 0; i < CPL; ++i)
#pragma unroll
                                    for (int k = 1; k < NWE; ++k)
                                        ready = ready && (uint32_t(wv[q][i * NWE + k] >> 32) == uint32_t(wv[q][i * NWE] >> 32));
                                if (!ready) { stalled = true; kb = b2; break; }
#pragma unroll
                                for (int i = 0; i < CPL; ++i) {
                                    if ((pend >> i) & 1u) {
                                        uint32_t w[NWE];
#pragma unroll
                                        for (int k = 0; k < NWE; ++k) w[k] = uint32_t(wv[q][i * NWE + k]);
                                        top[i] += from_words<T>(w);
                                        if ((uint32_t(wv[q][i * NWE] >> 32) & 3u) == 2u) pend &= ~(1u << i);
                                    }
                                }
                                ++hops;
                            }
                            if (stalled) { __nanosleep(32); guard.tick(); ++polls; }
                            else kb -= LBW;
                        }
                        if (p.hg > 0 && pend) {
                            // phase 2: every band g0 .. band-1 was an aggregate
                            const int grpi = band / p.hg;
                            const int64_t gimg = int64_t(img) * p.ngroups;
                            // the group's last band publishes the group aggregate
                            // (sum of its bands' aggregates) before walking on, so
                            // the bands below never wait on a chain of inclusives
                            if (publish && band == g0 + p.hg - 1 && pend == kAll) {
                                T ga[CPL];
#pragma unroll
                                for (int i = 0; i < CPL; ++i) ga[i] = top[i] + agg[i];
                                publish_words<T, CPL>(p.gdesc + ((gimg + grpi) * desc_w + c0) * NWE, tagbase | 1u, ga);
                            }
                            // group 0's word always ends inclusive (its walk meets
                            // band 0), so the walk stops at kg >= 0
                            int kg = grpi - 1;
                            while (pend) {
                                uint64_t wv[LBW][NW];
#pragma unroll
                                for (int q = 0; q < LBW; ++q) {
                                    const int g2 = kg - q;
                                    if (g2 >= 0) {
                                        load_words<NW>(p.gdesc + ((gimg + g2) * desc_w + c0) * NWE, wv[q]);
                                    } else {
#pragma unroll
                                        for (int i = 0; i < NW; ++i) wv[q][i] = 0;
                                    }
                                }
                                bool stalled = false;
#pragma unroll
                                for (int q = 0; q < LBW; ++q) {
                                    if (!pend || stalled) break;
                                    const int g2 = kg - q;
                                    const uint32_t tk = band_tag(kbase, gb - band + g2 * p.hg + p.hg - 1);
                                    bool ready = true;
#pragma unroll
                                    for (int i = 0; i < NW; ++i) {
                                        const uint32_t t = uint32_t(wv[q][i] >> 32);
                                        ready = ready && ((t & ~3u) == tk) && (t & 3u);
                                    }
#pragma unroll
                                    for (int i = 0; i < CPL; ++i)
#pragma unroll
                                        for (int k = 1; k < NWE; ++k)
                                            ready = ready && (uint32_t(wv[q][i * NWE + k] >> 32) == uint32_t(wv[q][i * NWE] >> 32));
                                    if (!ready) { stalled = true; kg = g2; break; }
#pragma unroll
                                    for (int i = 0; i < CPL; ++i) {
                                        if ((pend >> i) & 1u) {
                                            uint32_t w[NWE];
#pragma unroll
                                            for (int k = 0; k < NWE; ++k) w[k] = uint32_t(wv[q][i * NWE + k]);
                                            top[i] += from_words<T>(w);
                                            if ((uint32_t(wv[q][i * NWE] >> 32) & 3u) == 2u) pend &= ~(1u << i);
                                        }
                                    }
                                    ++hops;
                                }
                                if (stalled) { __nanosleep(32); guard.tick(); ++polls; }
                                else kg -= LBW;
                            }
                        }
                    }
                    if (publish) {
                        T inc[CPL];
#pragma unroll
                        for (int i = 0; i < CPL; ++i) inc[i] = agg[i] + top[i];
                        publish_words<T, CPL>(my, tagbase | 2u, inc);
                        // the group's last band: its inclusive is the group's
                        if (p.hg > 0 && (band + 1) % p.hg == 0)
                            publish_words<T, CPL>(p.gdesc + ((int64_t(img) * p.ngroups + band / p.hg) * desc_w + c0) * NWE,
                                                  tagbase | 2u, inc);
                    }
                    if constexpr (kDebug) {
                        if (traced && cw == grp * NS && lane == 0)
                            p.trace[(int64_t(gb) * p.nc + J) * 8 + 2] =
                                (globaltimer() & 0xFFFFFFFFFFFFull) | (min(hops, 255ull) << 48) | (min(polls, 255ull) << 56);
                    }
                    (void)hops; (void)polls;
                    // add vectors for finish(): top + bottom rows of the warps above
#pragma unroll
                    for (int w2 = 0; w2 < W; ++w2) {
                        T b[CPL];
                        lds_cols<T, CPL>(xb + w2 * TWK, b);
                        sts_cols<T, CPL>(xb + w2 * TWK, top);
#pragma unroll
                        for (int i = 0; i < CPL; ++i) top[i] += b[i];
                    }
                    mbar_arrive(&topr[it % XS]);
                    diag_mark(p.diag, uint32_t(unit), uint32_t(k), 4);
                }
            }
        } else {
            // ================= producer warp: TMA load ring =================
            if constexpr (TMA) {
                if (lane == 0) {
                    const uint64_t pol = policy_evict_first();
                    for (int k0 = 0; k0 < nch; k0 += SUB) {
                        const uint32_t q = gq + uint32_t(k0 / SUB);
                        const int s = q % S;
                        const int nsub = nch - k0 < SUB ? nch - k0 : SUB;
                        if (q >= uint32_t(S)) mbar_wait(&empty[s], ((q / S) & 1) ^ 1u);
                        if constexpr (kDebug) {
                            if (traced) p.trace[(int64_t(gb) * p.nc + j0 + k0) * 8 + 4] = globaltimer();
                        }
                        mbar_arrive_expect_tx(&full[s], TILE_BYTES * nsub);
                        for (int j = 0; j < nsub; ++j)   // adjacent boxes: SUB*512 B per row
                            tma_load_3d(tiles + size_t(s) * SM::slot_elems + size_t(j) * SM::tile_elems,
                                        &tm_in, &full[s], (j0 + k0 + j) * TWK, row0, img, pol);
                    }
                }
            }
        }
        diag_mark(p.diag, uint32_t(unit), uint32_t(nch), 5);
        g += nch;
        gq += uint32_t((nch + SUB - 1) / SUB);
    }
    if constexpr (HOLD) {
        // the last DT-1 parked chunks of the stream
        if (warp < W)
            for (uint32_t it = g > uint32_t(DT - 1) ? g - (DT - 1) : 0u; it < g; ++it) finish_it(it);
    }
    diag_mark(p.diag, 0xFFFFFFFFu, 0, 6);
    if (HOLD) {
        tmem_fence_before();
        __syncthreads();
        tmem_fence_after();
        if (warp == 0)
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;"
                         :: "r"(tmem_base), "r"(TC::alloc) : "memory");
    }
}

}  // namespace sat
