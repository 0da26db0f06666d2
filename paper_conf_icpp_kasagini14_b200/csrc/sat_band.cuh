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
//     right in TH x 128 chunks staged through a TMA ring in shared memory;
//   * the horizontal carry (the paper's R) is the per-row running sum L held
//     in registers by the warp that owns the row;
//   * the vertical carry (the paper's C and S, i.e. the SAT row above the
//     band) comes from a decoupled look-back over flag-guarded descriptors:
//     each (band, chunk) publishes the bottom row of its band-local SAT as an
//     "aggregate", then -- once it knows the SAT row above -- the final SAT
//     bottom row as "inclusive";
//   * inside a chunk, Step 3-1/3-2 of 2R1W become: row scan
//     (in-thread + warp shuffle) with L, column prefix down the warp's R rows,
//     a cross-warp exchange of warp bottom rows, then + (SAT row above).
//
// The same kernel, with MODE/TopSrc switches, is the column pass and row pass
// of 2R2W, Step 3 of 2R1W with external carries
// and the 1R1W band (C) of (1+r)R1W.
//
// Roles (warps): 0..W-1 compute (R rows each), W = control (descriptors,
// look-back), W+1 = producer (TMA loads and stores, one elected lane).
#pragma once
#include "sat_common.h"
#include "sat_device.cuh"

namespace sat {

template <typename T>
struct V4 { T x, y, z, w; };

template <typename T>
__device__ __forceinline__ V4<T> lds4(const T* p) {
    uint4 u = *reinterpret_cast<const uint4*>(p);
    return V4<T>{from_bits<T>(u.x), from_bits<T>(u.y), from_bits<T>(u.z), from_bits<T>(u.w)};
}
template <typename T>
__device__ __forceinline__ void sts4(T* p, const V4<T>& v) {
    *reinterpret_cast<uint4*>(p) = make_uint4(to_bits(v.x), to_bits(v.y), to_bits(v.z), to_bits(v.w));
}
template <typename T>
__device__ __forceinline__ void add4(V4<T>& a, const V4<T>& b) {
    a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
}

// Shared-memory footprint of one configuration.
template <typename T, int R, int W, int S>
struct BandSmem {
    static constexpr int TH = R * W;
    static constexpr size_t tile_elems = size_t(TH) * TW;
    static constexpr size_t tiles = S * tile_elems * sizeof(T);
    static constexpr size_t xbuf = size_t(S) * W * TW * sizeof(T);
    static constexpr size_t topb = size_t(S) * TW * sizeof(T);
    static constexpr size_t bars = size_t(4) * S * sizeof(uint64_t) + 16;
    static constexpr size_t total = tiles + xbuf + topb + bars;
};

template <typename T, int R, int W, int S, int MODE, bool TMA, int MINB>
__global__ void __launch_bounds__((W + 2) * 32, MINB)
sat_band_kernel(const __grid_constant__ CUtensorMap tm_in,
                const __grid_constant__ CUtensorMap tm_out,
                const BandParams p)
{
    constexpr int TH = R * W;
    constexpr int CW = W;          // control warp
    constexpr int PW = W + 1;      // producer warp
    constexpr uint32_t TILE_BYTES = uint32_t(TH) * TW * sizeof(T);
    using SM = BandSmem<T, R, W, S>;

    extern __shared__ __align__(1024) uint8_t smem[];
    T* tiles = reinterpret_cast<T*>(smem);
    T* xbuf = reinterpret_cast<T*>(smem + SM::tiles);
    T* topb = reinterpret_cast<T*>(smem + SM::tiles + SM::xbuf);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + SM::tiles + SM::xbuf + SM::topb);
    uint64_t* full = bars;
    uint64_t* colr = bars + S;
    uint64_t* topr = bars + 2 * S;
    uint64_t* done = bars + 3 * S;
    long long* s_unit = reinterpret_cast<long long*>(bars + 4 * S);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&colr[s], W * 32);
            mbar_init(&topr[s], 32);
            mbar_init(&done[s], W * 32);
        }
        fence_mbar_init();
    }
    if (TMA && warp == PW && lane == 0) { prefetch_tmap(&tm_in); prefetch_tmap(&tm_out); }
    __syncthreads();

    const int64_t img_elems = p.rows * p.cols;
    const int desc_w = p.nc * TW;
    const int64_t lx_stride = int64_t(p.total_bands) * TH;
    uint32_t g = 0;                              // CTA-local chunk counter (ring position)
    T seedrun = T(0);                            // control warp: running seed prefix

    for (;;) {
        if (threadIdx.x == 0)
            *s_unit = (long long)(atomicAdd(p.ticket, 1ull) - p.base);
        __syncthreads();
        const long long unit = *s_unit;
        if (unit >= p.total_units) break;

        int gb, j0, j1;
        if (p.tile_units) {
            gb = int(unit / p.nc);
            const int J = int(unit % p.nc);
            int r0, r1;
            region_range(p.region, p.tA, p.nb, p.nc, gb % p.nb, r0, r1);
            j0 = J; j1 = (J >= r0 && J < r1) ? J + 1 : J;
        } else {
            gb = int(unit);
            region_range(p.region, p.tA, p.nb, p.nc, gb % p.nb, j0, j1);
        }
        const int img = gb / p.nb;
        const int band = gb - img * p.nb;
        const int nch = j1 - j0;
        const int row0 = band * TH;

        if (warp < W) {
            // ================= compute warps =================
            const int rbase = warp * R;                  // first row of this warp in the band
            T L[R];
#pragma unroll
            for (int r = 0; r < R; ++r) L[r] = T(0);
            auto load_L = [&](int J) {
                if (p.Lx != nullptr) {
                    const T* lx = reinterpret_cast<const T*>(p.Lx) + int64_t(J) * lx_stride
                                  + int64_t(gb) * TH + rbase;
#pragma unroll
                    for (int r = 0; r < R; ++r) L[r] = lx[r];
                }
            };
            load_L(j0);

            const T* gin = reinterpret_cast<const T*>(p.in) + int64_t(img) * img_elems;
            T* gout = reinterpret_cast<T*>(p.out) + int64_t(img) * img_elems;

            // local(): load chunk k, row scans with L, column prefix, publish warp bottom row
            auto local = [&](V4<T> (&v)[R], int k) {
                const uint32_t it = g + k;
                const int s = it % S;
                const uint32_t ph = (it / S) & 1;
                const int J = j0 + k;
                if (p.tile_units && k == 0) load_L(J);
                if constexpr (!TMA) {
                    // generic path: slot s is free once every warp finished its previous use
                    if (it >= uint32_t(S)) mbar_wait(&done[s], ph ^ 1u);
                }
                if constexpr (TMA) {
                    mbar_wait(&full[s], ph);
                    if (p.trace && warp == 0 && lane == 0)
                        p.trace[(int64_t(gb) * p.nc + J) * 4 + 0] = globaltimer();
                    const T* t = tiles + size_t(s) * SM::tile_elems + size_t(rbase) * TW + 4 * lane;
#pragma unroll
                    for (int r = 0; r < R; ++r) v[r] = lds4<T>(t + r * TW);
                } else {
                    const int64_t c = int64_t(J) * TW + 4 * lane;
#pragma unroll
                    for (int r = 0; r < R; ++r) {
                        const int64_t row = row0 + rbase + r;
                        T e[4];
#pragma unroll
                        for (int i = 0; i < 4; ++i)
                            e[i] = (row < p.rows && c + i < p.cols) ? gin[row * p.cols + c + i] : T(0);
                        v[r] = V4<T>{e[0], e[1], e[2], e[3]};
                    }
                }
                if constexpr (MODE != MODE_COL) {
                    // row-wise prefix-sums (the paper's R carry lives in L)
#pragma unroll
                    for (int r = 0; r < R; ++r) {
                        v[r].y += v[r].x; v[r].z += v[r].y; v[r].w += v[r].z;
                        const T inc = warp_inclusive_scan(v[r].w, lane);
                        T exc = __shfl_up_sync(0xffffffffu, inc, 1);
                        if (lane == 0) exc = T(0);
                        const T off = L[r] + exc;
                        v[r].x += off; v[r].y += off; v[r].z += off; v[r].w += off;
                        L[r] += __shfl_sync(0xffffffffu, inc, 31);
                    }
                }
                if constexpr (MODE != MODE_ROW) {
                    // column-wise prefix-sums down this warp's rows
#pragma unroll
                    for (int r = 1; r < R; ++r) add4(v[r], v[r - 1]);
                    sts4(xbuf + (size_t(s) * W + warp) * TW + 4 * lane, v[R - 1]);
                    mbar_arrive(&colr[s]);
                }
            };
            // finish(): + (SAT row above the band) + (bottom rows of the warps above), store
            auto finish = [&](V4<T> (&v)[R], int k) {
                const uint32_t it = g + k;
                const int s = it % S;
                const uint32_t ph = (it / S) & 1;
                const int J = j0 + k;
                if constexpr (MODE != MODE_ROW) {
                    mbar_wait(&topr[s], ph);
                    V4<T> add = lds4<T>(topb + size_t(s) * TW + 4 * lane);
                    for (int w2 = 0; w2 < warp; ++w2)
                        add4(add, lds4<T>(xbuf + (size_t(s) * W + w2) * TW + 4 * lane));
#pragma unroll
                    for (int r = 0; r < R; ++r) add4(v[r], add);
                }
                if constexpr (TMA) {
                    T* t = tiles + size_t(s) * SM::tile_elems + size_t(rbase) * TW + 4 * lane;
#pragma unroll
                    for (int r = 0; r < R; ++r) sts4(t + r * TW, v[r]);
                    fence_proxy_async_smem();
                    mbar_arrive(&done[s]);
                } else {
                    const int64_t c = int64_t(J) * TW + 4 * lane;
#pragma unroll
                    for (int r = 0; r < R; ++r) {
                        const int64_t row = row0 + rbase + r;
                        if (row < p.rows) {
                            const T e[4] = {v[r].x, v[r].y, v[r].z, v[r].w};
#pragma unroll
                            for (int i = 0; i < 4; ++i)
                                if (c + i < p.cols) gout[row * p.cols + c + i] = e[i];
                        }
                    }
                    mbar_arrive(&done[s]);
                }
            };

            V4<T> va[R], vb[R];
            if (nch > 0) {
                local(va, 0);
                for (int k = 0; k < nch; k += 2) {
                    if (k + 1 < nch) local(vb, k + 1);
                    finish(va, k);
                    if (k + 1 >= nch) break;
                    if (k + 2 < nch) local(va, k + 2);
                    finish(vb, k + 1);
                }
            }
            if (p.Lb != nullptr && !p.tile_units && lane == 0) {
                T* lb = reinterpret_cast<T*>(p.Lb) + int64_t(gb) * TH + rbase;
#pragma unroll
                for (int r = 0; r < R; ++r) lb[r] = L[r];
            }
        } else if (warp == CW) {
            // ================= control warp: descriptors + look-back =================
            if constexpr (MODE != MODE_ROW) {
                const uint32_t tagbase = uint32_t((p.base + (unsigned long long)gb) & 0x3FFFFFFFull) << 2;
                if (band == 0) seedrun = T(0);
                for (int k = 0; k < nch; ++k) {
                    const uint32_t it = g + k;
                    const int s = it % S;
                    const uint32_t ph = (it / S) & 1;
                    const int J = j0 + k;
                    const int c0 = J * TW + 4 * lane;
                    mbar_wait(&colr[s], ph);
                    if (p.trace && lane == 0)
                        p.trace[(int64_t(gb) * p.nc + J) * 4 + 1] = globaltimer();
                    unsigned long long hops = 0;
                    V4<T> agg = lds4<T>(xbuf + size_t(s) * W * TW + 4 * lane);
                    for (int w2 = 1; w2 < W; ++w2)
                        add4(agg, lds4<T>(xbuf + (size_t(s) * W + w2) * TW + 4 * lane));
                    V4<T> top{T(0), T(0), T(0), T(0)};
                    if (p.top_src == TOP_EXTERNAL) {
                        top = lds4<T>(reinterpret_cast<const T*>(p.TopX) + int64_t(gb) * desc_w + c0);
                    } else {
                        uint64_t* my = p.desc + int64_t(gb) * desc_w + c0;
                        if (p.jitter) {
                            uint32_t h = (uint32_t(gb) * 2654435761u) ^ (uint32_t(J) * 40503u) ^ lane;
                            h ^= h >> 13; h *= 0x5bd1e995u; h ^= h >> 15;
                            __nanosleep(h % (uint32_t)p.jitter);
                        }
                        if (band == 0) {
                            if (p.seed_kind != SEED_NONE && img == 0) {
                                const T* sd = reinterpret_cast<const T*>(p.seed);
                                T e[4];
#pragma unroll
                                for (int i = 0; i < 4; ++i) e[i] = (c0 + i < p.cols) ? sd[c0 + i] : T(0);
                                if (p.seed_kind == SEED_COLSUM && MODE == MODE_SAT) {
                                    // SAT row above = row prefix of the column sums above
                                    e[1] += e[0]; e[2] += e[1]; e[3] += e[2];
                                    const T inc = warp_inclusive_scan(e[3], lane);
                                    T exc = __shfl_up_sync(0xffffffffu, inc, 1);
                                    if (lane == 0) exc = T(0);
                                    const T off = seedrun + exc;
#pragma unroll
                                    for (int i = 0; i < 4; ++i) e[i] += off;
                                    seedrun += __shfl_sync(0xffffffffu, inc, 31);
                                }
                                top = V4<T>{e[0], e[1], e[2], e[3]};
                            }
                        } else {
                            // publish aggregate (band-local), then look back
                            const uint32_t tA = tagbase | 1u;
                            st_relaxed_v2(my, (uint64_t(tA) << 32) | to_bits(agg.x), (uint64_t(tA) << 32) | to_bits(agg.y));
                            st_relaxed_v2(my + 2, (uint64_t(tA) << 32) | to_bits(agg.z), (uint64_t(tA) << 32) | to_bits(agg.w));
                            T acc[4] = {T(0), T(0), T(0), T(0)};
                            uint32_t pend = 0xFu;
                            int kb = band - 1;
                            const T* gout = reinterpret_cast<const T*>(p.out) + int64_t(img) * img_elems;
                            while (pend) {
                                if (p.region == REG_C && kb + J < p.tA) {
                                    // tile (kb, J) belongs to (A): its final SAT row is in `out`
                                    const int64_t row = int64_t(kb + 1) * TH - 1;
#pragma unroll
                                    for (int i = 0; i < 4; ++i)
                                        if ((pend >> i) & 1u)
                                            acc[i] += (c0 + i < p.cols) ? gout[row * p.cols + c0 + i] : T(0);
                                    pend = 0;
                                    break;
                                }
                                const uint64_t* q = p.desc + (int64_t(gb) - (band - kb)) * desc_w + c0;
                                const uint32_t tk = uint32_t((p.base + (unsigned long long)(gb - (band - kb))) & 0x3FFFFFFFull) << 2;
                                uint64_t w0, w1, w2, w3;
                                ld_relaxed_v2(q, w0, w1);
                                ld_relaxed_v2(q + 2, w2, w3);
                                const uint64_t ws[4] = {w0, w1, w2, w3};
                                bool ready = true;
#pragma unroll
                                for (int i = 0; i < 4; ++i) {
                                    const uint32_t t = uint32_t(ws[i] >> 32);
                                    ready = ready && ((t & ~3u) == tk) && (t & 3u);
                                }
                                if (!ready) { __nanosleep(16); continue; }
#pragma unroll
                                for (int i = 0; i < 4; ++i) {
                                    if ((pend >> i) & 1u) {
                                        acc[i] += from_bits<T>(uint32_t(ws[i]));
                                        if ((uint32_t(ws[i] >> 32) & 3u) == 2u) pend &= ~(1u << i);
                                    }
                                }
                                --kb;
                                ++hops;
                            }
                            top = V4<T>{acc[0], acc[1], acc[2], acc[3]};
                        }
                        if (p.nb > 1) {
                            V4<T> inc = agg;
                            add4(inc, top);
                            const uint32_t tP = tagbase | 2u;
                            st_relaxed_v2(my, (uint64_t(tP) << 32) | to_bits(inc.x), (uint64_t(tP) << 32) | to_bits(inc.y));
                            st_relaxed_v2(my + 2, (uint64_t(tP) << 32) | to_bits(inc.z), (uint64_t(tP) << 32) | to_bits(inc.w));
                        }
                    }
                    if (p.trace && lane == 0)
                        p.trace[(int64_t(gb) * p.nc + J) * 4 + 2] = (globaltimer() & 0xFFFFFFFFFFFFull) | (hops << 48);
                    sts4(topb + size_t(s) * TW + 4 * lane, top);
                    mbar_arrive(&topr[s]);
                }
            }
        } else {
            // ================= producer warp: TMA ring =================
            if constexpr (TMA) {
                if (lane == 0 && nch > 0) {
                    const uint64_t pol = policy_evict_first();
                    bulk_wait_read<0>();          // previous unit's stores done reading smem
                    auto load = [&](int k) {
                        const uint32_t it = g + k;
                        const int s = it % S;
                        mbar_arrive_expect_tx(&full[s], TILE_BYTES);
                        tma_load_3d(tiles + size_t(s) * SM::tile_elems, &tm_in, &full[s],
                                    (j0 + k) * TW, row0, img, pol);
                    };
                    const int pre = nch < S ? nch : S;
                    for (int k = 0; k < pre; ++k) load(k);
                    for (int k = 0; k < nch; ++k) {
                        const uint32_t it = g + k;
                        const int s = it % S;
                        const uint32_t ph = (it / S) & 1;
                        mbar_wait(&done[s], ph);
                        if (p.trace)
                            p.trace[(int64_t(gb) * p.nc + j0 + k) * 4 + 3] = globaltimer();
                        tma_store_3d(&tm_out, tiles + size_t(s) * SM::tile_elems, (j0 + k) * TW, row0, img, pol);
                        bulk_commit();
                        if (k + S < nch) { bulk_wait_read<0>(); load(k + S); }
                    }
                }
            }
        }
        g += nch;
        __syncthreads();
    }
    if (TMA && warp == PW && lane == 0) bulk_wait<0>();
}

}  // namespace sat
