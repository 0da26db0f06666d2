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
//     right in TH x 128 chunks staged through an S-slot TMA ring in smem;
//   * the horizontal carry (the paper's R) is the per-row running sum L held
//     in registers by the warp that owns the row;
//   * the vertical carry (the paper's C and S, i.e. the SAT row above the
//     band) comes from a decoupled look-back over self-validating descriptor
//     words: each (band, chunk) publishes the bottom row of its band-local SAT
//     as an "aggregate", then -- once it knows the SAT row above -- the final
//     SAT bottom row as "inclusive".  The look-back reads a
//     window of LBW bands per round trip;
//   * inside a chunk, Step 3-1/3-2 of 2R1W become two passes over
//     the smem slot: the compute warps' local() = row scans with L + column
//     prefix down the warp's R rows (written back in place; the warp's bottom
//     row goes to xbuf); the control warp's finish = + (SAT row above the
//     band + bottom rows of the warps above).  The compute warps never wait
//     for a look-back: they run ahead as far as the S-slot ring allows, and
//     NCW control warps keep NCW look-backs (and finishes) in flight.
//
// The same kernel, with MODE/TopSrc switches, is the column pass and row pass
// of 2R2W, Step 3 of 2R1W with external carries
// and the 1R1W band (C) of (1+r)R1W.
//
// Roles (warps): 0..W-1 compute (R rows each), W..W+NCW-1 control
// (descriptors and look-back; control warp c owns the chunks k = c mod NCW,
// so NCW look-backs are in flight at once), W+NCW = producer (TMA loads and
// stores, one elected lane).
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
    static constexpr int XS = S;                     // xbuf slots (one per ring slot)
    static constexpr size_t tile_elems = size_t(TH) * TW;
    static constexpr size_t tiles = S * tile_elems * sizeof(T);
    static constexpr size_t xbuf = size_t(XS) * W * TW * sizeof(T);
    static constexpr size_t bars = size_t(4) * S * sizeof(uint64_t) + 16;
    static constexpr size_t total = tiles + xbuf + bars;
};

constexpr int LBW = 4;   // look-back window: bands read per round trip

__device__ __forceinline__ uint32_t band_tag(unsigned long long base, int gb) {
    return uint32_t((base + (unsigned long long)gb) & 0x3FFFFFFFull) << 2;
}

template <typename T>
__device__ __forceinline__ void publish4(uint64_t* my, uint32_t tag, const V4<T>& v) {
    st_relaxed_v2(my, (uint64_t(tag) << 32) | to_bits(v.x), (uint64_t(tag) << 32) | to_bits(v.y));
    st_relaxed_v2(my + 2, (uint64_t(tag) << 32) | to_bits(v.z), (uint64_t(tag) << 32) | to_bits(v.w));
}

// Row-wise inclusive prefix-sums of R rows of 128 columns (lane owns 4
// consecutive columns), continuing from the running row sums L, which are
// advanced to the end of the chunk.  Rows are interleaved step by step so the
// shuffles of different rows overlap.
template <typename T, int R>
__device__ __forceinline__ void row_scan(V4<T> (&v)[R], T (&L)[R], int lane) {
    T inc[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
        v[r].y += v[r].x; v[r].z += v[r].y; v[r].w += v[r].z;
        inc[r] = v[r].w;
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
            exc = inc[r] - v[r].w;                 // exact in Z/2^32
        } else {
            exc = __shfl_up_sync(0xffffffffu, inc[r], 1);
            if (lane == 0) exc = T(0);
        }
        const T off = L[r] + exc;
        v[r].x += off; v[r].y += off; v[r].z += off; v[r].w += off;
        L[r] += __shfl_sync(0xffffffffu, inc[r], 31);
    }
}

template <typename T, int R, int W, int S, int NCW, int MODE, bool TMA, int MINB>
__global__ void __launch_bounds__((W + NCW + 1) * 32, MINB)
sat_band_kernel(const __grid_constant__ CUtensorMap tm_in,
                const __grid_constant__ CUtensorMap tm_out,
                const BandParams p)
{
    constexpr int TH = R * W;
    constexpr int CW = W;          // first control warp
    constexpr int PW = W + NCW;    // producer warp
    constexpr uint32_t TILE_BYTES = uint32_t(TH) * TW * sizeof(T);
    using SM = BandSmem<T, R, W, S>;
    constexpr int XS = SM::XS;
    // A control warp waits on colr[] of chunk k only after finishing chunk
    // k-NCW, which implies local(k-S) completed iff NCW <= S; otherwise the
    // parity wait could pass on a stale phase.
    static_assert(NCW <= S, "more control warps than ring slots");

    extern __shared__ __align__(1024) uint8_t smem[];
    T* tiles = reinterpret_cast<T*>(smem);
    T* xbuf = reinterpret_cast<T*>(smem + SM::tiles);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + SM::tiles + SM::xbuf);
    uint64_t* full = bars;          // TMA load landed (tx count)
    uint64_t* colr = bars + S;      // every compute warp finished local()
    uint64_t* done = bars + 3 * S;  // the slot holds final values (control warp / row pass)
    long long* s_unit = reinterpret_cast<long long*>(bars + 4 * S);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&colr[s], W * 32);
            mbar_init(&done[s], MODE == MODE_ROW ? W * 32 : 32);
        }
        fence_mbar_init();
    }
    if (TMA && warp == PW && lane == 0) { prefetch_tmap(&tm_in); prefetch_tmap(&tm_out); }
    __syncthreads();

    const int64_t img_elems = p.rows * p.cols;
    const int desc_w = p.nc * TW;
    const int64_t lx_stride = int64_t(p.total_bands) * TH;
    uint32_t g = 0;                              // CTA-local chunk counter (ring position)

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
            if (p.Lx != nullptr) {
                const T* lx = reinterpret_cast<const T*>(p.Lx) + int64_t(j0) * lx_stride
                              + int64_t(gb) * TH + rbase;
#pragma unroll
                for (int r = 0; r < R; ++r) L[r] = lx[r];
            }
            const T* gin = reinterpret_cast<const T*>(p.in) + int64_t(img) * img_elems;
            T* gout = reinterpret_cast<T*>(p.out) + int64_t(img) * img_elems;

            // local(k): row scans with L, column prefix down this warp's rows,
            // result back into the slot, warp bottom row into xbuf
            auto local = [&](int k) {
                const uint32_t it = g + k;
                const int s = it % S;
                const uint32_t ph = (it / S) & 1;
                T* t = tiles + size_t(s) * SM::tile_elems + size_t(rbase) * TW + 4 * lane;
                V4<T> v[R];
                if constexpr (!TMA) {
                    // the slot is free once the control warp finished chunk it-S
                    if (it >= uint32_t(S)) mbar_wait(&done[s], ph ^ 1u);
                }
                if constexpr (TMA) {
                    mbar_wait(&full[s], ph);
                    if (p.trace && warp == 0 && lane == 0)
                        p.trace[(int64_t(gb) * p.nc + j0 + k) * 8 + 0] = globaltimer();
#pragma unroll
                    for (int r = 0; r < R; ++r) v[r] = lds4<T>(t + r * TW);
                } else {
                    const int64_t c = int64_t(j0 + k) * TW + 4 * lane;
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
                if constexpr (MODE != MODE_COL) row_scan<T, R>(v, L, lane);
                if constexpr (MODE != MODE_ROW) {
#pragma unroll
                    for (int r = 1; r < R; ++r) add4(v[r], v[r - 1]);
                    sts4(xbuf + (size_t(it % XS) * W + warp) * TW + 4 * lane, v[R - 1]);
                }
                if constexpr (MODE == MODE_ROW && !TMA) {
                    // the row pass is final: write straight out
                    const int64_t c = int64_t(j0 + k) * TW + 4 * lane;
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
                } else {
#pragma unroll
                    for (int r = 0; r < R; ++r) sts4(t + r * TW, v[r]);
                }
                if constexpr (MODE == MODE_ROW) {
                    if constexpr (TMA) fence_proxy_async_smem();
                    mbar_arrive(&done[s]);
                } else {
                    mbar_arrive(&colr[s]);
                }
            };
            for (int k = 0; k < nch; ++k) local(k);
            if (p.Lb != nullptr && !p.tile_units && lane == 0) {
                T* lb = reinterpret_cast<T*>(p.Lb) + int64_t(gb) * TH + rbase;
#pragma unroll
                for (int r = 0; r < R; ++r) lb[r] = L[r];
            }
        } else if (warp < PW) {
            // ================= control warp: descriptors + look-back =================
            if constexpr (MODE != MODE_ROW) {
                const uint32_t tagbase = band_tag(p.base, gb);
                const bool lookback = (p.top_src == TOP_LOOKBACK);
                const bool publish = lookback && band + 1 < p.nb;   // the last band is never read
                const T* gout = reinterpret_cast<const T*>(p.out) + int64_t(img) * img_elems;
                for (int k = warp - CW; k < nch; k += NCW) {
                    const uint32_t it = g + k;
                    const int s = it % S;
                    const uint32_t ph = (it / S) & 1;
                    const int J = j0 + k;
                    const int c0 = J * TW + 4 * lane;
                    T* xb = xbuf + size_t(it % XS) * W * TW + 4 * lane;
                    mbar_wait(&colr[s], ph);
                    if (p.trace && lane == 0)
                        p.trace[(int64_t(gb) * p.nc + J) * 8 + 1] = globaltimer();
                    V4<T> agg = lds4<T>(xb);
#pragma unroll
                    for (int w2 = 1; w2 < W; ++w2) add4(agg, lds4<T>(xb + w2 * TW));
                    uint64_t* my = p.desc + int64_t(gb) * desc_w + c0;
                    if (p.jitter && lookback) {
                        uint32_t h = (uint32_t(gb) * 2654435761u) ^ (uint32_t(J) * 40503u) ^ lane;
                        h ^= h >> 13; h *= 0x5bd1e995u; h ^= h >> 15;
                        __nanosleep(h % (uint32_t)p.jitter);
                    }
                    if (publish && band > 0) publish4<T>(my, tagbase | 1u, agg);
                    V4<T> top{T(0), T(0), T(0), T(0)};
                    unsigned long long hops = 0, polls = 0;
                    if (!lookback) {
                        top = lds4<T>(reinterpret_cast<const T*>(p.TopX) + int64_t(gb) * desc_w + c0);
                    } else if (band == 0) {
                        if (p.seed_kind != SEED_NONE && img == 0) {
                            // the SAT row just above the matrix (sat_api.cu turns a
                            // column-sum seed into this row first)
                            const T* sd = reinterpret_cast<const T*>(p.seed);
                            T e[4];
#pragma unroll
                            for (int i = 0; i < 4; ++i) e[i] = (c0 + i < p.cols) ? sd[c0 + i] : T(0);
                            top = V4<T>{e[0], e[1], e[2], e[3]};
                        }
                    } else {
                        // decoupled look-back over bands band-1, band-2, ...,
                        // LBW descriptor rows per round trip
                        T acc[4] = {T(0), T(0), T(0), T(0)};
                        uint32_t pend = 0xFu;
                        int kb = band - 1;
                        SpinGuard guard;
                        while (pend) {
                            uint64_t wv[LBW][4];
#pragma unroll
                            for (int q = 0; q < LBW; ++q) {
                                const int b2 = kb - q;
                                if (b2 >= 0) {
                                    const uint64_t* qp = p.desc + (int64_t(gb) - (band - b2)) * desc_w + c0;
                                    ld_relaxed_v2(qp, wv[q][0], wv[q][1]);
                                    ld_relaxed_v2(qp + 2, wv[q][2], wv[q][3]);
                                } else {
                                    wv[q][0] = wv[q][1] = wv[q][2] = wv[q][3] = 0;
                                }
                            }
                            bool stalled = false;
#pragma unroll
                            for (int q = 0; q < LBW; ++q) {
                                if (!pend || stalled) break;
                                const int b2 = kb - q;
                                if (p.region == REG_C && b2 + J < p.tA) {
                                    // tile (b2, J) belongs to (A): its final SAT row is in `out`
                                    const int64_t row = int64_t(b2 + 1) * TH - 1;
#pragma unroll
                                    for (int i = 0; i < 4; ++i)
                                        if ((pend >> i) & 1u)
                                            acc[i] += (c0 + i < p.cols) ? gout[row * p.cols + c0 + i] : T(0);
                                    pend = 0;
                                    break;
                                }
                                const uint32_t tk = band_tag(p.base, gb - (band - b2));
                                bool ready = true;
#pragma unroll
                                for (int i = 0; i < 4; ++i) {
                                    const uint32_t t = uint32_t(wv[q][i] >> 32);
                                    ready = ready && ((t & ~3u) == tk) && (t & 3u);
                                }
                                if (!ready) { stalled = true; kb = b2; break; }
#pragma unroll
                                for (int i = 0; i < 4; ++i) {
                                    if ((pend >> i) & 1u) {
                                        acc[i] += from_bits<T>(uint32_t(wv[q][i]));
                                        if ((uint32_t(wv[q][i] >> 32) & 3u) == 2u) pend &= ~(1u << i);
                                    }
                                }
                                ++hops;
                            }
                            if (stalled) { __nanosleep(32); guard.tick(); ++polls; }
                            else kb -= LBW;
                        }
                        top = V4<T>{acc[0], acc[1], acc[2], acc[3]};
                    }
                    if (publish) {
                        V4<T> inc = agg;
                        add4(inc, top);
                        publish4<T>(my, tagbase | 2u, inc);
                    }
                    if (p.trace && lane == 0)
                        p.trace[(int64_t(gb) * p.nc + J) * 8 + 2] =
                            (globaltimer() & 0xFFFFFFFFFFFFull) | (min(hops, 255ull) << 48) | (min(polls, 255ull) << 56);
                    // finish: + (SAT row above the band + bottom rows of the
                    // warps above); the slot then holds final values
                    if (p.trace && lane == 0)
                        p.trace[(int64_t(gb) * p.nc + J) * 8 + 6] = globaltimer();
                    T* t = tiles + size_t(s) * SM::tile_elems + 4 * lane;
                    const int64_t cg = int64_t(J) * TW + 4 * lane;
                    T* go = reinterpret_cast<T*>(p.out) + int64_t(img) * img_elems;
                    V4<T> run = top;
#pragma unroll 1
                    for (int w2 = 0; w2 < W; ++w2) {
                        const V4<T> b = lds4<T>(xb + w2 * TW);
                        T* tr = t + (w2 * R) * TW;
                        V4<T> v[R];
#pragma unroll
                        for (int r = 0; r < R; ++r) v[r] = lds4<T>(tr + r * TW);   // loads first (ILP)
#pragma unroll
                        for (int r = 0; r < R; ++r) {
                            add4(v[r], run);
                            if constexpr (TMA) {
                                sts4(tr + r * TW, v[r]);
                            } else {
                                const int64_t row = row0 + w2 * R + r;
                                if (row < p.rows) {
                                    const T e[4] = {v[r].x, v[r].y, v[r].z, v[r].w};
#pragma unroll
                                    for (int i = 0; i < 4; ++i)
                                        if (cg + i < p.cols) go[row * p.cols + cg + i] = e[i];
                                }
                            }
                        }
                        add4(run, b);
                    }
                    if constexpr (TMA) fence_proxy_async_smem();
                    __syncwarp();
                    mbar_arrive(&done[s]);
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
                        if (p.trace)
                            p.trace[(int64_t(gb) * p.nc + j0 + k) * 8 + 4] = globaltimer();
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
                            p.trace[(int64_t(gb) * p.nc + j0 + k) * 8 + 3] = globaltimer();
                        tma_store_3d(&tm_out, tiles + size_t(s) * SM::tile_elems, (j0 + k) * TW, row0, img, pol);
                        bulk_commit();
                        if (k + S < nch) {
                            bulk_wait_read<0>();
                            if (p.trace)
                                p.trace[(int64_t(gb) * p.nc + j0 + k) * 8 + 5] = globaltimer();
                            load(k + S);
                        }
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
