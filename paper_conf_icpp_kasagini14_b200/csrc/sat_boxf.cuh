// sat_boxf.cuh -- the box filter fused with the SAT that serves it (SURVEY.md
// Sec. 8 row f2; the paper's motivating use, "the sum of any rectangular area
// can be computed in O(1)", Sec. I).
//
// out[i][j] = sum of a[k][l] over |k - i| <= rr, |l - j| <= rc (clipped to
// the image) = S[i2][j2] - S[i1-1][j2] - S[i2][j1-1] + S[i1-1][j1-1] with the
// SAT S.  The two-pass path (sat_box_kernel) writes S to HBM and reads it
// back: 1 + 4 + 4 + 4 bytes per uint8 pixel.  Here the SAT never leaves the
// chip: a CTA owns a band of TH output rows and computes the SAT of the rows
// the band's windows touch -- the band plus a halo of rr rows above and below
// -- chunk by chunk (128 columns, left to right, row carries in registers),
// keeping the last three chunks' SATs in shared memory, and evaluates the four
// corner reads for the chunk before.  The SAT is LOCAL: it starts at zero at
// the halo's first row.  The global SAT differs from it by one row vector X(j)
// (the SAT row above the halo), which cancels in S[i2][.] - S[i1-1][.] because
// both rows lie in the halo band -- so no look-back is needed, and the input is
// read (TH + 2 rr) / TH times: 1 x (1 + 2 rr / TH) + 4 bytes per uint8 pixel.
//
// Roles: NWARP (16) warps.  A chunk is a TMA box of 128 columns x MAXH rows (MAXH >= TH
// + 2 rr) of the input in an NS-slot ring (thread 0 issues, mbarrier
// complete_tx).  Warp w owns loaded rows [w*RPW, (w+1)*RPW): it widens its
// rows (uint8 -> uint32, float32 -> float64), row-scans them with its per-row
// carries, takes the column prefix down its rows and publishes its bottom row;
// after a barrier every warp adds the bottom rows of the warps above and
// stores its rows into the chunk's SAT buffer; after a second barrier the
// warps evaluate the box sums of the previous chunk (4 conflict-free scalar
// LDS per output) and store them with coalesced 128-B warp stores.
#pragma once
#include "sat_common.h"
#include "sat_device.cuh"

namespace sat {

struct BoxParams {
    const void* in;        // [batch][rows][cols] (the TMA map covers it)
    void* out;             // [batch][rows][cols]
    int rows, cols, batch;
    int rr, rc;            // radii (host-clamped to the image)
    int normalize;         // float only: divide by the clipped window's count
    int nb;                // bands per image = ceil(rows / TH)
    int nc;                // chunks = ceil(cols / 128)
    unsigned long long* ticket;
    unsigned long long base;
};

template <int MAXH, int NS, typename TI, typename TS, int NWARP>
struct BoxSmem {
    static constexpr size_t ring = size_t(NS) * MAXH * TW * sizeof(TI);
    static constexpr size_t ring_al = (ring + 127) / 128 * 128;
    static constexpr size_t satb = size_t(3) * (MAXH + 1) * TW * sizeof(TS);   // row 0 of each buffer: zeros
    static constexpr size_t bot = size_t(NWARP) * TW * sizeof(TS);
    static constexpr size_t bars = size_t(NS) * 8 + 16;
    static constexpr size_t total = ring_al + satb + bot + bars;
};

// scalar shared load from a 32-bit shared-window address
template <typename T>
__device__ __forceinline__ T lds_s(uint32_t a) {
    if constexpr (sizeof(T) == 4) {
        uint32_t v;
        asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a));
        return from_bits<T>(v);
    } else {
        double v;
        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
        return T(v);
    }
}

template <typename TI, typename TS, typename TO, int TH, int MAXH, int NS, int NWARP>
__global__ void __launch_bounds__(NWARP * 32, 1) sat_boxf_kernel(const __grid_constant__ CUtensorMap tm_in,
                                                                 const BoxParams bp) {
    constexpr int RPW = (MAXH + NWARP - 1) / NWARP;    // loaded rows per warp
    using SM = BoxSmem<MAXH, NS, TI, TS, NWARP>;
    extern __shared__ __align__(1024) uint8_t smem[];
    TI* ring = reinterpret_cast<TI*>(smem);
    TS* satb = reinterpret_cast<TS*>(smem + SM::ring_al);            // [3][1 + MAXH][TW]
    TS* bot = reinterpret_cast<TS*>(smem + SM::ring_al + SM::satb);  // [NWARP][TW]
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + SM::ring_al + SM::satb + SM::bot);
    long long* s_unit = reinterpret_cast<long long*>(full + NS);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < NS; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
        prefetch_tmap(&tm_in);
    }
    // row 0 of every chunk buffer holds the SAT row above the halo: zeros
    for (int i = threadIdx.x; i < 3 * TW; i += blockDim.x)
        satb[size_t(i / TW) * (MAXH + 1) * TW + (i % TW)] = TS(0);
    __syncthreads();
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const uint64_t pol = policy_evict_first();
    uint32_t q = 0;                                     // CTA-global chunk counter (ring parity)
    const int64_t img_elems = int64_t(bp.rows) * bp.cols;
    for (;;) {
        __syncthreads();                                // everyone done with the previous unit's buffers
        if (threadIdx.x == 0) *s_unit = (long long)(atomicAdd(bp.ticket, 1ull) - bp.base);
        __syncthreads();
        const long long unit = *s_unit;
        if (unit >= (long long)bp.batch * bp.nb) break;
        const int img = int(unit / bp.nb), band = int(unit % bp.nb);
        const int r0 = band * TH, r1 = min(bp.rows, r0 + TH);
        const int t0 = max(0, r0 - bp.rr), t1 = min(bp.rows, r1 + bp.rr);
        const int H = t1 - t0;                          // loaded rows (<= MAXH, host-checked)
        TO* gout = reinterpret_cast<TO*>(bp.out) + int64_t(img) * img_elems;
        // prologue: the first NS-1 chunks
        if (threadIdx.x == 0) {
            for (int k = 0; k < NS - 1 && k < bp.nc; ++k) {
                const uint32_t qq = q + k;
                mbar_arrive_expect_tx(&full[qq % NS], uint32_t(MAXH) * TW * sizeof(TI));
                tma_load_3d(ring + size_t(qq % NS) * MAXH * TW, &tm_in, &full[qq % NS], k * TW, t0, img, pol);
            }
        }
        TS L[RPW];
#pragma unroll
        for (int r = 0; r < RPW; ++r) L[r] = TS(0);
        for (int k = 0; k <= bp.nc; ++k) {
            if (k < bp.nc) {
                const uint32_t qk = q + k;
                if (threadIdx.x == 0 && k + NS - 1 < bp.nc) {
                    // refill the slot every thread released at the last barrier
                    fence_proxy_async_smem();
                    const uint32_t qn = qk + NS - 1;
                    mbar_arrive_expect_tx(&full[qn % NS], uint32_t(MAXH) * TW * sizeof(TI));
                    tma_load_3d(ring + size_t(qn % NS) * MAXH * TW, &tm_in, &full[qn % NS], (k + NS - 1) * TW,
                                t0, img, pol);
                }
                mbar_wait(&full[qk % NS], (qk / NS) & 1);
                // local SAT of this chunk: row scans with carries, column
                // prefix down this warp's rows
                const TI* src = ring + size_t(qk % NS) * MAXH * TW + 4 * lane;
                const bool cin = k * TW + 4 * lane < bp.cols;
                // warps whose rows all lie below the halo band (H < MAXH for
                // small radii) have nothing to do: their rows are never read
                const bool act = warp * RPW < H;
                TS v[RPW][4];
                TS run[4] = {TS(0), TS(0), TS(0), TS(0)};
#pragma unroll
                for (int r = 0; r < RPW; ++r) {
                    const int lr = warp * RPW + r;
                    if (!act) break;
                    TS e[4] = {TS(0), TS(0), TS(0), TS(0)};
                    if (lr < H && cin) {
                        if constexpr (sizeof(TI) == 1) {
                            const uint32_t w = *reinterpret_cast<const uint32_t*>(src + size_t(lr) * TW);
                            e[0] = TS(w & 255u); e[1] = TS((w >> 8) & 255u); e[2] = TS((w >> 16) & 255u); e[3] = TS(w >> 24);
                        } else {
                            const uint4 w = *reinterpret_cast<const uint4*>(src + size_t(lr) * TW);
                            e[0] = TS(from_bits<TI>(w.x)); e[1] = TS(from_bits<TI>(w.y));
                            e[2] = TS(from_bits<TI>(w.z)); e[3] = TS(from_bits<TI>(w.w));
                        }
                    }
                    e[1] += e[0]; e[2] += e[1]; e[3] += e[2];
                    const TS inc = warp_inclusive_scan(e[3], lane);
                    TS exc = __shfl_up_sync(0xffffffffu, inc, 1);
                    if (lane == 0) exc = TS(0);
                    const TS off = L[r] + exc;
                    L[r] += __shfl_sync(0xffffffffu, inc, 31);
#pragma unroll
                    for (int i = 0; i < 4; ++i) { run[i] += e[i] + off; v[r][i] = run[i]; }
                }
                TS* b = bot + warp * TW + 4 * lane;
#pragma unroll
                for (int i = 0; i < 4; ++i) b[i] = run[i];
                __syncthreads();                        // bottom rows published, ring slot read
                TS add[4] = {TS(0), TS(0), TS(0), TS(0)};
                for (int w2 = 0; act && w2 < warp; ++w2)
#pragma unroll
                    for (int i = 0; i < 4; ++i) add[i] += bot[w2 * TW + 4 * lane + i];
                TS* dst = satb + (size_t(k % 3) * (MAXH + 1) + 1) * TW + 4 * lane;
#pragma unroll
                for (int r = 0; r < RPW; ++r) {
                    const int lr = warp * RPW + r;
                    if (lr < H) {
                        if constexpr (sizeof(TS) == 4) {
                            *reinterpret_cast<uint4*>(dst + size_t(lr) * TW) =
                                make_uint4(to_bits(v[r][0] + add[0]), to_bits(v[r][1] + add[1]),
                                           to_bits(v[r][2] + add[2]), to_bits(v[r][3] + add[3]));
                        } else {
                            reinterpret_cast<double2*>(dst + size_t(lr) * TW)[0] =
                                make_double2(v[r][0] + add[0], v[r][1] + add[1]);
                            reinterpret_cast<double2*>(dst + size_t(lr) * TW)[1] =
                                make_double2(v[r][2] + add[2], v[r][3] + add[3]);
                        }
                    }
                }
            }
            __syncthreads();                            // chunk k's SAT complete
            if (k >= 1) {
                // box sums of chunk k-1 (needs chunks k-2 .. k: rc < 128)
                const int kc = k - 1;
                // lane owns columns kc*128 + lane + 32 e (e = 0..3): the four
                // corner reads of a warp hit 32 consecutive words (no bank
                // conflicts; a 4-consecutive-columns-per-lane mapping made
                // them 4-way)
                // per lane and e: shared addresses of the two corner columns
                // (buffer of their chunk + column in it; 32-bit shared-window
                // addresses, so a corner read is one IADD + LDS), and a mask
                // that zeroes the left corner terms when j1 - 1 < 0
                uint32_t o2[4], o1[4];
                TS m1[4];
                const uint32_t sb = smem_u32(satb);
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    const int j = kc * TW + lane + 32 * e;
                    const int j2 = min(j + bp.rc, bp.cols - 1);
                    const int j1 = max(j - bp.rc, 0) - 1;      // -1: column before the image (S = 0)
                    const int jl = max(j1, 0);
                    o2[e] = sb + uint32_t((((j2 >> 7) % 3) * (MAXH + 1) * TW + (j2 & (TW - 1))) * sizeof(TS));
                    o1[e] = sb + uint32_t((((jl >> 7) % 3) * (MAXH + 1) * TW + (jl & (TW - 1))) * sizeof(TS));
                    if constexpr (std::is_same<TS, uint32_t>::value) m1[e] = j1 >= 0 ? 0xFFFFFFFFu : 0u;
                    else m1[e] = j1 >= 0 ? TS(1) : TS(0);
                }
                const bool full_chunk = kc * TW + TW <= bp.cols;
                const int64_t rstride = int64_t(NWARP) * bp.cols;
                TO* prow = gout + int64_t(r0 + warp) * bp.cols + kc * TW + lane;
                for (int i = r0 + warp; i < r1; i += NWARP, prow += rstride) {
                    // byte offsets of the local SAT rows of the window's last row
                    // and of the row above its first (+1: row 0 of each buffer is zero)
                    const uint32_t a2 = uint32_t((min(i + bp.rr, bp.rows - 1) - t0 + 1) * TW * int(sizeof(TS)));
                    const uint32_t a1 = uint32_t((max(i - bp.rr, 0) - t0) * TW * int(sizeof(TS)));
                    TS s[4];
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        const TS right = lds_s<TS>(a2 + o2[e]) - lds_s<TS>(a1 + o2[e]);
                        const TS left = lds_s<TS>(a2 + o1[e]) - lds_s<TS>(a1 + o1[e]);
                        if constexpr (std::is_same<TS, uint32_t>::value) s[e] = right - (left & m1[e]);
                        else s[e] = right - left * m1[e];
                    }
                    if constexpr (!std::is_same<TS, uint32_t>::value) {
                        if (bp.normalize) {
                            const int hh = min(i + bp.rr, bp.rows - 1) - max(i - bp.rr, 0) + 1;
#pragma unroll
                            for (int e = 0; e < 4; ++e) {
                                const int j = kc * TW + lane + 32 * e;
                                const int ww = min(j + bp.rc, bp.cols - 1) - max(j - bp.rc, 0) + 1;
                                s[e] = s[e] / TS(int64_t(hh) * int64_t(ww));
                            }
                        }
                    }
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        if (full_chunk || kc * TW + lane + 32 * e < bp.cols) {
                            if constexpr (std::is_same<TS, uint32_t>::value) __stcs(prow + 32 * e, TO(int32_t(s[e])));
                            else __stcs(prow + 32 * e, TO(s[e]));
                        }
                    }
                }
            }
        }
        q += uint32_t(bp.nc);
    }
}

}  // namespace sat
