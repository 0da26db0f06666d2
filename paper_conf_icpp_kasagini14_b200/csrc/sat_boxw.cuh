// sat_boxw.cuh -- the box filter as a SAT evaluated on the fly, one warp per
// strip of output columns walking down the rows (
// the sum of any rectangle in O(1) from the SAT).
//
// out[i][j] = S[i2][j2] - S[i1-1][j2] - S[i2][j1-1] + S[i1-1][j1-1]
//           = sum_{k=i1..i2} D(k, j),   D(k, j) = P(k, j2) - P(k, j1 - 1),
// with i1 = i - rr, i2 = i + rr, j1 = j - rc, j2 = j + rc (clipped) and P the
// row prefix sums (the SAT's row pass).  The SAT's column pass, differenced
// over the window rows, is a running sum V(i) = V(i-1) + D(i+rr) - D(i-rr-1)
// down each column, so a warp that walks its strip top to bottom evaluates
// the four-corner formula with one row scan, two prefix reads and one
// add/subtract per pixel -- no SAT in HBM, no SAT tile in shared memory, no
// barrier between warps (every warp owns its own units).
//
// Unit = (image, strip c of SW = 32 OPL output columns, block of RB output
// rows): OPL = 4 (128 columns) for uint32 sums, 2 (64 columns) for float64
// sums, whose shared buffers are twice as wide.  Per input row k of
// [i0 - rr, i1 - 1 + rr]:
//   * lane L holds columns c*SW - 64 + EPS*L .. +EPS-1 (EPS = OPL + 4: the
//     strip plus a 64-column halo each side; rc <= 63), copied by cp.async
//     into a per-warp ring PF rows deep; pieces outside the image are
//     zero-filled, so the prefix P over the span is flat outside the image and
//     the clipping of the window comes for free;
//   * P: EPS-element serial scan per lane + warp shuffle scan, written to the
//     warp's shared P buffer (P is offset by the span's start, which cancels
//     in D);
//   * D for the lane's output columns j = c*SW + L + 32e (e < OPL:
//     consecutive lanes, consecutive words: conflict-free reads);
//   * V += D - D(k - 2rr - 1), the old D from a per-warp shared ring of
//     2rr + 1 rows; output row k - rr once the window is complete, stored as
//     OPL coalesced warp stores.
// The first 2rr rows of a unit are a warm-up (input re-read from L2); units
// are sized by the host to fill one wave of resident warps.  Input traffic
// ~ (1 + 2rr/RB) x eb_in per pixel from HBM (halo columns and warm-up rows
// hit L2), output eb_out per pixel.  DESIGN.md Sec. 4.12.
#pragma once
#include "sat_common.h"
#include "sat_device.cuh"

namespace sat {

struct BoxWParams {
    const void* in;        // [batch][rows][cols], element type TI
    void* out;             // [batch][rows][cols], element type TO
    int rows, cols, batch;
    int rr, rc;            // radii (host-clamped; rc <= 63)
    int normalize;         // float only
    int rb;                // output rows per unit
    int nrb;               // row blocks per image
    int nc;                // SW-column strips per image
    long long units;       // batch * nrb * nc
};

// A unit is SW = 32 * OPL output columns: lane L owns outputs c0 + L + 32e
// (e < OPL) and the span positions 8L' .. of the SW + 128 columns around them
// (a 64-column halo each side), EPS = OPL + 4 elements per lane.
template <int OPL>
struct BoxWGeom {
    static constexpr int SW = 32 * OPL;          // output columns per unit
    static constexpr int SPAN = SW + 128;        // loaded columns
    static constexpr int EPS = SPAN / 32;        // span elements per lane
};

// shared bytes per warp: raw-row ring (PF rows of the span, TI) + the P buffer
// (SPAN entries) + the D ring (2rr + 1 rows of SW)
template <typename TI, typename TS, int PF, int OPL = 4>
SAT_HD size_t boxw_warp_smem(int rr) {
    using G = BoxWGeom<OPL>;
    return size_t(PF) * G::SPAN * sizeof(TI) + (size_t(G::SPAN) + size_t(2 * rr + 1) * G::SW) * sizeof(TS);
}

// Asynchronous copy of the lane's EPS span elements into the warp's raw-row
// ring in pieces of 8 B (uint8: one piece of 8; 4-byte types with EPS = 8:
// two 16-B pieces; EPS = 6: three 8-B pieces); a piece outside the image
// copies nothing and is zero-filled (src-size 0), which is the window
// clipping.  ok = bit mask of the pieces inside the image.
// row = column 0 of the row; a piece outside the image reads from `row`
// itself (a valid address, no bytes taken)
template <typename TI, int EPS>
__device__ __forceinline__ void boxw_cp(uint32_t dst, const TI* row, int s0, uint32_t ok) {
    if constexpr (sizeof(TI) == 1) {
        static_assert(EPS == 8, "uint8: 8 span elements per lane");
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" :: "r"(dst), "l"(row + ((ok & 1u) ? s0 : 0)),
                     "r"((ok & 1u) ? 8 : 0) : "memory");
    } else if constexpr (EPS == 8) {
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            const bool in = (ok >> q) & 1u;
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" :: "r"(dst + 16 * q),
                         "l"(row + (in ? s0 + 4 * q : 0)), "r"(in ? 16 : 0) : "memory");
        }
    } else {
        static_assert(EPS % 2 == 0, "8-B pieces");
#pragma unroll
        for (int q = 0; q < EPS / 2; ++q) {
            const bool in = (ok >> q) & 1u;
            asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" :: "r"(dst + 8 * q),
                         "l"(row + (in ? s0 + 2 * q : 0)), "r"(in ? 8 : 0) : "memory");
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void boxw_cp_wait() { asm volatile("cp.async.wait_group %0;" :: "n"(N) : "memory"); }

template <typename TI, typename TS, int EPS>
__device__ __forceinline__ void boxw_widen(uint32_t raddr, TS (&e)[EPS]) {
    if constexpr (sizeof(TI) == 1) {
        uint32_t a, b;
        asm volatile("ld.shared.v2.b32 {%0, %1}, [%2];" : "=r"(a), "=r"(b) : "r"(raddr));
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            e[t] = TS(__byte_perm(a, 0u, 0x4440u + t));
            e[4 + t] = TS(__byte_perm(b, 0u, 0x4440u + t));
        }
    } else {
        uint32_t w[EPS];
#pragma unroll
        for (int q = 0; q < EPS / 2; ++q)
            asm volatile("ld.shared.v2.b32 {%0, %1}, [%2];" : "=r"(w[2 * q]), "=r"(w[2 * q + 1]) : "r"(raddr + 8 * q));
#pragma unroll
        for (int t = 0; t < EPS; ++t) {
            if constexpr (std::is_same<TI, float>::value) e[t] = TS(__uint_as_float(w[t]));
            else e[t] = TS(w[t]);
        }
    }
}

template <typename TS>
__device__ __forceinline__ TS boxw_lds(uint32_t a) {
    if constexpr (sizeof(TS) == 4) {
        uint32_t v;
        asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a));
        return TS(v);
    } else {
        double v;
        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
        return v;
    }
}
template <typename TS>
__device__ __forceinline__ void boxw_sts(uint32_t a, TS v) {
    if constexpr (sizeof(TS) == 4) asm volatile("st.shared.b32 [%0], %1;" :: "r"(a), "r"(uint32_t(v)));
    else asm volatile("st.shared.f64 [%0], %1;" :: "r"(a), "d"(v));
}

template <typename TI, typename TS, typename TO, int NWARP, int PF, int OPL = 4>
__global__ void __launch_bounds__(NWARP * 32) sat_boxw_kernel(const BoxWParams bp) {
    using G = BoxWGeom<OPL>;
    constexpr int SW = G::SW, SPAN = G::SPAN, EPS = G::EPS;
    extern __shared__ __align__(1024) uint8_t smem[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int ring_rows = 2 * bp.rr + 1;
    // per-warp shared layout: raw ring [PF][SPAN] TI | P [SPAN] TS | D ring [2rr+1][SW] TS
    const uint32_t wbase = smem_u32(smem) + uint32_t(warp * boxw_warp_smem<TI, TS, PF, OPL>(bp.rr));
    const uint32_t raw0 = wbase + uint32_t(EPS * lane * sizeof(TI));        // lane's slot in raw row 0
    constexpr uint32_t RAW_ROW = SPAN * sizeof(TI);
    const uint32_t pb = wbase + PF * RAW_ROW;
    const uint32_t ring0 = pb + SPAN * sizeof(TS) + lane * sizeof(TS);
    const uint32_t ring_end = ring0 + uint32_t(ring_rows) * SW * sizeof(TS);
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const long long unit = (long long)blockIdx.x * NWARP + warp;
    if (unit >= bp.units) return;
    const int c = int(unit % bp.nc);
    const long long r2 = unit / bp.nc;
    const int rbk = int(r2 % bp.nrb);
    const int img = int(r2 / bp.nrb);
    const int i0 = rbk * bp.rb, i1 = min(bp.rows, i0 + bp.rb);
    const int kstart = max(0, i0 - bp.rr), kend = i1 - 1 + bp.rr;   // inclusive
    const int klast = min(kend, bp.rows - 1);                        // last row that exists
    const int c0 = c * SW;
    const int s0 = c0 - 64 + EPS * lane;
    // copy pieces (8 B for uint8, 16 B at EPS 8, 8 B at EPS 6) lie wholly
    // inside or outside the image: host requires cols % 8 == 0 for uint8,
    // % 4 == 0 for 4-byte types
    constexpr int PIECE = sizeof(TI) == 1 ? 8 : (EPS == 8 ? 4 : 2);   // elements per piece
    uint32_t ok = 0;
#pragma unroll
    for (int q = 0; q < EPS / PIECE; ++q)
        if (s0 + PIECE * q >= 0 && s0 + PIECE * (q + 1) <= bp.cols) ok |= 1u << q;
    const TI* src = reinterpret_cast<const TI*>(bp.in) + (int64_t(img) * bp.rows + kstart) * bp.cols;  // row kstart
    TO* dst = reinterpret_cast<TO*>(bp.out) + (int64_t(img) * bp.rows + i0) * bp.cols + c0 + lane;
    // shared addresses of the window's corner columns in P (span index =
    // column - (c0 - 64)); clipping is done by the zero fill
    uint32_t ar[OPL], al[OPL];
    bool jin[OPL];
    int ww[OPL];
#pragma unroll
    for (int e = 0; e < OPL; ++e) {
        const int x = 64 + lane + 32 * e;
        ar[e] = pb + uint32_t((x + bp.rc) * sizeof(TS));
        al[e] = pb + uint32_t((x - bp.rc - 1) * sizeof(TS));
        const int j = c0 + lane + 32 * e;
        jin[e] = j < bp.cols;
        ww[e] = min(j + bp.rc, bp.cols - 1) - max(j - bp.rc, 0) + 1;
    }
    // prologue: rows kstart .. kstart + PF - 1 in flight (empty groups past klast)
#pragma unroll
    for (int u = 0; u < PF; ++u) {
        if (kstart + u <= klast) boxw_cp<TI, EPS>(raw0 + u * RAW_ROW, src + int64_t(u) * bp.cols, s0, ok);
        else asm volatile("cp.async.commit_group;" ::: "memory");
    }
    const TI* nxt = src + int64_t(PF) * bp.cols;                  // row k + PF
    TS V[OPL];
#pragma unroll
    for (int e = 0; e < OPL; ++e) V[e] = TS(0);
    uint32_t rs = ring0;                                          // ring slot of row k
    int q = 0;                                                    // raw ring slot of row k
    for (int k = kstart; k <= kend; ++k) {
        TS D[OPL];
#pragma unroll
        for (int e = 0; e < OPL; ++e) D[e] = TS(0);
        if (k <= klast) {
            boxw_cp_wait<PF - 1>();                               // row k landed (this lane's copies)
            TS e8[EPS];
            boxw_widen<TI, TS, EPS>(raw0 + q * RAW_ROW, e8);
            // refill the slot with row k + PF (an empty group keeps the count);
            // a lane reads and refills only its own bytes of the slot
            if (k + PF <= klast) boxw_cp<TI, EPS>(raw0 + q * RAW_ROW, nxt, s0, ok);
            else asm volatile("cp.async.commit_group;" ::: "memory");
            nxt += bp.cols;
#pragma unroll
            for (int t = 1; t < EPS; ++t) e8[t] += e8[t - 1];
            const TS inc = warp_inclusive_scan(e8[EPS - 1], lane);
            TS exc;
            if constexpr (std::is_same<TS, uint32_t>::value) {
                exc = inc - e8[EPS - 1];
            } else {
                exc = __shfl_up_sync(0xffffffffu, inc, 1);
                if (lane == 0) exc = TS(0);
            }
            const uint32_t pw = pb + uint32_t(EPS * lane * sizeof(TS));
            if constexpr (sizeof(TS) == 4) {
                static_assert(EPS == 8, "uint32 sums: 8 span elements per lane");
                asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" :: "r"(pw), "r"(e8[0] + exc), "r"(e8[1] + exc),
                             "r"(e8[2] + exc), "r"(e8[3] + exc) : "memory");
                asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" :: "r"(pw + 16), "r"(e8[4] + exc),
                             "r"(e8[5] + exc), "r"(e8[6] + exc), "r"(e8[7] + exc) : "memory");
            } else {
#pragma unroll
                for (int t = 0; t < EPS; t += 2)
                    asm volatile("st.shared.v2.f64 [%0], {%1, %2};" :: "r"(pw + 8 * t), "d"(e8[t] + exc),
                                 "d"(e8[t + 1] + exc) : "memory");
            }
            __syncwarp();
#pragma unroll
            for (int e = 0; e < OPL; ++e) D[e] = boxw_lds<TS>(ar[e]) - boxw_lds<TS>(al[e]);
            __syncwarp();                                         // P reads done before the next row's writes
            if (++q == PF) q = 0;
        }
        // vertical window: V(k - rr) = sum of D over rows k - 2rr .. k
        if (k - kstart >= ring_rows) {
#pragma unroll
            for (int e = 0; e < OPL; ++e) V[e] -= boxw_lds<TS>(rs + 32 * e * sizeof(TS));
        }
#pragma unroll
        for (int e = 0; e < OPL; ++e) {
            boxw_sts<TS>(rs + 32 * e * sizeof(TS), D[e]);
            V[e] += D[e];
        }
        rs += SW * sizeof(TS);
        if (rs == ring_end) rs = ring0;
        const int i = k - bp.rr;
        if (i >= i0) {
            if constexpr (std::is_same<TS, uint32_t>::value) {
#pragma unroll
                for (int e = 0; e < OPL; ++e)
                    if (jin[e]) __stcs(dst + 32 * e, TO(int32_t(V[e])));
            } else {
                int hh = 1;
                if (bp.normalize) hh = min(i + bp.rr, bp.rows - 1) - max(i - bp.rr, 0) + 1;
#pragma unroll
                for (int e = 0; e < OPL; ++e) {
                    TS sv = V[e];
                    if (bp.normalize) sv = sv / TS(int64_t(hh) * int64_t(ww[e]));
                    if (jin[e]) __stcs(dst + 32 * e, TO(sv));
                }
            }
            dst += bp.cols;
        }
    }
    boxw_cp_wait<0>();
}

}  // namespace sat
