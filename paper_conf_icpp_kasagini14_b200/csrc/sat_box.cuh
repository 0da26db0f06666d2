// sat_box.cuh -- consumers of a SAT: the reason the
// paper computes SATs at all -- "the sum of any rectangular area can be
// computed in O(1) time" from four SAT reads (Sec. I).
//
//  * sat_box_kernel: box filter, out[i][j] = sum of a over rows |k - i| <= rr
//    and columns |l - j| <= rc, clipped to the matrix, by inclusion-exclusion
//    over the SAT S:  S[i2][j2] - S[i1-1][j2] - S[i2][j1-1] + S[i1-1][j1-1]
//    (terms with index -1 are 0), optionally divided by the clipped window's
//    element count (box mean).  One thread per output element; a warp reads
//    two SAT rows at two column offsets, all coalesced; the 2rr+1 rows a
//    block row shares stay in L2.
//  * sat_rect_kernel: K arbitrary rectangle queries (image, r0, c0, r1, c1),
//    inclusive and clipped to the matrix, one thread each.
#pragma once
#include "sat_common.h"

namespace sat {

template <typename T>
__device__ __forceinline__ T rect_from_sat(const T* S, int64_t cols, int64_t i1, int64_t j1, int64_t i2,
                                           int64_t j2) {
    T v = S[i2 * cols + j2];
    if (i1 > 0) v -= S[(i1 - 1) * cols + j2];
    if (j1 > 0) v -= S[i2 * cols + j1 - 1];
    if (i1 > 0 && j1 > 0) v += S[(i1 - 1) * cols + j1 - 1];
    return v;
}

template <typename TO, typename T>
__device__ __forceinline__ TO box_out(T v) {
    if constexpr (std::is_same<T, uint32_t>::value) return TO(int32_t(v));   // int32 bits, mod 2^32
    else return TO(v);
}

// grid: (ceil(cols / 256), min(ceil(rows / BOX_RB), 65535), batch); block 256.
// A thread owns one column and BOX_RB consecutive rows per iteration and
// issues all 4*BOX_RB SAT loads before any arithmetic (memory-level
// parallelism: one row per thread left the kernel latency-bound).  IDX is the
// in-image index type: int32 when rows*cols < 2^31 (the kernel was
// instruction-bound on 64-bit index arithmetic: ncu SM throughput 65 %, DRAM
// 23 %); the image base is a 64-bit pointer either way.
constexpr int BOX_RB = 8;
template <typename T, typename TO, typename IDX>
__global__ void __launch_bounds__(256) sat_box_kernel(const T* __restrict__ S, TO* __restrict__ out,
                                                      IDX rows, IDX cols, int rr, int rc,
                                                      int normalize) {
    const IDX j = IDX(blockIdx.x) * IDX(blockDim.x) + IDX(threadIdx.x);
    if (j >= cols) return;
    const int64_t img = blockIdx.z;
    const T* Si = S + img * int64_t(rows) * int64_t(cols);
    TO* Oi = out + img * int64_t(rows) * int64_t(cols);
    const IDX j1 = j - rc > 0 ? j - rc : IDX(0);
    const IDX j2 = j + rc < cols - 1 ? j + rc : cols - 1;
    const bool left = j1 > 0;
    const IDX jl = left ? j1 - 1 : IDX(0);
    const IDX wc = j2 - j1 + 1;
    for (IDX i0 = IDX(blockIdx.y) * BOX_RB; i0 < rows; i0 += IDX(gridDim.y) * BOX_RB) {
        T a[BOX_RB], b[BOX_RB], c[BOX_RB], d[BOX_RB];
#pragma unroll
        for (int k = 0; k < BOX_RB; ++k) {
            const IDX i = i0 + k < rows ? i0 + k : rows - 1;
            const IDX i1 = i - rr > 0 ? i - rr : IDX(0);
            const IDX i2 = i + rr < rows - 1 ? i + rr : rows - 1;
            const T* s2 = Si + i2 * cols;
            const T* s1 = Si + (i1 > 0 ? i1 - 1 : IDX(0)) * cols;
            a[k] = s2[j2];
            b[k] = i1 > 0 ? s1[j2] : T(0);
            c[k] = left ? s2[jl] : T(0);
            d[k] = (i1 > 0 && left) ? s1[jl] : T(0);
        }
#pragma unroll
        for (int k = 0; k < BOX_RB; ++k) {
            const IDX i = i0 + k;
            if (i >= rows) break;
            T v = ((a[k] - b[k]) - c[k]) + d[k];
            if constexpr (!std::is_same<T, uint32_t>::value) {
                if (normalize) {
                    const IDX i1 = i - rr > 0 ? i - rr : IDX(0);
                    const IDX i2 = i + rr < rows - 1 ? i + rr : rows - 1;
                    v = v / T(int64_t(i2 - i1 + 1) * int64_t(wc));
                }
            }
            Oi[i * cols + j] = box_out<TO>(v);
        }
    }
}

// rects: [K][5] int32 = (image, r0, c0, r1, c1), inclusive; clipped to the
// matrix; an empty (clipped) rectangle or a bad image index sums to 0.
template <typename T>
__global__ void __launch_bounds__(256) sat_rect_kernel(const T* __restrict__ S, int64_t batch, int64_t rows,
                                                       int64_t cols, const int32_t* __restrict__ rects,
                                                       int64_t K, T* __restrict__ out) {
    for (int64_t q = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; q < K;
         q += int64_t(gridDim.x) * blockDim.x) {
        const int32_t* r = rects + q * 5;
        const int64_t b = r[0];
        int64_t i1 = r[1], j1 = r[2], i2 = r[3], j2 = r[4];
        if (i1 < 0) i1 = 0;
        if (j1 < 0) j1 = 0;
        if (i2 > rows - 1) i2 = rows - 1;
        if (j2 > cols - 1) j2 = cols - 1;
        T v = T(0);
        if (b >= 0 && b < batch && i1 <= i2 && j1 <= j2)
            v = rect_from_sat(S + b * rows * cols, cols, i1, j1, i2, j2);
        out[q] = v;
    }
}

}  // namespace sat
