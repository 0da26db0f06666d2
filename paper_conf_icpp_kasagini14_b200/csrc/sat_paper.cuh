// sat_paper.cuh -- the paper's remaining comparison variants on B200
// (SURVEY.md Sec. 8 row f3): 4R4W and 4R1W.  Neither is on the hot path; they
// complete the columns of Table II.
//
//  * 4R4W (Sec. IV, Lemma 3): column-wise prefix-sums,
//    transpose, column-wise prefix-sums, transpose -- four full read+write
//    passes, all coalesced.  The paper transposes through w x w shared-memory
//    blocks in diagonal arrangement (Fig. 7); here a 32 x 32 tile
//    with one padding column does the same job (the padding shifts each row by
//    one bank, which is what the diagonal arrangement achieves).  The column
//    passes are the band kernel in MODE_COL.
//  * 4R1W (Sec. VI, Formula (1)):
//      b[i][j] = a[i][j] + b[i-1][j] + b[i][j-1] - b[i-1][j-1]
//    (out-of-range terms are 0, R12), evaluated one anti-diagonal
//    t = i + j at a time: rows + cols - 1 stages, one kernel launch per stage
//    exactly as the paper's GPU implementation does, because every
//    element of stage t reads three results of stages t-1 and t-2.
#pragma once
#include "sat_common.h"

namespace sat {

// in: [batch][rows][cols] -> out: [batch][cols][rows].  Block (32, 8); one
// 32 x 32 tile per block iteration.
template <typename T>
__global__ void __launch_bounds__(256) sat_transpose_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                            int64_t rows, int64_t cols) {
    __shared__ T tile[32][33];
    const int64_t img = blockIdx.z;
    const T* src = in + img * rows * cols;
    T* dst = out + img * rows * cols;
    const int64_t ntr = (rows + 31) / 32;
    const int64_t c0 = int64_t(blockIdx.x) * 32;
    for (int64_t tr = blockIdx.y; tr < ntr; tr += gridDim.y) {
        const int64_t r0 = tr * 32;
#pragma unroll
        for (int k = threadIdx.y; k < 32; k += 8) {
            const int64_t r = r0 + k, c = c0 + threadIdx.x;
            if (r < rows && c < cols) tile[k][threadIdx.x] = src[r * cols + c];
        }
        __syncthreads();
#pragma unroll
        for (int k = threadIdx.y; k < 32; k += 8) {
            const int64_t c = c0 + k, r = r0 + threadIdx.x;
            if (r < rows && c < cols) dst[c * rows + r] = tile[threadIdx.x][k];
        }
        __syncthreads();
    }
}

// Wide transpose: 64 x 64 tiles, two consecutive elements per lane on both
// sides (8-B accesses for 4-byte types, 16-B for float64), so every warp reads
// and writes 256-B (512-B) row segments; smem rows padded by one element (at
// most a 2-way bank conflict on the transposed read).  Requires even rows and
// cols and 2-element-aligned pointers (the host falls back to the 32 x 32
// kernel otherwise).  Measured 16384^2 int32: see DESIGN.md Sec. 5.
template <typename T>
struct alignas(2 * sizeof(T)) Pair { T a, b; };

template <typename T>
__global__ void __launch_bounds__(256) sat_transpose64_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                              int64_t rows, int64_t cols) {
    __shared__ T tile[64][65];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t img = blockIdx.z;
    const T* src = in + img * rows * cols;
    T* dst = out + img * rows * cols;
    const int64_t ntr = (rows + 63) / 64;
    const int64_t c0 = int64_t(blockIdx.x) * 64;
    for (int64_t tr = blockIdx.y; tr < ntr; tr += gridDim.y) {
        const int64_t r0 = tr * 64;
        Pair<T> v[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const int64_t r = r0 + warp + 8 * k, c = c0 + 2 * lane;
            v[k] = (r < rows && c < cols) ? *reinterpret_cast<const Pair<T>*>(src + r * cols + c)
                                          : Pair<T>{T(0), T(0)};
        }
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            tile[warp + 8 * k][2 * lane] = v[k].a;
            tile[warp + 8 * k][2 * lane + 1] = v[k].b;
        }
        __syncthreads();
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const int cc = warp + 8 * k;                  // output row = input column c0 + cc
            const int64_t c = c0 + cc, r = r0 + 2 * lane;
            if (c < cols && r < rows)
                *reinterpret_cast<Pair<T>*>(dst + c * rows + r) = Pair<T>{tile[2 * lane][cc], tile[2 * lane + 1][cc]};
        }
        __syncthreads();
    }
}

// One stage of 4R1W: every element (i, t - i) of anti-diagonal t, i in
// [i0, i0 + cnt).  Formula (1) evaluated left to right,
// ((a + b_up) + b_left) - b_diag; uint32 wraps, floating point rounds per add.
template <typename T>
__global__ void __launch_bounds__(256) sat_4r1w_stage_kernel(const T* in, T* out, int64_t rows,
                                                             int64_t cols, int64_t t, int64_t i0,
                                                             int64_t cnt) {
    const int64_t img = blockIdx.y;
    const T* A = in + img * rows * cols;
    T* B = out + img * rows * cols;
    for (int64_t e = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; e < cnt;
         e += int64_t(gridDim.x) * blockDim.x) {
        const int64_t i = i0 + e, j = t - i;
        T v = A[i * cols + j];
        if (i > 0) v += B[(i - 1) * cols + j];
        if (j > 0) v += B[i * cols + j - 1];
        if (i > 0 && j > 0) v -= B[(i - 1) * cols + j - 1];
        B[i * cols + j] = v;
    }
}

}  // namespace sat
