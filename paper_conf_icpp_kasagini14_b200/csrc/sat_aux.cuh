// sat_aux.cuh -- the smaller kernels around the band kernel.
//
//  * 2R1W Step 1 (reduce) and Step 2 (carries), PAPER.md P:L1059-L1137,
//    P:L1855-L1871 (Sec. V): per tile the column sums C and row sums R are
//    reduced (1R, small W); Step 2 turns them into, per tile, the row carry L
//    (the paper's prefix of R, stored transposed as the paper stores R^T for
//    coalescing) and the SAT row above the tile (the paper's C prefix
//    plus the corner from SAT(S)).  Step 3 is the band kernel with external
//    carries.
//  * sharded mode (north star (3)): the strip's column totals and the
//    exclusive scan of the all-gathered totals over ranks.
#pragma once
#include "sat_common.h"
#include "sat_device.cuh"

namespace sat {

struct TileParams {
    const void* in;
    int64_t rows, cols;
    int batch, nb, nc, total_bands, th;
    int region, tA;
    void* Bt;        // [total_bands][nc*TW]: chunk-local prefix of the tile's column sums
    void* RS;        // [nc][total_bands*th]: the tile's row sums (R^T layout)
};

// Step 1: one CTA (8 warps) per tile; grid = (nc, total_bands).
template <typename T>
__global__ void __launch_bounds__(256)
sat_reduce_kernel(const TileParams p)
{
    const int J = blockIdx.x, gb = blockIdx.y;
    const int img = gb / p.nb, band = gb % p.nb;
    int j0, j1;
    region_range(p.region, p.tA, p.nb, p.nc, band, j0, j1);
    if (J < j0 || J >= j1) return;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    __shared__ T colp[8][TW];
    const T* gin = reinterpret_cast<const T*>(p.in) + int64_t(img) * p.rows * p.cols;
    const int64_t c = int64_t(J) * TW + 4 * lane;
    const bool vec = (p.cols % 4 == 0) && ((reinterpret_cast<uintptr_t>(p.in) & 15) == 0);
    T cs[4] = {T(0), T(0), T(0), T(0)};
    T* rs = reinterpret_cast<T*>(p.RS) + int64_t(J) * p.total_bands * p.th + int64_t(gb) * p.th;
    for (int r = warp; r < p.th; r += 8) {
        const int64_t row = int64_t(band) * p.th + r;
        T e[4] = {T(0), T(0), T(0), T(0)};
        if (row < p.rows) {
            if (vec && c + 3 < p.cols) {
                ldg4<T>(gin + row * p.cols + c, e);
            } else {
#pragma unroll
                for (int i = 0; i < 4; ++i) if (c + i < p.cols) e[i] = gin[row * p.cols + c + i];
            }
        }
        T sr = (e[0] + e[1]) + (e[2] + e[3]);
#pragma unroll
        for (int i = 0; i < 4; ++i) cs[i] += e[i];
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) sr += __shfl_xor_sync(0xffffffffu, sr, d);
        if (lane == 0) rs[r] = sr;
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) colp[warp][4 * lane + i] = cs[i];
    __syncthreads();
    if (warp == 0) {
        T v[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            T s = T(0);
            for (int w = 0; w < 8; ++w) s += colp[w][4 * lane + i];
            v[i] = s;
        }
        v[1] += v[0]; v[2] += v[1]; v[3] += v[2];
        const T inc = warp_inclusive_scan(v[3], lane);
        T exc = __shfl_up_sync(0xffffffffu, inc, 1);
        if (lane == 0) exc = T(0);
        T* bt = reinterpret_cast<T*>(p.Bt) + int64_t(gb) * p.nc * TW + c;
#pragma unroll
        for (int i = 0; i < 4; ++i) bt[i] = v[i] + exc;
    }
}

struct CarryParams {
    int64_t rows, cols;
    int batch, nb, nc, total_bands, th;
    int region, tA;
    const void* RS;      // [nc][total_bands*th]
    const void* Bt;      // [total_bands][nc*TW]
    const void* Lb;      // [total_bands*th] row carry at the region's first chunk (nullable = 0)
    void* Lx;            // [nc+1][total_bands*th] row carry at chunk start
    void* Lsum;          // [total_bands][nc+1] sum over the band's rows of Lx
    void* TopX;          // [total_bands][nc*TW] SAT row above each tile
    const void* out;     // final SAT values outside the region (region B boundary)
};

// Step 2a: row carries.  One CTA per band, one thread per row of the band.
// Writes Lx for J in [j0, j1] (j1 inclusive: the carry into the next region).
template <typename T>
__global__ void sat_carry_rows_kernel(const CarryParams p)
{
    const int gb = blockIdx.x;
    const int band = gb % p.nb;
    int j0, j1;
    region_range(p.region, p.tA, p.nb, p.nc, band, j0, j1);
    const int r = threadIdx.x;           // blockDim.x == th rounded up to 32
    const bool valid = r < p.th;
    const int64_t stride = int64_t(p.total_bands) * p.th;
    const int64_t idx = int64_t(gb) * p.th + r;
    T L = (p.Lb && valid) ? reinterpret_cast<const T*>(p.Lb)[idx] : T(0);
    __shared__ T red[32];
    const int warp = r >> 5, lane = r & 31, nw = (p.th + 31) / 32;
    for (int J = j0; J <= j1 && J <= p.nc; ++J) {
        if (valid) reinterpret_cast<T*>(p.Lx)[int64_t(J) * stride + idx] = L;
        T s = L;
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
        if (lane == 0) red[warp] = s;
        __syncthreads();
        if (r == 0) {
            T t = T(0);
            for (int w = 0; w < nw; ++w) t += red[w];
            reinterpret_cast<T*>(p.Lsum)[int64_t(gb) * (p.nc + 1) + J] = t;
        }
        __syncthreads();
        if (J < j1 && valid) L += reinterpret_cast<const T*>(p.RS)[int64_t(J) * stride + idx];
    }
}

// Step 2b: SAT row above every region tile.  One thread per (image, column).
// Walks down the region's tiles of the column's chunk:
//   Top(I+1) = Top(I) + Lsum(I, J) + Bt(I)[c]
// starting from 0 at the matrix top, or -- for region B -- from the final SAT
// row just above the region (already in `out`).
template <typename T>
__global__ void sat_carry_top_kernel(const CarryParams p)
{
    const int64_t c = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    const int img = blockIdx.y;
    const int W = p.nc * TW;
    if (c >= W) return;
    const int J = int(c / TW);
    // bands I of this image whose tile (I, J) is in the region: contiguous
    int i0 = -1, i1 = -1;
    for (int I = 0; I < p.nb; ++I) {
        int j0, j1;
        region_range(p.region, p.tA, p.nb, p.nc, I, j0, j1);
        if (J >= j0 && J < j1) { if (i0 < 0) i0 = I; i1 = I + 1; }
    }
    if (i0 < 0) return;
    T top = T(0);
    if (i0 > 0 && c < p.cols) {
        const T* o = reinterpret_cast<const T*>(p.out) + int64_t(img) * p.rows * p.cols;
        top = o[(int64_t(i0) * p.th - 1) * p.cols + c];
    }
    for (int I = i0; I < i1; ++I) {
        const int gb = img * p.nb + I;
        reinterpret_cast<T*>(p.TopX)[int64_t(gb) * W + c] = top;
        top += reinterpret_cast<const T*>(p.Lsum)[int64_t(gb) * (p.nc + 1) + J]
             + reinterpret_cast<const T*>(p.Bt)[int64_t(gb) * W + c];
    }
}

// Sharded mode: partial column sums of row segments.  grid = (nc, splits),
// 256 threads: warp w sums rows w, w+8, ... of the segment for 128 columns.
template <typename T>
__global__ void __launch_bounds__(256)
sat_colsum_partial_kernel(const T* __restrict__ in, T* __restrict__ part,
                          int64_t rows, int64_t cols, int64_t seg_rows)
{
    const int J = blockIdx.x, sp = blockIdx.y;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t c = int64_t(J) * TW + 4 * lane;
    const int64_t r0 = int64_t(sp) * seg_rows;
    int64_t r1 = r0 + seg_rows;
    if (r1 > rows) r1 = rows;
    const bool vec = (cols % 4 == 0) && ((reinterpret_cast<uintptr_t>(in) & 15) == 0) && (c + 3 < cols);
    T cs[4] = {T(0), T(0), T(0), T(0)};
    for (int64_t r = r0 + warp; r < r1; r += 8) {
        if (vec) {
            T e[4];
            ldg4<T>(in + r * cols + c, e);
#pragma unroll
            for (int i = 0; i < 4; ++i) cs[i] += e[i];
        } else {
#pragma unroll
            for (int i = 0; i < 4; ++i) if (c + i < cols) cs[i] += in[r * cols + c + i];
        }
    }
    __shared__ T sm[8][TW];
#pragma unroll
    for (int i = 0; i < 4; ++i) sm[warp][4 * lane + i] = cs[i];
    __syncthreads();
    if (threadIdx.x < TW) {
        T s = T(0);
        for (int w = 0; w < 8; ++w) s += sm[w][threadIdx.x];
        const int64_t cc = int64_t(J) * TW + threadIdx.x;
        part[int64_t(sp) * gridDim.x * TW + cc] = s;
    }
}

// Sum the partials in split order (deterministic); write cols entries.
template <typename T>
__global__ void sat_colsum_final_kernel(const T* __restrict__ part, T* __restrict__ totals,
                                        int64_t cols, int splits, int width)
{
    const int64_t c = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (c >= cols) return;
    T s = T(0);
    for (int sp = 0; sp < splits; ++sp) s += part[int64_t(sp) * width + c];
    totals[c] = s;
}

// carry[c] = sum_{q < rank} gathered[q][c]  (fixed q order)
template <typename T>
__global__ void sat_rank_exscan_kernel(const T* __restrict__ gathered, T* __restrict__ carry,
                                       int64_t cols, int rank)
{
    const int64_t c = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (c >= cols) return;
    T s = T(0);
    for (int q = 0; q < rank; ++q) s += gathered[int64_t(q) * cols + c];
    carry[c] = s;
}

// sat_row[c] = sum_{c' <= c} carry[c'] : the SAT row just above a strip whose
// column sums above are `carry` (seeded mode).  One CTA of 1024 threads walks
// the row in tiles of 8192 elements with a running carry.
template <typename T>
__global__ void __launch_bounds__(1024)
sat_row_prefix_kernel(const T* __restrict__ carry, T* __restrict__ sat_row, int64_t cols)
{
    __shared__ T wsum[32];
    __shared__ T s_run;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) s_run = T(0);
    __syncthreads();
    for (int64_t base = 0; base < cols; base += 8 * 1024) {
        const int64_t c = base + int64_t(threadIdx.x) * 8;
        T e[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) e[i] = (c + i < cols) ? carry[c + i] : T(0);
#pragma unroll
        for (int i = 1; i < 8; ++i) e[i] += e[i - 1];
        const T inc = warp_inclusive_scan(e[7], lane);
        if (lane == 31) wsum[warp] = inc;
        __syncthreads();
        if (warp == 0) {
            const T w = warp_inclusive_scan(wsum[lane], lane);
            wsum[lane] = w;
        }
        __syncthreads();
        const T off = s_run + (warp > 0 ? wsum[warp - 1] : T(0)) + (inc - e[7]);
#pragma unroll
        for (int i = 0; i < 8; ++i)
            if (c + i < cols) sat_row[c + i] = e[i] + off;
        __syncthreads();
        if (threadIdx.x == 0) s_run += wsum[31];
        __syncthreads();
    }
}

}  // namespace sat
