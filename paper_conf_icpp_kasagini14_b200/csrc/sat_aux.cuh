// sat_aux.cuh -- the smaller kernels around the band kernel.
//
//  * 2R1W Step 1 (reduce) and Step 2 (carries), PAPER.md P:L1059-L1137,
//    P:L1855-L1871 (Sec. V): per tile the column sums C and row sums R are
//    reduced (1R, small W); Step 2 turns them into, per tile, the row carry L
//    (the paper's prefix of R, stored transposed as the paper stores R^T for
//    coalescing) and the SAT row above the tile (the paper's C prefix
//    plus the corner from SAT(S)).  Step 3 is the band kernel with external
//    carries.
//  * sharded mode (north star (3)): the exclusive scan of all-gathered
//    totals over ranks (sat_rank_exscan; the sharded entry points fold it into
//    the band kernel's seed instead, sat_common.h ColSeed).
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
    // rows warp, warp+8, ... in batches of 8: all loads of a batch are issued
    // before the first shuffle reduction (memory-level parallelism)
    constexpr int B = 8;
    for (int r0 = warp; r0 < p.th; r0 += 8 * B) {
        T e[B][4];
#pragma unroll
        for (int q = 0; q < B; ++q) {
            const int r = r0 + 8 * q;
            const int64_t row = int64_t(band) * p.th + r;
#pragma unroll
            for (int i = 0; i < 4; ++i) e[q][i] = T(0);
            if (r < p.th && row < p.rows) {
                if (vec && c + 3 < p.cols) {
                    ldg4<T>(gin + row * p.cols + c, e[q]);
                } else {
#pragma unroll
                    for (int i = 0; i < 4; ++i) if (c + i < p.cols) e[q][i] = gin[row * p.cols + c + i];
                }
            }
        }
#pragma unroll
        for (int q = 0; q < B; ++q) {
            const int r = r0 + 8 * q;
            T sr = (e[q][0] + e[q][1]) + (e[q][2] + e[q][3]);
#pragma unroll
            for (int i = 0; i < 4; ++i) cs[i] += e[q][i];
#pragma unroll
            for (int d = 16; d > 0; d >>= 1) sr += __shfl_xor_sync(0xffffffffu, sr, d);
            if (lane == 0 && r < p.th) rs[r] = sr;
        }
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
// Writes Lx for J in [j0, j1] (j1 inclusive: the carry into the next region);
// the loads of RS are independent of the running sum, so batches of 8 are in
// flight at once.  Lsum(J) = sum over the band's rows of Lx(J) = sum(Lb) +
// the exclusive prefix over the region's chunks of the tile totals, and a tile
// total is the last entry of its chunk-local column-sum prefix Bt (Step 1).
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
    const T* __restrict__ RS = reinterpret_cast<const T*>(p.RS);
    T* __restrict__ Lx = reinterpret_cast<T*>(p.Lx);
    const T L0 = (p.Lb && valid) ? reinterpret_cast<const T*>(p.Lb)[idx] : T(0);
    const int jend = min(j1, p.nc);      // last Lx index written
    if (valid) {
        T L = L0;
        constexpr int B = 8;
        for (int J = j0; J <= jend; J += B) {
            T v[B];
#pragma unroll
            for (int q = 0; q < B; ++q)
                v[q] = (J + q < j1) ? RS[int64_t(J + q) * stride + idx] : T(0);
#pragma unroll
            for (int q = 0; q < B; ++q) {
                if (J + q <= jend) Lx[int64_t(J + q) * stride + idx] = L;
                L += v[q];
            }
        }
    }
    // sum over the band's rows of Lb
    __shared__ T red[32];
    const int warp = r >> 5, lane = r & 31, nw = (p.th + 31) / 32;
    T s = valid ? L0 : T(0);
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
    if (lane == 0) red[warp] = s;
    __syncthreads();
    if (warp == 0) {
        T base = T(0);
        for (int w = 0; w < nw; ++w) base += red[w];
        const int W = p.nc * TW;
        const T* bt = reinterpret_cast<const T*>(p.Bt) + int64_t(gb) * W;
        T* lsum = reinterpret_cast<T*>(p.Lsum) + int64_t(gb) * (p.nc + 1);
        for (int J0 = j0; J0 <= jend; J0 += 32) {
            const int J = J0 + lane;
            const T tot = (J < j1) ? bt[int64_t(J) * TW + TW - 1] : T(0);
            const T inc = warp_inclusive_scan(tot, lane);
            // exclusive prefix: by subtraction only in Z/2^32; floats shift
            // (inc - tot would turn an Inf total into NaN)
            T exc;
            if constexpr (std::is_same<T, uint32_t>::value) {
                exc = inc - tot;
            } else {
                exc = __shfl_up_sync(0xffffffffu, inc, 1);
                if (lane == 0) exc = T(0);
            }
            if (J <= jend) lsum[J] = base + exc;
            base += __shfl_sync(0xffffffffu, inc, 31);
        }
    }
}

// Step 2b: SAT row above every region tile:
//   Top(I+1) = Top(I) + Lsum(I, J) + Bt(I)[c]
// starting from 0 at the matrix top, or -- for region B -- from the final SAT
// row just above the region (already in `out`).  Block = 32 columns x 8 band
// groups: each thread sums its group's increments, an exclusive scan over the
// 8 groups gives every group its starting Top, then each thread writes its
// group's rows (loads independent of the running sum, 4 in flight).
template <typename T>
__global__ void __launch_bounds__(256) sat_carry_top_kernel(const CarryParams p)
{
    const int cx = threadIdx.x & 31, grp = threadIdx.x >> 5;
    const int64_t c = int64_t(blockIdx.x) * 32 + cx;
    const int img = blockIdx.y;
    const int W = p.nc * TW;
    const bool live = c < W;
    const int J = live ? int(c / TW) : 0;
    // bands I of this image whose tile (I, J) is in the region: contiguous
    int i0 = -1, i1 = -1;
    for (int I = 0; I < p.nb; ++I) {
        int j0, j1;
        region_range(p.region, p.tA, p.nb, p.nc, I, j0, j1);
        if (J >= j0 && J < j1) { if (i0 < 0) i0 = I; i1 = I + 1; }
    }
    const bool any = live && i0 >= 0;
    const int n = any ? i1 - i0 : 0;
    const int per = (n + 7) / 8;
    const int g0 = i0 + grp * per, g1 = min(i1, g0 + per);
    const T* __restrict__ lsum = reinterpret_cast<const T*>(p.Lsum);
    const T* __restrict__ bt = reinterpret_cast<const T*>(p.Bt);
    T* __restrict__ topx = reinterpret_cast<T*>(p.TopX);
    auto inc = [&](int I) {
        const int gb = img * p.nb + I;
        return lsum[int64_t(gb) * (p.nc + 1) + J] + bt[int64_t(gb) * W + c];
    };
    T part = T(0);
    if (any) {
        int I = g0;
        for (; I + 4 <= g1; I += 4) {
            const T a = inc(I), b = inc(I + 1), d = inc(I + 2), e = inc(I + 3);
            part += (a + b) + (d + e);
        }
        for (; I < g1; ++I) part += inc(I);
    }
    __shared__ T sums[8][32];
    sums[grp][cx] = part;
    __syncthreads();
    if (!any) return;
    T top = T(0);
    if (i0 > 0 && c < p.cols) {
        const T* o = reinterpret_cast<const T*>(p.out) + int64_t(img) * p.rows * p.cols;
        top = o[(int64_t(i0) * p.th - 1) * p.cols + c];
    }
    for (int g = 0; g < grp; ++g) top += sums[g][cx];
    int I = g0;
    for (; I + 4 <= g1; I += 4) {
        const T a = inc(I), b = inc(I + 1), d = inc(I + 2), e = inc(I + 3);
        const int64_t gb = int64_t(img) * p.nb + I;
        topx[gb * W + c] = top; top += a;
        topx[(gb + 1) * W + c] = top; top += b;
        topx[(gb + 2) * W + c] = top; top += d;
        topx[(gb + 3) * W + c] = top; top += e;
    }
    for (; I < g1; ++I) {
        topx[(int64_t(img) * p.nb + I) * W + c] = top;
        top += inc(I);
    }
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

}  // namespace sat
