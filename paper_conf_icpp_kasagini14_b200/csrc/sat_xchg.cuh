// sat_xchg.cuh -- the sharded mode's exchange fused into its kernels over
// peer memory (north star (3)).
//
// Row strips: rank p needs carry_p[j] = sum_{q<p}
// totals_q[j].  The NCCL path runs totals kernel -> all-gather -> exscan
// kernel -> seeded SAT.  Here:
//   * the totals kernel's epilogue stores rank p's totals straight into slot p
//     of every higher rank's mailbox (P2P stores over NVLink through
//     IPC-mapped pointers), and the last block to finish raises a flag
//     (st.release.sys) in each of those mailboxes;
//   * the SAT kernel's band 0 waits for the flags of ranks < p
//     (ld.acquire.sys), sums their slots in rank order into its first input
//     row and writes its acknowledgement back into each producer's mailbox.
// Mailboxes are double-buffered by call parity; before reusing a parity a
// producer waits for every consumer's acknowledgement of the call two back,
// so no data is overwritten before it is read and no barrier is needed.
#pragma once
#include "sat_common.h"
#include "sat_device.cuh"

namespace sat {

// The consumer side runs inside the band kernel (sat_band.cuh, ColSeed):
// band 0 waits for the flags of ranks < p, adds sum_{q<p} slot[par][q] (q
// ascending) to its first input row, and the last band-0 unit acknowledges.
//
// Mailbox layout (per rank, `cols` values of T per slot):
//   uint64 flag[2][P]     flag[par][q] = epoch of the totals q wrote in slot par
//   uint64 ack[P]         ack[c]       = last epoch consumer c finished reading
//   T      slot[2][P][cols]
struct XchgLayout {
    int P;
    int64_t cols;
    size_t esz;
    __host__ __device__ size_t flags_off() const { return 0; }
    __host__ __device__ size_t acks_off() const { return size_t(2) * P * 8; }
    __host__ __device__ size_t slots_off() const { return ((size_t(3) * P * 8 + 255) / 256) * 256; }
    __host__ __device__ size_t slot_off(int par, int q) const {
        return slots_off() + (size_t(par) * P + q) * ((size_t(cols) * esz + 255) / 256 * 256);
    }
    __host__ __device__ size_t bytes() const { return slot_off(2, 0); }
};

struct XchgParams {
    XchgLayout L;
    int rank;
    unsigned long long epoch;          // this call (>= 1)
    uint8_t* mine;                     // own mailbox (local pointer)
    uint8_t* peers[16];                // peers[q]: rank q's mailbox as seen from this rank
    unsigned int* done;                // per-rank block counter (local, zero between calls)
};

__device__ __forceinline__ void st_release_sys_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_sys_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void wait_at_least(const uint64_t* p, uint64_t want, uint32_t what) {
    if (ld_acquire_sys_u64(p) >= want) return;
    SpinGuard guard(what, uint32_t(want));
    while (ld_acquire_sys_u64(p) < want) { __nanosleep(128); guard.tick(); }
}

// Column totals of a strip in ONE launch (the sharded mode's extra read).
// grid = (nc, splits), 256 threads: block (J, sp) sums rows [sp*seg, (sp+1)*seg)
// of the 128 columns of chunk J (8 independent 16-B loads in flight per lane)
// into part[sp][J*128 ..]; the last block to arrive for chunk J (counter
// cnt[J]) adds the splits in split order (deterministic), writes the totals
// and -- in the fused exchange -- stores them straight into slot (epoch & 1,
// rank) of every higher rank's mailbox; the last chunk column to finish
// (counter cnt[nc]) raises those ranks' flags with st.release.sys.  Before
// the first store into a parity, the consumers' acknowledgements of the call
// two back are awaited.  Counters reset themselves.
struct TotalsParams {
    const void* in;
    int64_t rows, cols;
    int64_t seg_rows;
    int splits;
    void* part;                 // [splits][nc*TW]
    unsigned int* cnt;          // [nc + 1], zero between calls
    void* totals;               // nullable: cols entries on this device
    int push;                   // 1: fused exchange (x)
    XchgParams x;
};

template <typename T>
__global__ void __launch_bounds__(256) sat_colsum_kernel(const TotalsParams tp) {
    const int J = blockIdx.x, sp = blockIdx.y;
    const int nc = gridDim.x;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const T* in = static_cast<const T*>(tp.in);
    const int64_t cols = tp.cols;
    const int64_t c = int64_t(J) * TW + 4 * lane;
    const int64_t r0 = int64_t(sp) * tp.seg_rows;
    const int64_t r1 = min(tp.rows, r0 + tp.seg_rows);
    const bool vec = (cols % 4 == 0) && ((reinterpret_cast<uintptr_t>(in) & 15) == 0) && (c + 3 < cols);
    T cs[4] = {T(0), T(0), T(0), T(0)};
    int64_t r = r0 + warp;
    if (vec) {
        for (; r + 56 < r1; r += 64) {
            T e[8][4];
#pragma unroll
            for (int q = 0; q < 8; ++q) ldg4<T>(in + (r + 8 * q) * cols + c, e[q]);
#pragma unroll
            for (int q = 0; q < 8; ++q)
#pragma unroll
                for (int i = 0; i < 4; ++i) cs[i] += e[q][i];
        }
    }
    for (; r < r1; r += 8) {
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
    __shared__ int s_last;
#pragma unroll
    for (int i = 0; i < 4; ++i) sm[warp][4 * lane + i] = cs[i];
    __syncthreads();
    T* part = static_cast<T*>(tp.part);
    if (threadIdx.x < TW) {
        T s = T(0);
        for (int w = 0; w < 8; ++w) s += sm[w][threadIdx.x];
        part[int64_t(sp) * nc * TW + int64_t(J) * TW + threadIdx.x] = s;
    }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = atomicAdd(&tp.cnt[J], 1u) == unsigned(tp.splits - 1);
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    const XchgParams& x = tp.x;
    const int par = int(x.epoch & 1);
    const int P = x.L.P;
    if (tp.push && threadIdx.x == 0 && x.epoch > 2) {
        // the consumers of this parity's previous use (epoch - 2) are done
        for (int q = x.rank + 1; q < P; ++q)
            wait_at_least(reinterpret_cast<const uint64_t*>(x.mine + x.L.acks_off()) + q, x.epoch - 2,
                          0x10000000u | uint32_t(q));
    }
    __syncthreads();
    if (threadIdx.x < TW) {
        const int64_t cc = int64_t(J) * TW + threadIdx.x;
        if (cc < cols) {
            T s = T(0);
            for (int k = 0; k < tp.splits; ++k) s += __ldcg(part + int64_t(k) * nc * TW + cc);
            if (tp.totals) static_cast<T*>(tp.totals)[cc] = s;
            if (tp.push)
                for (int q = x.rank + 1; q < P; ++q)
                    reinterpret_cast<T*>(x.peers[q] + x.L.slot_off(par, x.rank))[cc] = s;
        }
    }
    if (threadIdx.x == 0) tp.cnt[J] = 0u;
    if (!tp.push) return;
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned int n = atomicAdd(&tp.cnt[nc], 1u);
        if (n == unsigned(nc - 1)) {
            tp.cnt[nc] = 0u;
            __threadfence_system();
            for (int q = x.rank + 1; q < P; ++q)
                st_release_sys_u64(reinterpret_cast<uint64_t*>(x.peers[q] + x.L.flags_off()) + par * P + x.rank,
                                   x.epoch);
        }
    }
}

// A rank with an empty strip still consumes its producers' totals: wait for
// the flags, acknowledge (keeps the double-buffered protocol in step).
__global__ void sat_xchg_drain_kernel(XchgParams x) {
    const int par = int(x.epoch & 1);
    const int P = x.L.P;
    const int q = threadIdx.x;
    if (q < x.rank) {
        wait_at_least(reinterpret_cast<const uint64_t*>(x.mine + x.L.flags_off()) + par * P + q, x.epoch,
                      0x18000000u | uint32_t(q));
        st_release_sys_u64(reinterpret_cast<uint64_t*>(x.peers[q] + x.L.acks_off()) + x.rank, x.epoch);
    }
}

}  // namespace sat
