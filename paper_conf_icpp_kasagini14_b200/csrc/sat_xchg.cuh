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
//   * the SAT prologue (the kernel that turns the carry into the SAT row above
//     the strip) waits for the flags of ranks < p (ld.acquire.sys), sums their
//     slots in rank order and writes its acknowledgement back into each
//     producer's mailbox.
// Mailboxes are double-buffered by call parity; before reusing a parity a
// producer waits for every consumer's acknowledgement of the call two back,
// so no data is overwritten before it is read and no barrier is needed.
#pragma once
#include "sat_common.h"
#include "sat_device.cuh"

namespace sat {

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

// Column totals from the partials (as sat_colsum_final_kernel), pushed into
// slot (epoch & 1, rank) of every higher rank's mailbox.
template <typename T>
__global__ void __launch_bounds__(256)
sat_colsum_push_kernel(const T* __restrict__ part, int64_t cols, int splits, int width, XchgParams x) {
    const int par = int(x.epoch & 1);
    const int P = x.L.P;
    if (threadIdx.x == 0 && x.epoch > 2) {
        // the consumers of this parity's previous use (epoch - 2) are done
        for (int c = x.rank + 1; c < P; ++c)
            wait_at_least(reinterpret_cast<const uint64_t*>(x.mine + x.L.acks_off()) + c, x.epoch - 2,
                          0x10000000u | uint32_t(c));
    }
    __syncthreads();
    for (int64_t c = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; c < cols;
         c += int64_t(gridDim.x) * blockDim.x) {
        T s = T(0);
        for (int sp = 0; sp < splits; ++sp) s += part[int64_t(sp) * width + c];
        for (int q = x.rank + 1; q < P; ++q)
            reinterpret_cast<T*>(x.peers[q] + x.L.slot_off(par, x.rank))[c] = s;
    }
    // last block: publish the flag in every consumer's mailbox
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned int n = atomicAdd(x.done, 1u);
        if (n == gridDim.x - 1) {
            __threadfence_system();
            for (int q = x.rank + 1; q < P; ++q)
                st_release_sys_u64(reinterpret_cast<uint64_t*>(x.peers[q] + x.L.flags_off()) + par * P + x.rank,
                                   x.epoch);
            *x.done = 0;
        }
    }
}

// Rank p's carry: wait for ranks < p, carry[c] = sum_{q<p} slot[par][q][c]
// (rank order), acknowledge, then the SAT row above the strip =
// row prefix of the carry (as sat_row_prefix_kernel).  One CTA of 1024.
template <typename T>
__global__ void __launch_bounds__(1024)
sat_seed_from_peers_kernel(T* __restrict__ sat_row, int64_t cols, XchgParams x) {
    __shared__ T wsum[32];
    __shared__ T s_run;
    const int par = int(x.epoch & 1);
    const int P = x.L.P;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x < x.rank)
        wait_at_least(reinterpret_cast<const uint64_t*>(x.mine + x.L.flags_off()) + par * P + threadIdx.x,
                      x.epoch, 0x18000000u | threadIdx.x);
    if (threadIdx.x == 0) s_run = T(0);
    __syncthreads();
    for (int64_t base = 0; base < cols; base += 8 * 1024) {
        const int64_t c = base + int64_t(threadIdx.x) * 8;
        T e[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            T s = T(0);
            if (c + i < cols)
                for (int q = 0; q < x.rank; ++q)
                    s += reinterpret_cast<const volatile T*>(x.mine + x.L.slot_off(par, q))[c + i];
            e[i] = s;
        }
#pragma unroll
        for (int i = 1; i < 8; ++i) e[i] += e[i - 1];
        const T inc = warp_inclusive_scan(e[7], lane);
        if (lane == 31) wsum[warp] = inc;
        __syncthreads();
        if (warp == 0) wsum[lane] = warp_inclusive_scan(wsum[lane], lane);
        __syncthreads();
        T exc = __shfl_up_sync(0xffffffffu, inc, 1);
        if (lane == 0) exc = T(0);
        const T off = s_run + (warp > 0 ? wsum[warp - 1] : T(0)) + exc;
#pragma unroll
        for (int i = 0; i < 8; ++i)
            if (c + i < cols) sat_row[c + i] = e[i] + off;
        __syncthreads();
        if (threadIdx.x == 0) s_run += wsum[31];
        __syncthreads();
    }
    // every slot read: acknowledge to each producer
    if (threadIdx.x < x.rank)
        st_release_sys_u64(reinterpret_cast<uint64_t*>(x.peers[threadIdx.x] + x.L.acks_off()) + x.rank, x.epoch);
}

}  // namespace sat
