// sat_common.h -- host/device shared definitions of libsat (not shared with
// the oracle).  Kernel parameter block and the (1+r)R1W region geometry.
#pragma once
#include <cstdint>

#ifdef __CUDACC__
#define SAT_HD __host__ __device__ __forceinline__
#else
#define SAT_HD inline
#endif

namespace sat {

constexpr int TW = 128;          // chunk width: 32 lanes x 4 elements (16 B)

enum Mode { MODE_COL = 1, MODE_ROW = 2, MODE_SAT = 3 };
enum TopSrc { TOP_LOOKBACK = 0, TOP_EXTERNAL = 1 };
enum Region { REG_ALL = 0, REG_A = 1, REG_C = 2, REG_B = 3 };
enum SeedKind { SEED_NONE = 0, SEED_COLSUM = 1, SEED_SATROW = 2 };  // the kernel sees NONE/SATROW

// Tile (I = band, J = chunk) regions of (1+r)R1W, bounded by tile
// anti-diagonals (reading R10; Fig. 12):
//   A: I + J < tA,   B: I + J > last - tA,   C: the rest;  last = nb + nc - 2.
// Returns the half-open chunk range [j0, j1) of band I inside `region`.
SAT_HD void region_range(int region, int tA, int nb, int nc, int I, int& j0, int& j1) {
    const int last = nb + nc - 2;
    int lo = 0, hi = nc;
    if (region == REG_A) { lo = 0; hi = tA - I; }
    else if (region == REG_C) { lo = tA - I; hi = last - tA - I + 1; }
    else if (region == REG_B) { lo = last - tA - I + 1; hi = nc; }
    if (lo < 0) lo = 0;
    if (lo > nc) lo = nc;
    if (hi > nc) hi = nc;
    if (hi < lo) hi = lo;
    j0 = lo; j1 = hi;
}

// Column-sum seed of a strip (row-strip sharding, north star (3)): the
// carry row c[j] = sum_{q < n} vec_q[j] (q ascending) is the column sum of
// everything above the strip.  Band 0 of image 0 adds it to its first input
// row before the row scan (SAT of [c; a] restricted to a's rows == the rows
// of the taller matrix's SAT), so neither a carry-prefix kernel nor an
// exclusive-scan kernel runs.  Sources: one vector (sat_compute_seeded), the
// all-gathered totals of ranks < p (NCCL path), or the slots of a peer
// mailbox after its flags (fused exchange, sat_xchg.cuh).
struct ColSeed {
    const void* base;               // vector q at base + q * stride (bytes); nullptr = none
    int64_t stride;
    int n;                          // vectors to sum (0 = no seed)
    const uint64_t* flags;          // nullable: wait flags[q] >= epoch (sys acquire) before reading vector q
    unsigned long long epoch;
    uint64_t* const* acks;          // nullable: [n] after the last read, st.release.sys(acks[q], epoch)
    unsigned int* done;             // band-0 units finished reading (self-resetting counter) when acks != nullptr
};

struct BandParams {
    const void* in;            // [batch][rows][cols] (generic path, not used by TMA path)
    void* out;                 // [batch][rows][cols]
    int64_t rows, cols;        // per image
    int batch;
    int nb;                    // bands per image = ceil(rows / TH)
    int nc;                    // chunks per band = ceil(cols / TW)
    int total_bands;           // batch * nb
    long long total_units;     // bands (band units) or bands*nc (tile units)
    int tile_units;            // K > 0: one ticket = K consecutive tiles of a band (external carries); 0 = whole bands
    uint64_t* desc;            // [total_bands][nc*TW] look-back descriptor words
    unsigned long long* ticket;
    unsigned long long base;   // ticket base of this launch (also the tag base)
    const unsigned long long* base_dev;   // nullable: read the base from device memory (graph capture)
    const void* seed;          // [cols] SAT row above band 0 of image 0, nullable
    int seed_kind;             // SEED_NONE or SEED_SATROW
    ColSeed cseed;             // column-sum seed added to row 0 of image 0 (n = 0: none)
    int top_src;               // TopSrc
    int region;                // Region
    int tA;                    // (1+r)R1W threshold
    const void* Lx;            // [nc+1][total_bands*TH] row carry at chunk start, nullable
    const void* TopX;          // [total_bands][nc*TW] external SAT row above, nullable
    void* Lb;                  // [total_bands*TH] band-final row carry out, nullable
    int jitter;                // stress tests: random publish delay (ns scale), 0 = off
    // Band segments (plain 1R1W, many waves): a ticket is (segment s, band b),
    // segment-major, so the last wave holds short units.  Segment s covers
    // chunks [s*segc, (s+1)*segc); the row carry L of band b crosses from
    // segment s-1 to s through Lseg (tagged 64-bit words).
    int nseg;                  // 1 = whole bands
    int segc;                  // chunks per segment
    uint64_t* Lseg;            // [total_bands][TH] row carry at the end of the band's last segment
    // Ticket order of the segment units (nullable = segment-major): order[t]
    // = (segment, band) of ticket t, sorted by band + K * segment: both
    // predecessors of a unit -- the same segment of the band above and the
    // previous segment of the same band -- hold earlier tickets.
    const int2* order;
    // Hierarchical look-back: hg > 0 groups the bands
    // of an image by hg; the last band of a group also publishes the group's
    // aggregate / inclusive words in gdesc[img * ngroups + group][column], and
    // a walk visits its own group band by band, then one word per group above.
    int hg;                    // 0 = flat look-back
    int ngroups;               // groups per image = ceil(nb / hg)
    uint64_t* gdesc;           // [batch * ngroups][nc*TW] group descriptor words
    unsigned long long* trace; // debug builds (SAT_DEBUG): [total_bands*nc][8] event times (ns), nullable
    unsigned int* diag;        // debug builds: host-mapped progress marks, nullable
};

}  // namespace sat
