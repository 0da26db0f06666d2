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
    int cluster;               // CTAs per cluster (1, or 8: one ticket = 8 bands)
    int big;                   // 1: one CTA per SM with a 2x ring of 1-KB row segments (TH 64)
    uint64_t* desc;            // [total_bands][nc*TW] look-back descriptor words
    unsigned long long* ticket;
    unsigned long long base;   // ticket base of this launch (also the tag base)
    const unsigned long long* base_dev;   // nullable: read the base from device memory (graph capture)
    const void* seed;          // [cols] SAT row above band 0 of image 0, nullable
    int seed_kind;             // SEED_NONE or SEED_SATROW
    int top_src;               // TopSrc
    int region;                // Region
    int tA;                    // (1+r)R1W threshold
    const void* Lx;            // [nc+1][total_bands*TH] row carry at chunk start, nullable
    const void* TopX;          // [total_bands][nc*TW] external SAT row above, nullable
    void* Lb;                  // [total_bands*TH] band-final row carry out, nullable
    int jitter;                // debug: random publish delay (ns scale), 0 = off
    int dbg;                   // debug: bit 0 = skip look-back and publication (top = 0; WRONG results, timing only)
    unsigned long long* trace; // debug: [total_bands*nc][4] event times (ns), nullable
    unsigned int* diag;        // debug: host-mapped progress marks (sat_debug_diag_enable), nullable
    // Band segments (plain 1R1W, many waves): a ticket is (segment s, band b),
    // segment-major, so the last wave holds short units.  Segment s covers
    // chunks [s*segc, (s+1)*segc); the row carry L of band b crosses from
    // segment s-1 to s through Lseg (tagged 64-bit words).
    int nseg;                  // 1 = whole bands
    int segc;                  // chunks per segment
    uint64_t* Lseg;            // [total_bands][TH] row carry at the end of the band's last segment
    int pf;                    // L2 prefetch distance in chunks (TMA path; 0 = off)
    int unit_sync;             // A/B: 1 = the next unit starts only after every warp finished this one
};

}  // namespace sat
