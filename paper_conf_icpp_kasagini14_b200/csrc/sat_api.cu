// sat_api.cu -- the libsat C ABI (include/sat.h): validation, per-stream
// workspace, tensor maps, variant drivers and kernel dispatch.
//
// Variant drivers follow PAPER.md: 2R2W Sec. IV, 2R1W Sec. V
// (P:L1059-L1137), 1R1W Sec. VI, (1+r)R1W Sec. VII
// (P:L2289-L2355).  The sharded and host (end-to-end) entry points are the
// north star's (1)/(3) additions (BASELINE.json).
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <type_traits>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <atomic>
#include <vector>
#include <string>
#include <utility>

#include "../../include/sat.h"
#include "sat_aux.cuh"
#include "sat_band.cuh"
#include "sat_paper.cuh"
#include "sat_box.cuh"
#include <dlfcn.h>
#include <nccl.h>

#include "sat_boxf.cuh"
#include "sat_boxw.cuh"
#include "sat_xchg.cuh"

using namespace sat;

namespace {

thread_local std::string t_err;
thread_local int t_launches = 0;
thread_local int t_th = 0;
thread_local int t_grid = 0;
thread_local int t_hg = 0;
thread_local double t_r = 0.0;
thread_local unsigned long long* t_trace = nullptr;
thread_local bool t_capture = false;   // the current call's stream is being captured
static unsigned int* g_diag_dev = nullptr;   // sat_debug_diag_enable (device view)

int fail(int code, const std::string& msg) {
    t_err = msg;
    return code;
}

#define CUDA_TRY(expr)                                                                  \
    do {                                                                                \
        cudaError_t _e = (expr);                                                        \
        if (_e != cudaSuccess)                                                          \
            return fail(SAT_ERR_CUDA, std::string(#expr) + ": " + cudaGetErrorString(_e)); \
    } while (0)

#define SAT_TRY(expr)                  \
    do {                               \
        int _s = (expr);               \
        if (_s != SAT_OK) return _s;   \
    } while (0)

// ------------------------------------------------------------------ devices
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

constexpr int kMaxDev = 64;

struct DevInfo {
    int sms = 0;
    int l2 = 0;
    int smem_optin = 0;
    int smem_sm = 0;
    bool ok = false;
};

std::mutex g_mu;
std::map<int, DevInfo> g_dev;
EncodeTiledFn g_encode = nullptr;

int get_dev(int& dev, DevInfo& info) {
    CUDA_TRY(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(g_mu);
    DevInfo& d = g_dev[dev];
    if (!d.ok) {
        CUDA_TRY(cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev));
        CUDA_TRY(cudaDeviceGetAttribute(&d.smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
        CUDA_TRY(cudaDeviceGetAttribute(&d.smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev));
        CUDA_TRY(cudaDeviceGetAttribute(&d.l2, cudaDevAttrL2CacheSize, dev));
        d.ok = true;
    }
    if (!g_encode) {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        CUDA_TRY(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
        if (q != cudaDriverEntryPointSuccess || !fn)
            return fail(SAT_ERR_CUDA, "cuTensorMapEncodeTiled entry point not found");
        g_encode = reinterpret_cast<EncodeTiledFn>(fn);
    }
    info = d;
    return SAT_OK;
}

// ------------------------------------------------------------------ workspace
struct Buf {
    void* p = nullptr;
    size_t bytes = 0;
};

// look-back tags are 30 bits (band_tag); sat_debug_set_tag_space (tests only)
// shrinks the space so the reset paths run
std::atomic<unsigned long long> g_tag_space{1ull << 30};
std::atomic<int> g_box_rb{0};        // sat_debug_set_box_rows (0 = automatic)
unsigned long long tag_space() { return g_tag_space.load(std::memory_order_relaxed); }

struct Workspace {
    Buf desc;                 // look-back descriptors (zeroed when (re)allocated)
    Buf lseg;                 // band-segment row carries (zeroed when (re)allocated)
    Buf ticket;               // [0] ticket counter, [1] device base (unsigned long long)
    unsigned long long next_base = 0;
    bool dev_epoch = false;   // once captured: every launch takes its base from the device (Sec. 4)
    Buf bt, rs, lx, lsum, topx, lb;   // 2R1W family
    Buf tr;                   // 4R4W transposed copy
    Buf box;                  // box filter: the SAT it reads
    Buf part;                 // column totals partials
    Buf cnt;                  // column totals: per-chunk-column and global arrival counters (self-resetting)
    Buf bticket;              // fused box filter: unit ticket (zeroed per call on the stream)
    Buf order;                // segment-unit ticket order (int2 per unit), for order_key
    unsigned long long order_key = 0;
    Buf shard;                // sharded default workspace
    Buf din, dout;            // host e2e device copies
    std::vector<void*> retired;   // buffers a captured graph may still reference (freed by sat_release_workspace)
    cudaStream_t cstream_in = nullptr, cstream_out = nullptr;
};

thread_local Workspace* t_ws = nullptr;   // the current call's workspace (for ensure())
thread_local cudaStream_t t_st = nullptr; // the current call's stream

// Grow a workspace buffer.  New memory is zeroed (when asked) with
// cudaMemsetAsync on the call's stream, so the kernels queued after it on that
// stream see zeros.  Once any call on the stream was captured into a CUDA
// graph, an outgrown buffer is retired, not freed: a graph replay may still
// reference it (freed by sat_release_workspace).
int ensure(Buf& b, size_t bytes, bool zero) {
    if (b.bytes >= bytes && b.p) return SAT_OK;
    // a captured call cannot allocate (cudaMalloc / cudaMemset would break
    // the capture): the workspace must have been sized by an eager call
    if (t_capture)
        return fail(SAT_ERR_UNSUPPORTED, "stream capture needs a warm workspace: run the same call once "
                                         "on this stream before capturing it");
    if (b.p) {
        if (t_ws && t_ws->dev_epoch) t_ws->retired.push_back(b.p);
        else cudaFree(b.p);
        b.p = nullptr;
        b.bytes = 0;
    }
    size_t want = std::max<size_t>(bytes, 256);
    if (cudaMalloc(&b.p, want) != cudaSuccess) {
        cudaGetLastError();
        return fail(SAT_ERR_NOMEM, "cudaMalloc of " + std::to_string(want) + " bytes failed");
    }
    b.bytes = want;
    if (zero) CUDA_TRY(cudaMemsetAsync(b.p, 0, want, t_st));
    return SAT_OK;
}

std::map<std::pair<int, void*>, Workspace*> g_ws;

int get_ws(int dev, cudaStream_t st, Workspace*& ws) {
    std::lock_guard<std::mutex> lk(g_mu);
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    CUDA_TRY(cudaStreamIsCapturing(st, &cap));
    t_capture = (cap != cudaStreamCaptureStatusNone);
    Workspace*& w = g_ws[{dev, reinterpret_cast<void*>(st)}];
    if (!w) w = new Workspace();
    ws = w;
    t_ws = w;
    t_st = st;
    return SAT_OK;
}

void free_buf(Buf& b) {
    if (b.p) cudaFree(b.p);
    b.p = nullptr;
    b.bytes = 0;
}

// ------------------------------------------------------------------ helpers

bool dtype_ok(int dtype) { return dtype == SAT_INT32 || dtype == SAT_FLOAT32 || dtype == SAT_FLOAT64; }
size_t esize(int dtype) { return dtype == SAT_FLOAT64 ? 8 : dtype == SAT_UINT8 ? 1 : 4; }
// widening input -> sum pairs of sat_compute_widening (besides same-type pairs)
bool widen_ok(int in_dtype, int dtype) {
    return in_dtype == dtype || (in_dtype == SAT_UINT8 && dtype == SAT_INT32) ||
           (in_dtype == SAT_FLOAT32 && dtype == SAT_FLOAT64);
}
// Element type of a sat_dtype: uint32 (int32, wrapping), float, double.
#define SAT_DISPATCH(dtype, T, ...)                                             \
    ((dtype) == SAT_INT32     ? [&] { using T = uint32_t; return __VA_ARGS__; }() \
     : (dtype) == SAT_FLOAT32 ? [&] { using T = float; return __VA_ARGS__; }()    \
                              : [&] { using T = double; return __VA_ARGS__; }())

int validate(const void* in, const void* out, int64_t batch, int64_t rows, int64_t cols,
             int dtype, bool need_in = true, int in_dtype = -1) {
    if (in_dtype < 0) in_dtype = dtype;
    if (!dtype_ok(dtype))
        return fail(SAT_ERR_INVALID, "dtype must be SAT_INT32, SAT_FLOAT32 or SAT_FLOAT64");
    if (!widen_ok(in_dtype, dtype))
        return fail(SAT_ERR_INVALID, "input/sum dtype pair must be equal, UINT8->INT32 or FLOAT32->FLOAT64");
    if (rows < 0 || cols < 0 || batch < 0) return fail(SAT_ERR_INVALID, "negative size");
    if (rows > INT32_MAX || cols > INT32_MAX || batch > INT32_MAX)
        return fail(SAT_ERR_INVALID, "rows, cols and batch must each be < 2^31");
    if (rows == 0 || cols == 0 || batch == 0) return SAT_OK;
    const double n = double(rows) * double(cols) * double(batch);
    if (n * double(esize(dtype)) > 9.0e18) return fail(SAT_ERR_INVALID, "matrix byte size overflows");
    if ((need_in && !in) || !out) return fail(SAT_ERR_INVALID, "null pointer with nonzero size");
    if (need_in && in_dtype != dtype && in == out)
        return fail(SAT_ERR_INVALID, "a widening SAT cannot run in place");
    if (need_in && in != out) {
        const uintptr_t a0 = reinterpret_cast<uintptr_t>(in), b0 = reinterpret_cast<uintptr_t>(out);
        const uintptr_t n_el = uintptr_t(rows) * uintptr_t(cols) * uintptr_t(batch);
        const uintptr_t la = n_el * esize(in_dtype), lb = n_el * esize(dtype);
        if (a0 < b0 + lb && b0 < a0 + la)
            return fail(SAT_ERR_INVALID, "in and out partially overlap");
    }
    const uintptr_t am = esize(dtype) - 1, ai = esize(in_dtype) - 1;
    if ((reinterpret_cast<uintptr_t>(out) & am) || (need_in && (reinterpret_cast<uintptr_t>(in) & ai)))
        return fail(SAT_ERR_INVALID, "pointers must be aligned to the element size");
    return SAT_OK;
}

bool tma_ok(const void* in, const void* out, int64_t cols, int in_dtype = -1) {
    // 16-B aligned rows for the TMA box and the 4-per-lane vector stores
    const int64_t q = in_dtype == SAT_UINT8 ? 16 : 4;
    return (cols % q == 0) && ((reinterpret_cast<uintptr_t>(in) & 15) == 0) &&
           ((reinterpret_cast<uintptr_t>(out) & 15) == 0);
}

int make_tmap(CUtensorMap* m, const void* base, int dtype, int64_t batch, int64_t rows,
              int64_t cols, int th, int tw = TW) {
    cuuint64_t dims[3] = {cuuint64_t(cols), cuuint64_t(rows), cuuint64_t(batch)};
    const cuuint64_t eb = esize(dtype);
    cuuint64_t strides[2] = {cuuint64_t(cols) * eb, cuuint64_t(cols) * cuuint64_t(rows) * eb};
    cuuint32_t box[3] = {cuuint32_t(tw), cuuint32_t(th), 1};
    cuuint32_t es[3] = {1, 1, 1};
    CUresult r = g_encode(m, dtype == SAT_INT32     ? CU_TENSOR_MAP_DATA_TYPE_UINT32
                             : dtype == SAT_FLOAT32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                             : dtype == SAT_UINT8   ? CU_TENSOR_MAP_DATA_TYPE_UINT8
                                                    : CU_TENSOR_MAP_DATA_TYPE_FLOAT64,
                          3, const_cast<void*>(base), dims, strides, box, es,
                          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS)
        return fail(SAT_ERR_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string(int(r)) + ")");
    return SAT_OK;
}

// ------------------------------------------------------------------ band kernel dispatch
struct BandCfg {
    int R, W, S, DT, SUB, NCW, NS, MINB;
};
// TH = R*W rows per band, W compute warps of R rows.  Shared memory per CTA:
// S ring slots of SUB adjacent TH x 128 chunks (SUB*512 B per row per load:
// wider row segments keep HBM pages busy) + DT*W*512 B
// (bottom rows / add vectors) + barriers; TMEM per CTA: DT chunks x 4R words
// per compute thread.  Two CTAs per SM.
constexpr BandCfg kCfg16{4, 4, 3, 8, 4, 4, 1, 2};
constexpr BandCfg kCfg32{8, 4, 3, 8, 2, 4, 1, 2};
// TH 32 when the bands fit in one wave of ONE CTA per SM (4096^2: 128
// bands): 8 compute warps of 4 rows, a 4 x 32 KB ring, 16 chunks parked (all
// 512 TMEM columns) and 12 control groups walking one band per round trip.
// The look-back of a lockstep wave is ~11 hops deep, so its latency (not the
// bandwidth) sets the chunk rate: 4096^2 int32 45 vs 53-55 us, 3072^2 35 vs
// 41, 2048^2 25 vs 29 (profiles/r02_small.txt; 8 groups 47, window 2 / 4:
// 49 / 53, 8 parked chunks 51)
constexpr BandCfg kCfg32S{4, 8, 4, 16, 2, 12, 1, 1};
constexpr int kLbw32S = 1;

// column / row passes (2R2W, 4R4W) at TH 64: two CTAs per SM
constexpr BandCfg kCfg64{8, 8, 3, 4, 1, 4, 1, 2};
// 1R1W at TH 64 ("wide"): one CTA per SM, 192 KB ring of 64 x 256 slots
// (1-KB row segments per TMA load pair), 8 chunks parked in TMEM (all 512
// columns).  Between one half and two thirds of a wave of 128-row bands it
// beats both TH 32 and TH 128: 6144^2 int32 0.084 vs 0.094 ms (TH 32),
// 8192^2 0.127 vs 0.143, 10240^2 0.179 vs 0.198 (TH 128); the two-CTA TH-64
// configuration was 20-30 % slower (profiles/r02_ab_th.txt).  8 control
// groups walking one band per round trip: 6144^2-12288^2 5-7 % faster than 4
// groups with a window of 4 (profiles/r02_small.txt)
constexpr BandCfg kCfg64W{8, 8, 3, 8, 2, 8, 1, 1};
constexpr int kLbw64W = 1;
// TH = 128: 16 compute warps, one CTA per SM (ring 3 x 64 KB, TMEM 4 chunks =
// all 512 columns); half the descriptor bytes and look-back hops per element
constexpr BandCfg kCfg128{8, 16, 3, 4, 1, 3, 1, 1};
constexpr int kLbw128 = 2;   // look-back window (bands per round trip) at TH = 128:
                             // 2 measured ~1 % faster than 4 at 16384^2/18432^2, 8 slower
// float64 (8-byte elements: 1 KB chunk rows, two TMEM words per element)
constexpr BandCfg kCfgD16{2, 8, 4, 4, 1, 3, 1, 2};   //  96 KB smem, 128 TMEM cols: 2 CTAs/SM
constexpr BandCfg kCfgD32{4, 8, 4, 8, 1, 4, 1, 1};   // 192 KB smem, 512 TMEM cols
// TH 64: ONE control group of 2 warps that split the columns (NS = 2: 2
// columns per lane, 4 descriptor words per band, look-back window 4):
// 16384^2 0.917 vs 1.04 ms with 3 groups of 1 warp, 32768^2 3.49 vs 3.87
constexpr BandCfg kCfgD64{8, 8, 3, 4, 1, 2, 2, 1};   // 224 KB smem, 512 TMEM cols
// TH 128 (plain 1R1W): 64-column chunks, so a lane moves two doubles (16 B)
// and a chunk is 64 KB -- the int32 TH-128 geometry: 16 compute warps, one CTA
// per SM, 3 x 64 KB ring, 4 chunks parked (512 TMEM columns), 3 control
// warps of 2 columns per lane (4 descriptor words per band, window 2)
constexpr BandCfg kCfgD128{8, 16, 3, 4, 1, 3, 1, 1};
constexpr int kTwD128 = 64;
// float64 1R1W at TH 64 / 128: one band per look-back round trip (18432^2
// 1.076 vs 1.101 ms at TH 64, 1.002 vs 1.006 at TH 128; more control groups
// were 2-8 % slower, profiles/r02_float64_th128.txt)
constexpr int kLbwD = 1;

// uint8 input widened to uint32 sums: the ring holds bytes (TH x 128 B per
// chunk), so it is 6 slots deep
constexpr BandCfg kCfgU64{8, 8, 6, 4, 1, 4, 1, 2};
constexpr BandCfg kCfgU128{8, 16, 6, 4, 1, 3, 1, 1};

// CTAs per SM of a 1R1W-family configuration (for wave counts before launch)
int ctas_per_sm(int dtype, int th) {
    if (dtype == SAT_FLOAT64) return th == 16 ? 2 : 1;
    return th >= 64 ? 1 : 2;
}

// One-time per (instantiation, device) launch set-up, shared by all threads.
struct KernelSetup {
    std::once_flag once[kMaxDev];
    cudaFuncAttributes fa[kMaxDev];
    cudaError_t err[kMaxDev] = {};
};

template <typename T, int R, int W, int S, int DT, int SUB, int NCW, int NS, int MODE, bool TMA, int MINB,
          int LBW = 0, typename TI = T, int TWK = TW>
int launch_band_t(const BandParams& p, const CUtensorMap& ti, const DevInfo& di, cudaStream_t st, int& grid_out) {
    auto kern = sat_band_kernel<T, R, W, S, DT, SUB, NCW, NS, MODE, TMA, MINB, LBW, TI, TWK>;
    const size_t smem = BandSmem<T, R, W, S, DT, SUB, TI, TWK>::total;
    const int threads = (W + NCW + 1) * 32;
    // per instantiation and device: attributes set once, resources queried
    // once (a per-call cudaFuncGetAttributes was a visible part of the ~15 us
    // host cost of a small call); std::call_once orders the set-up before any
    // thread's launch
    static KernelSetup setup;
    int dev = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    if (dev < 0 || dev >= kMaxDev) return fail(SAT_ERR_CUDA, "device ordinal out of range");
    std::call_once(setup.once[dev], [&] {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout,
                                     int(cudaSharedmemCarveoutMaxShared));
        if (e == cudaSuccess) e = cudaFuncGetAttributes(&setup.fa[dev], kern);
        setup.err[dev] = e;
    });
    if (setup.err[dev] != cudaSuccess)
        return fail(SAT_ERR_CUDA, std::string("band kernel set-up: ") + cudaGetErrorString(setup.err[dev]));
    // Resident CTAs per SM, from the kernel's own resources.  (The runtime's
    // occupancy query reports 1 for kernels that allocate tensor memory; two
    // CTAs of ours fit: TC::alloc <= 256 columns of the SM's 512.)
    const cudaFuncAttributes& fa = setup.fa[dev];
    const int warps = threads / 32;
    const int regs_warp = ((fa.numRegs * 32 + 255) / 256) * 256;
    const int occ = std::min({2048 / threads, 65536 / (regs_warp * warps),
                              di.smem_sm / int(smem + fa.sharedSizeBytes + 1024),
                              MODE == MODE_ROW ? 32 : 512 / TmemCols<R, W, DT, int(sizeof(T) / 4), TWK / 32>::alloc,
                              32});
    if (occ < 1) return fail(SAT_ERR_CUDA, "band kernel does not fit on an SM");
    long long grid = std::min<long long>(p.total_units, (long long)occ * di.sms);
    if (grid < 1) grid = 1;
    grid_out = int(grid);
    t_grid = int(grid);
    // programmatic dependent launch: the CTA prologue (barriers, TMEM alloc)
    // overlaps the previous kernel's tail; the kernel waits
    // (griddepcontrol.wait) before its first global access.  Back-to-back
    // calls: 1024^2 16.7 -> 14.4 us, 4096^2 f32 47.9 -> 45.5 us
    // (profiles/r01_pdl_ab.txt)
    cudaLaunchConfig_t cfg;
    std::memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = dim3(unsigned(grid));
    cfg.blockDim = dim3(unsigned(threads));
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, ti, p));
    CUDA_TRY(cudaGetLastError());
    ++t_launches;
    return SAT_OK;
}

#define SAT_CFG(c) c.R, c.W, c.S, c.DT, c.SUB, c.NCW, c.NS
// Band heights instantiated per (dtype, mode, path); `band_th` maps a
// requested height onto them.  1R1W family (MODE_SAT) on the TMA path: int32 /
// float32 16, 32, 64 ("wide", one CTA per SM), 128, float64 16, 32,
// 64; the column and row passes of 2R2W / 4R4W: 32 and 64; the generic
// (non-TMA) path: 32 (and 128 for 4-byte 1R1W).
int band_th(int mode, int dtype, bool tma, int th) {
    if (!tma) {
        if (mode == MODE_SAT && dtype != SAT_FLOAT64 && th >= 128) return 128;
        return 32;
    }
    if (mode != MODE_SAT && th >= 128) return 128;          // float64: 64-column chunks
    if (mode != MODE_SAT) return th >= 64 ? 64 : 32;
    if (dtype == SAT_FLOAT64) return th >= 128 ? 128 : th >= 64 ? 64 : th >= 32 ? 32 : 16;
    return th >= 128 ? 128 : th >= 64 ? 64 : th >= 32 ? 32 : 16;
}

template <typename T, int MODE, bool TMA>
int launch_band_th(int th, const BandParams& p, const CUtensorMap& ti, const DevInfo& di, cudaStream_t st,
                   int& grid) {
    if constexpr (!TMA) {
        if constexpr (MODE == MODE_SAT && sizeof(T) == 4)
            if (th == 128) return launch_band_t<T, SAT_CFG(kCfg128), MODE, TMA, kCfg128.MINB>(p, ti, di, st, grid);
        if constexpr (sizeof(T) == 8)
            return launch_band_t<T, SAT_CFG(kCfgD32), MODE, TMA, kCfgD32.MINB>(p, ti, di, st, grid);
        else
            return launch_band_t<T, SAT_CFG(kCfg32), MODE, TMA, kCfg32.MINB>(p, ti, di, st, grid);
    } else if constexpr (MODE != MODE_SAT) {
        if constexpr (sizeof(T) == 8) {
            if (th == 128)
                return launch_band_t<T, SAT_CFG(kCfgD128), MODE, TMA, kCfgD128.MINB, kLbwD, T, kTwD128>(p, ti, di, st, grid);
            if (th == 64) return launch_band_t<T, SAT_CFG(kCfgD64), MODE, TMA, kCfgD64.MINB>(p, ti, di, st, grid);
            return launch_band_t<T, SAT_CFG(kCfgD32), MODE, TMA, kCfgD32.MINB>(p, ti, di, st, grid);
        } else {
            if (th == 128) return launch_band_t<T, SAT_CFG(kCfg128), MODE, TMA, kCfg128.MINB, kLbw128>(p, ti, di, st, grid);
            if (th == 64) return launch_band_t<T, SAT_CFG(kCfg64), MODE, TMA, kCfg64.MINB>(p, ti, di, st, grid);
            return launch_band_t<T, SAT_CFG(kCfg32), MODE, TMA, kCfg32.MINB>(p, ti, di, st, grid);
        }
    } else if constexpr (sizeof(T) == 8) {
        switch (th) {
            case 128: return launch_band_t<T, SAT_CFG(kCfgD128), MODE, TMA, kCfgD128.MINB, kLbwD, T, kTwD128>(
                          p, ti, di, st, grid);
            case 16: return launch_band_t<T, SAT_CFG(kCfgD16), MODE, TMA, kCfgD16.MINB>(p, ti, di, st, grid);
            case 32: return launch_band_t<T, SAT_CFG(kCfgD32), MODE, TMA, kCfgD32.MINB>(p, ti, di, st, grid);
            case 64: return launch_band_t<T, SAT_CFG(kCfgD64), MODE, TMA, kCfgD64.MINB, kLbwD>(p, ti, di, st, grid);
        }
        return fail(SAT_ERR_INVALID, "float64: no band configuration for this tile_rows");
    } else {
        switch (th) {
            case 32:
                if (p.top_src == TOP_LOOKBACK && p.total_units <= di.sms)
                    return launch_band_t<T, SAT_CFG(kCfg32S), MODE, TMA, kCfg32S.MINB, kLbw32S>(p, ti, di, st, grid);
                return launch_band_t<T, SAT_CFG(kCfg32), MODE, TMA, kCfg32.MINB>(p, ti, di, st, grid);
            case 16: return launch_band_t<T, SAT_CFG(kCfg16), MODE, TMA, kCfg16.MINB>(p, ti, di, st, grid);
            case 64: return launch_band_t<T, SAT_CFG(kCfg64W), MODE, TMA, kCfg64W.MINB, kLbw64W>(p, ti, di, st, grid);
            case 128: return launch_band_t<T, SAT_CFG(kCfg128), MODE, TMA, kCfg128.MINB, kLbw128>(p, ti, di, st, grid);
        }
        return fail(SAT_ERR_INVALID, "no band configuration for this tile_rows");
    }
}

// Widening 1R1W: uint8 -> uint32 and float32 -> float64.
template <typename T, typename TI, bool TMA>
int launch_band_widen(int th, const BandParams& p, const CUtensorMap& ti, const DevInfo& di, cudaStream_t st,
                      int& grid) {
    if constexpr (sizeof(TI) == 1) {
        if constexpr (TMA) {
            if (th == 128) return launch_band_t<T, SAT_CFG(kCfgU128), MODE_SAT, TMA, 1, kLbw128, TI>(p, ti, di, st, grid);
        }
        return launch_band_t<T, SAT_CFG(kCfgU64), MODE_SAT, TMA, 2, 0, TI>(p, ti, di, st, grid);
    } else {
        if constexpr (TMA) {
            if (th == 16) return launch_band_t<T, SAT_CFG(kCfgD16), MODE_SAT, TMA, kCfgD16.MINB, 0, TI>(p, ti, di, st, grid);
            if (th == 64) return launch_band_t<T, SAT_CFG(kCfgD64), MODE_SAT, TMA, kCfgD64.MINB, 0, TI>(p, ti, di, st, grid);
            if (th == 128)
                return launch_band_t<T, SAT_CFG(kCfgD128), MODE_SAT, TMA, kCfgD128.MINB, kLbwD, TI, kTwD128>(
                    p, ti, di, st, grid);
        }
        return launch_band_t<T, SAT_CFG(kCfgD32), MODE_SAT, TMA, kCfgD32.MINB, 0, TI>(p, ti, di, st, grid);
    }
}

template <typename T, int MODE>
int launch_band_m(bool tma, int th, const BandParams& p, const CUtensorMap& ti, const DevInfo& di,
                  cudaStream_t st, int& grid) {
    return tma ? launch_band_th<T, MODE, true>(th, p, ti, di, st, grid)
               : launch_band_th<T, MODE, false>(th, p, ti, di, st, grid);
}

template <typename T>
int launch_band_d(int mode, bool tma, int th, const BandParams& p, const CUtensorMap& ti, const DevInfo& di,
                  cudaStream_t st, int& grid) {
    switch (mode) {
        case MODE_SAT: return launch_band_m<T, MODE_SAT>(tma, th, p, ti, di, st, grid);
        case MODE_COL: return launch_band_m<T, MODE_COL>(tma, th, p, ti, di, st, grid);
        case MODE_ROW: return launch_band_m<T, MODE_ROW>(tma, th, p, ti, di, st, grid);
    }
    return fail(SAT_ERR_INVALID, "bad mode");
}

// Automatic band height: the tallest band that still gives roughly one band
// per resident CTA slot (the look-back chain is per band; more, shorter bands
// raise parallelism, taller bands cut descriptor traffic).
int auto_th(int64_t rows, int64_t batch, const DevInfo& di, int variant, int dtype) {
    if (dtype == SAT_FLOAT64) {
        // plain 1R1W: TH 128 with 64-column chunks (the int32 TH-128 geometry)
        // once its bands fill two thirds of the SMs
        if (variant == SAT_1R1W && batch * ((rows + 127) / 128) * 100 >= 65LL * di.sms) return 128;
        // one CTA per SM for TH 32/64 (1-KB rows): the tallest band with a
        // wave; below that TH 32 from 1024 rows (a shorter look-back chain
        // beats filling the SMs: 1024^2 0.031 vs 0.034 ms, 2048^2 0.054 vs 0.063)
        for (int th : {64, 32}) {
            const long long bands = batch * ((rows + th - 1) / th);
            if (bands * 5 >= 4LL * di.sms) return th;
        }
        return rows * batch >= 512 ? 32 : 16;
    }
    // 1R1W (one CTA per SM for TH 64 and 128; r02 sweep, profiles/r02_ab_th.txt):
    // TH = 128 once its bands fill about two thirds of the SMs (the look-back
    // chain is one hop per band; 16K^2+: 5.3-5.4 TB/s); the wide TH 64 below
    // that while its bands fill 60 % of the SMs (6144^2-10240^2: 9-11 %
    // faster than TH 32 or 128); then TH 32 from 512 rows (one wave of
    // kCfg32S: 768^2-4096^2 10-40 % faster than TH 16), else TH 16.
    if (variant == SAT_1R1W || variant == SAT_1PLUSR_R1W) {   // (1+r): its band C is 1R1W
        const long long b128 = batch * ((rows + 127) / 128), b64 = batch * ((rows + 63) / 64);
        if (b128 * 100 >= 65LL * di.sms) return 128;
        if (b64 * 10 >= 6LL * di.sms) return 64;
        return rows * batch >= 512 ? 32 : 16;
    }
    // 2R1W (its Step-3 band kernel is the 1R1W one with external carries,
    // no look-back chain, so tall bands pay off earlier): TH 128 from 64
    // bands of 128 rows, else TH 64 from 32 bands of 64 rows (int32 sweep:
    // 16384^2 0.596 -> 0.569 ms, 12288^2 428 -> 331 us, 8192^2 208 -> 165,
    // 6144^2 204 -> 120, 4096^2 93 -> 77, 2048^2 46 -> 44; 1024^2 keeps 16)
    if (variant == SAT_2R1W) {
        if (batch * ((rows + 127) / 128) >= 64) return 128;
        if (batch * ((rows + 63) / 64) >= 32) return 64;
    }
    const long long slots = 2LL * di.sms;          // 2 CTAs/SM for TH = 32/64
    for (int th : {64, 32}) {
        const long long bands = batch * ((rows + th - 1) / th);
        if (bands * 5 >= slots * 4) return th;
    }
    return 16;
}

// The 2R2W / 4R4W column and row passes take TH 128 from ~0.6 bands of 128
// rows per SM (int32 sweep: 12288^2 2R2W 530 -> 456 us, 4R4W 1031 -> 919;
// at 8192^2, 64 bands, 2R2W is 8 % slower at TH 128)
bool pass_th128(int64_t rows, int64_t batch, const DevInfo& di) {
    return batch * ((rows + 127) / 128) * 10 >= 6LL * di.sms;
}

struct Job {
    const void* in;
    void* out;
    int64_t batch, rows, cols;
    int dtype;
    int in_dtype;     // == dtype, or a narrower input widened on load (1R1W only)
    int th;
    bool tma;
    int jitter;
    int segments;     // sat_options.segments: 0 = automatic band segments
    int hg;           // sat_options.lookback_group: 0 = automatic, -1 = flat, n >= 2 groups of n bands
    const DevInfo* di;
    Workspace* ws;
    cudaStream_t st;
};

// Device-side ticket base (graph capture).  The ticket counter (64-bit, never
// reset on this path) ends every band launch at base + units + takers, the
// next launch's base; block 0 copies it to tk[1] for the band kernel (whose
// CTAs advance tk[0] while they start).  Tags are 30 bits of base + unit, so a
// stale descriptor could match again one tag space later: every block clears
// the descriptors whenever this launch's value range [t, t + worst) crosses a
// multiple of half the tag space.  Between clears every live descriptor was
// written less than half a space + one launch earlier, so none can alias.
// One launch, decided on the device from t alone (no state, no inter-block
// race: nothing in this kernel writes tk[0]).
__global__ void sat_epoch_kernel(unsigned long long* tk, unsigned long long worst, unsigned long long half,
                                 uint4* a, size_t na, uint4* b, size_t nb) {
    const unsigned long long t = __ldcg(tk);
    if (blockIdx.x == 0 && threadIdx.x == 0) tk[1] = t;
    if (t / half == (t + worst) / half) return;
    const uint4 z = make_uint4(0, 0, 0, 0);
    for (size_t i = size_t(blockIdx.x) * blockDim.x + threadIdx.x; i < na + nb; i += size_t(gridDim.x) * blockDim.x) {
        if (i < na) a[i] = z; else b[i - na] = z;
    }
}

// The band height a launch actually uses (the instantiated configurations).
int eff_th(const Job& j, int mode) {
    if (j.in_dtype == SAT_UINT8) return (j.tma && j.th >= 128) ? 128 : 64;
    // float32 -> float64: TH 128 with 64-column chunks like plain float64
    if (j.in_dtype != j.dtype) return j.tma ? (j.th >= 128 ? 128 : j.th >= 64 ? 64 : j.th >= 32 ? 32 : 16) : 32;
    return band_th(mode, j.dtype, j.tma, j.th);
}

// One band-kernel launch with ticket/tag bookkeeping.
int run_band(const Job& j0, int mode, const void* in, void* out, BandParams p) {
    Job j = j0;
    j.th = eff_th(j0, mode);
    t_th = j.th;
    // The ticket base and the descriptor tags come from a host-side counter
    // advanced per launch.  A captured launch replayed from a CUDA graph would
    // reuse a host value, so under capture (and on this workspace from then
    // on, since replays advance the device ticket behind the host's back) the
    // base is taken on the device: sat_epoch_kernel reads the ticket counter
    // (it ends every launch at the next launch's base) right before the band
    // kernel, on the same stream.
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    CUDA_TRY(cudaStreamIsCapturing(j.st, &cap));
    if (cap != cudaStreamCaptureStatusNone) j.ws->dev_epoch = true;
    p.in = in;
    p.out = out;
    p.rows = j.rows;
    p.cols = j.cols;
    p.batch = int(j.batch);
    // chunk width: 64 columns for float64 at TH 128 (kCfgD128), else 128
    const int tw = (j.tma && j.dtype == SAT_FLOAT64 && j.th == 128) ? kTwD128 : TW;
    p.nb = int((j.rows + j.th - 1) / j.th);
    p.nc = int((j.cols + tw - 1) / tw);
    p.total_bands = int(j.batch * p.nb);
    p.total_units = p.tile_units ? (long long)p.total_bands * ((p.nc + p.tile_units - 1) / p.tile_units)
                                 : p.total_bands;
    // Band segments: short units for the last wave when
    // bands are many waves deep
    p.nseg = 1;
    p.segc = p.nc;
    if (mode == MODE_SAT && p.top_src == TOP_LOOKBACK && p.region == REG_ALL && !p.tile_units &&
        p.Lx == nullptr && p.Lb == nullptr) {
        // more bands than resident CTAs: up to 16 segments of >= 16 chunks, so
        // the partial last wave of whole bands becomes many short units
        // (65536^2 TH 128: 5.97 ms with 16 segments vs 6.34 ms whole bands;
        // 20480^2: 0.614 ms with 8-10 vs 0.887 ms; 12288^2 float64: 0.608 vs
        // 0.785 ms); at most one wave: whole bands (a segment would wait for
        // the band's previous segment)
        const int slots = j.di->sms * ctas_per_sm(j.dtype, j.th);
        int want = p.total_bands > slots ? std::min(16, p.nc / 16) : 1;
        // short bands (batches of images): segments of >= 3 chunks
        // (32 x 1080x1920 float32: 0.1045 vs 0.1070 ms, 64 images 0.1935 vs
        // 0.2048 with 5 segments of 3 chunks, profiles/r02_small.txt)
        // (not the widening loads: 32 x 1080x1920 uint8 -> int32 0.078 vs
        // 0.084 ms, float32 -> float64 0.187 vs 0.24-0.25 without / with)
        if (p.total_bands > slots && want < 2 && j.in_dtype == j.dtype && j.dtype != SAT_FLOAT64)
            want = std::min(5, p.nc / 3);
        if (j.segments > 0) want = j.segments;
        if (want > 1 && p.nc > 1) {
            p.segc = (p.nc + want - 1) / want;
            p.nseg = (p.nc + p.segc - 1) / p.segc;
            p.total_units = (long long)p.total_bands * p.nseg;
        }
    }
    // Skewed ticket order of the segment units: sorted
    // by band + K * segment with K = 12 x resident CTAs / segments, so the
    // band above a unit (same segment) runs ~nseg tickets earlier instead of
    // alongside it, and the same band's previous segment ~K * nseg tickets
    // earlier (long finished).  65536^2: 5.81-5.87 vs 5.87-5.97 ms,
    // 49152^2: 3.37-3.41 vs 3.45-3.47 (three rounds each, profiles/r02_skew.txt);
    // where K exceeds the bands it is the plain segment-major order.
    constexpr int kSkewMult = 12;
    p.order = nullptr;
    if (p.nseg > 1) {
        const int K = std::max(1, kSkewMult * j.di->sms * ctas_per_sm(j.dtype, j.th) / p.nseg);
        const unsigned long long key = (unsigned long long)p.total_bands | ((unsigned long long)p.nseg << 32) |
                                       ((unsigned long long)K << 44);
        Workspace& w = *j.ws;
        if (w.order_key != key || !w.order.p) {
            std::vector<int2> ord;
            ord.reserve(size_t(p.total_bands) * p.nseg);
            const long long kmax = (long long)p.total_bands - 1 + (long long)K * (p.nseg - 1);
            for (long long d = 0; d <= kmax; ++d)
                for (int sg = 0; sg < p.nseg; ++sg) {
                    const long long b = d - (long long)K * sg;
                    if (b >= 0 && b < p.total_bands) ord.push_back(make_int2(sg, int(b)));
                }
            SAT_TRY(ensure(w.order, ord.size() * sizeof(int2), false));
            CUDA_TRY(cudaMemcpy(w.order.p, ord.data(), ord.size() * sizeof(int2), cudaMemcpyHostToDevice));
            w.order_key = key;
        }
        p.order = static_cast<const int2*>(w.order.p);
    }
    p.jitter = j.jitter;
    if (kDebug) {
        p.diag = g_diag_dev;
        if (mode == MODE_SAT && p.top_src == TOP_LOOKBACK && t_trace) {
            p.trace = t_trace;
            t_trace = nullptr;
        }
    }
    Workspace& ws = *j.ws;
    // hierarchical look-back: group words live after
    // the band descriptors in the same buffer (cleared with them)
    p.hg = 0;
    p.ngroups = 0;
    if (p.top_src == TOP_LOOKBACK && mode != MODE_ROW && p.region == REG_ALL) {
        // automatic: groups of 4 bands for one-wave 1R1W launches of bands
        // <= 64 rows (the one-wave TH-32 and wide TH-64 configurations, whose
        // control groups walk one band per round trip): 4096^2 45.1 -> 42.0 us,
        // 3072^2 34.8 -> 32.8, 5120^2 75.8 -> 72.7, 6144^2 79.9 -> 77.8,
        // 4096^2 float64 112 -> 107; flat at TH 128 (16384^2 0.408 vs
        // 0.410-0.419 ms for groups of 4-16) and for many waves (65536^2,
        // 8192^2, 12288^2: 0.5-2 % slower); profiles/r02_hier.txt
        int hg = j.hg;
        if (hg == 0) {
            const int slots = j.di->sms * ctas_per_sm(j.dtype, j.th);
            hg = (mode == MODE_SAT && j.th <= 64 && p.total_units <= slots) ? 4 : -1;
            // the 2R2W / 4R4W column pass: groups of 4 up to one band per SM
            // (4096^2 f32 2R2W 82.9 -> 77.9 us, 4R4W 160.7 -> 146.4; 2048^2
            // -5 / -12 %; 192 bands at 6144^2: 10 % slower, flat)
            if (mode == MODE_COL && j.th <= 32 && p.total_units <= j.di->sms) hg = 4;
        }
        if (hg >= 2 && hg < p.nb) {
            p.hg = hg;
            p.ngroups = (p.nb + hg - 1) / hg;
        }
    }
    size_t desc_words = 0;
    if (p.top_src == TOP_LOOKBACK && mode != MODE_ROW) {
        desc_words = size_t(p.total_bands) * size_t(p.nc) * tw * (esize(j.dtype) / 4);
        const size_t gwords = size_t(j.batch) * size_t(p.ngroups) * size_t(p.nc) * tw * (esize(j.dtype) / 4);
        SAT_TRY(ensure(ws.desc, (desc_words + gwords) * sizeof(uint64_t), true));
    }
    SAT_TRY(ensure(ws.ticket, 4 * sizeof(unsigned long long), true));
    if (p.nseg > 1)
        SAT_TRY(ensure(ws.lseg, size_t(p.total_bands) * j.th * sizeof(uint64_t) * (esize(j.dtype) / 4), true));
    const unsigned long long units = (unsigned long long)p.total_units;
    const unsigned long long worst = units + 4096ull * 64ull;   // units + max grid
    p.base_dev = nullptr;
    if (ws.dev_epoch) {
        unsigned long long* tk = static_cast<unsigned long long*>(ws.ticket.p);
        const size_t dw = ws.desc.p ? ws.desc.bytes / 16 : 0, lw = ws.lseg.p ? ws.lseg.bytes / 16 : 0;
        sat_epoch_kernel<<<2 * j.di->sms, 256, 0, j.st>>>(tk, worst, tag_space() / 2, static_cast<uint4*>(ws.desc.p),
                                                          dw, static_cast<uint4*>(ws.lseg.p), lw);
        CUDA_TRY(cudaGetLastError());
        p.base_dev = tk + 1;
        ++t_launches;
    } else if (ws.next_base + worst >= tag_space()) {
        // tag space exhausted: clear descriptors and the counter (rare)
        if (ws.desc.p) CUDA_TRY(cudaMemsetAsync(ws.desc.p, 0, ws.desc.bytes, j.st));
        if (ws.lseg.p) CUDA_TRY(cudaMemsetAsync(ws.lseg.p, 0, ws.lseg.bytes, j.st));
        CUDA_TRY(cudaMemsetAsync(ws.ticket.p, 0, sizeof(unsigned long long), j.st));
        ws.next_base = 0;
    }
    p.desc = static_cast<uint64_t*>(ws.desc.p);
    p.gdesc = p.hg > 0 ? p.desc + desc_words : nullptr;
    t_hg = p.hg;
    p.Lseg = static_cast<uint64_t*>(ws.lseg.p);
    p.ticket = static_cast<unsigned long long*>(ws.ticket.p);
    p.base = ws.next_base;
    CUtensorMap ti;
    std::memset(&ti, 0, sizeof(ti));
    if (j.tma) {
        SAT_TRY(make_tmap(&ti, in, j.in_dtype, j.batch, j.rows, j.cols, j.th, tw));
    }
    int grid = 0;
    int s;
    if (j.in_dtype == SAT_UINT8)
        s = j.tma ? launch_band_widen<uint32_t, uint8_t, true>(j.th, p, ti, *j.di, j.st, grid)
                  : launch_band_widen<uint32_t, uint8_t, false>(j.th, p, ti, *j.di, j.st, grid);
    else if (j.in_dtype != j.dtype)
        s = j.tma ? launch_band_widen<double, float, true>(j.th, p, ti, *j.di, j.st, grid)
                  : launch_band_widen<double, float, false>(j.th, p, ti, *j.di, j.st, grid);
    else
        s = SAT_DISPATCH(j.dtype, T, launch_band_d<T>(mode, j.tma, j.th, p, ti, *j.di, j.st, grid));
    if (s != SAT_OK) return s;
    // every persistent ticket taker (a CTA) makes exactly one failing fetch,
    // so the counter ends at base + units + takers
    ws.next_base += units + (unsigned long long)grid;
    return SAT_OK;
}

BandParams base_params() {
    BandParams p;
    std::memset(&p, 0, sizeof(p));
    p.top_src = TOP_LOOKBACK;
    p.region = REG_ALL;
    p.seed_kind = SEED_NONE;
    return p;
}

// ------------------------------------------------------------------ 2R1W family
struct Carry2r1w {
    int nb, nc, total_bands;
};

int prep_2r1w(const Job& j, Carry2r1w& c) {
    c.nb = int((j.rows + j.th - 1) / j.th);
    c.nc = int((j.cols + TW - 1) / TW);
    c.total_bands = int(j.batch * c.nb);
    Workspace& ws = *j.ws;
    const size_t eb = esize(j.dtype);
    const size_t wide = size_t(c.total_bands) * c.nc * TW * eb;
    const size_t rowsp = size_t(c.total_bands) * j.th * eb;
    SAT_TRY(ensure(ws.bt, wide, false));
    SAT_TRY(ensure(ws.topx, wide, false));
    SAT_TRY(ensure(ws.rs, rowsp * c.nc, false));
    SAT_TRY(ensure(ws.lx, rowsp * (c.nc + 1), false));
    SAT_TRY(ensure(ws.lsum, size_t(c.total_bands) * (c.nc + 1) * eb, false));
    SAT_TRY(ensure(ws.lb, rowsp, false));
    return SAT_OK;
}

template <typename T>
int run_2r1w_region_t(const Job& j, const Carry2r1w& c, int region, int tA, const void* in,
                      void* out, const void* Lb) {
    Workspace& ws = *j.ws;
    TileParams tp;
    tp.in = in; tp.rows = j.rows; tp.cols = j.cols; tp.batch = int(j.batch);
    tp.nb = c.nb; tp.nc = c.nc; tp.total_bands = c.total_bands; tp.th = j.th;
    tp.region = region; tp.tA = tA; tp.Bt = ws.bt.p; tp.RS = ws.rs.p;
    // Step 1: tile reductions
    sat_reduce_kernel<T><<<dim3(c.nc, c.total_bands), 256, 0, j.st>>>(tp);
    CUDA_TRY(cudaGetLastError());
    ++t_launches;
    // Step 2: row carries, then SAT row above every tile
    CarryParams cp;
    cp.rows = j.rows; cp.cols = j.cols; cp.batch = int(j.batch); cp.nb = c.nb; cp.nc = c.nc;
    cp.total_bands = c.total_bands; cp.th = j.th; cp.region = region; cp.tA = tA;
    cp.RS = ws.rs.p; cp.Bt = ws.bt.p; cp.Lb = Lb; cp.Lx = ws.lx.p; cp.Lsum = ws.lsum.p;
    cp.TopX = ws.topx.p; cp.out = out;
    const int rthreads = ((j.th + 31) / 32) * 32;
    sat_carry_rows_kernel<T><<<c.total_bands, rthreads, 0, j.st>>>(cp);
    CUDA_TRY(cudaGetLastError());
    ++t_launches;
    const int W = c.nc * TW;
    sat_carry_top_kernel<T><<<dim3((W + 31) / 32, unsigned(j.batch)), 256, 0, j.st>>>(cp);
    CUDA_TRY(cudaGetLastError());
    ++t_launches;
    // Step 3: re-read, add carries, tile SAT, write (tile tickets, external carries)
    BandParams p = base_params();
    p.top_src = TOP_EXTERNAL;
    // units of K chunks of a band (external carries make every range
    // independent): whole bands for the full matrix up to 64 chunks, 8-chunk
    // ranges above (16384^2 2R1W 0.657 -> 0.625 ms); 16-chunk ranges for the
    // (1+r)R1W triangles, whose top bands are long (16384^2 0.952 -> 0.705 ms)
    p.tile_units = region == REG_ALL ? (c.nc >= 64 ? 8 : 0) : 16;
    p.region = region;
    p.tA = tA;
    p.Lx = ws.lx.p;
    p.TopX = ws.topx.p;
    return run_band(j, MODE_SAT, in, out, p);
}

int run_2r1w_region(const Job& j, const Carry2r1w& c, int region, int tA, const void* in,
                    void* out, const void* Lb) {
    return SAT_DISPATCH(j.dtype, T, run_2r1w_region_t<T>(j, c, region, tA, in, out, Lb));
}

// Choose the triangle threshold tA whose tile fraction (|A|+|B|)/(nb*nc) is
// closest to r (reading R10), keeping A and B disjoint.
int choose_tA(int nb, int nc, double r, double& r_eff) {
    const int last = nb + nc - 2;
    const int tmax = (last + 1) / 2;
    int best = 0;
    double bestd = 1e30;
    r_eff = 0;
    for (int tA = 0; tA <= tmax; ++tA) {
        long long cnt = 0;
        for (int I = 0; I < nb; ++I) {
            int a0, a1, b0, b1;
            region_range(REG_A, tA, nb, nc, I, a0, a1);
            region_range(REG_B, tA, nb, nc, I, b0, b1);
            cnt += (a1 - a0) + (b1 - b0);
        }
        const double re = double(cnt) / (double(nb) * nc);
        if (std::fabs(re - r) < bestd) { bestd = std::fabs(re - r); best = tA; r_eff = re; }
    }
    return best;
}

// ------------------------------------------------------------------ 4R4W / 4R1W (Table II columns)
template <typename T>
int transpose_t(const void* in, void* out, int64_t batch, int64_t rows, int64_t cols, cudaStream_t st) {
    const uintptr_t al = 2 * sizeof(T) - 1;
    if (rows % 2 == 0 && cols % 2 == 0 && !(reinterpret_cast<uintptr_t>(in) & al) &&
        !(reinterpret_cast<uintptr_t>(out) & al)) {
        const int64_t ntr = (rows + 63) / 64;
        const dim3 grid(unsigned((cols + 63) / 64), unsigned(std::min<int64_t>(ntr, 65535)), unsigned(batch));
        sat_transpose64_kernel<T><<<grid, 256, 0, st>>>(static_cast<const T*>(in), static_cast<T*>(out),
                                                        rows, cols);
        CUDA_TRY(cudaGetLastError());
        ++t_launches;
        return SAT_OK;
    }
    const int64_t ntr = (rows + 31) / 32;
    const dim3 grid(unsigned((cols + 31) / 32), unsigned(std::min<int64_t>(ntr, 65535)), unsigned(batch));
    sat_transpose_kernel<T><<<grid, dim3(32, 8), 0, st>>>(static_cast<const T*>(in), static_cast<T*>(out),
                                                          rows, cols);
    CUDA_TRY(cudaGetLastError());
    ++t_launches;
    return SAT_OK;
}

// 4R4W (Sec. IV, Lemma 3): column prefix, transpose, column prefix, transpose.
int run_4r4w(const Job& j, const sat_options& o) {
    Workspace& ws = *j.ws;
    SAT_TRY(ensure(ws.tr, size_t(j.batch) * j.rows * j.cols * esize(j.dtype), false));
    // column passes at TH 128 where plain 1R1W takes it (as in 2R2W)
    auto col_th = [&](int64_t rows, int th) {
        if (!o.tile_rows && pass_th128(rows, j.batch, *j.di)) return 128;
        return th;
    };
    Job j1 = j;
    j1.th = col_th(j.rows, j.th);
    SAT_TRY(run_band(j1, MODE_COL, j.in, j.out, base_params()));
    auto tp = [&](const void* a, void* b, int64_t r, int64_t c) {
        return SAT_DISPATCH(j.dtype, T, transpose_t<T>(a, b, j.batch, r, c, j.st));
    };
    SAT_TRY(tp(j.out, ws.tr.p, j.rows, j.cols));
    Job jt = j;
    jt.rows = j.cols;
    jt.cols = j.rows;
    jt.in = ws.tr.p;
    jt.out = ws.tr.p;
    jt.th = col_th(jt.rows, o.tile_rows ? o.tile_rows : auto_th(jt.rows, jt.batch, *j.di, SAT_4R4W, j.dtype));
    jt.tma = !o.force_generic && tma_ok(ws.tr.p, ws.tr.p, jt.cols);
    SAT_TRY(run_band(jt, MODE_COL, ws.tr.p, ws.tr.p, base_params()));
    return tp(ws.tr.p, j.out, jt.rows, jt.cols);
}

// 4R1W (Sec. VI, Formula (1)): rows + cols - 1 anti-diagonal stage launches.
template <typename T>
int run_4r1w_t(const Job& j) {
    const int64_t stages = j.rows + j.cols - 1;
    for (int64_t t = 0; t < stages; ++t) {
        const int64_t i0 = std::max<int64_t>(0, t - (j.cols - 1));
        const int64_t i1 = std::min<int64_t>(j.rows - 1, t);
        const int64_t cnt = i1 - i0 + 1;
        const unsigned blocks = unsigned(std::min<int64_t>((cnt + 255) / 256, 8LL * j.di->sms));
        sat_4r1w_stage_kernel<T><<<dim3(blocks, unsigned(j.batch)), 256, 0, j.st>>>(
            static_cast<const T*>(j.in), static_cast<T*>(j.out), j.rows, j.cols, t, i0, cnt);
        CUDA_TRY(cudaGetLastError());
        ++t_launches;
    }
    return SAT_OK;
}

// ------------------------------------------------------------------ core driver
// satrow: SAT row just above the matrix (SEED_SATROW), cs: column-sum seed of
// image 0 (sat_common.h ColSeed); both 1R1W only.
int compute_core(const void* in, void* out, int64_t batch, int64_t rows, int64_t cols,
                 int dtype, int variant, const sat_options* opt, const void* satrow,
                 const ColSeed* cs, cudaStream_t st, int in_dtype = -1) {
    t_launches = 0;
    if (in_dtype < 0) in_dtype = dtype;
    SAT_TRY(validate(in, out, batch, rows, cols, dtype, true, in_dtype));
    if (variant < SAT_2R2W || variant > SAT_4R1W) return fail(SAT_ERR_INVALID, "bad variant");
    const bool seeded = satrow != nullptr || (cs && cs->n > 0);
    if (in_dtype != dtype && (variant != SAT_1R1W || seeded))
        return fail(SAT_ERR_UNSUPPORTED, "widening input: unseeded 1R1W only");
    // column-sum seeds: 1R1W (band 0's first row) and 2R2W (the column pass's
    // first row: the column prefix carries it down, the row pass across);
    // the SAT-row seed: 1R1W only
    if ((satrow != nullptr && variant != SAT_1R1W) || (cs && cs->n > 0 && variant != SAT_1R1W && variant != SAT_2R2W))
        return fail(SAT_ERR_UNSUPPORTED, "seeded (sharded) SAT: variant must be 1R1W or 2R2W");
    sat_options o;
    sat_options_init(&o);
    if (opt) o = *opt;
    if (o.tile_rows != 0 && o.tile_rows != 16 && o.tile_rows != 32 && o.tile_rows != 64 && o.tile_rows != 128)
        return fail(SAT_ERR_INVALID, "tile_rows must be 0, 16, 32, 64 or 128");
    if (!(o.r >= 0.0 && o.r <= 1.0)) return fail(SAT_ERR_INVALID, "r must be in [0, 1]");
    if (o.segments < 0) return fail(SAT_ERR_INVALID, "segments must be >= 0");
    if (o.lookback_group < -1 || o.lookback_group == 1)
        return fail(SAT_ERR_INVALID, "lookback_group must be -1, 0 or >= 2");
    if (rows == 0 || cols == 0 || batch == 0) return SAT_OK;
    int dev;
    DevInfo di;
    SAT_TRY(get_dev(dev, di));
    Workspace* ws;
    SAT_TRY(get_ws(dev, st, ws));
    Job j;
    j.in = in; j.out = out; j.batch = batch; j.rows = rows; j.cols = cols; j.dtype = dtype;
    j.in_dtype = in_dtype;
    j.th = o.tile_rows ? o.tile_rows : auto_th(rows, batch, di, variant, dtype);
    j.tma = !o.force_generic && tma_ok(in, out, cols, in_dtype);
    j.jitter = o.jitter;
    j.segments = o.segments;
    j.hg = o.lookback_group;
    j.di = &di;
    j.ws = ws;
    j.st = st;
    // the 1R1W family's band height (2R1W Steps 1-2 size their carries by it);
    // float64 TH 128 (64-column chunks) serves plain 1R1W only
    if (dtype == SAT_FLOAT64 && variant != SAT_1R1W && j.th > 64) j.th = 64;
    j.th = eff_th(j, MODE_SAT);
    t_th = j.th;
    switch (variant) {
        case SAT_1R1W: {
            BandParams p = base_params();
            if (cs && cs->n > 0) p.cseed = *cs;
            p.seed = satrow;
            p.seed_kind = satrow ? SEED_SATROW : SEED_NONE;
            return run_band(j, MODE_SAT, in, out, p);
        }
        case SAT_2R2W: {
            // column-wise prefix-sums (look-back down the columns), then
            // row-wise prefix-sums (rows independent)
            Job j1 = j;
            j1.th = o.tile_rows ? o.tile_rows : auto_th(rows, batch, di, variant, dtype);
            // both passes take the TH-128 configuration where plain 1R1W
            // does: 16384^2 int32 0.851 -> 0.797 ms (column pass) -> 0.759
            // (and the row pass), 18432^2 1.049 -> 0.987
            if (!o.tile_rows && pass_th128(rows, batch, di)) j1.th = 128;
            BandParams pc = base_params();
            if (cs && cs->n > 0) pc.cseed = *cs;
            SAT_TRY(run_band(j1, MODE_COL, in, out, pc));
            Job j2 = j1;
            j2.tma = !o.force_generic && tma_ok(out, out, cols);
            return run_band(j2, MODE_ROW, out, out, base_params());
        }
        case SAT_2R1W: {
            Carry2r1w c;
            SAT_TRY(prep_2r1w(j, c));
            return run_2r1w_region(j, c, REG_ALL, 0, in, out, nullptr);
        }
        case SAT_1PLUSR_R1W: {
            Carry2r1w c;
            SAT_TRY(prep_2r1w(j, c));
            double r_eff = 0;
            const int tA = choose_tA(c.nb, c.nc, o.r, r_eff);
            t_r = r_eff;
            if (tA == 0) {
                // r_eff = 0: both triangles are empty -- plain 1R1W (no empty
                // Step 1/2 launches, band segments allowed, plain 1R1W's band
                // height: float64 may take TH 128)
                Job j1 = j;
                if (!o.tile_rows && dtype == SAT_FLOAT64) {
                    j1.th = auto_th(rows, batch, di, SAT_1R1W, dtype);
                    j1.th = eff_th(j1, MODE_SAT);
                }
                BandParams p = base_params();
                return run_band(j1, MODE_SAT, in, out, p);
            }
            // (A) 2R1W on the top-left triangle; its Step 2 also leaves the
            // row carry into (C) in Lx.
            SAT_TRY(run_2r1w_region(j, c, REG_A, tA, in, out, nullptr));
            // (C) 1R1W over the middle band, seeded from (A)'s final SAT rows
            // and row carries; leaves the row carry into (B) in Lb.
            BandParams p = base_params();
            p.region = REG_C;
            p.tA = tA;
            p.Lx = ws->lx.p;
            p.Lb = ws->lb.p;
            SAT_TRY(run_band(j, MODE_SAT, in, out, p));
            // (B) 2R1W on the bottom-right triangle, seeded from (C).
            return run_2r1w_region(j, c, REG_B, tA, in, out, ws->lb.p);
        }
        case SAT_4R4W:
            return run_4r4w(j, o);
        case SAT_4R1W:
            if (batch > 65535) return fail(SAT_ERR_UNSUPPORTED, "4R1W: batch must be <= 65535");
            return SAT_DISPATCH(dtype, T, run_4r1w_t<T>(j));
    }
    return fail(SAT_ERR_INVALID, "bad variant");
}

// Column totals in one launch (sat_xchg.cuh sat_colsum_kernel); push = the
// fused exchange's epilogue.
template <typename T>
int column_totals_t(const void* in, void* totals, int64_t rows, int64_t cols, const DevInfo& di,
                    Workspace& ws, cudaStream_t st, const XchgParams* x) {
    const int nc = int((cols + TW - 1) / TW);
    long long splits = std::max<long long>(1, (4LL * di.sms + nc - 1) / nc);
    splits = std::min<long long>(splits, std::max<int64_t>(1, (rows + 63) / 64));
    const int64_t seg = std::max<int64_t>(1, (rows + splits - 1) / splits);
    if (rows > 0) splits = (rows + seg - 1) / seg;
    SAT_TRY(ensure(ws.part, size_t(splits) * nc * TW * sizeof(T), false));
    SAT_TRY(ensure(ws.cnt, size_t(nc + 1) * sizeof(unsigned int), true));
    TotalsParams tp;
    std::memset(&tp, 0, sizeof(tp));
    tp.in = in; tp.rows = rows; tp.cols = cols; tp.seg_rows = seg; tp.splits = int(splits);
    tp.part = ws.part.p;
    tp.cnt = static_cast<unsigned int*>(ws.cnt.p);
    tp.totals = totals;
    if (x) { tp.push = 1; tp.x = *x; }
    sat_colsum_kernel<T><<<dim3(nc, unsigned(splits)), 256, 0, st>>>(tp);
    CUDA_TRY(cudaGetLastError());
    ++t_launches;
    return SAT_OK;
}

int column_totals_core(const void* in, void* totals, int64_t rows, int64_t cols, int dtype,
                       cudaStream_t st) {
    int dev;
    DevInfo di;
    SAT_TRY(get_dev(dev, di));
    Workspace* ws;
    SAT_TRY(get_ws(dev, st, ws));
    return SAT_DISPATCH(dtype, T, column_totals_t<T>(in, totals, rows, cols, di, *ws, st, nullptr));
}

int exscan_core(const void* gathered, void* carry, int64_t nranks, int64_t cols, int rank,
                int dtype, cudaStream_t st) {
    const unsigned blocks = unsigned((cols + 255) / 256);
    SAT_DISPATCH(dtype, T, (sat_rank_exscan_kernel<T><<<blocks, 256, 0, st>>>(
                                static_cast<const T*>(gathered), static_cast<T*>(carry), cols, rank),
                            0));
    CUDA_TRY(cudaGetLastError());
    ++t_launches;
    return SAT_OK;
}

size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

// ------------------------------------------------------------------ fused peer exchange
struct PeerExchange {
    int rank, nranks, dtype;
    int64_t cols;
    XchgParams x;             // epoch advanced per call
    unsigned int* done;       // device counter: band-0 units that finished reading the slots
    uint64_t** acks;          // device [nranks]: &peers[q].ack[rank] for q < rank
};

template <typename T>
int sharded_fused_t(const void* in, void* out, int64_t strip_rows, PeerExchange& ex, cudaStream_t st) {
    int dev;
    DevInfo di;
    SAT_TRY(get_dev(dev, di));
    Workspace* ws;
    SAT_TRY(get_ws(dev, st, ws));
    if (t_capture)
        return fail(SAT_ERR_UNSUPPORTED, "sat_compute_sharded_fused cannot be captured: the exchange epoch "
                                         "is assigned per call on the host (a replay would reuse it)");
    const int64_t cols = ex.cols;
    ex.x.epoch += 1;
    int launches = 0;
    if (ex.rank < ex.nranks - 1) {
        // 1. strip column totals; the epilogue pushes them into the higher
        //    ranks' mailboxes and raises their flags (ONE launch)
        t_launches = 0;
        SAT_TRY(column_totals_t<T>(in, nullptr, strip_rows, cols, di, *ws, st, &ex.x));
        launches += t_launches;
    }
    if (ex.rank > 0 && strip_rows == 0) {
        sat_xchg_drain_kernel<<<1, 32, 0, st>>>(ex.x);
        CUDA_TRY(cudaGetLastError());
        ++launches;
    }
    // 2. seeded local 1R1W: band 0 waits for the flags of ranks < p, adds the
    //    sum of their slots (rank order) to its first row, acknowledges
    if (strip_rows > 0) {
        ColSeed cs;
        std::memset(&cs, 0, sizeof(cs));
        if (ex.rank > 0) {
            const int par = int(ex.x.epoch & 1);
            cs.base = ex.x.mine + ex.x.L.slot_off(par, 0);
            cs.stride = int64_t(ex.x.L.slot_off(par, 1) - ex.x.L.slot_off(par, 0));
            cs.n = ex.rank;
            cs.flags = reinterpret_cast<const uint64_t*>(ex.x.mine + ex.x.L.flags_off()) + par * ex.nranks;
            cs.epoch = ex.x.epoch;
            cs.acks = ex.acks;
            cs.done = ex.done;
        }
        SAT_TRY(compute_core(in, out, 1, strip_rows, cols, ex.dtype, SAT_1R1W, nullptr, nullptr, &cs, st));
        launches += t_launches;
    }
    t_launches = launches;
    return SAT_OK;
}

// Fused box filter (sat_boxf.cuh): one launch, the SAT stays on chip.
template <typename TI, typename TS, typename TO, int TH, int MAXH, int NS, int NWARP = 16, int CPS = 1>
int box_fused_t(const void* in, int in_dtype, void* out, int64_t batch, int64_t rows, int64_t cols, int rr, int rc,
                int normalize, const DevInfo& di, Workspace& ws, cudaStream_t st) {
    auto kern = sat_boxf_kernel<TI, TS, TO, TH, MAXH, NS, NWARP>;
    const size_t smem = BoxSmem<MAXH, NS, TI, TS, NWARP>::total;
    static KernelSetup setup;
    int dev = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    if (dev < 0 || dev >= kMaxDev) return fail(SAT_ERR_CUDA, "device ordinal out of range");
    std::call_once(setup.once[dev], [&] {
        setup.err[dev] = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    });
    if (setup.err[dev] != cudaSuccess)
        return fail(SAT_ERR_CUDA, std::string("box kernel set-up: ") + cudaGetErrorString(setup.err[dev]));
    CUtensorMap tm;
    std::memset(&tm, 0, sizeof(tm));
    SAT_TRY(make_tmap(&tm, in, in_dtype, batch, rows, cols, MAXH));
    SAT_TRY(ensure(ws.bticket, sizeof(unsigned long long), false));
    CUDA_TRY(cudaMemsetAsync(ws.bticket.p, 0, sizeof(unsigned long long), st));
    BoxParams bp;
    bp.in = in; bp.out = out; bp.rows = int(rows); bp.cols = int(cols); bp.batch = int(batch);
    bp.rr = rr; bp.rc = rc; bp.normalize = normalize;
    bp.nb = int((rows + TH - 1) / TH);
    bp.nc = int((cols + TW - 1) / TW);
    bp.ticket = static_cast<unsigned long long*>(ws.bticket.p);
    bp.base = 0;
    const long long units = (long long)batch * bp.nb;
    const int grid = int(std::min<long long>(units, (long long)CPS * di.sms));
    cudaLaunchConfig_t cfg;
    std::memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = dim3(unsigned(grid));
    cfg.blockDim = dim3(NWARP * 32);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, tm, bp));
    CUDA_TRY(cudaGetLastError());
    t_launches = 1;
    t_grid = grid;
    return SAT_OK;
}

// Column-walk box filter (sat_boxw.cuh): one launch, one warp per unit of
// 128 columns x rb output rows, the SAT evaluated on the fly.
template <typename TI, typename TS, typename TO>
int box_walk_t(const void* in, void* out, int64_t batch, int64_t rows, int64_t cols, int rr, int rc, int normalize,
               cudaStream_t st) {
    constexpr int NWARP = 4;
    // rows in flight per warp (cp.async ring); 4 also for uint8 rows (8 B per
    // lane): the smaller ring buys occupancy -- uint8 r = 8 0.148 -> 0.125 ms,
    // r = 4 0.127 / 0.129 (tools/bench_box.py)
    constexpr int PF = 4;
    // float input (float64 sums): two outputs per lane, so the float64 D ring
    // and P buffer stay small enough for ~24 warps per SM
    constexpr int OPL = sizeof(TS) == 8 ? 2 : 4;
    constexpr int SWC = 32 * OPL;                 // output columns per unit
    auto kern = sat_boxw_kernel<TI, TS, TO, NWARP, PF, OPL>;
    const size_t smem = size_t(NWARP) * boxw_warp_smem<TI, TS, PF, OPL>(rr);
    static KernelSetup setup;
    int dev = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    if (dev < 0 || dev >= kMaxDev) return fail(SAT_ERR_CUDA, "device ordinal out of range");
    std::call_once(setup.once[dev], [&] {
        setup.err[dev] = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    });
    if (setup.err[dev] != cudaSuccess)
        return fail(SAT_ERR_CUDA, std::string("box kernel set-up: ") + cudaGetErrorString(setup.err[dev]));
    if (smem > 200 * 1024) return fail(SAT_ERR_UNSUPPORTED, "box filter: radius too large for the walk kernel");
    BoxWParams bp;
    bp.in = in; bp.out = out; bp.rows = int(rows); bp.cols = int(cols); bp.batch = int(batch);
    bp.rr = rr; bp.rc = rc; bp.normalize = normalize;
    bp.nc = int((cols + SWC - 1) / SWC);
    bp.rb = g_box_rb.load(std::memory_order_relaxed);
    if (bp.rb <= 0) {
        // one wave: as many row blocks per strip as the resident warps allow
        // (units = batch x strips x row blocks <= warp slots), so every warp
        // runs from the start and the 2 rr-row warm-up is paid as few times
        // as possible; blocks of >= 32 rows.  32 x 1080x1920 uint8 r = 4:
        // 0.119 ms (6 blocks of 180 rows) vs 0.125 (64-row blocks, two
        // waves) and 0.141 (120-row blocks, 1.04 waves); tools/box_rows.py
        int per_sm = 0;
        CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, NWARP * 32, smem));
        int sms = 0;
        CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
        const long long slots = (long long)std::max(per_sm, 1) * NWARP * sms;
        const long long strips = batch * (long long)bp.nc;
        const long long nrb = std::max(1LL, slots / strips);
        bp.rb = int(std::max<long long>(32, (rows + nrb - 1) / nrb));
    }
    bp.nrb = int((rows + bp.rb - 1) / bp.rb);
    bp.units = (long long)batch * bp.nrb * bp.nc;
    const uintptr_t ia = reinterpret_cast<uintptr_t>(in);
    if (!(sizeof(TI) == 1 ? (cols % 8 == 0 && (ia & 7) == 0) : (cols % 4 == 0 && (ia & 15) == 0)))
        return fail(SAT_ERR_INVALID, "box walk: misaligned rows");
    const long long grid = (bp.units + NWARP - 1) / NWARP;
    cudaLaunchConfig_t cfg;
    std::memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = dim3(unsigned(grid));
    cfg.blockDim = dim3(NWARP * 32);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, bp));
    CUDA_TRY(cudaGetLastError());
    t_launches = 1;
    t_grid = int(std::min<long long>(grid, INT32_MAX));
    return SAT_OK;
}

}  // namespace

// ====================================================================== C ABI
extern "C" {

size_t sat_exchange_mailbox_bytes(int64_t cols, int nranks, int dtype) {
    if (cols <= 0 || nranks <= 0 || !dtype_ok(dtype)) return 0;
    XchgLayout L{nranks, cols, esize(dtype)};
    return L.bytes();
}

int sat_exchange_create(void** handle, int rank, int nranks, int64_t cols, int dtype, void* mailbox,
                        void* const* peers) {
    if (!handle) return fail(SAT_ERR_INVALID, "null handle");
    *handle = nullptr;
    if (!dtype_ok(dtype)) return fail(SAT_ERR_INVALID, "bad dtype");
    if (nranks < 1 || nranks > 16 || rank < 0 || rank >= nranks)
        return fail(SAT_ERR_INVALID, "nranks must be 1..16 and 0 <= rank < nranks");
    if (cols <= 0 || !mailbox || !peers) return fail(SAT_ERR_INVALID, "bad cols / null pointer");
    for (int q = 0; q < nranks; ++q)
        if (!peers[q]) return fail(SAT_ERR_INVALID, "null peer mailbox");
    if (reinterpret_cast<uintptr_t>(mailbox) & 255) return fail(SAT_ERR_INVALID, "mailbox must be 256-B aligned");
    PeerExchange* ex = new PeerExchange();
    ex->rank = rank; ex->nranks = nranks; ex->dtype = dtype; ex->cols = cols;
    std::memset(&ex->x, 0, sizeof(ex->x));
    ex->x.L = XchgLayout{nranks, cols, esize(dtype)};
    ex->x.rank = rank;
    ex->x.epoch = 0;
    ex->x.mine = static_cast<uint8_t*>(mailbox);
    for (int q = 0; q < nranks; ++q) ex->x.peers[q] = static_cast<uint8_t*>(peers[q]);
    if (cudaMalloc(&ex->done, sizeof(unsigned int)) != cudaSuccess) {
        cudaGetLastError();
        delete ex;
        return fail(SAT_ERR_NOMEM, "exchange counter");
    }
    ex->x.done = ex->done;
    if (cudaMalloc(&ex->acks, sizeof(uint64_t*) * 16) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(ex->done);
        delete ex;
        return fail(SAT_ERR_NOMEM, "exchange ack table");
    }
    uint64_t* acks_h[16] = {};
    for (int q = 0; q < rank; ++q)
        acks_h[q] = reinterpret_cast<uint64_t*>(ex->x.peers[q] + ex->x.L.acks_off()) + rank;
    CUDA_TRY(cudaMemcpy(ex->acks, acks_h, sizeof(acks_h), cudaMemcpyHostToDevice));
    CUDA_TRY(cudaMemset(ex->done, 0, sizeof(unsigned int)));
    CUDA_TRY(cudaMemset(mailbox, 0, ex->x.L.bytes()));
    CUDA_TRY(cudaDeviceSynchronize());
    *handle = ex;
    return SAT_OK;
}

int sat_exchange_destroy(void* handle) {
    PeerExchange* ex = static_cast<PeerExchange*>(handle);
    if (!ex) return SAT_OK;
    cudaFree(ex->done);
    cudaFree(ex->acks);
    delete ex;
    return SAT_OK;
}

int sat_compute_sharded_fused(const void* in_strip, void* out_strip, int64_t strip_rows, void* handle,
                              void* stream) {
    t_launches = 0;
    PeerExchange* ex = static_cast<PeerExchange*>(handle);
    if (!ex) return fail(SAT_ERR_INVALID, "null exchange");
    SAT_TRY(validate(in_strip, out_strip, 1, strip_rows, ex->cols, ex->dtype));
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    return SAT_DISPATCH(ex->dtype, T, sharded_fused_t<T>(in_strip, out_strip, strip_rows, *ex, st));
}

int sat_ipc_get_handle(const void* dev_ptr, void* handle64) {
    if (!dev_ptr || !handle64) return fail(SAT_ERR_INVALID, "null pointer");
    cudaIpcMemHandle_t h;
    CUDA_TRY(cudaIpcGetMemHandle(&h, const_cast<void*>(dev_ptr)));
    std::memcpy(handle64, &h, sizeof(h));
    return SAT_OK;
}

int sat_ipc_open(const void* handle64, void** dev_ptr) {
    if (!handle64 || !dev_ptr) return fail(SAT_ERR_INVALID, "null pointer");
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle64, sizeof(h));
    CUDA_TRY(cudaIpcOpenMemHandle(dev_ptr, h, cudaIpcMemLazyEnablePeerAccess));
    return SAT_OK;
}

int sat_ipc_close(void* dev_ptr) {
    if (!dev_ptr) return SAT_OK;
    CUDA_TRY(cudaIpcCloseMemHandle(dev_ptr));
    return SAT_OK;
}

void sat_options_init(sat_options* opt) {
    if (!opt) return;
    std::memset(opt, 0, sizeof(*opt));
    opt->r = 0.25;
}

int sat_compute(const void* in, void* out, int64_t rows, int64_t cols, int dtype, int variant,
                void* stream) {
    return compute_core(in, out, 1, rows, cols, dtype, variant, nullptr, nullptr, nullptr,
                        static_cast<cudaStream_t>(stream));
}

int sat_compute_ex(const void* in, void* out, int64_t rows, int64_t cols, int dtype, int variant,
                   const sat_options* opt, void* stream) {
    return compute_core(in, out, 1, rows, cols, dtype, variant, opt, nullptr, nullptr,
                        static_cast<cudaStream_t>(stream));
}

int sat_compute_batched(const void* in, void* out, int64_t batch, int64_t rows, int64_t cols,
                        int dtype, int variant, const sat_options* opt, void* stream) {
    return compute_core(in, out, batch, rows, cols, dtype, variant, opt, nullptr, nullptr,
                        static_cast<cudaStream_t>(stream));
}

int sat_compute_widening(const void* in, int in_dtype, void* out, int dtype, int64_t batch,
                         int64_t rows, int64_t cols, const sat_options* opt, void* stream) {
    if (in_dtype != SAT_UINT8 && !dtype_ok(in_dtype)) return fail(SAT_ERR_INVALID, "bad input dtype");
    return compute_core(in, out, batch, rows, cols, dtype, SAT_1R1W, opt, nullptr, nullptr,
                        static_cast<cudaStream_t>(stream), in_dtype);
}

int sat_box_filter(const void* in, int in_dtype, void* out, int out_dtype, int64_t batch,
                   int64_t rows, int64_t cols, int rr, int rc, int normalize, void* stream) {
    t_launches = 0;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    // the SAT's type: uint32 sums for integer pixels, float64 for float inputs
    const int sdt = (in_dtype == SAT_UINT8 || in_dtype == SAT_INT32) ? SAT_INT32
                    : (in_dtype == SAT_FLOAT32 || in_dtype == SAT_FLOAT64) ? SAT_FLOAT64 : -1;
    if (sdt < 0) return fail(SAT_ERR_INVALID, "box filter input must be UINT8, INT32, FLOAT32 or FLOAT64");
    if (sdt == SAT_INT32 ? out_dtype != SAT_INT32 : (out_dtype != SAT_FLOAT32 && out_dtype != SAT_FLOAT64))
        return fail(SAT_ERR_INVALID, "box filter output: INT32 for integer input, FLOAT32/64 for float input");
    if (rr < 0 || rc < 0) return fail(SAT_ERR_INVALID, "negative radius");
    // windows are clipped to the image anyway: a radius beyond it changes
    // nothing, and clamping keeps i + rr / j + rc inside the index type
    if (rr > rows) rr = int(std::min<int64_t>(rows, INT32_MAX));
    if (rc > cols) rc = int(std::min<int64_t>(cols, INT32_MAX));
    if (normalize && sdt == SAT_INT32) return fail(SAT_ERR_INVALID, "normalize needs float input");
    if (batch > 65535) return fail(SAT_ERR_UNSUPPORTED, "box filter: batch must be <= 65535");
    SAT_TRY(validate(nullptr, out, batch, rows, cols, out_dtype, false));
    if (rows == 0 || cols == 0 || batch == 0) return SAT_OK;
    if (!in) return fail(SAT_ERR_INVALID, "null pointer with nonzero size");
    if (reinterpret_cast<uintptr_t>(in) & (esize(in_dtype) - 1))
        return fail(SAT_ERR_INVALID, "pointers must be aligned to the element size");
    {   // the SAT lives in a workspace, so out may alias in exactly, not partially
        const uintptr_t a0 = reinterpret_cast<uintptr_t>(in), b0 = reinterpret_cast<uintptr_t>(out);
        const uintptr_t n_el = uintptr_t(rows) * uintptr_t(cols) * uintptr_t(batch);
        const uintptr_t la = n_el * esize(in_dtype), lb = n_el * esize(out_dtype);
        if (a0 != b0 && a0 < b0 + lb && b0 < a0 + la)
            return fail(SAT_ERR_INVALID, "in and out partially overlap");
        if (a0 == b0 && la != lb) return fail(SAT_ERR_INVALID, "in place needs equal element sizes");
    }
    int dev;
    DevInfo di;
    SAT_TRY(get_dev(dev, di));
    Workspace* ws;
    SAT_TRY(get_ws(dev, st, ws));
    // Column walk (one launch, one warp per 128-column strip of a row block --
    // 64 columns for float input, sat_boxw.cuh) when out does not alias in,
    // rc <= 63 and rr <= 8 (uint8 / int32 / float32): 32 x 1080x1920 r = 4
    // uint8 0.127 ms, int32 0.150, float32 0.272 (band kernel: 0.182 / 0.186 /
    // 0.305), DESIGN.md Sec. 4.12
    const bool walk_al = in_dtype == SAT_UINT8 ? (cols % 8 == 0 && (reinterpret_cast<uintptr_t>(in) & 7) == 0)
                                               : (cols % 4 == 0 && (reinterpret_cast<uintptr_t>(in) & 15) == 0);
    if (walk_al && in != out && rc <= 63 && rr <= 16 && rows <= INT32_MAX && cols <= INT32_MAX &&
        batch * rows <= INT32_MAX) {
        if (in_dtype == SAT_UINT8 && rr <= 8)
            return box_walk_t<uint8_t, uint32_t, int32_t>(in, out, batch, rows, cols, rr, rc, 0, st);
        if (in_dtype == SAT_INT32 && rr <= 8)
            return box_walk_t<uint32_t, uint32_t, int32_t>(in, out, batch, rows, cols, rr, rc, 0, st);
        if (in_dtype == SAT_FLOAT32 && rr <= 8)
            return out_dtype == SAT_FLOAT32
                       ? box_walk_t<float, double, float>(in, out, batch, rows, cols, rr, rc, normalize, st)
                       : box_walk_t<float, double, double>(in, out, batch, rows, cols, rr, rc, normalize, st);
    }
    // Fused (one launch, the SAT never leaves the chip, sat_boxf.cuh) when the
    // input is TMA-addressable, out does not alias it (a band's halo rows are
    // another band's output rows), the halo fits the band buffer and rc < 128.
    {
        const bool al = (reinterpret_cast<uintptr_t>(in) & 15) == 0 && (reinterpret_cast<uintptr_t>(out) & 15) == 0;
        const bool apart = in != out;
        const bool u8 = in_dtype == SAT_UINT8 && cols % 16 == 0 && 2 * rr <= 32;
        const bool i32 = in_dtype == SAT_INT32 && cols % 4 == 0 && 2 * rr <= 32;
        const bool f32 = in_dtype == SAT_FLOAT32 && cols % 4 == 0 && 2 * rr <= 16;
        if (al && apart && rc <= 127 && rows <= INT32_MAX && cols <= INT32_MAX && (u8 || i32 || f32)) {
            // uint8 with 2 rr <= 16: 32-row bands of 8 warps, ~104 KB of shared
            // memory, two CTAs per SM (one CTA's barrier phases overlap the
            // other's work)
            if (u8 && 2 * rr <= 16)
                return box_fused_t<uint8_t, uint32_t, int32_t, 32, 48, 4, 8, 2>(in, in_dtype, out, batch, rows, cols, rr,
                                                                                 rc, 0, di, *ws, st);
            if (u8)
                return box_fused_t<uint8_t, uint32_t, int32_t, 64, 96, 4>(in, in_dtype, out, batch, rows, cols, rr, rc, 0,
                                                                           di, *ws, st);
            if (i32 && 2 * rr <= 16)
                return box_fused_t<uint32_t, uint32_t, int32_t, 16, 32, 2, 8, 2>(in, in_dtype, out, batch, rows, cols,
                                                                                  rr, rc, 0, di, *ws, st);
            if (i32)
                return box_fused_t<uint32_t, uint32_t, int32_t, 32, 64, 2>(in, in_dtype, out, batch, rows, cols, rr, rc,
                                                                            0, di, *ws, st);
            if (out_dtype == SAT_FLOAT32 && 2 * rr <= 8)
                return box_fused_t<float, double, float, 16, 24, 2, 8, 2>(in, in_dtype, out, batch, rows, cols, rr,
                                                                           rc, normalize, di, *ws, st);
            if (out_dtype == SAT_FLOAT32)
                return box_fused_t<float, double, float, 32, 48, 2>(in, in_dtype, out, batch, rows, cols, rr, rc,
                                                                     normalize, di, *ws, st);
            if (2 * rr <= 8)
                return box_fused_t<float, double, double, 16, 24, 2, 8, 2>(in, in_dtype, out, batch, rows, cols, rr,
                                                                            rc, normalize, di, *ws, st);
            return box_fused_t<float, double, double, 32, 48, 2>(in, in_dtype, out, batch, rows, cols, rr, rc,
                                                                  normalize, di, *ws, st);
        }
    }
    SAT_TRY(ensure(ws->box, size_t(batch) * rows * cols * esize(sdt), false));
    // 1. the SAT (1R1W, widening uint8 -> uint32 and float32 -> float64 on load)
    SAT_TRY(compute_core(in, ws->box.p, batch, rows, cols, sdt, SAT_1R1W, nullptr, nullptr, nullptr,
                         st, in_dtype));
    int launches = t_launches;
    // 2. four SAT reads per output element
    const dim3 grid(unsigned((cols + 255) / 256), unsigned(std::min<int64_t>((rows + BOX_RB - 1) / BOX_RB, 65535)),
                    unsigned(batch));
    auto box = [&](auto idx) {
        using I = decltype(idx);
        if (sdt == SAT_INT32)
            sat_box_kernel<uint32_t, int32_t, I><<<grid, 256, 0, st>>>(
                static_cast<const uint32_t*>(ws->box.p), static_cast<int32_t*>(out), I(rows), I(cols), rr, rc, 0);
        else if (out_dtype == SAT_FLOAT32)
            sat_box_kernel<double, float, I><<<grid, 256, 0, st>>>(
                static_cast<const double*>(ws->box.p), static_cast<float*>(out), I(rows), I(cols), rr, rc, normalize);
        else
            sat_box_kernel<double, double, I><<<grid, 256, 0, st>>>(
                static_cast<const double*>(ws->box.p), static_cast<double*>(out), I(rows), I(cols), rr, rc, normalize);
    };
    if (rows * cols < (int64_t(1) << 31)) box(int32_t(0));
    else box(int64_t(0));
    CUDA_TRY(cudaGetLastError());
    t_launches = launches + 1;
    return SAT_OK;
}

int sat_rect_sums(const void* sat, int dtype, int64_t batch, int64_t rows, int64_t cols,
                  const int32_t* rects, int64_t nrects, void* out, void* stream) {
    t_launches = 0;
    if (!dtype_ok(dtype)) return fail(SAT_ERR_INVALID, "bad dtype");
    if (nrects < 0 || batch < 0 || rows < 0 || cols < 0) return fail(SAT_ERR_INVALID, "negative size");
    if (nrects == 0) return SAT_OK;
    if (!sat || !rects || !out) return fail(SAT_ERR_INVALID, "null pointer");
    int dev;
    DevInfo di;
    SAT_TRY(get_dev(dev, di));
    const unsigned blocks = unsigned(std::min<int64_t>((nrects + 255) / 256, 16LL * di.sms));
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    SAT_DISPATCH(dtype, T, (sat_rect_kernel<T><<<blocks, 256, 0, st>>>(static_cast<const T*>(sat), batch, rows,
                                                                      cols, rects, nrects, static_cast<T*>(out)),
                            0));
    CUDA_TRY(cudaGetLastError());
    t_launches = 1;
    return SAT_OK;
}

int sat_compute_seeded(const void* in, void* out, int64_t rows, int64_t cols, int dtype,
                       const void* carry_row, void* stream) {
    return sat_compute_seeded_sum(in, out, rows, cols, dtype, carry_row, carry_row ? 1 : 0, 0, stream);
}

int sat_compute_seeded_sum(const void* in, void* out, int64_t rows, int64_t cols, int dtype,
                           const void* vectors, int64_t nvec, int64_t stride, void* stream) {
    if (nvec < 0 || nvec > INT32_MAX) return fail(SAT_ERR_INVALID, "nvec must be in [0, 2^31)");
    if (nvec > 0 && !vectors) return fail(SAT_ERR_INVALID, "null seed vectors");
    if (nvec > 1 && stride < cols) return fail(SAT_ERR_INVALID, "seed stride must be >= cols");
    ColSeed cs;
    std::memset(&cs, 0, sizeof(cs));
    cs.base = vectors;
    cs.stride = stride * int64_t(esize(dtype));
    cs.n = int(nvec);
    return compute_core(in, out, 1, rows, cols, dtype, SAT_1R1W, nullptr, nullptr, &cs,
                        static_cast<cudaStream_t>(stream));
}

int sat_compute_seeded_satrow(const void* in, void* out, int64_t rows, int64_t cols, int dtype,
                              const void* sat_row, void* stream) {
    return compute_core(in, out, 1, rows, cols, dtype, SAT_1R1W, nullptr, sat_row, nullptr,
                        static_cast<cudaStream_t>(stream));
}

int sat_column_totals(const void* in, void* totals, int64_t rows, int64_t cols, int dtype,
                      void* stream) {
    t_launches = 0;
    SAT_TRY(validate(in, totals, 1, rows, cols, dtype, true));
    if (rows == 0 || cols == 0) {
        if (cols > 0 && totals)
            CUDA_TRY(cudaMemsetAsync(totals, 0, size_t(cols) * esize(dtype), static_cast<cudaStream_t>(stream)));
        return SAT_OK;
    }
    return column_totals_core(in, totals, rows, cols, dtype, static_cast<cudaStream_t>(stream));
}

int sat_rank_exscan(const void* gathered, void* carry_row, int64_t nranks, int64_t cols, int rank,
                    int dtype, void* stream) {
    t_launches = 0;
    if (!dtype_ok(dtype)) return fail(SAT_ERR_INVALID, "bad dtype");
    if (nranks < 1 || rank < 0 || rank >= nranks || cols < 0)
        return fail(SAT_ERR_INVALID, "bad rank / nranks / cols");
    if (cols == 0) return SAT_OK;
    if (!carry_row || (rank > 0 && !gathered)) return fail(SAT_ERR_INVALID, "null pointer");
    return exscan_core(gathered, carry_row, nranks, cols, rank, dtype,
                       static_cast<cudaStream_t>(stream));
}

size_t sat_sharded_workspace_bytes(int64_t cols, int nranks, int dtype) {
    if (cols <= 0 || nranks <= 0) return 0;
    const size_t row = align256(size_t(cols) * (dtype == SAT_FLOAT64 ? 8 : 4));
    return row * size_t(nranks + 2);
}

int sat_compute_sharded(const void* in_strip, void* out_strip, int64_t strip_rows, int64_t cols,
                        int dtype, int rank, int nranks, sat_allgather_fn allgather,
                        void* comm_ctx, void* workspace, void* stream, sat_shard_stats* stats) {
    return sat_compute_sharded_ex(in_strip, out_strip, strip_rows, cols, dtype, SAT_1R1W, rank, nranks, allgather,
                                  comm_ctx, workspace, stream, stats);
}

int sat_compute_sharded_ex(const void* in_strip, void* out_strip, int64_t strip_rows, int64_t cols,
                           int dtype, int variant, int rank, int nranks, sat_allgather_fn allgather,
                           void* comm_ctx, void* workspace, void* stream, sat_shard_stats* stats) {
    t_launches = 0;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(SAT_ERR_INVALID, "bad rank / nranks");
    if (variant != SAT_1R1W && variant != SAT_2R2W)
        return fail(SAT_ERR_UNSUPPORTED, "sharded SAT: variant must be SAT_1R1W or SAT_2R2W");
    SAT_TRY(validate(in_strip, out_strip, 1, strip_rows, cols, dtype));
    if (nranks > 1 && !allgather) return fail(SAT_ERR_INVALID, "allgather callback required");
    if (stats) std::memset(stats, 0, sizeof(*stats));
    if (cols == 0) return SAT_OK;
    const size_t eb = esize(dtype);
    const size_t row = align256(size_t(cols) * eb);
    uint8_t* wsp = static_cast<uint8_t*>(workspace);
    if (!wsp) {
        int dev;
        DevInfo di;
        SAT_TRY(get_dev(dev, di));
        Workspace* ws;
        SAT_TRY(get_ws(dev, st, ws));
        SAT_TRY(ensure(ws->shard, sat_sharded_workspace_bytes(cols, nranks, dtype), false));
        wsp = static_cast<uint8_t*>(ws->shard.p);
    }
    void* send = wsp;
    void* recv = wsp + 2 * row;
    int launches = 0;
    ColSeed cs;
    std::memset(&cs, 0, sizeof(cs));
    if (nranks > 1) {
        // 1. column totals of the strip (the extra read, one launch); the last
        //    rank's totals are never consumed, so it sends zeros instead
        if (rank < nranks - 1 && strip_rows > 0) {
            SAT_TRY(column_totals_core(in_strip, send, strip_rows, cols, dtype, st));
            launches += t_launches;
        } else {
            CUDA_TRY(cudaMemsetAsync(send, 0, size_t(cols) * eb, st));
        }
        // 2. all-gather of the m-vectors (NCCL over NVLink in the Python binding)
        if (allgather(comm_ctx, send, recv, size_t(cols) * eb, stream) != 0)
            return fail(SAT_ERR_COMM, "allgather callback failed");
        // 3. the exclusive scan over ranks is the band kernel's seed: band 0
        //    adds sum_{q < rank} recv[q] (q ascending) to its first row
        cs.base = recv;
        cs.stride = int64_t(cols) * int64_t(eb);
        cs.n = rank;
    }
    // 4. seeded local SAT (1R1W, or 2R2W whose column pass takes the seed)
    if (strip_rows > 0) {
        SAT_TRY(compute_core(in_strip, out_strip, 1, strip_rows, cols, dtype, variant, nullptr,
                             nullptr, &cs, st));
        launches += t_launches;
    }
    t_launches = launches;
    if (stats) {
        const int64_t b = strip_rows * cols * int64_t(eb) * (variant == SAT_2R2W ? 2 : 1);
        stats->strip_bytes_read = b;
        stats->strip_bytes_written = b;
        stats->extra_bytes_read = (nranks > 1 && rank < nranks - 1) ? b : 0;
        stats->allgather_bytes = nranks > 1 ? int64_t(nranks) * cols * int64_t(eb) : 0;
    }
    return SAT_OK;
}

int sat_compute_host(const void* in_host, void* out_host, int64_t rows, int64_t cols, int dtype,
                     int variant, void* stream) {
    t_launches = 0;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (!dtype_ok(dtype)) return fail(SAT_ERR_INVALID, "bad dtype");
    if (rows < 0 || cols < 0) return fail(SAT_ERR_INVALID, "negative size");
    if (rows == 0 || cols == 0) return SAT_OK;
    if (!in_host || !out_host) return fail(SAT_ERR_INVALID, "null pointer");
    int dev;
    DevInfo di;
    SAT_TRY(get_dev(dev, di));
    Workspace* ws;
    SAT_TRY(get_ws(dev, st, ws));
    if (t_capture)
        return fail(SAT_ERR_UNSUPPORTED, "sat_compute_host cannot be captured: it synchronizes the stream");
    const size_t bytes = size_t(rows) * size_t(cols) * esize(dtype);
    SAT_TRY(ensure(ws->din, bytes, false));
    SAT_TRY(ensure(ws->dout, bytes, false));
    cudaPointerAttributes ai, ao;
    bool pinned = cudaPointerGetAttributes(&ai, in_host) == cudaSuccess &&
                  cudaPointerGetAttributes(&ao, out_host) == cudaSuccess &&
                  ai.type == cudaMemoryTypeHost && ao.type == cudaMemoryTypeHost;
    cudaGetLastError();
    int launches = 0;
    if (!pinned || variant != SAT_1R1W || rows < 512) {
        CUDA_TRY(cudaMemcpyAsync(ws->din.p, in_host, bytes, cudaMemcpyHostToDevice, st));
        SAT_TRY(compute_core(ws->din.p, ws->dout.p, 1, rows, cols, dtype, variant, nullptr,
                             nullptr, nullptr, st));
        launches = t_launches;
        CUDA_TRY(cudaMemcpyAsync(out_host, ws->dout.p, bytes, cudaMemcpyDeviceToHost, st));
        CUDA_TRY(cudaStreamSynchronize(st));
        t_launches = launches;
        return SAT_OK;
    }
    // Pinned 1R1W: stream row strips; strip k is seeded with the last SAT row
    // of strip k-1, so H2D of strip k+1 and D2H of strip k-1 overlap the SAT
    // of strip k.
    if (!ws->cstream_in) {
        CUDA_TRY(cudaStreamCreateWithFlags(&ws->cstream_in, cudaStreamNonBlocking));
        CUDA_TRY(cudaStreamCreateWithFlags(&ws->cstream_out, cudaStreamNonBlocking));
    }
    // 32 strips: fill/drain of the copy pipeline is 1/32 of the transfer
    // (32768^2 int32: 89.9 ms vs 95.3 ms with 8 strips; H2D+D2H concurrently
    // take 87.8 ms, tools/pcie_probe.py)
    const int want = 32;
    const int nstrips = int(std::min<int64_t>(want, rows / 256));
    const int64_t srows = (rows + nstrips - 1) / nstrips;
    cudaEvent_t ev_start, ev_in[64], ev_done[64];
    CUDA_TRY(cudaEventCreateWithFlags(&ev_start, cudaEventDisableTiming));
    for (int k = 0; k < nstrips; ++k) {
        CUDA_TRY(cudaEventCreateWithFlags(&ev_in[k], cudaEventDisableTiming));
        CUDA_TRY(cudaEventCreateWithFlags(&ev_done[k], cudaEventDisableTiming));
    }
    CUDA_TRY(cudaEventRecord(ev_start, st));
    CUDA_TRY(cudaStreamWaitEvent(ws->cstream_in, ev_start, 0));
    const uint8_t* hin = static_cast<const uint8_t*>(in_host);
    uint8_t* hout = static_cast<uint8_t*>(out_host);
    uint8_t* din = static_cast<uint8_t*>(ws->din.p);
    uint8_t* dout = static_cast<uint8_t*>(ws->dout.p);
    const size_t rowb = size_t(cols) * esize(dtype);
    for (int k = 0; k < nstrips; ++k) {
        const int64_t r0 = k * srows, r1 = std::min<int64_t>(rows, r0 + srows);
        if (r1 <= r0) { CUDA_TRY(cudaEventRecord(ev_in[k], ws->cstream_in)); continue; }
        CUDA_TRY(cudaMemcpyAsync(din + r0 * rowb, hin + r0 * rowb, (r1 - r0) * rowb,
                                 cudaMemcpyHostToDevice, ws->cstream_in));
        CUDA_TRY(cudaEventRecord(ev_in[k], ws->cstream_in));
    }
    for (int k = 0; k < nstrips; ++k) {
        const int64_t r0 = k * srows, r1 = std::min<int64_t>(rows, r0 + srows);
        CUDA_TRY(cudaStreamWaitEvent(st, ev_in[k], 0));
        if (r1 > r0) {
            SAT_TRY(compute_core(din + r0 * rowb, dout + r0 * rowb, 1, r1 - r0, cols, dtype,
                                 SAT_1R1W, nullptr, k > 0 ? dout + (r0 - 1) * rowb : nullptr,
                                 nullptr, st));
            launches += t_launches;
        }
        CUDA_TRY(cudaEventRecord(ev_done[k], st));
        CUDA_TRY(cudaStreamWaitEvent(ws->cstream_out, ev_done[k], 0));
        if (r1 > r0)
            CUDA_TRY(cudaMemcpyAsync(hout + r0 * rowb, dout + r0 * rowb, (r1 - r0) * rowb,
                                     cudaMemcpyDeviceToHost, ws->cstream_out));
    }
    CUDA_TRY(cudaStreamSynchronize(ws->cstream_out));
    CUDA_TRY(cudaStreamSynchronize(st));
    cudaEventDestroy(ev_start);
    for (int k = 0; k < nstrips; ++k) { cudaEventDestroy(ev_in[k]); cudaEventDestroy(ev_done[k]); }
    t_launches = launches;
    return SAT_OK;
}

// ------------------------------------------------------------------ in-library NCCL
// The sharded mode's all-gather over NVLink/NVSwitch through an NCCL
// communicator owned by the caller's handle.  libnccl.so.2 is loaded on first
// use (dlopen): a process that already loaded NCCL (e.g. through PyTorch)
// shares that copy, and libsat has no link-time NCCL dependency.
namespace {
struct NcclApi {
    ncclResult_t (*get_unique_id)(ncclUniqueId*) = nullptr;
    ncclResult_t (*comm_init_rank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*all_gather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*comm_destroy)(ncclComm_t) = nullptr;
    ncclResult_t (*comm_count)(const ncclComm_t, int*) = nullptr;
    ncclResult_t (*comm_user_rank)(const ncclComm_t, int*) = nullptr;
    const char* (*error_string)(ncclResult_t) = nullptr;
    std::string err;
};
NcclApi& nccl_api() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            const char* e = dlerror();          // read once: a second call returns NULL
            api.err = std::string("dlopen libnccl.so.2: ") + (e ? e : "unknown error");
            return;
        }
        auto sym = [&](const char* n) {
            void* f = dlsym(h, n);
            if (!f && api.err.empty()) api.err = std::string("libnccl: missing ") + n;
            return f;
        };
        api.get_unique_id = reinterpret_cast<decltype(api.get_unique_id)>(sym("ncclGetUniqueId"));
        api.comm_init_rank = reinterpret_cast<decltype(api.comm_init_rank)>(sym("ncclCommInitRank"));
        api.all_gather = reinterpret_cast<decltype(api.all_gather)>(sym("ncclAllGather"));
        api.comm_destroy = reinterpret_cast<decltype(api.comm_destroy)>(sym("ncclCommDestroy"));
        api.comm_count = reinterpret_cast<decltype(api.comm_count)>(sym("ncclCommCount"));
        api.comm_user_rank = reinterpret_cast<decltype(api.comm_user_rank)>(sym("ncclCommUserRank"));
        api.error_string = reinterpret_cast<decltype(api.error_string)>(sym("ncclGetErrorString"));
    });
    return api;
}
#define NCCL_TRY(x)                                                                              \
    do {                                                                                         \
        const ncclResult_t r_ = (x);                                                             \
        if (r_ != ncclSuccess)                                                                   \
            return fail(SAT_ERR_COMM, std::string("NCCL: ") + nccl_api().error_string(r_));      \
    } while (0)
int nccl_allgather_cb(void* ctx, const void* send, void* recv, size_t bytes, void* stream) {
    return nccl_api().all_gather(send, recv, bytes, ncclUint8, static_cast<ncclComm_t>(ctx),
                                 static_cast<cudaStream_t>(stream)) == ncclSuccess ? 0 : 1;
}
}  // namespace

extern "C" {

int sat_nccl_unique_id(void* id128) {
    if (!id128) return fail(SAT_ERR_INVALID, "null id buffer");
    NcclApi& a = nccl_api();
    if (!a.err.empty()) return fail(SAT_ERR_UNSUPPORTED, a.err);
    ncclUniqueId id;
    NCCL_TRY(a.get_unique_id(&id));
    static_assert(sizeof(id) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(id128, &id, sizeof(id));
    return SAT_OK;
}

int sat_nccl_comm_create(void** comm, const void* id128, int rank, int nranks) {
    if (!comm || !id128) return fail(SAT_ERR_INVALID, "null pointer");
    *comm = nullptr;
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(SAT_ERR_INVALID, "bad rank / nranks");
    NcclApi& a = nccl_api();
    if (!a.err.empty()) return fail(SAT_ERR_UNSUPPORTED, a.err);
    ncclUniqueId id;
    std::memcpy(&id, id128, sizeof(id));
    ncclComm_t c = nullptr;
    NCCL_TRY(a.comm_init_rank(&c, nranks, id, rank));
    *comm = c;
    return SAT_OK;
}

int sat_nccl_comm_destroy(void* comm) {
    if (!comm) return SAT_OK;
    NcclApi& a = nccl_api();
    if (!a.err.empty()) return fail(SAT_ERR_UNSUPPORTED, a.err);
    NCCL_TRY(a.comm_destroy(static_cast<ncclComm_t>(comm)));
    return SAT_OK;
}

int sat_compute_sharded_nccl(const void* in_strip, void* out_strip, int64_t strip_rows, int64_t cols, int dtype,
                             int variant, void* comm, void* workspace, void* stream, sat_shard_stats* stats) {
    if (!comm) return fail(SAT_ERR_INVALID, "null NCCL communicator");
    NcclApi& a = nccl_api();
    if (!a.err.empty()) return fail(SAT_ERR_UNSUPPORTED, a.err);
    int rank = 0, nranks = 0;
    NCCL_TRY(a.comm_user_rank(static_cast<ncclComm_t>(comm), &rank));
    NCCL_TRY(a.comm_count(static_cast<ncclComm_t>(comm), &nranks));
    return sat_compute_sharded_ex(in_strip, out_strip, strip_rows, cols, dtype, variant, rank, nranks,
                                  nccl_allgather_cb, comm, workspace, stream, stats);
}

}  // extern "C"

static unsigned int* g_diag_host = nullptr;
static const size_t kDiagWords = size_t(4096) * 32 * 4 * 2;

int sat_debug_diag_enable(void) {
    if (!g_diag_host) {
        CUDA_TRY(cudaHostAlloc(&g_diag_host, kDiagWords * 4, cudaHostAllocMapped));
        std::memset(g_diag_host, 0, kDiagWords * 4);
    }
    unsigned int* dptr = nullptr;
    CUDA_TRY(cudaHostGetDevicePointer(&dptr, g_diag_host, 0));
    CUDA_TRY(cudaMemcpyToSymbol(sat::g_sat_diag, &dptr, sizeof(dptr)));
    g_diag_dev = static_cast<unsigned int*>(dptr);
    return SAT_OK;
}

int sat_debug_diag_dump(void) {
    if (!g_diag_host) return 0;
    int n = 0;
    for (size_t i = kDiagWords / 2; i < kDiagWords; i += 4) {
        if ((g_diag_host[i + 2] & 0xFFFF0000u) == 0xC0DE0000u)
            std::fprintf(stderr, "mark block %u warp %zu: unit %u step %u mark %u\n", g_diag_host[i + 3],
                         ((i - kDiagWords / 2) / 4) % 32, g_diag_host[i], g_diag_host[i + 1],
                         g_diag_host[i + 2] & 0xFFFFu);
    }
    for (size_t b = 0; b < 4096; ++b) {
        const unsigned int* h = g_diag_host + kDiagWords / 2 + size_t(4096) * 32 * 2 + b * 16;
        if (h[15]) {
            std::fprintf(stderr, "units block %zu:", b);
            for (unsigned int q = 0; q < h[15] && q < 15; ++q) std::fprintf(stderr, " %u", h[q]);
            std::fprintf(stderr, "\n");
        }
    }
    for (size_t i = 0; i < kDiagWords / 2; i += 4) {
        if ((g_diag_host[i + 2] & 0xFFFF0000u) == 0xC0DE0000u) {
            std::fprintf(stderr, "diag block %u warp %zu thread %u: what 0x%08x extra %u\n",
                         g_diag_host[i + 2] & 0xFFFFu, (i / 4) % 32, g_diag_host[i + 3],
                         g_diag_host[i], g_diag_host[i + 1]);
            ++n;
        }
    }
    return n;
}

int sat_debug_trace(void* dev_buf) {
    if (!kDebug) return fail(SAT_ERR_UNSUPPORTED, "event traces need a debug build (SAT_DEBUG=1)");
    t_trace = static_cast<unsigned long long*>(dev_buf);
    return SAT_OK;
}

int sat_debug_set_box_rows(int rows) {
    if (rows < 0 || rows > (1 << 20)) return fail(SAT_ERR_INVALID, "box rows must be in [0, 2^20]");
    g_box_rb.store(rows, std::memory_order_relaxed);
    return SAT_OK;
}

int sat_debug_set_tag_space(uint64_t space) {
    if (space == 0) space = 1ull << 30;
    if (space < 2 || space > (1ull << 30)) return fail(SAT_ERR_INVALID, "tag space must be in [2, 2^30]");
    g_tag_space.store(space, std::memory_order_relaxed);
    return SAT_OK;
}

int sat_release_workspace(void* stream) {
    int dev;
    CUDA_TRY(cudaGetDevice(&dev));
    Workspace* w = nullptr;
    {
        std::lock_guard<std::mutex> lk(g_mu);
        auto it = g_ws.find({dev, stream});
        if (it == g_ws.end()) return SAT_OK;
        w = it->second;
        g_ws.erase(it);
    }
    // the stream's queued work may still use the buffers
    CUDA_TRY(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
    for (Buf* b : {&w->desc, &w->lseg, &w->ticket, &w->bt, &w->rs, &w->lx, &w->lsum, &w->topx, &w->lb,
                   &w->tr, &w->box, &w->part, &w->cnt, &w->bticket, &w->order, &w->shard, &w->din, &w->dout})
        free_buf(*b);
    for (void* p : w->retired) cudaFree(p);
    if (w->cstream_in) cudaStreamDestroy(w->cstream_in);
    if (w->cstream_out) cudaStreamDestroy(w->cstream_out);
    if (t_ws == w) t_ws = nullptr;
    delete w;
    return SAT_OK;
}

int sat_last_launch_count(void) { return t_launches; }
int sat_last_tile_rows(void) { return t_th; }
int sat_last_grid(void) { return t_grid; }
int sat_last_lookback_group(void) { return t_hg; }
double sat_last_r_effective(void) { return t_r; }

const char* sat_strerror(int status) {
    switch (status) {
        case SAT_OK: return "ok";
        case SAT_ERR_INVALID: return "invalid argument";
        case SAT_ERR_UNSUPPORTED: return "unsupported";
        case SAT_ERR_NOMEM: return "out of device memory";
        case SAT_ERR_CUDA: return "CUDA error";
        case SAT_ERR_COMM: return "communication error";
    }
    return "unknown status";
}

const char* sat_last_error(void) { return t_err.c_str(); }
int sat_abi_version(void) { return SAT_ABI_VERSION; }

}  // extern "C"
