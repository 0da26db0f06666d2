/*
 * sat.h -- libsat: B200 (sm_100a) summed area tables.  C ABI.
 *
 * The operation (Kasagi, Nakano, Ito, "Parallel Algorithms for the Summed Area
 * Table on the Asynchronous Hierarchical Memory Machine, with GPU
 * implementations", ICPP 2014; /root/reference/PAPER.md):
 *
 *   P:L187-L193 (Sec. I, Fig. 3): for an n x m matrix a the summed area table
 *   is the n x m matrix b with  b[i][j] = sum_{0<=k<=i, 0<=l<=j} a[k][l]
 *   (inclusive, 0-indexed), i.e. column-wise prefix-sums followed by row-wise
 *   prefix-sums.
 *
 * Conventions shared by every entry point:
 *   - Matrices are row-major and contiguous: element (i, j) of image b lives at
 *     index (b*rows + i)*cols + j.  Input and output have the same dtype.
 *   - All data pointers are DEVICE pointers owned by the caller (e.g. a torch
 *     tensor's data_ptr()), except sat_compute_host() which takes host pointers.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *     Every call is asynchronous on `stream` unless stated otherwise.
 *   - SAT_INT32 is computed in uint32 arithmetic, i.e. the result is exact
 *     modulo 2^32 (two's-complement wrap), bit-identical for every variant,
 *     tile shape and sharding.  SAT_FLOAT32 uses IEEE fp32 adds (round to
 *     nearest, no FTZ); its summation order differs between variants and may
 *     differ between runs (the look-back takes whichever predecessor state it
 *     finds first); every order stays within the documented 1e-5 max relative
 *     error for inputs in [0, 1).  SAT_FLOAT64 (the
 *     paper's "double (64-bit)" precision) uses IEEE fp64 adds with
 *     the same ordering caveats; for inputs k*2^-24 every partial sum below
 *     2^29 is exact, so those results are unique.  Float64 takes tile_rows
 *     16, 32 or 64 and needs 8-byte aligned pointers; the TMA path needs
 *     16-byte aligned pointers and cols % 4 == 0 (as for 4-byte types).
 *   - in == out (exact aliasing) is allowed for every entry point that takes
 *     both; a partial overlap returns SAT_ERR_INVALID.
 *   - rows == 0 or cols == 0 (or batch == 0) is a no-op returning SAT_OK.
 *   - Validation errors are returned synchronously and nothing is launched.
 *     Faults inside kernels surface as SAT_ERR_CUDA at this or a later call or
 *     at the caller's next synchronisation.  No C++ exception crosses the ABI.
 *     sat_last_error() returns a thread-local description of the last error.
 *   - The library keeps a per-(device, stream) workspace (look-back
 *     descriptors, a ticket counter, 2R1W carry buffers), grown on demand and
 *     never memset per call (descriptors carry per-launch tags).  Calls that
 *     share a stream are serialised by the stream; do not issue calls on two
 *     threads with the same stream concurrently.
 */
#ifndef LIBSAT_SAT_H
#define LIBSAT_SAT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SAT_ABI_VERSION 2

typedef enum { SAT_INT32 = 0, SAT_FLOAT32 = 1, SAT_FLOAT64 = 2,
               SAT_UINT8 = 3 /* input only: sat_compute_widening, sat_box_filter */ } sat_dtype;

/* Variants (Table I / Secs. IV-VII):
 *   SAT_2R2W        column-wise prefix pass then row-wise prefix pass, each a
 *                   full read+write of the matrix (Sec. IV, P:L847-L945,
 *                   Lemma 2).  The paper's row pass is strided; ours is
 *                   coalesced with the same byte count (R6).
 *   SAT_2R1W        Step 1 tile reductions (1R), Step 2 carry scans (small),
 *                   Step 3 re-read + carries + tile SAT (1R+1W) (Sec. V,
 *                   P:L1059-L1137, Lemma 4).
 *   SAT_1R1W        the hot path: one read and one write per element (Sec. VI,
 *                   P:L2151-L2163, Theorem 6), as one launch with a decoupled
 *                   look-back instead of 2n/w-1 stage launches.
 *   SAT_1PLUSR_R1W  2R1W on the top-left tile triangle A, 1R1W on the middle
 *                   band C, 2R1W on the bottom-right triangle B (Sec. VII,
 *                   P:L2289-L2355, Theorem 7); r from sat_options (0.25 =
 *                   the paper's 1.25R1W).
 *   SAT_4R4W        column-wise prefix pass, transpose, column-wise prefix
 *                   pass, transpose: four coalesced read+write passes (Sec. IV,
 *                   P:L1081-L1085, Lemma 3).  Needs a rows*cols*4-byte
 *                   workspace (allocated on first use per stream).
 *   SAT_4R1W        Formula (1) b[i][j] = a[i][j] + b[i-1][j] + b[i][j-1]
 *                   - b[i-1][j-1] one anti-diagonal per launch, rows+cols-1
 *                   launches (Sec. VI, Lemma 5).  Float32 loses
 *                   accuracy to the subtraction (R16); batch <= 65535.
 */
typedef enum { SAT_2R2W = 0, SAT_2R1W = 1, SAT_1R1W = 2, SAT_1PLUSR_R1W = 3,
               SAT_4R4W = 4, SAT_4R1W = 5 } sat_variant;

typedef enum {
    SAT_OK = 0,
    SAT_ERR_INVALID = -1,      /* bad pointer / size / enum / overlap */
    SAT_ERR_UNSUPPORTED = -2,  /* valid but not implemented (e.g. seeded batch) */
    SAT_ERR_NOMEM = -3,        /* workspace allocation failed */
    SAT_ERR_CUDA = -4,         /* a CUDA runtime/driver call failed */
    SAT_ERR_COMM = -5          /* the all-gather callback returned nonzero */
} sat_status;

typedef struct sat_options {
    double r;            /* SAT_1PLUSR_R1W: target fraction of tiles done by 2R1W
                            (0..1, default 0.25); the realised value is the tile
                            count ratio, see sat_last_r_effective() */
    int tile_rows;       /* 1R1W-family band height TH in {16, 32, 64, 128}
                            (float64: 16, 32, 64; uint8 input: 64, 128); 0 =
                            automatic (1R1W takes 128 once its
                            bands fill half the SMs, else 32 from 1536 rows,
                            else 16).  A height without an instantiated
                            configuration is rounded down to one that has it
                            (sat_last_tile_rows() reports the height used). */
    int force_generic;   /* 1 = use the non-TMA load/store path (tests) */
    int jitter;          /* stress tests: random delay (ns) before descriptor
                            publication, to shuffle the look-back; 0 = off */
    int segments;        /* 1R1W band segments: 0 =
                            automatic, n >= 1 = cut every band into n column
                            segments (tests) */
    int lookback_group;  /* look-back over bands: 0 =
                            automatic, -1 = flat (band by band), n >= 2 =
                            hierarchical: the last band of every group of n
                            bands also publishes the group's sums, and a walk
                            visits its own group band by band, then one word
                            per group above.  Same results either way. */
    int reserved[2];     /* must be 0 */
} sat_options;

/* Fill *opt with defaults (r = 0.25, automatic tile, TMA when eligible). */
void sat_options_init(sat_options *opt);

/* Stream capture (CUDA graphs) is supported by every entry point that
 * launches the band kernel on a device stream, except
 * sat_compute_sharded_fused (its exchange epoch is host-assigned) and
 * sat_compute_host (it synchronizes), which return SAT_ERR_UNSUPPORTED under
 * capture.  Requirement: one eager call of
 * the same shape/variant on the same stream first (a captured call cannot
 * allocate its workspace; otherwise SAT_ERR_UNSUPPORTED, "warm workspace").
 * From the first capture on, that stream's launches take their look-back
 * ticket base from the device (one extra small kernel per band launch,
 * DESIGN.md Sec. 4), so replays and later eager calls stay correct.
 * The captured launches keep using the capture stream's workspace
 * (descriptors, ticket): replays of graphs captured on one stream, and eager
 * calls on that stream, must not run concurrently with each other (replay
 * them in stream order, as with any graph that owns scratch memory). */

/* out = SAT(in) for one rows x cols matrix.  variant: sat_variant. */
int sat_compute(const void *in, void *out, int64_t rows, int64_t cols,
                int dtype, int variant, void *stream);

/* As sat_compute with options (NULL = defaults). */
int sat_compute_ex(const void *in, void *out, int64_t rows, int64_t cols,
                   int dtype, int variant, const sat_options *opt, void *stream);

/* `batch` independent rows x cols matrices stored back to back (the
 * data-parallel image workload, BASELINE.json config 5).  One launch for the
 * whole batch. */
int sat_compute_batched(const void *in, void *out, int64_t batch, int64_t rows,
                        int64_t cols, int dtype, int variant, const sat_options *opt,
                        void *stream);

/* Widening 1R1W: in holds in_dtype elements, out gets
 * the SAT in `dtype`, the input widened on load inside the kernel (no extra
 * pass).  Pairs: (SAT_UINT8 -> SAT_INT32) = the classic integral image of
 * 8-bit pixels, exact in uint32 arithmetic (1 + 4 bytes per pixel moved);
 * (SAT_FLOAT32 -> SAT_FLOAT64) = a float integral image in the paper's
 * precision (4 + 8 bytes); same-type pairs behave as sat_compute_batched with
 * SAT_1R1W.  batch x rows x cols, back to back.  in == out is invalid for a
 * widening pair.  TMA path needs 16-B aligned pointers and cols % 16 == 0
 * (uint8) or cols % 4 == 0; otherwise the generic path runs.  tile_rows: 64 or
 * 128 for uint8 input, 16/32/64/128 for float32 -> float64 (128: 64-column
 * chunks, as plain float64). */
int sat_compute_widening(const void *in, int in_dtype, void *out, int dtype,
                         int64_t batch, int64_t rows, int64_t cols,
                         const sat_options *opt, void *stream);

/* Box filter (the SAT's use, "the sum of any rectangular area
 * in O(1)"): out[b][i][j] = sum of in[b][k][l] over
 * |k - i| <= rr, |l - j| <= rc, clipped to the image; the four-corner SAT
 * formula with uint32 sums for SAT_UINT8/SAT_INT32 input and float64 sums for
 * SAT_FLOAT32/SAT_FLOAT64 input.  One launch, the SAT never in HBM, when out
 * does not alias in: uint8 / int32 / float32 input with
 * rr <= 8, rc <= 63 and 8-B (uint8, cols % 8 == 0) / 16-B (4-byte types,
 * cols % 4 == 0) aligned rows takes the column-walk kernel (row prefix sums
 * differenced, a running vertical window sum); other TMA-addressable cases with rc <= 127 and
 * 2 rr <= 32 (uint8/int32) or 16 (float32) the band kernel with the local SAT
 * in shared memory.  Otherwise (in place, larger radii, float64 input,
 * unaligned rows) a widening 1R1W SAT goes to a library workspace and a second
 * kernel does four SAT reads per output element.  out_dtype: SAT_INT32 for
 * integer input (sums mod 2^32), SAT_FLOAT32 or SAT_FLOAT64 for float input.
 * normalize != 0 divides by the clipped window's element count (box mean;
 * float input only).  rr, rc >= 0 (radii beyond the image are clamped);
 * batch <= 65535.  Bytes moved per pixel: in x (1 + halo rows) + out for the
 * one-launch paths, in + 2 x sum + out for the two-pass path. */
int sat_box_filter(const void *in, int in_dtype, void *out, int out_dtype,
                   int64_t batch, int64_t rows, int64_t cols, int rr, int rc,
                   int normalize, void *stream);

/* Rectangle sums from a SAT: for q < nrects, with
 * rects[5q .. 5q+4] = (image, r0, c0, r1, c1) (device int32, inclusive
 * bounds), out[q] = sum of the rectangle = S[r1][c1] - S[r0-1][c1]
 * - S[r1][c0-1] + S[r0-1][c0-1].  Bounds are clipped to the matrix; an empty
 * rectangle or an image index outside [0, batch) gives 0.  sat, out: device,
 * `dtype` elements (uint32 arithmetic for SAT_INT32). */
int sat_rect_sums(const void *sat, int dtype, int64_t batch, int64_t rows, int64_t cols,
                  const int32_t *rects, int64_t nrects, void *out, void *stream);

/* Seeded 1R1W: the rows x cols matrix is a strip of a taller matrix and
 * carry_row[j] (device, cols entries, same dtype) is the column sum of
 * everything above the strip in column j.  Result: the strip's rows of the
 * full matrix's SAT.  carry_row == NULL is the unseeded case.  One launch:
 * band 0 adds the carry to the strip's first input row before its row scan
 * (SAT([c; a]) restricted to a's rows), so no carry-prefix pass runs. */
int sat_compute_seeded(const void *in, void *out, int64_t rows, int64_t cols,
                       int dtype, const void *carry_row, void *stream);

/* As sat_compute_seeded with carry_row[j] = sum_{q < nvec} vectors[q*stride + j]
 * (q ascending; stride in elements, >= cols when nvec > 1): the row-strip
 * sharded mode passes the all-gathered column totals of all ranks and its rank
 * as nvec, so the exclusive scan over ranks happens inside the SAT kernel. */
int sat_compute_seeded_sum(const void *in, void *out, int64_t rows, int64_t cols,
                           int dtype, const void *vectors, int64_t nvec, int64_t stride,
                           void *stream);

/* As sat_compute_seeded, but sat_row[j] is the SAT row just above the strip
 * (the last SAT row of the strip above), not the column sums. */
int sat_compute_seeded_satrow(const void *in, void *out, int64_t rows, int64_t cols,
                              int dtype, const void *sat_row, void *stream);

/* ---- Fused peer exchange ----
 * The sharded mode without a collective call and with two launches per rank:
 * rank p's column-totals kernel (one launch) ends by storing its totals
 * straight into slot p of every higher rank's "mailbox" (peer memory over
 * NVLink, e.g. IPC-mapped) and raising a flag there (st.release.sys); rank
 * p's SAT kernel (one launch) waits in band 0 for the flags of ranks < p
 * (ld.acquire.sys), adds the sum of their slots in rank order (the exclusive
 * scan) to its first input row, and acknowledges once band 0 has read them.
 * Mailboxes are double-buffered by call parity with acknowledgements, so
 * consecutive calls need no barrier.  All ranks must make the same sequence of
 * calls.  Results are bit-identical to sat_compute_sharded (int32).
 *
 * sat_exchange_mailbox_bytes: size of one rank's mailbox.
 * sat_exchange_create: rank of nranks (<= 16); `mailbox` = this rank's own
 *   mailbox (device, 256-B aligned, zeroed here); peers[q] = rank q's mailbox
 *   as addressable from this rank's device (peers[rank] == mailbox).  The
 *   caller owns the memory and keeps it alive until sat_exchange_destroy.
 * sat_compute_sharded_fused: as sat_compute_sharded for this rank's strip. */
size_t sat_exchange_mailbox_bytes(int64_t cols, int nranks, int dtype);
int sat_exchange_create(void **exchange, int rank, int nranks, int64_t cols, int dtype,
                        void *mailbox, void *const *peers);
int sat_exchange_destroy(void *exchange);
int sat_compute_sharded_fused(const void *in_strip, void *out_strip, int64_t strip_rows,
                              void *exchange, void *stream);

/* CUDA IPC helpers for the mailboxes of other processes: a 64-byte handle of
 * a device allocation, and its mapping into this process (peer access over
 * NVLink enabled lazily). */
int sat_ipc_get_handle(const void *dev_ptr, void *handle64);
int sat_ipc_open(const void *handle64, void **dev_ptr);
int sat_ipc_close(void *dev_ptr);

/* totals[j] = sum_i in[i][j] (device, cols entries).  Deterministic order. */
int sat_column_totals(const void *in, void *totals, int64_t rows, int64_t cols,
                      int dtype, void *stream);

/* carry_row[j] = sum_{q < rank} gathered[q][j]; gathered is nranks x cols
 * (device), q ascending. */
int sat_rank_exscan(const void *gathered, void *carry_row, int64_t nranks,
                    int64_t cols, int rank, int dtype, void *stream);

/* All-gather callback for the sharded mode: gather `bytes` from every rank's
 * `send` into `recv` (rank-major, nranks * bytes), enqueued on or completed
 * before work on `stream`.  Return 0 on success. */
typedef int (*sat_allgather_fn)(void *ctx, const void *send, void *recv,
                                size_t bytes, void *stream);

typedef struct sat_shard_stats {
    int64_t strip_bytes_read;     /* SAT pass: rows*cols*eb */
    int64_t strip_bytes_written;  /* SAT pass: rows*cols*eb */
    int64_t extra_bytes_read;     /* column-totals pass (0 on the last rank) */
    int64_t allgather_bytes;      /* bytes received by this rank */
} sat_shard_stats;

/* Row-strip sharded SAT (north star (3)): this rank holds strip `rank` of
 * `nranks` consecutive row strips of one matrix (strips may have different
 * heights; every rank passes the same cols).  Steps: column totals of the
 * strip (skipped on the last rank, whose totals nobody needs -- it sends
 * zeros), all-gather through `allgather`, seeded 1R1W whose band 0 sums the
 * gathered totals of ranks < rank (the exclusive scan, in the SAT kernel).
 * Two launches per rank + the callback.  `workspace` is a caller-owned device buffer of at least
 * sat_sharded_workspace_bytes(cols, nranks, dtype) bytes (NULL = library
 * allocated).  stats may be NULL. */
int sat_compute_sharded(const void *in_strip, void *out_strip, int64_t strip_rows,
                        int64_t cols, int dtype, int rank, int nranks,
                        sat_allgather_fn allgather, void *comm_ctx, void *workspace,
                        void *stream, sat_shard_stats *stats);
size_t sat_sharded_workspace_bytes(int64_t cols, int nranks, int dtype);

/* As sat_compute_sharded with a variant: SAT_1R1W (the seeded band kernel) or
 * SAT_2R2W (the seed enters the column pass's first row; 2 x the strip bytes
 * in stats).  Other variants: SAT_ERR_UNSUPPORTED (their carry passes take no
 * seed). */
int sat_compute_sharded_ex(const void *in_strip, void *out_strip, int64_t strip_rows,
                           int64_t cols, int dtype, int variant, int rank, int nranks,
                           sat_allgather_fn allgather, void *comm_ctx, void *workspace,
                           void *stream, sat_shard_stats *stats);

/* In-library NCCL for the sharded mode (north star (3): the all-gather of the
 * strips' column totals over NVLink / NVSwitch).  libnccl.so.2 is loaded on
 * first use (dlopen; a copy already in the process, e.g. PyTorch's, is
 * shared); without it these return SAT_ERR_UNSUPPORTED.
 * sat_nccl_unique_id: 128 bytes for rank 0 to share out of band.
 * sat_nccl_comm_create: this process's rank of nranks on the current device
 *   (collective: every rank calls it with the same id); *comm is an opaque
 *   ncclComm_t, freed by sat_nccl_comm_destroy.
 * sat_compute_sharded_nccl: sat_compute_sharded_ex with rank / nranks taken
 *   from the communicator and the all-gather done by ncclAllGather on
 *   `stream` (NCCL errors: SAT_ERR_COMM). */
int sat_nccl_unique_id(void *id128);
int sat_nccl_comm_create(void **comm, const void *id128, int rank, int nranks);
int sat_nccl_comm_destroy(void *comm);
int sat_compute_sharded_nccl(const void *in_strip, void *out_strip, int64_t strip_rows,
                             int64_t cols, int dtype, int variant, void *comm,
                             void *workspace, void *stream, sat_shard_stats *stats);

/* End to end from HOST memory: copies in_host (rows*cols elements) to the
 * device, computes the SAT with `variant`, copies it back to out_host, and
 * synchronises `stream` before returning.  Pinned host buffers overlap the
 * copies with compute (the matrix is streamed in row strips, each seeded with
 * the SAT row above it); pageable buffers work but are slower. */
int sat_compute_host(const void *in_host, void *out_host, int64_t rows, int64_t cols,
                     int dtype, int variant, void *stream);

/* Debug/profiling (builds with SAT_DEBUG=1 only; SAT_ERR_UNSUPPORTED
 * otherwise): the next 1R1W-family band launch on this thread records,
 * per (band, chunk) of TH x 128 elements, eight 64-bit globaltimer stamps
 * (ns) into dev_buf[(band*nchunks + chunk)*8 + e]: e=0 tile data arrived,
 * e=1 band-local reductions done, e=2 look-back done (bits 48..55 = look-
 * back hops, 56..63 = polls of unpublished descriptors), e=3 tile store
 * issued, e=4 tile load issued, e=5 the store's smem read completed, e=6
 * finish (carry injection) starts, e=7 unused.  dev_buf (device, caller-owned) must hold
 * ceil(rows/TH)*batch*ceil(cols/128)*64 bytes; NULL disarms. */
int sat_debug_trace(void *dev_buf);

/* Watchdog diagnostics: record, in host-mapped memory, what every spinning warp waits on
 * once a wait exceeds half the 4-s watchdog (before the kernel traps);
 * sat_debug_diag_dump prints the records to stderr (also after a failed
 * launch) and returns their number. */
int sat_debug_diag_enable(void);
int sat_debug_diag_dump(void);

/* Free the library workspace of `stream` on the current device (look-back
 * descriptors, ticket, carry buffers, and buffers retired after a graph
 * capture).  Synchronizes the stream first.  CUDA graphs captured on that
 * stream must not be replayed afterwards.  The next call on the stream
 * allocates a fresh workspace. */
int sat_release_workspace(void *stream);

/* Tests only: shrink the look-back tag space (default and maximum 2^30;
 * 0 restores the default) so the tag-exhaustion paths run. */
int sat_debug_set_tag_space(uint64_t space);

/* Tests / tuning only: output rows per unit of the column-walk box filter
 * (DESIGN.md Sec. 4.12); 0 restores the automatic choice. */
int sat_debug_set_box_rows(int rows);

/* Number of kernels launched by the last successful call on this thread. */
int sat_last_launch_count(void);
/* Band height used by the last 1R1W-family call on this thread. */
int sat_last_tile_rows(void);
/* Grid size (persistent CTAs) of the last band-kernel launch on this thread. */
int sat_last_grid(void);
/* Look-back group size of the last band-kernel launch on this thread (0 =
 * flat walk; sat_options.lookback_group). */
int sat_last_lookback_group(void);
/* Realised r of the last SAT_1PLUSR_R1W call on this thread. */
double sat_last_r_effective(void);

const char *sat_strerror(int status);
const char *sat_last_error(void);
int sat_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* LIBSAT_SAT_H */
