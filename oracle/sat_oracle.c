/*
 * sat_oracle.c -- plain, slow, single-threaded CPU oracle for the summed area
 * table (SAT).  TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or helper with the CUDA path (libsat).
 *
 * What it computes (Kasagi, Nakano, Ito, ICPP 2014; /root/reference/PAPER.md):
 *   P:L187-L193 (Sec. I, Fig. 3): the SAT b of an n x m matrix a is the matrix
 *   of the same size with b[i][j] = sum_{0<=k<=i, 0<=l<=j} a[k][l] (inclusive,
 *   pinned by Fig. 3: b[0][3] = a[0][3] = 1).  "the SAT can be obtained by
 *   computing the column-wise prefix-sums and the row-wise prefix-sums".
 *
 * Element types (reading R3): int32 input -> uint32 arithmetic
 * (wraps mod 2^32, defined behaviour); float32 input -> float64 accumulation.
 *
 * Formulations (all reach the same plain definition):
 *   oracle_sat_*        column-wise prefix then row-wise prefix, row-fused and
 *                       streaming (running column sums carried in `colsum`, so
 *                       a matrix can be fed strip by strip);
 *   oracle_sat_*_eq1    Formula (1), b[i][j] = a[i][j] + b[i-1][j] + b[i][j-1]
 *                       - b[i-1][j-1], evaluated in raster order = the paper's
 *                       4R1W(CPU) baseline; out-of-range b terms are 0
 *                       (reading R12).
 *   oracle_sat_*_2pass  2R2W(CPU): the whole column-wise prefix pass in raster
 *                       order, then the whole row-wise pass.
 *   oracle_sat_*_brute  the double sum written out, O(n^2 m^2), tiny inputs.
 *   oracle_sat_*_at     one element b[i][j] by the double sum (sampled parity at
 *                       full size).
 */
#include <stdint.h>
#include <stddef.h>

/* ---------------- uint32 (int32 input, wrapping) ---------------- */

/* Column-wise prefix-sums then row-wise prefix-sums, one row at a time.
 * colsum[j] holds sum_{k<i} a[k][j] on entry to row i (zero for a fresh
 * matrix; the caller passes it back to continue with the next strip). */
void oracle_sat_u32(const uint32_t *a, uint32_t *b, int64_t rows, int64_t cols,
                    uint32_t *colsum)
{
    for (int64_t i = 0; i < rows; ++i) {
        uint32_t s = 0;
        for (int64_t j = 0; j < cols; ++j) {
            colsum[j] += a[i * cols + j];   /* column-wise prefix-sum */
            s += colsum[j];                 /* row-wise prefix-sum of it */
            b[i * cols + j] = s;
        }
    }
}

/* Formula (1) in raster order.  prev_row (nullable) = SAT row just above
 * row 0 (b[-1][*]); NULL means zeros. */
void oracle_sat_u32_eq1(const uint32_t *a, uint32_t *b, int64_t rows, int64_t cols,
                        const uint32_t *prev_row)
{
    for (int64_t i = 0; i < rows; ++i) {
        const uint32_t *up = (i > 0) ? b + (i - 1) * cols : prev_row;
        for (int64_t j = 0; j < cols; ++j) {
            uint32_t v = a[i * cols + j];
            uint32_t b_up = up ? up[j] : 0u;
            uint32_t b_left = (j > 0) ? b[i * cols + j - 1] : 0u;
            uint32_t b_diag = (up && j > 0) ? up[j - 1] : 0u;
            b[i * cols + j] = v + b_up + b_left - b_diag;
        }
    }
}

/* 2R2W(CPU): column-wise pass over the whole matrix, then row-wise pass. */
void oracle_sat_u32_2pass(const uint32_t *a, uint32_t *b, int64_t rows, int64_t cols)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j)
            b[i * cols + j] = a[i * cols + j] + (i > 0 ? b[(i - 1) * cols + j] : 0u);
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 1; j < cols; ++j)
            b[i * cols + j] += b[i * cols + j - 1];
}

uint32_t oracle_sat_u32_at(const uint32_t *a, int64_t rows, int64_t cols,
                           int64_t i, int64_t j)
{
    (void)rows;
    uint32_t s = 0;
    for (int64_t k = 0; k <= i; ++k)
        for (int64_t l = 0; l <= j; ++l)
            s += a[k * cols + l];
    return s;
}

void oracle_sat_u32_brute(const uint32_t *a, uint32_t *b, int64_t rows, int64_t cols)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j)
            b[i * cols + j] = oracle_sat_u32_at(a, rows, cols, i, j);
}

/* ---------------- float32 input, float64 accumulation ---------------- */

void oracle_sat_f64(const float *a, double *b, int64_t rows, int64_t cols,
                    double *colsum)
{
    for (int64_t i = 0; i < rows; ++i) {
        double s = 0.0;
        for (int64_t j = 0; j < cols; ++j) {
            colsum[j] += (double)a[i * cols + j];
            s += colsum[j];
            b[i * cols + j] = s;
        }
    }
}

void oracle_sat_f64_eq1(const float *a, double *b, int64_t rows, int64_t cols,
                        const double *prev_row)
{
    for (int64_t i = 0; i < rows; ++i) {
        const double *up = (i > 0) ? b + (i - 1) * cols : prev_row;
        for (int64_t j = 0; j < cols; ++j) {
            double v = (double)a[i * cols + j];
            double b_up = up ? up[j] : 0.0;
            double b_left = (j > 0) ? b[i * cols + j - 1] : 0.0;
            double b_diag = (up && j > 0) ? up[j - 1] : 0.0;
            b[i * cols + j] = v + b_up + b_left - b_diag;
        }
    }
}

void oracle_sat_f64_2pass(const float *a, double *b, int64_t rows, int64_t cols)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j)
            b[i * cols + j] = (double)a[i * cols + j] + (i > 0 ? b[(i - 1) * cols + j] : 0.0);
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 1; j < cols; ++j)
            b[i * cols + j] += b[i * cols + j - 1];
}

double oracle_sat_f64_at(const float *a, int64_t rows, int64_t cols,
                         int64_t i, int64_t j)
{
    (void)rows;
    double s = 0.0;
    for (int64_t k = 0; k <= i; ++k)
        for (int64_t l = 0; l <= j; ++l)
            s += (double)a[k * cols + l];
    return s;
}

void oracle_sat_f64_brute(const float *a, double *b, int64_t rows, int64_t cols)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j)
            b[i * cols + j] = oracle_sat_f64_at(a, rows, cols, i, j);
}

/* ---------------- float64 input, float64 arithmetic (the paper's precision,
 * "double (64-bit) numbers") ---------------- */

void oracle_sat_d64(const double *a, double *b, int64_t rows, int64_t cols,
                    double *colsum)
{
    for (int64_t i = 0; i < rows; ++i) {
        double s = 0.0;
        for (int64_t j = 0; j < cols; ++j) {
            colsum[j] += a[i * cols + j];   /* column-wise prefix-sum */
            s += colsum[j];                 /* row-wise prefix-sum of it */
            b[i * cols + j] = s;
        }
    }
}

void oracle_sat_d64_eq1(const double *a, double *b, int64_t rows, int64_t cols,
                        const double *prev_row)
{
    for (int64_t i = 0; i < rows; ++i) {
        const double *up = (i > 0) ? b + (i - 1) * cols : prev_row;
        for (int64_t j = 0; j < cols; ++j) {
            double v = a[i * cols + j];
            double b_up = up ? up[j] : 0.0;
            double b_left = (j > 0) ? b[i * cols + j - 1] : 0.0;
            double b_diag = (up && j > 0) ? up[j - 1] : 0.0;
            b[i * cols + j] = v + b_up + b_left - b_diag;
        }
    }
}

void oracle_sat_d64_2pass(const double *a, double *b, int64_t rows, int64_t cols)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j)
            b[i * cols + j] = a[i * cols + j] + (i > 0 ? b[(i - 1) * cols + j] : 0.0);
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 1; j < cols; ++j)
            b[i * cols + j] += b[i * cols + j - 1];
}

double oracle_sat_d64_at(const double *a, int64_t rows, int64_t cols,
                         int64_t i, int64_t j)
{
    (void)rows;
    double s = 0.0;
    for (int64_t k = 0; k <= i; ++k)
        for (int64_t l = 0; l <= j; ++l)
            s += a[k * cols + l];
    return s;
}

void oracle_sat_d64_brute(const double *a, double *b, int64_t rows, int64_t cols)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j)
            b[i * cols + j] = oracle_sat_d64_at(a, rows, cols, i, j);
}

/* ---------------- box filter (the SAT's motivating use, P:L193, L221;
 * SURVEY 8(f2)) written as its plain definition: the sum of the input over
 * the (2*rr+1) x (2*rc+1) window centred on (i, j), clipped to the matrix.
 * O(rows * cols * window): test sizes only. ---------------- */

static int64_t lo_clip(int64_t x) { return x < 0 ? 0 : x; }
static int64_t hi_clip(int64_t x, int64_t n) { return x > n - 1 ? n - 1 : x; }

void oracle_box_u32(const uint32_t *a, uint32_t *out, int64_t rows, int64_t cols,
                    int64_t rr, int64_t rc)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j) {
            uint32_t s = 0;
            for (int64_t k = lo_clip(i - rr); k <= hi_clip(i + rr, rows); ++k)
                for (int64_t l = lo_clip(j - rc); l <= hi_clip(j + rc, cols); ++l)
                    s += a[k * cols + l];
            out[i * cols + j] = s;
        }
}

/* float32 input summed in float64 */
void oracle_box_f64(const float *a, double *out, int64_t rows, int64_t cols,
                    int64_t rr, int64_t rc)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j) {
            double s = 0.0;
            for (int64_t k = lo_clip(i - rr); k <= hi_clip(i + rr, rows); ++k)
                for (int64_t l = lo_clip(j - rc); l <= hi_clip(j + rc, cols); ++l)
                    s += (double)a[k * cols + l];
            out[i * cols + j] = s;
        }
}

void oracle_box_d64(const double *a, double *out, int64_t rows, int64_t cols,
                    int64_t rr, int64_t rc)
{
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j) {
            double s = 0.0;
            for (int64_t k = lo_clip(i - rr); k <= hi_clip(i + rr, rows); ++k)
                for (int64_t l = lo_clip(j - rc); l <= hi_clip(j + rc, cols); ++l)
                    s += a[k * cols + l];
            out[i * cols + j] = s;
        }
}
