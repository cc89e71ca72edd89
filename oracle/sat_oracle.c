/*
 * sat_oracle.c -- CPU ORACLE for the summed area table (TEST INFRASTRUCTURE ONLY).
 *
 * This file is test infrastructure.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load it.  The product path
 * (libsat) shares no code, header, table or helper with it and never calls it.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, cited as P:<line>):
 *
 *   SAT definition, P:44 (Sec. I.A):  b[i][j] = sum_{0<=i'<=i, 0<=j'<=j} a[i'][j'].
 *
 *   Method, P:46 and Figure 2, repeated at P:54 (Sec. I.B): "the SAT can be
 *   obtained by computing the column-wise prefix-sums and then the row-wise prefix-sums".
 *   The oracle is that sentence written out literally, one thread, no blocking:
 *       pass 1 (column-wise prefix sums):  c[i][j] = c[i-1][j] + a[i][j]
 *       pass 2 (row-wise prefix sums):     b[i][j] = b[i][j-1] + c[i][j]
 *   where each 1-D prefix sum is the sequential recurrence p[i] <- p[i-1] + p[i] of
 *   P:42 ("by executing p[i] <- p[i-1]+p[i] for all i in turn").
 *
 *   Layout: row-major, element a[i][j] at offset i*pitch + j (the paper has
 *   pitch = n; reading R3 generalises to any pitch >= cols).
 *
 *   Arithmetic (reading R1; the paper only says "4-byte float"):
 *     - int32 inputs: sums taken modulo 2^32 (uint32 wraparound), i.e. the exact
 *       integer SAT reduced mod 2^32;
 *     - fp32 inputs: sums taken in IEEE fp64 from the exactly-converted fp32 values,
 *       together with the SAT of |a| (absSAT) that scales the fp32 tolerance.
 *
 *   Streaming form (same two passes, one row at a time): keeps the running column
 *   vector c (pass 1 state) and emits row i of b as the row-wise prefix of c.  Used for
 *   matrices too large to hold twice in host memory and for per-rank strips.
 *
 *   Region sum S[U:D][L:R] of P:128-130 (Sec. III), by its double-sum definition; it
 *   is the building block of the per-tile sums of Table II (reconstructed, R5).
 *
 * Parity pins for every function here live in tests/test_oracle.py (brute force over
 * the P:44 definition, Figure 2 golden tables, rectangle formula P:48, closed forms,
 * invariants); DESIGN.md Sec. 3 lists the pin of each function, including
 * oracle_region_sum_f64 (test_region_sum_f64_against_fsum).  No function in this file
 * is "parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_API __attribute__((visibility("default")))

/* ---------------------------------------------------------------- in-memory, uint32 */

/* Pass 1: column-wise prefix sums, c[i][j] = c[i-1][j] + a[i][j] (mod 2^32). */
ORACLE_API void oracle_col_prefix_u32(const uint32_t* a, uint32_t* c, int64_t rows, int64_t cols,
                                      int64_t pitch) {
    for (int64_t j = 0; j < cols; ++j) {
        uint32_t run = 0;
        for (int64_t i = 0; i < rows; ++i) {
            run = run + a[i * pitch + j];
            c[i * pitch + j] = run;
        }
    }
}

/* Pass 2: row-wise prefix sums, b[i][j] = b[i][j-1] + c[i][j] (mod 2^32). */
ORACLE_API void oracle_row_prefix_u32(const uint32_t* c, uint32_t* b, int64_t rows, int64_t cols,
                                      int64_t pitch) {
    for (int64_t i = 0; i < rows; ++i) {
        uint32_t run = 0;
        for (int64_t j = 0; j < cols; ++j) {
            run = run + c[i * pitch + j];
            b[i * pitch + j] = run;
        }
    }
}

/* SAT = column-wise prefix sums, then row-wise prefix sums (Fig. 2).  b may equal a. */
ORACLE_API void oracle_sat_u32(const uint32_t* a, uint32_t* b, int64_t rows, int64_t cols,
                               int64_t pitch) {
    oracle_col_prefix_u32(a, b, rows, cols, pitch);
    oracle_row_prefix_u32(b, b, rows, cols, pitch);
}

/* ---------------------------------------------------------------- in-memory, fp64 */

/* The same two passes in fp64 from fp32 input (each fp32 value converts to fp64 exactly).
 * Also produces absSAT = SAT(|a|), the scale of the fp32 tolerance (R10).
 * b and absb are dense rows x cols (pitch = cols) fp64 arrays. */
ORACLE_API void oracle_sat_f32_f64(const float* a, double* b, double* absb, int64_t rows,
                                   int64_t cols, int64_t pitch) {
    /* pass 1: column-wise prefix sums */
    for (int64_t j = 0; j < cols; ++j) {
        double run = 0.0, arun = 0.0;
        for (int64_t i = 0; i < rows; ++i) {
            double x = (double)a[i * pitch + j];
            run = run + x;
            arun = arun + fabs(x);
            b[i * cols + j] = run;
            if (absb) absb[i * cols + j] = arun;
        }
    }
    /* pass 2: row-wise prefix sums */
    for (int64_t i = 0; i < rows; ++i) {
        double run = 0.0, arun = 0.0;
        for (int64_t j = 0; j < cols; ++j) {
            run = run + b[i * cols + j];
            b[i * cols + j] = run;
            if (absb) {
                arun = arun + absb[i * cols + j];
                absb[i * cols + j] = arun;
            }
        }
    }
}

/* The same two passes for fp64 input (used by the pins with exact-integer doubles). */
ORACLE_API void oracle_sat_f64(const double* a, double* b, int64_t rows, int64_t cols) {
    for (int64_t j = 0; j < cols; ++j) {
        double run = 0.0;
        for (int64_t i = 0; i < rows; ++i) {
            run = run + a[i * cols + j];
            b[i * cols + j] = run;
        }
    }
    for (int64_t i = 0; i < rows; ++i) {
        double run = 0.0;
        for (int64_t j = 0; j < cols; ++j) {
            run = run + b[i * cols + j];
            b[i * cols + j] = run;
        }
    }
}

/* ---------------------------------------------------------------- streaming form */

/* State of pass 1 (the running column-wise prefix sums c[i][*]) for one matrix. */
typedef struct {
    int64_t cols;
    int64_t row;      /* rows consumed so far */
    uint32_t* c_u32;  /* running column sums, uint32 */
    double* c_f64;    /* running column sums, fp64 */
    double* ca_f64;   /* running column sums of |a|, fp64 */
} oracle_stream_t;

ORACLE_API oracle_stream_t* oracle_stream_new(int64_t cols) {
    oracle_stream_t* s = (oracle_stream_t*)calloc(1, sizeof(oracle_stream_t));
    if (!s) return NULL;
    s->cols = cols;
    s->c_u32 = (uint32_t*)calloc((size_t)(cols > 0 ? cols : 1), sizeof(uint32_t));
    s->c_f64 = (double*)calloc((size_t)(cols > 0 ? cols : 1), sizeof(double));
    s->ca_f64 = (double*)calloc((size_t)(cols > 0 ? cols : 1), sizeof(double));
    if (!s->c_u32 || !s->c_f64 || !s->ca_f64) {
        free(s->c_u32); free(s->c_f64); free(s->ca_f64); free(s);
        return NULL;
    }
    return s;
}

ORACLE_API void oracle_stream_free(oracle_stream_t* s) {
    if (!s) return;
    free(s->c_u32); free(s->c_f64); free(s->ca_f64); free(s);
}

/* Copy out the running column sums c[row-1][*] (the strip carry of a rank whose strip
 * starts at global row `row`; the carry of the top strip is the zero vector). */
ORACLE_API void oracle_stream_colsums_u32(const oracle_stream_t* s, uint32_t* out) {
    memcpy(out, s->c_u32, (size_t)s->cols * sizeof(uint32_t));
}
ORACLE_API void oracle_stream_colsums_f64(const oracle_stream_t* s, double* out) {
    memcpy(out, s->c_f64, (size_t)s->cols * sizeof(double));
}

/* Consume `nrows` input rows (uint32, row stride `pitch`) and emit the SAT rows:
 * pass 1 updates c, pass 2 writes the row-wise prefix of c.  out may be NULL (skip). */
ORACLE_API void oracle_stream_rows_u32(oracle_stream_t* s, const uint32_t* a, uint32_t* out,
                                       int64_t nrows, int64_t pitch, int64_t out_pitch) {
    const int64_t cols = s->cols;
    for (int64_t r = 0; r < nrows; ++r) {
        const uint32_t* ar = a + r * pitch;
        for (int64_t j = 0; j < cols; ++j) s->c_u32[j] = s->c_u32[j] + ar[j];  /* pass 1 */
        if (out) {
            uint32_t* br = out + r * out_pitch;
            uint32_t run = 0;
            for (int64_t j = 0; j < cols; ++j) {                              /* pass 2 */
                run = run + s->c_u32[j];
                br[j] = run;
            }
        }
        s->row += 1;
    }
}

/* fp32 input rows -> fp64 SAT rows and fp64 absSAT rows (either output may be NULL). */
ORACLE_API void oracle_stream_rows_f32(oracle_stream_t* s, const float* a, double* out,
                                       double* absout, int64_t nrows, int64_t pitch,
                                       int64_t out_pitch) {
    const int64_t cols = s->cols;
    for (int64_t r = 0; r < nrows; ++r) {
        const float* ar = a + r * pitch;
        for (int64_t j = 0; j < cols; ++j) {                                  /* pass 1 */
            double x = (double)ar[j];
            s->c_f64[j] = s->c_f64[j] + x;
            s->ca_f64[j] = s->ca_f64[j] + fabs(x);
        }
        double run = 0.0, arun = 0.0;
        for (int64_t j = 0; j < cols; ++j) {                                  /* pass 2 */
            run = run + s->c_f64[j];
            arun = arun + s->ca_f64[j];
            if (out) out[r * out_pitch + j] = run;
            if (absout) absout[r * out_pitch + j] = arun;
        }
        s->row += 1;
    }
}

/* ---------------------------------------------------------------- region sums */

/* S[U:D][L:R] of P:128-130: sum of a[i'][j'] for U<=i'<=D, L<=j'<=R (mod 2^32).
 * Empty ranges (D<U or R<L) sum to 0; this is how the out-of-range aggregates
 * GRS(I,-1), GCS(-1,J), GS(-1,*) = 0 of DESIGN.md R5 arise. */
ORACLE_API uint32_t oracle_region_sum_u32(const uint32_t* a, int64_t pitch, int64_t U, int64_t D,
                                          int64_t L, int64_t R) {
    uint32_t s = 0;
    for (int64_t i = U; i <= D; ++i)
        for (int64_t j = L; j <= R; ++j) s = s + a[i * pitch + j];
    return s;
}

ORACLE_API double oracle_region_sum_f64(const float* a, int64_t pitch, int64_t U, int64_t D,
                                        int64_t L, int64_t R) {
    double s = 0.0;
    for (int64_t i = U; i <= D; ++i)
        for (int64_t j = L; j <= R; ++j) s = s + (double)a[i * pitch + j];
    return s;
}
