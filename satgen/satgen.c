/*
 * satgen.c -- seeded, counter-based synthetic input generator (host side).
 *
 * Shared by the oracle side (tests, cpu baseline) and the product side (bench inputs);
 * it contains none of the SAT arithmetic.  Element (i, j) of a matrix with `cols`
 * columns gets the counter idx = i*cols + j (global row index i, independent of pitch
 * and of which rank holds the row), and its 64 random bits are
 *     z = splitmix64(key + idx),   key = splitmix64(seed)
 * The device generator (satgen_cuda.cu) and the numpy generator (__init__.py)
 * implement exactly the same function; tests check all three agree bit for bit.
 *
 * Distributions:
 *   SATGEN_U32  : int32 bits = z >> 32                  (full 32-bit range, exercises wraparound)
 *   SATGEN_U8   : z >> 56                               (0..255, image intensities)
 *   SATGEN_U2   : z >> 62                               (0..3, exact fp32 regime)
 *   SATGEN_F01  : (z >> 40) * 2^-24                     (fp32 uniform [0,1), exact)
 *   SATGEN_FSYM : (z >> 40) * 2^-23 - 1                 (fp32 uniform [-1,1), exact)
 *   SATGEN_FU2  : (float)(z >> 62)                      (fp32 in {0,1,2,3})
 */
#include <stdint.h>

#define SATGEN_API __attribute__((visibility("default")))

enum { SATGEN_U32 = 0, SATGEN_U8 = 1, SATGEN_U2 = 2, SATGEN_F01 = 3, SATGEN_FSYM = 4, SATGEN_FU2 = 5 };

static inline uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

static inline uint32_t satgen_bits(uint64_t z, int dist) {
    union { float f; uint32_t u; } cv;
    switch (dist) {
        case SATGEN_U32: return (uint32_t)(z >> 32);
        case SATGEN_U8: return (uint32_t)(z >> 56);
        case SATGEN_U2: return (uint32_t)(z >> 62);
        case SATGEN_F01: cv.f = (float)(z >> 40) * 0x1p-24f; return cv.u;
        case SATGEN_FSYM: cv.f = (float)(z >> 40) * 0x1p-23f - 1.0f; return cv.u;
        case SATGEN_FU2: cv.f = (float)(z >> 62); return cv.u;
        default: return 0u;
    }
}

/* Fill rows [row0, row0+nrows) x [0, cols) of the global matrix into out (row stride pitch,
 * 32-bit words; the bits are int32 or fp32 depending on dist).  Pad words are untouched. */
SATGEN_API void satgen_fill_host(uint32_t* out, int64_t nrows, int64_t cols, int64_t pitch,
                                 int64_t row0, uint64_t seed, int dist) {
    const uint64_t key = splitmix64(seed);
    for (int64_t r = 0; r < nrows; ++r) {
        const uint64_t base = key + (uint64_t)(row0 + r) * (uint64_t)cols;
        uint32_t* o = out + r * pitch;
        for (int64_t j = 0; j < cols; ++j) o[j] = satgen_bits(splitmix64(base + (uint64_t)j), dist);
    }
}
