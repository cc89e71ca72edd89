// satgen_cuda.cu -- device side of the seeded counter-based input generator.
// Same function as satgen.c / satgen/__init__.py (see satgen.c for the definition);
// no SAT arithmetic here.  Used by bench.py and the GPU tests to create large inputs
// directly in HBM; tests/test_satgen_gpu.py checks it bit-for-bit against the host copy.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__device__ __forceinline__ uint32_t bits_of(uint64_t z, int dist) {
    switch (dist) {
        case 0: return (uint32_t)(z >> 32);
        case 1: return (uint32_t)(z >> 56);
        case 2: return (uint32_t)(z >> 62);
        case 3: return __float_as_uint(__fmul_rn((float)(z >> 40), 0x1p-24f));
        case 4: return __float_as_uint(__fsub_rn(__fmul_rn((float)(z >> 40), 0x1p-23f), 1.0f));
        case 5: return __float_as_uint((float)(z >> 62));
        default: return 0u;
    }
}

__global__ void fill_kernel(uint32_t* out, int64_t nrows, int64_t cols, int64_t pitch, int64_t row0,
                            uint64_t key, int dist) {
    const int64_t total = nrows * cols;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = t / cols, j = t - r * cols;
        const uint64_t idx = (uint64_t)(row0 + r) * (uint64_t)cols + (uint64_t)j;
        out[r * pitch + j] = bits_of(splitmix64(key + idx), dist);
    }
}

uint64_t host_splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

}  // namespace

// Fill rows [row0, row0+nrows) of the global matrix into device memory `out` (row stride
// `pitch` 32-bit words) on `stream`.  Returns a cudaError_t value (0 = success).
extern "C" __attribute__((visibility("default"))) int satgen_fill_device(
    void* out, int64_t nrows, int64_t cols, int64_t pitch, int64_t row0, uint64_t seed, int dist,
    void* stream) {
    if (nrows <= 0 || cols <= 0) return 0;
    const int threads = 256;
    int64_t blocks = (nrows * cols + threads - 1) / threads;
    if (blocks > 148 * 64) blocks = 148 * 64;
    fill_kernel<<<(unsigned)blocks, threads, 0, (cudaStream_t)stream>>>(
        (uint32_t*)out, nrows, cols, pitch, row0, host_splitmix64(seed), dist);
    return (int)cudaGetLastError();
}
