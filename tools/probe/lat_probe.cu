// Loaded-latency probe: how long does an L2-resident ld.relaxed.gpu take while the other SMs stream
// HBM at full bandwidth?  (Design aid for the look-back; not part of libsat.)
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__global__ void stream_copy(const int4* __restrict__ a, int4* __restrict__ b, size_t n, int iters) {
    for (int it = 0; it < iters; ++it)
        for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
            b[i] = a[i];
}

__global__ void probe(const uint64_t* p, int n, long long* out, int stride) {
    long long tot = 0;
    uint64_t acc = 0;
    for (int i = 0; i < n; ++i) {
        const uint64_t* q = p + ((i * stride) & 4095) * 16;
        long long t0 = clock64();
        uint64_t v;
        asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(q) : "memory");
        acc += v;
        long long t1 = clock64();
        tot += t1 - t0;
    }
    if (threadIdx.x == 0) { out[0] = tot / n; out[1] = (long long)acc; }
}

extern "C" int run_probe(int load_sms, int iters, long long* idle_lat, long long* loaded_lat, float* copy_ms) {
    size_t n = (size_t)1 << 28;  // 4 GiB of int4
    int4 *a, *b;
    uint64_t* flags;
    long long* out;
    if (cudaMalloc(&a, n * 16) || cudaMalloc(&b, n * 16) || cudaMalloc(&flags, 4096 * 128) || cudaMalloc(&out, 64)) return 1;
    cudaMemset(flags, 0, 4096 * 128);
    cudaStream_t s1, s2;
    cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    probe<<<1, 32, 0, s2>>>(flags, 2000, out, 7);
    cudaStreamSynchronize(s2);
    probe<<<1, 32, 0, s2>>>(flags, 2000, out, 7);
    cudaStreamSynchronize(s2);
    cudaMemcpy(idle_lat, out, 8, cudaMemcpyDeviceToHost);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0, s1);
    stream_copy<<<load_sms * 4, 512, 0, s1>>>(a, b, n, iters);
    cudaEventRecord(e1, s1);
    probe<<<1, 32, 0, s2>>>(flags, 20000, out, 7);
    cudaStreamSynchronize(s2);
    cudaMemcpy(loaded_lat, out, 8, cudaMemcpyDeviceToHost);
    cudaStreamSynchronize(s1);
    cudaEventElapsedTime(copy_ms, e0, e1);
    cudaFree(a); cudaFree(b); cudaFree(flags); cudaFree(out);
    return (int)cudaGetLastError();
}

// Probe alone on `stream` (caller runs the load elsewhere): average latency of n polls, in cycles.
extern "C" int probe_async(void* flags, int n, long long* out_dev, void* stream) {
    probe<<<1, 32, 0, (cudaStream_t)stream>>>((const uint64_t*)flags, n, out_dev, 7);
    return (int)cudaGetLastError();
}
