// Probe: how fast can a persistent 1-CTA-per-SM TMA tile pipeline copy an n x n fp32 matrix on B200, as
// a function of tile height and stage count?  (The SAT kernel's data path without the SAT.)  Also
// reports the mean TMA load latency (issue -> mbarrier complete) seen by the loader.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC tma_copy.cu -o libtmacopy.so -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

namespace {

__device__ __forceinline__ uint32_t sa(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void minit(uint64_t* b, uint32_t c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void mexpect(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void marrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(b)) : "memory");
}
__device__ __forceinline__ bool mtest(uint64_t* b, uint32_t ph) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n}"
                 : "=r"(ok) : "r"(sa(b)), "r"(ph) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mwait(uint64_t* b, uint32_t ph) {
    while (!mtest(b, ph)) {}
}

template <int TR, int STAGES, int TC>
__global__ void __launch_bounds__(64, 1) copy_kernel(const __grid_constant__ CUtensorMap mi,
                                                     const __grid_constant__ CUtensorMap mo,
                                                     const __grid_constant__ CUtensorMap mo32, int R, int C,
                                                     unsigned long long* lat, int split_store) {
    extern __shared__ __align__(1024) unsigned char raw[];
    float* stage = reinterpret_cast<float*>(raw);
    __shared__ uint64_t full[STAGES], empty[STAGES];
    __shared__ long long issued[STAGES];
    constexpr uint32_t kBytes = TR * TC * 4;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) { minit(&full[s], 1); minit(&empty[s], 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int ntiles = R * C;
    if (warp == 0 && lane == 0) {
        unsigned long long sum = 0, cnt = 0;
        int k = 0;
        const int per = (ntiles + gridDim.x - 1) / gridDim.x;
        const bool chunk = (split_store & 2) != 0;
        for (int i = 0;; ++i, ++k) {
            const int t = chunk ? blockIdx.x * per + i : blockIdx.x + i * gridDim.x;
            if ((chunk && i >= per) || t >= ntiles) break;
            const int s = k % STAGES;
            if (k >= STAGES) mwait(&empty[s], ((k / STAGES) & 1) ^ 1);
            mexpect(&full[s], kBytes);
            issued[s] = clock64();
            const int I = t / C, J = t % C;
            asm volatile(
                "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                ::"r"(sa(stage + s * TR * TC)), "l"(&mi), "r"(J * TC), "r"(I * TR), "r"(sa(&full[s]))
                : "memory");
        }
        (void)sum; (void)cnt;
    } else if (warp == 1 && lane == 0) {
        unsigned long long sum = 0, cnt = 0;
        int k = 0;
        const int per = (ntiles + gridDim.x - 1) / gridDim.x;
        const bool chunk = (split_store & 2) != 0;
        for (int i = 0;; ++i, ++k) {
            const int t = chunk ? blockIdx.x * per + i : blockIdx.x + i * gridDim.x;
            if ((chunk && i >= per) || t >= ntiles) break;
            const int s = k % STAGES;
            mwait(&full[s], (k / STAGES) & 1);
            sum += clock64() - issued[s];
            ++cnt;
            const int I = t / C, J = t % C;
            if (split_store & 1) {
                for (int h = 0; h < TR; h += 32)
                    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                                 ::"l"(&mo32), "r"(J * TC), "r"(I * TR + h), "r"(sa(stage + s * TR * TC + h * TC)) : "memory");
            } else {
                asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                             ::"l"(&mo), "r"(J * TC), "r"(I * TR), "r"(sa(stage + s * TR * TC)) : "memory");
            }
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            marrive(&empty[s]);
        }
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
        atomicAdd(&lat[0], sum);
        atomicAdd(&lat[1], cnt);
    }
}

__global__ void __launch_bounds__(512) ldg_copy(const float4* __restrict__ src, float4* __restrict__ dst, long long n4) {
    for (long long i = blockIdx.x * 512LL + threadIdx.x; i < n4; i += 512LL * gridDim.x) {
        const float4 v = __ldcs(src + i);
        __stcs(dst + i, v);
    }
}

__global__ void __launch_bounds__(512) ldg_copy4(const float4* __restrict__ src, float4* __restrict__ dst, long long n4) {
    const long long stride = 512LL * gridDim.x;
    long long i = blockIdx.x * 512LL + threadIdx.x;
    for (; i + 3 * stride < n4; i += 4 * stride) {
        float4 v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) v[u] = __ldcs(src + i + u * stride);
#pragma unroll
        for (int u = 0; u < 4; ++u) __stcs(dst + i + u * stride, v[u]);
    }
    for (; i < n4; i += stride) __stcs(dst + i, __ldcs(src + i));
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int make_map(CUtensorMap* m, void* p, int n, int tr, int tc) {
    static EncodeFn enc = nullptr;
    if (!enc) {
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", reinterpret_cast<void**>(&enc), cudaEnableDefault, &q) !=
            cudaSuccess)
            return -1;
    }
    cuuint64_t dims[2] = {static_cast<cuuint64_t>(n), static_cast<cuuint64_t>(n)};
    cuuint64_t strides[1] = {static_cast<cuuint64_t>(n) * 4};
    cuuint32_t box[2] = {static_cast<cuuint32_t>(tc), static_cast<cuuint32_t>(tr)};
    cuuint32_t es[2] = {1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, p, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) ==
                   CUDA_SUCCESS
               ? 0
               : -2;
}

template <int TR, int ST, int TC>
int run(const float* src, float* dst, int n, int ctas, int reps, int split, float* ms, double* lat_cyc) {
    CUtensorMap mi, mo, mo32;
    if (make_map(&mi, const_cast<float*>(src), n, TR, TC) || make_map(&mo, dst, n, TR, TC) || make_map(&mo32, dst, n, 32, TC))
        return -3;
    const size_t smem = static_cast<size_t>(ST) * TR * TC * 4;
    auto k = copy_kernel<TR, ST, TC>;
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem)) != cudaSuccess)
        return -4;
    unsigned long long* lat;
    cudaMalloc(&lat, 16);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int w = 0; w < 2; ++w) k<<<ctas, 64, smem>>>(mi, mo, mo32, n / TR, n / TC, lat, split);
    cudaMemset(lat, 0, 16);
    cudaEventRecord(e0);
    for (int r = 0; r < reps; ++r) k<<<ctas, 64, smem>>>(mi, mo, mo32, n / TR, n / TC, lat, split);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(ms, e0, e1);
    *ms /= reps;
    unsigned long long h[2];
    cudaMemcpy(h, lat, 16, cudaMemcpyDeviceToHost);
    *lat_cyc = h[1] ? static_cast<double>(h[0]) / h[1] : 0.0;
    cudaFree(lat);
    const cudaError_t err = cudaGetLastError();
    return err == cudaSuccess ? 0 : -100 - static_cast<int>(err);
}

}  // namespace

extern "C" int ldg_copy_run(const float* src, float* dst, long long n, int blocks, int unroll, int reps, float* ms) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto go = [&]() {
        if (unroll) ldg_copy4<<<blocks, 512>>>(reinterpret_cast<const float4*>(src), reinterpret_cast<float4*>(dst), n / 4);
        else ldg_copy<<<blocks, 512>>>(reinterpret_cast<const float4*>(src), reinterpret_cast<float4*>(dst), n / 4);
    };
    go();
    cudaEventRecord(e0);
    for (int r = 0; r < reps; ++r) go();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(ms, e0, e1);
    *ms /= reps;
    return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

extern "C" int tma_copy(const float* src, float* dst, int n, int tr, int stages, int ctas, int reps, int split,
                        float* ms, double* lat_cyc, int tc) {
#define CASE(A, B, C) \
    if (tr == A && stages == B && tc == C) return run<A, B, C>(src, dst, n, ctas, reps, split, ms, lat_cyc);
    CASE(128, 3, 128) CASE(128, 2, 128) CASE(128, 1, 128) CASE(64, 6, 128) CASE(64, 4, 128) CASE(64, 3, 128)
    CASE(32, 12, 128) CASE(32, 6, 128) CASE(64, 3, 256) CASE(64, 2, 256) CASE(32, 6, 256) CASE(32, 4, 256)
    CASE(32, 3, 256) CASE(96, 2, 256) CASE(16, 12, 256) CASE(16, 6, 256)
#undef CASE
    return -1;
}
