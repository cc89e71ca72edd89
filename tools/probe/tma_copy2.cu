// Probe 2: copy ceiling of a persistent 1-CTA-per-SM TMA tile pipeline on B200 as a function of the
// tile SHAPE (contiguous bytes per tile row), stage count and the data path through the SM:
//   mode 0: TMA load -> stage -> TMA store from the same stage (pure DMA)
//   mode 1: TMA load -> stage -> 16 warps copy through registers into an output buffer -> TMA store
//           (the SAT kernel's data path, without the SAT)
// Tiles wider than 256 elements use a 3-D tensor map {256, TC/256, rows} so that one box row is TC
// contiguous elements.  Tile order: row-major (t -> (t / C, t % C)) or anti-diagonal bands.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC tma_copy2.cu -o libtmacopy2.so
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
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n}"
                 : "=r"(ok) : "r"(sa(b)), "r"(ph) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mwait(uint64_t* b, uint32_t ph) {
    while (!mtest(b, ph)) {}
}
__device__ __forceinline__ uint64_t pol_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

template <int TR, int TC>
__device__ __forceinline__ void load_tile(void* dst, const CUtensorMap* m, uint64_t* bar, int I, int J, uint64_t pol) {
    if constexpr (TC <= 256) {
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, "
            "%3}], [%4], %5;" ::"r"(sa(dst)),
            "l"(m), "r"(J * TC), "r"(I * TR), "r"(sa(bar)), "l"(pol)
            : "memory");
    } else {
        asm volatile(
            "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, "
            "%3, %4}], [%5], %6;" ::"r"(sa(dst)),
            "l"(m), "r"(0), "r"(J * (TC / 256)), "r"(I * TR), "r"(sa(bar)), "l"(pol)
            : "memory");
    }
}
template <int TR, int TC>
__device__ __forceinline__ void store_tile(const CUtensorMap* m, const void* src, int I, int J, uint64_t pol) {
    if constexpr (TC <= 256) {
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%1, %2}], [%3], %4;"
                     ::"l"(m), "r"(J * TC), "r"(I * TR), "r"(sa(src)), "l"(pol) : "memory");
    } else {
        asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%1, %2, %3}], [%4], %5;"
                     ::"l"(m), "r"(0), "r"(J * (TC / 256)), "r"(I * TR), "r"(sa(src)), "l"(pol) : "memory");
    }
}

__device__ __forceinline__ long long tri(long long k) { return k * (k + 1) / 2; }
__device__ __forceinline__ long long tri_inv(long long s) {
    long long k = static_cast<long long>((sqrt(8.0 * static_cast<double>(s) + 1.0) - 1.0) * 0.5);
    while (tri(k + 1) <= s) ++k;
    while (k > 0 && tri(k) > s) --k;
    return k;
}
__device__ void tile_ij(int t, int R, int C, int order, int& I, int& J) {
    if (order == 0) { I = t / C; J = t % C; return; }
    if (order >= 10) {  // anti-diagonal order of g-wide groups, tiles of a group left to right
        const int g = order - 10;
        int I2, J2;
        tile_ij(t / g, R, C / g, 2, I2, J2);
        I = I2;
        J = J2 * g + t % g;
        return;
    }
    if (order == 2) {  // compact anti-diagonal order (I ascending)
        const long long s = t, m = R < C ? R : C, M = R < C ? C : R;
        const long long hA = tri(m), hB = hA + (M - m) * m;
        long long d, base;
        if (s < hA) { d = tri_inv(s); base = tri(d); }
        else if (s < hB) { d = m + (s - hA) / m; base = hA + (d - m) * m; }
        else {
            const long long r = static_cast<long long>(R) * C - 1 - s, e = tri_inv(r);
            d = static_cast<long long>(R) + C - 2 - e;
            base = static_cast<long long>(R) * C - tri(e + 1);
        }
        const long long i0 = d - C + 1 > 0 ? d - C + 1 : 0;
        I = static_cast<int>(i0 + (s - base));
        J = static_cast<int>(d - I);
        return;
    }
    // column-major
    I = t % R; J = t / R;
}

constexpr int NW = 16;

template <int TR, int TC, int ST, int MODE>
__global__ void __launch_bounds__((NW + 2) * 32, 1) copy_kernel(const __grid_constant__ CUtensorMap mi,
                                                                 const __grid_constant__ CUtensorMap mo, int R, int C,
                                                                 int order, unsigned int* counter,
                                                                 unsigned long long* lat, float* dst, int n) {
    extern __shared__ __align__(1024) unsigned char raw[];
    float* stage = reinterpret_cast<float*>(raw);
    constexpr int NO = (ST + 2) * TR * TC * 4 <= 227 * 1024 ? 2 : 1;
    float* out = stage + ST * TR * TC;  // MODE 1: NO output buffers
    __shared__ uint64_t full[ST], empty[ST], ofull[2], ofree[2];
    __shared__ int tid_of[ST];
    __shared__ int otid[2];
    __shared__ long long issued[ST];
    constexpr uint32_t kBytes = TR * TC * 4;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < ST; ++s) { minit(&full[s], 1); minit(&empty[s], MODE >= 1 ? NW : 1); }
        for (int s = 0; s < 2; ++s) { minit(&ofull[s], NW); minit(&ofree[s], 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int ntiles = R * C;
    const uint64_t pol = pol_first();
    if (warp == NW) {
        if (lane == 0) {  // loader
            unsigned long long sum = 0, cnt = 0;
            for (int k = 0;; ++k) {
                const int s = k % ST;
                if (k >= ST) mwait(&empty[s], ((k / ST) & 1) ^ 1);
                const int t = static_cast<int>(atomicAdd(counter, 1u));
                tid_of[s] = t;
                if (t >= ntiles) { marrive(&full[s]); break; }
                int I, J;
                tile_ij(t, R, C, order, I, J);
                mexpect(&full[s], kBytes);
                issued[s] = clock64();
                load_tile<TR, TC>(stage + s * TR * TC, &mi, &full[s], I, J, pol);
            }
            (void)sum; (void)cnt;
        }
    } else if (warp == NW + 1) {
        if (MODE != 2 && lane == 0) {  // storer
            unsigned long long sum = 0, cnt = 0;
            for (int k = 0;; ++k) {
                const int s = k % ST;
                if (MODE == 0) {
                    mwait(&full[s], (k / ST) & 1);
                    const int t = tid_of[s];
                    if (t >= ntiles) break;
                    sum += clock64() - issued[s];
                    ++cnt;
                    int I, J;
                    tile_ij(t, R, C, order, I, J);
                    store_tile<TR, TC>(&mo, stage + s * TR * TC, I, J, pol);
                    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
                    marrive(&empty[s]);
                } else {
                    const int o = k % NO;
                    mwait(&ofull[o], (k / NO) & 1);
                    const int t = otid[o];
                    if (t >= ntiles) break;
                    int I, J;
                    tile_ij(t, R, C, order, I, J);
                    store_tile<TR, TC>(&mo, out + o * TR * TC, I, J, pol);
                    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
                    marrive(&ofree[o]);
                }
            }
            asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
            atomicAdd(&lat[0], sum);
            atomicAdd(&lat[1], cnt);
        }
    } else if (MODE >= 1) {
        // compute warps: stage -> registers -> out
        constexpr int RPW = TR / NW > 0 ? TR / NW : 1;
        constexpr int V4 = TC / 128;  // float4 per lane per row
        for (int k = 0;; ++k) {
            const int s = k % ST;
            mwait(&full[s], (k / ST) & 1);
            const int t = tid_of[s];
            const int o = k % NO;
            if (t >= ntiles) {
                if (MODE == 2) break;
                if (k >= NO) mwait(&ofree[o], ((k / NO) & 1) ^ 1);
                if (warp == 0 && lane == 0) otid[o] = t;
                __syncwarp();
                if (lane == 0) marrive(&ofull[o]);
                break;
            }
            float4 v[RPW][V4];
            const float* st = stage + s * TR * TC;
#pragma unroll
            for (int r = 0; r < RPW; ++r)
#pragma unroll
                for (int u = 0; u < V4; ++u)
                    v[r][u] = *reinterpret_cast<const float4*>(&st[(warp * RPW + r) * TC + u * 128 + lane * 4]);
            __syncwarp();
            if (lane == 0) marrive(&empty[s]);
            if constexpr (MODE == 2) {
                int I, J;
                tile_ij(t, R, C, order, I, J);
#pragma unroll
                for (int r = 0; r < RPW; ++r)
#pragma unroll
                    for (int u = 0; u < V4; ++u) {
                        float4* g = reinterpret_cast<float4*>(dst + static_cast<long long>(I * TR + warp * RPW + r) * n +
                                                              J * TC + u * 128 + lane * 4);
                        __stcs(g, v[r][u]);
                    }
                continue;
            }
            if (k >= NO) mwait(&ofree[o], ((k / NO) & 1) ^ 1);
            if (warp == 0 && lane == 0) otid[o] = t;
            float* ob = out + o * TR * TC;
#pragma unroll
            for (int r = 0; r < RPW; ++r)
#pragma unroll
                for (int u = 0; u < V4; ++u)
                    *reinterpret_cast<float4*>(&ob[(warp * RPW + r) * TC + u * 128 + lane * 4]) = v[r][u];
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (lane == 0) marrive(&ofull[o]);
        }
    }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int make_map(CUtensorMap* m, void* p, int n, int tr, int tc, int promo) {
    static EncodeFn enc = nullptr;
    if (!enc) {
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", reinterpret_cast<void**>(&enc), cudaEnableDefault, &q) !=
            cudaSuccess)
            return -1;
    }
    const CUtensorMapL2promotion pr = promo == 0 ? CU_TENSOR_MAP_L2_PROMOTION_NONE
                                      : promo == 1 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B
                                                   : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
    cuuint32_t es[3] = {1, 1, 1};
    if (tc <= 256) {
        cuuint64_t dims[2] = {static_cast<cuuint64_t>(n), static_cast<cuuint64_t>(n)};
        cuuint64_t strides[1] = {static_cast<cuuint64_t>(n) * 4};
        cuuint32_t box[2] = {static_cast<cuuint32_t>(tc), static_cast<cuuint32_t>(tr)};
        return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, p, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, pr, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS ? 0 : -2;
    }
    cuuint64_t dims[3] = {256, static_cast<cuuint64_t>(n / 256), static_cast<cuuint64_t>(n)};
    cuuint64_t strides[2] = {256 * 4, static_cast<cuuint64_t>(n) * 4};
    cuuint32_t box[3] = {256, static_cast<cuuint32_t>(tc / 256), static_cast<cuuint32_t>(tr)};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, p, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               CU_TENSOR_MAP_SWIZZLE_NONE, pr, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS ? 0 : -2;
}

template <int TR, int TC, int ST, int MODE>
int run(const float* src, float* dst, int n, int ctas, int reps, int order, int promo, float* ms, double* lat_cyc) {
    CUtensorMap mi, mo;
    if (make_map(&mi, const_cast<float*>(src), n, TR, TC, promo) || make_map(&mo, dst, n, TR, TC, promo)) return -3;
    const int no = (ST + 2) * TR * TC * 4 <= 227 * 1024 ? 2 : 1;
    const size_t smem = static_cast<size_t>(ST + (MODE == 1 ? no : 0)) * TR * TC * 4;
    auto k = copy_kernel<TR, TC, ST, MODE>;
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem)) != cudaSuccess)
        return -4;
    unsigned long long* lat;
    unsigned int* ctr;
    cudaMalloc(&lat, 16);
    cudaMalloc(&ctr, 4 * (reps + 2));
    cudaMemset(ctr, 0, 4 * (reps + 2));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int w = 0; w < 2; ++w) k<<<ctas, (NW + 2) * 32, smem>>>(mi, mo, n / TR, n / TC, order, ctr + reps + w, lat, dst, n);
    cudaMemset(lat, 0, 16);
    cudaEventRecord(e0);
    for (int r = 0; r < reps; ++r) k<<<ctas, (NW + 2) * 32, smem>>>(mi, mo, n / TR, n / TC, order, ctr + r, lat, dst, n);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(ms, e0, e1);
    *ms /= reps;
    unsigned long long h[2];
    cudaMemcpy(h, lat, 16, cudaMemcpyDeviceToHost);
    *lat_cyc = h[1] ? static_cast<double>(h[0]) / h[1] : 0.0;
    cudaFree(lat);
    cudaFree(ctr);
    const cudaError_t err = cudaGetLastError();
    return err == cudaSuccess ? 0 : -100 - static_cast<int>(err);
}

}  // namespace

extern "C" int tma_copy2(const float* src, float* dst, int n, int tr, int tc, int stages, int mode, int ctas, int reps,
                         int order, int promo, float* ms, double* lat_cyc) {
#define CASE(A, B, C, M) \
    if (tr == A && tc == B && stages == C && mode == M) return run<A, B, C, M>(src, dst, n, ctas, reps, order, promo, ms, lat_cyc);
#define CASES(A, B, C) CASE(A, B, C, 0) CASE(A, B, C, 1) CASE(A, B, C, 2)
    CASES(128, 128, 2) CASES(128, 128, 3) CASES(64, 256, 2) CASES(64, 256, 3) CASES(32, 512, 2) CASES(32, 512, 3)
    CASES(16, 1024, 2) CASES(16, 1024, 3) CASES(32, 256, 4) CASES(32, 256, 6) CASES(16, 512, 4) CASES(16, 512, 6)
    CASES(64, 512, 1) CASES(32, 1024, 1) CASES(32, 1024, 2) CASES(16, 2048, 2) CASES(32, 128, 4) CASES(64, 128, 4)
#undef CASES
#undef CASE
    return -1;
}
