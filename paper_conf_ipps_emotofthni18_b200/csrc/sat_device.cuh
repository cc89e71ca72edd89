// sat_device.cuh -- sm_100a device primitives for libsat: TMA 2-D tile moves with mbarriers,
// relaxed gpu-scope status words, warp scans.  No SAT-specific logic here (see sat_kernel.cuh).
#pragma once

#include <cstdint>
#include <cstdio>
#include <cuda.h>  // CUtensorMap (header only; the driver entry point is resolved at run time)
#include <cuda_runtime.h>

namespace sat {

constexpr unsigned kFull = 0xffffffffu;

// ------------------------------------------------------------------ element arithmetic
// int32 SAT is computed in uint32 (two's-complement wraparound, R1); fp32 in IEEE fp32.
__device__ __forceinline__ uint32_t to_bits(uint32_t v) { return v; }
__device__ __forceinline__ uint32_t to_bits(float v) { return __float_as_uint(v); }
template <typename V> __device__ __forceinline__ V from_bits(uint32_t b);
template <> __device__ __forceinline__ uint32_t from_bits<uint32_t>(uint32_t b) { return b; }
template <> __device__ __forceinline__ float from_bits<float>(uint32_t b) { return __uint_as_float(b); }

// Warp prefix-sum algorithm of P:118-124 (Kogge-Stone, log2(32) = 5 shuffle steps; the "a[i+2^j]"
// of P:124 is read as a[i-2^j], reading R15).  Inclusive; lane 31 ends with the warp total.
template <typename V>
__device__ __forceinline__ V warp_inclusive_scan(V x, int lane) {
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        V y = __shfl_up_sync(kFull, x, d);
        if (lane >= d) x = x + y;
    }
    return x;
}

// Exclusive prefix over the 32 lanes of a warp for N independent rows at once (tot[r] = this lane's
// value in row r; ex[r] = sum over lanes < lane), through a transpose in shared memory instead of
// N shuffle scans: G = 32/N lanes take one row each, sum N consecutive lane values serially, and
// scan their G partial sums with log2(G) shuffles.  S: N*32 elements of warp-private, 16-byte
// aligned scratch.  Same prefix sums as warp_inclusive_scan (different association for floats).
template <typename V, int N>
__device__ __forceinline__ void warp_rows_exclusive_smem(const V (&tot)[N], V (&ex)[N], V* S, int lane) {
    static_assert(N >= 4 && N <= 32 && 32 % N == 0, "rows per transposed scan");
    constexpr int G = 32 / N;
#pragma unroll
    for (int r = 0; r < N; ++r) S[r * 32 + lane] = tot[r];
    __syncwarp();
    const int row = lane / G, g = lane % G;
    V x[N];
#pragma unroll
    for (int i = 0; i < N; i += 4) {
        const uint4 q = *reinterpret_cast<const uint4*>(&S[row * 32 + g * N + i]);
        x[i] = from_bits<V>(q.x); x[i + 1] = from_bits<V>(q.y); x[i + 2] = from_bits<V>(q.z); x[i + 3] = from_bits<V>(q.w);
    }
#pragma unroll
    for (int i = 1; i < N; ++i) x[i] = x[i] + x[i - 1];
    V inc = x[N - 1];
#pragma unroll
    for (int d = 1; d < G; d <<= 1) {
        const V y = __shfl_up_sync(kFull, inc, d, G);
        if (g >= d) inc = inc + y;
    }
    V base = __shfl_up_sync(kFull, inc, 1, G);
    if (g == 0) base = V(0);
    __syncwarp();
#pragma unroll
    for (int i = 0; i < N; i += 4) {
        const V e0 = i == 0 ? base : base + x[i - 1];
        *reinterpret_cast<uint4*>(&S[row * 32 + g * N + i]) =
            make_uint4(to_bits(e0), to_bits(base + x[i]), to_bits(base + x[i + 1]), to_bits(base + x[i + 2]));
    }
    __syncwarp();
#pragma unroll
    for (int r = 0; r < N; ++r) ex[r] = S[r * 32 + lane];
}

template <typename V>
__device__ __forceinline__ V warp_sum(V x) {
#pragma unroll
    for (int d = 16; d >= 1; d >>= 1) x = x + __shfl_xor_sync(kFull, x, d);
    return x;
}

// ------------------------------------------------------------------ protocol-stress builds
// (PAPER.md:21 -- the method must be correct and deadlock-free under any CTA -> SM
// assignment and any relative speed of the CTAs.)  Neither switch is on in the product build.
//   -DSAT_JITTER=1    before every publication of status words a warp sleeps a pseudo-random 0 .. 4 us
//                     (one time in four), so words land in orders the production timing never shows.
//   -DSAT_WATCHDOG=1  every spin loop is bounded: after kWatchdogNs of waiting without progress the
//                     thread prints what it waited for and traps, so a protocol deadlock becomes a launch
//                     error (cudaErrorLaunchFailure) instead of a hung GPU.
__device__ __forceinline__ uint64_t sat_now_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// Jitter is applied per warp at publication points where the whole warp is converged (SAT_JITTER_WARP()
// in the kernels): the lanes of a warp sleep the same time, so the perturbation is between warps and CTAs
// -- what the look-back protocol must tolerate -- not inside a warp's lock-step code.
#if SAT_JITTER
__device__ __forceinline__ void sat_jitter_warp() {
    uint64_t z = static_cast<uint64_t>(clock64()) ^ (static_cast<uint64_t>(blockIdx.x) << 40) ^
                 (static_cast<uint64_t>(threadIdx.x >> 5) << 20);
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    z ^= z >> 31;
    z = __shfl_sync(0xffffffffu, z, 0);
    if ((z & 3u) == 0u) __nanosleep(static_cast<unsigned>((z >> 8) & 4095u));
}
#define SAT_JITTER_WARP() ::sat::sat_jitter_warp()
#else
#define SAT_JITTER_WARP() (void)0
#endif
#if SAT_WATCHDOG
constexpr uint64_t kWatchdogNs = 10000000000ull;  // 10 s without progress
__device__ __noinline__ void sat_watchdog_fire(const char* what) {
    printf("libsat watchdog: block %d thread %d waited > 10 s for %s\n", static_cast<int>(blockIdx.x),
           static_cast<int>(threadIdx.x), what);
    __trap();
}
#define SAT_SPIN_DECL uint64_t sat_spin_t0_ = ::sat::sat_now_ns()
#define SAT_SPIN_RESET (sat_spin_t0_ = ::sat::sat_now_ns())
#define SAT_SPIN_CHECK(what)                                                                                  \
    do {                                                                                                      \
        if (::sat::sat_now_ns() - sat_spin_t0_ > ::sat::kWatchdogNs) ::sat::sat_watchdog_fire(what);          \
    } while (0)
#else
#define SAT_SPIN_DECL (void)0
#define SAT_SPIN_RESET (void)0
#define SAT_SPIN_CHECK(what) (void)0
#endif
// spin (with a nanosleep back-off) until `cond` holds
#define sat_spin_until(cond, ns)                                                                              \
    do {                                                                                                      \
        SAT_SPIN_DECL;                                                                                        \
        while (!(cond)) {                                                                                     \
            SAT_SPIN_CHECK(#cond);                                                                            \
            __nanosleep(ns);                                                                                  \
        }                                                                                                     \
    } while (0)

// ------------------------------------------------------------------ shared memory / mbarrier
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
                 : "memory");
}

// Blocking wait on an mbarrier phase.  The suspend-time hint lets the hardware park the warp until
// the phase completes instead of spinning (a spinning warp steals issue slots from working warps).
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(smem_addr(bar)), "r"(parity), "r"(1000000u)
        : "memory");
    return ok != 0u;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
#if SAT_WATCHDOG
    SAT_SPIN_DECL;
    while (!mbar_try_wait(bar, parity)) SAT_SPIN_CHECK("an mbarrier phase");
    return;
#endif
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "SAT_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
        "@!p bra SAT_WAIT_%=;\n}" ::"r"(smem_addr(bar)),
        "r"(parity), "r"(1000000u)
        : "memory");
}

// ------------------------------------------------------------------ TMA (cp.async.bulk.tensor)
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// 2-D tile global -> shared, completion signalled on `bar` as transaction bytes.  Out-of-bounds
// box elements are zero-filled (partial edge tiles, R2).
__device__ __forceinline__ void tma_load_2d(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int x, int y,
                                            uint64_t policy) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%2, %3}], [%4], %5;" ::"r"(smem_addr(smem_dst)),
        "l"(map), "r"(x), "r"(y), "r"(smem_addr(bar)), "l"(policy)
        : "memory");
}

// 1-D bulk copy global -> shared (TMA engine), completion signalled on `bar` as transaction bytes.
// src, dst 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_load_1d(void* smem_dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_addr(smem_dst)),
                 "l"(src), "r"(bytes), "r"(smem_addr(bar))
                 : "memory");
}

// 2-D tile global -> L2 only (no shared memory, no completion): warms L2 ahead of the real load.
__device__ __forceinline__ void tma_prefetch_2d(const CUtensorMap* map, int x, int y) {
    asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global [%0, {%1, %2}];" ::"l"(map), "r"(x), "r"(y) : "memory");
}
// ... with an L2 eviction-priority hint for the prefetched lines
__device__ __forceinline__ void tma_prefetch_2d_hint(const CUtensorMap* map, int x, int y, uint64_t policy) {
    asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global.L2::cache_hint [%0, {%1, %2}], %3;" ::"l"(map), "r"(x),
                 "r"(y), "l"(policy)
                 : "memory");
}

// 2-D tile shared -> global; out-of-bounds box elements are not written (edge tiles, pitch pad).
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, const void* smem_src, int x, int y) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(map), "r"(x),
                 "r"(y), "r"(smem_addr(smem_src))
                 : "memory");
}

// Same with an L2 eviction policy (evict_first for the streamed output, so it does not push the
// look-back status words out of L2).
__device__ __forceinline__ void tma_store_2d_hint(const CUtensorMap* map, const void* smem_src, int x, int y,
                                                  uint64_t policy) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%1, %2}], [%3], %4;" ::"l"(
                     map),
                 "r"(x), "r"(y), "r"(smem_addr(smem_src)), "l"(policy)
                 : "memory");
}

// 16-byte global store with an L2 eviction policy (the streamed SAT output, written from registers).
__device__ __forceinline__ void st_global_v4_hint(void* p, uint32_t a, uint32_t b, uint32_t c, uint32_t d,
                                                  uint64_t pol) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.b32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p), "r"(a),
                 "r"(b), "r"(c), "r"(d), "l"(pol)
                 : "memory");
}

__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}


__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }

template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}

__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// Generic-proxy smem writes -> visible to the async proxy (the TMA store that follows).
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void prefetch_tensormap(const CUtensorMap* map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}

// ------------------------------------------------------------------ gpu-scope status words
// A status word is 64 bits: high 32 = (epoch << 2) | kind, low 32 = value bits.  One aligned
// 64-bit access is single-copy atomic, so value and status can never tear; relaxed gpu-scope
// accesses go to L2 (coherent point for all SMs) and need no fence (R11).
__device__ __forceinline__ void st_relaxed(uint64_t* p, uint64_t a) {
    asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(a) : "memory");
}
__device__ __forceinline__ void st_relaxed2(uint64_t* p, uint64_t a, uint64_t b) {
    asm volatile("st.relaxed.gpu.global.v2.b64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t* p) {
    uint64_t a;
    asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(a) : "l"(p) : "memory");
    return a;
}
__device__ __forceinline__ void ld_relaxed2(const uint64_t* p, uint64_t& a, uint64_t& b) {
    asm volatile("ld.relaxed.gpu.global.v2.b64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

// Status-word accesses with an L2 evict_last policy: the words must survive in L2 between their
// publication and their successors' look-backs while the matrix streams through.
__device__ __forceinline__ void st_relaxed_p(uint64_t* p, uint64_t a, uint64_t pol) {
    asm volatile("st.relaxed.gpu.global.L2::cache_hint.b64 [%0], %1, %2;" ::"l"(p), "l"(a), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_relaxed2_p(uint64_t* p, uint64_t a, uint64_t b, uint64_t pol) {
    asm volatile("st.relaxed.gpu.global.L2::cache_hint.v2.b64 [%0], {%1, %2}, %3;" ::"l"(p), "l"(a), "l"(b), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed_p(const uint64_t* p, uint64_t pol) {
    uint64_t a;
    asm volatile("ld.relaxed.gpu.global.L2::cache_hint.b64 %0, [%1], %2;" : "=l"(a) : "l"(p), "l"(pol) : "memory");
    return a;
}
__device__ __forceinline__ void ld_relaxed2_p(const uint64_t* p, uint64_t& a, uint64_t& b, uint64_t pol) {
    asm volatile("ld.relaxed.gpu.global.L2::cache_hint.v2.b64 {%0, %1}, [%2], %3;"
                 : "=l"(a), "=l"(b)
                 : "l"(p), "l"(pol)
                 : "memory");
}

// System-scope status words: the chained strip partition's inbox, written by a peer GPU over NVLink
// (peer-mapped pointers) and polled by the owner; single-copy atomic 64-bit accesses as above.
__device__ __forceinline__ void st_relaxed2_sys(uint64_t* p, uint64_t a, uint64_t b) {
    asm volatile("st.relaxed.sys.global.v2.b64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void ld_relaxed2_sys(const uint64_t* p, uint64_t& a, uint64_t& b) {
    asm volatile("ld.relaxed.sys.global.v2.b64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ void st_relaxed_sys_u32(uint32_t* p, uint32_t a) {
    asm volatile("st.relaxed.sys.global.b32 [%0], %1;" ::"l"(p), "r"(a) : "memory");
}
__device__ __forceinline__ uint32_t ld_relaxed_sys_u32(const uint32_t* p) {
    uint32_t a;
    asm volatile("ld.relaxed.sys.global.b32 %0, [%1];" : "=r"(a) : "l"(p) : "memory");
    return a;
}
template <int E>
__device__ __forceinline__ void st_words_sys(uint64_t* p, const uint64_t (&w)[E]) {
    static_assert(E % 2 == 0, "16-byte aligned word pairs");
#pragma unroll
    for (int e = 0; e < E; e += 2) st_relaxed2_sys(p + e, w[e], w[e + 1]);
}
template <int E>
__device__ __forceinline__ void ld_words_sys(const uint64_t* p, uint64_t (&w)[E]) {
    static_assert(E % 2 == 0, "16-byte aligned word pairs");
#pragma unroll
    for (int e = 0; e < E; e += 2) ld_relaxed2_sys(p + e, w[e], w[e + 1]);
}

template <int E>
__device__ __forceinline__ void st_words_p(uint64_t* p, const uint64_t (&w)[E], uint64_t pol) {
    if constexpr (E % 2 != 0) {  // odd vectors are not 16-byte aligned per lane: scalar accesses
#pragma unroll
        for (int e = 0; e < E; ++e) st_relaxed_p(p + e, w[e], pol);
    } else {
#pragma unroll
        for (int e = 0; e < E; e += 2) st_relaxed2_p(p + e, w[e], w[e + 1], pol);
    }
}

template <int E>
__device__ __forceinline__ void ld_words_p(const uint64_t* p, uint64_t (&w)[E], uint64_t pol) {
    if constexpr (E % 2 != 0) {  // odd vectors are not 16-byte aligned per lane: scalar accesses
#pragma unroll
        for (int e = 0; e < E; ++e) w[e] = ld_relaxed_p(p + e, pol);
    } else {
#pragma unroll
        for (int e = 0; e < E; e += 2) ld_relaxed2_p(p + e, w[e], w[e + 1], pol);
    }
}

template <int E>
__device__ __forceinline__ void st_words(uint64_t* p, const uint64_t (&w)[E]) {
    if constexpr (E % 2 != 0) {  // odd vectors are not 16-byte aligned per lane: scalar accesses
#pragma unroll
        for (int e = 0; e < E; ++e) st_relaxed(p + e, w[e]);
    } else {
#pragma unroll
        for (int e = 0; e < E; e += 2) st_relaxed2(p + e, w[e], w[e + 1]);
    }
}

template <int E>
__device__ __forceinline__ void ld_words(const uint64_t* p, uint64_t (&w)[E]) {
    if constexpr (E % 2 != 0) {  // odd vectors are not 16-byte aligned per lane: scalar accesses
#pragma unroll
        for (int e = 0; e < E; ++e) w[e] = ld_relaxed(p + e);
    } else {
#pragma unroll
        for (int e = 0; e < E; e += 2) ld_relaxed2(p + e, w[e], w[e + 1]);
    }
}

}  // namespace sat
