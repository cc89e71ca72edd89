// sat_api.cu -- libsat host side: the C ABI of include/sat.h.  Argument validation, the cached
// per-(device, stream) workspace, TMA tensor maps, kernel variant selection and launch, the
// end-to-end host-buffer pipeline and the NCCL strip-partitioned path.
#include <dlfcn.h>

#include <cstdarg>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <type_traits>
#include <utility>
#include <vector>

#include <cudaTypedefs.h>  // PFN_cuTensorMapEncodeTiled

#include "sat.h"
#include "sat_aux_kernels.cuh"
#include "sat_kernel.cuh"
#include "sat_tm_kernel.cuh"
#include "sat_query_kernels.cuh"
#include "sat_batch_kernel.cuh"
#include "sat_wide_kernel.cuh"

#if defined(SAT_HAVE_NCCL_H)
#include <nccl.h>
#endif

#define SAT_API extern "C" __attribute__((visibility("default")))

namespace {

using sat::Ctrl;
using sat::KParams;

// ------------------------------------------------------------------ error reporting
thread_local std::string g_detail;

sat_status_t fail(sat_status_t s, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_detail = buf;
    return s;
}

sat_status_t cuda_fail(cudaError_t e, const char* what) {
    return fail(SAT_ERR_CUDA, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
}

#define SAT_CUDA(call)                                  \
    do {                                                \
        cudaError_t e_ = (call);                        \
        if (e_ != cudaSuccess) return cuda_fail(e_, #call); \
    } while (0)

// ------------------------------------------------------------------ kernel variants
using LaunchFn = cudaError_t (*)(bool tma, bool carry, dim3 grid, cudaStream_t st, const CUtensorMap& mi,
                                 const CUtensorMap& mo, const void* params);
using PrepareFn = cudaError_t (*)(bool tma, bool carry, int* occupancy);

struct Variant {
    int TR, TC, NW, STAGES;
    int TB;                // TMA box width in elements (TC, or 256 for flat tiles: NB = TC / TB boxes)
    int OBR;               // rows of the output TMA box (TR, or TR/4 for quarter stores)
    int family;            // 2 = TMEM-parked (sat_tm_kernel), 1 = warp-specialised (sat_ws_kernel), 0 = classic
    bool chain;            // chained-strip configuration (sat_compute_chained only)
    size_t smem;           // dynamic shared memory bytes (same for int32 / fp32)
    LaunchFn launch[3];    // [dtype]; [kU8] = u8 input -> uint32 SAT (TMEM-parked family only, else null)
    PrepareFn prepare[3];  // [dtype]
};

// Kernel family traits: the classic kernel (sat_kernel.cuh, TileCfg) and the warp-specialised
// kernel (sat_ws_kernel.cuh, WsCfg) share one launch interface.
template <typename Cfg>
struct Family;

template <int TR, int TC, int NW, int ST>
struct Family<sat::TileCfg<TR, TC, NW, ST>> {
    using Cfg = sat::TileCfg<TR, TC, NW, ST>;
    static constexpr int threads = NW * 32;
    static constexpr int family = 0;
    template <typename V>
    static constexpr size_t smem() { return sizeof(sat::Smem<V, Cfg>); }
    template <typename V, bool TMA, bool CARRY>
    static void* kernel() { return reinterpret_cast<void*>(&sat::sat_tiles_kernel<V, Cfg, TMA, CARRY>); }
};

#if SAT_EXPERIMENTAL
template <int TR, int NW, int ST, int NT, int NQ, int FLAGS>
struct Family<sat::WsCfg<TR, NW, ST, NT, NQ, FLAGS>> {
    using Cfg = sat::WsCfg<TR, NW, ST, NT, NQ, FLAGS>;
    static constexpr int threads = Cfg::THREADS;
    static constexpr int family = 1;
    template <typename V>
    static constexpr size_t smem() { return sizeof(sat::WsSmem<V, Cfg>); }
    template <typename V, bool TMA, bool CARRY>
    static void* kernel() { return reinterpret_cast<void*>(&sat::sat_ws_kernel<V, Cfg, TMA, CARRY>); }
};

#endif

template <int NW, int IN, int NQ, int NT, int WPUB, int D, int DIRECT, int QS, int TR, int TC, int LB, int CT, int DW,
          int CH, int MINB, int RW2>
struct Family<sat::TmCfg<NW, IN, NQ, NT, WPUB, D, DIRECT, QS, TR, TC, LB, CT, DW, CH, MINB, RW2>> {
    using Cfg = sat::TmCfg<NW, IN, NQ, NT, WPUB, D, DIRECT, QS, TR, TC, LB, CT, DW, CH, MINB, RW2>;
    static constexpr int box_cols = Cfg::TB;
    static constexpr int out_box_rows = Cfg::OBR;
    static constexpr int threads = Cfg::THREADS;
    static constexpr int family = 2;
    template <typename V>
    static constexpr size_t smem() { return sizeof(sat::TmSmem<V, Cfg>); }
    template <typename V, bool TMA, bool CARRY>
    static void* kernel() { return reinterpret_cast<void*>(&sat::sat_tm_kernel<V, Cfg, TMA, CARRY>); }
    // u8 pixels in, uint32 integral image out
    static constexpr size_t smem_u8() { return sizeof(sat::TmSmem<uint32_t, Cfg, uint8_t>); }
    template <bool TMA, bool CARRY>
    static void* kernel_u8() { return reinterpret_cast<void*>(&sat::sat_tm_kernel<uint32_t, Cfg, TMA, CARRY, uint8_t>); }
};

template <typename F, typename = void>
struct HasOBR { static constexpr bool value = false; };
template <typename F>
struct HasOBR<F, std::void_t<decltype(F::out_box_rows)>> { static constexpr bool value = true; };

template <typename F, typename = void>
struct HasBox { static constexpr bool value = false; };
template <typename F>
struct HasBox<F, std::void_t<decltype(F::box_cols)>> { static constexpr bool value = true; };

template <typename F, typename = void>
struct HasU8 { static constexpr bool value = false; };
template <typename F>
struct HasU8<F, std::void_t<decltype(F::smem_u8())>> { static constexpr bool value = true; };

template <typename Cfg, typename = void>
struct IsChain { static constexpr bool value = false; };
template <typename Cfg>
struct IsChain<Cfg, std::void_t<decltype(Cfg::CHAIN)>> { static constexpr bool value = Cfg::CHAIN; };

template <typename V, typename F>
void* pick_kernel(bool tma, bool carry) {
    if constexpr (IsChain<typename F::Cfg>::value) {  // chained strips take no carry row
        (void)carry;
        return tma ? F::template kernel<V, true, false>() : F::template kernel<V, false, false>();
    } else {
        return tma ? (carry ? F::template kernel<V, true, true>() : F::template kernel<V, true, false>())
                   : (carry ? F::template kernel<V, false, true>() : F::template kernel<V, false, false>());
    }
}

template <typename V, typename Cfg>
cudaError_t launch_variant(bool tma, bool carry, dim3 grid, cudaStream_t st, const CUtensorMap& mi,
                           const CUtensorMap& mo, const void* params) {
    using F = Family<Cfg>;
    const KParams<V>& p = *static_cast<const KParams<V>*>(params);
    void* args[] = {const_cast<CUtensorMap*>(&mi), const_cast<CUtensorMap*>(&mo), const_cast<KParams<V>*>(&p)};
    return cudaLaunchKernel(pick_kernel<V, F>(tma, carry), grid, dim3(F::threads), args, F::template smem<V>(), st);
}

template <typename V, typename Cfg>
cudaError_t prepare_variant(bool tma, bool carry, int* occupancy) {
    using F = Family<Cfg>;
    void* k = pick_kernel<V, F>(tma, carry);
    const int smem = static_cast<int>(F::template smem<V>());
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occupancy, k, F::threads, smem);
}

constexpr int kU8 = 2;  // internal dtype index: u8 input, uint32 output

template <typename F>
void* pick_kernel_u8(bool tma, bool carry) {
    return tma ? (carry ? F::template kernel_u8<true, true>() : F::template kernel_u8<true, false>())
               : (carry ? F::template kernel_u8<false, true>() : F::template kernel_u8<false, false>());
}

template <typename Cfg>
cudaError_t launch_variant_u8(bool tma, bool carry, dim3 grid, cudaStream_t st, const CUtensorMap& mi,
                              const CUtensorMap& mo, const void* params) {
    using F = Family<Cfg>;
    const KParams<uint32_t>& p = *static_cast<const KParams<uint32_t>*>(params);
    void* args[] = {const_cast<CUtensorMap*>(&mi), const_cast<CUtensorMap*>(&mo), const_cast<KParams<uint32_t>*>(&p)};
    return cudaLaunchKernel(pick_kernel_u8<F>(tma, carry), grid, dim3(F::threads), args, F::smem_u8(), st);
}

template <typename Cfg>
cudaError_t prepare_variant_u8(bool tma, bool carry, int* occupancy) {
    using F = Family<Cfg>;
    void* k = pick_kernel_u8<F>(tma, carry);
    const int smem = static_cast<int>(F::smem_u8());
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occupancy, k, F::threads, smem);
}

template <typename Cfg, bool U8 = false>
Variant make_variant() {
    Variant v;
    v.TR = Cfg::TR;
    v.TC = Cfg::TC;
    v.NW = Cfg::NW;
    v.STAGES = Cfg::STAGES;
    v.family = Family<Cfg>::family;
    v.chain = IsChain<Cfg>::value;
    if constexpr (HasOBR<Family<Cfg>>::value) v.OBR = Family<Cfg>::out_box_rows;
    else v.OBR = Cfg::TR;
    v.smem = Family<Cfg>::template smem<uint32_t>();
    v.launch[SAT_INT32] = &launch_variant<uint32_t, Cfg>;
    v.launch[SAT_FLOAT32] = &launch_variant<float, Cfg>;
    v.prepare[SAT_INT32] = &prepare_variant<uint32_t, Cfg>;
    v.prepare[SAT_FLOAT32] = &prepare_variant<float, Cfg>;
    if constexpr (HasBox<Family<Cfg>>::value) v.TB = Family<Cfg>::box_cols;
    else v.TB = Cfg::TC;
    if constexpr (U8 && HasU8<Family<Cfg>>::value && Cfg::TC <= 256 && !IsChain<Cfg>::value) {
        v.launch[kU8] = &launch_variant_u8<Cfg>;
        v.prepare[kU8] = &prepare_variant_u8<Cfg>;
    } else {
        v.launch[kU8] = nullptr;
        v.prepare[kU8] = nullptr;
    }
    return v;
}

// Shipped kernel variants (auto_variant picks among them; sat_set_tuning can force one, test hook).
// Tuning builds (-DSAT_EXPERIMENTAL=1) append the configurations measured and not kept in round 1
// (DESIGN.md Sec. 5), so that they can still be re-measured.
enum : int { kVarClassic = 0, kVarTm128 = 1, kVarU8 = 2, kVarFlat = 3, kVarChain = 4, kVarU8Flat = 5 };
const std::vector<Variant>& variants() {
    static const std::vector<Variant> vs = {
        make_variant<sat::TileCfg<64, 128, 8, 2>>(),                   // 0: classic, 64 x 128 tiles (small matrices)
        // 1: TMEM-parked, 128 x 128 tiles, two row walker warps (even / odd tiles): 4K^2 38.3 -> 34.8 us,
        //    8K^2 103.5 -> 99.5 us (the row + diagonal walks are the medium sizes' long pole)
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4, 0, 0, 128, 128, 2, 0, 4, 0, 1, 1>, true>(),
        make_variant<sat::TmCfg<16, 4, 9, 1, 3, 4>, true>(),            // 2: u8 integral images (4 stages of 16 KiB)
        make_variant<sat::TmCfg<8, 2, 6, 1, 3, 4, 0, 0, 64, 256>>(),    // 3: TMEM-parked, flat 64 x 256 tiles
        // 4: chained strips (sat_compute_chained only); look-back window 2 (64K^2 / 8 per rank: 0.739 ms; windows
        //    of 4 / 8 0.740 / 0.756, diagonal window 4 0.783, a ring of 8 0.783, two row walkers 0.863)
        make_variant<sat::TmCfg<8, 2, 7, 1, 3, 4, 0, 0, 128, 128, 2, 0, 32, 1>>(),
        // 5: u8 integral images on flat 64 x 256 tiles (4 stages of 16 KiB, 8 compute warps), above 2^25 pixels:
        //    32K^2 1.145 -> 1.044 ms, 16K^2 0.331 -> 0.304 ms (tools/u8_probe.py; 3 / 6 stages, a ring of 8
        //    and the 2-tile-group order measured no better)
        make_variant<sat::TmCfg<8, 4, 7, 1, 3, 4, 0, 0, 64, 256>, true>(),
#if SAT_EXPERIMENTAL
        // tuning builds only (numbering continues after the shipped variants 0-5):
        // round-2 candidates, measured and not shipped (medium sizes): 8 compute warps on 128 x 128 tiles, wider look-back windows
        make_variant<sat::TmCfg<8, 2, 7, 1, 3, 4, 0, 0, 128, 128, 2>>(),            // 5
        make_variant<sat::TmCfg<8, 2, 7, 1, 3, 4, 0, 0, 128, 128, 4, 0, 32>>(),     // 6
        make_variant<sat::TmCfg<8, 2, 7, 1, 3, 4, 0, 0, 128, 128, 8, 0, 32>>(),     // 7
        make_variant<sat::TmCfg<8, 2, 7, 1, 3, 4, 0, 0, 128, 128, 8, 0, 4>>(),      // 8
        make_variant<sat::TmCfg<8, 2, 6, 1, 3, 4, 0, 0, 64, 256, 2, 0, 32>>(),      // 9: flat, diagonal 32
        make_variant<sat::TmCfg<8, 2, 8, 1, 3, 4, 0, 0, 64, 256>>(),                // 10: flat, tile ring of 8
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4>, true>(),             // round-1 variant 1 (one row walker)
        make_variant<sat::TmCfg<16, 4, 9, 1, 3, 4, 0, 0, 128, 128, 2, 0, 4, 0, 1, 1>, true>(),  // u8 + two row walkers
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4, 0, 0, 128, 128, 8, 0, 32, 1, 1, 1>>(),       // chain, 16 warps + RW2
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4, 0, 0, 128, 128, 8, 0, 32, 1>>(),             // chain, 16 warps
        make_variant<sat::TmCfg<8, 2, 6, 1, 3, 4, 0, 0, 64, 256, 2, 0, 4, 0, 1, 1>>(),  // flat + two row walkers
        // round-2 medium-size candidates: 64 x 128 tiles (32 KiB), 2 CTAs per SM (registers capped at 85)
        make_variant<sat::TmCfg<8, 2, 5, 1, 3, 4, 0, 0, 64, 128, 2, 0, 4, 0, 2>>(),    // 11
        make_variant<sat::TmCfg<8, 2, 5, 1, 3, 4, 0, 0, 64, 128, 4, 0, 32, 0, 2>>(),   // 12
        make_variant<sat::TmCfg<16, 2, 5>>(),  // walkers publish (blocking ws_walker)
        make_variant<sat::WsCfg<128, 16, 3, 1, 5, sat::kWsPrefetch | sat::kWsDefer | sat::kWsDirect>>(),  // 6
        make_variant<sat::WsCfg<128, 16, 3, 1, 5, sat::kWsPrefetch>>(),  // 7: warp-specialised, TMA store
        make_variant<sat::TmCfg<16, 2, 5, 1, 2>>(),  // 8
        make_variant<sat::TileCfg<128, 128, 16, 2>>(),  // 9: classic, 128 x 128 tiles
        make_variant<sat::TmCfg<16, 2, 7, 1, 1, 4>>(),  // 10
        make_variant<sat::TmCfg<16, 3, 8, 1, 3, 4, 1>>(),  // 11: GSAT from registers
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4, 1>>(),  // 12
        make_variant<sat::TmCfg<8, 2, 8, 1, 3, 4, 0, 0, 64, 256>>(),    // 13: flat, ring of 8
        make_variant<sat::TmCfg<8, 2, 7, 1, 3, 4, 0, 0, 64, 256>>(),    // 14: flat, ring of 7
        make_variant<sat::TmCfg<8, 2, 10, 1, 3, 4, 0, 0, 64, 256>>(),   // 15: flat, ring of 10
        make_variant<sat::TmCfg<16, 2, 6, 1, 3, 4, 0, 0, 64, 256>>(),   // 16: flat, 16 compute warps
        make_variant<sat::TmCfg<8, 3, 7, 1, 3, 4, 1, 0, 64, 256>>(),    // 17: flat, GSAT from registers
        make_variant<sat::TmCfg<8, 2, 6, 1, 3, 4, 0, 0, 64, 256, 2, 1>>(),  // 18: flat, 8 contiguous columns
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4, 0, 0, 128, 128, 4>>(),         // 19: 128^2, look-back 4 per round
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4, 0, 0, 128, 128, 8>>(),         // 20: 128^2, 8 per round
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4, 0, 0, 128, 128, 8, 0, 32>>(),  // 21: ... diagonal 32 per round
        make_variant<sat::TmCfg<16, 2, 7, 1, 3, 4, 0, 0, 128, 128, 2, 0, 32>>(),  // 22: 128^2, diagonal 32 per round
        make_variant<sat::TmCfg<8, 2, 6, 1, 3, 4, 0, 0, 64, 256, 4>>(),           // 23: flat, look-back 4 per round
        make_variant<sat::TmCfg<8, 2, 6, 1, 3, 4, 0, 0, 64, 256, 4, 0, 32>>(),    // 24: ... diagonal 32 per round
        make_variant<sat::TmCfg<16, 2, 9, 1, 3, 4, 0, 0, 128, 128, 8, 0, 32>>(),  // 25: 21 + ring of 9
        make_variant<sat::TmCfg<8, 2, 6, 1, 3, 4, 0, 0, 64, 256, 4, 0, 32, 1>>(),   // 26: chained strips, flat 64 x 256
#endif
    };
    return vs;
}

// process-wide tuning knobs (sat_set_tuning)
std::mutex g_mu;
int g_variant = -1;
int g_order = 0;
int g_ctas_per_sm = 0;
int g_max_ctas = 0;

int auto_variant(int64_t rows, int64_t cols) {
    // measured device times (tools/graph_sweep.py, tools/sweep_variants.py): up to
    // ~1.4K x 1.4K (<= 128 tiles of 128^2) the classic kernel with 64 x 128 tiles has the shortest
    // latency; up to 8K x 8K the TMEM-parked kernel on 128 x 128 tiles with two row walkers (round 2:
    // 4K^2 34.8 us, 8K^2 99.5 us vs 37.4 / 102.1 on flat tiles); above, the TMEM-parked kernel with
    // decoupled walkers (parking depth 4) on flat 64 x 256 tiles
    const int64_t n = rows * cols;
    return n <= (int64_t(1) << 21) ? kVarClassic : (n <= (int64_t(1) << 26) ? kVarTm128 : kVarFlat);
}

// L2 prefetch of a tile's boxes when the loader acquires it (cp.async.bulk.prefetch.tensor): the DRAM read
// of a tile then starts up to NQ - IN tiles before an input stage is free for it, so the read stream no
// longer waits on the compute warps' stage release.  Measured on the flat 64 x 256 kernel at 32K^2
// (tools/gpu_r02c.sh, profiles/r02_sweep_prefetch.jsonl): fp32 1.417 -> 1.384 ms, int32 1.409 -> 1.378 ms;
// with a tile ring of 8 it over-fetches (1.50 ms).  It pays at every size (profiles/r02_sweep_prefetch_sizes.jsonl:
// 4K^2 40.9 -> 36.7 us, 8K^2 108 -> 102 us, 64K^2 5.55 -> 5.48 ms).  Marking the prefetched lines evict_last
// (mode 2) keeps them in L2 until their TMA load (which reads them evict_first): 32K^2 fp32 1.383 -> 1.355 ms,
// int32 1.378 -> 1.351 ms, 16K^2 0.374 -> 0.365 ms, 64K^2 5.48 -> 5.37 ms, chained strip 0.741 -> 0.715 ms per rank;
// on the 128 x 128 kernel at 4K^2 / 8K^2 it costs 1-3% (tools/gpu_pf.sh).  Default: evict_last for the flat,
// chained and flat-u8 kernels, plain for the 128 x 128 ones, none for the classic kernel (no tile ring);
// SAT_L2_PREFETCH=0/1/2 (read once) forces off / plain / evict_last (tuning switch).
int l2_prefetch_mode(int vi) {
    static const int mode = [] {
        const char* e = std::getenv("SAT_L2_PREFETCH");
        return e ? std::atoi(e) : -1;
    }();
    if (mode >= 0) return mode;
    if (variants()[vi].family != 2) return 0;
    return (vi == kVarFlat || vi == kVarChain || vi == kVarU8Flat) ? 2 : 1;
}

int auto_order(int vi, int64_t cols) {
    // flat 64 x 256 tiles with >= 128 tile columns (>= 32K columns): anti-diagonal order of 2-wide tile
    // groups (each DRAM row visit 2 KiB); narrower grids keep the plain anti-diagonal order, which
    // measured faster there (tools/sweep_variants.py, profiles/r01_sweep_sizes.jsonl)
    return (vi == kVarFlat && (cols + 255) / 256 >= 128) ? 0x200 : 0;
}

// ------------------------------------------------------------------ device info caches
struct DeviceInfo {
    int sms = 0;
    std::map<std::pair<int, int>, int> occ;  // (variant*8 + dtype*4 + tma*2 + carry) -> occupancy
};
std::map<int, DeviceInfo> g_dev;

sat_status_t device_info(int dev, DeviceInfo** out) {
    auto it = g_dev.find(dev);
    if (it == g_dev.end()) {
        DeviceInfo di;
        SAT_CUDA(cudaDeviceGetAttribute(&di.sms, cudaDevAttrMultiProcessorCount, dev));
        it = g_dev.emplace(dev, di).first;
    }
    *out = &it->second;
    return SAT_OK;
}

// SM count of `dev` (cached; takes g_mu)
sat_status_t device_sms(int dev, int* sms) {
    std::lock_guard<std::mutex> lk(g_mu);
    DeviceInfo* di = nullptr;
    sat_status_t s = device_info(dev, &di);
    if (s == SAT_OK) *sms = di->sms;
    return s;
}

sat_status_t occupancy(int dev, int vi, int dt, bool tma, bool carry, int* occ) {
    DeviceInfo* di = nullptr;
    sat_status_t s = device_info(dev, &di);
    if (s != SAT_OK) return s;
    const std::pair<int, int> key(vi, dt * 4 + (tma ? 2 : 0) + (carry ? 1 : 0));
    auto it = di->occ.find(key);
    if (it == di->occ.end()) {
        int o = 0;
        if (!variants()[vi].prepare[dt]) return fail(SAT_ERR_UNSUPPORTED, "kernel variant %d lacks this dtype", vi);
        cudaError_t e = variants()[vi].prepare[dt](tma, carry, &o);
        if (e == cudaErrorInvalidValue) {  // dynamic shared memory above the per-block limit
            cudaGetLastError();
            return fail(SAT_ERR_UNSUPPORTED, "kernel variant %d does not fit on an SM for this dtype", vi);
        }
        if (e != cudaSuccess) return cuda_fail(e, "kernel attribute / occupancy query");
        if (o < 1) return fail(SAT_ERR_UNSUPPORTED, "kernel variant %d does not fit on an SM", vi);
        it = di->occ.emplace(key, o).first;
    }
    *occ = it->second;
    return SAT_OK;
}

// ------------------------------------------------------------------ workspace
struct Workspace {
    int dev = 0;
    cudaStream_t stream = nullptr;
    std::mutex mu;  // growth + launch on this (device, stream); g_mu only guards the map
    Ctrl* ctrl = nullptr;
    uint64_t* slots = nullptr;
    size_t slot_words = 0;
    uint64_t calls = 0;
    long long* stats = nullptr;  // SAT_STATS builds: [ctas][kNumStats] of the last launch, then the trace
    int stats_ctas = 0;
    size_t stats_words = 0;
    int64_t trace_tiles = 0;
    void* scratch = nullptr;  // colsum partials etc.
    size_t scratch_bytes = 0;
    int last_TR = 0, last_TC = 0, last_R = 0, last_C = 0;  // tile grid of the last launch (sat_debug_workspace)
};
std::map<std::pair<int, cudaStream_t>, Workspace*> g_ws;
Workspace* g_last_stats = nullptr;

sat_status_t reset_ctrl(Workspace* w) {
    Ctrl init{0u, 0u, 1u, 0u};
    SAT_CUDA(cudaMemcpyAsync(w->ctrl, &init, sizeof(Ctrl), cudaMemcpyHostToDevice, w->stream));
    SAT_CUDA(cudaStreamSynchronize(w->stream));  // `init` lives on this stack frame
    return SAT_OK;
}

// The workspace of (dev, st), created on first use (one synchronising control-block reset).  The
// caller locks w->mu before growing it (grow_slots) or launching with it.
sat_status_t find_workspace(int dev, cudaStream_t st, Workspace** out) {
    std::lock_guard<std::mutex> lk(g_mu);
    auto key = std::make_pair(dev, st);
    auto it = g_ws.find(key);
    if (it != g_ws.end()) {
        *out = it->second;
        return SAT_OK;
    }
    Workspace* w = new Workspace();
    w->dev = dev;
    w->stream = st;
    cudaError_t e = cudaMalloc(&w->ctrl, 256);
    if (e != cudaSuccess) {
        cudaGetLastError();
        delete w;
        return fail(SAT_ERR_OUT_OF_MEMORY, "workspace control block: %s", cudaGetErrorString(e));
    }
    sat_status_t s = reset_ctrl(w);
    if (s != SAT_OK) {
        cudaFree(w->ctrl);
        delete w;
        return s;
    }
    g_ws[key] = w;
    *out = w;
    return SAT_OK;
}

// Grow the status-word slots to >= slot_words (stream-ordered: cudaFreeAsync / cudaMallocAsync /
// cudaMemsetAsync on the workspace's stream, no host synchronisation).  New words are zeroed: epoch 0
// never matches a launch epoch (>= 1), so they read "not published".
sat_status_t grow_slots(Workspace* w, size_t slot_words) {
    if (slot_words > w->slot_words) {
        const size_t want = slot_words + slot_words / 4;
        if (w->slots) SAT_CUDA(cudaFreeAsync(w->slots, w->stream));
        w->slots = nullptr;
        w->slot_words = 0;
        cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&w->slots), want * sizeof(uint64_t), w->stream);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(SAT_ERR_OUT_OF_MEMORY, "workspace slots (%zu bytes): %s", want * 8, cudaGetErrorString(e));
        }
        SAT_CUDA(cudaMemsetAsync(w->slots, 0, want * sizeof(uint64_t), w->stream));
        w->slot_words = want;
    }
    // Epoch wrap (after ~2^30 launches on this workspace): clear the slots and restart at epoch 1.
    if (w->calls + 2 >= sat::kEpochMax) {
        SAT_CUDA(cudaMemsetAsync(w->slots, 0, w->slot_words * sizeof(uint64_t), w->stream));
        sat_status_t s = reset_ctrl(w);
        if (s != SAT_OK) return s;
        w->calls = 0;
    }
    return SAT_OK;
}

sat_status_t get_scratch(Workspace* w, size_t bytes, void** out) {
    if (bytes > w->scratch_bytes) {
        if (w->scratch) SAT_CUDA(cudaFreeAsync(w->scratch, w->stream));
        w->scratch = nullptr;
        w->scratch_bytes = 0;
        cudaError_t e = cudaMallocAsync(&w->scratch, bytes, w->stream);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(SAT_ERR_OUT_OF_MEMORY, "scratch (%zu bytes): %s", bytes, cudaGetErrorString(e));
        }
        w->scratch_bytes = bytes;
    }
    *out = w->scratch;
    return SAT_OK;
}

// Synchronises the workspace's stream and frees its buffers (the caller has removed it from g_ws).
void free_workspace(Workspace* w) {
    {
        std::lock_guard<std::mutex> wlk(w->mu);
        cudaStreamSynchronize(w->stream);
        if (w->slots) cudaFree(w->slots);
        if (w->scratch) cudaFree(w->scratch);
        if (w->ctrl) cudaFree(w->ctrl);
        if (w->stats) cudaFree(w->stats);
    }
    delete w;
}

// ------------------------------------------------------------------ TMA tensor maps
PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;

sat_status_t get_encoder() {
    if (g_encode) return SAT_OK;
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
        return fail(SAT_ERR_CUDA, "cuTensorMapEncodeTiled entry point unavailable (%s)", cudaGetErrorString(e));
    g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
    return SAT_OK;
}

sat_status_t encode_map(CUtensorMap* m, sat_dtype_t dt, const void* ptr, int64_t rows, int64_t cols, int64_t pitch,
                        int TR, int TC) {
    cuuint64_t dims[2] = {static_cast<cuuint64_t>(cols), static_cast<cuuint64_t>(rows)};
    cuuint64_t strides[1] = {static_cast<cuuint64_t>(pitch) * 4u};
    cuuint32_t box[2] = {static_cast<cuuint32_t>(TC), static_cast<cuuint32_t>(TR)};
    cuuint32_t estr[2] = {1u, 1u};
    CUresult r = g_encode(m, dt == SAT_FLOAT32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_UINT32, 2,
                          const_cast<void*>(ptr), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return fail(SAT_ERR_CUDA, "cuTensorMapEncodeTiled failed (CUresult %d)", (int)r);
    return SAT_OK;
}

sat_status_t encode_map_u8(CUtensorMap* m, const void* ptr, int64_t rows, int64_t cols, int64_t pitch_bytes, int TR,
                           int TC) {
    cuuint64_t dims[2] = {static_cast<cuuint64_t>(cols), static_cast<cuuint64_t>(rows)};
    cuuint64_t strides[1] = {static_cast<cuuint64_t>(pitch_bytes)};
    cuuint32_t box[2] = {static_cast<cuuint32_t>(TC), static_cast<cuuint32_t>(TR)};
    cuuint32_t estr[2] = {1u, 1u};
    CUresult r = g_encode(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, const_cast<void*>(ptr), dims, strides, box, estr,
                          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return fail(SAT_ERR_CUDA, "cuTensorMapEncodeTiled (u8) failed (CUresult %d)", (int)r);
    return SAT_OK;
}

// ------------------------------------------------------------------ validation / planning
sat_status_t validate(const void* src, const void* dst, int64_t rows, int64_t cols, int64_t pitch) {
    if (rows < 0 || cols < 0 || pitch < cols)
        return fail(SAT_ERR_INVALID_VALUE, "bad sizes rows=%lld cols=%lld pitch=%lld", (long long)rows,
                    (long long)cols, (long long)pitch);
    if (rows == 0 || cols == 0) return SAT_OK;
    if (!src || !dst) return fail(SAT_ERR_INVALID_VALUE, "null pointer");
    if ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 3u)
        return fail(SAT_ERR_MISALIGNED, "pointers must be 4-byte aligned");
    if (src != dst) {
        const uintptr_t bytes = static_cast<uintptr_t>(((rows - 1) * pitch + cols) * 4);
        const uintptr_t a = reinterpret_cast<uintptr_t>(src), b = reinterpret_cast<uintptr_t>(dst);
        if (a < b + bytes && b < a + bytes) return fail(SAT_ERR_INVALID_VALUE, "src and dst partially overlap");
    }
    if (rows > (int64_t(1) << 31) - 1 || cols > (int64_t(1) << 31) - 1)
        return fail(SAT_ERR_UNSUPPORTED, "rows and cols must be < 2^31");
    return SAT_OK;
}

bool tma_ok(const void* src, const void* dst, int64_t pitch) {
    return ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 15u) == 0 &&
           ((pitch * 4) % 16) == 0 && pitch * 4 < (int64_t(1) << 40);
}

struct Plan {
    int vi, TR, TC, R, C, order;
    int64_t ntiles;
    bool tma;
};

sat_status_t make_plan(int64_t rows, int64_t cols, int64_t pitch, const void* src, const void* dst, Plan* pl,
                       bool u8 = false, int64_t src_pitch = 0, int force_vi = -1) {
    int vi, order;
    if (force_vi >= 0) {
        vi = force_vi;
        order = 0;
    } else {
        std::lock_guard<std::mutex> lk(g_mu);
        const bool forced = g_variant >= 0 && !variants()[g_variant].chain;  // chain configs: chained calls only
        vi = forced ? g_variant
                    : (u8 ? (rows * cols <= (int64_t(1) << 25) ? kVarU8 : kVarU8Flat) : auto_variant(rows, cols));
        order = (!forced && g_order == 0) ? auto_order(vi, cols) : g_order;
    }
    const Variant& v = variants()[vi];
    pl->vi = vi;
    pl->TR = v.TR;
    pl->TC = v.TC;
    pl->R = static_cast<int>((rows + v.TR - 1) / v.TR);
    pl->C = static_cast<int>((cols + v.TC - 1) / v.TC);
    pl->ntiles = static_cast<int64_t>(pl->R) * pl->C;
    pl->order = order;
    pl->tma = u8 ? (((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 15u) == 0 &&
                    src_pitch % 16 == 0 && (pitch * 4) % 16 == 0 && pitch * 4 < (int64_t(1) << 40) &&
                    src_pitch < (int64_t(1) << 40))
                 : tma_ok(src, dst, pitch);
    if (pl->ntiles > (int64_t(1) << 31) - 4096)
        return fail(SAT_ERR_UNSUPPORTED, "too many tiles (%lld)", (long long)pl->ntiles);
    return SAT_OK;
}

// ------------------------------------------------------------------ the hot path
sat_status_t validate_u8(const void* src, int64_t src_pitch, const void* dst, int64_t rows, int64_t cols,
                         int64_t pitch) {
    if (rows < 0 || cols < 0 || pitch < cols || src_pitch < cols)
        return fail(SAT_ERR_INVALID_VALUE, "bad sizes rows=%lld cols=%lld pitch=%lld src_pitch=%lld", (long long)rows,
                    (long long)cols, (long long)pitch, (long long)src_pitch);
    if (rows == 0 || cols == 0) return SAT_OK;
    if (!src || !dst) return fail(SAT_ERR_INVALID_VALUE, "null pointer");
    if (reinterpret_cast<uintptr_t>(dst) & 3u) return fail(SAT_ERR_MISALIGNED, "dst must be 4-byte aligned");
    const uintptr_t a = reinterpret_cast<uintptr_t>(src), b = reinterpret_cast<uintptr_t>(dst);
    const uintptr_t na = static_cast<uintptr_t>((rows - 1) * src_pitch + cols);
    const uintptr_t nb = static_cast<uintptr_t>(((rows - 1) * pitch + cols) * 4);
    if (a < b + nb && b < a + na) return fail(SAT_ERR_INVALID_VALUE, "src and dst overlap");
    if (rows > (int64_t(1) << 31) - 1 || cols > (int64_t(1) << 31) - 1)
        return fail(SAT_ERR_UNSUPPORTED, "rows and cols must be < 2^31");
    return SAT_OK;
}

// dt: SAT_INT32, SAT_FLOAT32, or kU8 (u8 input with row stride src_pitch bytes -> uint32 output)
sat_status_t compute_impl(int dt, const void* src, void* dst, int64_t rows, int64_t cols, int64_t pitch,
                          const void* carry, cudaStream_t st, int64_t src_pitch = 0) {
    if (dt != SAT_INT32 && dt != SAT_FLOAT32 && dt != kU8) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype %d", dt);
    const bool u8 = dt == kU8;
    sat_status_t s = u8 ? validate_u8(src, src_pitch, dst, rows, cols, pitch) : validate(src, dst, rows, cols, pitch);
    if (s != SAT_OK || rows == 0 || cols == 0) return s;
    if (carry && (reinterpret_cast<uintptr_t>(carry) & 3u)) return fail(SAT_ERR_MISALIGNED, "carry misaligned");
    Plan pl;
    if ((s = make_plan(rows, cols, pitch, src, dst, &pl, u8, src_pitch)) != SAT_OK) return s;
    const Variant& v = variants()[pl.vi];

    int dev = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    int occ = 0, sms = 0, max_ctas = 0, ctas_per_sm = 0;
    {
        std::lock_guard<std::mutex> lk(g_mu);
        if ((s = occupancy(dev, pl.vi, dt, pl.tma, carry != nullptr, &occ)) != SAT_OK) return s;
        DeviceInfo* di = nullptr;
        if ((s = device_info(dev, &di)) != SAT_OK) return s;
        sms = di->sms;
        max_ctas = g_max_ctas;
        ctas_per_sm = g_ctas_per_sm;
    }
    int per_sm = (ctas_per_sm > 0 && ctas_per_sm < occ) ? ctas_per_sm : occ;
    int64_t grid = static_cast<int64_t>(sms) * per_sm;
    // the classic kernel is launched the paper's way, one CTA per tile (CTAs beyond the resident
    // ones take their tickets when they start, so any grid is deadlock-free): its persistent loop only
    // runs under a CTA cap (sat_set_max_ctas, the forward-progress tests)
    if (v.family == 0) grid = pl.ntiles;
    if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;
    if (grid > pl.ntiles) grid = pl.ntiles;

    Workspace* w;
    if ((s = find_workspace(dev, st, &w)) != SAT_OK) return s;
    std::lock_guard<std::mutex> wlk(w->mu);
    const size_t words = static_cast<size_t>(pl.ntiles) * (v.TR + v.TC + 1);
    if ((s = grow_slots(w, words)) != SAT_OK) return s;

    CUtensorMap mi, mo;
    std::memset(&mi, 0, sizeof(mi));
    std::memset(&mo, 0, sizeof(mo));
    if (pl.tma) {
        if ((s = get_encoder()) != SAT_OK) return s;
        if (u8) {
            if ((s = encode_map_u8(&mi, src, rows, cols, src_pitch, v.TR, v.TC)) != SAT_OK) return s;
            if ((s = encode_map(&mo, SAT_INT32, dst, rows, cols, pitch, v.OBR, v.TC)) != SAT_OK) return s;
        } else {
            if ((s = encode_map(&mi, static_cast<sat_dtype_t>(dt), src, rows, cols, pitch, v.TR, v.TB)) != SAT_OK)
                return s;
            if ((s = encode_map(&mo, static_cast<sat_dtype_t>(dt), dst, rows, cols, pitch, v.OBR, v.TB)) != SAT_OK)
                return s;
        }
    }
    KParams<uint32_t> p;  // identical layout for float
    std::memset(&p, 0, sizeof(p));  // epoch_override = 0, no chain
    p.src = static_cast<const uint32_t*>(src);
    p.dst = static_cast<uint32_t*>(dst);
    p.rows = rows;
    p.cols = cols;
    p.pitch = pitch;
    p.R = pl.R;
    p.C = pl.C;
    p.ntiles = static_cast<int>(pl.ntiles);
    p.order = pl.order;
    p.row_slots = w->slots;
    p.col_slots = w->slots + static_cast<size_t>(pl.ntiles) * v.TR;
    p.corner_slots = w->slots + static_cast<size_t>(pl.ntiles) * (v.TR + v.TC);
    p.ctrl = w->ctrl;
    p.carry = static_cast<const uint32_t*>(carry);
    p.stats = nullptr;
    p.trace = nullptr;
    p.src8 = u8 ? static_cast<const uint8_t*>(src) : nullptr;
    p.src_pitch = u8 ? src_pitch : pitch;
    if (u8) p.src = nullptr;
    p.l2_prefetch = l2_prefetch_mode(pl.vi);
#if SAT_STATS
    {
        std::lock_guard<std::mutex> lk(g_mu);
        const size_t need = static_cast<size_t>(grid) * sat::kNumStats + 8 * static_cast<size_t>(pl.ntiles);
        if (w->stats_words < need) {
            if (w->stats) cudaFree(w->stats);
            SAT_CUDA(cudaMalloc(&w->stats, need * 8));
            w->stats_words = need;
        }
        w->stats_ctas = static_cast<int>(grid);
        w->trace_tiles = pl.ntiles;
        SAT_CUDA(cudaMemsetAsync(w->stats, 0, need * 8, st));
        p.stats = w->stats;
        p.trace = w->stats + static_cast<size_t>(grid) * sat::kNumStats;
        g_last_stats = w;
    }
#endif
    cudaError_t e = v.launch[dt](pl.tma, carry != nullptr, dim3(static_cast<unsigned>(grid)), st, mi, mo, &p);
    if (e != cudaSuccess) return cuda_fail(e, "SAT kernel launch");
    w->calls++;
    w->last_TR = v.TR;
    w->last_TC = v.TC;
    w->last_R = pl.R;
    w->last_C = pl.C;
    return SAT_OK;
}

// 64-bit output elements: moments = false -> fp64 SAT of fp32 input, true ->
// (SAT(a), SAT(a*a)) fp32 pairs.  One CTA per 64 x 128 tile (sat_wide_kernel.cuh).
sat_status_t wide_impl(bool moments, const float* src, int64_t src_pitch, void* dst, int64_t dst_pitch, int64_t rows,
                       int64_t cols, cudaStream_t st) {
    if (rows < 0 || cols < 0 || src_pitch < cols || dst_pitch < cols)
        return fail(SAT_ERR_INVALID_VALUE, "bad sizes rows=%lld cols=%lld src_pitch=%lld dst_pitch=%lld", (long long)rows,
                    (long long)cols, (long long)src_pitch, (long long)dst_pitch);
    if (rows == 0 || cols == 0) return SAT_OK;
    if (!src || !dst) return fail(SAT_ERR_INVALID_VALUE, "null pointer");
    const uintptr_t a = reinterpret_cast<uintptr_t>(src), b = reinterpret_cast<uintptr_t>(dst);
    if ((a & 3u) || (b & 7u)) return fail(SAT_ERR_MISALIGNED, "src must be 4-byte and dst 8-byte aligned");
    if (rows > (int64_t(1) << 31) - 1 || cols > (int64_t(1) << 31) - 1)
        return fail(SAT_ERR_UNSUPPORTED, "rows and cols must be < 2^31");
    const uintptr_t na = static_cast<uintptr_t>(((rows - 1) * src_pitch + cols) * 4);
    const uintptr_t nb = static_cast<uintptr_t>(((rows - 1) * dst_pitch + cols) * 8);
    if (a < b + nb && b < a + na) return fail(SAT_ERR_INVALID_VALUE, "src and dst overlap");
    constexpr int TR = sat::kWideTR, TC = sat::kWideTC;
    const int64_t R = (rows + TR - 1) / TR, C = (cols + TC - 1) / TC, ntiles = R * C;
    if (ntiles > (int64_t(1) << 31) - 1) return fail(SAT_ERR_UNSUPPORTED, "too many tiles");
    int dev = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    Workspace* w;
    sat_status_t s = find_workspace(dev, st, &w);
    if (s != SAT_OK) return s;
    std::lock_guard<std::mutex> wlk(w->mu);
    if ((s = grow_slots(w, static_cast<size_t>(ntiles) * 2 * (TR + TC + 1))) != SAT_OK) return s;
    sat::WideParams p;
    std::memset(&p, 0, sizeof(p));
    p.src = src;
    p.dst = dst;
    p.rows = rows;
    p.cols = cols;
    p.src_pitch = src_pitch;
    p.dst_pitch = dst_pitch;
    p.R = static_cast<int>(R);
    p.C = static_cast<int>(C);
    p.ntiles = static_cast<int>(ntiles);
    p.row_slots = w->slots;
    p.col_slots = w->slots + static_cast<size_t>(ntiles) * 2 * TR;
    p.corner_slots = w->slots + static_cast<size_t>(ntiles) * 2 * (TR + TC);
    p.ctrl = w->ctrl;
    p.vec = ((a & 15u) == 0 && (b & 15u) == 0 && (src_pitch * 4) % 16 == 0 && (dst_pitch * 8) % 16 == 0) ? 1 : 0;
    if (moments) sat::sat_wide_kernel<float2><<<static_cast<unsigned>(ntiles), sat::kWideNW * 32, 0, st>>>(p);
    else sat::sat_wide_kernel<double><<<static_cast<unsigned>(ntiles), sat::kWideNW * 32, 0, st>>>(p);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "sat_wide_kernel launch");
    w->calls++;
    w->last_TR = w->last_TC = w->last_R = w->last_C = 0;  // two words per value: not sat_debug_workspace's layout
    return SAT_OK;
}

sat_status_t colsum_impl(sat_dtype_t dt, const void* src, void* colsum, int64_t rows, int64_t cols, int64_t pitch,
                         cudaStream_t st) {
    if (dt != SAT_INT32 && dt != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype %d", (int)dt);
    if (rows < 0 || cols < 0 || pitch < cols) return fail(SAT_ERR_INVALID_VALUE, "bad sizes");
    if (cols == 0) return SAT_OK;
    if (!colsum || (rows > 0 && !src)) return fail(SAT_ERR_INVALID_VALUE, "null pointer");
    if ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(colsum)) & 3u)
        return fail(SAT_ERR_MISALIGNED, "pointers must be 4-byte aligned");
    if (rows == 0) {
        SAT_CUDA(cudaMemsetAsync(colsum, 0, cols * 4, st));
        return SAT_OK;
    }
    int dev = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    int sms = 0;
    sat_status_t s = device_sms(dev, &sms);
    if (s != SAT_OK) return s;
    const bool vec = ((reinterpret_cast<uintptr_t>(src) & 15u) == 0) && (pitch % 4 == 0);
    const int64_t bx = (cols + (vec ? 1023 : 255)) / (vec ? 1024 : 256);
    // one full wave: at most 8 blocks of 256 threads per SM (a partial second wave doubles the time)
    int64_t nseg = (static_cast<int64_t>(sms) * 8) / bx;
    const int64_t max_seg = (rows + 7) / 8;
    if (nseg > max_seg) nseg = max_seg;
    if (nseg > 65535) nseg = 65535;
    if (nseg < 1) nseg = 1;
    const int64_t seg = (rows + nseg - 1) / nseg;
    nseg = (rows + seg - 1) / seg;
    Workspace* w;
    if ((s = find_workspace(dev, st, &w)) != SAT_OK) return s;
    std::lock_guard<std::mutex> wlk(w->mu);
    void* partial;
    if ((s = get_scratch(w, static_cast<size_t>(nseg * cols) * 4, &partial)) != SAT_OK) return s;
    dim3 g1(static_cast<unsigned>(bx), static_cast<unsigned>(nseg));
    if (dt == SAT_INT32) {
        if (vec)
            sat::colsum_partial_kernel<uint32_t, true><<<g1, 256, 0, st>>>(
                static_cast<const uint32_t*>(src), static_cast<uint32_t*>(partial), rows, cols, pitch, seg);
        else
            sat::colsum_partial_kernel<uint32_t, false><<<g1, 256, 0, st>>>(
                static_cast<const uint32_t*>(src), static_cast<uint32_t*>(partial), rows, cols, pitch, seg);
        sat::colsum_reduce_kernel<uint32_t><<<static_cast<unsigned>((cols + 255) / 256), 256, 0, st>>>(
            static_cast<const uint32_t*>(partial), static_cast<uint32_t*>(colsum), cols, static_cast<int>(nseg));
    } else {
        if (vec)
            sat::colsum_partial_kernel<float, true><<<g1, 256, 0, st>>>(
                static_cast<const float*>(src), static_cast<float*>(partial), rows, cols, pitch, seg);
        else
            sat::colsum_partial_kernel<float, false><<<g1, 256, 0, st>>>(
                static_cast<const float*>(src), static_cast<float*>(partial), rows, cols, pitch, seg);
        sat::colsum_reduce_kernel<float><<<static_cast<unsigned>((cols + 255) / 256), 256, 0, st>>>(
            static_cast<const float*>(partial), static_cast<float*>(colsum), cols, static_cast<int>(nseg));
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "colsum kernels");
    return SAT_OK;
}

sat_status_t carry_impl(sat_dtype_t dt, const void* gathered, int nranks, int rank, int64_t cols, void* carry,
                        cudaStream_t st) {
    if (dt != SAT_INT32 && dt != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype %d", (int)dt);
    if (nranks < 1 || rank < 0 || rank >= nranks || cols < 0) return fail(SAT_ERR_INVALID_VALUE, "bad rank/sizes");
    if (cols == 0) return SAT_OK;
    if (!carry || (rank > 0 && !gathered)) return fail(SAT_ERR_INVALID_VALUE, "null pointer");
    if (dt == SAT_INT32)
        sat::carry_prefix_kernel<uint32_t><<<1, 1024, 0, st>>>(static_cast<const uint32_t*>(gathered), rank, cols,
                                                               static_cast<uint32_t*>(carry));
    else
        sat::carry_prefix_kernel<float><<<1, 1024, 0, st>>>(static_cast<const float*>(gathered), rank, cols,
                                                            static_cast<float*>(carry));
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "carry_prefix_kernel");
    return SAT_OK;
}

// ------------------------------------------------------------------ rectangle queries
sat_status_t box_impl(sat_dtype_t dt, const void* b, void* out, int64_t rows, int64_t cols, int64_t pitch, int64_t rh,
                      int64_t rw, cudaStream_t st) {
    if (dt != SAT_INT32 && dt != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype %d", (int)dt);
    if (rh < 0 || rw < 0) return fail(SAT_ERR_INVALID_VALUE, "negative box radius");
    sat_status_t s = validate(b, out, rows, cols, pitch);
    if (s != SAT_OK || rows == 0 || cols == 0) return s;
    if (b == out) return fail(SAT_ERR_INVALID_VALUE, "box sums cannot be computed in place");
    int dev = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    int sms = 0;
    if ((s = device_sms(dev, &sms)) != SAT_OK) return s;
    const int64_t gx = (cols + 1023) / 1024;
    int64_t gy = (static_cast<int64_t>(sms) * 8 + gx - 1) / gx;
    if (gy > rows) gy = rows;
    if (gy > 65535) gy = 65535;
    const dim3 grid(static_cast<unsigned>(gx), static_cast<unsigned>(gy));
    const bool vec = ((reinterpret_cast<uintptr_t>(out) & 15u) == 0) && ((pitch * 4) % 16 == 0);
    // band kernel (production): one wave of sms x occ blocks cut into px column panels x bands row bands,
    // the fewest bands (least re-read halo) whose panel is >= 128 columns wide and whose two rings of
    // kBandQ x kBandRows row segments fit the shared memory of `occ` blocks per SM
    if (vec && ((reinterpret_cast<uintptr_t>(b) & 15u) == 0) && cols % 4 == 0 && rows < (int64_t(1) << 31) - 1 &&
        rh < (1 << 28) && rw < (1 << 20)) {
        using CfgB = sat::BandCfg<8, 1>;  // 8 rows per slot, one slot ahead (measured: 4 blocks/SM, 32K^2 r = 8:
                                          // 1.62 ms; <16, 1> at 2 blocks/SM 2.42 ms; <4, 4> 2.45 ms; <2, 4> 2.93 ms)
        static const int band_occ_max = [] {
            const char* e = std::getenv("SAT_BOX_BAND_OCC");  // tuning switch (0 = staged kernel)
            return e ? std::atoi(e) : 4;
        }();
        // only at 4 blocks per SM (fewer leave the band walk latency-bound: r = 64 at 3 blocks/SM 2.87 ms vs
        // 2.58 ms staged) and while the rows re-read as u stay in L2 (bands x (2 rh + 1) rows <= 48 MB)
        static const int band_cfg = [] {  // tuning switch: 0 = <8,1> (default), 1 = <6,2>, 2 = <4,3>
            const char* e = std::getenv("SAT_BOX_BAND_CFG");
            return e ? std::atoi(e) : 0;
        }();
        for (int occ : {band_occ_max >= 5 ? 5 : 4}) {
            if (occ > band_occ_max) continue;
            const int64_t S = static_cast<int64_t>(sms) * occ;
            const size_t limit = (228 * 1024) / occ - 1024;
            for (int64_t bands = 1; bands <= S && bands <= rows; ++bands) {
                if (S % bands) continue;
                const int64_t px = S / bands;
                const int64_t W = ((cols + px - 1) / px + 3) & ~int64_t(3);
                if (W < 128 && px > 1) continue;
                const int64_t segw = (W + 2 * rw + 8 + 3) & ~int64_t(3);  // 16-byte segment rows
                const size_t bytes = band_cfg == 1 ? sat::BandCfg<6, 2>::smem(segw)
                                     : band_cfg == 2 ? sat::BandCfg<4, 3>::smem(segw) : CfgB::smem(segw);
                if (bytes > limit) break;  // more bands only widen the panels
                if (static_cast<double>(bands) * (2 * rh + 1) * cols * 4 > 48.0 * (1 << 20)) break;
                const int64_t H = (rows + bands - 1) / bands;
                const dim3 g(static_cast<unsigned>((cols + W - 1) / W), static_cast<unsigned>((rows + H - 1) / H));
                auto go = [&](auto cfg) -> cudaError_t {
                    using C = decltype(cfg);
                    const void* k = dt == SAT_INT32 ? reinterpret_cast<const void*>(&sat::box_band_kernel<uint32_t, C>)
                                                    : reinterpret_cast<const void*>(&sat::box_band_kernel<float, C>);
                    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                         static_cast<int>(bytes));
                    if (e != cudaSuccess) return e;
                    if (dt == SAT_INT32)
                        sat::box_band_kernel<uint32_t, C><<<g, 256, bytes, st>>>(
                            static_cast<const uint32_t*>(b), static_cast<uint32_t*>(out), static_cast<int>(rows), cols,
                            pitch, static_cast<int>(rh), static_cast<int>(rw), static_cast<int>(W), static_cast<int>(H),
                            static_cast<int>(segw));
                    else
                        sat::box_band_kernel<float, C><<<g, 256, bytes, st>>>(
                            static_cast<const float*>(b), static_cast<float*>(out), static_cast<int>(rows), cols, pitch,
                            static_cast<int>(rh), static_cast<int>(rw), static_cast<int>(W), static_cast<int>(H),
                            static_cast<int>(segw));
                    return cudaGetLastError();
                };
                cudaError_t e = band_cfg == 1 ? go(sat::BandCfg<6, 2>{}) : band_cfg == 2 ? go(sat::BandCfg<4, 3>{})
                                                                       : go(CfgB{});
                if (e != cudaSuccess) return cuda_fail(e, "box_band_kernel");
                return SAT_OK;
            }
        }
    }
    // staged kernel: both pointers 16-byte aligned and kBoxBufs pairs of row segments in 48 KB
    const int64_t nv = (sat::kBoxPanel + 2 * rw + 8) / 4 + 1;
    const size_t smem = static_cast<size_t>(nv) * 4 * 4 * 2 * sat::kBoxBufs;
    if (vec && ((reinterpret_cast<uintptr_t>(b) & 15u) == 0) && smem <= 48 * 1024) {
        if (dt == SAT_INT32)
            sat::box_sum_smem_kernel<uint32_t><<<grid, sat::kBoxThreads, smem, st>>>(
                static_cast<const uint32_t*>(b), static_cast<uint32_t*>(out), rows, cols, pitch, rh, rw,
                static_cast<int>(nv));
        else
            sat::box_sum_smem_kernel<float><<<grid, sat::kBoxThreads, smem, st>>>(
                static_cast<const float*>(b), static_cast<float*>(out), rows, cols, pitch, rh, rw, static_cast<int>(nv));
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_fail(e, "box_sum_smem_kernel");
        return SAT_OK;
    }
    if (dt == SAT_INT32) {
        const uint32_t* bb = static_cast<const uint32_t*>(b);
        uint32_t* oo = static_cast<uint32_t*>(out);
        if (vec) sat::box_sum_kernel<uint32_t, true><<<grid, 256, 0, st>>>(bb, oo, rows, cols, pitch, rh, rw);
        else sat::box_sum_kernel<uint32_t, false><<<grid, 256, 0, st>>>(bb, oo, rows, cols, pitch, rh, rw);
    } else {
        const float* bb = static_cast<const float*>(b);
        float* oo = static_cast<float*>(out);
        if (vec) sat::box_sum_kernel<float, true><<<grid, 256, 0, st>>>(bb, oo, rows, cols, pitch, rh, rw);
        else sat::box_sum_kernel<float, false><<<grid, 256, 0, st>>>(bb, oo, rows, cols, pitch, rh, rw);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "box_sum_kernel");
    return SAT_OK;
}

sat_status_t rects_impl(sat_dtype_t dt, const void* b, int64_t rows, int64_t cols, int64_t pitch, const int64_t* rects,
                        int64_t n, void* out, cudaStream_t st) {
    if (dt != SAT_INT32 && dt != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype %d", (int)dt);
    if (n < 0 || rows < 0 || cols < 0 || pitch < cols) return fail(SAT_ERR_INVALID_VALUE, "bad sizes");
    if (n == 0) return SAT_OK;
    if (!rects || !out || (rows > 0 && cols > 0 && !b)) return fail(SAT_ERR_INVALID_VALUE, "null pointer");
    if ((reinterpret_cast<uintptr_t>(rects) & 15u) || (reinterpret_cast<uintptr_t>(out) & 3u) ||
        (reinterpret_cast<uintptr_t>(b) & 3u))
        return fail(SAT_ERR_MISALIGNED, "rects must be 16-byte aligned, b and out 4-byte aligned");
    if (rows == 0 || cols == 0) {
        SAT_CUDA(cudaMemsetAsync(out, 0, static_cast<size_t>(n) * 4, st));
        return SAT_OK;
    }
    int64_t blocks = (n + 255) / 256;
    if (blocks > 148 * 32) blocks = 148 * 32;
    if (dt == SAT_INT32)
        sat::rect_sums_kernel<uint32_t><<<static_cast<unsigned>(blocks), 256, 0, st>>>(
            static_cast<const uint32_t*>(b), rows, cols, pitch, rects, n, static_cast<uint32_t*>(out));
    else
        sat::rect_sums_kernel<float><<<static_cast<unsigned>(blocks), 256, 0, st>>>(
            static_cast<const float*>(b), rows, cols, pitch, rects, n, static_cast<float*>(out));
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "rect_sums_kernel");
    return SAT_OK;
}

// ------------------------------------------------------------------ batched small matrices (NEXT-2)
template <typename V, typename TIn, int NWR>
cudaError_t launch_batch(bool vec, unsigned grid, const void* src, void* dst, int64_t batch, int64_t rows,
                         int64_t cols, int64_t pitch, int64_t stride, int64_t spitch, int64_t sstride, cudaStream_t st) {
    const TIn* a = static_cast<const TIn*>(src);
    V* b = static_cast<V*>(dst);
    constexpr int threads = NWR * 32 * sat::kBatchIpb<NWR>;
    if (vec)
        sat::sat_batch_kernel<V, TIn, NWR, true>
            <<<grid, threads, 0, st>>>(a, b, batch, rows, cols, pitch, stride, spitch, sstride);
    else
        sat::sat_batch_kernel<V, TIn, NWR, false>
            <<<grid, threads, 0, st>>>(a, b, batch, rows, cols, pitch, stride, spitch, sstride);
    return cudaGetLastError();
}

template <typename V, typename TIn>
cudaError_t launch_batch_w(int nwr, bool vec, unsigned grid, const void* src, void* dst, int64_t batch, int64_t rows,
                           int64_t cols, int64_t pitch, int64_t stride, int64_t spitch, int64_t sstride,
                           cudaStream_t st) {
    switch (nwr) {
        case 1: return launch_batch<V, TIn, 1>(vec, grid, src, dst, batch, rows, cols, pitch, stride, spitch, sstride, st);
        case 2: return launch_batch<V, TIn, 2>(vec, grid, src, dst, batch, rows, cols, pitch, stride, spitch, sstride, st);
        case 4: return launch_batch<V, TIn, 4>(vec, grid, src, dst, batch, rows, cols, pitch, stride, spitch, sstride, st);
        default: return launch_batch<V, TIn, 8>(vec, grid, src, dst, batch, rows, cols, pitch, stride, spitch, sstride, st);
    }
}

// grid / CTA width of sat_batch_kernel for `batch` matrices of `cols` columns
int batch_nwr(int64_t cols) { return cols <= 128 ? 1 : cols <= 256 ? 2 : cols <= 512 ? 4 : 8; }
sat_status_t batch_grid(int64_t batch, int nwr, unsigned* grid) {
    int dev = 0, sms = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    sat_status_t s = device_sms(dev, &sms);
    if (s != SAT_OK) return s;
    const int64_t cap = static_cast<int64_t>(sms) * 64;  // resident blocks are far fewer; the rest queue
    const int64_t ctas = nwr == 1 ? (batch + 3) / 4 : batch;  // one-warp CTAs hold 4 matrices (kBatchIpb)
    *grid = static_cast<unsigned>(ctas < cap ? ctas : cap);
    return SAT_OK;
}

sat_status_t batched_u8_impl(const void* src, int64_t spitch, int64_t sstride, void* dst, int64_t batch, int64_t rows,
                             int64_t cols, int64_t pitch, int64_t stride, cudaStream_t st) {
    if (batch < 0 || rows < 0 || cols < 0 || pitch < cols || spitch < cols)
        return fail(SAT_ERR_INVALID_VALUE, "bad sizes");
    if (batch == 0 || rows == 0 || cols == 0) return SAT_OK;
    if (!src || !dst) return fail(SAT_ERR_INVALID_VALUE, "null pointer");
    if (reinterpret_cast<uintptr_t>(dst) & 3u) return fail(SAT_ERR_MISALIGNED, "dst must be 4-byte aligned");
    if (rows > (int64_t(1) << 31) - 1 || cols > (int64_t(1) << 31) - 1)
        return fail(SAT_ERR_UNSUPPORTED, "rows and cols must be < 2^31");
    const int64_t span = (rows - 1) * pitch + cols, sspan = (rows - 1) * spitch + cols;
    if (batch > 1 && (stride < span || sstride < sspan))
        return fail(SAT_ERR_INVALID_VALUE, "matrix strides smaller than a matrix (matrices overlap)");
    const uintptr_t a = reinterpret_cast<uintptr_t>(src), b = reinterpret_cast<uintptr_t>(dst);
    const uintptr_t abytes = static_cast<uintptr_t>((batch - 1) * sstride + sspan);
    const uintptr_t bbytes = static_cast<uintptr_t>(((batch - 1) * stride + span) * 4);
    if (a < b + bbytes && b < a + abytes) return fail(SAT_ERR_INVALID_VALUE, "src and dst overlap");
    const bool vec = ((a & 3u) == 0) && ((b & 15u) == 0) && spitch % 4 == 0 && pitch % 4 == 0 &&
                     (batch == 1 || (sstride % 4 == 0 && stride % 4 == 0));
    const int nwr = batch_nwr(cols);
    unsigned grid = 0;
    sat_status_t s = batch_grid(batch, nwr, &grid);
    if (s != SAT_OK) return s;
    const cudaError_t e =
        launch_batch_w<uint32_t, uint8_t>(nwr, vec, grid, src, dst, batch, rows, cols, pitch, stride, spitch, sstride, st);
    if (e != cudaSuccess) return cuda_fail(e, "sat_batch_kernel (u8)");
    return SAT_OK;
}

sat_status_t batched_impl(sat_dtype_t dt, const void* src, void* dst, int64_t batch, int64_t rows, int64_t cols,
                          int64_t pitch, int64_t stride, cudaStream_t st) {
    if (dt != SAT_INT32 && dt != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype %d", (int)dt);
    if (batch < 0) return fail(SAT_ERR_INVALID_VALUE, "negative batch");
    sat_status_t s = validate(batch ? src : nullptr, batch ? dst : nullptr, batch ? rows : 0, cols, pitch);
    if (s != SAT_OK) return s;
    if (batch == 0 || rows == 0 || cols == 0) return SAT_OK;
    const int64_t span = (rows - 1) * pitch + cols;  // elements of one matrix
    if (batch > 1 && stride < span)
        return fail(SAT_ERR_INVALID_VALUE, "image_stride %lld < (rows-1)*pitch+cols = %lld (matrices overlap)",
                    (long long)stride, (long long)span);
    if (src != dst) {
        const uintptr_t bytes = static_cast<uintptr_t>(((batch - 1) * stride + span) * 4);
        const uintptr_t a = reinterpret_cast<uintptr_t>(src), b = reinterpret_cast<uintptr_t>(dst);
        if (a < b + bytes && b < a + bytes) return fail(SAT_ERR_INVALID_VALUE, "src and dst batches partially overlap");
    }
    const bool vec = (((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 15u) == 0) &&
                     (pitch % 4 == 0) && (batch == 1 || stride % 4 == 0);
    const int nwr = batch_nwr(cols);
    unsigned grid = 0;
    s = batch_grid(batch, nwr, &grid);
    if (s != SAT_OK) return s;
    const cudaError_t e =
        dt == SAT_INT32
            ? launch_batch_w<uint32_t, uint32_t>(nwr, vec, grid, src, dst, batch, rows, cols, pitch, stride, pitch, stride, st)
            : launch_batch_w<float, float>(nwr, vec, grid, src, dst, batch, rows, cols, pitch, stride, pitch, stride, st);
    if (e != cudaSuccess) return cuda_fail(e, "sat_batch_kernel");
    return SAT_OK;
}

// ------------------------------------------------------------------ end-to-end host pipeline
// One staging buffer, copy-stream pair and event set per device.  `mu` is held for a whole
// sat_compute_host call (through its final synchronisations), so concurrent calls on one device
// run one after the other instead of sharing the buffer.
constexpr int kHostMaxStrips = 64;
struct Staging {
    std::mutex mu;
    void* buf = nullptr;
    size_t bytes = 0;
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t ev[2 * kHostMaxStrips] = {};
};
std::map<int, Staging*> g_staging;

// ------------------------------------------------------------------ NCCL (dlopen)
#if defined(SAT_HAVE_NCCL_H)
struct NcclApi {
    void* h = nullptr;
    ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*allGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    const char* (*errStr)(ncclResult_t) = nullptr;
};
NcclApi g_nccl;

sat_status_t load_nccl() {
    if (g_nccl.h) return SAT_OK;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return fail(SAT_ERR_NCCL, "dlopen(libnccl.so.2) failed: %s", dlerror());
    g_nccl.getUniqueId = reinterpret_cast<decltype(g_nccl.getUniqueId)>(dlsym(h, "ncclGetUniqueId"));
    g_nccl.commInitRank = reinterpret_cast<decltype(g_nccl.commInitRank)>(dlsym(h, "ncclCommInitRank"));
    g_nccl.commDestroy = reinterpret_cast<decltype(g_nccl.commDestroy)>(dlsym(h, "ncclCommDestroy"));
    g_nccl.allGather = reinterpret_cast<decltype(g_nccl.allGather)>(dlsym(h, "ncclAllGather"));
    g_nccl.errStr = reinterpret_cast<decltype(g_nccl.errStr)>(dlsym(h, "ncclGetErrorString"));
    if (!g_nccl.getUniqueId || !g_nccl.commInitRank || !g_nccl.commDestroy || !g_nccl.allGather || !g_nccl.errStr)
        return fail(SAT_ERR_NCCL, "libnccl.so.2 lacks a required symbol");
    g_nccl.h = h;
    return SAT_OK;
}

sat_status_t nccl_fail(ncclResult_t r, const char* what) {
    return fail(SAT_ERR_NCCL, "%s: %s", what, g_nccl.errStr ? g_nccl.errStr(r) : "?");
}
#endif

}  // namespace

struct sat_comm_s {
#if defined(SAT_HAVE_NCCL_H)
    ncclComm_t comm = nullptr;
#endif
    int nranks = 0, rank = 0, dev = 0;
    void* buf = nullptr;  // colsum [cols] | gathered [nranks*cols] | carry [cols]
    size_t bytes = 0;
};

// ====================================================================== C ABI
SAT_API sat_status_t sat_compute(sat_dtype_t dtype, const void* src, void* dst, int64_t rows, int64_t cols,
                                 int64_t pitch, const void* carry, void* stream) {
    return compute_impl(dtype, src, dst, rows, cols, pitch, carry, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_compute_i32(const int32_t* src, int32_t* dst, int64_t rows, int64_t cols, int64_t pitch,
                                     void* stream) {
    return compute_impl(SAT_INT32, src, dst, rows, cols, pitch, nullptr, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_compute_f32(const float* src, float* dst, int64_t rows, int64_t cols, int64_t pitch,
                                     void* stream) {
    return compute_impl(SAT_FLOAT32, src, dst, rows, cols, pitch, nullptr, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_compute_u8(const uint8_t* src, int64_t src_pitch, uint32_t* dst, int64_t rows, int64_t cols,
                                    int64_t pitch, void* stream) {
    return compute_impl(kU8, src, dst, rows, cols, pitch, nullptr, static_cast<cudaStream_t>(stream), src_pitch);
}

SAT_API sat_status_t sat_compute_f32_f64(const float* src, int64_t src_pitch, double* dst, int64_t dst_pitch,
                                         int64_t rows, int64_t cols, void* stream) {
    return wide_impl(false, src, src_pitch, dst, dst_pitch, rows, cols, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_compute_moments_f32(const float* src, int64_t src_pitch, float* dst, int64_t dst_pitch,
                                             int64_t rows, int64_t cols, void* stream) {
    return wide_impl(true, src, src_pitch, dst, dst_pitch, rows, cols, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_strip_colsum(sat_dtype_t dtype, const void* src, void* colsum, int64_t rows, int64_t cols,
                                      int64_t pitch, void* stream) {
    return colsum_impl(dtype, src, colsum, rows, cols, pitch, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_carry_prefix(sat_dtype_t dtype, const void* gathered, int nranks, int rank, int64_t cols,
                                      void* carry, void* stream) {
    return carry_impl(dtype, gathered, nranks, rank, cols, carry, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_box_sum(sat_dtype_t dtype, const void* sat, void* out, int64_t rows, int64_t cols,
                                 int64_t pitch, int64_t rh, int64_t rw, void* stream) {
    return box_impl(dtype, sat, out, rows, cols, pitch, rh, rw, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_rect_sums(sat_dtype_t dtype, const void* sat, int64_t rows, int64_t cols, int64_t pitch,
                                   const int64_t* rects, int64_t n, void* out, void* stream) {
    return rects_impl(dtype, sat, rows, cols, pitch, rects, n, out, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_compute_batched(sat_dtype_t dtype, const void* src, void* dst, int64_t batch, int64_t rows,
                                         int64_t cols, int64_t pitch, int64_t image_stride, void* stream) {
    return batched_impl(dtype, src, dst, batch, rows, cols, pitch, image_stride, static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_compute_batched_u8(const uint8_t* src, int64_t src_pitch, int64_t src_image_stride,
                                            uint32_t* dst, int64_t batch, int64_t rows, int64_t cols, int64_t pitch,
                                            int64_t image_stride, void* stream) {
    return batched_u8_impl(src, src_pitch, src_image_stride, dst, batch, rows, cols, pitch, image_stride,
                           static_cast<cudaStream_t>(stream));
}

SAT_API sat_status_t sat_compute_host(sat_dtype_t dtype, const void* host_src, void* host_dst, int64_t rows,
                                      int64_t cols, int64_t pitch, void* stream) {
    if (dtype != SAT_INT32 && dtype != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype");
    if (rows < 0 || cols < 0 || pitch < cols) return fail(SAT_ERR_INVALID_VALUE, "bad sizes");
    if (rows == 0 || cols == 0) return SAT_OK;
    if (!host_src || !host_dst) return fail(SAT_ERR_INVALID_VALUE, "null pointer");
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    int dev = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    Staging* sg;
    {
        std::lock_guard<std::mutex> lk(g_mu);
        auto it = g_staging.find(dev);
        if (it == g_staging.end()) it = g_staging.emplace(dev, new Staging()).first;
        sg = it->second;
    }
    std::lock_guard<std::mutex> slk(sg->mu);
    const size_t bytes = static_cast<size_t>(rows) * pitch * 4;
    if (!sg->h2d) {
        SAT_CUDA(cudaStreamCreateWithFlags(&sg->h2d, cudaStreamNonBlocking));
        SAT_CUDA(cudaStreamCreateWithFlags(&sg->d2h, cudaStreamNonBlocking));
        for (auto& e : sg->ev) SAT_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    if (bytes > sg->bytes) {
        // the previous call synchronised all three streams before releasing sg->mu
        if (sg->buf) SAT_CUDA(cudaFree(sg->buf));
        sg->buf = nullptr;
        sg->bytes = 0;
        cudaError_t e = cudaMalloc(&sg->buf, bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(SAT_ERR_OUT_OF_MEMORY, "staging buffer (%zu bytes)", bytes);
        }
        sg->bytes = bytes;
    }
    // strips of >= 2 MiB, at most kHostMaxStrips, multiples of 128 rows
    const int64_t row_bytes = pitch * 4;
    int64_t nstrips = (rows * row_bytes) / (int64_t(2) << 20);
    if (nstrips < 1) nstrips = 1;
    if (nstrips > kHostMaxStrips) nstrips = kHostMaxStrips;
    int64_t h = (rows + nstrips - 1) / nstrips;
    h = ((h + 127) / 128) * 128;
    nstrips = (rows + h - 1) / h;
    sat_status_t status = SAT_OK;
    char* dbuf = static_cast<char*>(sg->buf);
    for (int64_t k = 0; k < nstrips && status == SAT_OK; ++k) {
        const int64_t r0 = k * h;
        const int64_t nr = (r0 + h <= rows) ? h : rows - r0;
        char* dstrip = dbuf + r0 * row_bytes;
        const char* hs = static_cast<const char*>(host_src) + r0 * row_bytes;
        char* hd = static_cast<char*>(host_dst) + r0 * row_bytes;
        cudaError_t e = cudaMemcpy2DAsync(dstrip, row_bytes, hs, row_bytes, cols * 4, nr, cudaMemcpyHostToDevice,
                                          sg->h2d);
        if (e == cudaSuccess) e = cudaEventRecord(sg->ev[2 * k], sg->h2d);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(st, sg->ev[2 * k], 0);
        if (e != cudaSuccess) {
            status = cuda_fail(e, "host pipeline H2D");
            break;
        }
        const void* carry = (k > 0) ? static_cast<const void*>(dstrip - row_bytes) : nullptr;
        status = compute_impl(dtype, dstrip, dstrip, nr, cols, pitch, carry, st);
        if (status != SAT_OK) break;
        e = cudaEventRecord(sg->ev[2 * k + 1], st);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(sg->d2h, sg->ev[2 * k + 1], 0);
        if (e == cudaSuccess)
            e = cudaMemcpy2DAsync(hd, row_bytes, dstrip, row_bytes, cols * 4, nr, cudaMemcpyDeviceToHost, sg->d2h);
        if (e != cudaSuccess) status = cuda_fail(e, "host pipeline D2H");
    }
    cudaError_t e1 = cudaStreamSynchronize(sg->d2h);
    cudaError_t e2 = cudaStreamSynchronize(st);
    cudaError_t e3 = cudaStreamSynchronize(sg->h2d);
    if (status != SAT_OK) return status;
    if (e1 != cudaSuccess) return cuda_fail(e1, "host pipeline sync");
    if (e2 != cudaSuccess) return cuda_fail(e2, "host pipeline sync");
    if (e3 != cudaSuccess) return cuda_fail(e3, "host pipeline sync");
    return SAT_OK;
}

SAT_API sat_status_t sat_comm_get_unique_id(unsigned char id[128]) {
#if defined(SAT_HAVE_NCCL_H)
    if (!id) return fail(SAT_ERR_INVALID_VALUE, "null id");
    sat_status_t s = load_nccl();
    if (s != SAT_OK) return s;
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    ncclUniqueId uid;
    ncclResult_t r = g_nccl.getUniqueId(&uid);
    if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
    std::memcpy(id, &uid, 128);
    return SAT_OK;
#else
    (void)id;
    return fail(SAT_ERR_UNSUPPORTED, "libsat was built without nccl.h");
#endif
}

SAT_API sat_status_t sat_comm_init(sat_comm_t* comm, const unsigned char id[128], int nranks, int rank) {
#if defined(SAT_HAVE_NCCL_H)
    if (!comm || !id || nranks < 1 || rank < 0 || rank >= nranks) return fail(SAT_ERR_INVALID_VALUE, "bad args");
    sat_status_t s = load_nccl();
    if (s != SAT_OK) return s;
    auto* c = new sat_comm_s();
    c->nranks = nranks;
    c->rank = rank;
    cudaGetDevice(&c->dev);
    ncclUniqueId uid;
    std::memcpy(&uid, id, 128);
    ncclResult_t r = g_nccl.commInitRank(&c->comm, nranks, uid, rank);
    if (r != ncclSuccess) {
        delete c;
        return nccl_fail(r, "ncclCommInitRank");
    }
    *comm = c;
    return SAT_OK;
#else
    (void)comm; (void)id; (void)nranks; (void)rank;
    return fail(SAT_ERR_UNSUPPORTED, "libsat was built without nccl.h");
#endif
}

SAT_API sat_status_t sat_comm_destroy(sat_comm_t comm) {
    if (!comm) return SAT_OK;
#if defined(SAT_HAVE_NCCL_H)
    if (comm->comm) g_nccl.commDestroy(comm->comm);
#endif
    if (comm->buf) cudaFree(comm->buf);
    delete comm;
    return SAT_OK;
}

SAT_API sat_status_t sat_compute_sharded(sat_comm_t comm, sat_dtype_t dtype, const void* strip_src, void* strip_dst,
                                         int64_t strip_rows, int64_t cols, int64_t pitch, void* stream) {
#if defined(SAT_HAVE_NCCL_H)
    if (!comm) return fail(SAT_ERR_INVALID_VALUE, "null comm");
    if (dtype != SAT_INT32 && dtype != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype");
    if (cols <= 0) return fail(SAT_ERR_INVALID_VALUE, "bad sizes");  // cols, dtype, comm: equal on all ranks
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const size_t need = static_cast<size_t>(cols) * 4 * (comm->nranks + 2);
    if (need > comm->bytes) {
        if (comm->buf) SAT_CUDA(cudaFree(comm->buf));
        comm->buf = nullptr;
        comm->bytes = 0;
        cudaError_t e = cudaMalloc(&comm->buf, need);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(SAT_ERR_OUT_OF_MEMORY, "sharded buffers");
        }
        comm->bytes = need;
    }
    char* base = static_cast<char*>(comm->buf);
    void* colsum = base;
    void* gathered = base + cols * 4;
    void* carry = base + cols * 4 * (comm->nranks + 1);
    // Every rank-local check runs before the collective.  A rank whose arguments or column-sum launch
    // fail still joins the all-gather (with a zero vector) so that no other rank blocks in it, then
    // returns its own error.
    sat_status_t local = (strip_rows < 0 || pitch < cols)
                             ? fail(SAT_ERR_INVALID_VALUE, "bad sizes strip_rows=%lld pitch=%lld", (long long)strip_rows,
                                    (long long)pitch)
                             : (strip_rows > 0 ? validate(strip_src, strip_dst, strip_rows, cols, pitch) : SAT_OK);
    if (local == SAT_OK) local = colsum_impl(dtype, strip_src, colsum, strip_rows, cols, pitch, st);
    if (local != SAT_OK) {
        const std::string detail = g_detail;
        cudaMemsetAsync(colsum, 0, cols * 4, st);
        g_nccl.allGather(colsum, gathered, static_cast<size_t>(cols), dtype == SAT_INT32 ? ncclUint32 : ncclFloat32,
                         comm->comm, st);
        g_detail = detail;
        return local;
    }
    ncclResult_t r = g_nccl.allGather(colsum, gathered, static_cast<size_t>(cols),
                                      dtype == SAT_INT32 ? ncclUint32 : ncclFloat32, comm->comm, st);
    if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather");
    sat_status_t s;
    if ((s = carry_impl(dtype, gathered, comm->nranks, comm->rank, cols, carry, st)) != SAT_OK) return s;
    if (strip_rows == 0) return SAT_OK;
    return compute_impl(dtype, strip_src, strip_dst, strip_rows, cols, pitch, carry, st);
#else
    (void)comm; (void)dtype; (void)strip_src; (void)strip_dst; (void)strip_rows; (void)cols; (void)pitch; (void)stream;
    return fail(SAT_ERR_UNSUPPORTED, "libsat was built without nccl.h");
#endif
}

// ====================================================================== chained strip partition
// (DESIGN.md Sec. 7): one persistent launch per rank and call, the strip column
// sums travel rank -> downstream ranks inside the kernels through peer-mapped inbox memory.
struct sat_chain_s {
    std::mutex mu;
    int nranks = 0, rank = 0, dev = 0;
    int64_t cols = 0, inbox_cols = 0;
    void* mem = nullptr;  // exported: inbox [2][inbox_cols] uint64 | done [kMaxChainRanks] uint32
    size_t inbox_bytes = 0, mem_bytes = 0;
    void* peer[sat::kMaxChainRanks] = {};
    bool opened[sat::kMaxChainRanks] = {};
    uint64_t calls = 0;
    Ctrl* ctrl = nullptr;
    uint64_t* slots = nullptr;
    size_t slot_words = 0;
};

SAT_API sat_status_t sat_chain_create(int nranks, int rank, int64_t cols, sat_chain_t* out) {
    if (!out || nranks < 1 || nranks > sat::kMaxChainRanks || rank < 0 || rank >= nranks || cols < 1 ||
        cols > (int64_t(1) << 31) - 1)
        return fail(SAT_ERR_INVALID_VALUE, "bad chain arguments (nranks %d, rank %d, cols %lld; nranks <= %d)", nranks,
                    rank, (long long)cols, sat::kMaxChainRanks);
    auto* c = new sat_chain_s();
    c->nranks = nranks;
    c->rank = rank;
    c->cols = cols;
    c->inbox_cols = (cols + 255) / 256 * 256;  // whole tiles of the widest chain configuration (TC = 256)
    c->inbox_bytes = static_cast<size_t>(2) * c->inbox_cols * 8;
    c->mem_bytes = c->inbox_bytes + 256;
    cudaError_t e = cudaGetDevice(&c->dev);
    if (e == cudaSuccess) e = cudaMalloc(&c->mem, c->mem_bytes);  // cudaMalloc: exportable with cudaIpcGetMemHandle
    if (e == cudaSuccess) e = cudaMemset(c->mem, 0, c->mem_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&c->ctrl, 256);
    if (e == cudaSuccess) e = cudaMemset(c->ctrl, 0, 256);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        cudaGetLastError();
        if (c->mem) cudaFree(c->mem);
        if (c->ctrl) cudaFree(c->ctrl);
        delete c;
        return fail(SAT_ERR_OUT_OF_MEMORY, "chain buffers: %s", cudaGetErrorString(e));
    }
    c->peer[rank] = c->mem;
    *out = c;
    return SAT_OK;
}

SAT_API sat_status_t sat_chain_export(sat_chain_t chain, unsigned char handle[64]) {
    if (!chain || !handle) return fail(SAT_ERR_INVALID_VALUE, "null argument");
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "cudaIpcMemHandle_t size");
    cudaIpcMemHandle_t h;
    SAT_CUDA(cudaIpcGetMemHandle(&h, chain->mem));
    std::memcpy(handle, &h, 64);
    return SAT_OK;
}

SAT_API sat_status_t sat_chain_connect(sat_chain_t chain, const unsigned char* handles) {
    if (!chain || !handles) return fail(SAT_ERR_INVALID_VALUE, "null argument");
    std::lock_guard<std::mutex> lk(chain->mu);
    for (int g = 0; g < chain->nranks; ++g) {
        if (g == chain->rank || chain->peer[g]) continue;
        cudaIpcMemHandle_t h;
        std::memcpy(&h, handles + 64 * g, 64);
        void* ptr = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle (chain peer)");
        chain->peer[g] = ptr;
        chain->opened[g] = true;
    }
    return SAT_OK;
}

SAT_API sat_status_t sat_chain_connect_local(sat_chain_t* chains, int n) {
    if (!chains || n < 1 || n > sat::kMaxChainRanks) return fail(SAT_ERR_INVALID_VALUE, "bad chain list");
    for (int r = 0; r < n; ++r)
        if (!chains[r] || chains[r]->nranks != n || chains[r]->rank != r || chains[r]->dev != chains[0]->dev ||
            chains[r]->cols != chains[0]->cols)
            return fail(SAT_ERR_INVALID_VALUE, "chains[r] must be rank r of %d on one device with equal cols", n);
    for (int r = 0; r < n; ++r)
        for (int g = 0; g < n; ++g) chains[r]->peer[g] = chains[g]->mem;
    return SAT_OK;
}

SAT_API sat_status_t sat_chain_destroy(sat_chain_t chain) {
    if (!chain) return SAT_OK;
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(chain->dev);
    cudaDeviceSynchronize();
    for (int g = 0; g < chain->nranks; ++g)
        if (chain->opened[g]) cudaIpcCloseMemHandle(chain->peer[g]);
    if (chain->slots) cudaFree(chain->slots);
    if (chain->ctrl) cudaFree(chain->ctrl);
    if (chain->mem) cudaFree(chain->mem);
    cudaSetDevice(cur);
    delete chain;
    cudaGetLastError();
    return SAT_OK;
}

// Tile order of a chained strip with R tile rows: anti-diagonal over groups of g vertically adjacent tiles
// (order 3, tile_of_serial), g the largest of 8, 4, 2 dividing R: the strip's bottom tile of column J
// resolves R/g group diagonals after its top tile -- the chain's lag per rank, (R/g) / (R/g + C) of a
// strip -- and a column look-back spans the g - 1 tiles above in the group
// plus the inclusive word of the group above (a few poll rounds).  SAT_CHAIN_ORDER overrides it (tuning:
// 2 = column-major).
int chain_order(int R) {
    if (const char* e = std::getenv("SAT_CHAIN_ORDER")) return std::atoi(e);
    for (int g : {8, 4, 2})
        if (R % g == 0) return 3 | (g << 8);
    return 3;
}

SAT_API sat_status_t sat_compute_chained(sat_chain_t chain, sat_dtype_t dtype, const void* strip_src, void* strip_dst,
                                         int64_t strip_rows, int64_t cols, int64_t pitch, void* stream) {
    if (!chain) return fail(SAT_ERR_INVALID_VALUE, "null chain");
    if (dtype != SAT_INT32 && dtype != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype %d", (int)dtype);
    if (cols != chain->cols) return fail(SAT_ERR_INVALID_VALUE, "cols %lld != the chain's %lld", (long long)cols,
                                         (long long)chain->cols);
    if (strip_rows < 1) return fail(SAT_ERR_INVALID_VALUE, "chained strips need >= 1 row per rank");
    sat_status_t s = validate(strip_src, strip_dst, strip_rows, cols, pitch);
    if (s != SAT_OK) return s;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    std::lock_guard<std::mutex> lk(chain->mu);
    for (int g = 0; g < chain->nranks; ++g)
        if (!chain->peer[g]) return fail(SAT_ERR_INVALID_VALUE, "chain not connected (rank %d)", g);
    if (chain->calls + 2 >= sat::kEpochMax) return fail(SAT_ERR_UNSUPPORTED, "chain epoch exhausted: recreate it");
    Plan pl;
    int cvi = kVarChain;
    {
        std::lock_guard<std::mutex> g(g_mu);
        if (g_variant >= 0 && g_variant < static_cast<int>(variants().size()) && variants()[g_variant].chain)
            cvi = g_variant;  // tuning hook: another chained configuration
    }
    if ((s = make_plan(strip_rows, cols, pitch, strip_src, strip_dst, &pl, false, 0, cvi)) != SAT_OK) return s;
    const Variant& v = variants()[cvi];
    int dev = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    if (dev != chain->dev) return fail(SAT_ERR_INVALID_VALUE, "chain lives on device %d, current device %d", chain->dev, dev);
    int occ = 0, sms = 0, max_ctas = 0;
    {
        std::lock_guard<std::mutex> g(g_mu);
        if ((s = occupancy(dev, cvi, dtype, pl.tma, false, &occ)) != SAT_OK) return s;
        DeviceInfo* di = nullptr;
        if ((s = device_info(dev, &di)) != SAT_OK) return s;
        sms = di->sms;
        max_ctas = g_max_ctas;
    }
    int64_t grid = static_cast<int64_t>(sms) * occ;
    if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;
    if (grid > pl.ntiles) grid = pl.ntiles;
    const size_t words = static_cast<size_t>(pl.ntiles) * (v.TR + v.TC + 1);
    if (words > chain->slot_words) {
        const size_t want = words + words / 4;
        if (chain->slots) SAT_CUDA(cudaFreeAsync(chain->slots, st));
        chain->slots = nullptr;
        chain->slot_words = 0;
        cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&chain->slots), want * 8, st);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(SAT_ERR_OUT_OF_MEMORY, "chain slots (%zu bytes)", want * 8);
        }
        SAT_CUDA(cudaMemsetAsync(chain->slots, 0, want * 8, st));
        chain->slot_words = want;
    }
    CUtensorMap mi, mo;
    std::memset(&mi, 0, sizeof(mi));
    std::memset(&mo, 0, sizeof(mo));
    if (pl.tma) {
        if ((s = get_encoder()) != SAT_OK) return s;
        if ((s = encode_map(&mi, dtype, strip_src, strip_rows, cols, pitch, v.TR, v.TB)) != SAT_OK) return s;
        if ((s = encode_map(&mo, dtype, strip_dst, strip_rows, cols, pitch, v.OBR, v.TB)) != SAT_OK) return s;
    }
    const uint32_t epoch = static_cast<uint32_t>(chain->calls + 1);
    KParams<uint32_t> p;
    std::memset(&p, 0, sizeof(p));
    p.src = static_cast<const uint32_t*>(strip_src);
    p.dst = static_cast<uint32_t*>(strip_dst);
    p.rows = strip_rows;
    p.cols = cols;
    p.pitch = pitch;
    p.R = pl.R;
    p.C = pl.C;
    p.ntiles = static_cast<int>(pl.ntiles);
    p.order = chain_order(pl.R);
    p.l2_prefetch = l2_prefetch_mode(cvi);
    p.row_slots = chain->slots;
    p.col_slots = chain->slots + static_cast<size_t>(pl.ntiles) * v.TR;
    p.corner_slots = chain->slots + static_cast<size_t>(pl.ntiles) * (v.TR + v.TC);
    p.ctrl = chain->ctrl;
    p.carry = nullptr;
    p.src_pitch = pitch;
    p.epoch_override = epoch;
    p.chain.rank = chain->rank;
    p.chain.nranks = chain->nranks;
    p.chain.parity = epoch & 1u;
    p.chain.inbox_cols = chain->inbox_cols;
    for (int g = 0; g < chain->nranks; ++g) {
        p.chain.peer_inbox[g] = static_cast<uint64_t*>(chain->peer[g]);
        p.chain.peer_done[g] = reinterpret_cast<uint32_t*>(static_cast<char*>(chain->peer[g]) + chain->inbox_bytes);
    }
    cudaError_t e = v.launch[dtype](pl.tma, false, dim3(static_cast<unsigned>(grid)), st, mi, mo, &p);
    if (e != cudaSuccess) return cuda_fail(e, "chained SAT kernel launch");
    chain->calls++;
    return SAT_OK;
}

SAT_API sat_status_t sat_query_plan(sat_dtype_t dtype, int64_t rows, int64_t cols, int64_t pitch, const void* src,
                                    const void* dst, sat_plan_t* plan) {
    if (!plan) return fail(SAT_ERR_INVALID_VALUE, "null plan");
    if (dtype != SAT_INT32 && dtype != SAT_FLOAT32) return fail(SAT_ERR_INVALID_VALUE, "unknown dtype");
    if (rows <= 0 || cols <= 0 || pitch < cols) return fail(SAT_ERR_INVALID_VALUE, "bad sizes");
    Plan pl;
    sat_status_t s = make_plan(rows, cols, pitch, src, dst, &pl);
    if (s != SAT_OK) return s;
    const Variant& v = variants()[pl.vi];
    plan->tile_rows = v.TR;
    plan->tile_cols = v.TC;
    plan->tma = pl.tma ? 1 : 0;
    plan->tiles = pl.ntiles;
    plan->aux_bytes = pl.ntiles * (v.TR + v.TC + 1) * 8;
    plan->variant = pl.vi;
    plan->order = pl.order;
    plan->family = v.family;
    plan->reserved = 0;
    plan->ctas = 0;
    int dev = 0;
    if (cudaGetDevice(&dev) == cudaSuccess) {
        std::lock_guard<std::mutex> lk(g_mu);
        int occ = 0;
        DeviceInfo* di = nullptr;
        if (occupancy(dev, pl.vi, dtype, pl.tma, false, &occ) == SAT_OK && device_info(dev, &di) == SAT_OK) {
            int per_sm = (g_ctas_per_sm > 0 && g_ctas_per_sm < occ) ? g_ctas_per_sm : occ;
            int64_t grid = static_cast<int64_t>(di->sms) * per_sm;
            if (g_max_ctas > 0 && grid > g_max_ctas) grid = g_max_ctas;
            plan->ctas = static_cast<int32_t>(grid < pl.ntiles ? grid : pl.ntiles);
        }
    }
    cudaGetLastError();  // a CPU-only host has no device: plan->ctas stays 0
    return SAT_OK;
}

SAT_API sat_status_t sat_set_tuning(int variant, int order, int ctas_per_sm) {
    if (variant < -1 || variant >= static_cast<int>(variants().size()))
        return fail(SAT_ERR_INVALID_VALUE, "unknown variant %d", variant);
#if SAT_STATS
    if (order < 0 || (order & 15) > 1 || order > 0xffff) return fail(SAT_ERR_INVALID_VALUE, "unknown order %d", order);
#else
    if (order < 0 || (order & ~0xff0f) != 0 || (order & 15) > 3)
        return fail(SAT_ERR_INVALID_VALUE, "unknown order %d", order);
#endif
    if (ctas_per_sm < 0) return fail(SAT_ERR_INVALID_VALUE, "ctas_per_sm < 0");
    std::lock_guard<std::mutex> lk(g_mu);
    g_variant = variant;
    g_order = order;
    g_ctas_per_sm = ctas_per_sm;
    return SAT_OK;
}

SAT_API sat_status_t sat_set_max_ctas(int max_ctas) {
    if (max_ctas < 0) return fail(SAT_ERR_INVALID_VALUE, "max_ctas < 0");
    std::lock_guard<std::mutex> lk(g_mu);
    g_max_ctas = max_ctas;
    return SAT_OK;
}

SAT_API int sat_num_variants(void) { return static_cast<int>(variants().size()); }

SAT_API sat_status_t sat_debug_occupy(int ctas, int64_t ns, int64_t smem_bytes, void* stream) {
    if (ctas < 1 || ns < 0 || ns > 10000000000LL || smem_bytes < 0 || smem_bytes > 227 * 1024)
        return fail(SAT_ERR_INVALID_VALUE, "bad occupy arguments");
    const int smem = static_cast<int>(smem_bytes);
    SAT_CUDA(cudaFuncSetAttribute(reinterpret_cast<const void*>(&sat::occupy_kernel),
                                  cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    sat::occupy_kernel<<<ctas, 32, smem, static_cast<cudaStream_t>(stream)>>>(static_cast<long long>(ns));
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "occupy_kernel");
    return SAT_OK;
}

SAT_API sat_status_t sat_variant_info(int variant, int32_t* tile_rows, int32_t* tile_cols) {
    if (variant < 0 || variant >= static_cast<int>(variants().size()))
        return fail(SAT_ERR_INVALID_VALUE, "unknown variant %d", variant);
    if (tile_rows) *tile_rows = variants()[variant].TR;
    if (tile_cols) *tile_cols = variants()[variant].TC;
    return SAT_OK;
}

SAT_API sat_status_t sat_debug_tile_order(int64_t R, int64_t C, int order, int32_t* out, void* stream) {
    if (R <= 0 || C <= 0 || R * C > (int64_t(1) << 30) || !out || order < 0 || (order & ~0xff0f) != 0 ||
        (order & 15) > 3)
        return fail(SAT_ERR_INVALID_VALUE, "bad args");
    const int64_t n = R * C;
    int blocks = static_cast<int>((n + 255) / 256);
    if (blocks > 4096) blocks = 4096;
    sat::tile_order_kernel<<<blocks, 256, 0, static_cast<cudaStream_t>(stream)>>>(static_cast<int>(R),
                                                                                  static_cast<int>(C), order, out);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "tile_order_kernel");
    return SAT_OK;
}

SAT_API sat_status_t sat_debug_stats(int64_t* out, int max_ctas, int* n_ctas, int* n_stats) {
#if SAT_STATS
    std::lock_guard<std::mutex> lk(g_mu);
    if (!g_last_stats || !out || !n_ctas || !n_stats) return fail(SAT_ERR_INVALID_VALUE, "no stats");
    Workspace* w = g_last_stats;
    const int n = w->stats_ctas < max_ctas ? w->stats_ctas : max_ctas;
    SAT_CUDA(cudaStreamSynchronize(w->stream));
    SAT_CUDA(cudaMemcpy(out, w->stats, static_cast<size_t>(n) * sat::kNumStats * 8, cudaMemcpyDeviceToHost));
    *n_ctas = n;
    *n_stats = sat::kNumStats;
    return SAT_OK;
#else
    (void)out; (void)max_ctas; (void)n_ctas; (void)n_stats;
    return fail(SAT_ERR_UNSUPPORTED, "libsat built without SAT_STATS");
#endif
}

SAT_API sat_status_t sat_debug_trace(int64_t* out, int64_t max_tiles, int64_t* n_tiles) {
#if SAT_STATS
    std::lock_guard<std::mutex> lk(g_mu);
    if (!g_last_stats || !out || !n_tiles) return fail(SAT_ERR_INVALID_VALUE, "no trace");
    Workspace* w = g_last_stats;
    const int64_t n = w->trace_tiles < max_tiles ? w->trace_tiles : max_tiles;
    SAT_CUDA(cudaStreamSynchronize(w->stream));
    SAT_CUDA(cudaMemcpy(out, w->stats + static_cast<size_t>(w->stats_ctas) * sat::kNumStats,
                        static_cast<size_t>(n) * 64, cudaMemcpyDeviceToHost));
    *n_tiles = n;
    return SAT_OK;
#else
    (void)out; (void)max_tiles; (void)n_tiles;
    return fail(SAT_ERR_UNSUPPORTED, "libsat built without SAT_STATS");
#endif
}

SAT_API sat_status_t sat_release_stream_workspace(void* stream) {
    int dev = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    Workspace* w = nullptr;
    {
        std::lock_guard<std::mutex> lk(g_mu);
        auto it = g_ws.find(std::make_pair(dev, static_cast<cudaStream_t>(stream)));
        if (it == g_ws.end()) return SAT_OK;
        w = it->second;
        g_ws.erase(it);
        if (g_last_stats == w) g_last_stats = nullptr;
    }
    free_workspace(w);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "release");
    return SAT_OK;
}

SAT_API sat_status_t sat_debug_workspace(void* stream, uint64_t* host_out, int64_t max_words, sat_ws_info_t* info) {
    if (!info) return fail(SAT_ERR_INVALID_VALUE, "null info");
    int dev = 0;
    SAT_CUDA(cudaGetDevice(&dev));
    Workspace* w = nullptr;
    {
        std::lock_guard<std::mutex> lk(g_mu);
        auto it = g_ws.find(std::make_pair(dev, static_cast<cudaStream_t>(stream)));
        if (it == g_ws.end()) return fail(SAT_ERR_INVALID_VALUE, "no workspace for this (device, stream)");
        w = it->second;
    }
    std::lock_guard<std::mutex> wlk(w->mu);
    const int64_t tiles = static_cast<int64_t>(w->last_R) * w->last_C;
    info->tile_rows = w->last_TR;
    info->tile_cols = w->last_TC;
    info->R = w->last_R;
    info->C = w->last_C;
    info->words = tiles * (w->last_TR + w->last_TC + 1);
    if (!host_out) return SAT_OK;
    if (max_words < info->words) return fail(SAT_ERR_INVALID_VALUE, "host_out holds %lld < %lld words",
                                             (long long)max_words, (long long)info->words);
    SAT_CUDA(cudaStreamSynchronize(w->stream));
    if (info->words > 0)
        SAT_CUDA(cudaMemcpy(host_out, w->slots, static_cast<size_t>(info->words) * 8, cudaMemcpyDeviceToHost));
    return SAT_OK;
}

SAT_API sat_status_t sat_release_workspaces(void) {
    std::lock_guard<std::mutex> lk(g_mu);
    int cur = 0;
    cudaGetDevice(&cur);
    for (auto& kv : g_ws) {
        cudaSetDevice(kv.second->dev);
        free_workspace(kv.second);
    }
    g_ws.clear();
    g_last_stats = nullptr;
    for (auto& kv : g_staging) {
        cudaSetDevice(kv.first);
        Staging* sg = kv.second;
        {
            std::lock_guard<std::mutex> slk(sg->mu);
            if (sg->buf) cudaFree(sg->buf);
            if (sg->h2d) {
                cudaStreamDestroy(sg->h2d);
                cudaStreamDestroy(sg->d2h);
                for (auto& e : sg->ev) cudaEventDestroy(e);
            }
        }
        delete sg;
    }
    g_staging.clear();
    cudaSetDevice(cur);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "release");
    return SAT_OK;
}

SAT_API const char* sat_status_string(sat_status_t s) {
    switch (s) {
        case SAT_OK: return "SAT_OK";
        case SAT_ERR_INVALID_VALUE: return "SAT_ERR_INVALID_VALUE";
        case SAT_ERR_MISALIGNED: return "SAT_ERR_MISALIGNED";
        case SAT_ERR_UNSUPPORTED: return "SAT_ERR_UNSUPPORTED";
        case SAT_ERR_OUT_OF_MEMORY: return "SAT_ERR_OUT_OF_MEMORY";
        case SAT_ERR_CUDA: return "SAT_ERR_CUDA";
        case SAT_ERR_NCCL: return "SAT_ERR_NCCL";
    }
    return "SAT_ERR_UNKNOWN";
}

SAT_API const char* sat_last_error_detail(void) { return g_detail.c_str(); }

SAT_API int sat_version(void) { return SAT_VERSION; }
