// sat_pipe.cuh -- pipeline plumbing shared by the persistent SAT kernels (sat_tm_kernel.cuh, and the
// experimental sat_ws_kernel.cuh): mbarrier arrive / try / test, named barriers, the tile-ring slot
// counter, the end-of-tiles test of the walkers, the kernel exit (ticket counter reset and epoch
// advance by the last CTA out, R12) and the per-CTA stats counters of SAT_STATS builds.
#pragma once

#include "sat_kernel.cuh"

namespace sat {

// Stats builds (-DSAT_STATS=1): per-CTA counters in shared memory, role-tagged slots.
enum WsStat {
    kWsTiles = 0, kWsFullWait, kWsLocal, kWsWalkWait, kWsFinish, kWsRowRounds, kWsColRounds,
    kWsStResultWait, kWsStStore, kWsLdIssue, kWsLdEmptyWait, kWsBandBar, kWsRowTiles, kWsColTiles,
    kWsRowRoundCyc, kWsColRoundCyc, kWsRowResolve, kWsColResolve, kWsRowIdle, kWsColIdle, kWsRowLat, kWsColLat,
    kWsFastHits, kWsScan
};
#if SAT_STATS
__shared__ unsigned long long ws_stats[kNumStats];
#define WS_ST(k, v) atomicAdd(&ws_stats[k], static_cast<unsigned long long>(v))
#else
#define WS_ST(k, v) (void)0
#endif

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}

// One bounded try_wait (the hardware may suspend the thread a while before reporting "not yet").
__device__ __forceinline__ bool mbar_try(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(smem_addr(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

// Non-blocking probe of an mbarrier phase.
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(smem_addr(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Position of tile k in the stage ring: stage s = k % STAGES, barrier phase parity (k / STAGES) & 1,
// advanced incrementally (no division in the loops).
template <int STAGES>
struct Slot {
    int k = 0, s = 0;
    uint32_t ph = 0;
    __device__ __forceinline__ void next() {
        ++k;
        if (++s == STAGES) { s = 0; ph ^= 1u; }
    }
};

// Walkers only wait for their next tile's acquisition; once the loader has drawn the end marker they
// stop.  Returns false when tile k will never exist.
template <typename SM>
__device__ __forceinline__ bool wait_acquired(SM& sm, int s, uint32_t parity, int k) {
    SAT_SPIN_DECL;
    while (!mbar_try(&sm.acq[s], parity)) {
        if (k >= *reinterpret_cast<volatile int*>(&sm.end_n)) return false;
        SAT_SPIN_CHECK("a tile acquisition");
    }
    return true;
}

// Kernel exit (one thread per CTA, after all its tiles are stored): the last CTA out resets the ticket
// counter and advances the epoch for the next launch (R9).
template <typename V>
__device__ __forceinline__ void ws_exit(const KParams<V>& p, uint32_t epoch) {
    __threadfence();
    const unsigned int done = atomicAdd(&p.ctrl->exit_count, 1u);
#if SAT_STATS
    if (p.stats)
        for (int k = 0; k < kNumStats; ++k)
            p.stats[static_cast<long long>(blockIdx.x) * kNumStats + k] = static_cast<long long>(ws_stats[k]);
#endif
    if (done == gridDim.x - 1) {
        p.ctrl->counter = 0u;
        p.ctrl->exit_count = 0u;
        if (p.epoch_override == 0u) p.ctrl->epoch = (epoch >= kEpochMax) ? 1u : epoch + 1u;
        __threadfence();
        // chained strips: every CTA of this rank is done reading its inbox for this call; tell the rank
        // above (the only writer of this inbox), which may then reuse this parity two calls later
        if (p.chain.rank > 0) st_relaxed_sys_u32(p.chain.peer_done[p.chain.rank - 1] + p.chain.rank, epoch);
    }
}

}  // namespace sat
