// sat_tm_kernel.cuh -- single-pass SAT kernel for sm_100a with the local SAT parked in tensor memory.
//
// The method is 1R1W-SKSS-LB of PAPER.md Sec. IV with prefix-form slots and epoch-tagged
// status words (sat_kernel.cuh).  What this kernel is built around is where a tile waits for its
// look-backs: with HBM saturated a look-back round trip costs ~1 us on B200, so a compute warp that
// held its tile until the walks land would idle and pin a 64 KiB stage (the superseded warp-
// specialised sat_ws_kernel, now only in -DSAT_EXPERIMENTAL tuning builds).  Here:
//
//   * a tile's pixels are read out of their input stage into registers right away and the stage is
//     handed back to the loader (the ring refills while the tile is still being computed);
//   * after the local SAT and the local aggregates (Steps 2.A.1, 2.B.1) each compute warp
//     parks its 8x128 block in TMEM (tcgen05.st; 2 slots x NW/4 warps x 32 columns, 256 of the
//     512 columns) and goes on with the local SAT of the NEXT tile;
//   * only then does it reload the parked block (tcgen05.ld), wait for the walks of the previous tile,
//     publish its inclusive aggregates (Steps 2.A.3, 2.B.3, 3.1, 3.3) and apply Step 4 (rule
//     P:150) into a dedicated output buffer, which the storer lane writes with a TMA 2-D store.
//
// Roles: loader lane (tickets + TMA loads), row / column walker warps (ws_walker), NW compute warps,
// storer lane.  Barriers: acq / rowwalk / colwalk / tfree / result per tile slot (tile ring, NQ
// deep); full / empty per input stage; ofree per output buffer.  The storer releases a tile slot
// (tfree) once it has taken the tile's result, so every per-slot barrier is at most one phase ahead
// of each of its waiters.
#pragma once

#include "sat_pipe.cuh"
#if SAT_EXPERIMENTAL
#include "sat_ws_kernel.cuh"  // ws_walker (non-decoupled walker configurations, tuning builds only)
#endif

namespace sat {

// TR_ x TC_ tiles: TC_ = 128 * G (a lane owns G chunks of 4 columns, 128 apart); flat tiles (TC_ > 128)
// keep the tile's 64 KiB but make every DRAM row visit 4 B * TC_ long (tile shape).
template <int NW_, int IN_, int NQ_, int NT_ = 1, int WPUB_ = 1, int D_ = 2, int DIRECT_ = 0, int QS_ = 0,
          int TR_ = 128, int TC_ = 128, int LB_ = 2, int CT_ = 0, int DW_ = 4, int CH_ = 0, int MINB_ = 1, int RW2_ = 0>
struct TmCfg {
    static constexpr int MINB = MINB_;              // resident CTAs per SM the registers are capped for
    static constexpr int RW2 = RW2_;                // 1: two row walker warps, even / odd tiles
    // Chained strip partition (sat_compute_chained): column-major tile order, column carries = strip-local
    // vertical look-back + the upstream ranks' strip column sums from the inbox, corners by a horizontal
    // look-back; bottom tiles push their strip column sums to the downstream ranks.
    static constexpr bool CHAIN = CH_ != 0;
    static constexpr int DW = DW_;                  // diagonal look-back: corner words polled per round (<= 32)
    static constexpr bool CT = CT_ != 0;            // a lane owns 4 G contiguous columns (one warp scan per row)
    static constexpr int LB = LB_;                  // row / column look-back: predecessors polled per round
    static constexpr int TR = TR_, TC = TC_, NW = NW_;
    static constexpr int G = TC / 128;             // column chunks per lane
    static constexpr int TB = TC < 256 ? TC : 256;  // TMA box width (boxDim <= 256 elements)
    static constexpr int NB = TC / TB;              // TMA boxes per tile (stage / output layout [NB][TR][TB])
    static constexpr bool SBAND = TC > 128;         // single-parity band buffer (two barriers per tile)
    static constexpr int IN = IN_;    // input stages
    static constexpr int STAGES = IN;
    static constexpr int NQ = NQ_;    // tile ring
    static constexpr int NT = NT_;    // tiles in flight per walker
    static constexpr bool FAST = false;
    static constexpr bool WPUB = WPUB_ != 0;  // the walkers publish the inclusive aggregates
    static constexpr bool WPUB_WAIT = WPUB_ == 2;  // ... blocking on the tile's local aggregates
    static constexpr bool DECOUPLED = WPUB_ == 3;  // tm_walker: GLS published as a local corner word
    static constexpr int RPW = TR / NW, ER = TR / 32, EC = TC / 32;
    static constexpr int NREG = RPW * 4 * G;     // 32-bit registers per thread parked per tile
    static constexpr int D = D_;                 // TMEM parking depth: finish(k) runs after local(k + D - 1)
    static constexpr bool DIRECT = DIRECT_ != 0; // GSAT stored from registers (st.global.cs), no output buffer
    static constexpr bool QS = QS_ != 0;         // output buffer handed over in quarters (4 TMA stores of TR/4 rows)
    static constexpr int OBR = QS ? TR / 4 : TR; // rows per TMA store box
    static constexpr int TM_COLS_PER_SLOT = (NW / 4) * NREG;
    static constexpr int TM_COLS = D * TM_COLS_PER_SLOT <= 32 ? 32 : D * TM_COLS_PER_SLOT <= 64 ? 64
                                 : D * TM_COLS_PER_SLOT <= 128 ? 128 : D * TM_COLS_PER_SLOT <= 256 ? 256 : 512;
    static constexpr int ROW_WARP = NW, COL_WARP = NW + 1, STORE_WARP = NW + 2, LOAD_WARP = NW + 3, ROW2_WARP = NW + 4;
    static constexpr int THREADS = (NW + 4 + RW2) * 32;
    static_assert(NW % 4 == 0 && TR % NW == 0 && RPW % 4 == 0, "compute warps cover the 4 TMEM lane quarters");
    static_assert(NREG == 16 || NREG == 32 || NREG == 64, "tcgen05 32x32b.x16 / .x32 parking");
    static_assert(TC % 128 == 0 && TC % TB == 0 && TR >= 32 && (TR * TC == 128 * 128 || (TR * TC == 64 * 128 && MINB == 2)),
                  "64 KiB tiles (32 KiB tiles for 2 CTAs per SM), TC = 128 G");
    static_assert(!SBAND || !QS, "flat tiles: whole-tile TMA stores");
    static_assert(!CT || (TC == 256 && !DIRECT), "contiguous lane columns: 64 x 256 tiles");
    static_assert(D >= 2 && D * TM_COLS_PER_SLOT <= 512, "TMEM columns");
    static_assert(DW >= 1 && DW <= 32 && (DW & (DW - 1)) == 0, "diagonal window: a power of two <= 32");
    static_assert(IN >= 1 && NQ >= IN + D - 1 && NQ <= 16, "rings");
#if !SAT_EXPERIMENTAL
    static_assert(DECOUPLED, "product builds ship the decoupled walkers only (-DSAT_EXPERIMENTAL=1 for the rest)");
#endif
};

template <typename V, typename Cfg, typename TIn = V>
struct TmSmem {
    alignas(1024) TIn stage[Cfg::IN][Cfg::TR * Cfg::TC];  // input ring (TMA loads; u8 for integral images)
    alignas(1024) V out[Cfg::DIRECT ? 4 : Cfg::TR * Cfg::TC];  // GSAT of one tile (TMA store source)
    alignas(16) V band[Cfg::SBAND ? 1 : 2][Cfg::NW][Cfg::TC];
    alignas(16) V rp[Cfg::NQ][Cfg::TR];
    alignas(16) V cp[Cfg::NQ][Cfg::TC];
    V corner[Cfg::NQ];
    alignas(16) V lrs[Cfg::NQ][Cfg::TR];  // local row aggregates (prefix form) of the slot's tile (WPUB)
    alignas(16) V lcs[Cfg::NQ][Cfg::TC];  // local column aggregates
    alignas(8) uint64_t acq[Cfg::NQ];
    uint64_t ldone[Cfg::NQ];  // lrs / lcs written (NW arrivals)
    int rdone[Cfg::NQ];       // k + 1 once the row walk of tile k (slot) has written rp / corner (WPUB)
    int cdone[Cfg::NQ];       // k + 1 once the column walk of tile k has written cp
    int rres[Cfg::NQ];        // DECOUPLED: k + 1 once the row walk of tile k has written rp (corner maybe not)
    int lw[Cfg::NQ][Cfg::NW]; // DECOUPLED: k + 1 once compute warp w has written its lrs (and lcs) of tile k
    uint64_t rowwalk[Cfg::NQ];
    uint64_t colwalk[Cfg::NQ];
    uint64_t tfree[Cfg::NQ];
    uint64_t result[Cfg::NQ];  // GSAT of the slot's tile is in `out` (NW arrivals)
    uint64_t full[Cfg::IN];
    uint64_t empty[Cfg::IN];   // input stage read into registers (NW arrivals)
    uint64_t ofree[4];         // quarter q of `out` read by its TMA store (only [0] without QS: the whole buffer)
    uint64_t qready[4];        // QS: quarter q of `out` written (NW/4 arrivals)
    alignas(16) TileInfo info[Cfg::NQ];
    uint32_t epoch;
    int end_n;
    uint32_t tmem_base;
};

// ------------------------------------------------------------------ tcgen05 TMEM helpers
__device__ __forceinline__ void tmem_alloc(uint32_t* dst_smem, int ncols) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_addr(dst_smem)),
                 "r"(ncols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t base, int ncols) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(base), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// Park / reload the warp's RPW x 4 block: thread t of the warp uses TMEM lane (32 * (warp % 4) + t),
// NREG consecutive columns from `col`.
template <int N>
__device__ __forceinline__ void tmem_st(uint32_t taddr, const uint32_t (&r)[N]);
template <>
__device__ __forceinline__ void tmem_st<32>(uint32_t taddr, const uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31, %32};" ::"r"(taddr),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
        "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]),
        "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]),
        "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
        : "memory");
}
template <>
__device__ __forceinline__ void tmem_st<16>(uint32_t taddr, const uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15, %16};" ::"r"(taddr),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
        "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
        : "memory");
}
// tcgen05.st is asynchronous: completion is awaited (tmem_st_wait) only before the block is read back
// (the source registers are consumed at issue)
__device__ __forceinline__ void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void tmem_ld(uint32_t taddr, uint32_t (&r)[N]);
template <>
__device__ __forceinline__ void tmem_ld<32>(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
          "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),
          "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
          "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr)
        : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
template <>
__device__ __forceinline__ void tmem_ld<16>(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
          "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr)
        : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

template <typename Cfg>
__device__ __forceinline__ uint32_t tm_addr(uint32_t base, int warp, int slot) {
    return base + (static_cast<uint32_t>(32 * (warp & 3)) << 16) +
           static_cast<uint32_t>(slot * Cfg::TM_COLS_PER_SLOT + (warp >> 2) * Cfg::NREG);
}

// First column (within the tile) of chunk g of a lane: chunks 128 apart, or 4 G contiguous columns (CT)
template <typename Cfg>
__device__ __forceinline__ int tm_cb(int lane, int g) {
    return Cfg::CT ? lane * 4 * Cfg::G + 4 * g : g * 128 + lane * 4;
}

// Element (r, c) of a stage / the output buffer: NB boxes of TR x TB, each row-major.
template <typename Cfg>
__device__ __forceinline__ constexpr int tm_sidx(int r, int c) {
    return (c / Cfg::TB) * (Cfg::TR * Cfg::TB) + r * Cfg::TB + (c % Cfg::TB);
}

template <int N>
__device__ __forceinline__ void tmem_st_blk(uint32_t taddr, const uint32_t (&r)[N]) {
    if constexpr (N == 64) {
        tmem_st<32>(taddr, *reinterpret_cast<const uint32_t(*)[32]>(&r[0]));
        tmem_st<32>(taddr + 32, *reinterpret_cast<const uint32_t(*)[32]>(&r[32]));
    } else {
        tmem_st<N>(taddr, r);
    }
}
template <int N>
__device__ __forceinline__ void tmem_ld_blk(uint32_t taddr, uint32_t (&r)[N]) {
    if constexpr (N == 64) {
        tmem_ld<32>(taddr, *reinterpret_cast<uint32_t(*)[32]>(&r[0]));
        tmem_ld<32>(taddr + 32, *reinterpret_cast<uint32_t(*)[32]>(&r[32]));
    } else {
        tmem_ld<N>(taddr, r);
    }
}

// Step 1 + local SAT + Steps 2.A.1 / 2.B.1 of tile k (input stage sl, tile slot tq); parks the block in
// TMEM slot k % D.  Returns false at the end marker.
template <typename V, typename Cfg, bool TMA, typename TIn>
__device__ __forceinline__ bool tm_local(TmSmem<V, Cfg, TIn>& sm, const KParams<V>& p, const Slot<Cfg::IN>& sl,
                                         const Slot<Cfg::NQ>& tq, uint32_t epoch, int warp, int lane) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC, NW = Cfg::NW, RPW = Cfg::RPW, G = Cfg::G, X = 4 * Cfg::G;
    const int s = sl.s;
    const int row0 = warp * RPW, col0 = lane * 4;  // this lane's columns: tm_cb<Cfg>(lane, g) + c
    SAT_CLK(c0);
    mbar_wait(&sm.full[s], sl.ph);
    SAT_CLK(c1);
    if (warp == 0 && lane == 0) { WS_ST(kWsFullWait, c1 - c0); WS_ST(kWsTiles, 1); }
    const TileInfo ti = sm.info[tq.s];
    if (ti.t >= p.ntiles) return false;
#if SAT_STATS
    if (p.trace && warp == 0 && lane == 0) p.trace[8LL * ti.t + 1] = static_cast<long long>(globaltimer_ns());
#endif
    const int I = ti.I, J = ti.J;
    const long long tidx = static_cast<long long>(I) * p.C + J;
    const int par = tq.k & 1;
    V v[RPW][X];
    if constexpr (TMA && sizeof(TIn) == 1) {
        // u8 pixels (integral image): each of a lane's chunks of 4 columns is one 32-bit word of the stage row
        static_assert(TC <= 256, "u8 tiles: one TMA box per row");
        const TIn* tile = sm.stage[s];
#pragma unroll
        for (int r = 0; r < RPW; ++r)
#pragma unroll
            for (int g = 0; g < G; ++g) {
                const uint32_t w = *reinterpret_cast<const uint32_t*>(&tile[(row0 + r) * TC + tm_cb<Cfg>(lane, g)]);
#pragma unroll
                for (int c = 0; c < 4; ++c) v[r][4 * g + c] = V((w >> (8 * c)) & 0xffu);
            }
    } else if constexpr (TMA && Cfg::CT) {
        // two 16-byte halves per row, the lanes of each quarter-warp in swapped order (conflict-free)
        const TIn* tile = sm.stage[s];
        const int swz = (lane >> 2) & 1;
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const uint4 qa = *reinterpret_cast<const uint4*>(&tile[tm_sidx<Cfg>(row0 + r, tm_cb<Cfg>(lane, swz))]);
            const uint4 qb = *reinterpret_cast<const uint4*>(&tile[tm_sidx<Cfg>(row0 + r, tm_cb<Cfg>(lane, swz ^ 1))]);
            const uint4 q0 = swz ? qb : qa, q1 = swz ? qa : qb;
            v[r][0] = from_bits<V>(q0.x); v[r][1] = from_bits<V>(q0.y); v[r][2] = from_bits<V>(q0.z);
            v[r][3] = from_bits<V>(q0.w); v[r][4] = from_bits<V>(q1.x); v[r][5] = from_bits<V>(q1.y);
            v[r][6] = from_bits<V>(q1.z); v[r][7] = from_bits<V>(q1.w);
        }
    } else if constexpr (TMA) {
        const TIn* tile = sm.stage[s];
#pragma unroll
        for (int r = 0; r < RPW; ++r)
#pragma unroll
            for (int g = 0; g < G; ++g) {
                const uint4 q = *reinterpret_cast<const uint4*>(&tile[tm_sidx<Cfg>(row0 + r, tm_cb<Cfg>(lane, g))]);
                v[r][4 * g] = from_bits<V>(q.x); v[r][4 * g + 1] = from_bits<V>(q.y);
                v[r][4 * g + 2] = from_bits<V>(q.z); v[r][4 * g + 3] = from_bits<V>(q.w);
            }
    } else {
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const long long gi = static_cast<long long>(I) * TR + row0 + r;
#pragma unroll
            for (int x = 0; x < X; ++x) {
                const long long gj = static_cast<long long>(J) * TC + tm_cb<Cfg>(lane, x / 4) + (x % 4);
                const bool in = gi < p.rows && gj < p.cols;
                if constexpr (sizeof(TIn) == 1) v[r][x] = in ? V(p.src8[gi * p.src_pitch + gj]) : V(0);
                else v[r][x] = in ? p.src[gi * p.pitch + gj] : V(0);
            }
        }
    }
    // the pixels are in registers: the loader may refill the stage now
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.empty[s]);
    if (TMA && J == p.C - 1) {  // right edge: zero columns >= cols (16-byte TMA granules, reading R2)
#pragma unroll
        for (int x = 0; x < X; ++x)
            if (static_cast<long long>(J) * TC + tm_cb<Cfg>(lane, x / 4) + (x % 4) >= p.cols) {
#pragma unroll
                for (int r = 0; r < RPW; ++r) v[r][x] = V(0);
            }
    }
#if SAT_STATS
    const bool skip = (p.order & 64) != 0;  // timing experiment only: no local SAT / publication (wrong sums)
#else
    constexpr bool skip = false;
#endif
    if (!skip) {
    // local SAT: column prefix in the band, warp prefix-sum rows, bands above
#pragma unroll
    for (int r = 1; r < RPW; ++r)
#pragma unroll
        for (int x = 0; x < X; ++x) v[r][x] = v[r][x] + v[r - 1][x];
    if constexpr (Cfg::CT) {
        // lane-sequential scan of the lane's X contiguous columns, then one warp scan per row (step-major)
        V incl[RPW];
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
#pragma unroll
            for (int x = 1; x < X; ++x) v[r][x] = v[r][x] + v[r][x - 1];
            incl[r] = v[r][X - 1];
        }
#pragma unroll
        for (int d = 1; d < 32; d <<= 1)
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                const V y = __shfl_up_sync(kFull, incl[r], d);
                if (lane >= d) incl[r] = incl[r] + y;
            }
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            V excl = __shfl_up_sync(kFull, incl[r], 1);
            if (lane == 0) excl = V(0);
#pragma unroll
            for (int x = 0; x < X; ++x) v[r][x] = v[r][x] + excl;
        }
    } else if constexpr (G == 1) {
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            V* w = &v[r][0];
            w[1] = w[1] + w[0];
            w[2] = w[2] + w[1];
            w[3] = w[3] + w[2];
            const V incl = warp_inclusive_scan(w[3], lane);
            V excl = __shfl_up_sync(kFull, incl, 1);
            if (lane == 0) excl = V(0);
#pragma unroll
            for (int c = 0; c < 4; ++c) w[c] = w[c] + excl;
        }
    } else {
        // RPW x G independent warp scans, step-major so that their shuffles overlap
        V incl[RPW][G];
#pragma unroll
        for (int r = 0; r < RPW; ++r)
#pragma unroll
            for (int g = 0; g < G; ++g) {
                V* w = &v[r][4 * g];
                w[1] = w[1] + w[0];
                w[2] = w[2] + w[1];
                w[3] = w[3] + w[2];
                incl[r][g] = w[3];
            }
#pragma unroll
        for (int d = 1; d < 32; d <<= 1)
#pragma unroll
            for (int r = 0; r < RPW; ++r)
#pragma unroll
                for (int g = 0; g < G; ++g) {
                    const V y = __shfl_up_sync(kFull, incl[r][g], d);
                    if (lane >= d) incl[r][g] = incl[r][g] + y;
                }
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            V carry = V(0);  // row total of the chunks to the left
#pragma unroll
            for (int g = 0; g < G; ++g) {
                V excl = __shfl_up_sync(kFull, incl[r][g], 1);
                if (lane == 0) excl = V(0);
                if (g > 0) excl = excl + carry;
                V* w = &v[r][4 * g];
#pragma unroll
                for (int c = 0; c < 4; ++c) w[c] = w[c] + excl;
                if (g + 1 < G) carry = carry + __shfl_sync(kFull, incl[r][g], 31);
            }
        }
    }
    {   // band offsets: warp w adds the bottoms of bands 0 .. w-1 (no serial scan)
        V off[X];
#pragma unroll
        for (int x = 0; x < X; ++x) off[x] = V(0);
        if constexpr (Cfg::SBAND) {
            // one band buffer: every warp is done with the previous tile's bottoms before it is rewritten
            V* bands = &sm.band[0][0][0];
            named_bar_sync(1, NW * 32);
#pragma unroll
            for (int g = 0; g < G; ++g)
                *reinterpret_cast<uint4*>(&bands[warp * TC + tm_cb<Cfg>(lane, g)]) =
                    make_uint4(to_bits(v[RPW - 1][4 * g]), to_bits(v[RPW - 1][4 * g + 1]),
                               to_bits(v[RPW - 1][4 * g + 2]), to_bits(v[RPW - 1][4 * g + 3]));
            named_bar_sync(1, NW * 32);
#pragma unroll 2
            for (int u = 0; u < warp; ++u)
#pragma unroll
                for (int g = 0; g < G; ++g) {
                    const uint4 q = *reinterpret_cast<const uint4*>(&bands[u * TC + tm_cb<Cfg>(lane, g)]);
                    off[4 * g] = off[4 * g] + from_bits<V>(q.x); off[4 * g + 1] = off[4 * g + 1] + from_bits<V>(q.y);
                    off[4 * g + 2] = off[4 * g + 2] + from_bits<V>(q.z);
                    off[4 * g + 3] = off[4 * g + 3] + from_bits<V>(q.w);
                }
        } else {
            *reinterpret_cast<uint4*>(&sm.band[par][warp][col0]) = make_uint4(
                to_bits(v[RPW - 1][0]), to_bits(v[RPW - 1][1]), to_bits(v[RPW - 1][2]), to_bits(v[RPW - 1][3]));
            named_bar_sync(1, NW * 32);
#pragma unroll 4
            for (int u = 0; u < warp; ++u) {
                const uint4 q = *reinterpret_cast<const uint4*>(&sm.band[par][u][col0]);
                off[0] = off[0] + from_bits<V>(q.x); off[1] = off[1] + from_bits<V>(q.y);
                off[2] = off[2] + from_bits<V>(q.z); off[3] = off[3] + from_bits<V>(q.w);
            }
        }
#pragma unroll
        for (int r = 0; r < RPW; ++r)
#pragma unroll
            for (int x = 0; x < X; ++x) v[r][x] = v[r][x] + off[x];
    }
    SAT_JITTER_WARP();
    // Steps 2.A.1 / 2.B.1 (edge tiles publish inclusive at once: their carry is zero)
    const uint64_t pol = policy_evict_last();
    if (lane == 31) {
        uint64_t* rs = p.row_slots + tidx * TR + row0;
        const uint32_t kind = (J == 0) ? kIncl : kLocal;
#pragma unroll
        for (int r = 0; r < RPW; r += 2)
            st_relaxed2_p(rs + r, pack(epoch, kind, to_bits(v[r][X - 1])), pack(epoch, kind, to_bits(v[r + 1][X - 1])),
                          pol);
    }
    if (warp == NW - 1) {
        const uint32_t kind = (I == 0) ? kIncl : kLocal;
#pragma unroll
        for (int g = 0; g < G; ++g) {
            uint64_t* cs = p.col_slots + tidx * TC + tm_cb<Cfg>(lane, g);
            const V* b = &v[RPW - 1][4 * g];
            st_relaxed2_p(cs, pack(epoch, kind, to_bits(b[0])), pack(epoch, kind, to_bits(b[1])), pol);
            st_relaxed2_p(cs + 2, pack(epoch, kind, to_bits(b[2])), pack(epoch, kind, to_bits(b[3])), pol);
        }
    }
    if constexpr (Cfg::WPUB) {
        if (lane == 31) {
#pragma unroll
            for (int r = 0; r < RPW; r += 4)
                *reinterpret_cast<uint4*>(&sm.lrs[tq.s][row0 + r]) =
                    make_uint4(to_bits(v[r][X - 1]), to_bits(v[r + 1][X - 1]), to_bits(v[r + 2][X - 1]),
                               to_bits(v[r + 3][X - 1]));
        }
        if (warp == NW - 1)
#pragma unroll
            for (int g = 0; g < G; ++g)
                *reinterpret_cast<uint4*>(&sm.lcs[tq.s][tm_cb<Cfg>(lane, g)]) =
                    make_uint4(to_bits(v[RPW - 1][4 * g]), to_bits(v[RPW - 1][4 * g + 1]),
                               to_bits(v[RPW - 1][4 * g + 2]), to_bits(v[RPW - 1][4 * g + 3]));
        __syncwarp();
        if (lane == 0) mbar_arrive(&sm.ldone[tq.s]);
        if constexpr (Cfg::DECOUPLED) {
            // whoever comes last publishes (see tm_walker): raise this warp's flag, then look at the walkers'
            __threadfence_block();
            if (lane == 0) *reinterpret_cast<volatile int*>(&sm.lw[tq.s][warp]) = tq.k + 1;
            __threadfence_block();
            if (lane == 31 && J > 0 && *reinterpret_cast<volatile int*>(&sm.rres[tq.s]) == tq.k + 1) {
                __threadfence_block();
                uint64_t* rs = p.row_slots + tidx * TR + row0;
#pragma unroll
                for (int r = 0; r < RPW; r += 2)
                    st_relaxed2_p(rs + r, pack(epoch, kIncl, to_bits(v[r][X - 1] + sm.rp[tq.s][row0 + r])),
                                  pack(epoch, kIncl, to_bits(v[r + 1][X - 1] + sm.rp[tq.s][row0 + r + 1])), pol);
            }
            if (!Cfg::CHAIN && warp == NW - 1) {  // chained strips: the column walker publishes these
                const int cd = __shfl_sync(kFull, *reinterpret_cast<volatile int*>(&sm.cdone[tq.s]), 0);
                if (cd == tq.k + 1) {
                    __threadfence_block();
                    if (I > 0) {
#pragma unroll
                        for (int g = 0; g < G; ++g) {
                            const uint4 c4 = *reinterpret_cast<const uint4*>(&sm.cp[tq.s][tm_cb<Cfg>(lane, g)]);
                            uint64_t* cs = p.col_slots + tidx * TC + tm_cb<Cfg>(lane, g);
                            const V* b = &v[RPW - 1][4 * g];
                            st_relaxed2_p(cs, pack(epoch, kIncl, to_bits(b[0] + from_bits<V>(c4.x))),
                                          pack(epoch, kIncl, to_bits(b[1] + from_bits<V>(c4.y))), pol);
                            st_relaxed2_p(cs + 2, pack(epoch, kIncl, to_bits(b[2] + from_bits<V>(c4.z))),
                                          pack(epoch, kIncl, to_bits(b[3] + from_bits<V>(c4.w))), pol);
                        }
                    }
                    if (lane == 31 && *reinterpret_cast<volatile int*>(&sm.rdone[tq.s]) == tq.k + 1) {
                        __threadfence_block();
                        const V gs =
                            sm.corner[tq.s] + ((v[RPW - 1][X - 1] + sm.rp[tq.s][TR - 1]) + sm.cp[tq.s][TC - 1]);
                        st_relaxed_p(p.corner_slots + tidx, pack(epoch, kIncl, to_bits(gs)), pol);
                    }
                }
            }
        }
    }
    }
    // park the block
    uint32_t r32[Cfg::NREG];
#pragma unroll
    for (int r = 0; r < RPW; ++r)
#pragma unroll
        for (int x = 0; x < X; ++x) r32[r * X + x] = to_bits(v[r][x]);
    tmem_st_blk<Cfg::NREG>(tm_addr<Cfg>(sm.tmem_base, warp, tq.k % Cfg::D), r32);
    SAT_CLK(c2);
    if (warp == 0 && lane == 0) WS_ST(kWsLocal, c2 - c1);
#if SAT_STATS
    if (p.trace && warp == NW - 1 && lane == 0) p.trace[8LL * ti.t + 2] = static_cast<long long>(globaltimer_ns());
#endif
    return true;
}

// Steps 2.A.3 / 2.B.3 / 3.1 / 3.3 and Step 4 of tile k (tile slot tq; its block parked in TMEM slot
// k % D), GSAT into the output buffer (use number `ou` of it).
template <typename V, typename Cfg, bool TMA, bool CARRY, typename TIn>
__device__ __forceinline__ void tm_finish(TmSmem<V, Cfg, TIn>& sm, const KParams<V>& p, const Slot<Cfg::NQ>& tq,
                                          uint32_t ou, uint32_t epoch, int warp, int lane) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC, NW = Cfg::NW, RPW = Cfg::RPW, G = Cfg::G, X = 4 * Cfg::G;
    const int q = tq.s;
    const int row0 = warp * RPW, col0 = lane * 4;
    const TileInfo ti = sm.info[q];
    const int I = ti.I, J = ti.J;
    const long long tidx = static_cast<long long>(I) * p.C + J;
    const uint64_t pol = policy_evict_last();
    V v[RPW][X];
    {
        uint32_t r32[Cfg::NREG];
        tmem_st_wait();
        tmem_ld_blk<Cfg::NREG>(tm_addr<Cfg>(sm.tmem_base, warp, tq.k % Cfg::D), r32);
#pragma unroll
        for (int r = 0; r < RPW; ++r)
#pragma unroll
            for (int x = 0; x < X; ++x) v[r][x] = from_bits<V>(r32[r * X + x]);
    }
    SAT_CLK(c0);
    mbar_wait(&sm.rowwalk[q], tq.ph);
    mbar_wait(&sm.colwalk[q], tq.ph);
    SAT_CLK(c1);
    if (warp == 0 && lane == 0) WS_ST(kWsWalkWait, c1 - c0);
    V rt[RPW];
#pragma unroll
    for (int r = 0; r < RPW; r += 4) {
        const uint4 u = *reinterpret_cast<const uint4*>(&sm.rp[q][row0 + r]);
        rt[r] = from_bits<V>(u.x); rt[r + 1] = from_bits<V>(u.y); rt[r + 2] = from_bits<V>(u.z);
        rt[r + 3] = from_bits<V>(u.w);
    }
    V cpv[X];
#pragma unroll
    for (int g = 0; g < G; ++g) {
        const uint4 c4 = *reinterpret_cast<const uint4*>(&sm.cp[q][tm_cb<Cfg>(lane, g)]);
        cpv[4 * g] = from_bits<V>(c4.x); cpv[4 * g + 1] = from_bits<V>(c4.y); cpv[4 * g + 2] = from_bits<V>(c4.z);
        cpv[4 * g + 3] = from_bits<V>(c4.w);
    }
    const V corner = sm.corner[q];
    if (!Cfg::WPUB && lane == 31 && J > 0) {
        uint64_t* rs = p.row_slots + tidx * TR + row0;
#pragma unroll
        for (int r = 0; r < RPW; r += 2)
            st_relaxed2_p(rs + r, pack(epoch, kIncl, to_bits(v[r][X - 1] + rt[r])),
                          pack(epoch, kIncl, to_bits(v[r + 1][X - 1] + rt[r + 1])), pol);
    }
    if (!Cfg::WPUB && warp == NW - 1) {
        if (I > 0) {
#pragma unroll
            for (int g = 0; g < G; ++g) {
                uint64_t* cs = p.col_slots + tidx * TC + tm_cb<Cfg>(lane, g);
                const V* b = &v[RPW - 1][4 * g];
                const V* c = &cpv[4 * g];
                st_relaxed2_p(cs, pack(epoch, kIncl, to_bits(b[0] + c[0])), pack(epoch, kIncl, to_bits(b[1] + c[1])),
                              pol);
                st_relaxed2_p(cs + 2, pack(epoch, kIncl, to_bits(b[2] + c[2])),
                              pack(epoch, kIncl, to_bits(b[3] + c[3])), pol);
            }
        }
        if (lane == 31) {  // GLS = total + rp[TR-1] + cp[TC-1];  GS = GS(I-1,J-1) + GLS
            const V gls = v[RPW - 1][X - 1] + rt[RPW - 1] + cpv[X - 1];
            st_relaxed_p(p.corner_slots + tidx, pack(epoch, kIncl, to_bits(corner + gls)), pol);
        }
    }
    V colterm[X];
#pragma unroll
    for (int x = 0; x < X; ++x) colterm[x] = cpv[x] + corner;
    if constexpr (CARRY) {
#pragma unroll
        for (int x = 0; x < X; ++x) {
            const long long gj = static_cast<long long>(J) * TC + tm_cb<Cfg>(lane, x / 4) + (x % 4);
            colterm[x] = colterm[x] + (gj < p.cols ? p.carry[gj] : V(0));
        }
    }
#pragma unroll
    for (int r = 0; r < RPW; ++r)
#pragma unroll
        for (int x = 0; x < X; ++x) v[r][x] = v[r][x] + (rt[r] + colterm[x]);
    const bool ragged = !TMA || ((J == p.C - 1) && (p.cols & 3) != 0);
    if (Cfg::DIRECT && !ragged) {
        // Step 4 store straight from registers: a lane writes 16 contiguous bytes of each of its rows
        // (a warp row = 512 contiguous bytes); columns >= cols are clipped, rows >= rows skipped
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const long long gi = static_cast<long long>(I) * TR + row0 + r;
#pragma unroll
            for (int g = 0; g < G; ++g) {
                const long long gj = static_cast<long long>(J) * TC + tm_cb<Cfg>(lane, g);
                if (gi < p.rows && gj < p.cols)
                    __stcs(reinterpret_cast<uint4*>(p.dst + gi * p.pitch + gj),
                           make_uint4(to_bits(v[r][4 * g]), to_bits(v[r][4 * g + 1]), to_bits(v[r][4 * g + 2]),
                                      to_bits(v[r][4 * g + 3])));
            }
        }
    } else if (!ragged) {
        constexpr int WPQ = NW / 4;  // warps per quarter of the buffer
        const int qq = Cfg::QS ? warp / WPQ : 0;
        SAT_CLK(o0);
        mbar_wait(&sm.ofree[qq], (ou & 1u) ^ 1u);  // the previous tile's store has read (this quarter of) `out`
        SAT_CLK(o1);
        if (warp == 0 && lane == 0) WS_ST(kWsFastHits, o1 - o0);
        if constexpr (Cfg::CT) {
            const int swz = (lane >> 2) & 1;  // same quarter-warp order as the stage read
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                const uint4 q0 = make_uint4(to_bits(v[r][0]), to_bits(v[r][1]), to_bits(v[r][2]), to_bits(v[r][3]));
                const uint4 q1 = make_uint4(to_bits(v[r][4]), to_bits(v[r][5]), to_bits(v[r][6]), to_bits(v[r][7]));
                *reinterpret_cast<uint4*>(&sm.out[tm_sidx<Cfg>(row0 + r, tm_cb<Cfg>(lane, swz))]) = swz ? q1 : q0;
                *reinterpret_cast<uint4*>(&sm.out[tm_sidx<Cfg>(row0 + r, tm_cb<Cfg>(lane, swz ^ 1))]) = swz ? q0 : q1;
            }
        } else {
#pragma unroll
            for (int r = 0; r < RPW; ++r)
#pragma unroll
                for (int g = 0; g < G; ++g)
                    *reinterpret_cast<uint4*>(&sm.out[tm_sidx<Cfg>(row0 + r, tm_cb<Cfg>(lane, g))]) =
                        make_uint4(to_bits(v[r][4 * g]), to_bits(v[r][4 * g + 1]), to_bits(v[r][4 * g + 2]),
                                   to_bits(v[r][4 * g + 3]));
        }
        fence_proxy_async_smem();
        if constexpr (Cfg::QS) {
            __syncwarp();
            if (lane == 0) mbar_arrive(&sm.qready[qq]);
        }
    } else {
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const long long gi = static_cast<long long>(I) * TR + row0 + r;
#pragma unroll
            for (int x = 0; x < X; ++x) {
                const long long gj = static_cast<long long>(J) * TC + tm_cb<Cfg>(lane, x / 4) + (x % 4);
                if (gi < p.rows && gj < p.cols) p.dst[gi * p.pitch + gj] = v[r][x];
            }
        }
    }
#if SAT_STATS
    if (p.trace && warp == 0 && lane == 0) p.trace[8LL * ti.t + 5] = static_cast<long long>(globaltimer_ns());
#endif
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.result[q]);
    SAT_CLK(c2);
    if (warp == 0 && lane == 0) WS_ST(kWsFinish, c2 - c1);
}

// Look-back step over up to NP predecessors loaded in one round (w[h] = words of predecessor pos - h):
// consumed in order until one has a not-yet-published element that is still pending.
template <typename V, int E, int NP>
__device__ __forceinline__ bool lb_consume_n(uint32_t& pending, int& pos, V (&acc)[E], const uint64_t (&w)[NP][E],
                                             uint32_t epoch) {
    bool progress = false;
#pragma unroll
    for (int h = 0; h < NP; ++h) {
        if (!pending || pos < 0) break;
        bool ok = true;
#pragma unroll
        for (int e = 0; e < E; ++e)
            if (((pending >> e) & 1u) && !word_ready(w[h][e], epoch)) ok = false;
        if (!ok) break;
#pragma unroll
        for (int e = 0; e < E; ++e) {
            if ((pending >> e) & 1u) {
                acc[e] = acc[e] + from_bits<V>(static_cast<uint32_t>(w[h][e]));
                if (word_kind(w[h][e]) == kIncl) pending &= ~(1u << e);
            }
        }
        pos -= 1;
        progress = true;
    }
    return progress;
}

// Chained strips (Cfg::CHAIN), column walker, once the strip-local column look-back of tile (I,J) has
// resolved (acc = prefix_j of the column sums of this strip's rows above the tile, VP):
//  1. the strip-local inclusive column words VP + LCS(I,J) (Step 2.B.3 within the strip), once the owning
//     compute warp has written its local column aggregates;
//  2. acc += the carry T(rank-1) of the rank above from this rank's inbox: acc = prefix_j GCS(I-1,J) of the
//     full matrix, the column carry of Step 4 (the virtual tile row above the strip, R12);
//  3. bottom tile row: LCS(I,J) + acc = T(rank), the column sums of every row of ranks 0..rank over tile
//     column J (prefix form) -- pushed into the inbox of rank + 1 only (system-scope stores to peer
//     memory), after rank + 1 has released this inbox half (back-pressure: it finished call epoch - 2).
// The carry is forwarded cumulatively, T(r) = LCS + (VP + T(r-1)): every rank polls one vector and pushes
// one, whatever N (reading R12': fp32 carries are associated rank by rank, top to bottom).  The push
// of tile column J waits for T(rank-1)[J], which the top tile of column J needed already, so the chain
// lags one tile column per rank.
template <typename V, typename Cfg, typename SM>
__device__ __forceinline__ void tm_chain_column(SM& sm, const KParams<V>& p, int s, int k, int I, int J,
                                                V (&acc)[Cfg::EC], uint64_t* own, uint32_t epoch, int lane, bool& bp_ok) {
    constexpr int E = Cfg::EC, NW = Cfg::NW, TC = Cfg::TC;
    const uint64_t pol = policy_evict_last();
    const ChainParams& ch = p.chain;
    sat_spin_until(*reinterpret_cast<const volatile int*>(&sm.lw[s][NW - 1]) == k + 1, 20);
    __threadfence_block();
    V lcs[E];
#pragma unroll
    for (int e = 0; e < E; ++e) lcs[e] = sm.lcs[s][lane * E + e];
    if (I > 0) {  // I == 0: published inclusive by the compute warp
        uint64_t wv[E];
#pragma unroll
        for (int e = 0; e < E; ++e) wv[e] = pack(epoch, kIncl, to_bits(lcs[e] + acc[e]));
        st_words_p<E>(own + lane * E, wv, pol);
    }
    const long long col = static_cast<long long>(J) * TC + lane * E;
    if (ch.rank > 0) {
        const uint64_t* inbox = ch.peer_inbox[ch.rank] + static_cast<long long>(ch.parity) * ch.inbox_cols + col;
        uint64_t w[E];
        SAT_SPIN_DECL;
        while (true) {
            ld_words_sys<E>(inbox, w);
            bool ok = true;
#pragma unroll
            for (int e = 0; e < E; ++e) ok = ok && word_ready(w[e], epoch);
            if (__all_sync(kFull, ok)) break;
            SAT_SPIN_CHECK("chain inbox");
            __nanosleep(64);
        }
#pragma unroll
        for (int e = 0; e < E; ++e) acc[e] = acc[e] + from_bits<V>(static_cast<uint32_t>(w[e]));
    }
    if (I == p.R - 1 && ch.rank + 1 < ch.nranks) {
        SAT_JITTER_WARP();
        if (!bp_ok) {
            if (lane == 0)
                sat_spin_until(static_cast<long long>(ld_relaxed_sys_u32(ch.peer_done[ch.rank] + ch.rank + 1)) >=
                                   static_cast<long long>(epoch) - 2, 64);
            __syncwarp();
            bp_ok = true;
        }
        uint64_t wv[E];
#pragma unroll
        for (int e = 0; e < E; ++e) wv[e] = pack(epoch, kIncl, to_bits(lcs[e] + acc[e]));
        st_words_sys<E>(ch.peer_inbox[ch.rank + 1] + static_cast<long long>(ch.parity) * ch.inbox_cols + col, wv);
    }
}

// Walker with a decoupled diagonal look-back (Cfg::DECOUPLED), one tile at a time, in acquisition order.
//
// Row walker: row look-back (Step 2.A.2) and diagonal look-back (Step 3.2).  Column
// walker: column look-back (Step 2.B.2).  A walker never waits for anything but the words it polls: it
// hands a tile's carries to the compute warps (smem + rowwalk / colwalk) and goes on with the next tile.
// The inclusive words need the local aggregates too, so they are published by whichever side comes
// last, each raising its flag before it looks at the other's:
//   row words (Step 2.A.3)  compute warp w (flag lw[w], its RPW rows)   vs the row walker (rres)
//   column words (2.B.3)    compute warp NW-1 (lw[NW-1])                 vs the column walker (cdone)
//   GS (Step 3.3)           compute warp NW-1, column walker, row walker (rdone: rp and the corner)
// Both sides compute the same sums from the same operands, so a double publication writes equal bits.
// The corner word goes through two states like the vector words: while its diagonal look-back is
// still open, the row walker publishes GLS(I,J) = total + rp[TR-1] + cp[TC-1] (Step 3.1)
// with kind "local"; GS(I,J) = GS(I-1,J-1) + GLS(I,J) follows with kind "inclusive" (only after rdone,
// which the row walker raises after any GLS store; should another warp's GS store still land first,
// the word merely reads "local" again: readers then walk one tile further, and the edge tiles, whose
// walk is empty, only ever publish GS).  A diagonal look-back therefore sums GLS words up to
// the first GS word (reading R8) instead of waiting for GS(I-1,J-1): no chain in any of the
// three directions waits for a neighbour's completion.
template <typename V, typename Cfg, bool ROW, typename TIn>
__device__ __forceinline__ void tm_walker(TmSmem<V, Cfg, TIn>& sm, const KParams<V>& p, uint32_t epoch, int lane,
                                          int first = 0, int stride = 1) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC, RPW = Cfg::RPW, NW = Cfg::NW;
    constexpr int E = ROW ? Cfg::ER : Cfg::EC;
    constexpr int DW = Cfg::DW;  // diagonal predecessors polled per round
    // predecessors polled per round: LB, capped at 32 words (64 registers) per lane
    constexpr int NP = Cfg::LB * E <= 32 ? Cfg::LB : (32 / E >= 1 ? 32 / E : 1);
    const uint64_t pol = policy_evict_last();
    auto flag = [&](const int* f) { return *reinterpret_cast<const volatile int*>(f); };
    bool bp_ok = false;  // chain mode: the downstream ranks have released this call's inbox half
    Slot<Cfg::NQ> nx;
    for (int f = 0; f < first; ++f) nx.next();
    for (;; [&] { for (int f = 0; f < stride; ++f) nx.next(); }()) {
        if (!wait_acquired(sm, nx.s, nx.ph, nx.k)) break;
        const TileInfo ti = sm.info[nx.s];
        if (ti.t >= p.ntiles) break;
        const int s = nx.s, k = nx.k, I = ti.I, J = ti.J;
        const long long tidx = static_cast<long long>(I) * p.C + J;
        const long long step = ROW ? static_cast<long long>(TR) : static_cast<long long>(p.C) * TC;
        uint64_t* const own = ROW ? p.row_slots + tidx * TR : p.col_slots + tidx * TC;
        int pos = ROW ? J - 1 : I - 1;
        uint32_t pend = pos >= 0 ? (1u << E) - 1u : 0u;
        V acc[E];
#pragma unroll
        for (int e = 0; e < E; ++e) acc[e] = V(0);
        // diagonal look-back (Step 3.2) -- in chain mode a horizontal one over the corner words X / XG
        bool ddone = ROW ? (Cfg::CHAIN ? J == 0 : (I == 0 || J == 0)) : true;
#if SAT_STATS
        if (p.order & 16) { pend = 0u; ddone = true; }  // timing experiment only: no look-back (wrong sums)
#endif
        V dacc = V(0);
        int dbase = 1;
        bool cin = false, lpub = false;
        SAT_SPIN_DECL;
        while (true) {
            // ---- issue this round's loads
            uint64_t w[NP][E], wd = 0;
            if (pend) {
                const uint64_t* q = own - (ROW ? static_cast<long long>(J - pos) * TR
                                               : static_cast<long long>(I - pos) * p.C * TC) + lane * E;
#pragma unroll
                for (int h = 0; h < NP; ++h)
                    if (pos - h >= 0) ld_words_p<E>(q - h * step, w[h], pol);
            }
            const int kk = dbase + lane;
            const int dI = Cfg::CHAIN ? I : I - kk;
            const bool dinr = ROW && !ddone && lane < DW && (dI >= 0) && (J - kk >= 0);
            if (dinr) wd = ld_relaxed_p(p.corner_slots + static_cast<long long>(dI) * p.C + (J - kk), pol);
            // ---- consume
            bool progress = false;
            if (pend) progress = lb_consume_n<V, E, NP>(pend, pos, acc, w, epoch);
            if (ROW && !ddone) {
                const bool ready = !dinr || word_ready(wd, epoch);
                const unsigned incl = __ballot_sync(kFull, dinr && ready && word_kind(wd) == kIncl);
                const unsigned notready = __ballot_sync(kFull, !ready);
                const int f = incl ? (__ffs(incl) - 1) : DW;
                const unsigned need = (2u << (f < DW ? f : DW - 1)) - 1u;
                if (!(notready & need)) {
                    V val = (dinr && lane <= f) ? from_bits<V>(static_cast<uint32_t>(wd)) : V(0);
#pragma unroll
                    for (int d = DW / 2; d >= 1; d >>= 1) val = val + __shfl_xor_sync(kFull, val, d);
                    dacc = dacc + __shfl_sync(kFull, val, 0);
                    if (f < DW) ddone = true; else dbase += DW;
                    progress = true;
                }
            }
            if constexpr (Cfg::CHAIN && !ROW) {
                if (!cin && __all_sync(kFull, pend == 0u)) tm_chain_column<V, Cfg>(sm, p, s, k, I, J, acc, own, epoch, lane,
                                                                                    bp_ok);
            }
            if (!cin && __all_sync(kFull, pend == 0u)) {
                SAT_JITTER_WARP();
                // carries -> smem, raise the flag, then publish the inclusive words of the rows / columns
                // whose local aggregates are already in
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    if (ROW) sm.rp[s][lane * E + e] = acc[e];
                    else sm.cp[s][lane * E + e] = acc[e];
                }
                if (Cfg::CHAIN && !ROW && lane == 31)  // X(I,J): local corner word (inclusive on the left edge)
                    st_relaxed_p(p.corner_slots + tidx, pack(epoch, J == 0 ? kIncl : kLocal, to_bits(acc[E - 1])), pol);
                __syncwarp();
                __threadfence_block();
                if (lane == 0) *reinterpret_cast<volatile int*>(ROW ? &sm.rres[s] : &sm.cdone[s]) = k + 1;
                __threadfence_block();
                const int owner = ROW ? (lane * E) / RPW : NW - 1;  // compute warp holding these locals
                if ((ROW ? J > 0 : (I > 0 && !Cfg::CHAIN)) && flag(&sm.lw[s][owner]) == k + 1) {
                    __threadfence_block();
                    uint64_t wv[E];
#pragma unroll
                    for (int e = 0; e < E; ++e) {
                        const V l = ROW ? sm.lrs[s][lane * E + e] : sm.lcs[s][lane * E + e];
                        wv[e] = pack(epoch, kIncl, to_bits(l + acc[e]));
                    }
                    st_words_p<E>(own + lane * E, wv, pol);
                }
                cin = true;
                progress = true;
            }
            if (!Cfg::CHAIN && ROW && cin && !ddone && !lpub) {  // Step 3.1: GLS, published as a local corner word
                SAT_JITTER_WARP();
                int go = 0;
                if (lane == 31 && flag(&sm.cdone[s]) == k + 1 && flag(&sm.lw[s][NW - 1]) == k + 1) {
                    __threadfence_block();
                    const V gls = (sm.lrs[s][TR - 1] + acc[E - 1]) + sm.cp[s][TC - 1];
                    st_relaxed_p(p.corner_slots + tidx, pack(epoch, kLocal, to_bits(gls)), pol);
                    go = 1;
                }
                lpub = __shfl_sync(kFull, go, 31) != 0;
            }
            if (cin && ddone) break;
            if (progress) {
                SAT_SPIN_RESET;
            } else {
                SAT_SPIN_CHECK(ROW ? "row / diagonal look-back words" : "column look-back words");
                __nanosleep(32);
            }
        }
        SAT_JITTER_WARP();
        // ---- Step 3.3 (GS, by whoever comes last) and the hand-off
        if (ROW && Cfg::CHAIN) {
            // corner = GS(I-1,J-1) = sum of X(I,J') over J' < J; then XG(I,J) = corner + X(I,J) = GS(I-1,J),
            // once the column walker has published X (it never waits for this warp)
            if (lane == 0) sm.corner[s] = dacc;
            __syncwarp();
            __threadfence_block();
            if (lane == 0) *reinterpret_cast<volatile int*>(&sm.rdone[s]) = k + 1;
            if (J > 0) {
                sat_spin_until(flag(&sm.cdone[s]) == k + 1, 20);
                __threadfence_block();
                if (lane == 31) st_relaxed_p(p.corner_slots + tidx, pack(epoch, kIncl, to_bits(dacc + sm.cp[s][TC - 1])), pol);
            }
        } else if (ROW) {
            if (lane == 0) sm.corner[s] = dacc;
            __syncwarp();
            __threadfence_block();
            if (lane == 0) *reinterpret_cast<volatile int*>(&sm.rdone[s]) = k + 1;
            __threadfence_block();
            if (lane == 31 && flag(&sm.cdone[s]) == k + 1 && flag(&sm.lw[s][NW - 1]) == k + 1) {
                __threadfence_block();
                const V gs = dacc + ((sm.lrs[s][TR - 1] + acc[E - 1]) + sm.cp[s][TC - 1]);
                st_relaxed_p(p.corner_slots + tidx, pack(epoch, kIncl, to_bits(gs)), pol);
            }
        } else if (!Cfg::CHAIN) {
            if (lane == 31 && flag(&sm.rdone[s]) == k + 1 && flag(&sm.lw[s][NW - 1]) == k + 1) {
                __threadfence_block();
                const V gs = sm.corner[s] + ((sm.lrs[s][TR - 1] + sm.rp[s][TR - 1]) + acc[E - 1]);
                st_relaxed_p(p.corner_slots + tidx, pack(epoch, kIncl, to_bits(gs)), pol);
            }
        }
#if SAT_STATS
        if (p.trace && lane == 0) p.trace[8LL * ti.t + (ROW ? 3 : 4)] = static_cast<long long>(globaltimer_ns());
#endif
        __syncwarp();
        if (lane == 0) mbar_arrive(ROW ? &sm.rowwalk[s] : &sm.colwalk[s]);
    }
}

template <typename V, typename Cfg, bool TMA, bool CARRY, typename TIn = V>
__global__ void __launch_bounds__(Cfg::THREADS, Cfg::MINB)
sat_tm_kernel(const __grid_constant__ CUtensorMap map_in, const __grid_constant__ CUtensorMap map_out,
              const KParams<V> p) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC, NW = Cfg::NW, IN = Cfg::IN;
    constexpr uint32_t kTileBytes = TR * TC * sizeof(TIn);
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    TmSmem<V, Cfg, TIn>& sm = *reinterpret_cast<TmSmem<V, Cfg, TIn>*>(smem_raw);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

#if SAT_STATS
    if (threadIdx.x < kNumStats) ws_stats[threadIdx.x] = 0ull;
#endif
    if (warp == 0) tmem_alloc(&sm.tmem_base, Cfg::TM_COLS);
    if (threadIdx.x == 32) {
        sm.epoch = p.epoch_override ? p.epoch_override : *reinterpret_cast<volatile unsigned int*>(&p.ctrl->epoch);
        sm.end_n = 0x7fffffff;
#pragma unroll
        for (int q = 0; q < Cfg::NQ; ++q) {
            mbar_init(&sm.acq[q], 1);
            mbar_init(&sm.rowwalk[q], 1);
            mbar_init(&sm.colwalk[q], 1);
            mbar_init(&sm.tfree[q], 1);
            mbar_init(&sm.result[q], NW);
            mbar_init(&sm.ldone[q], NW);
            sm.rdone[q] = 0;
            sm.cdone[q] = 0;
            sm.rres[q] = 0;
            for (int w = 0; w < NW; ++w) sm.lw[q][w] = 0;
        }
#pragma unroll
        for (int s = 0; s < IN; ++s) {
            mbar_init(&sm.full[s], 1);
            mbar_init(&sm.empty[s], NW);
        }
        for (int q = 0; q < 4; ++q) {
            mbar_init(&sm.ofree[q], 1);
            mbar_init(&sm.qready[q], NW / 4);
        }
        fence_mbar_init();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t epoch = sm.epoch;

    if (warp < NW) {
        // ================================================================ compute warps
        // local(0 .. D-2), then {local(k+D-1), finish(k)}: the walks of tile k run during the D-1 locals
        // that follow it
        Slot<IN> sl;
        Slot<Cfg::NQ> tql, tqf;
        uint32_t ou = 0;  // uses of the output buffer so far
        int parked = 0;
        bool more = true;
        while (more && parked < Cfg::D - 1) {
            more = tm_local<V, Cfg, TMA, TIn>(sm, p, sl, tql, epoch, warp, lane);
            if (more) { ++parked; sl.next(); tql.next(); }
        }
        while (parked > 0) {
            if (more) {
                more = tm_local<V, Cfg, TMA, TIn>(sm, p, sl, tql, epoch, warp, lane);
                if (more) { ++parked; sl.next(); tql.next(); }
            }
            const TileInfo ti = sm.info[tqf.s];
            const bool ragged = !TMA || ((ti.J == p.C - 1) && (p.cols & 3) != 0);
            tm_finish<V, Cfg, TMA, CARRY, TIn>(sm, p, tqf, ou, epoch, warp, lane);
            if (!ragged) ++ou;
            tqf.next();
            --parked;
        }
        tmem_st_wait();
        tc_fence_before();
        named_bar_sync(2, NW * 32);
        if (warp == 0) tmem_dealloc(sm.tmem_base, Cfg::TM_COLS);
    } else if (warp == Cfg::ROW_WARP) {
#if SAT_EXPERIMENTAL
        if constexpr (!Cfg::DECOUPLED) ws_walker<V, Cfg, true>(sm, p, epoch, lane);
        else
#endif
        tm_walker<V, Cfg, true, TIn>(sm, p, epoch, lane, 0, Cfg::RW2 ? 2 : 1);
    } else if (Cfg::RW2 && warp == Cfg::ROW2_WARP) {
        tm_walker<V, Cfg, true, TIn>(sm, p, epoch, lane, 1, 2);  // the odd tiles' row / diagonal walks
    } else if (warp == Cfg::COL_WARP) {
#if SAT_EXPERIMENTAL
        if constexpr (!Cfg::DECOUPLED) ws_walker<V, Cfg, false>(sm, p, epoch, lane);
        else
#endif
        tm_walker<V, Cfg, false, TIn>(sm, p, epoch, lane);
    } else if (warp == Cfg::STORE_WARP) {
        // ================================================================ storer (one lane)
        if (lane == 0) {
            if constexpr (TMA) prefetch_tensormap(&map_out);
            const uint64_t spol = policy_evict_first();
            uint32_t sou = 0;  // QS: uses of the output buffer so far
            for (Slot<Cfg::NQ> tq;; tq.next()) {
                mbar_wait(&sm.acq[tq.s], tq.ph);
                const TileInfo ti = sm.info[tq.s];
                if (ti.t >= p.ntiles) break;
                SAT_CLK(u0);
                if constexpr (Cfg::QS && !Cfg::DIRECT) {
                    // quarters go out as soon as their warps have written them
                    const bool qragged = !TMA || ((ti.J == p.C - 1) && (p.cols & 3) != 0);
                    if (!qragged) {
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            mbar_wait(&sm.qready[q], sou & 1u);
                            tma_store_2d_hint(&map_out, sm.out + q * Cfg::OBR * TC, ti.J * TC, ti.I * TR + q * Cfg::OBR,
                                              spol);
                            bulk_commit();
                            if (q > 0) {
                                bulk_wait_read<1>();
                                mbar_arrive(&sm.ofree[q - 1]);
                            }
                        }
                        bulk_wait_read<0>();
                        mbar_arrive(&sm.ofree[3]);
                        ++sou;
                    }
                }
                mbar_wait(&sm.result[tq.s], tq.ph);
                // tile k is done with its slot (walks, carries, id): tile k + NQ may be acquired.  Released
                // only here so that no barrier of the slot can run a phase ahead of this lane.
                mbar_arrive(&sm.tfree[tq.s]);
                SAT_CLK(u1);
                WS_ST(kWsStResultWait, u1 - u0);
                const bool ragged = !TMA || ((ti.J == p.C - 1) && (p.cols & 3) != 0);
                if (!Cfg::DIRECT && !Cfg::QS && !ragged) {
#pragma unroll
                    for (int bx = 0; bx < Cfg::NB; ++bx)
                        tma_store_2d_hint(&map_out, sm.out + bx * TR * Cfg::TB, ti.J * TC + bx * Cfg::TB, ti.I * TR,
                                          spol);
                    bulk_commit();
#if SAT_STATS
                    if (p.trace) p.trace[8LL * ti.t + 6] = static_cast<long long>(globaltimer_ns());
#endif
                    bulk_wait_read<0>();
                    mbar_arrive(&sm.ofree[0]);
                }
                SAT_CLK(u2);
                WS_ST(kWsStStore, u2 - u1);
            }
            if constexpr (TMA) bulk_wait_all();
            ws_exit(p, epoch);
        }
    } else if (lane == 0) {
        // ================================================================ loader (one lane)
        const uint64_t policy = TMA ? policy_evict_first() : 0ull;
        if constexpr (TMA) prefetch_tensormap(&map_in);
        Slot<Cfg::NQ> ta, tl;
        Slot<IN> sl;
        bool acq_done = false;
        SAT_SPIN_DECL;
        while (true) {
            bool progress = false;
            if (!acq_done && (ta.k < Cfg::NQ || mbar_test(&sm.tfree[ta.s], ta.ph ^ 1u))) {
                const int t = static_cast<int>(atomicAdd(&p.ctrl->counter, 1u));
                const bool valid = t < p.ntiles;
                TileInfo ti{t, 0, 0, 0};
                if (valid) tile_of_serial(t, p.R, p.C, p.order, ti.I, ti.J);
                if (TMA && valid && p.l2_prefetch) {  // warm L2 while the tile waits for an input stage
                    if (p.l2_prefetch == 2) {  // tuning: prefetched lines marked evict_last
                        const uint64_t lpol = policy_evict_last();
#pragma unroll
                        for (int bx = 0; bx < Cfg::NB; ++bx)
                            tma_prefetch_2d_hint(&map_in, ti.J * TC + bx * Cfg::TB, ti.I * TR, lpol);
                    } else {
#pragma unroll
                        for (int bx = 0; bx < Cfg::NB; ++bx) tma_prefetch_2d(&map_in, ti.J * TC + bx * Cfg::TB, ti.I * TR);
                    }
                }
                sm.info[ta.s] = ti;
                if (!valid) {
                    *reinterpret_cast<volatile int*>(&sm.end_n) = ta.k;
                    acq_done = true;
                }
                mbar_arrive(&sm.acq[ta.s]);
#if SAT_STATS
                if (p.trace && valid) p.trace[8LL * t] = static_cast<long long>(globaltimer_ns());
#endif
                ta.next();
                progress = true;
            }
            if (tl.k < ta.k && (sl.k < IN || mbar_test(&sm.empty[sl.s], sl.ph ^ 1u))) {
                const TileInfo ti = sm.info[tl.s];
                const bool valid = ti.t < p.ntiles;
                if (TMA && valid) {
                    WS_ST(kWsLdIssue, 1);
                    mbar_arrive_expect_tx(&sm.full[sl.s], kTileBytes);
#pragma unroll
                    for (int bx = 0; bx < Cfg::NB; ++bx)
                        tma_load_2d(sm.stage[sl.s] + bx * TR * Cfg::TB, &map_in, &sm.full[sl.s],
                                    ti.J * TC + bx * Cfg::TB, ti.I * TR, policy);
#if SAT_STATS
                    if (p.trace) p.trace[8LL * ti.t + 7] = static_cast<long long>(globaltimer_ns());
#endif
                } else {
                    mbar_arrive(&sm.full[sl.s]);
                }
                tl.next();
                sl.next();
                progress = true;
                if (!valid) break;
            }
#if SAT_STATS
            if (!progress) {
                SAT_CLK(b0);
                __nanosleep(32);
                SAT_CLK(b1);
                if (!acq_done && ta.k >= Cfg::NQ) WS_ST(kWsBandBar, b1 - b0);     // ring full: tile slots busy
                if (tl.k < ta.k) WS_ST(kWsLdEmptyWait, b1 - b0);                 // stage not yet read
            }
#else
            if (progress) {
                SAT_SPIN_RESET;
            } else {
                SAT_SPIN_CHECK("a free tile slot or input stage (loader)");
                __nanosleep(32);
            }
#endif
        }
    }
}

}  // namespace sat
