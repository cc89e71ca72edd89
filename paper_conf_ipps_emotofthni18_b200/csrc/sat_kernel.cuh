// sat_kernel.cuh -- the single-pass SAT kernel for sm_100a (1R1W-SKSS-LB, Sec. IV,
// P:182-249, re-designed for B200; DESIGN.md sections "Kernel" and "Differences from the paper").
//
// One persistent launch.  Every CTA loops:
//   tile t = atomicAdd(&counter, 1)                 SKSS dynamic tile counter
//   t -> (I, J) in diagonal-major order             Fig. 9
//   TMA 2-D load of T(I, J), prefetched one tile ahead                            Step 1
//   local SAT of the tile in registers (column prefix within a warp's row band, row scans with
//     the warp prefix-sum algorithm, cross-band offsets through shared memory)
//   publish the local row/column aggregates                                   Steps 2.A.1/2.B.1
//   row look-back (warp 0), column look-back (warp 1), diagonal look-back (warp 2)
//                                                      Steps 2.A.2-3, 2.B.2-3, 3.1-3.3
//   GSAT(I,J) = localSAT + prefix_i GRS(I,J-1) + prefix_j GCS(I-1,J) + GS(I-1,J-1)
//     (the injection rule of P:150 applied after the local SAT, by linearity)     Step 4
//   TMA 2-D store of GSAT(I, J)                                                   Step 4
//
// Aggregates are published in PREFIX form (R5'): the row slot of T(I,J) carries
// prefix_i LRS(I,J) (= last column of the local SAT) while local and prefix_i GRS(I,J) when
// inclusive; the column slot carries prefix_j LCS / prefix_j GCS; the corner slot carries GLS(I,J)
// while local and GS(I,J) when inclusive.  Prefix sums are linear, so the paper's look-back sums
// carry over unchanged and the carries are directly the corrections Step 4 needs.
//
// Status words (R, C of P:224-229) are folded into the aggregate slots: every 64-bit slot holds
// (epoch << 2 | kind) : value, kind 1 = local, 2 = inclusive.  The epoch changes every launch, so no
// workspace reset is needed between calls (R12).
#pragma once

#include "sat_device.cuh"

namespace sat {

constexpr uint32_t kLocal = 1u;
constexpr uint32_t kIncl = 2u;
constexpr uint32_t kEpochMax = (1u << 30) - 1u;

struct Ctrl {
    unsigned int counter;     // SKSS tile counter c, reset by the last CTA to exit
    unsigned int exit_count;  // CTAs that have exited this launch
    unsigned int epoch;       // current launch epoch, 1 .. kEpochMax
    unsigned int pad;
};

template <typename V>
struct KParams {
    const V* src;  // generic path only
    V* dst;        // generic path only
    int64_t rows, cols, pitch;
    int R, C;          // tile grid
    int ntiles;
    int order;         // 0 = diagonal-major (Fig. 9), 1 = row-major
    uint64_t* row_slots;     // [R*C][TR]
    uint64_t* col_slots;     // [R*C][TC]
    uint64_t* corner_slots;  // [R*C]
    Ctrl* ctrl;
    const V* carry;    // [cols] or nullptr
};

__device__ __forceinline__ uint64_t pack(uint32_t epoch, uint32_t kind, uint32_t bits) {
    return (static_cast<uint64_t>((epoch << 2) | kind) << 32) | bits;
}
__device__ __forceinline__ bool word_ready(uint64_t w, uint32_t epoch) {
    return static_cast<uint32_t>(w >> 34) == epoch;
}
__device__ __forceinline__ uint32_t word_kind(uint64_t w) { return static_cast<uint32_t>(w >> 32) & 3u; }

// ------------------------------------------------------------------ serial number -> tile
// Number of tiles T(I,J) of an R x C grid with I + J < d.
__device__ __forceinline__ long long diag_count(long long d, long long R, long long C) {
    long long m = d < R ? d : R;  // I ranges over [0, m)
    if (m <= 0) return 0;
    long long a = d - C + 1;      // for I < a the diagonal is cut by the right edge: C tiles
    a = a < 0 ? 0 : (a > m ? m : a);
    return a * C + (m - a) * d - (a + m - 1) * (m - a) / 2;
}

// Fig. 9 order generalised to R x C (reading R6): diagonals I+J = 0,1,2,... in turn, I ascending.
__device__ __forceinline__ void tile_of_serial(int s, int R, int C, int order, int& I, int& J) {
    if (order == 1) {
        I = s / C;
        J = s - I * C;
        return;
    }
    long long lo = 0, hi = (long long)R + C - 2;  // largest d with diag_count(d) <= s
    while (lo < hi) {
        long long mid = (lo + hi + 1) >> 1;
        if (diag_count(mid, R, C) <= s) lo = mid; else hi = mid - 1;
    }
    long long d = lo;
    long long i0 = d - C + 1 > 0 ? d - C + 1 : 0;
    I = static_cast<int>(i0 + (s - diag_count(d, R, C)));
    J = static_cast<int>(d - I);
}

// ------------------------------------------------------------------ look-backs
// Row / column look-back (Steps 2.A.2 / 2.B.2, Fig. 10): walk predecessors
// p, p+step, p+2*step, ... summing local aggregates until an inclusive one is found.  Each lane
// owns E consecutive elements of the vector and resolves each element independently (an element
// stops at its first inclusive word); the warp walks until every element of every lane is done.
// Termination: the tile at the grid edge (J=0 / I=0) always publishes inclusive (reading R10').
template <typename V, int E>
__device__ __forceinline__ void lookback_vec(const uint64_t* p, long long step, uint32_t epoch, V (&acc)[E]) {
    uint32_t pending = (1u << E) - 1u;
#pragma unroll
    for (int e = 0; e < E; ++e) acc[e] = V(0);
    while (true) {
        if (pending) {
            uint64_t w[E];
            while (true) {
                ld_words<E>(p, w);
                bool ok = true;
#pragma unroll
                for (int e = 0; e < E; ++e)
                    if (((pending >> e) & 1u) && !word_ready(w[e], epoch)) ok = false;
                if (ok) break;
                __nanosleep(32);
            }
#pragma unroll
            for (int e = 0; e < E; ++e) {
                if ((pending >> e) & 1u) {
                    acc[e] = acc[e] + from_bits<V>(static_cast<uint32_t>(w[e]));
                    if (word_kind(w[e]) == kIncl) pending &= ~(1u << e);
                }
            }
        }
        if (__all_sync(kFull, pending == 0u)) break;
        p += step;
    }
}

// Diagonal look-back (Step 3.2): GS(I-1,J-1) = GS(I-k,J-k) + sum_{0<k'<k} GLS(I-k',J-k').
// The warp inspects a window of 32 diagonal predecessors at once (lane k-1 <-> tile (I-k, J-k)).
// Non-blocking mode returns false as soon as a needed word is not yet published.
template <typename V>
__device__ __forceinline__ bool lookback_diag(const uint64_t* corner_slots, int I, int J, int C, uint32_t epoch,
                                              bool blocking, int lane, V& out) {
    if (I == 0 || J == 0) {
        out = V(0);
        return true;
    }
    V acc = V(0);
    int base = 1;
    while (true) {
        const int k = base + lane;
        const bool inrange = (I - k >= 0) && (J - k >= 0);
        uint64_t w = 0;
        bool ready = true;
        if (inrange) {
            w = ld_relaxed(corner_slots + static_cast<long long>(I - k) * C + (J - k));
            ready = word_ready(w, epoch);
        }
        const unsigned incl = __ballot_sync(kFull, inrange && ready && word_kind(w) == kIncl);
        const unsigned notready = __ballot_sync(kFull, inrange && !ready);
        const int f = incl ? (__ffs(incl) - 1) : 32;
        const unsigned need = (f >= 31) ? kFull : ((2u << f) - 1u);
        if (notready & need) {
            if (!blocking) return false;
            __nanosleep(32);
            continue;
        }
        V val = (inrange && lane <= f) ? from_bits<V>(static_cast<uint32_t>(w)) : V(0);
        acc = acc + warp_sum(val);
        if (f < 32) {
            out = acc;
            return true;
        }
        base += 32;
    }
}

// ------------------------------------------------------------------ the kernel
template <int TR_, int TC_, int NW_, int STAGES_>
struct TileCfg {
    static constexpr int TR = TR_, TC = TC_, NW = NW_, STAGES = STAGES_;
    static constexpr int RPW = TR / NW;       // rows per warp band
    static constexpr int ER = TR / 32;        // row-vector elements per lane (look-back)
    static constexpr int EC = TC / 32;        // column-vector elements per lane
    static constexpr int PRODUCER_WARP = 3;   // issues the tile counter atomics and the TMA ops
    static_assert(TC == 128, "a lane owns 4 consecutive columns (one 16-byte vector)");
    static_assert(TR % NW == 0 && TR % 32 == 0 && NW >= 4, "tile shape");
    static_assert(ER == 1 || ER % 2 == 0, "row vector split");
};

template <typename V, typename Cfg>
struct Smem {
    alignas(1024) V stage[Cfg::STAGES][Cfg::TR * Cfg::TC];
    alignas(16) V band[Cfg::NW][Cfg::TC];
    alignas(16) V lrsp[Cfg::TR];
    alignas(16) V lcsp[Cfg::TC];
    alignas(16) V rp[Cfg::TR];
    alignas(16) V cp[Cfg::TC];
    alignas(8) uint64_t full[Cfg::STAGES];
    int tile_id[Cfg::STAGES];
    V corner;
    int corner_ok;
    uint32_t epoch;
};

template <typename V, typename Cfg, bool TMA, bool CARRY>
__global__ void __launch_bounds__(Cfg::NW * 32)
sat_tiles_kernel(const __grid_constant__ CUtensorMap map_in, const __grid_constant__ CUtensorMap map_out,
                 const KParams<V> p) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC, NW = Cfg::NW, STAGES = Cfg::STAGES;
    constexpr int RPW = Cfg::RPW, ER = Cfg::ER, EC = Cfg::EC;
    constexpr uint32_t kTileBytes = TR * TC * sizeof(V);
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    Smem<V, Cfg>& sm = *reinterpret_cast<Smem<V, Cfg>*>(smem_raw);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const bool producer = (warp == Cfg::PRODUCER_WARP) && (lane == 0);
    uint64_t policy = 0;

    if (producer) {
        sm.epoch = *reinterpret_cast<volatile unsigned int*>(&p.ctrl->epoch);
        if constexpr (TMA) {
            prefetch_tensormap(&map_in);
            prefetch_tensormap(&map_out);
            policy = policy_evict_first();
#pragma unroll
            for (int s = 0; s < STAGES; ++s) mbar_init(&sm.full[s], 1);
            fence_mbar_init();
        }
        const int t0 = static_cast<int>(atomicAdd(&p.ctrl->counter, 1u));
        sm.tile_id[0] = t0;
        if constexpr (TMA) {
            if (t0 < p.ntiles) {
                int I0, J0;
                tile_of_serial(t0, p.R, p.C, p.order, I0, J0);
                mbar_arrive_expect_tx(&sm.full[0], kTileBytes);
                tma_load_2d(sm.stage[0], &map_in, &sm.full[0], J0 * TC, I0 * TR, policy);
            }
        }
    }
    __syncthreads();
    const uint32_t epoch = sm.epoch;

    uint32_t phase_bits = 0;  // parity of each stage's mbarrier
    int s = 0;
    while (true) {
        const int t = sm.tile_id[s];
        if (t >= p.ntiles) break;
        const int sn = (s + 1 == STAGES) ? 0 : s + 1;

        // ---- acquire the next tile and prefetch it (one tile ahead)
        if (producer) {
            const int tn = static_cast<int>(atomicAdd(&p.ctrl->counter, 1u));
            sm.tile_id[sn] = tn;
            if constexpr (TMA) {
                if (tn < p.ntiles) {
                    int In, Jn;
                    tile_of_serial(tn, p.R, p.C, p.order, In, Jn);
                    // the stage being refilled was last stored STAGES-1 tiles ago
                    bulk_wait_read<STAGES - 2>();
                    mbar_arrive_expect_tx(&sm.full[sn], kTileBytes);
                    tma_load_2d(sm.stage[sn], &map_in, &sm.full[sn], Jn * TC, In * TR, policy);
                }
            }
        }

        int I, J;
        tile_of_serial(t, p.R, p.C, p.order, I, J);
        const long long tidx = static_cast<long long>(I) * p.C + J;
        V* tile = sm.stage[s];
        const int row0 = warp * RPW;
        const int col0 = lane * 4;

        // ---- Step 1: tile -> registers (lane owns 4 columns of RPW rows)
        V v[RPW][4];
        if constexpr (TMA) {
            mbar_wait(&sm.full[s], (phase_bits >> s) & 1u);
            phase_bits ^= (1u << s);
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                const uint4 q = *reinterpret_cast<const uint4*>(&tile[(row0 + r) * TC + col0]);
                v[r][0] = from_bits<V>(q.x); v[r][1] = from_bits<V>(q.y);
                v[r][2] = from_bits<V>(q.z); v[r][3] = from_bits<V>(q.w);
            }
        } else {
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                const long long gi = static_cast<long long>(I) * TR + row0 + r;
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    const long long gj = static_cast<long long>(J) * TC + col0 + c;
                    v[r][c] = (gi < p.rows && gj < p.cols) ? p.src[gi * p.pitch + gj] : V(0);
                }
            }
        }

        // ---- local SAT, part 1: column prefix inside the warp's band, then row scans
#pragma unroll
        for (int r = 1; r < RPW; ++r)
#pragma unroll
            for (int c = 0; c < 4; ++c) v[r][c] = v[r][c] + v[r - 1][c];
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            v[r][1] = v[r][1] + v[r][0];
            v[r][2] = v[r][2] + v[r][1];
            v[r][3] = v[r][3] + v[r][2];
            const V incl = warp_inclusive_scan(v[r][3], lane);
            V excl = __shfl_up_sync(kFull, incl, 1);
            if (lane == 0) excl = V(0);
#pragma unroll
            for (int c = 0; c < 4; ++c) v[r][c] = v[r][c] + excl;
        }
        *reinterpret_cast<uint4*>(&sm.band[warp][col0]) =
            make_uint4(to_bits(v[RPW - 1][0]), to_bits(v[RPW - 1][1]), to_bits(v[RPW - 1][2]),
                       to_bits(v[RPW - 1][3]));
        __syncthreads();  // (1) band bottoms visible

        // ---- local SAT, part 2: add the SAT rows of the bands above
        {
            V off[4] = {V(0), V(0), V(0), V(0)};
            for (int w2 = 0; w2 < warp; ++w2) {
                const uint4 q = *reinterpret_cast<const uint4*>(&sm.band[w2][col0]);
                off[0] = off[0] + from_bits<V>(q.x); off[1] = off[1] + from_bits<V>(q.y);
                off[2] = off[2] + from_bits<V>(q.z); off[3] = off[3] + from_bits<V>(q.w);
            }
#pragma unroll
            for (int r = 0; r < RPW; ++r)
#pragma unroll
                for (int c = 0; c < 4; ++c) v[r][c] = v[r][c] + off[c];
        }
        // local aggregates in prefix form: last column / bottom row of the local SAT
        if (lane == 31) {
#pragma unroll
            for (int r = 0; r < RPW; ++r) sm.lrsp[row0 + r] = v[r][3];
        }
        if (warp == NW - 1) {
            *reinterpret_cast<uint4*>(&sm.lcsp[col0]) =
                make_uint4(to_bits(v[RPW - 1][0]), to_bits(v[RPW - 1][1]), to_bits(v[RPW - 1][2]),
                           to_bits(v[RPW - 1][3]));
        }
        __syncthreads();  // (2) lrsp / lcsp visible

        // ---- Steps 2.A / 2.B / 3.2: publish local aggregates and look back (three warps at once)
        if (warp == 0) {
            V mine[ER];
            uint64_t w[ER];
#pragma unroll
            for (int e = 0; e < ER; ++e) mine[e] = sm.lrsp[lane * ER + e];
            uint64_t* slot = p.row_slots + tidx * TR + lane * ER;
            V acc[ER];
            if (J == 0) {
#pragma unroll
                for (int e = 0; e < ER; ++e) { acc[e] = V(0); w[e] = pack(epoch, kIncl, to_bits(mine[e])); }
                st_words<ER>(slot, w);
            } else {
#pragma unroll
                for (int e = 0; e < ER; ++e) w[e] = pack(epoch, kLocal, to_bits(mine[e]));
                st_words<ER>(slot, w);
                lookback_vec<V, ER>(slot - TR, -static_cast<long long>(TR), epoch, acc);
#pragma unroll
                for (int e = 0; e < ER; ++e) w[e] = pack(epoch, kIncl, to_bits(acc[e] + mine[e]));
                st_words<ER>(slot, w);
            }
#pragma unroll
            for (int e = 0; e < ER; ++e) sm.rp[lane * ER + e] = acc[e];
        } else if (warp == 1) {
            V mine[EC];
            uint64_t w[EC];
#pragma unroll
            for (int e = 0; e < EC; ++e) mine[e] = sm.lcsp[lane * EC + e];
            uint64_t* slot = p.col_slots + tidx * TC + lane * EC;
            V acc[EC];
            if (I == 0) {
#pragma unroll
                for (int e = 0; e < EC; ++e) { acc[e] = V(0); w[e] = pack(epoch, kIncl, to_bits(mine[e])); }
                st_words<EC>(slot, w);
            } else {
#pragma unroll
                for (int e = 0; e < EC; ++e) w[e] = pack(epoch, kLocal, to_bits(mine[e]));
                st_words<EC>(slot, w);
                lookback_vec<V, EC>(slot - static_cast<long long>(p.C) * TC,
                                    -static_cast<long long>(p.C) * TC, epoch, acc);
#pragma unroll
                for (int e = 0; e < EC; ++e) w[e] = pack(epoch, kIncl, to_bits(acc[e] + mine[e]));
                st_words<EC>(slot, w);
            }
#pragma unroll
            for (int e = 0; e < EC; ++e) sm.cp[lane * EC + e] = acc[e];
        } else if (warp == 2) {
            V corner;
            const bool ok = lookback_diag<V>(p.corner_slots, I, J, p.C, epoch, /*blocking=*/false, lane, corner);
            if (lane == 0) {
                sm.corner = ok ? corner : V(0);
                sm.corner_ok = ok ? 1 : 0;
            }
        }
        __syncthreads();  // (3) rp, cp, corner (if resolved) visible

        // ---- Steps 3.1 / 3.3: GLS(I,J) and GS(I,J) = GS(I-1,J-1) + GLS(I,J)
        if (warp == 2) {
            const V gls = sm.lcsp[TC - 1] + sm.rp[TR - 1] + sm.cp[TC - 1];
            uint64_t* cslot = p.corner_slots + tidx;
            V corner = sm.corner;
            if (!sm.corner_ok) {
                if (lane == 0) st_relaxed(cslot, pack(epoch, kLocal, to_bits(gls)));
                lookback_diag<V>(p.corner_slots, I, J, p.C, epoch, /*blocking=*/true, lane, corner);
                if (lane == 0) sm.corner = corner;
            }
            if (lane == 0) st_relaxed(cslot, pack(epoch, kIncl, to_bits(corner + gls)));
        }
        __syncthreads();  // (4) corner visible

        // ---- Step 4: GSAT(I,J) = localSAT + rp[i] + cp[j] + corner (+ carry[j])
        {
            V colterm[4];
            const V corner = sm.corner;
            {
                const uint4 q = *reinterpret_cast<const uint4*>(&sm.cp[col0]);
                colterm[0] = from_bits<V>(q.x) + corner; colterm[1] = from_bits<V>(q.y) + corner;
                colterm[2] = from_bits<V>(q.z) + corner; colterm[3] = from_bits<V>(q.w) + corner;
            }
            if constexpr (CARRY) {
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    const long long gj = static_cast<long long>(J) * TC + col0 + c;
                    colterm[c] = colterm[c] + (gj < p.cols ? p.carry[gj] : V(0));
                }
            }
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                const V rt = sm.rp[row0 + r];
#pragma unroll
                for (int c = 0; c < 4; ++c) v[r][c] = v[r][c] + (rt + colterm[c]);
            }
        }

        if constexpr (TMA) {
#pragma unroll
            for (int r = 0; r < RPW; ++r)
                *reinterpret_cast<uint4*>(&tile[(row0 + r) * TC + col0]) =
                    make_uint4(to_bits(v[r][0]), to_bits(v[r][1]), to_bits(v[r][2]), to_bits(v[r][3]));
            fence_proxy_async_smem();
            __syncthreads();  // (5) tile in smem; tile_id[sn] visible
            if (producer) {
                tma_store_2d(&map_out, tile, J * TC, I * TR);
                bulk_commit();
            }
        } else {
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                const long long gi = static_cast<long long>(I) * TR + row0 + r;
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    const long long gj = static_cast<long long>(J) * TC + col0 + c;
                    if (gi < p.rows && gj < p.cols) p.dst[gi * p.pitch + gj] = v[r][c];
                }
            }
            __syncthreads();  // (5) tile_id[sn] visible
        }
        s = sn;
    }

    // ---- teardown: drain TMA stores; the last CTA to leave resets the counter and bumps the epoch
    if (producer) {
        if constexpr (TMA) bulk_wait_all();
        __threadfence();
        const unsigned int done = atomicAdd(&p.ctrl->exit_count, 1u);
        if (done == gridDim.x - 1) {
            p.ctrl->counter = 0u;
            p.ctrl->exit_count = 0u;
            p.ctrl->epoch = (epoch >= kEpochMax) ? 1u : epoch + 1u;
            __threadfence();
        }
    }
}

// Test hook: the serial -> (I, J) map exactly as the kernel evaluates it.
__global__ void tile_order_kernel(int R, int C, int order, int32_t* out) {
    const int n = R * C;
    for (int s = blockIdx.x * blockDim.x + threadIdx.x; s < n; s += gridDim.x * blockDim.x) {
        int I, J;
        tile_of_serial(s, R, C, order, I, J);
        out[2 * s] = I;
        out[2 * s + 1] = J;
    }
}

}  // namespace sat
