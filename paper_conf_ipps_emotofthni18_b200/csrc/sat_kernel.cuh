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
//   row look-back (warp 0), column look-back (warp 1), diagonal look-back (warp 2), each started
//     speculatively at the top of the tile so its first L2 round trip overlaps the local SAT
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

// Diagnosis builds only (-DSAT_DIAG_SITE=k): a per-THREAD pseudo-random sleep at publication site k
#if defined(SAT_DIAG_SITE)
#define SAT_DIAG_SLEEP(site)                                                                                   \
    do {                                                                                                      \
        if ((site) == SAT_DIAG_SITE) {                                                                        \
            uint64_t z_ = static_cast<uint64_t>(clock64()) ^ (static_cast<uint64_t>(blockIdx.x) << 40) ^      \
                          (static_cast<uint64_t>(threadIdx.x) << 20);                                         \
            z_ = (z_ ^ (z_ >> 30)) * 0xbf58476d1ce4e5b9ull;                                                   \
            z_ ^= z_ >> 31;                                                                                   \
            if ((z_ & 3u) == 0u) __nanosleep(static_cast<unsigned>((z_ >> 8) & 4095u));                      \
        }                                                                                                     \
    } while (0)
#else
#define SAT_DIAG_SLEEP(site) (void)0
#endif

constexpr uint32_t kLocal = 1u;
constexpr uint32_t kIncl = 2u;
constexpr uint32_t kEpochMax = (1u << 30) - 1u;

// Optional per-CTA phase counters (build with -DSAT_STATS=1; tools/stats.py reads them).
#ifndef SAT_STATS
#define SAT_STATS 0
#endif
// Tuning builds (-DSAT_EXPERIMENTAL=1): the kernel configurations measured in round 1 and not shipped.
#ifndef SAT_EXPERIMENTAL
#define SAT_EXPERIMENTAL 0
#endif
constexpr int kNumStats = 24;
enum StatSlot {
    kStTiles = 0, kStLoop, kStTicket, kStFullWait, kStCompute, kStRowLb, kStRowSteps, kStRowSpins, kStColLb,
    kStColSteps, kStColSpins, kStDiagTry, kStDiagUnresolved, kStDiagLate, kStBar3Producer, kStStore,
    kStStoreWait, kStBar1, kStPublish, kStBar3
};
#if SAT_STATS
#define SAT_CLK(x) const long long x = clock64()
#define SAT_ST(k, v) st[k] += (v)
#else
#define SAT_CLK(x) (void)0
#define SAT_ST(k, v) (void)0
#endif

struct Ctrl {
    unsigned int counter;     // SKSS tile counter c, reset by the last CTA to exit
    unsigned int exit_count;  // CTAs that have exited this launch
    unsigned int epoch;       // current launch epoch, 1 .. kEpochMax
    unsigned int pad;
};

// Chained strip partition (sat_compute_chained): rank r's
// strip takes its column carry T(r-1) = the column sums of all rows of ranks 0 .. r-1, which rank r-1
// pushes (as epoch-tagged status words, prefix form over each tile's columns) into rank r's inbox over
// NVLink peer memory as soon as its bottom tile of that tile column resolves (T(r-1) = its own strip
// column sums + the T(r-2) it received).
constexpr int kMaxChainRanks = 8;
struct ChainParams {
    int rank, nranks;
    uint32_t parity;                         // inbox half of this call (epoch & 1)
    int64_t inbox_cols;                      // words per inbox vector (>= C * TC)
    uint64_t* peer_inbox[kMaxChainRanks];    // inbox of every rank: [2][inbox_cols] words (written by rank - 1)
    uint32_t* peer_done[kMaxChainRanks];     // back-pressure words of every rank: [kMaxChainRanks] (rank + 1's used)
};

template <typename V>
struct KParams {
    const V* src;  // generic path only
    V* dst;        // generic path, and ragged right-edge tiles of the TMA path
    int64_t rows, cols, pitch;
    int R, C;          // tile grid
    int ntiles;
    int order;         // 0 = diagonal-major (Fig. 9), 1 = row-major
    uint64_t* row_slots;     // [R*C][TR]
    uint64_t* col_slots;     // [R*C][TC]
    uint64_t* corner_slots;  // [R*C]
    Ctrl* ctrl;
    const V* carry;    // [cols] or nullptr
    long long* stats;  // [gridDim.x][kNumStats] (SAT_STATS builds only) or nullptr
    long long* trace;  // [ntiles][2]: acquisition / store-issue globaltimer ns (SAT_STATS builds only)
    const uint8_t* src8;  // u8 input (integral images, sat_compute_u8): generic path only, else nullptr
    int64_t src_pitch;    // row stride of src8 in bytes
    uint32_t epoch_override;  // != 0: the launch epoch chosen by the host (chained calls); ctrl->epoch untouched
    int l2_prefetch;          // TMEM-parked kernels: L2 prefetch of a tile's boxes as soon as it is acquired
    ChainParams chain;        // chained strip partition only
};

__device__ __forceinline__ uint64_t pack(uint32_t epoch, uint32_t kind, uint32_t bits) {
    return (static_cast<uint64_t>((epoch << 2) | kind) << 32) | bits;
}
__device__ __forceinline__ bool word_ready(uint64_t w, uint32_t epoch) {
    return static_cast<uint32_t>(w >> 34) == epoch;
}
__device__ __forceinline__ uint32_t word_kind(uint64_t w) { return static_cast<uint32_t>(w >> 32) & 3u; }

// ------------------------------------------------------------------ serial number -> tile
// Fig. 9 order generalised to an R x C tile grid (reading R6): diagonals d = I+J = 0, 1, 2, ... in
// turn, I ascending within a diagonal.  With m = min(R,C), M = max(R,C), diagonal d holds d+1 tiles
// for d < m, m tiles for m <= d < M and R+C-1-d tiles for d >= M, so the serial number of the
// first tile of a diagonal is a closed form and its inverse needs one square root.
__device__ __forceinline__ long long tri(long long k) { return k * (k + 1) / 2; }

__device__ __forceinline__ long long tri_floor_inv(long long s) {  // largest k with tri(k) <= s
    long long k = static_cast<long long>((sqrt(8.0 * static_cast<double>(s) + 1.0) - 1.0) * 0.5);
    while (tri(k + 1) <= s) ++k;
    while (k > 0 && tri(k) > s) --k;
    return k;
}

__device__ __forceinline__ void diag_of_serial(long long s, int R, int C, int& I, int& J) {
    const long long m = R < C ? R : C, M = R < C ? C : R;
    const long long headA = tri(m);            // tiles on diagonals d < m
    const long long headB = headA + (M - m) * m;  // ... on diagonals d < M
    long long d, base;
    if (s < headA) {
        d = tri_floor_inv(s);       // tri(d) <= s < tri(d+1): s lies on diagonal d
        base = tri(d);
    } else if (s < headB) {
        d = m + (s - headA) / m;
        base = headA + (d - m) * m;
    } else {
        const long long r = static_cast<long long>(R) * C - 1 - s;  // index from the end
        const long long e = tri_floor_inv(r);                       // diagonal counted from the end
        d = static_cast<long long>(R) + C - 2 - e;
        base = static_cast<long long>(R) * C - tri(e + 1);
    }
    const long long i0 = d - C + 1 > 0 ? d - C + 1 : 0;
    I = static_cast<int>(i0 + (s - base));
    J = static_cast<int>(d - I);
}

// order & 15: 0 = anti-diagonal (Fig. 9), 1 = row-major, 2 = column-major.  (order >> 8) & 255 = g > 1 with order & 15
// == 0 and g | C: anti-diagonal order of g-wide tile groups, the g tiles of a group consecutive and
// left to right (a topological order too: a tile's left neighbour is earlier in its group or on the
// previous group diagonal, its upper neighbours on the previous group diagonal).  The g tiles of a
// group share their DRAM rows, so the rows concurrent tiles touch are g times longer.  order & 15 == 3
// with g | R: anti-diagonal order of g-TALL tile groups, the g tiles of a group consecutive and top to
// bottom (chained strips: the bottom tile of tile column J resolves R/g group diagonals after the top one,
// and a column look-back spans at most the g - 1 tiles above in the group plus one inclusive word).
__device__ __forceinline__ void tile_of_serial(int s_, int R, int C, int order, int& I, int& J) {
    if ((order & 15) == 1) {
        I = s_ / C;
        J = s_ - I * C;
        return;
    }
    if ((order & 15) == 2) {  // column-major (chained strips: a tile column's tiles are consecutive)
        J = s_ / R;
        I = s_ - J * R;
        return;
    }
    const int g = (order >> 8) & 255;
    if ((order & 15) == 3) {
        if (g > 1 && R % g == 0) {
            diag_of_serial(s_ / g, R / g, C, I, J);
            I = I * g + s_ % g;
        } else {
            diag_of_serial(s_, R, C, I, J);
        }
        return;
    }
    if (g > 1 && C % g == 0) {
        int J2;
        diag_of_serial(s_ / g, R, C / g, I, J2);
        J = J2 * g + s_ % g;
        return;
    }
    diag_of_serial(s_, R, C, I, J);
}

// ------------------------------------------------------------------ look-backs
// Row / column look-back (Steps 2.A.2 / 2.B.2, Fig. 10): walk predecessors
// p, p+step, p+2*step, ... summing local aggregates until an inclusive one is found.  Each lane
// owns E consecutive elements of the vector and resolves each element independently (an element
// stops at its first inclusive word); the warp walks until every element of every lane is done.
// `w` holds words already loaded from p (a speculative early poll); not-ready words are re-polled.
// Termination: the tile at the grid edge (J=0 / I=0) always publishes inclusive (reading R10').
template <typename V, int E>
__device__ __forceinline__ void lookback_vec(const uint64_t* p, long long step, uint32_t epoch, V (&acc)[E],
                                             uint64_t (&w)[E], int& steps, int& spins) {
    uint32_t pending = (1u << E) - 1u;
#pragma unroll
    for (int e = 0; e < E; ++e) acc[e] = V(0);
    SAT_SPIN_DECL;
    while (true) {
        if (pending) {
            ++steps;
            while (true) {
                bool ok = true;
#pragma unroll
                for (int e = 0; e < E; ++e)
                    if (((pending >> e) & 1u) && !word_ready(w[e], epoch)) ok = false;
                if (ok) break;
                ++spins;
                SAT_SPIN_CHECK("a row / column look-back word");
                __nanosleep(20);
                ld_words<E>(p, w);
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
        if (pending) ld_words<E>(p, w);
    }
}

// Diagonal look-back (Step 3.2): GS(I-1,J-1) = GS(I-k,J-k) + sum_{0<k'<k} GLS(I-k',J-k').
// The warp inspects a window of 32 diagonal predecessors at once (lane k-1 <-> tile (I-k, J-k)).
__device__ __forceinline__ uint64_t diag_word(const uint64_t* corner_slots, int I, int J, int C, int k) {
    return (I - k >= 0 && J - k >= 0) ? ld_relaxed(corner_slots + static_cast<long long>(I - k) * C + (J - k)) : 0ull;
}

// Non-blocking mode returns false as soon as a needed word is not yet published.  `w` is the word of
// window position base=1 for this lane (speculative early poll).
template <typename V>
__device__ __forceinline__ bool lookback_diag(const uint64_t* corner_slots, int I, int J, int C, uint32_t epoch,
                                              bool blocking, int lane, uint64_t w, V& out) {
    if (I == 0 || J == 0) {
        out = V(0);
        return true;
    }
    V acc = V(0);
    int base = 1;
    SAT_SPIN_DECL;
    while (true) {
        const int k = base + lane;
        const bool inrange = (I - k >= 0) && (J - k >= 0);
        const bool ready = !inrange || word_ready(w, epoch);
        const unsigned incl = __ballot_sync(kFull, inrange && ready && word_kind(w) == kIncl);
        const unsigned notready = __ballot_sync(kFull, !ready);
        const int f = incl ? (__ffs(incl) - 1) : 32;
        const unsigned need = (f >= 31) ? kFull : ((2u << f) - 1u);
        if (notready & need) {
            if (!blocking) return false;
            SAT_SPIN_CHECK("a diagonal look-back word");
            __nanosleep(20);
            w = diag_word(corner_slots, I, J, C, k);
            continue;
        }
        V val = (inrange && lane <= f) ? from_bits<V>(static_cast<uint32_t>(w)) : V(0);
        acc = acc + warp_sum(val);
        if (f < 32) {
            out = acc;
            return true;
        }
        base += 32;
        w = diag_word(corner_slots, I, J, C, base + lane);
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
    static_assert(RPW % 2 == 0 || RPW == 1, "row slots are published in pairs");
    static_assert(ER == 1 || ER % 2 == 0, "row vector split");
};

struct TileInfo {
    int t, I, J, pad;
};

template <typename V, typename Cfg>
struct Smem {
    alignas(1024) V stage[Cfg::STAGES][Cfg::TR * Cfg::TC];
    alignas(16) V band[Cfg::NW][Cfg::TC];
    alignas(16) V rp[Cfg::TR];
    alignas(16) V cp[Cfg::TC];
    alignas(8) uint64_t full[Cfg::STAGES];
    alignas(16) TileInfo info[Cfg::STAGES];
    V corner;
    V total;
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
#if SAT_STATS
    long long st[kNumStats];
#pragma unroll
    for (int k = 0; k < kNumStats; ++k) st[k] = 0;
#endif
    int n_steps = 0, n_spins = 0;

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
        TileInfo ti{t0, 0, 0, 0};
        if (t0 < p.ntiles) tile_of_serial(t0, p.R, p.C, p.order, ti.I, ti.J);
        sm.info[0] = ti;
        if constexpr (TMA) {
            if (t0 < p.ntiles) {
                mbar_arrive_expect_tx(&sm.full[0], kTileBytes);
                tma_load_2d(sm.stage[0], &map_in, &sm.full[0], ti.J * TC, ti.I * TR, policy);
            }
        }
    }
    __syncthreads();
    const uint32_t epoch = sm.epoch;

    uint32_t phase_bits = 0;  // parity of each stage's mbarrier
    int s = 0;
    while (true) {
        SAT_CLK(c_top);
        const TileInfo ti = sm.info[s];
        if (ti.t >= p.ntiles) break;
        const int I = ti.I, J = ti.J;
        const int sn = (s + 1 == STAGES) ? 0 : s + 1;
        const long long tidx = static_cast<long long>(I) * p.C + J;
        V* tile = sm.stage[s];
        const int row0 = warp * RPW;
        const int col0 = lane * 4;
        SAT_ST(kStTiles, 1);

        // ---- ticket for the next tile: issued now, consumed after the local scans (latency hidden)
        unsigned int ticket = 0;
        if (producer) ticket = atomicAdd(&p.ctrl->counter, 1u);

        // ---- speculative first polls of the look-backs (their L2 round trip overlaps the local SAT)
        uint64_t wr[ER], wc[EC], wd = 0;
        if (warp == 0 && J > 0) ld_words<ER>(p.row_slots + (tidx - 1) * TR + lane * ER, wr);
        if (warp == 1 && I > 0) ld_words<EC>(p.col_slots + (tidx - p.C) * TC + lane * EC, wc);
        if (warp == 2) wd = diag_word(p.corner_slots, I, J, p.C, 1 + lane);

        // ---- Step 1: tile -> registers (lane owns 4 columns of RPW rows)
        SAT_CLK(c_fw0);
        V v[RPW][4];
        if constexpr (TMA) {
            mbar_wait(&sm.full[s], (phase_bits >> s) & 1u);
            phase_bits ^= (1u << s);
            SAT_CLK(c_fw1);
            SAT_ST(kStFullWait, c_fw1 - c_fw0);
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                const uint4 q = *reinterpret_cast<const uint4*>(&tile[(row0 + r) * TC + col0]);
                v[r][0] = from_bits<V>(q.x); v[r][1] = from_bits<V>(q.y);
                v[r][2] = from_bits<V>(q.z); v[r][3] = from_bits<V>(q.w);
            }
            // Right-edge tile: TMA moves 16-byte granules, so a row whose width is not a multiple of
            // 4 elements may bring in pad words; zero every column >= cols (partial tiles are
            // zero-padded, reading R2).
            if (J == p.C - 1) {
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    if (static_cast<long long>(J) * TC + col0 + c >= p.cols) {
#pragma unroll
                        for (int r = 0; r < RPW; ++r) v[r][c] = V(0);
                    }
                }
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

        // ---- producer: consume the ticket, prefetch the next tile into the next stage
        if (producer) {
            SAT_CLK(c_tk);
            const int tn = static_cast<int>(ticket);
            TileInfo nx{tn, 0, 0, 0};
            if (tn < p.ntiles) tile_of_serial(tn, p.R, p.C, p.order, nx.I, nx.J);
            sm.info[sn] = nx;
            SAT_CLK(c_tk2);
            SAT_ST(kStTicket, c_tk2 - c_tk);
            if constexpr (TMA) {
                if (tn < p.ntiles) {
                    // the stage being refilled was last stored STAGES-1 tiles ago
                    bulk_wait_read<STAGES - 2>();
                    SAT_CLK(c_sw1);
                    SAT_ST(kStStoreWait, c_sw1 - c_tk2);
                    mbar_arrive_expect_tx(&sm.full[sn], kTileBytes);
                    tma_load_2d(sm.stage[sn], &map_in, &sm.full[sn], nx.J * TC, nx.I * TR, policy);
                }
            }
        }
        SAT_CLK(c_b1a);
        SAT_ST(kStCompute, c_b1a - c_fw0);
        __syncthreads();  // (1) band bottoms visible
        SAT_CLK(c_b1b);
        SAT_ST(kStBar1, c_b1b - c_b1a);

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

        SAT_JITTER_WARP();
        // ---- Steps 2.A.1 / 2.B.1: publish the local aggregates straight from the owning lanes.
        //      Row slots: lane 31 of every warp (last column of its rows); column slots: the last
        //      warp (bottom row).  Edge tiles publish inclusive at once (their carry is zero).
        if (lane == 31) {
            SAT_DIAG_SLEEP(1);
            uint64_t* rs = p.row_slots + tidx * TR + row0;
            const uint32_t kind = (J == 0) ? kIncl : kLocal;
#pragma unroll
            for (int r = 0; r < RPW; r += 2) {
                if constexpr (RPW == 1) {
                    st_relaxed(rs, pack(epoch, kind, to_bits(v[0][3])));
                } else {
                    st_relaxed2(rs + r, pack(epoch, kind, to_bits(v[r][3])), pack(epoch, kind, to_bits(v[r + 1][3])));
                }
            }
        }
        if (warp == NW - 1) {
            uint64_t* cs = p.col_slots + tidx * TC + col0;
            const uint32_t kind = (I == 0) ? kIncl : kLocal;
            SAT_DIAG_SLEEP(2);
            st_relaxed2(cs, pack(epoch, kind, to_bits(v[RPW - 1][0])), pack(epoch, kind, to_bits(v[RPW - 1][1])));
            st_relaxed2(cs + 2, pack(epoch, kind, to_bits(v[RPW - 1][2])), pack(epoch, kind, to_bits(v[RPW - 1][3])));
            if (lane == 31) sm.total = v[RPW - 1][3];
        }
        SAT_CLK(c_pub);
        SAT_ST(kStPublish, c_pub - c_b1b);

        // ---- Steps 2.A.2 / 2.B.2 / 3.2: the look-backs (three warps at once)
        if (warp == 0) {
            V acc[ER];
            if (J == 0) {
#pragma unroll
                for (int e = 0; e < ER; ++e) acc[e] = V(0);
            } else {
                lookback_vec<V, ER>(p.row_slots + (tidx - 1) * TR + lane * ER, -static_cast<long long>(TR), epoch,
                                    acc, wr, n_steps, n_spins);
            }
#pragma unroll
            for (int e = 0; e < ER; ++e) sm.rp[lane * ER + e] = acc[e];
        } else if (warp == 1) {
            V acc[EC];
            if (I == 0) {
#pragma unroll
                for (int e = 0; e < EC; ++e) acc[e] = V(0);
            } else {
                lookback_vec<V, EC>(p.col_slots + (tidx - p.C) * TC + lane * EC, -static_cast<long long>(p.C) * TC,
                                    epoch, acc, wc, n_steps, n_spins);
            }
            *reinterpret_cast<uint4*>(&sm.cp[lane * EC]) =
                make_uint4(to_bits(acc[0]), to_bits(acc[1]), to_bits(acc[2]), to_bits(acc[3]));
        } else if (warp == 2) {
            V corner;
            const bool ok = lookback_diag<V>(p.corner_slots, I, J, p.C, epoch, /*blocking=*/false, lane, wd, corner);
            if (lane == 0) {
                sm.corner = ok ? corner : V(0);
                sm.corner_ok = ok ? 1 : 0;
            }
        }
        SAT_CLK(c_b3a);
#if SAT_STATS
        if (warp == 0) { SAT_ST(kStRowLb, c_b3a - c_pub); }
        if (warp == 1) { SAT_ST(kStColLb, c_b3a - c_pub); }
        if (warp == 2) { SAT_ST(kStDiagTry, c_b3a - c_pub); SAT_ST(kStDiagUnresolved, sm.corner_ok ? 0 : 1); }
#endif
        __syncthreads();  // (3) rp, cp, corner (if resolved), total visible
        SAT_CLK(c_b3b);
        if (warp == 3) SAT_ST(kStBar3Producer, c_b3b - c_b3a); else SAT_ST(kStBar3, c_b3b - c_b3a);

        SAT_JITTER_WARP();
        // ---- Steps 2.A.3 / 2.B.3: publish the inclusive aggregates (owners of the local values)
        if (lane == 31 && J > 0) {
            SAT_DIAG_SLEEP(5);
            uint64_t* rs = p.row_slots + tidx * TR + row0;
#pragma unroll
            for (int r = 0; r < RPW; r += 2) {
                if constexpr (RPW == 1) {
                    st_relaxed(rs, pack(epoch, kIncl, to_bits(v[0][3] + sm.rp[row0])));
                } else {
                    st_relaxed2(rs + r, pack(epoch, kIncl, to_bits(v[r][3] + sm.rp[row0 + r])),
                                pack(epoch, kIncl, to_bits(v[r + 1][3] + sm.rp[row0 + r + 1])));
                }
            }
        }
        if (warp == NW - 1 && I > 0) {
            SAT_DIAG_SLEEP(6);
            uint64_t* cs = p.col_slots + tidx * TC + col0;
            const uint4 q = *reinterpret_cast<const uint4*>(&sm.cp[col0]);
            st_relaxed2(cs, pack(epoch, kIncl, to_bits(v[RPW - 1][0] + from_bits<V>(q.x))),
                        pack(epoch, kIncl, to_bits(v[RPW - 1][1] + from_bits<V>(q.y))));
            st_relaxed2(cs + 2, pack(epoch, kIncl, to_bits(v[RPW - 1][2] + from_bits<V>(q.z))),
                        pack(epoch, kIncl, to_bits(v[RPW - 1][3] + from_bits<V>(q.w))));
        }

        // ---- Steps 3.1 / 3.3: GLS(I,J) = total + rp[TR-1] + cp[TC-1]; GS(I,J) = GS(I-1,J-1) + GLS(I,J)
        const V gls = sm.total + sm.rp[TR - 1] + sm.cp[TC - 1];
        uint64_t* cslot = p.corner_slots + tidx;
        if (!sm.corner_ok) {  // uniform: read after barrier (3)
            if (warp == 2) {
                if (lane == 0) {
                    SAT_DIAG_SLEEP(3);
                    st_relaxed(cslot, pack(epoch, kLocal, to_bits(gls)));
                }
                V corner;
                lookback_diag<V>(p.corner_slots, I, J, p.C, epoch, /*blocking=*/true, lane,
                                 diag_word(p.corner_slots, I, J, p.C, 1 + lane), corner);
                if (lane == 0) sm.corner = corner;
            }
            __syncthreads();  // (4) corner visible (rare)
        }
        const V corner = sm.corner;
        if (warp == 2 && lane == 0) {
            SAT_DIAG_SLEEP(4);
            st_relaxed(cslot, pack(epoch, kIncl, to_bits(corner + gls)));
        }
        SAT_CLK(c_b4);
        SAT_ST(kStDiagLate, c_b4 - c_b3b);

        // ---- Step 4: GSAT(I,J) = localSAT + rp[i] + cp[j] + corner (+ carry[j])
        {
            V colterm[4];
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

        // A right-edge tile whose row width is not a multiple of 4 elements is stored element by
        // element (a TMA store would write whole 16-byte granules, i.e. pad words, P:54 layout / R3).
        const bool ragged = TMA && (J == p.C - 1) && (p.cols & 3) != 0;
        if (TMA && !ragged) {
#pragma unroll
            for (int r = 0; r < RPW; ++r)
                *reinterpret_cast<uint4*>(&tile[(row0 + r) * TC + col0]) =
                    make_uint4(to_bits(v[r][0]), to_bits(v[r][1]), to_bits(v[r][2]), to_bits(v[r][3]));
            fence_proxy_async_smem();
            __syncthreads();  // (5) tile in smem; info[sn] visible
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
            __syncthreads();  // (5) info[sn] visible
            if (TMA && producer) bulk_commit();  // empty bulk group: keep one group per tile
        }
        SAT_CLK(c_end);
        SAT_ST(kStStore, c_end - c_b4);
        SAT_ST(kStLoop, c_end - c_top);
        s = sn;
    }
#if SAT_STATS
    if (warp == 0) { st[kStRowSteps] = n_steps; st[kStRowSpins] = n_spins; }
    if (warp == 1) { st[kStColSteps] = n_steps; st[kStColSpins] = n_spins; }
    if (p.stats && lane == 0 && warp < 4) {
        long long* out = p.stats + static_cast<long long>(blockIdx.x) * kNumStats;
        for (int k = 0; k < kNumStats; ++k) {
            const bool mine = (warp == 0 && (k == kStTiles || k == kStLoop || k == kStCompute || k == kStRowLb ||
                                              k == kStRowSteps || k == kStRowSpins || k == kStStore ||
                                              k == kStBar1 || k == kStPublish || k == kStBar3 ||
                                              k == kStFullWait)) ||
                              (warp == 1 && (k == kStColLb || k == kStColSteps || k == kStColSpins)) ||
                              (warp == 2 && (k == kStDiagTry || k == kStDiagUnresolved || k == kStDiagLate)) ||
                              (warp == 3 && (k == kStTicket || k == kStStoreWait || k == kStBar3Producer));
            if (mine) out[k] = st[k];
        }
    }
#endif
    (void)n_steps;
    (void)n_spins;

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
