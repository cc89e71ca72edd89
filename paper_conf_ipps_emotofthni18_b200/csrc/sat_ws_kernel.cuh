// sat_ws_kernel.cuh -- warp-specialised single-pass SAT kernel for sm_100a (the production kernel).
//
// Same method and same published aggregates as sat_tiles_kernel (sat_kernel.cuh: 1R1W-SKSS-LB of
// PAPER.md Sec. IV, prefix-form slots, epoch-tagged status words), but the steps of a tile
// run on dedicated warps so that their latencies overlap.  Measured on B200: with HBM saturated an
// L2 round trip (a look-back poll) costs ~1-2 us, the same order as one tile's whole compute, so the
// look-backs must run ahead of the tile they serve.  Roles of a persistent CTA:
//
//   loader (1 lane)    SKSS ticket c <- atomicAdd(&c,1) (drawn one tile ahead),
//                      Fig. 9 serial -> (I,J), TMA 2-D load of T(I,J) into a ring of STAGES
//                      shared-memory stages (Step 1).
//   row walker warp    row look-back (Step 2.A.2) and diagonal look-back (Step 3.2,
//                      P:241) of the CTA's tiles, started as soon as a tile is acquired, several
//                      tiles per polling round; results -> the tile's stage slots (rp, corner).
//   column walker warp column look-back (Step 2.B.2); result -> cp.
//   NW compute warps   local SAT of the tile in registers; local aggregates published
//                      from the owning lanes (Steps 2.A.1, 2.B.1); once the walks are in, the
//                      inclusive aggregates GRS/GCS/GS from the same lanes (Steps 2.A.3, 2.B.3, 3.1,
//                      3.3) and the Step 4 correction (rule P:150) written to the stage.
//   storer (1 lane)    TMA 2-D store of GSAT(I,J) (Step 4), two in flight; frees stages.
//
// Hand-offs are mbarriers per stage: acq (tile id written), full (TMA bytes landed, or "no more
// tiles"), rowwalk / colwalk (carries in smem), result (GSAT in smem, NW arrivals), empty (stage read
// by its TMA store).  Each completes once per use of its stage (tile k: stage k % STAGES, parity
// (k / STAGES) & 1, tracked incrementally by Slot).  Forward progress: tiles are acquired in serial
// order; every role handles its CTA's tiles in that order; a walk only waits on tiles with smaller
// serial numbers, whose local aggregates depend on nothing but their own data.
#pragma once

#include "sat_pipe.cuh"

namespace sat {
// Option bits of WsCfg (see the roles above).
enum WsFlags : int {
    kWsFast = 1,      // compute warps poll the direct predecessors themselves (walkers as fallback)
    kWsDefer = 2,     // finish tile k after the local SAT of tile k+1 (local SAT parked in its stage)
    kWsDirect = 4,    // GSAT stored from registers (no TMA store, no storer)
    kWsPrefetch = 8,  // L2 prefetch of a tile's pixels as soon as it is acquired
    kWsSmemScan = 16, // row scans transposed through shared memory instead of shuffle scans
};

template <int TR_, int NW_, int STAGES_, int NT_, int NQ_, int FLAGS_ = 0>
struct WsCfg {
    static constexpr int TR = TR_, TC = 128, NW = NW_, STAGES = STAGES_;
    static constexpr int NQ = NQ_;        // tile ring: tiles acquired ahead of their data stage
    static constexpr int NT = NT_;        // tiles in flight per walker
    static constexpr int FLAGS = FLAGS_;
    static constexpr bool FAST = (FLAGS & kWsFast) != 0;
    static constexpr bool DEFER = (FLAGS & kWsDefer) != 0;
    static constexpr bool DIRECT = (FLAGS & kWsDirect) != 0;
    static constexpr bool PREFETCH = (FLAGS & kWsPrefetch) != 0;
    static constexpr bool SMEM_SCAN = (FLAGS & kWsSmemScan) != 0;
    static constexpr bool WPUB = false;  // inclusive aggregates published by the compute warps
    static constexpr bool WPUB_WAIT = false;
    static constexpr int RPW = TR / NW;   // rows per compute-warp band
    static constexpr int ER = TR / 32;    // row-vector elements per walker lane
    static constexpr int EC = TC / 32;    // column-vector elements per walker lane
    static constexpr int ROW_WARP = NW, COL_WARP = NW + 1, STORE_WARP = NW + 2, LOAD_WARP = NW + 3;
    static constexpr int THREADS = (NW + 4) * 32;
    static constexpr int MINB = 1;
    static_assert(TR % NW == 0 && TR % 32 == 0, "tile shape");
    static_assert(RPW % 2 == 0, "row slots are published in pairs");
    static_assert(STAGES >= 2 && STAGES <= 8 && NT >= 1 && NQ >= STAGES && NQ <= 16, "rings");
    static_assert(!FAST || (NW >= 3 && ER <= 4 && ER % 2 == 0), "fast-path poll warps 0, 1, NW-1");
    static_assert(!(FAST && DEFER), "the fast-path poll registers would not survive the deferred finish");
    static_assert(!(FAST && DIRECT), "fast path releases tile slots through the storer");
};

// Two rings: the data stages (tile k's pixels live in stage k % STAGES) and the tile ring (tile k's
// id, carries and hand-off barriers live in slot k % NQ).  Tiles are acquired up to NQ ahead of the
// storer, i.e. before a data stage is free, so their look-backs start earlier.
template <typename V, typename Cfg>
struct WsSmem {
    alignas(1024) V stage[Cfg::STAGES][Cfg::TR * Cfg::TC];
    alignas(16) V band[2][Cfg::NW][Cfg::TC];
    alignas(16) V rp[Cfg::NQ][Cfg::TR];  // row carry    prefix_i GRS(I,J-1)
    alignas(16) V cp[Cfg::NQ][Cfg::TC];  // column carry prefix_j GCS(I-1,J)
    V corner[Cfg::NQ];                   // GS(I-1,J-1)
    alignas(16) V rpf[Cfg::TR];          // fast path: the same carries read from inclusive predecessors
    alignas(16) V cpf[Cfg::TC];
    V cornerf;
    int fok[3];                          // fast path: row / column / corner predecessor inclusive
    int fdone[Cfg::NQ];                  // tile slot resolved by the fast path (walkers may stop)
    alignas(8) uint64_t acq[Cfg::NQ];    // tile id written (tile ring)
    uint64_t rowwalk[Cfg::NQ];
    uint64_t colwalk[Cfg::NQ];
    uint64_t tfree[Cfg::NQ];             // tile slot released by the storer
    uint64_t full[Cfg::STAGES];          // data ring
    uint64_t result[Cfg::STAGES];
    uint64_t empty[Cfg::STAGES];
    alignas(16) TileInfo info[Cfg::NQ];
    uint32_t epoch;
    int end_n;  // index of the end marker once the loader has drawn an invalid ticket, else INT_MAX
};

// One round of a 2-deep windowed vector look-back (Steps 2.A.2 / 2.B.2): the lane's E elements,
// predecessor position `pos` (and pos-1) along the walk, words already loaded.  Consumes ready
// predecessors in order, stops at the first not-ready one.  Returns true if it made progress.
template <typename V, int E>
__device__ __forceinline__ bool lb_consume(uint32_t& pending, int& pos, V (&acc)[E], const uint64_t (&w0)[E],
                                           const uint64_t (&w1)[E], bool have1, uint32_t epoch) {
    bool progress = false;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        if (!pending || (h == 1 && !have1)) break;
        const uint64_t(&w)[E] = h == 0 ? w0 : w1;
        bool ok = true;
#pragma unroll
        for (int e = 0; e < E; ++e)
            if (((pending >> e) & 1u) && !word_ready(w[e], epoch)) ok = false;
        if (!ok) break;
#pragma unroll
        for (int e = 0; e < E; ++e) {
            if ((pending >> e) & 1u) {
                acc[e] = acc[e] + from_bits<V>(static_cast<uint32_t>(w[e]));
                if (word_kind(w[e]) == kIncl) pending &= ~(1u << e);
            }
        }
        pos -= 1;
        progress = true;
    }
    return progress;
}

// (SM: WsSmem, or any shared-memory layout with the same walker-facing members: acq, info, end_n,
// rp, cp, corner, rowwalk, colwalk.)
template <typename V, typename Cfg, bool ROW, typename SM>
__device__ __forceinline__ void ws_walker(SM& sm, const KParams<V>& p, uint32_t epoch, int lane) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC;
    constexpr int E = ROW ? Cfg::ER : Cfg::EC;
    constexpr int NT = Cfg::NT;
    struct Walk {
        int active, s, k, I, J, pos;
        uint32_t ph;
        uint32_t pend;
        V acc[E];
        V dacc;
        int dbase, ddone;
        long long t_acq;
    };
    Walk wk[NT];
#pragma unroll
    for (int w = 0; w < NT; ++w) wk[w].active = 0;
    // WPUB: a resolved tile whose local aggregates were not in yet (published, and handed to the
    // compute warps, as soon as they are; meanwhile the walker goes on with the next tiles)
    struct Pend {
        int on, s, k, I, J;
        uint32_t ph;
        V acc[E];
        V dacc;
    } pd;
    pd.on = 0;
    Slot<Cfg::NQ> next;
    bool ended = false;
    int steps = 0;
    const uint64_t pol = policy_evict_last();
    constexpr int DW = 4;  // diagonal predecessors polled per round (the first is almost always inclusive)
    // WPUB: Steps 2.A.3 / 2.B.3 (and 3.1 / 3.3 if the other walk of the tile is in) of a resolved tile
    // whose local aggregates (lrs / lcs, kept in smem by the compute warps) are in.  The walkers are then
    // the only publishers of inclusive aggregates: each tile's row / column words by its own walker, GS
    // by whichever of the two publishes second (each raises its rdone / cdone flag before it looks at
    // the other's, so at least one of them sees both).
    auto publish = [&](int s, int k, int I, int J, const V (&acc)[E], V dacc, bool gs_only = false) {
        if constexpr (Cfg::WPUB) {
            const long long tidx = static_cast<long long>(I) * p.C + J;
            V l[E];
            uint64_t wv[E];
#pragma unroll
            for (int e = 0; e < E; ++e) {
                l[e] = ROW ? sm.lrs[s][lane * E + e] : sm.lcs[s][lane * E + e];
                wv[e] = pack(epoch, kIncl, to_bits(l[e] + acc[e]));
            }
            if (!gs_only && (ROW ? J > 0 : I > 0))
                st_words_p<E>((ROW ? p.row_slots + tidx * TR : p.col_slots + tidx * TC) + lane * E, wv, pol);
            if (lane == 31 && *reinterpret_cast<volatile int*>(ROW ? &sm.cdone[s] : &sm.rdone[s]) == k + 1) {
                // GLS = total + rp[TR-1] + cp[TC-1];  GS = GS(I-1,J-1) + GLS
                __threadfence_block();  // acquire: the other walker's carries were written before its flag
                const V rp1 = ROW ? acc[E - 1] : sm.rp[s][TR - 1];
                const V cp1 = ROW ? sm.cp[s][TC - 1] : acc[E - 1];
                const V cor = ROW ? dacc : sm.corner[s];
                st_relaxed_p(p.corner_slots + tidx, pack(epoch, kIncl, to_bits(cor + ((l[E - 1] + rp1) + cp1))), pol);
            }
        }
    };
    auto hand_off = [&](int s) {
        __syncwarp();
        if (lane == 0) mbar_arrive(ROW ? &sm.rowwalk[s] : &sm.colwalk[s]);
    };
    while (true) {
        // ---- take newly acquired tiles into free walk slots (block only when nothing is in flight)
#pragma unroll
        for (int w = 0; w < NT; ++w) {
            if (wk[w].active || ended) continue;
            bool busy = pd.on != 0;
#pragma unroll
            for (int v2 = 0; v2 < NT; ++v2) busy = busy || wk[v2].active;
            bool got;
            if (busy) {
                got = mbar_test(&sm.acq[next.s], next.ph);
                if (!got && next.k >= *reinterpret_cast<volatile int*>(&sm.end_n)) ended = true;
            } else {
                got = wait_acquired(sm, next.s, next.ph, next.k);
                if (!got) ended = true;
            }
            if (!got) continue;
            const TileInfo ti = sm.info[next.s];
            if (ti.t >= p.ntiles) {
                ended = true;
                continue;
            }
            Walk& x = wk[w];
            x.active = 1;
            x.s = next.s;
            x.k = next.k;
            x.ph = next.ph;
            x.I = ti.I;
            x.J = ti.J;
            x.pos = ROW ? ti.J - 1 : ti.I - 1;
            x.pend = (x.pos >= 0) ? ((1u << E) - 1u) : 0u;
#pragma unroll
            for (int e = 0; e < E; ++e) x.acc[e] = V(0);
            x.dacc = V(0);
            x.dbase = 1;
            x.ddone = ROW ? (ti.I == 0 || ti.J == 0) : 1;
#if SAT_STATS
            x.t_acq = clock64();
#endif
            next.next();
        }
        bool any = pd.on != 0;
#pragma unroll
        for (int w = 0; w < NT; ++w) any = any || wk[w].active;
        if (!any) {
            if (ended) break;
            continue;
        }
        // ---- one polling round: issue every load first ...
        uint64_t w0[NT][E], w1[NT][E], wd[NT];
        bool fd[NT];
#pragma unroll
        for (int w = 0; w < NT; ++w) {
            const Walk& x = wk[w];
            wd[w] = 0;
            fd[w] = false;
            if (!x.active) continue;
            if constexpr (Cfg::FAST) {
                // the compute warps found the direct predecessors inclusive: nothing left to walk
                fd[w] = __shfl_sync(kFull, *reinterpret_cast<volatile int*>(&sm.fdone[x.s]), 0) != 0;
                if (fd[w]) continue;
            }
            if (x.pend) {
                if (ROW) {
                    const long long base = static_cast<long long>(x.I) * p.C;
                    ld_words_p<E>(p.row_slots + (base + x.pos) * TR + lane * E, w0[w], pol);
                    if (x.pos >= 1) ld_words_p<E>(p.row_slots + (base + x.pos - 1) * TR + lane * E, w1[w], pol);
                } else {
                    ld_words_p<E>(p.col_slots + (static_cast<long long>(x.pos) * p.C + x.J) * TC + lane * E, w0[w],
                                  pol);
                    if (x.pos >= 1)
                        ld_words_p<E>(p.col_slots + (static_cast<long long>(x.pos - 1) * p.C + x.J) * TC + lane * E,
                                      w1[w], pol);
                }
            }
            if (ROW && !x.ddone && lane < DW) {
                const int kk = x.dbase + lane;
                if (x.I - kk >= 0 && x.J - kk >= 0)
                    wd[w] = ld_relaxed_p(p.corner_slots + static_cast<long long>(x.I - kk) * p.C + (x.J - kk), pol);
            }
        }
        ++steps;
        SAT_CLK(r0);
#if SAT_STATS
        {   // stats only: wait for the round's loads to measure their latency apart from processing
            uint64_t sink = 0;
#pragma unroll
            for (int w = 0; w < NT; ++w) {
                if (wk[w].active && wk[w].pend) {
#pragma unroll
                    for (int e = 0; e < E; ++e) sink ^= w0[w][e];
                }
                sink ^= wd[w];
            }
            if (sink == 0x123456789abcdefull) wk[0].J = -7;  // never true; forces the loads to land
            SAT_CLK(rl);
            if (lane == 0) WS_ST(ROW ? kWsRowLat : kWsColLat, rl - r0);
        }
#endif
        // ---- ... then consume them
        bool progress = false;
#pragma unroll
        for (int w = 0; w < NT; ++w) {
            Walk& x = wk[w];
            if (!x.active) continue;
            if (fd[w]) {
                if (lane == 0) mbar_arrive(ROW ? &sm.rowwalk[x.s] : &sm.colwalk[x.s]);
                x.active = 0;
                progress = true;
                continue;
            }
            if (x.pend) progress |= lb_consume<V, E>(x.pend, x.pos, x.acc, w0[w], w1[w], x.pos >= 1, epoch);
            if (ROW && !x.ddone) {
                // Step 3.2: GS(I-1,J-1) = GS(I-k,J-k) + sum of GLS of the tiles between
                // window of DW lanes; the grid-edge tile of a diagonal is always inclusive
                const int kk = x.dbase + lane;
                const bool inrange = lane < DW && (x.I - kk >= 0) && (x.J - kk >= 0);
                const bool ready = !inrange || word_ready(wd[w], epoch);
                const unsigned incl = __ballot_sync(kFull, inrange && ready && word_kind(wd[w]) == kIncl);
                const unsigned notready = __ballot_sync(kFull, !ready);
                const int f = incl ? (__ffs(incl) - 1) : DW;
                const unsigned need = (2u << (f < DW ? f : DW - 1)) - 1u;
                if (!(notready & need)) {
                    V val = (inrange && lane <= f) ? from_bits<V>(static_cast<uint32_t>(wd[w])) : V(0);
#pragma unroll
                    for (int d = DW / 2; d >= 1; d >>= 1) val = val + __shfl_xor_sync(kFull, val, d);
                    x.dacc = x.dacc + __shfl_sync(kFull, val, 0);
                    if (f < DW) x.ddone = 1; else x.dbase += DW;
                    progress = true;
                }
            }
            if (x.ddone && __all_sync(kFull, x.pend == 0u)) {
                if (ROW) {
#pragma unroll
                    for (int e = 0; e < E; ++e) sm.rp[x.s][lane * E + e] = x.acc[e];
                    if (lane == 0) sm.corner[x.s] = x.dacc;
                } else {
#pragma unroll
                    for (int e = 0; e < E; ++e) sm.cp[x.s][lane * E + e] = x.acc[e];
                }
                __syncwarp();
                bool handed = true;
                if constexpr (Cfg::WPUB) {
                    // announce this half of the tile's carries to the other walker (for GS), then publish
                    // now if the local aggregates are in, else park the tile and go on walking
                    if (lane == 0) {
                        *reinterpret_cast<volatile int*>(ROW ? &sm.rdone[x.s] : &sm.cdone[x.s]) = x.k + 1;
                        __threadfence_block();
                    }
                    __syncwarp();
                    if (pd.on) {  // rare: two tiles waiting for their local aggregates
                        mbar_wait(&sm.ldone[pd.s], pd.ph);
                        publish(pd.s, pd.k, pd.I, pd.J, pd.acc, pd.dacc);
                        hand_off(pd.s);
                        pd.on = 0;
                    }
                    if (Cfg::WPUB_WAIT) {
                        mbar_wait(&sm.ldone[x.s], x.ph);
                        publish(x.s, x.k, x.I, x.J, x.acc, x.dacc);
                        if (ROW && __shfl_sync(kFull, *reinterpret_cast<volatile int*>(&sm.cdone[x.s]) != x.k + 1, 31)) {
                            // GS needs the column carry too: wait for the column walker, then publish it
                            mbar_wait(&sm.colwalk[x.s], x.ph);
                            publish(x.s, x.k, x.I, x.J, x.acc, x.dacc, true);
                        }
                    } else if (__shfl_sync(kFull, static_cast<int>(mbar_test(&sm.ldone[x.s], x.ph)), 0)) {
                        publish(x.s, x.k, x.I, x.J, x.acc, x.dacc);
                    } else {
                        pd.on = 1;
                        pd.s = x.s;
                        pd.k = x.k;
                        pd.I = x.I;
                        pd.J = x.J;
                        pd.ph = x.ph;
#pragma unroll
                        for (int e = 0; e < E; ++e) pd.acc[e] = x.acc[e];
                        pd.dacc = x.dacc;
                        handed = false;
                    }
                }
                if (lane == 0) {
#if SAT_STATS
                    if (p.trace) p.trace[8LL * sm.info[x.s].t + (ROW ? 3 : 4)] = static_cast<long long>(globaltimer_ns());
#endif
                    WS_ST(ROW ? kWsRowTiles : kWsColTiles, 1);
#if SAT_STATS
                    WS_ST(ROW ? kWsRowResolve : kWsColResolve, clock64() - x.t_acq);
#endif
                }
                if (handed) hand_off(x.s);
                x.active = 0;
                progress = true;
            }
        }
        if constexpr (Cfg::WPUB) {
            if (pd.on && __shfl_sync(kFull, static_cast<int>(mbar_test(&sm.ldone[pd.s], pd.ph)), 0)) {
                publish(pd.s, pd.k, pd.I, pd.J, pd.acc, pd.dacc);
                hand_off(pd.s);
                pd.on = 0;
                progress = true;
            }
        }
        SAT_CLK(r1);
        if (lane == 0) WS_ST(ROW ? kWsRowRoundCyc : kWsColRoundCyc, r1 - r0);
        if (!__any_sync(kFull, progress)) {
            if (lane == 0) WS_ST(ROW ? kWsRowIdle : kWsColIdle, 1);
            __nanosleep(64);
        }
    }
    if (lane == 0) WS_ST(ROW ? kWsRowRounds : kWsColRounds, steps);
}

// Step 1, local SAT, Steps 2.A.1 / 2.B.1 of the tile in stage sl.s into registers `v`.  Returns false
// at the end marker.
template <typename V, typename Cfg, bool TMA>
__device__ __forceinline__ bool ws_local(WsSmem<V, Cfg>& sm, const KParams<V>& p, V (&v)[Cfg::RPW][4],
                                         uint64_t (&fw)[4], const Slot<Cfg::STAGES>& sl, const Slot<Cfg::NQ>& tq,
                                         int& I, int& J, uint32_t epoch, int warp, int lane) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC, NW = Cfg::NW, RPW = Cfg::RPW;
    const int s = sl.s;
    const int row0 = warp * RPW, col0 = lane * 4;
    SAT_CLK(c0);
    mbar_wait(&sm.full[s], sl.ph);
    SAT_CLK(c1);
    if (warp == 0 && lane == 0) { WS_ST(kWsFullWait, c1 - c0); WS_ST(kWsTiles, 1); }
    const TileInfo ti = sm.info[tq.s];
    if (ti.t >= p.ntiles) return false;
#if SAT_STATS
    if (p.trace && warp == 0 && lane == 0) p.trace[8LL * ti.t + 1] = static_cast<long long>(globaltimer_ns());
#endif
    I = ti.I;
    J = ti.J;
    const long long tidx = static_cast<long long>(I) * p.C + J;
    const int par = sl.k & 1;
    const uint64_t pol = policy_evict_last();
    if constexpr (Cfg::FAST) {
        // Fast path of Steps 2.A.2 / 2.B.2 / 3.2: the direct predecessors (I,J-1), (I-1,J), (I-1,J-1)
        // have usually published their inclusive aggregates by now; poll them once, here, so the
        // round trip overlaps the local SAT (consumed in ws_finish; the walkers are the fallback).
        constexpr int ER = Cfg::ER;
        if (warp == 0) {
            if (J > 0) {
#pragma unroll
                for (int e = 0; e < ER; e += 2)
                    ld_relaxed2_p(p.row_slots + (tidx - 1) * TR + lane * ER + e, fw[e], fw[e + 1], pol);
            }
        } else if (warp == NW - 1) {
            if (I > 0) {
                const uint64_t* cs = p.col_slots + (tidx - p.C) * TC + col0;
                ld_relaxed2_p(cs, fw[0], fw[1], pol);
                ld_relaxed2_p(cs + 2, fw[2], fw[3], pol);
            }
        } else if (warp == 1 && lane == 0 && I > 0 && J > 0) {
            fw[0] = ld_relaxed_p(p.corner_slots + tidx - p.C - 1, pol);
        }
    }

    // ---- Step 1 (data in smem, or read from global on the generic path): tile -> registers
    if constexpr (TMA) {
        const V* tile = sm.stage[s];
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const uint4 q = *reinterpret_cast<const uint4*>(&tile[(row0 + r) * TC + col0]);
            v[r][0] = from_bits<V>(q.x); v[r][1] = from_bits<V>(q.y);
            v[r][2] = from_bits<V>(q.z); v[r][3] = from_bits<V>(q.w);
        }
        if (J == p.C - 1) {  // right edge: zero columns >= cols (16-byte TMA granules, reading R2)
#pragma unroll
            for (int c = 0; c < 4; ++c)
                if (static_cast<long long>(J) * TC + col0 + c >= p.cols) {
#pragma unroll
                    for (int r = 0; r < RPW; ++r) v[r][c] = V(0);
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

    if constexpr (Cfg::DIRECT && !Cfg::DEFER && !Cfg::SMEM_SCAN) {
        // the tile now lives in registers: hand the stage back to the loader at once
        __syncwarp();
        if (lane == 0) mbar_arrive(&sm.empty[s]);
    }

    // ---- local SAT: column prefix inside the warp's band, row scans with the warp prefix-sum
    //      algorithm, then the SAT rows of the bands above
#pragma unroll
    for (int r = 1; r < RPW; ++r)
#pragma unroll
        for (int c = 0; c < 4; ++c) v[r][c] = v[r][c] + v[r - 1][c];
    if constexpr (Cfg::SMEM_SCAN) {
        // scratch: this warp's own rows of the stage (already in registers, rewritten only in ws_finish)
        V tot[RPW], ex[RPW];
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            v[r][1] = v[r][1] + v[r][0];
            v[r][2] = v[r][2] + v[r][1];
            v[r][3] = v[r][3] + v[r][2];
            tot[r] = v[r][3];
        }
        warp_rows_exclusive_smem<V, RPW>(tot, ex, sm.stage[s] + row0 * TC, lane);
#pragma unroll
        for (int r = 0; r < RPW; ++r)
#pragma unroll
            for (int c = 0; c < 4; ++c) v[r][c] = v[r][c] + ex[r];
        if constexpr (Cfg::DIRECT && !Cfg::DEFER) {
            __syncwarp();
            if (lane == 0) mbar_arrive(&sm.empty[s]);
        }
    } else {
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
    }
    *reinterpret_cast<uint4*>(&sm.band[par][warp][col0]) =
        make_uint4(to_bits(v[RPW - 1][0]), to_bits(v[RPW - 1][1]), to_bits(v[RPW - 1][2]), to_bits(v[RPW - 1][3]));
    SAT_CLK(cb0);
    named_bar_sync(1, NW * 32);
    SAT_CLK(cb1);
    if (warp == 0 && lane == 0) { WS_ST(kWsBandBar, cb1 - cb0); WS_ST(kWsScan, cb0 - c1); }
    {
        // column-wise exclusive scan of the NW band bottoms, in place, by the first TC compute
        // threads (one column each); then every warp reads its band's offset in one 16-byte load
        const int tid = warp * 32 + lane;
        if (tid < TC) {
            V b[NW];
#pragma unroll
            for (int u = 0; u < NW; ++u) b[u] = sm.band[par][u][tid];
            V run = V(0);
#pragma unroll
            for (int u = 0; u < NW; ++u) {
                sm.band[par][u][tid] = run;
                run = run + b[u];
            }
        }
        named_bar_sync(1, NW * 32);
        const uint4 q = *reinterpret_cast<const uint4*>(&sm.band[par][warp][col0]);
        const V off[4] = {from_bits<V>(q.x), from_bits<V>(q.y), from_bits<V>(q.z), from_bits<V>(q.w)};
#pragma unroll
        for (int r = 0; r < RPW; ++r)
#pragma unroll
            for (int c = 0; c < 4; ++c) v[r][c] = v[r][c] + off[c];
    }

    // ---- Steps 2.A.1 / 2.B.1: local aggregates (prefix form) from the owning lanes: the last column
    //      (lane 31 of every warp) and the bottom row (last warp).  Edge tiles publish inclusive at
    //      once: their carry is zero.
    if (lane == 31) {
        uint64_t* rs = p.row_slots + tidx * TR + row0;
        const uint32_t kind = (J == 0) ? kIncl : kLocal;
#pragma unroll
        for (int r = 0; r < RPW; r += 2)
            st_relaxed2_p(rs + r, pack(epoch, kind, to_bits(v[r][3])), pack(epoch, kind, to_bits(v[r + 1][3])), pol);
    }
    if (warp == NW - 1) {
        uint64_t* cs = p.col_slots + tidx * TC + col0;
        const uint32_t kind = (I == 0) ? kIncl : kLocal;
        st_relaxed2_p(cs, pack(epoch, kind, to_bits(v[RPW - 1][0])), pack(epoch, kind, to_bits(v[RPW - 1][1])), pol);
        st_relaxed2_p(cs + 2, pack(epoch, kind, to_bits(v[RPW - 1][2])), pack(epoch, kind, to_bits(v[RPW - 1][3])),
                      pol);
    }
    if constexpr (Cfg::DEFER) {
        // park the local SAT in the tile's stage; ws_finish reloads it after the next tile's local
        V* tile = sm.stage[s];
#pragma unroll
        for (int r = 0; r < RPW; ++r)
            *reinterpret_cast<uint4*>(&tile[(row0 + r) * TC + col0]) =
                make_uint4(to_bits(v[r][0]), to_bits(v[r][1]), to_bits(v[r][2]), to_bits(v[r][3]));
    }
    SAT_CLK(c2);
    if (warp == 0 && lane == 0) WS_ST(kWsLocal, c2 - c1);
#if SAT_STATS
    if (p.trace && warp == NW - 1 && lane == 0) p.trace[8LL * ti.t + 2] = static_cast<long long>(globaltimer_ns());
#endif
    return true;
}

// Steps 2.A.3 / 2.B.3 / 3.1 / 3.3 and Step 4 for the tile in stage sl.s whose local SAT is in `v`.
template <typename V, typename Cfg, bool TMA, bool CARRY>
__device__ __forceinline__ void ws_finish(WsSmem<V, Cfg>& sm, const KParams<V>& p, V (&v)[Cfg::RPW][4],
                                          const uint64_t (&fw)[4], const Slot<Cfg::STAGES>& sl,
                                          const Slot<Cfg::NQ>& tq, int I, int J, uint32_t epoch, int warp,
                                          int lane) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC, NW = Cfg::NW, RPW = Cfg::RPW;
    const int s = sl.s, q = tq.s;
    const int row0 = warp * RPW, col0 = lane * 4;
    const long long tidx = static_cast<long long>(I) * p.C + J;
    const uint64_t pol = policy_evict_last();
#if SAT_STATS
    const int trace_t = sm.info[q].t;  // the slot may be reacquired once released below
#endif
    SAT_CLK(c0);
    bool fast = false;
    if constexpr (Cfg::FAST) {
        // An inclusive predecessor word IS the carry (prefix-form slots): if all three are inclusive
        // the walks are not needed.  Decided CTA-wide (all or nothing) after one barrier.
        constexpr int ER = Cfg::ER;
        auto incl_ok = [&](uint64_t w) { return word_ready(w, epoch) && word_kind(w) == kIncl; };
        if (warp == 0) {
            bool ok = true;
            V val[ER];
#pragma unroll
            for (int e = 0; e < ER; ++e) {
                val[e] = (J > 0) ? from_bits<V>(static_cast<uint32_t>(fw[e])) : V(0);
                if (J > 0) ok = ok && incl_ok(fw[e]);
            }
            ok = __all_sync(kFull, ok);
            if (ok) {
#pragma unroll
                for (int e = 0; e < ER; ++e) sm.rpf[lane * ER + e] = val[e];
            }
            if (lane == 0) sm.fok[0] = ok;
        } else if (warp == NW - 1) {
            bool ok = true;
            V val[4];
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                val[c] = (I > 0) ? from_bits<V>(static_cast<uint32_t>(fw[c])) : V(0);
                if (I > 0) ok = ok && incl_ok(fw[c]);
            }
            ok = __all_sync(kFull, ok);
            if (ok)
                *reinterpret_cast<uint4*>(&sm.cpf[col0]) =
                    make_uint4(to_bits(val[0]), to_bits(val[1]), to_bits(val[2]), to_bits(val[3]));
            if (lane == 0) sm.fok[1] = ok;
        } else if (warp == 1 && lane == 0) {
            const bool edge = (I == 0 || J == 0);
            const bool ok = edge || incl_ok(fw[0]);
            sm.cornerf = edge ? V(0) : from_bits<V>(static_cast<uint32_t>(fw[0]));
            sm.fok[2] = ok;
        }
        named_bar_sync(2, NW * 32);
        fast = sm.fok[0] && sm.fok[1] && sm.fok[2];
        if (warp == 0 && lane == 0) {
            if (fast) *reinterpret_cast<volatile int*>(&sm.fdone[q]) = 1;
            WS_ST(kWsFastHits, fast ? 1 : 0);
        }
    }
    if (!fast) {
        mbar_wait(&sm.rowwalk[q], tq.ph);
        mbar_wait(&sm.colwalk[q], tq.ph);
    }
    SAT_CLK(c1);
    if (warp == 0 && lane == 0) WS_ST(kWsWalkWait, c1 - c0);
    const V* rps = fast ? sm.rpf : sm.rp[q];
    const V* cps = fast ? sm.cpf : sm.cp[q];
    V rt[RPW];
#pragma unroll
    for (int r = 0; r < RPW; ++r) rt[r] = rps[row0 + r];
    V cpv[4];
    {
        const uint4 c4 = *reinterpret_cast<const uint4*>(&cps[col0]);
        cpv[0] = from_bits<V>(c4.x); cpv[1] = from_bits<V>(c4.y); cpv[2] = from_bits<V>(c4.z);
        cpv[3] = from_bits<V>(c4.w);
    }
    const V corner = fast ? sm.cornerf : sm.corner[q];
    if constexpr (Cfg::DEFER) {
        const V* tile = sm.stage[s];
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const uint4 u = *reinterpret_cast<const uint4*>(&tile[(row0 + r) * TC + col0]);
            v[r][0] = from_bits<V>(u.x); v[r][1] = from_bits<V>(u.y);
            v[r][2] = from_bits<V>(u.z); v[r][3] = from_bits<V>(u.w);
        }
    }
    if constexpr (Cfg::DIRECT) {
        // carries are in registers, and (deferred) so is the local SAT: release the tile slot and stage
        __syncwarp();
        if (lane == 0) {
            mbar_arrive(&sm.tfree[q]);
            if constexpr (Cfg::DEFER) mbar_arrive(&sm.empty[s]);
        }
    }
    // inclusive aggregates (Steps 2.A.3, 2.B.3, 3.1, 3.3), from the lanes that hold the local ones, at
    // once (successors are waiting for them; publishing after the stage hand-off measured no faster)
    V rinc[RPW], cinc[4];
#pragma unroll
    for (int r = 0; r < RPW; ++r) rinc[r] = v[r][3] + rt[r];
#pragma unroll
    for (int c = 0; c < 4; ++c) cinc[c] = v[RPW - 1][c] + cpv[c];
    const V gs = corner + (v[RPW - 1][3] + rt[RPW - 1] + cpv[3]);  // GS = GS(I-1,J-1) + GLS
    auto publish_incl = [&]() {
        if (lane == 31 && J > 0) {
            uint64_t* rs = p.row_slots + tidx * TR + row0;
#pragma unroll
            for (int r = 0; r < RPW; r += 2)
                st_relaxed2_p(rs + r, pack(epoch, kIncl, to_bits(rinc[r])), pack(epoch, kIncl, to_bits(rinc[r + 1])),
                              pol);
        }
        if (warp == NW - 1) {
            if (I > 0) {
                uint64_t* cs = p.col_slots + tidx * TC + col0;
                st_relaxed2_p(cs, pack(epoch, kIncl, to_bits(cinc[0])), pack(epoch, kIncl, to_bits(cinc[1])), pol);
                st_relaxed2_p(cs + 2, pack(epoch, kIncl, to_bits(cinc[2])), pack(epoch, kIncl, to_bits(cinc[3])), pol);
            }
            if (lane == 31) st_relaxed_p(p.corner_slots + tidx, pack(epoch, kIncl, to_bits(gs)), pol);
        }
    };
    publish_incl();
    // GSAT(I,J) = localSAT + rp[i] + cp[j] + corner (+ carry[j])
    V colterm[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) colterm[c] = cpv[c] + corner;
    if constexpr (CARRY) {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
            const long long gj = static_cast<long long>(J) * TC + col0 + c;
            colterm[c] = colterm[c] + (gj < p.cols ? p.carry[gj] : V(0));
        }
    }
#pragma unroll
    for (int r = 0; r < RPW; ++r)
#pragma unroll
        for (int c = 0; c < 4; ++c) v[r][c] = v[r][c] + (rt[r] + colterm[c]);
    const bool ragged = !TMA || ((J == p.C - 1) && (p.cols & 3) != 0);
    if constexpr (Cfg::DIRECT && TMA) {
        // 16-byte aligned rows (TMA path preconditions): one vector store per row chunk
        const uint64_t spol = policy_evict_first();
        const long long gj0 = static_cast<long long>(J) * TC + col0;
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const long long gi = static_cast<long long>(I) * TR + row0 + r;
            if (gi >= p.rows) continue;
            V* dst = p.dst + gi * p.pitch + gj0;
            if (gj0 + 3 < p.cols) {
                st_global_v4_hint(dst, to_bits(v[r][0]), to_bits(v[r][1]), to_bits(v[r][2]), to_bits(v[r][3]), spol);
            } else {
#pragma unroll
                for (int c = 0; c < 4; ++c)
                    if (gj0 + c < p.cols) dst[c] = v[r][c];
            }
        }
    } else if (!ragged) {
        V* tile = sm.stage[s];
#pragma unroll
        for (int r = 0; r < RPW; ++r)
            *reinterpret_cast<uint4*>(&tile[(row0 + r) * TC + col0]) =
                make_uint4(to_bits(v[r][0]), to_bits(v[r][1]), to_bits(v[r][2]), to_bits(v[r][3]));
        fence_proxy_async_smem();
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
    }
#if SAT_STATS
    if (p.trace && warp == 0 && lane == 0) p.trace[8LL * trace_t + 5] = static_cast<long long>(globaltimer_ns());
#endif
    if constexpr (!Cfg::DIRECT) {
        __syncwarp();
        if (lane == 0) mbar_arrive(&sm.result[s]);
    }
    SAT_CLK(c2);
    if (warp == 0 && lane == 0) WS_ST(kWsFinish, c2 - c1);
}

template <typename V, typename Cfg, bool TMA, bool CARRY>
__global__ void __launch_bounds__(Cfg::THREADS, Cfg::MINB)
sat_ws_kernel(const __grid_constant__ CUtensorMap map_in, const __grid_constant__ CUtensorMap map_out,
              const KParams<V> p) {
    constexpr int TR = Cfg::TR, TC = Cfg::TC, NW = Cfg::NW, STAGES = Cfg::STAGES, RPW = Cfg::RPW;
    constexpr uint32_t kTileBytes = TR * TC * sizeof(V);
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    WsSmem<V, Cfg>& sm = *reinterpret_cast<WsSmem<V, Cfg>*>(smem_raw);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

#if SAT_STATS
    if (threadIdx.x < kNumStats) ws_stats[threadIdx.x] = 0ull;
#endif
    if (threadIdx.x == 0) {
        sm.epoch = *reinterpret_cast<volatile unsigned int*>(&p.ctrl->epoch);
        sm.end_n = 0x7fffffff;
#pragma unroll
        for (int q = 0; q < Cfg::NQ; ++q) {
            mbar_init(&sm.acq[q], 1);
            mbar_init(&sm.rowwalk[q], 1);
            mbar_init(&sm.colwalk[q], 1);
            mbar_init(&sm.tfree[q], Cfg::DIRECT ? NW : 1);
        }
#pragma unroll
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&sm.full[s], 1);
            mbar_init(&sm.result[s], NW);
            mbar_init(&sm.empty[s], Cfg::DIRECT ? NW : 1);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const uint32_t epoch = sm.epoch;

    if (warp < NW) {
        // ================================================================ compute warps
        V v[RPW][4];
        uint64_t fw[4] = {0ull, 0ull, 0ull, 0ull};
        Slot<STAGES> sl;
        Slot<Cfg::NQ> tq;
        if constexpr (Cfg::DEFER) {
            // local(k+1) runs while the walks of tile k finish: local(0), {local(k+1), finish(k)}...
            int I, J;
            bool have = ws_local<V, Cfg, TMA>(sm, p, v, fw, sl, tq, I, J, epoch, warp, lane);
            while (have) {
                Slot<STAGES> sl2 = sl;
                Slot<Cfg::NQ> tq2 = tq;
                sl2.next();
                tq2.next();
                int I2, J2;
                const bool have2 = ws_local<V, Cfg, TMA>(sm, p, v, fw, sl2, tq2, I2, J2, epoch, warp, lane);
                ws_finish<V, Cfg, TMA, CARRY>(sm, p, v, fw, sl, tq, I, J, epoch, warp, lane);
                sl = sl2;
                tq = tq2;
                I = I2;
                J = J2;
                have = have2;
            }
        } else {
            for (;; tq.next(), sl.next()) {
                int I, J;
                if (!ws_local<V, Cfg, TMA>(sm, p, v, fw, sl, tq, I, J, epoch, warp, lane)) break;
                ws_finish<V, Cfg, TMA, CARRY>(sm, p, v, fw, sl, tq, I, J, epoch, warp, lane);
            }
        }
        if constexpr (Cfg::DIRECT) {
            __threadfence();
            named_bar_sync(3, (NW + 1) * 32);
        }
    } else if (warp == Cfg::ROW_WARP) {
        ws_walker<V, Cfg, true>(sm, p, epoch, lane);
    } else if (warp == Cfg::COL_WARP) {
        ws_walker<V, Cfg, false>(sm, p, epoch, lane);
    } else if (warp == Cfg::STORE_WARP && Cfg::DIRECT) {
        // compute warps store from registers: this warp only runs the exit protocol once they are done
        named_bar_sync(3, (NW + 1) * 32);
        if (lane == 0) ws_exit(p, epoch);
    } else if (warp == Cfg::STORE_WARP) {
        // ================================================================ storer (one lane)
        if (lane == 0) {
            if constexpr (TMA) prefetch_tensormap(&map_out);
            const uint64_t spol = policy_evict_first();
            Slot<STAGES> sl;
            for (Slot<Cfg::NQ> tq;; tq.next(), sl.next()) {
                const int s = sl.s;
                mbar_wait(&sm.acq[tq.s], tq.ph);
                const TileInfo ti = sm.info[tq.s];  // stays valid until this lane releases the slot
                if (ti.t >= p.ntiles) break;
                SAT_CLK(u0);
                mbar_wait(&sm.result[s], sl.ph);
                SAT_CLK(u1);
                WS_ST(kWsStResultWait, u1 - u0);
                bool stored = false;
                if constexpr (TMA) {
                    const bool ragged = (ti.J == p.C - 1) && (p.cols & 3) != 0;
                    if (!ragged) {
                        tma_store_2d_hint(&map_out, sm.stage[s], ti.J * TC, ti.I * TR, spol);
                        bulk_commit();
                        stored = true;
                    }
                }
                // the walkers may still be winding down a tile the fast path resolved
                mbar_wait(&sm.rowwalk[tq.s], tq.ph);
                mbar_wait(&sm.colwalk[tq.s], tq.ph);
                mbar_arrive(&sm.tfree[tq.s]);  // the tile slot (id, carries) is no longer needed
#if SAT_STATS
                if (p.trace) p.trace[8LL * ti.t + 6] = static_cast<long long>(globaltimer_ns());
#endif
                // release the stage as soon as its store has read the shared memory
                if (stored) bulk_wait_read<0>();
                mbar_arrive(&sm.empty[s]);
                SAT_CLK(u2);
                WS_ST(kWsStStore, u2 - u1);
            }
            if constexpr (TMA) bulk_wait_all();
            ws_exit(p, epoch);
        }
    } else if (lane == 0) {
        // ================================================================ loader (one lane)
        // Two independent cursors: tickets are drawn into the tile ring as soon as a tile slot is free
        // (so the walkers start early); TMA loads follow into the data ring as stages free up.
        const uint64_t policy = TMA ? policy_evict_first() : 0ull;
        if constexpr (TMA) prefetch_tensormap(&map_in);
        Slot<Cfg::NQ> ta, tl;  // acquisition cursor; load cursor (tile ring)
        Slot<STAGES> sl;       // load cursor (data ring)
        bool acq_done = false;
        while (true) {
            bool progress = false;
            if (!acq_done && (ta.k < Cfg::NQ || mbar_test(&sm.tfree[ta.s], ta.ph ^ 1u))) {
                SAT_CLK(t0);
                const int t = static_cast<int>(atomicAdd(&p.ctrl->counter, 1u));
                const bool valid = t < p.ntiles;
                TileInfo ti{t, 0, 0, 0};
                if (valid) tile_of_serial(t, p.R, p.C, p.order, ti.I, ti.J);
                sm.info[ta.s] = ti;
                sm.fdone[ta.s] = 0;
                if (!valid) {
                    *reinterpret_cast<volatile int*>(&sm.end_n) = ta.k;
                    acq_done = true;
                }
                mbar_arrive(&sm.acq[ta.s]);
                if constexpr (TMA && Cfg::PREFETCH) {
                    if (valid) tma_prefetch_2d(&map_in, ti.J * TC, ti.I * TR);
                }
#if SAT_STATS
                if (p.trace && valid) p.trace[8LL * t] = static_cast<long long>(globaltimer_ns());
#endif
                ta.next();
                progress = true;
                SAT_CLK(t1);
                WS_ST(kWsLdIssue, t1 - t0);
            }
            if (tl.k < ta.k && (sl.k < STAGES || mbar_test(&sm.empty[sl.s], sl.ph ^ 1u))) {
                const TileInfo ti = sm.info[tl.s];
                const bool valid = ti.t < p.ntiles;
                if (TMA && valid) {
                    mbar_arrive_expect_tx(&sm.full[sl.s], kTileBytes);
                    tma_load_2d(sm.stage[sl.s], &map_in, &sm.full[sl.s], ti.J * TC, ti.I * TR, policy);
#if SAT_STATS
                    if (p.trace) p.trace[8LL * ti.t + 7] = static_cast<long long>(globaltimer_ns());
#endif
                } else {
                    mbar_arrive(&sm.full[sl.s]);  // generic path (data read from global) or end marker
                }
                tl.next();
                sl.next();
                progress = true;
                if (!valid) break;
            }
            if (!progress) __nanosleep(32);
        }
    }
}

}  // namespace sat
