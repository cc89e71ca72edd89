// sat_wide_kernel.cuh -- single-pass SATs with 64-bit output elements:
//
//   * fp32 input, fp64 SAT (sat_compute_f32_f64): the accumulation the 4-byte float of P:253 cannot hold
//     exactly at large n; 4 B read + 8 B written per element;
//   * summed-area variance shadow map moments (sat_compute_moments_f32; P:50 and ref. [8] at P:311): the
//     SAT of a and the SAT of a*a in fp32, stored as interleaved float pairs; 4 B read + 8 B written.
//
// The method is the one of sat_kernel.cuh (1R1W-SKSS-LB, Sec. IV): a CTA takes a
// ticket from the SKSS counter, maps it to a tile in Fig. 9's anti-diagonal order,
// computes the tile's local SAT, publishes its local row / column aggregates in prefix form
// (Steps 2.A.1 / 2.B.1, reading R5'), looks back along its tile row, tile column and diagonal (Steps
// 2.A.2, 2.B.2, 3.2), publishes the inclusive aggregates (2.A.3, 2.B.3, 3.1, 3.3) and writes
// GSAT (Step 4, rule P:150).  One CTA per tile, as in the paper: CTAs that are not yet
// resident take their tickets when they start, so any grid size is deadlock-free.
//
// What changes with 64-bit elements is the status word: a value no longer fits next to its epoch / kind
// tag in one single-copy-atomic 64-bit word (reading R11).  Each value is published as TWO tagged words,
// (epoch, kind, low 32 bits) and (epoch, kind, high 32 bits).  A slot goes "empty -> local -> inclusive"
// within a launch, each state written once by the same thread, so a reader that sees both halves with the
// current epoch and the SAME kind holds a consistent value; halves of different kinds are re-polled.
#pragma once

#include "sat_kernel.cuh"

namespace sat {

// ------------------------------------------------------------------ element types
__device__ __forceinline__ double wide_from_in(float x, double*) { return static_cast<double>(x); }
__device__ __forceinline__ float2 wide_from_in(float x, float2*) { return make_float2(x, __fmul_rn(x, x)); }
__device__ __forceinline__ double wadd(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ float2 wadd(float2 a, float2 b) { return make_float2(__fadd_rn(a.x, b.x), __fadd_rn(a.y, b.y)); }
template <typename W> __device__ __forceinline__ W wzero();
template <> __device__ __forceinline__ double wzero<double>() { return 0.0; }
template <> __device__ __forceinline__ float2 wzero<float2>() { return make_float2(0.f, 0.f); }
__device__ __forceinline__ uint64_t wbits(double a) { return static_cast<uint64_t>(__double_as_longlong(a)); }
__device__ __forceinline__ uint64_t wbits(float2 a) {
    return static_cast<uint64_t>(__float_as_uint(a.x)) | (static_cast<uint64_t>(__float_as_uint(a.y)) << 32);
}
template <typename W> __device__ __forceinline__ W wof(uint64_t b);
template <> __device__ __forceinline__ double wof<double>(uint64_t b) { return __longlong_as_double(static_cast<long long>(b)); }
template <> __device__ __forceinline__ float2 wof<float2>(uint64_t b) {
    return make_float2(__uint_as_float(static_cast<uint32_t>(b)), __uint_as_float(static_cast<uint32_t>(b >> 32)));
}
template <typename W>
__device__ __forceinline__ W wshfl_up(W v, int d) {
    return wof<W>(__shfl_up_sync(kFull, static_cast<unsigned long long>(wbits(v)), d));
}
template <typename W>
__device__ __forceinline__ W wshfl(W v, int src) {
    return wof<W>(__shfl_sync(kFull, static_cast<unsigned long long>(wbits(v)), src));
}

// two tagged words per value
__device__ __forceinline__ void wpack(uint32_t epoch, uint32_t kind, uint64_t b, uint64_t& w0, uint64_t& w1) {
    w0 = pack(epoch, kind, static_cast<uint32_t>(b));
    w1 = pack(epoch, kind, static_cast<uint32_t>(b >> 32));
}
// both halves published in this epoch with the same kind
__device__ __forceinline__ bool wready(uint64_t w0, uint64_t w1, uint32_t epoch) {
    return word_ready(w0, epoch) && word_ready(w1, epoch) && word_kind(w0) == word_kind(w1);
}
__device__ __forceinline__ uint64_t wjoin(uint64_t w0, uint64_t w1) {
    return static_cast<uint64_t>(static_cast<uint32_t>(w0)) | (static_cast<uint64_t>(static_cast<uint32_t>(w1)) << 32);
}

struct WideParams {
    const float* src;
    void* dst;                 // W elements
    int64_t rows, cols, src_pitch, dst_pitch;  // pitches in elements of the respective type
    int R, C, ntiles;
    uint64_t* row_slots;       // [R*C][TR][2]
    uint64_t* col_slots;       // [R*C][TC][2]
    uint64_t* corner_slots;    // [R*C][2]
    Ctrl* ctrl;
    int vec;                   // 16-byte aligned src / dst rows: vector loads and stores
};

constexpr int kWideTR = 64, kWideTC = 128, kWideNW = 8, kWideRPW = kWideTR / kWideNW;

template <typename W>
struct WideSmem {
    alignas(16) W band[kWideNW][kWideTC];
    alignas(16) W rp[kWideTR];
    alignas(16) W cp[kWideTC];
    W corner, total;
    int t, I, J, corner_ok;
    uint32_t epoch;
};

// Row / column look-back over E values per lane (2E words): predecessors p, p + step, ... (step in words)
template <typename W, int E>
__device__ __forceinline__ void wide_lookback(const uint64_t* p, long long step, uint32_t epoch, W (&acc)[E]) {
    uint32_t pending = (1u << E) - 1u;
#pragma unroll
    for (int e = 0; e < E; ++e) acc[e] = wzero<W>();
    SAT_SPIN_DECL;
    while (true) {
        uint64_t w[2 * E];
        ld_words<2 * E>(p, w);
        bool ok = true;
#pragma unroll
        for (int e = 0; e < E; ++e)
            if (((pending >> e) & 1u) && !wready(w[2 * e], w[2 * e + 1], epoch)) ok = false;
        if (!ok) {
            SAT_SPIN_CHECK("a wide row / column look-back word");
            __nanosleep(20);
            continue;
        }
#pragma unroll
        for (int e = 0; e < E; ++e) {
            if ((pending >> e) & 1u) {
                acc[e] = wadd(acc[e], wof<W>(wjoin(w[2 * e], w[2 * e + 1])));
                if (word_kind(w[2 * e]) == kIncl) pending &= ~(1u << e);
            }
        }
        if (__all_sync(kFull, pending == 0u)) break;
        p += step;
    }
}

// Diagonal look-back (Step 3.2, reading R8): GS(I-1,J-1) = sum of the corner words of (I-k, J-k),
// k = 1, 2, ... up to and including the first inclusive one (GLS words are "local").  32 predecessors per
// round, lane k-1 <-> tile (I-k, J-k).  Non-blocking mode returns false at the first unpublished word.
template <typename W>
__device__ __forceinline__ bool wide_diag(const uint64_t* corner, int I, int J, int C, uint32_t epoch, bool blocking,
                                          int lane, W& out) {
    if (I == 0 || J == 0) {
        out = wzero<W>();
        return true;
    }
    W acc = wzero<W>();
    int base = 1;
    SAT_SPIN_DECL;
    while (true) {
        const int k = base + lane;
        const bool inr = (I - k >= 0) && (J - k >= 0);
        uint64_t w0 = 0, w1 = 0;
        if (inr) {
            const uint64_t* q = corner + 2 * (static_cast<long long>(I - k) * C + (J - k));
            ld_relaxed2(q, w0, w1);
        }
        const bool ready = !inr || wready(w0, w1, epoch);
        const unsigned incl = __ballot_sync(kFull, inr && ready && word_kind(w0) == kIncl);
        const unsigned notready = __ballot_sync(kFull, !ready);
        const int f = incl ? (__ffs(incl) - 1) : 32;
        const unsigned need = (f >= 31) ? kFull : ((2u << f) - 1u);
        if (notready & need) {
            if (!blocking) return false;
            SAT_SPIN_CHECK("a wide diagonal look-back word");
            __nanosleep(20);
            continue;
        }
        W val = (inr && lane <= f) ? wof<W>(wjoin(w0, w1)) : wzero<W>();
#pragma unroll
        for (int d = 16; d >= 1; d >>= 1) val = wadd(val, wof<W>(__shfl_xor_sync(kFull, static_cast<unsigned long long>(wbits(val)), d)));
        acc = wadd(acc, val);
        if (f < 32) {
            out = acc;
            return true;
        }
        base += 32;
    }
}

template <typename W>
__global__ void __launch_bounds__(kWideNW * 32) sat_wide_kernel(const WideParams p) {
    constexpr int TR = kWideTR, TC = kWideTC, NW = kWideNW, RPW = kWideRPW, ER = TR / 32, EC = TC / 32;
    __shared__ WideSmem<W> sm;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        sm.epoch = *reinterpret_cast<volatile unsigned int*>(&p.ctrl->epoch);
        const int t = static_cast<int>(atomicAdd(&p.ctrl->counter, 1u));  // SKSS ticket
        int I = 0, J = 0;
        if (t < p.ntiles) tile_of_serial(t, p.R, p.C, 0, I, J);
        sm.t = t;
        sm.I = I;
        sm.J = J;
    }
    __syncthreads();
    const uint32_t epoch = sm.epoch;
    const int I = sm.I, J = sm.J;
    if (sm.t < p.ntiles) {
        const long long tidx = static_cast<long long>(I) * p.C + J;
        const int row0 = warp * RPW, col0 = lane * 4;
        const long long gj0 = static_cast<long long>(J) * TC + col0;
        // ---- Step 1: the lane's 4 columns of the warp's RPW rows
        W v[RPW][4];
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const long long gi = static_cast<long long>(I) * TR + row0 + r;
            float x[4] = {0.f, 0.f, 0.f, 0.f};
            if (gi < p.rows) {
                const float* s = p.src + gi * p.src_pitch + gj0;
                if (p.vec && gj0 + 3 < p.cols) {
                    const float4 q = __ldcs(reinterpret_cast<const float4*>(s));
                    x[0] = q.x; x[1] = q.y; x[2] = q.z; x[3] = q.w;
                } else {
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        if (gj0 + c < p.cols) x[c] = __ldcs(s + c);
                }
            }
#pragma unroll
            for (int c = 0; c < 4; ++c) v[r][c] = wide_from_in(x[c], static_cast<W*>(nullptr));
        }
        // ---- local SAT: column prefix in the band, in-lane row prefix, warp scan, bands above
#pragma unroll
        for (int r = 1; r < RPW; ++r)
#pragma unroll
            for (int c = 0; c < 4; ++c) v[r][c] = wadd(v[r][c], v[r - 1][c]);
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            v[r][1] = wadd(v[r][1], v[r][0]);
            v[r][2] = wadd(v[r][2], v[r][1]);
            v[r][3] = wadd(v[r][3], v[r][2]);
            W incl = v[r][3];
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const W y = wshfl_up(incl, d);
                if (lane >= d) incl = wadd(incl, y);
            }
            W excl = wshfl_up(incl, 1);
            if (lane == 0) excl = wzero<W>();
#pragma unroll
            for (int c = 0; c < 4; ++c) v[r][c] = wadd(v[r][c], excl);
        }
#pragma unroll
        for (int c = 0; c < 4; ++c) sm.band[warp][col0 + c] = v[RPW - 1][c];
        __syncthreads();
        {
            W off[4] = {wzero<W>(), wzero<W>(), wzero<W>(), wzero<W>()};
            for (int w2 = 0; w2 < warp; ++w2)
#pragma unroll
                for (int c = 0; c < 4; ++c) off[c] = wadd(off[c], sm.band[w2][col0 + c]);
#pragma unroll
            for (int r = 0; r < RPW; ++r)
#pragma unroll
                for (int c = 0; c < 4; ++c) v[r][c] = wadd(v[r][c], off[c]);
        }
        SAT_JITTER_WARP();
        // ---- Steps 2.A.1 / 2.B.1: local aggregates (edge tiles publish inclusive at once: no carry)
        if (lane == 31) {
            uint64_t* rs = p.row_slots + 2 * (tidx * TR + row0);
            const uint32_t kind = (J == 0) ? kIncl : kLocal;
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                uint64_t w0, w1;
                wpack(epoch, kind, wbits(v[r][3]), w0, w1);
                st_relaxed2(rs + 2 * r, w0, w1);
            }
        }
        if (warp == NW - 1) {
            uint64_t* cs = p.col_slots + 2 * (tidx * TC + col0);
            const uint32_t kind = (I == 0) ? kIncl : kLocal;
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                uint64_t w0, w1;
                wpack(epoch, kind, wbits(v[RPW - 1][c]), w0, w1);
                st_relaxed2(cs + 2 * c, w0, w1);
            }
            if (lane == 31) sm.total = v[RPW - 1][3];
        }
        // ---- Steps 2.A.2 / 2.B.2 / 3.2 (three warps at once)
        if (warp == 0) {
            W acc[ER];
            if (J == 0) {
#pragma unroll
                for (int e = 0; e < ER; ++e) acc[e] = wzero<W>();
            } else {
                wide_lookback<W, ER>(p.row_slots + 2 * ((tidx - 1) * TR + lane * ER), -2LL * TR, epoch, acc);
            }
#pragma unroll
            for (int e = 0; e < ER; ++e) sm.rp[lane * ER + e] = acc[e];
        } else if (warp == 1) {
            W acc[EC];
            if (I == 0) {
#pragma unroll
                for (int e = 0; e < EC; ++e) acc[e] = wzero<W>();
            } else {
                wide_lookback<W, EC>(p.col_slots + 2 * ((tidx - p.C) * TC + lane * EC), -2LL * p.C * TC, epoch, acc);
            }
#pragma unroll
            for (int e = 0; e < EC; ++e) sm.cp[lane * EC + e] = acc[e];
        } else if (warp == 2) {
            W corner;
            const bool ok = wide_diag<W>(p.corner_slots, I, J, p.C, epoch, false, lane, corner);
            if (lane == 0) {
                sm.corner = ok ? corner : wzero<W>();
                sm.corner_ok = ok ? 1 : 0;
            }
        }
        __syncthreads();
        SAT_JITTER_WARP();
        // ---- Steps 2.A.3 / 2.B.3: inclusive aggregates, by the owners of the local values
        if (lane == 31 && J > 0) {
            uint64_t* rs = p.row_slots + 2 * (tidx * TR + row0);
#pragma unroll
            for (int r = 0; r < RPW; ++r) {
                uint64_t w0, w1;
                wpack(epoch, kIncl, wbits(wadd(v[r][3], sm.rp[row0 + r])), w0, w1);
                st_relaxed2(rs + 2 * r, w0, w1);
            }
        }
        if (warp == NW - 1 && I > 0) {
            uint64_t* cs = p.col_slots + 2 * (tidx * TC + col0);
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                uint64_t w0, w1;
                wpack(epoch, kIncl, wbits(wadd(v[RPW - 1][c], sm.cp[col0 + c])), w0, w1);
                st_relaxed2(cs + 2 * c, w0, w1);
            }
        }
        // ---- Steps 3.1 / 3.3: GLS = total + rp[TR-1] + cp[TC-1]; GS = GS(I-1,J-1) + GLS
        const W gls = wadd(wadd(sm.total, sm.rp[TR - 1]), sm.cp[TC - 1]);
        uint64_t* cslot = p.corner_slots + 2 * tidx;
        if (!sm.corner_ok) {  // uniform (read after the barrier)
            if (warp == 2) {
                if (lane == 0) {
                    uint64_t w0, w1;
                    wpack(epoch, kLocal, wbits(gls), w0, w1);
                    st_relaxed2(cslot, w0, w1);
                }
                W corner;
                wide_diag<W>(p.corner_slots, I, J, p.C, epoch, true, lane, corner);
                if (lane == 0) sm.corner = corner;
            }
            __syncthreads();
        }
        const W corner = sm.corner;
        if (warp == 2 && lane == 0) {
            uint64_t w0, w1;
            wpack(epoch, kIncl, wbits(wadd(corner, gls)), w0, w1);
            st_relaxed2(cslot, w0, w1);
        }
        // ---- Step 4: GSAT = local SAT + rp[i] + (cp[j] + corner), streamed out
        W colterm[4];
#pragma unroll
        for (int c = 0; c < 4; ++c) colterm[c] = wadd(sm.cp[col0 + c], corner);
        W* dst = static_cast<W*>(p.dst);
#pragma unroll
        for (int r = 0; r < RPW; ++r) {
            const long long gi = static_cast<long long>(I) * TR + row0 + r;
            if (gi >= p.rows) continue;
            const W rt = sm.rp[row0 + r];
            W o[4];
#pragma unroll
            for (int c = 0; c < 4; ++c) o[c] = wadd(v[r][c], wadd(rt, colterm[c]));
            W* d = dst + gi * p.dst_pitch + gj0;
            if (p.vec && gj0 + 3 < p.cols) {
                const uint64_t b0 = wbits(o[0]), b1 = wbits(o[1]), b2 = wbits(o[2]), b3 = wbits(o[3]);
                __stcs(reinterpret_cast<ulonglong2*>(d), make_ulonglong2(b0, b1));
                __stcs(reinterpret_cast<ulonglong2*>(d) + 1, make_ulonglong2(b2, b3));
            } else {
#pragma unroll
                for (int c = 0; c < 4; ++c)
                    if (gj0 + c < p.cols) d[c] = o[c];
            }
        }
    }
    // ---- exit: the last CTA out resets the counter and advances the epoch (a0, no memset per call)
    __syncthreads();
    if (threadIdx.x == 0) {
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

}  // namespace sat
