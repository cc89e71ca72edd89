// sat_query_kernels.cuh -- O(1) rectangle queries on a summed area table.
//
// sum_{u < i <= d, l < j <= r} a[i][j] = b[d][r] - b[u][r] - b[d][l] + b[u][l], where b is the SAT
// of a.  Entries with a row or column index of -1 are zero (the empty prefix).  Evaluated in the
// SAT's own arithmetic (uint32 wraparound for int32, fp32 for float) left to right:
// ((b[d][r] - b[u][r]) - b[d][l]) + b[u][l]  (reading R17).
//
// box_sum_kernel: the box filter that motivates SATs: out[i][j] = sum of a over the window
// rows [i-rh, i+rh] x columns [j-rw, j+rw] clipped to the matrix, i.e. P:48 with
// u = i-rh-1, d = min(i+rh, rows-1), l = j-rw-1, r = min(j+rw, cols-1).  HBM-bound stencil: each SAT
// row is read by the two output rows that use it (the reuse distance is 2*rh+1 rows, so the second
// read is an L2 hit for any practical radius); algorithmic bytes 4 read + 4 written per element.
#pragma once

#include <cstdint>

#include "sat_device.cuh"

namespace sat {

template <typename V>
__device__ __forceinline__ V sat_at(const V* b, int64_t pitch, int64_t i, int64_t j) {
    return (i < 0 || j < 0) ? V(0) : __ldg(b + i * pitch + j);
}

template <typename V>
__device__ __forceinline__ V rect_from_sat(const V* b, int64_t pitch, int64_t u, int64_t d, int64_t l, int64_t r) {
    const V drr = sat_at(b, pitch, d, r), urr = sat_at(b, pitch, u, r);
    const V dll = sat_at(b, pitch, d, l), ull = sat_at(b, pitch, u, l);
    return ((drr - urr) - dll) + ull;
}

// One thread: 4 consecutive output columns of one row.  Grid: x over column groups of 4 * blockDim.x,
// y strides over rows.
template <typename V, bool VEC>
__global__ void __launch_bounds__(256) box_sum_kernel(const V* __restrict__ b, V* __restrict__ out, int64_t rows,
                                                      int64_t cols, int64_t pitch, int64_t rh, int64_t rw) {
    const int64_t j0 = (static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x) * 4;
    if (j0 >= cols) return;
    for (int64_t i = blockIdx.y; i < rows; i += gridDim.y) {
        const int64_t u = i - rh - 1;
        const int64_t d = i + rh < rows - 1 ? i + rh : rows - 1;
        V o[4];
#pragma unroll
        for (int c = 0; c < 4; ++c) {
            const int64_t j = j0 + c;
            const int64_t l = j - rw - 1;
            const int64_t r = j + rw < cols - 1 ? j + rw : cols - 1;
            o[c] = (j < cols) ? rect_from_sat(b, pitch, u, d, l, r) : V(0);
        }
        V* dst = out + i * pitch + j0;
        if (VEC && j0 + 3 < cols) {
            __stcs(reinterpret_cast<uint4*>(dst), make_uint4(to_bits(o[0]), to_bits(o[1]), to_bits(o[2]), to_bits(o[3])));
        } else {
#pragma unroll
            for (int c = 0; c < 4; ++c)
                if (j0 + c < cols) dst[c] = o[c];
        }
    }
}

// Staged box filter (the production path when the two row segments fit in shared memory).  A block
// owns a panel of kBoxPanel output columns and walks output rows i = blockIdx.y, +gridDim.y, ...  Per
// row it copies the two SAT row segments the panel needs, rows d and u over columns
// [panel - rw - 1, panel + kBoxPanel - 1 + rw] (clipped to the matrix; index -1 and the rows above
// row 0 read as zero), into shared memory with 16-byte coalesced loads, then evaluates P:48 for
// its 4 columns (256 apart, so a warp reads consecutive shared-memory words) from shared memory in
// the same left-to-right order as box_sum_kernel.  Global traffic per
// output row: one read of each SAT row segment (row u is row d of the output row 2*rh+1 above, an L2
// hit) and coalesced streaming stores, instead of 16 scalar L2 loads per 4 outputs.
// Requires pitch * 4 and both pointers 16-byte aligned (VEC).  The segments of the next kBoxBufs - 1
// rows are in flight (cp.async) while the current row is evaluated.
constexpr int kBoxThreads = 256;
constexpr int kBoxPanel = 4 * kBoxThreads;

constexpr int kBoxBufs = 3;  // row-segment pairs in flight per block (cp.async groups)

template <typename V>
__device__ __forceinline__ void box_load_seg(const V* __restrict__ b, int64_t pitch, int64_t row, int64_t a0,
                                             int64_t hi, int nv, V* seg) {
    // seg[k] = b[row][a0 + k] for a0 + k in [0, hi], else 0 (a0 is a multiple of 4; hi = last column);
    // 16-byte cp.async with a source size of 0..16 bytes (the rest of the 16 bytes is zero-filled)
    for (int q = threadIdx.x; q < nv; q += blockDim.x) {
        const int64_t j = a0 + 4 * static_cast<int64_t>(q);
        int bytes = 0;
        const V* src = b;
        if (row >= 0 && j >= 0 && j <= hi) {
            bytes = (hi - j + 1 >= 4) ? 16 : static_cast<int>(hi - j + 1) * 4;
            src = b + row * pitch + j;
        }
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_addr(seg + 4 * q)), "l"(src),
                     "r"(bytes)
                     : "memory");
    }
}

template <typename V>
__global__ void __launch_bounds__(kBoxThreads) box_sum_smem_kernel(const V* __restrict__ b, V* __restrict__ out,
                                                                   int64_t rows, int64_t cols, int64_t pitch,
                                                                   int64_t rh, int64_t rw, int nv) {
    extern __shared__ __align__(16) unsigned char box_smem[];
    V* buf = reinterpret_cast<V*>(box_smem);  // [kBoxBufs][2 rows (d, u)][4 * nv]
    const int64_t p0 = static_cast<int64_t>(blockIdx.x) * kBoxPanel;
    const int64_t a0 = ((p0 - rw - 1) >= 0) ? ((p0 - rw - 1) & ~int64_t(3)) : -((-(p0 - rw - 1) + 3) & ~int64_t(3));
    const int64_t hi = cols - 1;
    const int seglen = 4 * nv;
    auto load_row = [&](int64_t i, int sb) {  // always commits one group (empty past the last row)
        if (i < rows) {
            const int64_t u = i - rh - 1;
            const int64_t d = i + rh < rows - 1 ? i + rh : rows - 1;
            box_load_seg(b, pitch, d, a0, hi, nv, buf + (2 * sb) * seglen);
            box_load_seg(b, pitch, u, a0, hi, nv, buf + (2 * sb + 1) * seglen);
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    const int64_t step = gridDim.y;
    int64_t i = blockIdx.y;
#pragma unroll
    for (int k = 0; k < kBoxBufs - 1; ++k) load_row(i + k * step, k);
    int sb = 0;
    for (; i < rows; i += step) {
        asm volatile("cp.async.wait_group %0;" ::"n"(kBoxBufs - 2) : "memory");
        __syncthreads();  // row i's segments are visible to the block; every thread is done with row i - step
        // prefetch row i + (kBoxBufs-1) step into the buffer of row i - step
        load_row(i + (kBoxBufs - 1) * step, (sb + kBoxBufs - 1) % kBoxBufs);
        const V* D = buf + (2 * sb) * seglen;
        const V* U = D + seglen;
        V* dst = out + i * pitch;
#pragma unroll
        for (int c = 0; c < 4; ++c) {  // column p0 + threadIdx.x + 256 c: a warp reads consecutive words
            const int64_t j = p0 + threadIdx.x + kBoxThreads * c;
            if (j < cols) {
                const int64_t l = j - rw - 1;
                const int64_t r = j + rw < hi ? j + rw : hi;
                const int kr = static_cast<int>(r - a0), kl = static_cast<int>(l - a0);
                __stcs(dst + j, ((D[kr] - U[kr]) - D[kl]) + U[kl]);
            }
        }
        sb = (sb + 1) % kBoxBufs;
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
}

// Band box filter (production): the matrix is cut into gridDim.x column panels of W output columns and
// gridDim.y row bands of H output rows, one block each, sized by the host so the grid is one full wave
// (blocks = SMs x resident blocks per SM).  A block walks its band top to bottom; output row i needs the
// SAT row segments d = min(i + rh, rows - 1) and u = i - rh - 1 (columns [p0 - rw - 1, p0 + W - 1 + rw]).
// Warp 0 fetches both with 1-D bulk copies (TMA engine, one instruction per segment, completion on the
// ring slot's mbarrier), RB output rows per ring slot, AHEAD slots ahead; a thread evaluates its column
// for the slot's RB rows as RB independent chains with hoisted offsets.  Measured at 32K^2 int32, r = 8
// (tools/bench_box.py): row-at-a-time variants ran at 1.1-1.5 TB/s (instruction-issue
// bound: ncu issue slots 68% busy at ~50 instructions per output); <8, 1> at 4 blocks per SM 1.62 ms =
// 5.3 TB/s of the algorithmic 8 B/elem, with ncu DRAM read + write 1.00x algorithmic (the strided-row
// staged kernel below reads the SAT twice from DRAM: 12.9 GB for 8.6 GB algorithmic); the slot's copies
// issued by 8 lanes instead of thread 0: 1.547 ms = 5.55 TB/s.
// Row d is new data (one DRAM read per SAT row and band); row u is the row d of 2 rh + 1 output rows
// earlier -- an L2 hit while the concurrent bands' working set, bands x (2 rh + 1) rows x cols x 4 B, fits
// in L2 (32K columns, rh = 64, two bands: 33 MB of 126 MB).  All blocks walk rows top-down at about the
// same rate, so the panels' horizontal halos (2 rw + 1 columns, read by both neighbours) are L2 hits too.
// Segment columns outside [0, cols) are zeroed once and never copied.  P:48 is evaluated left to right as
// box_sum_kernel; columns < 0, rows < 0 read as 0.  Requires 16-byte aligned b, pitch % 4 == 0,
// cols % 4 == 0 (whole 16-byte bulk-copy granules).
// RB output rows per ring slot (one barrier and one mbarrier wait per slot), AHEAD slots in flight ahead of
// the one being evaluated, Q = AHEAD + 2 ring slots (in flight, read now, read by laggards)
template <int RB_, int AHEAD_>
struct BandCfg {
    static constexpr int RB = RB_, AHEAD = AHEAD_, Q = AHEAD_ + 2;
    static constexpr size_t smem(int64_t segw) { return 256 + static_cast<size_t>(2) * Q * RB * segw * 4; }
};

template <typename V, typename Cfg>
__global__ void __launch_bounds__(256) box_band_kernel(const V* __restrict__ b, V* __restrict__ out, int rows,
                                                       int64_t cols, int64_t pitch, int rh, int rw, int W, int H,
                                                       int segw) {
    constexpr int Q = Cfg::Q, RB = Cfg::RB, kBandAhead = Cfg::AHEAD;
    extern __shared__ __align__(128) unsigned char band_smem[];
    uint64_t* full = reinterpret_cast<uint64_t*>(band_smem);  // [Q] mbarriers
    V* ringD = reinterpret_cast<V*>(band_smem + 256);           // [Q][RB][segw]
    V* ringU = ringD + Q * RB * segw;                           // [Q][RB][segw]
    const int64_t p0 = static_cast<int64_t>(blockIdx.x) * W;
    const int i0 = static_cast<int>(blockIdx.y) * H;
    if (p0 >= cols || i0 >= rows) return;  // uniform per block
    const int i1 = i0 + H < rows ? i0 + H : rows;
    const int64_t pend = p0 + W < cols ? p0 + W : cols;
    const int64_t a0 = (p0 - rw - 1) >= 0 ? ((p0 - rw - 1) & ~int64_t(3)) : -((-(p0 - rw - 1) + 3) & ~int64_t(3));
    const int64_t hi = cols - 1;
    const int64_t lo_c = a0 > 0 ? a0 : 0;                                  // first valid column of a segment
    const int64_t hi_c = a0 + segw < cols ? a0 + segw : cols;              // one past the last valid column
    const uint32_t seg_bytes = static_cast<uint32_t>((hi_c - lo_c) * sizeof(V));
    const int seg_off = static_cast<int>(lo_c - a0);
    // zero both rings (the invalid columns stay zero: copies only ever write [lo_c, hi_c)), init barriers
    for (int k = threadIdx.x; k < 2 * Q * RB * segw; k += blockDim.x) ringD[k] = V(0);
    if (threadIdx.x == 0) {
        for (int q = 0; q < Q; ++q) mbar_init(&full[q], 1);
        fence_mbar_init();
    }
    fence_proxy_async_smem();  // the zeros (generic proxy) before the bulk copies (async proxy)
    __syncthreads();
    const int nslots = (i1 - i0 + RB - 1) / RB;
    // warp 0: segments of output rows i0 + n*RB .. + RB - 1, lane k < RB issuing row k's copies (the copies
    // of a slot go out in parallel instead of one after another from a single thread)
    auto issue_slot = [&](int n, int slot) {
        if (n >= nslots) return;
        const int ia = i0 + n * RB, ib = ia + RB < i1 ? ia + RB : i1;
        const int lane = threadIdx.x & 31;
        if (lane == 0) {
            uint32_t bytes = 0;
            for (int i = ia; i < ib; ++i) bytes += (i - rh - 1 >= 0) ? 2 * seg_bytes : seg_bytes;
            mbar_arrive_expect_tx(&full[slot], bytes);
        }
        __syncwarp();
        const int i = ia + lane;
        if (lane < RB && i < ib) {
            const int d = i + rh < rows - 1 ? i + rh : rows - 1, u = i - rh - 1;
            V* sd = ringD + (slot * RB + lane) * segw + seg_off;
            bulk_load_1d(sd, b + static_cast<int64_t>(d) * pitch + lo_c, seg_bytes, &full[slot]);
            if (u >= 0)
                bulk_load_1d(ringU + (slot * RB + lane) * segw + seg_off, b + static_cast<int64_t>(u) * pitch + lo_c,
                             seg_bytes, &full[slot]);
        }
    };
    if (threadIdx.x < 32)
        for (int n = 0; n < kBandAhead; ++n) issue_slot(n, n);
    const int64_t jcol = p0 + threadIdx.x;  // the fast path's column of this thread
    const int kr0 = static_cast<int>((jcol + rw < hi ? jcol + rw : hi) - a0), kl0 = static_cast<int>(jcol - rw - 1 - a0);
    int slot = 0;
    uint32_t phase = 0;
    for (int n = 0; n < nslots; ++n) {
        if (threadIdx.x < 32) {  // that slot was last read for slot number n + kBandAhead - Q = n - 2 (barrier below)
            const int f = slot + kBandAhead < Q ? slot + kBandAhead : slot + kBandAhead - Q;
            issue_slot(n + kBandAhead, f);
        }
        mbar_wait(&full[slot], phase);
        const int ia = i0 + n * RB, ib = ia + RB < i1 ? ia + RB : i1;
        const V* D = ringD + slot * RB * segw;
        const V* U = ringU + slot * RB * segw;
        if (ib - ia == RB && ia - rh - 1 >= 0 && W <= static_cast<int>(blockDim.x)) {
            // fast path (every slot but the band's first and last few): one column per thread, all RB rows
            // present and below the top halo -- RB independent load / add / store chains, offsets hoisted
            if (jcol < pend) {
                V* dst = out + static_cast<int64_t>(ia) * pitch + jcol;
#pragma unroll
                for (int rr = 0; rr < RB; ++rr) {
                    const V dr = D[rr * segw + kr0], dl = D[rr * segw + kl0];
                    const V ur = U[rr * segw + kr0], ul = U[rr * segw + kl0];
                    __stcs(dst + rr * pitch, ((dr - ur) - dl) + ul);
                }
            }
        } else {
            for (int64_t j = p0 + threadIdx.x; j < pend; j += blockDim.x) {
                const int64_t r = j + rw < hi ? j + rw : hi;
                const int kr = static_cast<int>(r - a0), kl = static_cast<int>(j - rw - 1 - a0);
                V* dst = out + static_cast<int64_t>(ia) * pitch + j;
#pragma unroll
                for (int rr = 0; rr < RB; ++rr) {
                    if (ia + rr < ib) {
                        const V dr = D[rr * segw + kr], dl = D[rr * segw + kl];
                        const bool has_u = ia + rr - rh - 1 >= 0;
                        const V ur = has_u ? U[rr * segw + kr] : V(0), ul = has_u ? U[rr * segw + kl] : V(0);
                        __stcs(dst + rr * pitch, ((dr - ur) - dl) + ul);
                    }
                }
            }
        }
        if (++slot == Q) {
            slot = 0;
            phase ^= 1u;
        }
        __syncthreads();  // every thread is done with this slot before it is refilled (two slots later)
    }
}

// Batched rectangle queries: rects[k] = (u, d, l, r) in the convention of P:48 (u < i <= d,
// l < j <= r).  Indices are clamped into [-1, rows-1] / [-1, cols-1] (memory safety); an empty
// rectangle (u >= d or l >= r after clamping) gives 0.
template <typename V>
__global__ void __launch_bounds__(256) rect_sums_kernel(const V* __restrict__ b, int64_t rows, int64_t cols,
                                                        int64_t pitch, const int64_t* __restrict__ rects, int64_t n,
                                                        V* __restrict__ out) {
    for (int64_t k = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; k < n;
         k += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const longlong2 ud = *reinterpret_cast<const longlong2*>(rects + 4 * k);
        const longlong2 lr = *reinterpret_cast<const longlong2*>(rects + 4 * k + 2);
        auto clampi = [](int64_t x, int64_t hi) { return x < -1 ? int64_t(-1) : (x > hi ? hi : x); };
        const int64_t u = clampi(ud.x, rows - 1), d = clampi(ud.y, rows - 1);
        const int64_t l = clampi(lr.x, cols - 1), r = clampi(lr.y, cols - 1);
        out[k] = (u >= d || l >= r) ? V(0) : rect_from_sat(b, pitch, u, d, l, r);
    }
}

}  // namespace sat
