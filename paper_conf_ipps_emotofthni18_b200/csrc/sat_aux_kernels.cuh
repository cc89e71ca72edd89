// sat_aux_kernels.cuh -- the multi-GPU strip-carry kernels (not in the paper; BASELINE.json
// north_star): strip column sums and the carry row of a rank.  Deterministic summation orders.
#pragma once

#include "sat_device.cuh"

namespace sat {

// Partial column sums: block (x, y) sums rows [y*seg, min((y+1)*seg, rows)) of columns
// [x*256*W, (x+1)*256*W) into partial[y][col], W = 4 columns per thread with 16-byte loads (VEC) or
// 1 with 4-byte loads.  Every warp reads 512 (128) contiguous bytes per row; 8 independent rows in
// flight per thread.  Per column: 8 row-residue accumulators, summed in ascending order at the end.
template <typename V, bool VEC>
__global__ void __launch_bounds__(256) colsum_partial_kernel(const V* __restrict__ src, V* __restrict__ partial,
                                                              int64_t rows, int64_t cols, int64_t pitch,
                                                              int64_t seg) {
    constexpr int W = VEC ? 4 : 1;
    const int64_t j = (static_cast<int64_t>(blockIdx.x) * 256 + threadIdx.x) * W;
    if (j >= cols) return;
    const int64_t r0 = static_cast<int64_t>(blockIdx.y) * seg;
    int64_t r1 = r0 + seg;
    if (r1 > rows) r1 = rows;
    V acc[8][W];
#pragma unroll
    for (int u = 0; u < 8; ++u)
#pragma unroll
        for (int c = 0; c < W; ++c) acc[u][c] = V(0);
    const bool full = j + W <= cols;
    int64_t i = r0;
    if (VEC && full) {
        for (; i + 8 <= r1; i += 8) {
            uint4 q[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) q[u] = __ldcs(reinterpret_cast<const uint4*>(src + (i + u) * pitch + j));
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                acc[u][0] = acc[u][0] + from_bits<V>(q[u].x);
                if constexpr (W == 4) {
                    acc[u][1] = acc[u][1] + from_bits<V>(q[u].y);
                    acc[u][2] = acc[u][2] + from_bits<V>(q[u].z);
                    acc[u][3] = acc[u][3] + from_bits<V>(q[u].w);
                }
            }
        }
        for (; i < r1; ++i) {
            const uint4 q = __ldcs(reinterpret_cast<const uint4*>(src + i * pitch + j));
            acc[0][0] = acc[0][0] + from_bits<V>(q.x);
            if constexpr (W == 4) {
                acc[0][1] = acc[0][1] + from_bits<V>(q.y);
                acc[0][2] = acc[0][2] + from_bits<V>(q.z);
                acc[0][3] = acc[0][3] + from_bits<V>(q.w);
            }
        }
    } else {
        for (; i + 8 <= r1; i += 8) {
#pragma unroll
            for (int u = 0; u < 8; ++u)
#pragma unroll
                for (int c = 0; c < W; ++c)
                    if (j + c < cols) acc[u][c] = acc[u][c] + __ldcs(src + (i + u) * pitch + j + c);
        }
        for (; i < r1; ++i)
#pragma unroll
            for (int c = 0; c < W; ++c)
                if (j + c < cols) acc[0][c] = acc[0][c] + __ldcs(src + i * pitch + j + c);
    }
#pragma unroll
    for (int c = 0; c < W; ++c) {
        if (j + c >= cols) break;
        V tot = V(0);
#pragma unroll
        for (int u = 0; u < 8; ++u) tot = tot + acc[u][c];
        partial[static_cast<int64_t>(blockIdx.y) * cols + j + c] = tot;
    }
}

// colsum[j] = sum over segments y = 0, 1, ... of partial[y][j] (ascending y).
template <typename V>
__global__ void colsum_reduce_kernel(const V* __restrict__ partial, V* __restrict__ colsum, int64_t cols,
                                     int nseg) {
    const int64_t j = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (j >= cols) return;
    V acc = V(0);
    for (int y = 0; y < nseg; ++y) acc = acc + partial[static_cast<int64_t>(y) * cols + j];
    colsum[j] = acc;
}

// Carry row of `rank`: C[j] = sum_{g<rank} gathered[g][j] (ascending g), carry = inclusive
// row-wise prefix of C.  One CTA of 1024 threads walking the columns in blocks of 1024: thread t
// sums column base + t over the lower ranks (coalesced loads), a block scan (warp scans + a scan of the
// 32 warp totals) gives the in-block prefix, and a running offset carries it across blocks.
template <typename V>
__global__ void __launch_bounds__(1024) carry_prefix_kernel(const V* __restrict__ gathered, int rank, int64_t cols,
                                                             V* __restrict__ carry) {
    __shared__ V warp_tot[32];
    __shared__ V block_tot;
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    V offset = V(0);  // sum of C over all earlier blocks (same value in every thread)
    for (int64_t base = 0; base < cols; base += 1024) {
        const int64_t j = base + t;
        V c = V(0);
        if (j < cols)
            for (int g = 0; g < rank; ++g) c = c + gathered[static_cast<int64_t>(g) * cols + j];
        const V incl = warp_inclusive_scan(c, lane);
        if (lane == 31) warp_tot[warp] = incl;
        __syncthreads();
        if (warp == 0) {
            const V x = warp_inclusive_scan(warp_tot[lane], lane);
            warp_tot[lane] = x;
            if (lane == 31) block_tot = x;
        }
        __syncthreads();
        const V pre = warp > 0 ? warp_tot[warp - 1] : V(0);
        if (j < cols) carry[j] = offset + (pre + incl);
        offset = offset + block_tot;
        __syncthreads();  // warp_tot / block_tot are rewritten by the next block
    }
}

// Test hook (sat_debug_occupy): each CTA holds `smem` bytes of shared memory and spins for `ns`
// nanoseconds, so that a SAT launched next on another stream finds most SMs taken -- its persistent CTAs
// then start over a long interval (forward progress under any CTA -> SM assignment).
__global__ void occupy_kernel(long long ns) {
    extern __shared__ unsigned char occ_smem[];
    const uint64_t t0 = sat_now_ns();
    if (threadIdx.x == 0) occ_smem[0] = 0;
    while (sat_now_ns() - t0 < static_cast<uint64_t>(ns)) __nanosleep(1000);
}

}  // namespace sat
