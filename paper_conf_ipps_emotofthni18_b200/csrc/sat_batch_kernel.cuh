// sat_batch_kernel.cuh -- SATs of a batch of small matrices in one launch.
//
// The single-matrix kernels parallelise one SAT over tiles with a look-back; a 256 x 256
// image has only 2-8 such tiles, so a batch of images launched one by one is latency-bound (the paper's
// own small-n weak spot).  Here the batch is the parallelism: one CTA computes one
// image at a time in a single pass (1R1W per element), walking down the image in bands of BR rows
// with the running column sums in registers -- the plain column-then-row definition:
//     c_i[j] = c_{i-1}[j] + a[i][j]          (column prefix; c_{-1} = 0)
//     b[i][j] = b[i][c0 - 1] + sum_{c0 <= j' <= j} c_i[j']   (row prefix over a column chunk [c0, c0 + CW))
// A CTA has NWR warps; a lane owns 4 consecutive columns of a CW = 128 NWR column chunk and BR rows of
// the band.  Per band: 16-byte loads (one band ahead for 8-warp CTAs), in-lane column prefix (+ the carried c), in-lane 4-column row
// prefix, one Kogge-Stone warp scan per row, warp totals exchanged through shared memory
// (one barrier, two buffers), 16-byte stores.  Images wider than CW are processed chunk by chunk; the
// left term b[i][c0 - 1] is read back from the output written by this CTA (ordered by the barriers).
// In place (src == dst) is safe: every element is read by the thread that later overwrites it.
#pragma once

#include <cstdint>

#include "sat_device.cuh"

namespace sat {

constexpr int kBatchBR = 8;  // rows per band

// matrices per CTA: one-warp CTAs (matrices <= 128 columns) are grouped 4 to a CTA, each warp on its
// own matrix, so that the 32-CTAs-per-SM limit does not cap the resident warps at 32
template <int NWR>
constexpr int kBatchIpb = NWR == 1 ? 4 : 1;

// rows [i0, i0 + BR) x columns [j0, j0 + 4) of one matrix; zeros outside it.  TIn = V (16-byte
// loads) or uint8_t (u8 pixels, one 32-bit load of 4 pixels, widened to V = uint32).
template <typename V, typename TIn, bool VEC>
__device__ __forceinline__ void load_band(V (&v)[kBatchBR][4], const TIn* a, int64_t i0, int64_t rows, int64_t cols,
                                          int64_t pitch, int64_t j0) {
#pragma unroll
    for (int r = 0; r < kBatchBR; ++r) {
        const int64_t i = i0 + r;
        const TIn* p = a + i * pitch + j0;
        if (VEC && i < rows && j0 + 3 < cols) {
            if constexpr (sizeof(TIn) == 1) {
                const uint32_t w = *reinterpret_cast<const uint32_t*>(p);
#pragma unroll
                for (int x = 0; x < 4; ++x) v[r][x] = V((w >> (8 * x)) & 0xffu);
            } else {
                const uint4 q = *reinterpret_cast<const uint4*>(p);
                v[r][0] = from_bits<V>(q.x); v[r][1] = from_bits<V>(q.y);
                v[r][2] = from_bits<V>(q.z); v[r][3] = from_bits<V>(q.w);
            }
        } else {
#pragma unroll
            for (int x = 0; x < 4; ++x) v[r][x] = (i < rows && j0 + x < cols) ? p[x] : V(0);
        }
    }
}

// u8 pixels of rows [i0, i0 + BR) x columns [j0, j0 + 4) as raw 32-bit words (pixel x in byte x);
// zeros outside the matrix.  Prefetching these costs BR registers instead of 4 BR.
template <bool VEC>
__device__ __forceinline__ void load_words_u8(uint32_t (&w)[kBatchBR], const uint8_t* a, int64_t i0, int64_t rows,
                                              int64_t cols, int64_t pitch, int64_t j0) {
#pragma unroll
    for (int r = 0; r < kBatchBR; ++r) {
        const int64_t i = i0 + r;
        const uint8_t* p = a + i * pitch + j0;
        if (VEC && i < rows && j0 + 3 < cols) {
            w[r] = *reinterpret_cast<const uint32_t*>(p);
        } else {
            uint32_t x = 0;
#pragma unroll
            for (int c = 0; c < 4; ++c)
                if (i < rows && j0 + c < cols) x |= static_cast<uint32_t>(p[c]) << (8 * c);
            w[r] = x;
        }
    }
}

// src: matrices of TIn with row stride spitch / matrix stride sstride; dst: V with pitch / stride
template <typename V, typename TIn, int NWR, bool VEC>
// >= 768 resident threads per SM (<= 85 registers) for the narrow CTAs and for u8 input: unbounded,
// ptxas used 130-190 registers there and left 10-14 warps per SM (ncu: 12% warps active for u8
// 256 x 256).  The 8-warp int32 / fp32 CTAs get 2 CTAs per SM (<= 128 registers): the one-band-ahead
// loads spill under the 85-register cap (1024^2: +19.5% over copy) and 150 unbounded registers leave
// one CTA per SM (+22.6%); at 128 registers +4.9% (measured)
__global__ void __launch_bounds__(NWR * 32 * kBatchIpb<NWR>,
                                  (sizeof(TIn) == 1 || NWR < 8) ? 768 / (NWR * 32 * kBatchIpb<NWR>) : 2)
    sat_batch_kernel(const TIn* src, V* dst, int64_t batch,
                                                            int64_t rows, int64_t cols, int64_t pitch,
                                                            int64_t stride, int64_t spitch, int64_t sstride) {
    constexpr int BR = kBatchBR, CW = 128 * NWR;
    __shared__ V wtot[2][NWR][BR];
    constexpr int IPB = kBatchIpb<NWR>;
    const int lane = threadIdx.x & 31, warp = IPB > 1 ? 0 : threadIdx.x >> 5;
    const int64_t first = static_cast<int64_t>(blockIdx.x) * IPB + (IPB > 1 ? threadIdx.x >> 5 : 0);
    int par = 0;
    for (int64_t img = first; img < batch; img += static_cast<int64_t>(gridDim.x) * IPB) {
        const TIn* a = src + img * sstride;
        V* b = dst + img * stride;
        for (int64_t c0 = 0; c0 < cols; c0 += CW) {
            const int64_t j0 = c0 + warp * 128 + lane * 4;  // this lane's first column
            V carry[4] = {V(0), V(0), V(0), V(0)};         // c_{i0 - 1}[j0 .. j0 + 3]
            // 8-warp CTAs (few, wide matrices) load the next band one band ahead so that its loads
            // overlap this band's scans; narrower int32 / fp32 CTAs are numerous enough to hide the
            // latency and run faster without the extra registers (measured).  u8
            // input always loads one band ahead, as raw words (8 registers; a warp row is only 128 B)
            constexpr bool PF = NWR >= 8;
            constexpr bool U8 = sizeof(TIn) == 1;
            V nx[PF && !U8 ? BR : 1][4];
            uint32_t nw[U8 ? BR : 1];
            if constexpr (U8) load_words_u8<VEC>(nw, reinterpret_cast<const uint8_t*>(a), 0, rows, cols, spitch, j0);
            else if constexpr (PF) load_band<V, TIn, VEC>(nx, a, 0, rows, cols, spitch, j0);
            for (int64_t i0 = 0; i0 < rows; i0 += BR) {
                V v[BR][4];
                if constexpr (U8) {
#pragma unroll
                    for (int r = 0; r < BR; ++r)
#pragma unroll
                        for (int x = 0; x < 4; ++x) v[r][x] = V((nw[r] >> (8 * x)) & 0xffu);
                    if (i0 + BR < rows)
                        load_words_u8<VEC>(nw, reinterpret_cast<const uint8_t*>(a), i0 + BR, rows, cols, spitch, j0);
                } else if constexpr (PF) {
#pragma unroll
                    for (int r = 0; r < BR; ++r)
#pragma unroll
                        for (int x = 0; x < 4; ++x) v[r][x] = nx[r][x];
                    if (i0 + BR < rows) load_band<V, TIn, VEC>(nx, a, i0 + BR, rows, cols, spitch, j0);
                } else {
                    load_band<V, TIn, VEC>(v, a, i0, rows, cols, spitch, j0);
                }
                // left term b[i][c0 - 1] (0 for the first chunk); written by this CTA one chunk earlier
                V left[BR];
#pragma unroll
                for (int r = 0; r < BR; ++r)
                    left[r] = (c0 > 0 && i0 + r < rows) ? b[(i0 + r) * pitch + c0 - 1] : V(0);
                // column prefix: c_i = c_{i-1} + a[i]
#pragma unroll
                for (int x = 0; x < 4; ++x) {
                    v[0][x] = carry[x] + v[0][x];
#pragma unroll
                    for (int r = 1; r < BR; ++r) v[r][x] = v[r - 1][x] + v[r][x];
                    carry[x] = v[BR - 1][x];
                }
                // row prefix of c_i over the chunk: in-lane, warp scan, warps to the left
                V incl[BR];
#pragma unroll
                for (int r = 0; r < BR; ++r) {
                    v[r][1] = v[r][0] + v[r][1];
                    v[r][2] = v[r][1] + v[r][2];
                    v[r][3] = v[r][2] + v[r][3];
                    incl[r] = v[r][3];
                }
#pragma unroll
                for (int d = 1; d < 32; d <<= 1)
#pragma unroll
                    for (int r = 0; r < BR; ++r) {
                        const V y = __shfl_up_sync(kFull, incl[r], d);
                        if (lane >= d) incl[r] = incl[r] + y;
                    }
                V off[BR];
#pragma unroll
                for (int r = 0; r < BR; ++r) {
                    V e = __shfl_up_sync(kFull, incl[r], 1);
                    off[r] = lane == 0 ? V(0) : e;
                }
                if constexpr (NWR > 1) {
                    if (lane == 31) {
#pragma unroll
                        for (int r = 0; r < BR; ++r) wtot[par][warp][r] = incl[r];
                    }
                    __syncthreads();
                    V wl[BR];
#pragma unroll
                    for (int r = 0; r < BR; ++r) wl[r] = V(0);
                    for (int u = 0; u < warp; ++u)
#pragma unroll
                        for (int r = 0; r < BR; ++r) wl[r] = wl[r] + wtot[par][u][r];
#pragma unroll
                    for (int r = 0; r < BR; ++r) off[r] = off[r] + wl[r];
                    par ^= 1;
                }
#pragma unroll
                for (int r = 0; r < BR; ++r) {
                    const V o = left[r] + off[r];
                    const int64_t i = i0 + r;
                    V* p = b + i * pitch + j0;
                    if (VEC && i < rows && j0 + 3 < cols) {
                        *reinterpret_cast<uint4*>(p) = make_uint4(to_bits(o + v[r][0]), to_bits(o + v[r][1]),
                                                                  to_bits(o + v[r][2]), to_bits(o + v[r][3]));
                    } else {
#pragma unroll
                        for (int x = 0; x < 4; ++x)
                            if (i < rows && j0 + x < cols) p[x] = o + v[r][x];
                    }
                }
            }
            // the next chunk reads this chunk's last column (global memory; same warp when NWR == 1)
            if constexpr (NWR == 1) __syncwarp();
            else __syncthreads();
        }
    }
}

}  // namespace sat
