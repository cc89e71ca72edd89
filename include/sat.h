/*
 * sat.h -- libsat: single-pass summed area tables on NVIDIA B200 (sm_100a).  C ABI.
 *
 * PAPER.md = /root/reference/PAPER.md (Emoto et al., "An Optimal Parallel Algorithm for
 * Computing the Summed Area Table on the GPU", IPDPSW 2018), cited as P:<line>.
 *
 * The operation (Sec. I.A; restated P:132, Sec. III):
 *     dst[i][j] = sum_{0<=i'<=i, 0<=j'<=j} src[i'][j']        0 <= i < rows, 0 <= j < cols
 * for a row-major matrix "stored in the global memory of the GPU", the result "written in the
 * global memory" (Sec. I.C), element [i][j] at offset i*pitch + j (pitch >= cols is
 * reading R3 of DESIGN.md).  It is computed in ONE kernel pass that reads every element once and
 * writes every element once (the 1R1W-SKSS-LB method of Sec. IV: a dynamic tile
 * counter, per-tile published aggregates and look-back), re-designed for sm_100a.
 *
 * General rules for every entry point:
 *   - extern "C", never throws, returns sat_status_t; on failure sat_last_error_detail() gives a
 *     thread-local human-readable detail (CUDA/NCCL error text included).
 *   - Pointers documented as "device" must point to memory of the CURRENT CUDA device (the device
 *     of `stream`); "host" pointers are ordinary (pageable or pinned) host memory.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  Device-pointer
 *     calls are stream-ordered and asynchronous (no host synchronisation).
 *   - Sizes are int64_t element counts.  rows == 0 or cols == 0 is a no-op returning SAT_OK.
 *     Negative sizes or pitch < cols return SAT_ERR_INVALID_VALUE.
 *   - Pointers not aligned to the 4-byte element size return SAT_ERR_MISALIGNED.  16-byte alignment
 *     of both pointers and of pitch*4 selects the TMA fast path; otherwise a slower path is used.
 *   - Pad elements [cols, pitch) of every row of dst are never written.
 *   - src == dst (in place) is allowed; any other overlap returns SAT_ERR_INVALID_VALUE.
 *   - int32: two's-complement wraparound (the exact SAT reduced mod 2^32), bit-exact and
 *     deterministic.  fp32: IEEE adds in an unspecified, run-dependent association; every entry
 *     satisfies |dst - exact| <= (rows+cols) * 1.2e-7 * SAT(|src|) at that entry (R10).
 *   - libsat owns its workspace (per-tile aggregates, status words, tile counter), cached per
 *     (device, stream) and grown on demand, stream-ordered (cudaMallocAsync / cudaFreeAsync on
 *     that stream, no host synchronisation); the first call on a new (device, stream) resets the
 *     workspace's control block synchronously, so call once before capturing a CUDA graph.
 *     sat_release_stream_workspace frees one stream's workspace (e.g. before destroying the stream),
 *     sat_release_workspaces all of them.
 *   - Thread safety: calls on different streams run concurrently; calls on the same stream from
 *     several host threads are serialised per workspace.  sat_compute_host is serialised per device.
 */
#ifndef LIBSAT_SAT_H
#define LIBSAT_SAT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SAT_VERSION 100 /* 1.0.0 */

typedef enum {
    SAT_OK = 0,
    SAT_ERR_INVALID_VALUE = 1,
    SAT_ERR_MISALIGNED = 2,
    SAT_ERR_UNSUPPORTED = 3,
    SAT_ERR_OUT_OF_MEMORY = 4,
    SAT_ERR_CUDA = 5,
    SAT_ERR_NCCL = 6
} sat_status_t;

typedef enum { SAT_INT32 = 0, SAT_FLOAT32 = 1 } sat_dtype_t;

/* Opaque multi-GPU communicator (owns an ncclComm_t).  Created by sat_comm_init, freed by
 * sat_comm_destroy; owned by the caller. */
typedef struct sat_comm_s* sat_comm_t;

/* ------------------------------------------------------------------ single GPU (the hot path) */

/* SAT of an int32 matrix, one pass, uint32 wraparound.
 *   src   device, rows x cols, row stride `pitch` elements; read once.
 *   dst   device, same shape and pitch; written once; may equal src.
 * Errors: INVALID_VALUE (sizes, overlap), MISALIGNED, OUT_OF_MEMORY (workspace), CUDA (launch). */
sat_status_t sat_compute_i32(const int32_t* src, int32_t* dst, int64_t rows, int64_t cols,
                             int64_t pitch, void* stream);

/* SAT of an fp32 matrix (the paper's "4-byte float"); tolerance rule above.
 * CUDA graphs: after one call on a stream (which creates that stream's workspace), calls on that stream
 * are capturable and replayable -- the launch epoch lives on the device, nothing synchronises the host --
 * as long as no captured call needs a larger workspace than the calls made before capture
 * (tests/test_gpu_batched.py::test_sat_calls_replay_from_a_cuda_graph). */
sat_status_t sat_compute_f32(const float* src, float* dst, int64_t rows, int64_t cols,
                             int64_t pitch, void* stream);

/* Integral image of an 8-bit image (the computer-vision use of SATs): src is u8, the SAT
 * is uint32 (exact while the total stays below 2^32, i.e. rows*cols*255 < 2^32; modulo 2^32
 * beyond, like sat_compute_i32).  Same single-pass method; 1 B read + 4 B written per element.
 *   src        device, rows x cols bytes, row stride src_pitch BYTES (>= cols).
 *   dst        device, rows x cols uint32, row stride `pitch` ELEMENTS (>= cols); must not overlap src.
 * 16-byte aligned src/dst with src_pitch % 16 == 0 and pitch*4 % 16 == 0 take the TMA path, any other
 * layout the generic path.  Errors: INVALID_VALUE (sizes, overlap), MISALIGNED (dst not 4-byte
 * aligned), UNSUPPORTED (a forced variant without u8 support), OUT_OF_MEMORY, CUDA. */
sat_status_t sat_compute_u8(const uint8_t* src, int64_t src_pitch, uint32_t* dst, int64_t rows,
                            int64_t cols, int64_t pitch, void* stream);

/* fp32 input, fp64 SAT (the accumulation the paper's 4-byte float, P:253,
 * cannot hold exactly at large n).  dst[i][j] = sum of src[0..i][0..j], every addition in IEEE
 * fp64 (round to nearest); the fp32 -> fp64 widening is exact.  Same single-pass look-back method
 * (Sec. IV) with each 64-bit aggregate published as two tagged status words; one CTA per
 * 64 x 128 tile.  4 B read + 8 B written per element.
 *   src  device fp32, rows x cols, row stride src_pitch ELEMENTS (>= cols); read once.
 *   dst  device fp64, rows x cols, row stride dst_pitch ELEMENTS (>= cols); must not overlap src;
 *        pad elements are never written.
 * Accuracy: |dst - exact| <= (rows + cols) * 2.3e-16 * SAT(|src|) at every entry (the R10 argument
 * with the fp64 unit roundoff); exact while every partial sum is an integer < 2^53.  16-byte aligned
 * pointers with src_pitch % 4 == 0 and dst_pitch % 2 == 0 take the vector path.
 * Errors: INVALID_VALUE (sizes, overlap, NULL), MISALIGNED (src not 4-byte or dst not 8-byte
 * aligned), UNSUPPORTED (rows or cols >= 2^31), OUT_OF_MEMORY (workspace), CUDA.  Stream-ordered. */
sat_status_t sat_compute_f32_f64(const float* src, int64_t src_pitch, double* dst, int64_t dst_pitch,
                                 int64_t rows, int64_t cols, void* stream);

/* Moments for summed-area variance shadow maps (Lauritzen, ref. [8] at P:311): the SAT of a and
 * the SAT of a*a, in fp32, interleaved: dst[2*(i*dst_pitch + j)] = SAT(a)[i][j],
 * dst[2*(i*dst_pitch + j) + 1] = SAT(a*a)[i][j] (a*a rounded to fp32 once, then summed like
 * sat_compute_f32).  Same method and kernel as sat_compute_f32_f64 (the pair is one 64-bit element).
 *   src  device fp32, row stride src_pitch ELEMENTS (>= cols).
 *   dst  device fp32 pairs, row stride dst_pitch PAIRS (>= cols); must not overlap src.
 * Accuracy: each channel within (rows + cols) * 1.2e-7 * its absSAT (SAT(|a|), resp. SAT(a*a)).
 * Errors: as sat_compute_f32_f64. */
sat_status_t sat_compute_moments_f32(const float* src, int64_t src_pitch, float* dst, int64_t dst_pitch,
                                     int64_t rows, int64_t cols, void* stream);

/* Same as above for either dtype, plus an optional carry row.
 *   carry  device, `cols` elements of the same dtype, or NULL.  When given, carry[j] is added to
 *          every element of column j of the result: dst[i][j] = carry[j] + SAT(src)[i][j].  With
 *          carry = the last SAT row of the matrix above (a strip's "carry row", R12),
 *          dst is that strip of the SAT of the stacked matrix. */
sat_status_t sat_compute(sat_dtype_t dtype, const void* src, void* dst, int64_t rows, int64_t cols,
                         int64_t pitch, const void* carry, void* stream);

/* End-to-end call with HOST buffers: copies src host->device, computes the SAT, copies the result
 * device->host and synchronises `stream` before returning.  The matrix is pipelined in horizontal
 * strips (H2D of strip k+1, SAT of strip k and D2H of strip k-1 overlap; strip k uses the last SAT
 * row of strip k-1 as its carry row).  host_src/host_dst: rows x cols, row stride `pitch`
 * elements, may be the same buffer; pinned memory gives full PCIe bandwidth.  Device staging
 * buffers, copy streams and events are owned by libsat (cached per device); concurrent calls on one
 * device are serialised (a per-device lock held until the call's final synchronisation).
 * Synchronous. */
sat_status_t sat_compute_host(sat_dtype_t dtype, const void* host_src, void* host_dst, int64_t rows,
                              int64_t cols, int64_t pitch, void* stream);

/* SATs of a batch of equally shaped matrices in one launch (P:42 per matrix; SURVEY Sec. 8(f)
 * NEXT-2: many small images, where one matrix has too few tiles to fill 148 SMs):
 *   dst + k*image_stride = SAT(src + k*image_stride)   for 0 <= k < batch,
 * each matrix rows x cols with row stride `pitch` elements.  src/dst device; src == dst (in place)
 * allowed, partial overlap rejected.  image_stride (elements) >= (rows-1)*pitch + cols when
 * batch > 1.  One CTA per matrix, a single 1R1W pass (column-then-row); meant for
 * matrices up to ~1K x 1K -- a few large matrices are faster through sat_compute.  16-byte aligned
 * pointers with pitch and image_stride multiples of 4 take the vector path.  int32 wraps mod 2^32;
 * fp32 within the tolerance of sat_compute_f32.  Pads are never written.  batch == 0, rows == 0
 * or cols == 0 is a no-op.
 * Errors: INVALID_VALUE (sizes, stride, overlap, dtype), MISALIGNED (4-byte), UNSUPPORTED (rows or
 * cols >= 2^31), CUDA. */
sat_status_t sat_compute_batched(sat_dtype_t dtype, const void* src, void* dst, int64_t batch, int64_t rows,
                                 int64_t cols, int64_t pitch, int64_t image_stride, void* stream);

/* Integral images of a batch of 8-bit images (sat_compute_u8 per image, in one launch like
 * sat_compute_batched): dst + k*image_stride = uint32 SAT of (src + k*src_image_stride).
 *   src  device u8, row stride src_pitch BYTES (>= cols), image stride src_image_stride BYTES
 *        (>= (rows-1)*src_pitch + cols when batch > 1).
 *   dst  device uint32, row stride `pitch` ELEMENTS (>= cols), image stride image_stride ELEMENTS;
 *        must not overlap src.  Exact while an image's total is < 2^32, modulo 2^32 beyond.
 * 4-byte aligned src with src_pitch and src_image_stride multiples of 4, and 16-byte aligned dst
 * with pitch and image_stride multiples of 4, take the vector path.
 * Errors: INVALID_VALUE (sizes, strides, overlap), MISALIGNED (dst not 4-byte aligned),
 * UNSUPPORTED (rows or cols >= 2^31), CUDA. */
sat_status_t sat_compute_batched_u8(const uint8_t* src, int64_t src_pitch, int64_t src_image_stride,
                                    uint32_t* dst, int64_t batch, int64_t rows, int64_t cols, int64_t pitch,
                                    int64_t image_stride, void* stream);

/* ------------------------------------------------------------------ queries on a SAT */

/* Box filter from a SAT b (the O(1) rectangle sum of P:48 that motivates SATs):
 *   out[i][j] = sum of a[i'][j'] over i' in [i-rh, i+rh] and j' in [j-rw, j+rw], clipped to the
 *               matrix, = ((b[d][r] - b[u][r]) - b[d][l]) + b[u][l] with u = i-rh-1,
 *               d = min(i+rh, rows-1), l = j-rw-1, r = min(j+rw, cols-1); entries with a negative
 *               index are 0.  Evaluated in b's arithmetic (uint32 wraparound / fp32), left to right.
 *   sat, out  device, rows x cols, row stride `pitch` elements; out must not overlap sat.
 *   rh, rw    window half-heights / half-widths, >= 0.
 * Errors: INVALID_VALUE (sizes, negative radius, overlap), MISALIGNED (4-byte), CUDA. */
sat_status_t sat_box_sum(sat_dtype_t dtype, const void* sat, void* out, int64_t rows, int64_t cols,
                         int64_t pitch, int64_t rh, int64_t rw, void* stream);

/* Batched rectangle sums: out[k] = sum of a[i][j] for u < i <= d, l < j <= r, where
 * rects[4k..4k+3] = (u, d, l, r).  Indices are clamped to [-1, rows-1] / [-1, cols-1]; an empty
 * rectangle gives 0.  rects: device, n x 4 int64, 16-byte aligned; out: device, n elements.
 * Errors: INVALID_VALUE, MISALIGNED, CUDA. */
sat_status_t sat_rect_sums(sat_dtype_t dtype, const void* sat, int64_t rows, int64_t cols,
                           int64_t pitch, const int64_t* rects, int64_t n, void* out, void* stream);

/* ------------------------------------------------------------------ multi-GPU strip partition */

/* Column sums of a strip (not in the paper; BASELINE.json north_star's strip carry):
 *   colsum[j] = sum_i src[i][j], 0 <= i < rows.   src device (rows x cols, pitch); colsum device,
 *   cols elements.  Deterministic (fixed summation order). */
sat_status_t sat_strip_colsum(sat_dtype_t dtype, const void* src, void* colsum, int64_t rows,
                              int64_t cols, int64_t pitch, void* stream);

/* Carry row of rank `rank` from the gathered column sums of all ranks:
 *   C[j] = sum_{g < rank} gathered[g*cols + j]   (ascending g: same association on every rank)
 *   carry[j] = C[0] + ... + C[j]                  (row-wise prefix)
 * gathered device (nranks x cols), carry device (cols).  rank 0 gets the zero vector. */
sat_status_t sat_carry_prefix(sat_dtype_t dtype, const void* gathered, int nranks, int rank,
                              int64_t cols, void* carry, void* stream);

/* NCCL bootstrap.  Rank 0 calls sat_comm_get_unique_id and ships the 128 bytes to the other
 * ranks (the Python binding broadcasts them over the torch process group); every rank then calls
 * sat_comm_init collectively.  NCCL is loaded with dlopen("libnccl.so.2") at first use (the copy
 * torch already loaded).  Errors: NCCL (load or NCCL call failure), UNSUPPORTED (built without
 * nccl.h). */
sat_status_t sat_comm_get_unique_id(unsigned char id[128]);
sat_status_t sat_comm_init(sat_comm_t* comm, const unsigned char id[128], int nranks, int rank);
sat_status_t sat_comm_destroy(sat_comm_t comm);

/* Strip-partitioned SAT over `nranks` GPUs, one process per GPU, called collectively in the same
 * order on every rank with equal `cols`.  Rank r passes ITS horizontal strip: global rows
 * [row0_r, row0_r + strip_rows) with row0_r = sum of strip_rows of ranks < r (strips may differ in
 * height).  Steps: sat_strip_colsum -> ncclAllGather of the colsum vectors -> sat_carry_prefix ->
 * sat_compute with that carry.  strip_src/strip_dst device (this rank), may be equal.
 * Errors: a null comm, unknown dtype or cols <= 0 (arguments equal on every rank) return before the
 * collective; a rank-local failure (bad strip_rows / pitch, overlap, misalignment, column-sum launch)
 * still joins the all-gather with a zero vector, so no other rank blocks, and is then returned. */
sat_status_t sat_compute_sharded(sat_comm_t comm, sat_dtype_t dtype, const void* strip_src,
                                 void* strip_dst, int64_t strip_rows, int64_t cols, int64_t pitch,
                                 void* stream);

/* ------------------------------------------------------------------ chained strip partition (NEXT-1)
 *
 * The same horizontal strip partition as sat_compute_sharded (rank r holds global rows
 * [row0_r, row0_r + strip_rows)), computed in ONE pass per rank: each element is read once and written
 * once (2 accesses instead of the 3 of colsum + all-gather + SAT).  A rank walks its strip in the
 * anti-diagonal order of groups of 8 vertically adjacent tiles (Fig. 9's order over tall groups); each
 * tile's column walker adds the carry T(r-1) -- the column sums of all rows of ranks 0..r-1 over its tile
 * column -- from the rank's inbox to its strip-local column carry, and as soon as the bottom tile of tile
 * column J has resolved, the kernel pushes T(r) = its strip column sums + T(r-1) -- as epoch-tagged 64-bit
 * status words, the single-copy-atomic protocol of the look-back (R11) -- into the inbox of
 * rank r+1 only, through peer-mapped memory over NVLink (CUDA IPC).  Every rank polls one vector and pushes
 * one per tile column, whatever nranks; a rank lags the one above by ~1/8 of its strip's tile rows
 * (DESIGN.md Sec. 7).  No NCCL call on the data path.
 *
 * Setup (collective, once per partition): every rank calls sat_chain_create on its own device,
 * exports its 64-byte IPC handle with sat_chain_export, the ranks all-gather the handles (the Python
 * binding does this over the torch process group), and every rank calls sat_chain_connect with the
 * nranks x 64 handle bytes (its own entry is ignored).  sat_chain_connect_local instead connects n
 * chains created in ONE process on ONE device (rank r = chains[r]): the single-GPU emulation used by
 * the tests and by bench.py's per-rank measurements.  nranks <= 8 (one node).
 *
 * sat_compute_chained must be called by every rank, in the same order, with equal cols (the chain's),
 * and >= 1 strip row per rank.  Calls are stream-ordered and asynchronous; a rank's kernel waits
 * inside the GPU for its upstream ranks' column sums of the same call, and a rank may run at most
 * two calls ahead of its downstream ranks (the inbox is double-buffered; back-pressure words are
 * written by the downstream kernels at exit).  strip_src / strip_dst device (this rank), may be
 * equal; TMA alignment rules as sat_compute.  int32 bit-exact; fp32 within the sat_compute_f32
 * tolerance with global rows / cols.
 * Errors: INVALID_VALUE (arguments, not connected, wrong device), OUT_OF_MEMORY, CUDA (IPC, launch),
 * UNSUPPORTED (2^30 calls on one chain: recreate it). */
typedef struct sat_chain_s* sat_chain_t;
sat_status_t sat_chain_create(int nranks, int rank, int64_t cols, sat_chain_t* chain);
sat_status_t sat_chain_export(sat_chain_t chain, unsigned char handle[64]);
sat_status_t sat_chain_connect(sat_chain_t chain, const unsigned char* handles);
sat_status_t sat_chain_connect_local(sat_chain_t* chains, int n);
sat_status_t sat_chain_destroy(sat_chain_t chain);
sat_status_t sat_compute_chained(sat_chain_t chain, sat_dtype_t dtype, const void* strip_src, void* strip_dst,
                                 int64_t strip_rows, int64_t cols, int64_t pitch, void* stream);

/* ------------------------------------------------------------------ introspection */

typedef struct {
    int32_t tile_rows;     /* TR: rows per tile */
    int32_t tile_cols;     /* TC: columns per tile */
    int32_t tma;           /* 1 = TMA path, 0 = generic load/store path */
    int32_t ctas;          /* persistent CTAs launched */
    int64_t tiles;         /* ceil(rows/TR) * ceil(cols/TC) */
    int64_t aux_bytes;     /* bytes of per-tile aggregate slots for this shape */
    int32_t variant;       /* kernel variant index */
    int32_t order;         /* 0 = diagonal-major (Fig. 9), 1 = row-major */
    int32_t family;        /* 2 = TMEM-parked kernel (sat_tm_kernel), 0 = classic (sat_tiles_kernel) */
    int32_t reserved;
} sat_plan_t;

/* Fill `plan` with what sat_compute would launch for this problem (no launch, no allocation). */
sat_status_t sat_query_plan(sat_dtype_t dtype, int64_t rows, int64_t cols, int64_t pitch,
                            const void* src, const void* dst, sat_plan_t* plan);

/* TEST / TUNING HOOKS (process-wide; for sweeps and tests -- not part of the computing API).
 * variant: -1 = automatic choice, else an index < sat_num_variants() (the shipped library has the
 * variants auto-selection uses: 0 classic 64x128, 1 TMEM-parked 128x128 with two row walkers,
 * 2 u8 integral images on 128x128, 3 TMEM-parked flat 64x256, 4 chained strips (sat_compute_chained
 * only; ignored by sat_compute), 5 u8 integral images on flat 64x256; -DSAT_EXPERIMENTAL builds append
 * the unshipped tuning configurations); order: 0 = diagonal-major (Fig. 9), 1 = row-major,
 * 2 = column-major, (g << 8) = diagonal-major over g-wide tile groups, 3 | (g << 8) = diagonal-major
 * over g-tall groups (the chained strips' order); ctas_per_sm: 0 = occupancy maximum.  Returns
 * INVALID_VALUE for an unknown variant or order. */
sat_status_t sat_set_tuning(int variant, int order, int ctas_per_sm);
int sat_num_variants(void);
/* Cap the total number of persistent CTAs (0 = no cap).  A cap of 1 runs the whole matrix on one
 * CTA: the forward-progress test of the tile-counter protocol. */
sat_status_t sat_set_max_ctas(int max_ctas);
/* Tile shape of variant v (TR, TC), or INVALID_VALUE. */
sat_status_t sat_variant_info(int variant, int32_t* tile_rows, int32_t* tile_cols);

/* Test hook: run the kernel's serial-number -> tile mapping on the device for an R x C tile grid.
 * out: device int32[2*R*C], out[2s] = I, out[2s+1] = J of serial s. */
sat_status_t sat_debug_tile_order(int64_t R, int64_t C, int order, int32_t* out, void* stream);

/* Test hook: launch `ctas` CTAs on `stream` that each hold `smem_bytes` (<= 227 KiB) of shared memory and
 * spin for `ns` (<= 1e10) nanoseconds.  With ctas close to the SM count and smem_bytes large enough that a
 * SAT CTA cannot share an SM, a SAT launched next on another stream starts with only a few resident
 * CTAs and gets the rest as the occupying CTAs retire: the forward-progress condition of P:21 / the
 * SKSS counter under an adversarial CTA -> SM assignment.  INVALID_VALUE on bad arguments,
 * SAT_ERR_CUDA on a launch error. */
sat_status_t sat_debug_occupy(int ctas, int64_t ns, int64_t smem_bytes, void* stream);

/* Test/tuning hook: per-CTA phase counters (cycles, look-back steps) of the most recent launch.
 * out: host int64[max_ctas * n_stats].  Only libsat_stats.so (built with -DSAT_STATS=1) records
 * them; the production library returns SAT_ERR_UNSUPPORTED. */
sat_status_t sat_debug_stats(int64_t* out, int max_ctas, int* n_ctas, int* n_stats);

/* Test/tuning hook: per-tile timeline of the most recent launch (libsat_stats.so only): out[8t + e]
 * for tile serial t, %globaltimer ns: e = 0 acquired, 1 data landed (compute starts), 2 local
 * aggregates published, 3 row walk resolved, 4 column walk resolved, 5 Step 4 done, 6 store issued,
 * 7 TMA load issued (0 where a step does not apply to the variant). */
sat_status_t sat_debug_trace(int64_t* out, int64_t max_tiles, int64_t* n_tiles);

/* Test hook: the published aggregate words of the most recent sat_compute launch on (current
 * device, `stream`) -- the per-tile slots of Steps 2.A/2.B/3 in their final state.
 * info (required) receives the tile grid; host_out (NULL = only fill info) receives info->words
 * 64-bit status words (synchronises `stream`): row slots [R*C][tile_rows], column slots
 * [R*C][tile_cols], corner slots [R*C], tile t = I*C + J.  A word is (epoch << 34 | kind << 32 |
 * value bits), kind 1 = local, 2 = inclusive; row / column slots hold prefix sums over the tile's
 * rows / columns (R5'), the corner GLS (local) or GS (inclusive).  Classic-kernel launches
 * (small matrices) share the layout.  Errors: INVALID_VALUE (no workspace, max_words too small), CUDA. */
typedef struct {
    int32_t tile_rows, tile_cols, R, C;
    int64_t words;
} sat_ws_info_t;
sat_status_t sat_debug_workspace(void* stream, uint64_t* host_out, int64_t max_words, sat_ws_info_t* info);

/* Free the cached workspace of (current device, `stream`) (synchronises the stream); a later call
 * on that stream allocates a new one.  Call before destroying a stream libsat has used. */
sat_status_t sat_release_stream_workspace(void* stream);

/* Free every cached workspace and staging buffer (synchronises the devices that own them). */
sat_status_t sat_release_workspaces(void);

const char* sat_status_string(sat_status_t s);
const char* sat_last_error_detail(void);
int sat_version(void);

#ifdef __cplusplus
}
#endif

#endif /* LIBSAT_SAT_H */
