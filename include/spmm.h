/*
 * spmm.h -- C ABI of the B200-native row-permuted CSR SpMM library (libspmm_b200.so).
 *
 * Method: Mehrabi et al., "Learning Sparse Matrix Row Permutations for Efficient SpMM on GPU
 * Architectures", ISPASS 2021 (/root/reference/PAPER.md, cited P:L<n> + section).
 *   C[M][K] = A[M][N] . B[N][K]                      (Alg.1 "Input: CSR A[M][N], float B[N][K]")
 * computed on a row-PERMUTED copy of the CSR matrix (§III: "re-order rows ... yet preserve
 * the CSR representation"), the inverse permutation being applied when C is written (C is always in
 * ORIGINAL row order).  Policies: §III.A load balancing, §III.B cache-aware,
 * §III.C hybrids, DCSR.  Features: Table II.  Predictor: §V.B
 * (P:L273-277).  Exact definitions and readings: DESIGN.md §"Readings".
 *
 * Conventions for every entry point
 *   - extern "C", plain pointers and sizes; nothing throws across the ABI; every call returns an
 *     spmm_status and on failure leaves a detail message in spmm_last_error() (thread-local).
 *   - "device" pointers are CUDA device addresses on the device that was current when the handle
 *     was created; "host" pointers are ordinary (preferably pinned) host memory.
 *   - cuda_stream is a cudaStream_t passed as void* (NULL = legacy default stream).  Every call that
 *     takes a stream is stream-ordered; calls that return host data synchronise that stream.
 *   - Layouts: CSR rowidx int64[M+1], colidx int32[nnz] (strictly increasing within a row),
 *     value float32[nnz].  Dense B float32 row-major [N][K], C float32 row-major [M][K], both
 *     16-byte aligned, K % 4 == 0, 4 <= K <= 1024 (B rows are read as float4 vectors along K).
 *   - Limits: 0 <= M, N < 2^31, 0 <= nnz < 2^31 (device offsets are int32).
 */
#ifndef SPMM_B200_H
#define SPMM_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct spmm_ctx *spmm_handle;

typedef enum {
    SPMM_OK = 0,
    SPMM_ERR_INVALID_ARG = 1,  /* NULL pointer, negative size, size >= 2^31, bad window/params   */
    SPMM_ERR_INVALID_CSR = 2,  /* rowidx[0]!=0, rowidx[M]!=nnz, decreasing offsets, column out of
                                  range, or columns not strictly increasing within a row         */
    SPMM_ERR_UNSUPPORTED = 3,  /* K % 4 != 0, K > 1024, misaligned B/C                            */
    SPMM_ERR_CUDA = 4,         /* a CUDA runtime error (text in spmm_last_error)                  */
    SPMM_ERR_OOM = 5,          /* device allocation failed                                        */
    SPMM_ERR_STATE = 6         /* handle used on a device other than the one it was created on    */
} spmm_status;

/* Row-permutation policies.  perm[p] = ORIGINAL row placed at position p (gather form). */
typedef enum {
    SPMM_POLICY_IDENTITY = 0,   /* plain CSR order ("original CSR")                     */
    SPMM_POLICY_NNZ_SORT = 1,   /* stable sort by nnz_i, descending; ties by row id (north star)       */
    SPMM_POLICY_PLAIN_SORT = 2, /* stable sort by warp load ceil(nnz_i/nt), descending   */
    SPMM_POLICY_CTA_AWARE = 3,  /* greedy chain: next row = min Hamming to previous row       */
    SPMM_POLICY_HYBRID_1 = 4,   /* Plain Sort, ties (equal warp load) broken by Hamming       */
    SPMM_POLICY_HYBRID_2_1 = 5, /* CTA-aware, Hamming ties broken by warp-load difference     */
    SPMM_POLICY_FLIPPED = 6,    /* Plain Sort with every odd nw-row chunk reversed            */
    SPMM_POLICY_LPT = 7,        /* LPT: rows in desc. warp load to the least-loaded warp      */
    SPMM_POLICY_WARP_AWARE = 8, /* row at q minimises Hamming to row q-nw                 */
    SPMM_POLICY_HYBRID_2_2 = 9, /* CTA-aware, ties broken by Hamming to row q-nw              */
    SPMM_POLICY_HYBRID_2_3 = 10,/* Warp-aware, ties broken by warp-load difference            */
    SPMM_POLICY_DCSR = 11,      /* non-empty rows first in original order, then empty rows     */
    SPMM_POLICY_COUNT = 12
} spmm_policy;

typedef struct {
    int32_t nw;             /* warps per CTA in the paper's model, default 32                */
    int32_t nt;             /* threads per warp, default 32                                  */
    int32_t bw;             /* columns per B cache-line block, default 32 = 128 B / 4 B */
    int32_t split_nnz;      /* rows longer than this are cut into chunks of this many nnz whose
                               partial sums are combined in a fixed pairwise order; default 128
                               (bounds every fp32 accumulation chain, DESIGN.md §"Accuracy")         */
    int64_t window;         /* greedy-chain window W (multiple of nw); 0 = whole matrix (paper-exact,
                               P:L118-122).  Every chain policy at any W (up to W = M); above 32768
                               rows through the inverted-index builder (f3,
                               DESIGN.md §8; cost grows with the posting lists of hub blocks).
                               Default 1024                                                            */
    int32_t preorder;       /* chain policies: windows over 0 = the original order, 1 = the MinHash key
                               order, 2 = the median-column-block order (DESIGN.md §2 "pre-orders")    */
    int32_t fuse_rows;      /* row fusion in spmm_run (a7/a8): 0 = auto -- take the short rows R consecutive
                               positions at a time and walk the union of their columns once (each shared B
                               row loaded once) when the unions hold <= 3/4 of those rows' nnz; 1 = off;
                               2 = always (where the K geometry has a fused kernel: R = 4 at K = 64,
                               R = 2 at K = 128).  C is bit-identical in every setting.                 */
    uint64_t seed;          /* MinHash seed                                                          */
} spmm_params;

/* Fill *p with the defaults (nw=nt=bw=32, split_nnz=128, window=1024, preorder=0, fuse_rows=0, seed=0). */
spmm_status spmm_default_params(spmm_params *p);

/* Optional device allocator (e.g. PyTorch's caching allocator).  alloc(bytes, stream, ctx) returns a
 * device pointer or NULL; free_(ptr, stream, ctx) releases it stream-ordered.  Pass NULLs to restore
 * the built-in cudaMallocAsync allocator.  Process-wide; set it before creating handles. */
spmm_status spmm_set_allocator(void *(*alloc)(size_t bytes, void *stream, void *ctx),
                               void (*free_)(void *ptr, void *stream, void *ctx), void *ctx);

/* Create a handle: copies and validates the CSR (§II.A) into handle-owned device memory
 * (inputs_on_device = 1: the three arrays are device pointers, else host pointers; caller buffers
 * may be freed on return).  Synchronises cuda_stream (validation result).  The current policy is
 * IDENTITY until spmm_permute is called. */
spmm_status spmm_create(spmm_handle *out, int64_t M, int64_t N, int64_t nnz, const int64_t *rowidx,
                        const int32_t *colidx, const float *value, int inputs_on_device, void *cuda_stream);

/* Build permutation `policy` (params NULL = defaults), the permuted CSR it implies and its row-class
 * counts, all on the device (offline / amortised), then replace the current permutation with it.
 * Atomic: everything is built into new buffers first; on any failure (e.g. SPMM_ERR_OOM) the handle keeps
 * its previous permutation, permuted CSR and schedules and stays usable.  Synchronises cuda_stream, and waits
 * for this handle's runs still in flight (they read the arrays being replaced).  Drops the cached run
 * schedules (rebuild: spmm_prepare).  Must not be called concurrently with other calls on the same handle. */
spmm_status spmm_permute(spmm_handle h, spmm_policy policy, const spmm_params *params, void *cuda_stream);

/* Build the K-dependent run schedule of the current permutation (a7: empty / whole / split rows packed into
 * warp tasks for the lane geometry of K, row-fusion unions where they pay) so that spmm_run with this K is
 * fully asynchronous.  B / C (device, may be NULL) only select the lane geometry: 32-byte aligned (or NULL)
 * -> 256-bit lane loads, else 128-bit; pass the buffers the runs will use.  Up to 4 geometries are cached per
 * permutation.  A run whose geometry was not prepared builds it itself (and then synchronises its stream).
 * Also sizes the scratch of runs captured into CUDA graphs (spmm_run).
 * Synchronises cuda_stream.  Errors: INVALID_ARG (NULL h, K <= 0), UNSUPPORTED (K), STATE, OOM, CUDA. */
spmm_status spmm_prepare(spmm_handle h, int64_t K, const float *B, const float *C, void *cuda_stream);

/* Install a caller-supplied permutation instead of building one -- e.g. a permutation computed offline and cached
 * ("row permutations happen offline or the cost is amortized"; SURVEY §5 checkpoint / resume: the Python
 * package's permcache stores spmm_get_perm results keyed by a hash of the CSR, policy and parameters).  perm: HOST
 * int32[M], perm[p] = original row at position p; checked on the device to be a bijection on [0, M).  Builds the
 * permuted CSR and row classes as spmm_permute does (params: split_nnz; NULL = defaults), atomically: on any error
 * the handle keeps its previous permutation.  Synchronises cuda_stream.  Errors: INVALID_ARG (NULL, not a
 * bijection, bad params), STATE, OOM, CUDA. */
spmm_status spmm_set_perm(spmm_handle h, const int32_t *perm, const spmm_params *params, void *cuda_stream);

/* Copy the current permutation (M int32, HOST buffer).  Reads it back on the handle's own non-blocking
 * stream (the permutation is complete when spmm_permute returns); no device-wide synchronisation. */
spmm_status spmm_get_perm(spmm_handle h, int32_t *perm_out);

/* Copy the current permuted CSR to HOST buffers: rowidx int64[M+1], colidx int32[nnz], value f32[nnz]. */
spmm_status spmm_get_permuted_csr(spmm_handle h, int64_t *rowidx, int32_t *colidx, float *value);

/* Row classes of the current permutation (a7): out[0]=empty rows (nnz==0, zero-filled), out[1]=non-empty
 * rows handled whole (nnz <= split_nnz), out[2]=split (long) rows, out[3]=split_nnz-chunks of the split
 * rows, out[4]=max row nnz. */
spmm_status spmm_get_info(spmm_handle h, int64_t out[5]);

/* Run schedule (a7) used by the most recent spmm_run on h: out[0] = rows per warp task (lane groups; 0 = no
 * schedule yet), out[1] = row-fusion factor R in use (1 = none), out[2] = warp tasks, out[3] = fusion groups,
 * out[4] = union records of those groups, out[5] = nnz of the fused rows (out[4] / out[5] = B-row loads per
 * nnz on the fused rows).  Errors: INVALID_ARG (NULL). */
spmm_status spmm_get_schedule_info(spmm_handle h, int64_t out[6]);

/* The 24 Table II features (definitions DESIGN.md §"Features") computed on the device,
 * of the ORIGINAL order (use_current_order = 0) or of the current permutation (1), with nw/nt/bw from
 * params (NULL = 32/32/32).  out: 24 doubles, HOST.  Synchronises cuda_stream. */
spmm_status spmm_features(spmm_handle h, int use_current_order, const spmm_params *params, double out[24],
                          void *cuda_stream);

/* B200 platform features g0..g6 ("platform-aware features are crucial", P:L267,
 * P:L330-332; definitions DESIGN.md readings A24-A26) of the ORIGINAL order (use_current_order = 0) or of the
 * current permutation, for right-hand-side width K: out[0] / out[1] = column-union of 2 / 4 consecutive rows
 * per nnz (row fusion's B-row loads per nnz), out[2] = distinct columns per 1024-row window per nnz, out[3] =
 * B-row share 4K*Cn / (4(M+1) + 8 nnz + 4K*Cn + 4MK) of the algorithmic bytes (Cn = distinct columns),
 * out[4] = empty-row fraction, out[5] = fraction of nnz in rows longer than 128, out[6] = lane-slot efficiency
 * of the short rows at the kernel's rows per warp task for K.  Integer counts on the device, ratios
 * (double)int64 / (double)int64 (0 on an empty denominator): bit-identical to the oracle.  out: 7 doubles,
 * HOST.  Scratch up to 12 bytes per nnz (a (window, column) key sort).  Synchronises cuda_stream.
 * Errors: INVALID_ARG (NULL, K <= 0), STATE, OOM, CUDA. */
spmm_status spmm_features_b200(spmm_handle h, int use_current_order, int64_t K, double out[7], void *cuda_stream);

/* C = A . B on the device (beta = 0: C is fully overwritten; empty rows get zeros).
 * B: device, float32 row-major [N][K]; C: device, float32 row-major [M][K] in ORIGINAL row order.
 * Asynchronous on cuda_stream once the schedule of K's geometry exists (spmm_prepare, or an earlier run
 * with this K): no host synchronisation, and runs on one handle may be issued concurrently from several
 * streams / host threads -- each run takes one of 4 handle-owned scratch slots (task counter, split-row
 * partials, zero-fill side stream) round-robin and waits, on its own stream, for that slot's previous run.
 * (The kernel-timing aid, spmm_set_kernel_timing, is the exception: its events belong to the handle.)
 * CUDA graphs: a run may be captured (cudaStreamBeginCapture on cuda_stream, e.g. torch.cuda.graph) once
 * spmm_prepare has built its K's schedule and sized the handle's capture scratch; the captured run allocates
 * nothing and waits on nothing outside the graph (its zero-fill side stream forks from and joins the capture).
 * Replays of graphs holding runs of one handle share that scratch and must be ordered (e.g. one stream).
 * Capturing an unprepared K fails with SPMM_ERR_STATE before any work is queued.  A graph holds device addresses
 * of the handle's permuted CSR, schedule and capture scratch: spmm_permute / spmm_set_perm (new arrays), an
 * spmm_prepare that grows the capture scratch (a larger K), and spmm_destroy invalidate graphs captured from the
 * handle -- re-capture after them. */
spmm_status spmm_run(spmm_handle h, const float *B, int64_t K, float *C, void *cuda_stream);

/* spmm_run with the C all-gather fused into the epilogue (SURVEY §8(f) f2 ii): every row this handle computes
 * (its shard, M rows) is stored to each of n_dsts (1..8) destinations at row row_offset + r, r = the handle's
 * original row index -- C_dsts: HOST array of DEVICE pointers to [>= row_offset + M][K] float32 row-major
 * buffers, typically this GPU's full-C buffer and its peers' (peer-mapped / symmetric-memory addresses on an
 * NVLink/NVSwitch node: the SpMM's own stores carry the exchange, no separate collective).  When every rank
 * calls it with all ranks' buffers and its shard's row offset, each buffer ends up holding the full C once all
 * ranks are done (the caller orders that, e.g. a barrier).  Other rows are untouched.  Asynchrony and
 * concurrency as spmm_run.  Errors: INVALID_ARG (NULL, n_dsts out of range, negative row_offset), UNSUPPORTED (K, or a
 * destination row not 16-byte aligned), STATE, CUDA. */
spmm_status spmm_run_to(spmm_handle h, const float *B, int64_t K, float *const *C_dsts, int32_t n_dsts,
                        int64_t row_offset, void *cuda_stream);

/* spmm_run into a C whose rows are ldc floats apart (ldc >= K, ldc % 4 == 0): C[r * ldc + k], k < K; the other
 * columns are untouched.  Lets a caller compute column blocks of a wider C, e.g. the column chunks of a B that
 * arrives in pieces (ShardedSpMM.run_pipelined: the SpMM of chunk c overlaps the transfer of chunk c + 1,
 * SURVEY §8(f) f2 iii).  Errors as spmm_run, plus UNSUPPORTED for a bad ldc. */
spmm_status spmm_run_ld(spmm_handle h, const float *B, int64_t K, float *C, int64_t ldc, void *cuda_stream);

/* spmm_run_to through an NVLink-SHARP multicast address (SURVEY §8(f) f2 ii, NVLS): C_mc is the multicast
 * address of a [>= row_offset + M][K] float32 buffer bound on every GPU of the group (e.g. torch symmetric
 * memory's multicast_ptr); every C row this handle computes is stored ONCE, with multimem.st, and the NVSwitch
 * delivers it to the buffer on every member GPU (this one included) -- one store per element instead of one
 * per peer.  Needs K % 8 == 0 and 32-byte aligned B and destination rows (the 256-bit lane geometry).
 * Asynchrony as spmm_run; the caller orders completion across GPUs (e.g. a barrier after the kernels).
 * Errors: INVALID_ARG (NULL, negative row_offset), UNSUPPORTED (K / alignment), STATE, OOM, CUDA. */
spmm_status spmm_run_multicast(spmm_handle h, const float *B, int64_t K, float *C_mc, int64_t row_offset,
                               void *cuda_stream);

/* End-to-end variant: B_host -> device, spmm_run, C -> C_host, all on cuda_stream with handle-owned
 * staging buffers (grown on demand).  Host buffers should be pinned for full copy bandwidth.
 * Synchronises cuda_stream before returning. */
spmm_status spmm_run_host(spmm_handle h, const float *B_host, int64_t K, float *C_host, void *cuda_stream);

/* Pipelined end-to-end variant for a stream of n right-hand sides (serving): for i = 0..n-1, C_host[i] =
 * A . B_host[i] (each B_host[i]: HOST float32 [N][K] row-major, each C_host[i]: HOST float32 [M][K], original
 * row order; all should be pinned so the copies are asynchronous).  Double-buffered handle-owned device
 * slots and two handle-owned copy streams: the H2D of B_{i+1} and the D2H of C_{i-1} overlap the SpMM of step
 * i (PCIe is full duplex), so a step costs about max(H2D, D2H) instead of their sum.  Every step still copies
 * its whole B in and its whole C out.  All work is ordered after what is already queued on cuda_stream; the
 * call synchronises cuda_stream before returning (all C_host[i] complete).  Errors as spmm_run_host (every
 * pair is checked before any work is queued); n = 0 is a no-op. */
spmm_status spmm_run_host_batch(spmm_handle h, int64_t n, const float *const *B_host, int64_t K,
                                float *const *C_host, void *cuda_stream);

/* Predictor inference (§V.B): z = (log1p(f) - mu)/sigma; h1 = relu(W1 z + b1) (64);
 * h2 = relu(W2 h1 + b2) (32); t = W3 h2 + b3 (n_policies predicted times); policy = argmin t, ties to
 * the lowest index.  weights: HOST float32, flat mu[24] sigma[24] W1[64][24] b1[64] W2[32][64] b2[32]
 * W3[P][32] b3[P]; n_weights must equal 48+1536+64+2048+32+33*P.  times_out may be NULL. */
spmm_status spmm_predict(const double features[24], const float *mlp_weights, int64_t n_weights,
                         int32_t n_policies, int32_t *policy_out, double *times_out);

/* The same inference for F input features (e.g. F = 31: the 24 Table II features followed by the 7 B200
 * platform features of spmm_features_b200, f4): weights mu[F] sigma[F] W1[64][F] b1[64] W2[32][64] b2[32]
 * W3[P][32] b3[P]; n_weights must equal 2F + 64F + 64 + 2048 + 32 + 33P.  spmm_predict is spmm_predict_n
 * with F = 24. */
spmm_status spmm_predict_n(const double *features, int32_t n_features, const float *mlp_weights, int64_t n_weights,
                           int32_t n_policies, int32_t *policy_out, double *times_out);

/* Row-sharded mode (north star (4)): bounds[0]=0, bounds[P]=M,
 * bounds[p] = min{ r : rowidx[r] >= ceil(p*nnz/P) }.  rowidx: HOST int64[M+1]; bounds: HOST int64[P+1]. */
spmm_status spmm_partition_by_nnz(const int64_t *rowidx, int64_t M, int32_t P, int64_t *bounds);

/* Release the handle and all its device memory (stream-ordered frees).  Waits for the handle's own runs and
 * copies (their slot events and streams) -- not for other work on the device. */
spmm_status spmm_destroy(spmm_handle h);

const char *spmm_status_string(spmm_status s);
const char *spmm_last_error(void);

/* Number of kernel launches issued by the most recent spmm_run on this thread (bench accounting). */
int32_t spmm_last_run_launches(void);

/* Measurement aid (bench.py's roofline of the dominant kernel): while enabled (enable != 0), every
 * spmm_run on h records two CUDA events on its cuda_stream around the main SpMM kernel (the row-group
 * kernel of a8; the empty-row zero fill and the split-row combine are separate launches outside them).
 * spmm_last_kernel_ms synchronises the second event of the most recent run on h and returns the kernel's
 * duration in milliseconds (0 when that run launched no SpMM kernel or timing is off).  Events are
 * owned by the handle.  Errors: INVALID_ARG (NULL), STATE (wrong device), CUDA. */
spmm_status spmm_set_kernel_timing(spmm_handle h, int enable);
spmm_status spmm_last_kernel_ms(spmm_handle h, float *ms);

#ifdef __cplusplus
}
#endif
#endif /* SPMM_B200_H */
