// internal.cuh -- shared internals of libspmm_b200 (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stddef.h>
#include <atomic>
#include <mutex>
#include <string>
#include <utility>
#include "../../include/spmm.h"

namespace spmm {

// ---- error plumbing -------------------------------------------------------------------------
void set_error(const std::string &msg);
spmm_status fail(spmm_status s, const std::string &msg);
spmm_status cuda_fail(cudaError_t e, const char *what);

#define SPMM_CUDA(call)                                                   \
    do {                                                                  \
        cudaError_t e_ = (call);                                          \
        if (e_ != cudaSuccess) return ::spmm::cuda_fail(e_, #call);       \
    } while (0)
#define SPMM_TRY(call)                                                    \
    do {                                                                  \
        spmm_status s_ = (call);                                          \
        if (s_ != SPMM_OK) return s_;                                     \
    } while (0)

// ---- allocation (optional user hook, else cudaMallocAsync) ------------------------------------
void *dev_alloc(size_t bytes, cudaStream_t s);
void dev_free(void *p, cudaStream_t s);

// RAII device buffer (stream-ordered free)
struct DevBuf {
    void *p = nullptr;
    size_t bytes = 0;
    cudaStream_t s = nullptr;
    DevBuf() = default;
    DevBuf(const DevBuf &) = delete;
    DevBuf &operator=(const DevBuf &) = delete;
    ~DevBuf() { release(); }
    spmm_status alloc(size_t n, cudaStream_t st) {
        release();
        s = st;
        bytes = n;
        if (n == 0) return SPMM_OK;
        p = dev_alloc(n, st);
        if (!p) { bytes = 0; return fail(SPMM_ERR_OOM, "device allocation of " + std::to_string(n) + " bytes failed"); }
        return SPMM_OK;
    }
    void release() {
        if (p) dev_free(p, s);
        p = nullptr;
        bytes = 0;
    }
    void swap(DevBuf &o) {
        std::swap(p, o.p);
        std::swap(bytes, o.bytes);
        std::swap(s, o.s);
    }
    template <class T> T *as() const { return reinterpret_cast<T *>(p); }
};

// ---- the handle -----------------------------------------------------------------------------
// a7 row classes (counts, K-independent; computed by spmm_permute)
struct RowClasses {
    int64_t n_long = 0;       // rows with nnz > split_nnz
    int64_t n_chunks = 0;     // split_nnz-chunks over those rows
};

// a7 run schedule for one lanes-per-row geometry (rows per warp RPW), built by spmm_prepare (or the first
// spmm_run of that geometry) after a permute; up to SCHED_CACHE geometries are kept per permutation.  Warp task t owns units [t*RPW, (t+1)*RPW): either up to RPW consecutive
// non-empty short rows of the permuted order, or RPW consecutive chunks of one long row (a chunk group,
// reduced across the warp into one partial).  Units: int4 (start, len, dst, 0); dst >= 0: C row,
// dst == INT_MIN: padding, dst < 0: chunk group -> partial slot -(dst+1).
// Row fusion (spmm_params.fuse_rows): the short rows of a run are taken R consecutive positions at a time
// (a fusion group); the group's unit walks the sorted UNION of the R rows' columns once, so a B row shared
// by several of them is loaded once and feeds every member's accumulator (each member still accumulates its
// own terms in ascending column order: the rounding of every row is unchanged).  Records: R = 2 -> int4
// (col, mask, v0, v1); R = 4 -> 2 x int4 (col, mask, v0, v1, v2, v3, 0, 0); mask bit r = row r has the column.
// Fused unit: int4 (first record, union length, group id, 1); gdst[group * R + r] = C row of member r.
struct Schedule {
    int32_t rpw = 0;          // 0 = not built
    int32_t fuse_req = 1;     // R the schedule was requested with (1 = none)
    int32_t fuse = 1;         // R actually used (1 = no fused units)
    int64_t n_groups = 0;     // fusion groups
    int64_t n_records = 0;    // union records over all groups
    int64_t fused_nnz = 0;    // nnz of the rows in fusion groups
    DevBuf recs;              // int4[n_records * (R / 2)]
    DevBuf gdst;              // int32[n_groups * R]
    int64_t n_tasks = 0;
    DevBuf units;             // int4[n_tasks * rpw]
    int64_t n_long = 0;
    DevBuf long_dst;          // int32[n_long]      C row of each long row
    DevBuf pslot_ptr;         // int32[n_long + 1]  partial-slot range of each long row
    int64_t n_pslots = 0;
    int64_t n_empty = 0;
    DevBuf empty_dst;         // int32[n_empty]     C rows of empty rows (zero-filled)
    uint64_t built = 0;       // build sequence number (0 = free slot): the oldest slot is rebuilt first
};
constexpr int SCHED_CACHE = 4;

// Per-run scratch (the task counter, split-row partials and the side stream of the empty-row zero fill).  A run
// takes the next of RUN_SLOTS slots round-robin and waits (on its own stream, no host sync) for the slot's
// previous user to finish, so runs on one handle may be issued concurrently from several streams / threads.
struct RunSlot {
    DevBuf counters;          // unsigned[64]: dynamic warp-task counters, one per column tile
    DevBuf partials;          // float[n_pslots * K]: split-row chunk-group partials
    cudaEvent_t done = nullptr;        // recorded on the run's stream after its last launch
    bool used = false;
    cudaStream_t side = nullptr;       // empty-row zero fill (forked from / joined to the run's stream)
    cudaEvent_t fork = nullptr, join = nullptr;
};
constexpr int RUN_SLOTS = 4;

}  // namespace spmm

// Extra C destinations of one spmm_run_to (f2 ii): every C row the run writes is also stored to p[0..n-1]
// (device or peer-mapped pointers, already offset to this shard's first row) -- the all-gather of C fused into
// the SpMM epilogue.  n = 0 for plain runs.
constexpr int SPMM_MAX_CDST = 8;
struct CExtra {
    float4 *p[SPMM_MAX_CDST - 1];
    int32_t n;
    uint32_t mc;          // bit i: p[i] is an NVLS multicast address (stores through multimem.st)
    int32_t skip_main;    // 1: the main C pointer is not written (every row goes to p[0..n-1] only)
};

struct spmm_ctx {
    int device = 0;
    cudaStream_t create_stream = nullptr;
    int64_t M = 0, N = 0, nnz = 0;
    int32_t max_row_nnz = 0;
    int64_t n_empty = 0;
    // original CSR on the device
    spmm::DevBuf rowidx;   // int32[M+1]
    spmm::DevBuf colidx;   // int32[nnz]
    spmm::DevBuf value;    // float[nnz]
    // current permutation and its permuted CSR (internal interleaved layout)
    spmm_policy policy = SPMM_POLICY_IDENTITY;
    spmm_params params{};
    spmm::DevBuf perm;     // int32[M]
    spmm::DevBuf rowptr_p; // int32[M+1]
    spmm::DevBuf cv_p;     // int2[nnz]: (colidx', bits(value'))
    spmm::RowClasses rc;
    spmm::Schedule sched[spmm::SCHED_CACHE];
    uint64_t sched_seq = 0;                 // build counter of the schedule slots
    std::atomic<int> last_sched{-1};        // slot of the most recent run (spmm_get_schedule_info)
    std::mutex mu;                          // schedule builds and run-slot hand-out
    spmm::RunSlot slots[spmm::RUN_SLOTS];
    spmm::RunSlot cap_slot;                 // scratch of runs captured into CUDA graphs (sized by spmm_prepare)
    uint32_t next_slot = 0;
    cudaStream_t aux = nullptr;             // non-blocking stream of host read-backs (no device-wide sync)
    // host-run staging (spmm_run_host: one slot; spmm_run_host_batch: two slots each, double-buffered)
    spmm::DevBuf stage_B, stage_C;
    cudaStream_t cin = nullptr, cout = nullptr;          // spmm_run_host_batch copy streams
    cudaEvent_t ev_start = nullptr, ev_in[2] = {nullptr, nullptr}, ev_comp[2] = {nullptr, nullptr},
                ev_out[2] = {nullptr, nullptr};
    int num_sms = 148;
    // optional kernel timing (spmm_set_kernel_timing): events around the main SpMM kernel of spmm_run
    // (a measurement aid: the events belong to the handle, so timed runs must not overlap)
    int timing = 0;
    bool timed = false;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    ~spmm_ctx() {
        if (aux) cudaStreamDestroy(aux);
    }
};

namespace spmm {

// kernels / device algorithms (defined in the .cu files)
spmm_status exclusive_scan_i32(const int32_t *in, int32_t *out, int64_t n, int32_t *total_host,
                               cudaStream_t s);   // out[n] = total when out has n+1 slots
spmm_status exclusive_scan_i64(const int64_t *in, int64_t *out, int64_t n, cudaStream_t s);
spmm_status reduce_max_i32(const int32_t *in, int64_t n, int32_t *result_host, cudaStream_t s);
spmm_status radix_sort_pairs(uint64_t *keys, uint32_t *vals, int64_t n, int begin_bit, int end_bit,
                             cudaStream_t s);     // stable, ascending, in place (uses scratch)

// permutation `policy` into perm (int32[M]); the permuted CSR of perm into rowptr_p / cv_p and its row classes
// (the handle's current permutation is untouched: spmm_permute swaps the results in only on success)
spmm_status build_permutation(spmm_ctx *h, spmm_policy policy, const spmm_params &p, DevBuf &perm, cudaStream_t s);
spmm_status build_permuted_csr(spmm_ctx *h, int32_t split, const DevBuf &perm, DevBuf &rowptr_p, DevBuf &cv_p,
                               RowClasses &rc, cudaStream_t s);
// a7 schedule for the K geometry (built if no cached slot matches; synchronises s when it builds)
spmm_status prepare_schedule(spmm_ctx *h, int64_t K, const float *B, const float *C, cudaStream_t s);
spmm_status compute_features(spmm_ctx *h, bool current_order, const spmm_params &p, double out[24],
                             cudaStream_t s);
spmm_status compute_features_b200(spmm_ctx *h, bool current_order, int64_t K, double out[7], cudaStream_t s);
spmm_status launch_spmm(spmm_ctx *h, const float *B, int64_t K, float *C, int64_t ldc, cudaStream_t s,
                        int32_t *launches, const CExtra &cx);
void release_run_slots(spmm_ctx *h);   // waits for the slots' last runs, frees their scratch and streams

// signatures of the rows (sorted unique col/bw), used by chains and features
struct Signatures {
    DevBuf ptr;   // int32[M+1]
    DevBuf blk;   // int32[S]
    int64_t S = 0;
};
spmm_status build_signatures(const int32_t *rowidx, const int32_t *colidx, const int32_t *order, int64_t M,
                             int64_t nnz, int32_t bw, Signatures &sig, cudaStream_t s);

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

}  // namespace spmm
