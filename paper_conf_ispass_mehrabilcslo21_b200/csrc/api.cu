// api.cu -- the C ABI of include/spmm.h: argument checking, CSR ingest + validation (a1), handle
// lifetime, dispatch to the permutation builders, the SpMM launch, features and the predictor.
#include "internal.cuh"
#include <nvtx3/nvToolsExt.h>
#include <algorithm>
#include <cmath>
#include <cstring>
#include <memory>
#include <mutex>
#include <new>
#include <vector>

namespace spmm {

// NVTX range per C-ABI call (SURVEY §5 tracing: phases show up by name in nsys / ncu timelines; a no-op without a
// tool attached -- NVTX v3 is header-only and binds to an injection library only when one is loaded)
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

static thread_local std::string g_last_error;
static thread_local int32_t g_last_launches = 0;

void set_error(const std::string &msg) { g_last_error = msg; }
spmm_status fail(spmm_status s, const std::string &msg) {
    g_last_error = msg;
    return s;
}
spmm_status cuda_fail(cudaError_t e, const char *what) {
    g_last_error = std::string(what) + ": " + cudaGetErrorString(e);
    return (e == cudaErrorMemoryAllocation) ? SPMM_ERR_OOM : SPMM_ERR_CUDA;
}

// ---- allocator ------------------------------------------------------------------------------
static void *(*g_alloc)(size_t, void *, void *) = nullptr;
static void (*g_free)(void *, void *, void *) = nullptr;
static void *g_alloc_ctx = nullptr;

void *dev_alloc(size_t bytes, cudaStream_t s) {
    if (g_alloc) return g_alloc(bytes, (void *)s, g_alloc_ctx);
    void *p = nullptr;
    if (cudaMallocAsync(&p, bytes, s) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return p;
}
void dev_free(void *p, cudaStream_t s) {
    if (!p) return;
    if (g_free) { g_free(p, (void *)s, g_alloc_ctx); return; }
    cudaFreeAsync(p, s);
}

namespace {

// a1: rowidx int64 -> int32 with checks (rowidx[0]=0, rowidx[M]=nnz, non-decreasing)
__global__ void k_ingest_rowidx(const int64_t *r64, int64_t M, int64_t nnz, int32_t *r32, int *err) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= M; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t v = r64[i];
        if ((i == 0 && v != 0) || (i == M && v != nnz) || v < 0 || v > nnz || (i > 0 && r64[i - 1] > v))
            atomicOr(err, 1);
        r32[i] = (int32_t)v;
    }
}
// columns in range and strictly increasing within each row (warp per row)
__global__ void k_check_cols(const int32_t *rowidx, const int32_t *colidx, int64_t M, int64_t N, int *err) {
    const int lane = threadIdx.x & 31;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < M;
         i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        int32_t a = rowidx[i], b = rowidx[i + 1];
        bool bad = false;
        for (int32_t j = a + lane; j < b; j += 32) {
            int32_t c = colidx[j];
            bad |= c < 0 || (int64_t)c >= N || (j > a && colidx[j - 1] >= c);
        }
        if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(err, 2);
    }
}
__global__ void k_row_len_stats(const int32_t *rowidx, int64_t M, int32_t *maxlen, unsigned long long *empty) {
    int32_t m = 0;
    unsigned long long e = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
        int32_t l = rowidx[i + 1] - rowidx[i];
        m = max(m, l);
        e += (l == 0);
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
        e += __shfl_xor_sync(0xffffffffu, e, o);
    }
    if ((threadIdx.x & 31) == 0) { atomicMax(maxlen, m); atomicAdd(empty, e); }
}

// a caller-supplied permutation must be a bijection on [0, M): every value in range and seen exactly once
__global__ void k_check_perm(const int32_t *perm, int64_t M, unsigned int *seen, int *err) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        const int32_t r = perm[p];
        if (r < 0 || (int64_t)r >= M) { atomicOr(err, 1); continue; }
        if (atomicAdd(seen + r, 1u) != 0u) atomicOr(err, 2);
    }
}

// drop every cached run schedule (they describe the previous permutation) and free their arrays; the caller has
// waited for the handle's runs in flight
void clear_schedules(spmm_ctx *h) {
    for (int i = 0; i < SCHED_CACHE; ++i) {
        Schedule &S = h->sched[i];
        S.built = 0;
        S.rpw = 0;
        S.recs.release();
        S.gdst.release();
        S.units.release();
        S.long_dst.release();
        S.pslot_ptr.release();
        S.empty_dst.release();
    }
    h->last_sched.store(-1);
}

unsigned grid1d(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 32)); }

spmm_status check_device(spmm_ctx *h) {
    int d = -1;
    SPMM_CUDA(cudaGetDevice(&d));
    if (d != h->device) return fail(SPMM_ERR_STATE, "handle created on device " + std::to_string(h->device) +
                                                         " used on device " + std::to_string(d));
    return SPMM_OK;
}

spmm_status check_params(const spmm_params &p) {
    if (p.nw <= 0 || p.nw > 1024 || p.nt <= 0 || p.bw <= 0 || p.split_nnz < 1 || p.window < 0 ||
        (p.window % p.nw) != 0 || (p.preorder < 0 || p.preorder > 2) || p.fuse_rows < 0 || p.fuse_rows > 2)
        return fail(SPMM_ERR_INVALID_ARG, "invalid spmm_params (nw/nt/bw > 0, nw <= 1024, split_nnz >= 1, "
                                          "window >= 0 and a multiple of nw, preorder in {0,1,2}, fuse_rows in {0,1,2})");
    return SPMM_OK;
}

spmm_status do_create(spmm_handle *out, int64_t M, int64_t N, int64_t nnz, const int64_t *rowidx,
                      const int32_t *colidx, const float *value, int on_device, cudaStream_t s) {
    if (!out) return fail(SPMM_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (M < 0 || N < 0 || nnz < 0) return fail(SPMM_ERR_INVALID_ARG, "negative size");
    if (M >= ((int64_t)1 << 31) || N >= ((int64_t)1 << 31) || nnz >= ((int64_t)1 << 31))
        return fail(SPMM_ERR_INVALID_ARG, "M, N and nnz must be < 2^31");
    if (!rowidx || (nnz > 0 && (!colidx || !value))) return fail(SPMM_ERR_INVALID_ARG, "NULL CSR array");
    auto *h = new (std::nothrow) spmm_ctx();
    if (!h) return fail(SPMM_ERR_OOM, "host allocation failed");
    std::unique_ptr<spmm_ctx> guard(h);
    SPMM_CUDA(cudaGetDevice(&h->device));
    SPMM_CUDA(cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, h->device));
    h->create_stream = s;
    SPMM_CUDA(cudaStreamCreateWithFlags(&h->aux, cudaStreamNonBlocking));
    h->M = M; h->N = N; h->nnz = nnz;
    spmm_default_params(&h->params);
    const cudaMemcpyKind kind = on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    DevBuf r64, flags;
    SPMM_TRY(r64.alloc((M + 1) * sizeof(int64_t), s));
    SPMM_TRY(flags.alloc(sizeof(int) + sizeof(int32_t) + sizeof(unsigned long long) + 8, s));
    SPMM_TRY(h->rowidx.alloc((M + 1) * sizeof(int32_t), s));
    SPMM_TRY(h->colidx.alloc(std::max<int64_t>(nnz, 1) * sizeof(int32_t), s));
    SPMM_TRY(h->value.alloc(std::max<int64_t>(nnz, 1) * sizeof(float), s));
    SPMM_CUDA(cudaMemcpyAsync(r64.p, rowidx, (M + 1) * sizeof(int64_t), kind, s));
    if (nnz > 0) {
        SPMM_CUDA(cudaMemcpyAsync(h->colidx.p, colidx, nnz * sizeof(int32_t), kind, s));
        SPMM_CUDA(cudaMemcpyAsync(h->value.p, value, nnz * sizeof(float), kind, s));
    }
    SPMM_CUDA(cudaMemsetAsync(flags.p, 0, flags.bytes, s));
    int *err = flags.as<int>();
    int32_t *maxlen = reinterpret_cast<int32_t *>(flags.as<char>() + 8);
    unsigned long long *nempty = reinterpret_cast<unsigned long long *>(flags.as<char>() + 16);
    k_ingest_rowidx<<<grid1d(M + 1), 256, 0, s>>>(r64.as<int64_t>(), M, nnz, h->rowidx.as<int32_t>(), err);
    SPMM_CUDA(cudaGetLastError());
    int herr = 0;
    SPMM_CUDA(cudaMemcpyAsync(&herr, err, sizeof(int), cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    if (herr) return fail(SPMM_ERR_INVALID_CSR, "invalid rowidx (rowidx[0] != 0, rowidx[M] != nnz or decreasing)");
    if (M > 0) {
        k_check_cols<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(M * 32, 256), 148 * 64)), 256, 0, s>>>(
            h->rowidx.as<int32_t>(), h->colidx.as<int32_t>(), M, N, err);
        k_row_len_stats<<<grid1d(M), 256, 0, s>>>(h->rowidx.as<int32_t>(), M, maxlen, nempty);
        SPMM_CUDA(cudaGetLastError());
    }
    unsigned long long ne = 0;
    SPMM_CUDA(cudaMemcpyAsync(&herr, err, sizeof(int), cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaMemcpyAsync(&h->max_row_nnz, maxlen, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaMemcpyAsync(&ne, nempty, sizeof(ne), cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    if (herr) return fail(SPMM_ERR_INVALID_CSR, "invalid colidx (out of [0,N) or not strictly increasing in a row)");
    h->n_empty = (int64_t)ne;
    r64.release();
    flags.release();
    // current policy: IDENTITY
    h->policy = SPMM_POLICY_IDENTITY;
    SPMM_TRY(build_permutation(h, SPMM_POLICY_IDENTITY, h->params, h->perm, s));
    SPMM_TRY(build_permuted_csr(h, h->params.split_nnz, h->perm, h->rowptr_p, h->cv_p, h->rc, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    *out = guard.release();
    return SPMM_OK;
}

}  // namespace
}  // namespace spmm

using namespace spmm;

extern "C" {

spmm_status spmm_default_params(spmm_params *p) {
    if (!p) return fail(SPMM_ERR_INVALID_ARG, "params is NULL");
    std::memset(p, 0, sizeof(*p));
    p->nw = 32;
    p->nt = 32;
    p->bw = 32;
    p->split_nnz = 128;
    p->window = 1024;
    p->preorder = 0;
    p->seed = 0;
    return SPMM_OK;
}

spmm_status spmm_set_allocator(void *(*alloc)(size_t, void *, void *), void (*free_)(void *, void *, void *),
                               void *ctx) {
    if ((alloc == nullptr) != (free_ == nullptr)) return fail(SPMM_ERR_INVALID_ARG, "alloc and free must both be set");
    g_alloc = alloc;
    g_free = free_;
    g_alloc_ctx = ctx;
    return SPMM_OK;
}

spmm_status spmm_create(spmm_handle *out, int64_t M, int64_t N, int64_t nnz, const int64_t *rowidx,
                        const int32_t *colidx, const float *value, int inputs_on_device, void *cuda_stream) {
    NvtxRange nvtx_("spmm_create");
    try {
        return do_create(out, M, N, nnz, rowidx, colidx, value, inputs_on_device, (cudaStream_t)cuda_stream);
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
}

spmm_status spmm_permute(spmm_handle h, spmm_policy policy, const spmm_params *params, void *cuda_stream) {
    NvtxRange nvtx_("spmm_permute");
    if (!h) return fail(SPMM_ERR_INVALID_ARG, "handle is NULL");
    if ((int)policy < 0 || (int)policy >= SPMM_POLICY_COUNT) return fail(SPMM_ERR_INVALID_ARG, "unknown policy");
    SPMM_TRY(check_device(h));
    spmm_params p;
    if (params) p = *params; else spmm_default_params(&p);
    SPMM_TRY(check_params(p));
    cudaStream_t s = (cudaStream_t)cuda_stream;
    try {
        // build into temporaries; the handle keeps its current permutation, permuted CSR and schedules unless
        // every step succeeds (a failed permute -- e.g. SPMM_ERR_OOM -- leaves a usable handle)
        DevBuf perm, rowptr_p, cv_p;
        RowClasses rc;
        SPMM_TRY(build_permutation(h, policy, p, perm, s));
        SPMM_TRY(build_permuted_csr(h, p.split_nnz, perm, rowptr_p, cv_p, rc, s));
        SPMM_CUDA(cudaStreamSynchronize(s));
        std::lock_guard<std::mutex> lk(h->mu);
        for (int i = 0; i < RUN_SLOTS; ++i)        // runs still in flight read the old arrays
            if (h->slots[i].used) SPMM_CUDA(cudaEventSynchronize(h->slots[i].done));
        h->perm.swap(perm);
        h->rowptr_p.swap(rowptr_p);
        h->cv_p.swap(cv_p);
        h->rc = rc;
        h->params = p;
        h->policy = policy;
        clear_schedules(h);
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
    return SPMM_OK;
}

spmm_status spmm_set_perm(spmm_handle h, const int32_t *perm_in, const spmm_params *params, void *cuda_stream) {
    NvtxRange nvtx_("spmm_set_perm");
    if (!h || (!perm_in && h->M > 0)) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    SPMM_TRY(check_device(h));
    spmm_params p;
    if (params) p = *params; else spmm_default_params(&p);
    SPMM_TRY(check_params(p));
    cudaStream_t s = (cudaStream_t)cuda_stream;
    const int64_t M = h->M;
    try {
        DevBuf perm, rowptr_p, cv_p, seen, flag;
        RowClasses rc;
        SPMM_TRY(perm.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
        if (M > 0) {
            SPMM_TRY(seen.alloc(M * sizeof(unsigned int), s));
            SPMM_TRY(flag.alloc(sizeof(int), s));
            SPMM_CUDA(cudaMemcpyAsync(perm.p, perm_in, M * sizeof(int32_t), cudaMemcpyHostToDevice, s));
            SPMM_CUDA(cudaMemsetAsync(seen.p, 0, M * sizeof(unsigned int), s));
            SPMM_CUDA(cudaMemsetAsync(flag.p, 0, sizeof(int), s));
            k_check_perm<<<grid1d(M), 256, 0, s>>>(perm.as<int32_t>(), M, seen.as<unsigned int>(), flag.as<int>());
            SPMM_CUDA(cudaGetLastError());
            int herr = 0;
            SPMM_CUDA(cudaMemcpyAsync(&herr, flag.p, sizeof(int), cudaMemcpyDeviceToHost, s));
            SPMM_CUDA(cudaStreamSynchronize(s));
            if (herr) return fail(SPMM_ERR_INVALID_ARG, "perm is not a bijection on [0, M)");
        }
        SPMM_TRY(build_permuted_csr(h, p.split_nnz, perm, rowptr_p, cv_p, rc, s));
        SPMM_CUDA(cudaStreamSynchronize(s));
        std::lock_guard<std::mutex> lk(h->mu);
        for (int i = 0; i < RUN_SLOTS; ++i)
            if (h->slots[i].used) SPMM_CUDA(cudaEventSynchronize(h->slots[i].done));
        h->perm.swap(perm);
        h->rowptr_p.swap(rowptr_p);
        h->cv_p.swap(cv_p);
        h->rc = rc;
        h->params = p;
        h->policy = SPMM_POLICY_COUNT;      // a caller-supplied order (no builder)
        clear_schedules(h);
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
    return SPMM_OK;
}

spmm_status spmm_get_perm(spmm_handle h, int32_t *perm_out) {
    NvtxRange nvtx_("spmm_get_perm");
    if (!h || (!perm_out && h->M > 0)) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    SPMM_TRY(check_device(h));
    if (h->M == 0) return SPMM_OK;
    // the permutation is complete (spmm_create / spmm_permute synchronise their stream); read it back on the
    // handle's own non-blocking stream -- no device-wide synchronisation
    SPMM_CUDA(cudaMemcpyAsync(perm_out, h->perm.p, h->M * sizeof(int32_t), cudaMemcpyDeviceToHost, h->aux));
    SPMM_CUDA(cudaStreamSynchronize(h->aux));
    return SPMM_OK;
}

spmm_status spmm_get_permuted_csr(spmm_handle h, int64_t *rowidx, int32_t *colidx, float *value) {
    NvtxRange nvtx_("spmm_get_permuted_csr");
    if (!h || !rowidx || (h->nnz > 0 && (!colidx || !value))) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    SPMM_TRY(check_device(h));
    std::vector<int32_t> r32(h->M + 1);
    SPMM_CUDA(cudaMemcpyAsync(r32.data(), h->rowptr_p.p, (h->M + 1) * sizeof(int32_t), cudaMemcpyDeviceToHost, h->aux));
    SPMM_CUDA(cudaStreamSynchronize(h->aux));
    for (int64_t i = 0; i <= h->M; ++i) rowidx[i] = r32[i];
    if (h->nnz > 0) {
        std::vector<int2> cv(h->nnz);
        SPMM_CUDA(cudaMemcpyAsync(cv.data(), h->cv_p.p, h->nnz * sizeof(int2), cudaMemcpyDeviceToHost, h->aux));
        SPMM_CUDA(cudaStreamSynchronize(h->aux));
        for (int64_t j = 0; j < h->nnz; ++j) {
            colidx[j] = cv[j].x;
            std::memcpy(&value[j], &cv[j].y, sizeof(float));
        }
    }
    return SPMM_OK;
}

spmm_status spmm_get_info(spmm_handle h, int64_t out[5]) {
    if (!h || !out) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    out[0] = h->n_empty;
    out[1] = h->M - h->n_empty - h->rc.n_long;
    out[2] = h->rc.n_long;
    out[3] = h->rc.n_chunks;
    out[4] = h->max_row_nnz;
    return SPMM_OK;
}

spmm_status spmm_get_schedule_info(spmm_handle h, int64_t out[6]) {
    if (!h || !out) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    const int i = h->last_sched.load();
    const bool ok = i >= 0 && h->sched[i].built;
    const Schedule &S = h->sched[ok ? i : 0];
    out[0] = ok ? S.rpw : 0;
    out[1] = ok ? S.fuse : 1;
    out[2] = ok ? S.n_tasks : 0;
    out[3] = ok ? S.n_groups : 0;
    out[4] = ok ? S.n_records : 0;
    out[5] = ok ? S.fused_nnz : 0;
    return SPMM_OK;
}

spmm_status spmm_features(spmm_handle h, int use_current_order, const spmm_params *params, double out[24],
                          void *cuda_stream) {
    NvtxRange nvtx_("spmm_features");
    if (!h || !out) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    SPMM_TRY(check_device(h));
    spmm_params p;
    if (params) p = *params; else spmm_default_params(&p);
    SPMM_TRY(check_params(p));
    try {
        return compute_features(h, use_current_order != 0, p, out, (cudaStream_t)cuda_stream);
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
}

spmm_status spmm_features_b200(spmm_handle h, int use_current_order, int64_t K, double out[7], void *cuda_stream) {
    NvtxRange nvtx_("spmm_features_b200");
    if (!h || !out) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    if (K <= 0) return fail(SPMM_ERR_INVALID_ARG, "K must be positive");
    SPMM_TRY(check_device(h));
    try {
        return compute_features_b200(h, use_current_order != 0, K, out, (cudaStream_t)cuda_stream);
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
}

static spmm_status check_run_args(spmm_handle h, const void *B, int64_t K, const void *C, bool device) {
    if (!h || (h->M > 0 && !C) || (h->N > 0 && h->nnz > 0 && !B)) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    if (K <= 0) return fail(SPMM_ERR_INVALID_ARG, "K must be positive");
    if (K % 4 != 0 || K > 1024) return fail(SPMM_ERR_UNSUPPORTED, "K must be a multiple of 4 and <= 1024");
    if (device && ((reinterpret_cast<uintptr_t>(B) | reinterpret_cast<uintptr_t>(C)) & 15u))
        return fail(SPMM_ERR_UNSUPPORTED, "B and C must be 16-byte aligned");
    return SPMM_OK;
}

spmm_status spmm_run(spmm_handle h, const float *B, int64_t K, float *C, void *cuda_stream) {
    NvtxRange nvtx_("spmm_run");
    g_last_launches = 0;
    SPMM_TRY(check_run_args(h, B, K, C, true));
    SPMM_TRY(check_device(h));
    try {
        return launch_spmm(h, B, K, C, K, (cudaStream_t)cuda_stream, &g_last_launches, CExtra{});
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
}

spmm_status spmm_prepare(spmm_handle h, int64_t K, const float *B, const float *C, void *cuda_stream) {
    NvtxRange nvtx_("spmm_prepare");
    if (!h) return fail(SPMM_ERR_INVALID_ARG, "handle is NULL");
    if (K <= 0) return fail(SPMM_ERR_INVALID_ARG, "K must be positive");
    if (K % 4 != 0 || K > 1024) return fail(SPMM_ERR_UNSUPPORTED, "K must be a multiple of 4 and <= 1024");
    SPMM_TRY(check_device(h));
    if (h->M == 0) return SPMM_OK;
    // B / C only decide the lane geometry (32-byte alignment); NULL = the aligned (256-bit load) geometry
    static const float kAligned[8] __attribute__((aligned(32))) = {0};
    try {
        return prepare_schedule(h, K, B ? B : kAligned, C ? C : kAligned, (cudaStream_t)cuda_stream);
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
}

spmm_status spmm_run_to(spmm_handle h, const float *B, int64_t K, float *const *C_dsts, int32_t n_dsts,
                        int64_t row_offset, void *cuda_stream) {
    NvtxRange nvtx_("spmm_run_to");
    g_last_launches = 0;
    if (!h || !C_dsts) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    if (n_dsts < 1 || n_dsts > SPMM_MAX_CDST) return fail(SPMM_ERR_INVALID_ARG, "n_dsts must be in [1, 8]");
    if (row_offset < 0) return fail(SPMM_ERR_INVALID_ARG, "negative row_offset");
    for (int32_t i = 0; i < n_dsts; ++i) {
        SPMM_TRY(check_run_args(h, B, K, C_dsts[i], true));
        if (((uintptr_t)(C_dsts[i] + row_offset * K)) & 15u)
            return fail(SPMM_ERR_UNSUPPORTED, "destination rows must be 16-byte aligned");
    }
    SPMM_TRY(check_device(h));
    CExtra cx{};
    cx.n = n_dsts - 1;
    for (int32_t i = 1; i < n_dsts; ++i) cx.p[i - 1] = reinterpret_cast<float4 *>(C_dsts[i] + row_offset * K);
    try {
        return launch_spmm(h, B, K, C_dsts[0] + row_offset * K, K, (cudaStream_t)cuda_stream, &g_last_launches, cx);
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
}

spmm_status spmm_run_ld(spmm_handle h, const float *B, int64_t K, float *C, int64_t ldc, void *cuda_stream) {
    NvtxRange nvtx_("spmm_run_ld");
    g_last_launches = 0;
    SPMM_TRY(check_run_args(h, B, K, C, true));
    if (ldc < K || ldc % 4 != 0) return fail(SPMM_ERR_UNSUPPORTED, "ldc must be >= K and a multiple of 4");
    SPMM_TRY(check_device(h));
    try {
        return launch_spmm(h, B, K, C, ldc, (cudaStream_t)cuda_stream, &g_last_launches, CExtra{});
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
}

spmm_status spmm_run_multicast(spmm_handle h, const float *B, int64_t K, float *C_mc, int64_t row_offset,
                               void *cuda_stream) {
    NvtxRange nvtx_("spmm_run_multicast");
    g_last_launches = 0;
    if (!h || !C_mc) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    if (row_offset < 0) return fail(SPMM_ERR_INVALID_ARG, "negative row_offset");
    SPMM_TRY(check_run_args(h, B, K, C_mc, true));
    float *dst = C_mc + row_offset * K;
    if (K % 8 != 0 || (((uintptr_t)B | (uintptr_t)dst) & 31u))
        return fail(SPMM_ERR_UNSUPPORTED, "multicast stores need K % 8 == 0 and 32-byte aligned B and C rows");
    SPMM_TRY(check_device(h));
    CExtra cx{};
    cx.n = 1;
    cx.p[0] = reinterpret_cast<float4 *>(dst);
    cx.mc = 1u;
    cx.skip_main = 1;     // the multicast store also reaches this GPU's buffer: no second local store
    try {
        return launch_spmm(h, B, K, dst, K, (cudaStream_t)cuda_stream, &g_last_launches, cx);
    } catch (const std::exception &e) {
        return fail(SPMM_ERR_OOM, e.what());
    }
}

spmm_status spmm_run_host(spmm_handle h, const float *B_host, int64_t K, float *C_host, void *cuda_stream) {
    NvtxRange nvtx_("spmm_run_host");
    g_last_launches = 0;
    SPMM_TRY(check_run_args(h, B_host, K, C_host, false));
    SPMM_TRY(check_device(h));
    cudaStream_t s = (cudaStream_t)cuda_stream;
    const size_t bB = (size_t)h->N * K * sizeof(float), bC = (size_t)h->M * K * sizeof(float);
    if (h->stage_B.bytes < bB) SPMM_TRY(h->stage_B.alloc(bB, s));
    if (h->stage_C.bytes < bC) SPMM_TRY(h->stage_C.alloc(bC, s));
    if (bB) SPMM_CUDA(cudaMemcpyAsync(h->stage_B.p, B_host, bB, cudaMemcpyHostToDevice, s));
    SPMM_TRY(launch_spmm(h, h->stage_B.as<float>(), K, h->stage_C.as<float>(), K, s, &g_last_launches, CExtra{}));
    if (bC) SPMM_CUDA(cudaMemcpyAsync(C_host, h->stage_C.p, bC, cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    return SPMM_OK;
}

spmm_status spmm_run_host_batch(spmm_handle h, int64_t n, const float *const *B_host, int64_t K,
                                float *const *C_host, void *cuda_stream) {
    NvtxRange nvtx_("spmm_run_host_batch");
    g_last_launches = 0;
    if (!h || n < 0 || (n > 0 && (!B_host || !C_host))) return fail(SPMM_ERR_INVALID_ARG, "NULL argument or n < 0");
    for (int64_t i = 0; i < n; ++i) SPMM_TRY(check_run_args(h, B_host[i], K, C_host[i], false));
    SPMM_TRY(check_device(h));
    if (n == 0) return SPMM_OK;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    const size_t bB = (size_t)h->N * K * sizeof(float), bC = (size_t)h->M * K * sizeof(float);
    // two slots each: step i uses slot i & 1 (B rows padded to 256 B so both slots stay 32-byte aligned)
    const size_t sB = (bB + 255) / 256 * 256, sC = (bC + 255) / 256 * 256;
    if (h->stage_B.bytes < 2 * sB) SPMM_TRY(h->stage_B.alloc(2 * sB, s));
    if (h->stage_C.bytes < 2 * sC) SPMM_TRY(h->stage_C.alloc(2 * sC, s));
    if (!h->cin) {
        SPMM_CUDA(cudaStreamCreateWithFlags(&h->cin, cudaStreamNonBlocking));
        SPMM_CUDA(cudaStreamCreateWithFlags(&h->cout, cudaStreamNonBlocking));
        SPMM_CUDA(cudaEventCreateWithFlags(&h->ev_start, cudaEventDisableTiming));
        for (int k = 0; k < 2; ++k) {
            SPMM_CUDA(cudaEventCreateWithFlags(&h->ev_in[k], cudaEventDisableTiming));
            SPMM_CUDA(cudaEventCreateWithFlags(&h->ev_comp[k], cudaEventDisableTiming));
            SPMM_CUDA(cudaEventCreateWithFlags(&h->ev_out[k], cudaEventDisableTiming));
        }
    }
    // everything below is ordered after the work already queued on s
    SPMM_CUDA(cudaEventRecord(h->ev_start, s));
    SPMM_CUDA(cudaStreamWaitEvent(h->cin, h->ev_start, 0));
    SPMM_CUDA(cudaStreamWaitEvent(h->cout, h->ev_start, 0));
    int32_t launches = 0;
    for (int64_t i = 0; i < n; ++i) {
        const int k = (int)(i & 1);
        float *Bs = reinterpret_cast<float *>(h->stage_B.as<char>() + k * sB);
        float *Cs = reinterpret_cast<float *>(h->stage_C.as<char>() + k * sC);
        // H2D of B_i once step i-2 (same slot) has finished reading it
        if (i >= 2) SPMM_CUDA(cudaStreamWaitEvent(h->cin, h->ev_comp[k], 0));
        if (bB) SPMM_CUDA(cudaMemcpyAsync(Bs, B_host[i], bB, cudaMemcpyHostToDevice, h->cin));
        SPMM_CUDA(cudaEventRecord(h->ev_in[k], h->cin));
        // SpMM i once B_i is in and the D2H of step i-2 has drained the C slot
        SPMM_CUDA(cudaStreamWaitEvent(s, h->ev_in[k], 0));
        if (i >= 2) SPMM_CUDA(cudaStreamWaitEvent(s, h->ev_out[k], 0));
        int32_t l = 0;
        SPMM_TRY(launch_spmm(h, Bs, K, Cs, K, s, &l, CExtra{}));
        launches += l;
        SPMM_CUDA(cudaEventRecord(h->ev_comp[k], s));
        // D2H of C_i (overlaps the H2D of B_{i+1}: PCIe is full duplex)
        SPMM_CUDA(cudaStreamWaitEvent(h->cout, h->ev_comp[k], 0));
        if (bC) SPMM_CUDA(cudaMemcpyAsync(C_host[i], Cs, bC, cudaMemcpyDeviceToHost, h->cout));
        SPMM_CUDA(cudaEventRecord(h->ev_out[k], h->cout));
    }
    for (int k = 0; k < 2 && k < n; ++k) SPMM_CUDA(cudaStreamWaitEvent(s, h->ev_out[k], 0));
    SPMM_CUDA(cudaStreamSynchronize(s));
    g_last_launches = launches;
    return SPMM_OK;
}

spmm_status spmm_predict_n(const double *features, int32_t F, const float *w, int64_t n_weights, int32_t P,
                           int32_t *policy_out, double *times_out) {
    if (!features || !w || !policy_out || P <= 0 || F <= 0) return fail(SPMM_ERR_INVALID_ARG, "NULL argument, P <= 0 or F <= 0");
    if (n_weights != 2 * (int64_t)F + 64 * (int64_t)F + 64 + 32 * 64 + 32 + 33 * (int64_t)P)
        return fail(SPMM_ERR_INVALID_ARG, "n_weights does not match the F-64-32-P layout");
    const float *mu = w, *sg = w + F, *W1 = w + 2 * F, *b1 = W1 + 64 * (int64_t)F, *W2 = b1 + 64, *b2 = W2 + 32 * 64,
                *W3 = b2 + 32, *b3 = W3 + (int64_t)P * 32;
    std::vector<double> z(F);
    double h1[64], h2[32];
    for (int i = 0; i < F; ++i) z[i] = (std::log1p(features[i]) - (double)mu[i]) / (double)sg[i];
    for (int o = 0; o < 64; ++o) {
        double s = b1[o];
        for (int i = 0; i < F; ++i) s += (double)W1[(int64_t)o * F + i] * z[i];
        h1[o] = s > 0 ? s : 0;
    }
    for (int o = 0; o < 32; ++o) {
        double s = b2[o];
        for (int i = 0; i < 64; ++i) s += (double)W2[o * 64 + i] * h1[i];
        h2[o] = s > 0 ? s : 0;
    }
    int32_t best = 0;
    double bestv = 0;
    for (int o = 0; o < P; ++o) {
        double s = b3[o];
        for (int i = 0; i < 32; ++i) s += (double)W3[o * 32 + i] * h2[i];
        if (times_out) times_out[o] = s;
        if (o == 0 || s < bestv) { best = o; bestv = s; }
    }
    *policy_out = best;
    return SPMM_OK;
}

spmm_status spmm_predict(const double features[24], const float *w, int64_t n_weights, int32_t P, int32_t *policy_out,
                         double *times_out) {
    return spmm_predict_n(features, 24, w, n_weights, P, policy_out, times_out);
}

spmm_status spmm_partition_by_nnz(const int64_t *rowidx, int64_t M, int32_t P, int64_t *bounds) {
    if (!rowidx || !bounds || M < 0 || P <= 0) return fail(SPMM_ERR_INVALID_ARG, "invalid partition arguments");
    const int64_t nnz = rowidx[M];
    bounds[0] = 0;
    for (int32_t p = 1; p < P; ++p) {
        const int64_t target = (p * nnz + P - 1) / P;
        bounds[p] = std::lower_bound(rowidx, rowidx + M + 1, target) - rowidx;   // first r with rowidx[r] >= target
    }
    bounds[P] = M;
    return SPMM_OK;
}

spmm_status spmm_destroy(spmm_handle h) {
    NvtxRange nvtx_("spmm_destroy");
    if (!h) return SPMM_OK;
    // wait for this handle's own work only (its runs' slot events, its copy streams), not the whole device
    release_run_slots(h);
    if (h->cin) cudaStreamSynchronize(h->cin);
    if (h->cout) cudaStreamSynchronize(h->cout);
    if (h->aux) cudaStreamSynchronize(h->aux);   // (destroyed with the handle)
    if (h->ev0) cudaEventDestroy(h->ev0);
    if (h->ev1) cudaEventDestroy(h->ev1);
    if (h->ev_start) cudaEventDestroy(h->ev_start);
    for (int k = 0; k < 2; ++k) {
        if (h->ev_in[k]) cudaEventDestroy(h->ev_in[k]);
        if (h->ev_comp[k]) cudaEventDestroy(h->ev_comp[k]);
        if (h->ev_out[k]) cudaEventDestroy(h->ev_out[k]);
    }
    if (h->cin) cudaStreamDestroy(h->cin);
    if (h->cout) cudaStreamDestroy(h->cout);
    delete h;
    return SPMM_OK;
}

const char *spmm_status_string(spmm_status s) {
    switch (s) {
        case SPMM_OK: return "SPMM_OK";
        case SPMM_ERR_INVALID_ARG: return "SPMM_ERR_INVALID_ARG";
        case SPMM_ERR_INVALID_CSR: return "SPMM_ERR_INVALID_CSR";
        case SPMM_ERR_UNSUPPORTED: return "SPMM_ERR_UNSUPPORTED";
        case SPMM_ERR_CUDA: return "SPMM_ERR_CUDA";
        case SPMM_ERR_OOM: return "SPMM_ERR_OOM";
        case SPMM_ERR_STATE: return "SPMM_ERR_STATE";
        default: return "SPMM_ERR_UNKNOWN";
    }
}

const char *spmm_last_error(void) { return g_last_error.c_str(); }

int32_t spmm_last_run_launches(void) { return g_last_launches; }

spmm_status spmm_set_kernel_timing(spmm_handle h, int enable) {
    if (!h) return fail(SPMM_ERR_INVALID_ARG, "handle is NULL");
    SPMM_TRY(check_device(h));
    if (enable && !h->ev0) {
        SPMM_CUDA(cudaEventCreate(&h->ev0));
        SPMM_CUDA(cudaEventCreate(&h->ev1));
    }
    h->timing = enable != 0;
    h->timed = false;
    return SPMM_OK;
}

spmm_status spmm_last_kernel_ms(spmm_handle h, float *ms) {
    if (!h || !ms) return fail(SPMM_ERR_INVALID_ARG, "NULL argument");
    *ms = 0.f;
    if (!h->timed) return SPMM_OK;
    SPMM_CUDA(cudaEventSynchronize(h->ev1));
    SPMM_CUDA(cudaEventElapsedTime(ms, h->ev0, h->ev1));
    return SPMM_OK;
}

}  // extern "C"
