// panel.cu -- a7 for kernel mode 2 (panel-staged SpMM): the schedule that lets the rows a CTA processes
// together share their B rows through shared memory.
//
// The paper's CTA-aware idea ("clusters of N_w consecutive rows ... processed in parallel ... cache
// lines requested by one warp are re-used by another warp running at the same time") relies on the
// hardware cache.  On B200 every nnz of the row-group kernel pulls its whole B row (4K bytes) through L2
// (measured L2->SM ceiling ~17.8 TB/s), so reuse among concurrently processed rows is made
// explicit: positions are cut into panels of `pr` consecutive rows of the permuted order; for each panel the
// columns referenced >= t times (t >= 2 chosen per panel so that at most `cap` B rows are selected, `cap`
// = shared-memory budget / 4K) are staged once into shared memory, and their nnz read B from there.  The
// row order decides how much reuse a panel has, so the locality policies pay off directly.
//
// Build (all on the device): key = (panel, col) per nnz -> stable radix sort -> runs of equal key (=
// per-panel column frequencies) -> per-panel frequency histogram -> threshold -> slots (scan) -> a copy of
// the interleaved permuted CSR whose staged columns are replaced by (slot | 0x80000000).  Work units are
// the panel's rows cut into <= split_nnz chunks (chunks of long rows write partials, combined pairwise).
#include "internal.cuh"
#include <algorithm>

namespace spmm {
namespace {

constexpr int HBINS = 64;

inline unsigned gb(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 32)); }
inline unsigned gw(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n * 32, 256), 148 * 64)); }

// key = (panel << colbits) | col for every nnz of the permuted CSR (warp per row)
__global__ void k_panel_keys(const int32_t *rowptr, const int2 *cv, int64_t M, int32_t pr, int colbits, uint64_t *keys,
                             uint32_t *vals) {
    const int lane = threadIdx.x & 31;
    for (int64_t p = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; p < M; p += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const uint64_t panel = (uint64_t)(p / pr);
        for (int32_t j = rowptr[p] + lane; j < rowptr[p + 1]; j += 32) {
            keys[j] = (panel << colbits) | (uint64_t)(uint32_t)cv[j].x;
            vals[j] = (uint32_t)j;
        }
    }
}

__global__ void k_run_flags(const uint64_t *keys, int64_t n, int32_t *flag) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        flag[i] = (i == 0 || keys[i] != keys[i - 1]) ? 1 : 0;
}

// run id (inclusive) of element i from the exclusive scan of run-start flags
__global__ void k_inclusive_ids(const int32_t *flag, int32_t *rid, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        rid[i] = rid[i] + flag[i] - 1;
}

__global__ void k_run_starts(const int32_t *flag, const int32_t *rid, int64_t n, int32_t *run_start) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (flag[i]) run_start[rid[i]] = (int32_t)i;
}

// per run: panel, count; histogram of counts per panel
__global__ void k_run_hist(const uint64_t *keys, const int32_t *run_start, int64_t n_runs, int64_t n, int colbits,
                           int32_t *run_count, int32_t *hist) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n_runs; r += (int64_t)gridDim.x * blockDim.x) {
        const int32_t s0 = run_start[r], s1 = r + 1 < n_runs ? run_start[r + 1] : (int32_t)n;
        const int32_t c = s1 - s0;
        run_count[r] = c;
        const int64_t panel = (int64_t)(keys[s0] >> colbits);
        atomicAdd(&hist[panel * HBINS + min(c, HBINS - 1)], 1);
    }
}

// per panel: smallest threshold t >= 2 with sum_{c >= t} hist[c] <= cap (t = HBINS-1 if none)
__global__ void k_panel_threshold(const int32_t *hist, int64_t n_panels, int32_t cap, int32_t *thr) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n_panels; p += (int64_t)gridDim.x * blockDim.x) {
        int32_t acc = 0, t = HBINS - 1;
        for (int c = HBINS - 1; c >= 2; --c) {
            acc += hist[p * HBINS + c];
            if (acc > cap) break;
            t = c;
        }
        thr[p] = t;
    }
}

__global__ void k_run_stage_flag(const uint64_t *keys, const int32_t *run_start, const int32_t *run_count,
                                 const int32_t *thr, int64_t n_runs, int colbits, int32_t *flag) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n_runs; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t panel = (int64_t)(keys[run_start[r]] >> colbits);
        flag[r] = run_count[r] >= max(thr[panel], 2) ? 1 : 0;
    }
}

// slot within the panel = global staged index - first staged index of the panel; enforce cap
__global__ void k_panel_first(const uint64_t *keys, const int32_t *run_start, const int32_t *gs, int64_t n_runs,
                              int colbits, int32_t *panel_first) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n_runs; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t panel = (int64_t)(keys[run_start[r]] >> colbits);
        const bool first = r == 0 || (int64_t)(keys[run_start[r - 1]] >> colbits) != panel;
        if (first) panel_first[panel] = gs[r];
    }
}

__global__ void k_run_final(const uint64_t *keys, const int32_t *run_start, const int32_t *flag, const int32_t *gs,
                            const int32_t *panel_first, int64_t n_runs, int colbits, int32_t cap, int32_t *final_flag,
                            int32_t *panel_cnt) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n_runs; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t panel = (int64_t)(keys[run_start[r]] >> colbits);
        const bool f = flag[r] && (gs[r] - panel_first[panel]) < cap;
        final_flag[r] = f;
        if (f) atomicAdd(&panel_cnt[panel], 1);
    }
}

// staged column list + rewritten cv (slot | 0x80000000) for every nnz of a staged run
__global__ void k_stage_write(const uint64_t *keys, const uint32_t *vals, const int32_t *rid, const int32_t *run_start,
                              const int32_t *final_flag, const int32_t *fs, const int32_t *stage_ptr, int64_t n,
                              int colbits, int32_t *staged_cols, int2 *cv_ps, unsigned long long *staged_nnz) {
    unsigned long long cnt = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t r = rid[i];
        if (!final_flag[r]) continue;
        const int64_t panel = (int64_t)(keys[i] >> colbits);
        const int32_t slot = fs[r] - stage_ptr[panel];
        if (run_start[r] == (int32_t)i) staged_cols[fs[r]] = (int32_t)(keys[i] & ((1ULL << colbits) - 1));
        cv_ps[vals[i]].x = (int32_t)((uint32_t)slot | 0x80000000u);
        ++cnt;
    }
    atomicAdd(staged_nnz, cnt);
}

// work units: every non-empty row cut into <= split chunks, in position order
__global__ void k_unit_counts(const int32_t *rowptr, int64_t M, int32_t split, int32_t *nunits, int32_t *is_long,
                              int32_t *nch_long, int32_t *is_empty) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        const int32_t len = rowptr[p + 1] - rowptr[p];
        const int32_t nc = (len + split - 1) / split;
        nunits[p] = nc;
        is_long[p] = len > split;
        nch_long[p] = len > split ? nc : 0;
        is_empty[p] = len == 0;
    }
}

__global__ void k_unit_fill(const int32_t *rowptr, const int32_t *perm, const int32_t *uoff, const int32_t *is_long,
                            const int32_t *lidx, const int32_t *poff, int64_t M, int32_t split, int4 *units,
                            int32_t *long_dst) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        const int32_t a = rowptr[p], len = rowptr[p + 1] - a;
        if (len == 0) continue;
        if (!is_long[p]) {
            units[uoff[p]] = make_int4(a, len, perm[p], 0);
        } else {
            const int32_t nc = (len + split - 1) / split;
            for (int32_t c = 0; c < nc; ++c)
                units[uoff[p] + c] = make_int4(a + c * split, min(split, len - c * split), -(poff[p] + c) - 1, 0);
            long_dst[lidx[p]] = perm[p];
        }
    }
}

__global__ void k_panel_unit_ptr(const int32_t *uoff, int64_t M, int32_t pr, int64_t n_panels, int32_t *ptr) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q <= n_panels; q += (int64_t)gridDim.x * blockDim.x)
        ptr[q] = uoff[q * pr < M ? q * pr : M];
}

__global__ void k_long_pslot_ptr(const int32_t *is_long, const int32_t *lidx, const int32_t *poff, int64_t M, int32_t *ptr) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x)
        if (is_long[p]) ptr[lidx[p]] = poff[p];
}

__global__ void k_scatter_pos(const int32_t *flag, const int32_t *pos, const int32_t *val, int64_t M, int32_t *out) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x)
        if (flag[p]) out[pos[p]] = val[p];
}

__global__ void k_set1(int32_t *a, int64_t i, int32_t v) { a[i] = v; }

int bits_for(uint64_t v) {
    int b = 0;
    while (b < 64 && (v >> b) != 0) ++b;
    return std::max(b, 1);
}

}  // namespace

spmm_status build_panel_schedule(spmm_ctx *h, int64_t K, int32_t pr, int32_t cap, cudaStream_t s) {
    PanelSchedule &P = h->psched;
    P.K = 0;
    const int64_t M = h->M, nnz = h->nnz;
    const int32_t split = h->params.split_nnz;
    const int32_t *rowptr = h->rowptr_p.as<int32_t>();
    P.pr = pr;
    P.cap = cap;
    P.n_panels = ceil_div(M, pr);
    const int colbits = bits_for((uint64_t)std::max<int64_t>(h->N - 1, 1));
    const int panelbits = bits_for((uint64_t)std::max<int64_t>(P.n_panels - 1, 1));
    if (colbits + panelbits > 62) return fail(SPMM_ERR_UNSUPPORTED, "panel schedule: key does not fit 64 bits");

    // ---- staged columns per panel ----
    SPMM_TRY(P.cv_ps.alloc(std::max<int64_t>(nnz, 1) * sizeof(int2), s));
    if (nnz > 0) SPMM_CUDA(cudaMemcpyAsync(P.cv_ps.p, h->cv_p.p, nnz * sizeof(int2), cudaMemcpyDeviceToDevice, s));
    SPMM_TRY(P.stage_ptr.alloc((P.n_panels + 1) * sizeof(int32_t), s));
    int32_t n_staged = 0;
    unsigned long long staged_nnz = 0;
    if (nnz > 0) {
        DevBuf keys, vals, flag, rid, run_start, run_count, hist, thr, sflag, gs, pfirst, fflag, fs, pcnt, snz;
        SPMM_TRY(keys.alloc(nnz * sizeof(uint64_t), s));
        SPMM_TRY(vals.alloc(nnz * sizeof(uint32_t), s));
        k_panel_keys<<<gw(M), 256, 0, s>>>(rowptr, h->cv_p.as<int2>(), M, pr, colbits, keys.as<uint64_t>(), vals.as<uint32_t>());
        SPMM_CUDA(cudaGetLastError());
        SPMM_TRY(radix_sort_pairs(keys.as<uint64_t>(), vals.as<uint32_t>(), nnz, 0, colbits + panelbits, s));
        SPMM_TRY(flag.alloc(nnz * sizeof(int32_t), s));
        SPMM_TRY(rid.alloc((nnz + 1) * sizeof(int32_t), s));
        k_run_flags<<<gb(nnz), 256, 0, s>>>(keys.as<uint64_t>(), nnz, flag.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        int32_t n_runs = 0;
        SPMM_TRY(exclusive_scan_i32(flag.as<int32_t>(), rid.as<int32_t>(), nnz, &n_runs, s));
        // rid = exclusive count of run starts before i: run of element i = rid[i] + flag[i] - 1
        // (convert to the inclusive run id in place)
        SPMM_TRY(run_start.alloc(n_runs * sizeof(int32_t), s));
        SPMM_TRY(run_count.alloc(n_runs * sizeof(int32_t), s));
        SPMM_TRY(hist.alloc(P.n_panels * HBINS * sizeof(int32_t), s));
        SPMM_TRY(thr.alloc(P.n_panels * sizeof(int32_t), s));
        SPMM_TRY(sflag.alloc(n_runs * sizeof(int32_t), s));
        SPMM_TRY(gs.alloc((n_runs + 1) * sizeof(int32_t), s));
        SPMM_TRY(pfirst.alloc(P.n_panels * sizeof(int32_t), s));
        SPMM_TRY(fflag.alloc(n_runs * sizeof(int32_t), s));
        SPMM_TRY(fs.alloc((n_runs + 1) * sizeof(int32_t), s));
        SPMM_TRY(pcnt.alloc(P.n_panels * sizeof(int32_t), s));
        SPMM_TRY(snz.alloc(sizeof(unsigned long long), s));
        SPMM_CUDA(cudaMemsetAsync(hist.p, 0, hist.bytes, s));
        SPMM_CUDA(cudaMemsetAsync(pcnt.p, 0, pcnt.bytes, s));
        SPMM_CUDA(cudaMemsetAsync(snz.p, 0, snz.bytes, s));
        SPMM_CUDA(cudaMemsetAsync(pfirst.p, 0, pfirst.bytes, s));
        k_inclusive_ids<<<gb(nnz), 256, 0, s>>>(flag.as<int32_t>(), rid.as<int32_t>(), nnz);
        k_run_starts<<<gb(nnz), 256, 0, s>>>(flag.as<int32_t>(), rid.as<int32_t>(), nnz, run_start.as<int32_t>());
        k_run_hist<<<gb(n_runs), 256, 0, s>>>(keys.as<uint64_t>(), run_start.as<int32_t>(), n_runs, nnz, colbits,
                                              run_count.as<int32_t>(), hist.as<int32_t>());
        k_panel_threshold<<<gb(P.n_panels), 256, 0, s>>>(hist.as<int32_t>(), P.n_panels, cap, thr.as<int32_t>());
        k_run_stage_flag<<<gb(n_runs), 256, 0, s>>>(keys.as<uint64_t>(), run_start.as<int32_t>(), run_count.as<int32_t>(),
                                                    thr.as<int32_t>(), n_runs, colbits, sflag.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        SPMM_TRY(exclusive_scan_i32(sflag.as<int32_t>(), gs.as<int32_t>(), n_runs, nullptr, s));
        k_panel_first<<<gb(n_runs), 256, 0, s>>>(keys.as<uint64_t>(), run_start.as<int32_t>(), gs.as<int32_t>(), n_runs,
                                                 colbits, pfirst.as<int32_t>());
        k_run_final<<<gb(n_runs), 256, 0, s>>>(keys.as<uint64_t>(), run_start.as<int32_t>(), sflag.as<int32_t>(),
                                               gs.as<int32_t>(), pfirst.as<int32_t>(), n_runs, colbits, cap,
                                               fflag.as<int32_t>(), pcnt.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        SPMM_TRY(exclusive_scan_i32(fflag.as<int32_t>(), fs.as<int32_t>(), n_runs, &n_staged, s));
        SPMM_TRY(exclusive_scan_i32(pcnt.as<int32_t>(), P.stage_ptr.as<int32_t>(), P.n_panels, nullptr, s));
        SPMM_TRY(P.staged_cols.alloc(std::max<int32_t>(n_staged, 1) * sizeof(int32_t), s));
        k_stage_write<<<gb(nnz), 256, 0, s>>>(keys.as<uint64_t>(), vals.as<uint32_t>(), rid.as<int32_t>(),
                                              run_start.as<int32_t>(), fflag.as<int32_t>(), fs.as<int32_t>(),
                                              P.stage_ptr.as<int32_t>(), nnz, colbits, P.staged_cols.as<int32_t>(),
                                              P.cv_ps.as<int2>(), snz.as<unsigned long long>());
        SPMM_CUDA(cudaGetLastError());
        SPMM_CUDA(cudaMemcpyAsync(&staged_nnz, snz.p, sizeof(staged_nnz), cudaMemcpyDeviceToHost, s));
    } else {
        SPMM_CUDA(cudaMemsetAsync(P.stage_ptr.p, 0, P.stage_ptr.bytes, s));
        SPMM_TRY(P.staged_cols.alloc(sizeof(int32_t), s));
    }
    // ---- work units, long rows, empty rows ----
    DevBuf nun, isl, nchl, ise, uoff, lidx, poff, eoff, pidx;
    SPMM_TRY(nun.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
    SPMM_TRY(isl.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
    SPMM_TRY(nchl.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
    SPMM_TRY(ise.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
    SPMM_TRY(uoff.alloc((M + 1) * sizeof(int32_t), s));
    SPMM_TRY(lidx.alloc((M + 1) * sizeof(int32_t), s));
    SPMM_TRY(poff.alloc((M + 1) * sizeof(int32_t), s));
    SPMM_TRY(eoff.alloc((M + 1) * sizeof(int32_t), s));
    SPMM_TRY(pidx.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
    k_unit_counts<<<gb(M), 256, 0, s>>>(rowptr, M, split, nun.as<int32_t>(), isl.as<int32_t>(), nchl.as<int32_t>(),
                                        ise.as<int32_t>());
    SPMM_CUDA(cudaGetLastError());
    int32_t n_units = 0, n_long = 0, n_pslots = 0, n_empty = 0;
    SPMM_TRY(exclusive_scan_i32(nun.as<int32_t>(), uoff.as<int32_t>(), M, &n_units, s));
    SPMM_TRY(exclusive_scan_i32(isl.as<int32_t>(), lidx.as<int32_t>(), M, &n_long, s));
    SPMM_TRY(exclusive_scan_i32(nchl.as<int32_t>(), poff.as<int32_t>(), M, &n_pslots, s));
    SPMM_TRY(exclusive_scan_i32(ise.as<int32_t>(), eoff.as<int32_t>(), M, &n_empty, s));
    P.n_units = n_units;
    P.n_long = n_long;
    P.n_pslots = n_pslots;
    P.n_empty = n_empty;
    SPMM_TRY(P.units.alloc(std::max<int64_t>(n_units, 1) * sizeof(int4), s));
    SPMM_TRY(P.long_dst.alloc(std::max<int32_t>(n_long, 1) * sizeof(int32_t), s));
    SPMM_TRY(P.pslot_ptr.alloc((n_long + 1) * sizeof(int32_t), s));
    SPMM_TRY(P.empty_dst.alloc(std::max<int32_t>(n_empty, 1) * sizeof(int32_t), s));
    SPMM_TRY(P.panel_unit_ptr.alloc((P.n_panels + 1) * sizeof(int32_t), s));
    if (M > 0) {
        k_unit_fill<<<gb(M), 256, 0, s>>>(rowptr, h->perm.as<int32_t>(), uoff.as<int32_t>(), isl.as<int32_t>(),
                                          lidx.as<int32_t>(), poff.as<int32_t>(), M, split, P.units.as<int4>(),
                                          P.long_dst.as<int32_t>());
        k_panel_unit_ptr<<<gb(P.n_panels + 1), 256, 0, s>>>(uoff.as<int32_t>(), M, pr, P.n_panels,
                                                            P.panel_unit_ptr.as<int32_t>());
        k_long_pslot_ptr<<<gb(M), 256, 0, s>>>(isl.as<int32_t>(), lidx.as<int32_t>(), poff.as<int32_t>(), M,
                                               P.pslot_ptr.as<int32_t>());
        k_set1<<<1, 1, 0, s>>>(P.pslot_ptr.as<int32_t>(), n_long, n_pslots);
        k_scatter_pos<<<gb(M), 256, 0, s>>>(ise.as<int32_t>(), eoff.as<int32_t>(), h->perm.as<int32_t>(), M,
                                            P.empty_dst.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    SPMM_CUDA(cudaStreamSynchronize(s));
    P.n_staged = n_staged;
    P.staged_nnz = (int64_t)staged_nnz;
    P.K = K;
    return SPMM_OK;
}

}  // namespace spmm
