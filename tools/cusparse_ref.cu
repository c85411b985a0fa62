// cusparse_ref.cu -- measurement baseline (not the method): cuSPARSE SpMM on the same CSR and B, so bench.py can
// report the library's time beside ours (BASELINE.json north star: "cuSPARSE SpMM on the same inputs"; SURVEY.md
// §8(d): CSR ALG1/ALG2/ALG3 row-major, best-of, mirroring the paper's comparison P:L166).
//
//   int cusparse_ref_spmm(M, N, nnz, rowptr (int32 device), colidx (int32 device), value (f32 device),
//                         B (f32 device, N x K row-major), K, C (f32 device, M x K row-major), alg, reps,
//                         flush (device scratch, may be NULL), flush_bytes, stream, times_ms (host, reps))
// alg: 1, 2, 3 = CUSPARSE_SPMM_CSR_ALG1/2/3, 0 = CUSPARSE_SPMM_ALG_DEFAULT.  Each rep: memset of the flush
// buffer (L2 flush, outside the events), then cusparseSpMM between two CUDA events on `stream`.  The
// work buffer and the preprocessing (ALG3) are outside the timed region, as a library user would amortise them.
// Returns 0, or a negative cuSPARSE / CUDA status (the caller reports the algorithm as unavailable).
#include <cuda_runtime.h>
#include <cusparse.h>
#include <stdint.h>

#define CK(x)                                  \
    do {                                       \
        cusparseStatus_t s_ = (x);             \
        if (s_ != CUSPARSE_STATUS_SUCCESS) {   \
            rc = -1000 - (int)s_;              \
            goto done;                         \
        }                                      \
    } while (0)
#define CC(x)                                  \
    do {                                       \
        cudaError_t e_ = (x);                  \
        if (e_ != cudaSuccess) {               \
            rc = -(int)e_;                     \
            goto done;                         \
        }                                      \
    } while (0)

extern "C" int cusparse_ref_spmm(int64_t M, int64_t N, int64_t nnz, const int32_t *rowptr, const int32_t *colidx,
                                 const float *value, const float *B, int64_t K, float *C, int alg, int reps,
                                 void *flush, size_t flush_bytes, void *stream, float *times_ms) {
    int rc = 0;
    cusparseHandle_t h = nullptr;
    cusparseSpMatDescr_t A = nullptr;
    cusparseDnMatDescr_t Bd = nullptr, Cd = nullptr;
    void *work = nullptr;
    size_t wbytes = 0;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    const float alpha = 1.0f, beta = 0.0f;
    cudaStream_t s = (cudaStream_t)stream;
    const cusparseSpMMAlg_t a = alg == 1 ? CUSPARSE_SPMM_CSR_ALG1 : alg == 2 ? CUSPARSE_SPMM_CSR_ALG2
                              : alg == 3 ? CUSPARSE_SPMM_CSR_ALG3 : CUSPARSE_SPMM_ALG_DEFAULT;
    CK(cusparseCreate(&h));
    CK(cusparseSetStream(h, s));
    CK(cusparseCreateCsr(&A, M, N, nnz, (void *)rowptr, (void *)colidx, (void *)value, CUSPARSE_INDEX_32I,
                         CUSPARSE_INDEX_32I, CUSPARSE_INDEX_BASE_ZERO, CUDA_R_32F));
    CK(cusparseCreateDnMat(&Bd, N, K, K, (void *)B, CUDA_R_32F, CUSPARSE_ORDER_ROW));
    CK(cusparseCreateDnMat(&Cd, M, K, K, (void *)C, CUDA_R_32F, CUSPARSE_ORDER_ROW));
    CK(cusparseSpMM_bufferSize(h, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE, &alpha, A, Bd,
                               &beta, Cd, CUDA_R_32F, a, &wbytes));
    if (wbytes) CC(cudaMalloc(&work, wbytes));
    if (a == CUSPARSE_SPMM_CSR_ALG3)
        CK(cusparseSpMM_preprocess(h, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE, &alpha, A,
                                   Bd, &beta, Cd, CUDA_R_32F, a, work));
    CC(cudaEventCreate(&e0));
    CC(cudaEventCreate(&e1));
    for (int r = -2; r < reps; ++r) {      // two untimed warm-ups
        if (flush && flush_bytes) CC(cudaMemsetAsync(flush, r & 0xff, flush_bytes, s));
        CC(cudaEventRecord(e0, s));
        CK(cusparseSpMM(h, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE, &alpha, A, Bd, &beta,
                        Cd, CUDA_R_32F, a, work));
        CC(cudaEventRecord(e1, s));
        CC(cudaEventSynchronize(e1));
        if (r >= 0) CC(cudaEventElapsedTime(&times_ms[r], e0, e1));
    }
done:
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    if (work) cudaFree(work);
    if (Cd) cusparseDestroyDnMat(Cd);
    if (Bd) cusparseDestroyDnMat(Bd);
    if (A) cusparseDestroySpMat(A);
    if (h) cusparseDestroy(h);
    return rc;
}
