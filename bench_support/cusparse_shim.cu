// BASELINE ONLY (not part of libnm): cuSPARSE CSR SpMM on the same graph, the comparison
// the paper draws (DGL's CUSPARSE_SPMM_CSR_ALG2; Fig. 4 "speedup over
// cuSPARSE", L615-636).  A and X 16-bit, fp32 accumulation, Y fp32 when cuSPARSE accepts
// that mix (else Y in the 16-bit type -- reported by cs_info).
#include <cuda_runtime.h>
#include <cusparse.h>

#include <cstdint>
#include <cstdio>

struct CsHandle {
  cusparseHandle_t h = nullptr;
  cusparseSpMatDescr_t A = nullptr;
  cusparseDnMatDescr_t X = nullptr, Y = nullptr;
  void* buf = nullptr;
  cusparseSpMMAlg_t alg;
  int y_is_f32 = 1;
};

extern "C" {

// rp32: int32 row offsets [n+1] (device), ci: int32 [nnz] (device), val: 16-bit [nnz]
// (device), X: 16-bit n x F row-major (ld = ldx), Y: n x F row-major (ld = ldy), fp32 (or
// 16-bit if cuSPARSE rejects the mixed types: then *y_f32 = 0 and Y must hold 16-bit).
int cs_create(int64_t n, int64_t nnz, const int32_t* rp32, const int32_t* ci, const void* val, int bf16, int F,
              const void* X, int64_t ldx, void* Y, int64_t ldy, int alg, void** out, int* y_f32) {
  CsHandle* c = new CsHandle();
  c->alg = alg == 2 ? CUSPARSE_SPMM_CSR_ALG2 : (alg == 1 ? CUSPARSE_SPMM_CSR_ALG1 : CUSPARSE_SPMM_ALG_DEFAULT);
  cudaDataType_t t16 = bf16 ? CUDA_R_16BF : CUDA_R_16F;
  if (cusparseCreate(&c->h) != CUSPARSE_STATUS_SUCCESS) return 1;
  if (cusparseCreateCsr(&c->A, n, n, nnz, (void*)rp32, (void*)ci, (void*)val, CUSPARSE_INDEX_32I,
                        CUSPARSE_INDEX_32I, CUSPARSE_INDEX_BASE_ZERO, t16) != CUSPARSE_STATUS_SUCCESS)
    return 2;
  if (cusparseCreateDnMat(&c->X, n, F, ldx, (void*)X, t16, CUSPARSE_ORDER_ROW) != CUSPARSE_STATUS_SUCCESS) return 3;
  float one = 1.f, zero = 0.f;
  size_t bytes = 0;
  for (int attempt = 0; attempt < 2; ++attempt) {
    cudaDataType_t ty = attempt == 0 ? CUDA_R_32F : t16;
    if (c->Y) cusparseDestroyDnMat(c->Y);
    c->Y = nullptr;
    if (cusparseCreateDnMat(&c->Y, n, F, ldy, Y, ty, CUSPARSE_ORDER_ROW) != CUSPARSE_STATUS_SUCCESS) return 4;
    cusparseStatus_t st = cusparseSpMM_bufferSize(c->h, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE,
                                                  &one, c->A, c->X, &zero, c->Y, CUDA_R_32F, c->alg, &bytes);
    if (st == CUSPARSE_STATUS_SUCCESS) {
      c->y_is_f32 = attempt == 0;
      break;
    }
    if (attempt == 1) return 5;
  }
  if (bytes && cudaMalloc(&c->buf, bytes) != cudaSuccess) return 6;
  *out = c;
  *y_f32 = c->y_is_f32;
  return 0;
}

int cs_run(void* hp, void* stream) {
  CsHandle* c = (CsHandle*)hp;
  float one = 1.f, zero = 0.f;
  cusparseSetStream(c->h, (cudaStream_t)stream);
  return (int)cusparseSpMM(c->h, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE, &one, c->A, c->X,
                           &zero, c->Y, CUDA_R_32F, c->alg, c->buf);
}

void cs_destroy(void* hp) {
  CsHandle* c = (CsHandle*)hp;
  if (!c) return;
  if (c->buf) cudaFree(c->buf);
  if (c->A) cusparseDestroySpMat(c->A);
  if (c->X) cusparseDestroyDnMat(c->X);
  if (c->Y) cusparseDestroyDnMat(c->Y);
  if (c->h) cusparseDestroy(c->h);
  delete c;
}

}  // extern "C"
