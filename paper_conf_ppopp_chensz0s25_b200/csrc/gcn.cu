// nm_gcn_layer: one GCN layer, Eq. 1: Hout = ReLU(Ahat (H W) + b).
// Linear first ("GCN aggregates after its linear layer", L564): the dense H W is a plain
// library GEMM (cuBLASLt, bf16/fp16 in, fp32 accumulate); the aggregation is nm_spmm on the
// packed Ahat (sparse tensor cores + residual); bias + activation + down-convert are fused in
// one elementwise pass over the fp32 aggregation result.
#include <cublasLt.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "nm_internal.h"

namespace nm {
namespace {

constexpr size_t kLtWorkspace = 32u << 20;

inline size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

template <int BF>
__global__ void k_bias_act(const float* __restrict__ Y, int64_t rows, int F, const float* __restrict__ bias,
                           int relu, uint16_t* __restrict__ out) {
  const int64_t total = rows * F;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    float v = Y[i] + (bias ? bias[i % F] : 0.f);
    if (relu) v = fmaxf(v, 0.f);
    uint16_t b;
    if (BF) {
      __nv_bfloat16 h = __float2bfloat16_rn(v);
      b = *(uint16_t*)&h;
    } else {
      __half h = __float2half_rn(v);
      b = *(uint16_t*)&h;
    }
    out[i] = b;
  }
}

struct LtHandle {
  cublasLtHandle_t h = nullptr;
  ~LtHandle() { if (h) cublasLtDestroy(h); }
};

nm_status lt_fail(cublasStatus_t s, const char* what) {
  return fail(NM_ERR_CUDA, std::string(what) + ": cublasLt status " + std::to_string((int)s));
}

#define NM_LT(call)                                       \
  do {                                                    \
    cublasStatus_t s_ = (call);                           \
    if (s_ != CUBLAS_STATUS_SUCCESS) return lt_fail(s_, #call); \
  } while (0)

// C[n x Fo] = H[n x Fi] * W[Fi x Fo], all row-major 16-bit; computed as the column-major
// product C^T = W^T H^T (no transposes needed).
nm_status dense_xw(const void* H, const void* W, void* C, int64_t n, int Fi, int Fo, nm_dtype dt, void* ws,
                   cudaStream_t s) {
  static thread_local LtHandle lt;
  if (!lt.h) NM_LT(cublasLtCreate(&lt.h));
  const cudaDataType_t ty = dt == NM_BF16 ? CUDA_R_16BF : CUDA_R_16F;
  cublasLtMatmulDesc_t op = nullptr;
  cublasLtMatrixLayout_t la = nullptr, lb = nullptr, lc = nullptr;
  cublasLtMatmulPreference_t pref = nullptr;
  nm_status st = NM_OK;
  do {
    if (cublasLtMatmulDescCreate(&op, CUBLAS_COMPUTE_32F, CUDA_R_32F) != CUBLAS_STATUS_SUCCESS) { st = fail(NM_ERR_CUDA, "cublasLtMatmulDescCreate"); break; }
    if (cublasLtMatrixLayoutCreate(&la, ty, Fo, Fi, Fo) != CUBLAS_STATUS_SUCCESS ||
        cublasLtMatrixLayoutCreate(&lb, ty, Fi, n, Fi) != CUBLAS_STATUS_SUCCESS ||
        cublasLtMatrixLayoutCreate(&lc, ty, Fo, n, Fo) != CUBLAS_STATUS_SUCCESS) { st = fail(NM_ERR_CUDA, "cublasLtMatrixLayoutCreate"); break; }
    if (cublasLtMatmulPreferenceCreate(&pref) != CUBLAS_STATUS_SUCCESS) { st = fail(NM_ERR_CUDA, "pref"); break; }
    size_t wsb = kLtWorkspace;
    cublasLtMatmulPreferenceSetAttribute(pref, CUBLASLT_MATMUL_PREF_MAX_WORKSPACE_BYTES, &wsb, sizeof(wsb));
    cublasLtMatmulHeuristicResult_t heur;
    int nres = 0;
    if (cublasLtMatmulAlgoGetHeuristic(lt.h, op, la, lb, lc, lc, pref, 1, &heur, &nres) != CUBLAS_STATUS_SUCCESS ||
        nres == 0) { st = fail(NM_ERR_CUDA, "cublasLt: no algorithm"); break; }
    const float one = 1.f, zero = 0.f;
    cublasStatus_t r = cublasLtMatmul(lt.h, op, &one, W, la, H, lb, &zero, C, lc, C, lc, &heur.algo, ws, wsb, s);
    if (r != CUBLAS_STATUS_SUCCESS) st = lt_fail(r, "cublasLtMatmul");
  } while (0);
  if (pref) cublasLtMatmulPreferenceDestroy(pref);
  if (la) cublasLtMatrixLayoutDestroy(la);
  if (lb) cublasLtMatrixLayoutDestroy(lb);
  if (lc) cublasLtMatrixLayoutDestroy(lc);
  if (op) cublasLtMatmulDescDestroy(op);
  return st;
}

}  // namespace
}  // namespace nm

using namespace nm;

extern "C" size_t nm_gcn_workspace_bytes(int64_t n, int F_out) {
  return align256((size_t)n * F_out * 2) + align256((size_t)n * F_out * 4) + kLtWorkspace;
}

extern "C" nm_status nm_gcn_layer(const nm_packed* Ahat, const void* H, const void* W, const float* bias,
                                  void* Hout, int F_in, int F_out, int flags, void* ws, size_t ws_bytes,
                                  void* stream) {
  if (!Ahat || !H || !W || !Hout || !ws) return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer: NULL argument");
  if (F_in < 1 || F_out < 1 || F_out % 8 != 0 || F_in % 8 != 0)
    return fail(NM_ERR_UNSUPPORTED, "nm_gcn_layer: F_in and F_out must be positive multiples of 8");
  const int64_t n = Ahat->n, rows = Ahat->row_end - Ahat->row_begin;
  if (ws_bytes < nm_gcn_workspace_bytes(n, F_out)) return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer: workspace too small");
  cudaStream_t s = (cudaStream_t)stream;
  uint8_t* w8 = (uint8_t*)ws;
  void* XW = w8;
  float* Yp = (float*)(w8 + align256((size_t)n * F_out * 2));
  void* lt_ws = w8 + align256((size_t)n * F_out * 2) + align256((size_t)n * F_out * 4);
  nm_status st = dense_xw(H, W, XW, n, F_in, F_out, Ahat->dtype, lt_ws, s);
  if (st != NM_OK) return st;
  st = nm_spmm(Ahat, XW, F_out, Yp, F_out, F_out, stream);
  if (st != NM_OK) return st;
  const int64_t total = rows * F_out;
  int grid = (int)((total + 255) / 256);
  if (grid > 148 * 16) grid = 148 * 16;
  if (grid < 1) grid = 1;
  if (Ahat->dtype == NM_BF16)
    k_bias_act<1><<<grid, 256, 0, s>>>(Yp, rows, F_out, bias, flags & NM_RELU, (uint16_t*)Hout);
  else
    k_bias_act<0><<<grid, 256, 0, s>>>(Yp, rows, F_out, bias, flags & NM_RELU, (uint16_t*)Hout);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}
