// nm_gcn_layer: one GCN layer, Eq. 1: Hout = act(Ahat (H W) + b).
// Two execution orders with the same result up to rounding:
//  * linear first (GCN's own order, L564: "GCN aggregates after its linear layer"):
//      XW = H W (cuBLASLt, 16-bit out) -> Y = Ahat XW (nm_spmm, fp32) -> act(Y + b)
//  * aggregate first (fewer SpMM columns when F_out > F_in, e.g. ogbn-products 100 -> 256):
//      Ya = Ahat H (nm_spmm, fp32) -> 16-bit -> Z = Ya W (cuBLASLt, fp32 out) -> act(Z + b)
// The dense products are plain library GEMMs (cuBLASLt, fp32 accumulation); the aggregation
// is libnm's sparse-tensor-core SpMM; bias + activation + down-convert are one fused pass.
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

template <int BF>
__global__ void k_to16(const float* __restrict__ Y, int64_t total, uint16_t* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    uint16_t b;
    if (BF) {
      __nv_bfloat16 h = __float2bfloat16_rn(Y[i]);
      b = *(uint16_t*)&h;
    } else {
      __half h = __float2half_rn(Y[i]);
      b = *(uint16_t*)&h;
    }
    out[i] = b;
  }
}

struct LtHandle {
  cublasLtHandle_t h = nullptr;
  ~LtHandle() {
    if (h) cublasLtDestroy(h);
  }
};

nm_status lt_fail(cublasStatus_t s, const char* what) {
  return fail(NM_ERR_CUDA, std::string(what) + ": cublasLt status " + std::to_string((int)s));
}

// C[m x nc] = A[m x k] * W[k x nc], all row-major; A, W 16-bit, C 16-bit or fp32.  Computed as
// the column-major product C^T = W^T A^T (no transposes needed).
nm_status dense_gemm(const void* A, const void* W, void* C, int64_t m, int k, int nc, nm_dtype dt, bool c_f32,
                     void* ws, cudaStream_t s) {
  static thread_local LtHandle lt;
  if (!lt.h) {
    cublasStatus_t r = cublasLtCreate(&lt.h);
    if (r != CUBLAS_STATUS_SUCCESS) return lt_fail(r, "cublasLtCreate");
  }
  if (m == 0) return NM_OK;
  const cudaDataType_t ty = dt == NM_BF16 ? CUDA_R_16BF : CUDA_R_16F;
  const cudaDataType_t cty = c_f32 ? CUDA_R_32F : ty;
  cublasLtMatmulDesc_t op = nullptr;
  cublasLtMatrixLayout_t la = nullptr, lb = nullptr, lc = nullptr;
  cublasLtMatmulPreference_t pref = nullptr;
  nm_status st = NM_OK;
  do {
    if (cublasLtMatmulDescCreate(&op, CUBLAS_COMPUTE_32F, CUDA_R_32F) != CUBLAS_STATUS_SUCCESS) {
      st = fail(NM_ERR_CUDA, "cublasLtMatmulDescCreate");
      break;
    }
    if (cublasLtMatrixLayoutCreate(&la, ty, nc, k, nc) != CUBLAS_STATUS_SUCCESS ||
        cublasLtMatrixLayoutCreate(&lb, ty, k, m, k) != CUBLAS_STATUS_SUCCESS ||
        cublasLtMatrixLayoutCreate(&lc, cty, nc, m, nc) != CUBLAS_STATUS_SUCCESS) {
      st = fail(NM_ERR_CUDA, "cublasLtMatrixLayoutCreate");
      break;
    }
    if (cublasLtMatmulPreferenceCreate(&pref) != CUBLAS_STATUS_SUCCESS) {
      st = fail(NM_ERR_CUDA, "cublasLtMatmulPreferenceCreate");
      break;
    }
    size_t wsb = kLtWorkspace;
    cublasLtMatmulPreferenceSetAttribute(pref, CUBLASLT_MATMUL_PREF_MAX_WORKSPACE_BYTES, &wsb, sizeof(wsb));
    cublasLtMatmulHeuristicResult_t heur;
    int nres = 0;
    if (cublasLtMatmulAlgoGetHeuristic(lt.h, op, la, lb, lc, lc, pref, 1, &heur, &nres) != CUBLAS_STATUS_SUCCESS ||
        nres == 0) {
      st = fail(NM_ERR_CUDA, "cublasLt: no algorithm");
      break;
    }
    const float one = 1.f, zero = 0.f;
    cublasStatus_t r = cublasLtMatmul(lt.h, op, &one, W, la, A, lb, &zero, C, lc, C, lc, &heur.algo, ws, wsb, s);
    if (r != CUBLAS_STATUS_SUCCESS) st = lt_fail(r, "cublasLtMatmul");
  } while (0);
  if (pref) cublasLtMatmulPreferenceDestroy(pref);
  if (la) cublasLtMatrixLayoutDestroy(la);
  if (lb) cublasLtMatrixLayoutDestroy(lb);
  if (lc) cublasLtMatrixLayoutDestroy(lc);
  if (op) cublasLtMatmulDescDestroy(op);
  return st;
}

inline int grid_for(int64_t total) {
  int64_t g = (total + 255) / 256;
  if (g > 148 * 16) g = 148 * 16;
  return (int)(g < 1 ? 1 : g);
}

}  // namespace
}  // namespace nm

using namespace nm;

extern "C" size_t nm_gcn_workspace_bytes(int64_t n, int F_in, int F_out) {
  const size_t fmax = (size_t)(F_in > F_out ? F_in : F_out);
  return align256((size_t)n * fmax * 2) + align256((size_t)n * fmax * 4) + align256((size_t)n * F_out * 4) +
         kLtWorkspace;
}

extern "C" nm_status nm_gcn_layer(const nm_packed* Ahat, const void* H, const void* W, const float* bias,
                                  void* Hout, int F_in, int F_out, int flags, void* ws, size_t ws_bytes,
                                  void* stream) {
  if (!Ahat || !H || !W || !Hout || !ws) return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer: NULL argument");
  if (F_in < 1 || F_out < 1 || F_out % 8 != 0 || F_in % 8 != 0)
    return fail(NM_ERR_UNSUPPORTED, "nm_gcn_layer: F_in and F_out must be positive multiples of 8");
  if (flags & ~(NM_RELU | NM_AGG_FIRST | NM_ORDER_AUTO)) return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer: unknown flags");
  if (Ahat->row_map) return fail(NM_ERR_UNSUPPORTED, "nm_gcn_layer: needs a pack in permuted order (flags 0)");
  const int64_t n = Ahat->n, rows = Ahat->row_end - Ahat->row_begin;
  if (ws_bytes < nm_gcn_workspace_bytes(n, F_in, F_out))
    return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer: workspace too small");
  const bool agg_first = (flags & NM_AGG_FIRST) || ((flags & NM_ORDER_AUTO) && F_out > F_in);
  cudaStream_t s = (cudaStream_t)stream;
  const size_t fmax = (size_t)(F_in > F_out ? F_in : F_out);
  uint8_t* w8 = (uint8_t*)ws;
  void* buf16 = w8;                                                   // n x fmax 16-bit
  float* buf32 = (float*)(w8 + align256((size_t)n * fmax * 2));       // n x fmax fp32
  float* out32 = (float*)((uint8_t*)buf32 + align256((size_t)n * fmax * 4));  // n x F_out fp32
  void* lt_ws = (uint8_t*)out32 + align256((size_t)n * F_out * 4);
  const bool bf = Ahat->dtype == NM_BF16;
  nm_status st;
  const float* pre;  // rows x F_out fp32 before bias / activation
  if (!agg_first) {
    st = dense_gemm(H, W, buf16, n, F_in, F_out, Ahat->dtype, false, lt_ws, s);  // XW (n x F_out)
    if (st != NM_OK) return st;
    st = nm_spmm(Ahat, buf16, F_out, buf32, F_out, F_out, stream);
    if (st != NM_OK) return st;
    pre = buf32;
  } else {
    st = nm_spmm(Ahat, H, F_in, buf32, F_in, F_in, stream);                     // Ahat H (rows x F_in)
    if (st != NM_OK) return st;
    if (bf) k_to16<1><<<grid_for(rows * F_in), 256, 0, s>>>(buf32, rows * F_in, (uint16_t*)buf16);
    else k_to16<0><<<grid_for(rows * F_in), 256, 0, s>>>(buf32, rows * F_in, (uint16_t*)buf16);
    NM_CUDA(cudaGetLastError());
    st = dense_gemm(buf16, W, out32, rows, F_in, F_out, Ahat->dtype, true, lt_ws, s);  // (Ahat H) W
    if (st != NM_OK) return st;
    pre = out32;
  }
  if (bf) k_bias_act<1><<<grid_for(rows * F_out), 256, 0, s>>>(pre, rows, F_out, bias, flags & NM_RELU, (uint16_t*)Hout);
  else k_bias_act<0><<<grid_for(rows * F_out), 256, 0, s>>>(pre, rows, F_out, bias, flags & NM_RELU, (uint16_t*)Hout);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}
