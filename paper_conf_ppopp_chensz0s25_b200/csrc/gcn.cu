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

// bias + activation + down-convert of 8 consecutive features per thread, the 16-byte result
// stored into every destination buffer (row dst_row0 + l): the fused all-gather of
// nm_gcn_layer_bcast -- on a multi-GPU node the destinations are the ranks' peer-mapped
// (NVLink) buffers, so the rows reach every GPU from this kernel's own stores
constexpr int kMaxDst = 16;
struct DstList {
  uint16_t* p[kMaxDst];
  int n;
};

template <int BF>
__global__ void k_bias_act_bcast(const float* __restrict__ Y, int64_t rows, int F, const float* __restrict__ bias,
                                 int relu, DstList dst, int64_t dst_row0) {
  const int vpr = F / 8;  // 16-byte vectors per row (F % 8 == 0)
  const int64_t total = rows * vpr;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / vpr;
    const int c = (int)(i % vpr) * 8;
    const float4 a = *(const float4*)(Y + r * F + c), b = *(const float4*)(Y + r * F + c + 4);
    float v[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
    uint32_t w[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      float x0 = v[2 * q] + (bias ? bias[c + 2 * q] : 0.f), x1 = v[2 * q + 1] + (bias ? bias[c + 2 * q + 1] : 0.f);
      if (relu) {
        x0 = fmaxf(x0, 0.f);
        x1 = fmaxf(x1, 0.f);
      }
      uint16_t h0, h1;
      if (BF) {
        __nv_bfloat16 t0 = __float2bfloat16_rn(x0), t1 = __float2bfloat16_rn(x1);
        h0 = *(uint16_t*)&t0;
        h1 = *(uint16_t*)&t1;
      } else {
        __half t0 = __float2half_rn(x0), t1 = __float2half_rn(x1);
        h0 = *(uint16_t*)&t0;
        h1 = *(uint16_t*)&t1;
      }
      w[q] = (uint32_t)h0 | ((uint32_t)h1 << 16);
    }
    const uint4 o = make_uint4(w[0], w[1], w[2], w[3]);
    for (int d = 0; d < dst.n; ++d) *(uint4*)(dst.p[d] + (dst_row0 + r) * F + c) = o;
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

nm_status lt_fail(cublasStatus_t s, const char* what) {
  return fail(NM_ERR_CUDA, std::string(what) + ": cublasLt status " + std::to_string((int)s));
}

// One cuBLASLt problem: descriptors, layouts and the heuristic's algorithm, built once per
// shape and kept (per thread) for later calls -- nm_gcn_layer and the models call the same
// shapes every layer / step.
struct LtPlan {
  bool ta, tb, c_f32;
  int64_t m, nn, k, lda, ldb, ldc;
  nm_dtype dt;
  cublasLtMatmulDesc_t op = nullptr;
  cublasLtMatrixLayout_t la = nullptr, lb = nullptr, lc = nullptr;
  cublasLtMatmulAlgo_t algo;
  void destroy() {
    if (la) cublasLtMatrixLayoutDestroy(la);
    if (lb) cublasLtMatrixLayoutDestroy(lb);
    if (lc) cublasLtMatrixLayoutDestroy(lc);
    if (op) cublasLtMatmulDescDestroy(op);
    la = lb = lc = nullptr;
    op = nullptr;
  }
  bool same(bool ta_, bool tb_, int64_t m_, int64_t nn_, int64_t k_, int64_t lda_, int64_t ldb_, int64_t ldc_,
            nm_dtype dt_, bool c_) const {
    return ta == ta_ && tb == tb_ && m == m_ && nn == nn_ && k == k_ && lda == lda_ && ldb == ldb_ && ldc == ldc_ &&
           dt == dt_ && c_f32 == c_;
  }
};

struct LtCache {
  cublasLtHandle_t h = nullptr;
  static constexpr int kSlots = 16;
  LtPlan plans[kSlots];
  int used = 0, next = 0;
  ~LtCache() {
    for (int i = 0; i < used; ++i) plans[i].destroy();
    if (h) cublasLtDestroy(h);
  }
};

// General column-major product C[m x nn] = op(A)[m x k] op(B)[k x nn] (cuBLASLt, fp32
// accumulation); A/B 16-bit, C 16-bit or fp32; lda/ldb/ldc are column-major leading dims.
nm_status lt_gemm(bool ta, bool tb, int64_t m, int64_t nn, int64_t k, const void* A, int64_t lda, const void* B,
                  int64_t ldb, void* C, int64_t ldc, nm_dtype dt, bool c_f32, void* ws, cudaStream_t s) {
  static thread_local LtCache lt;
  if (!lt.h) {
    cublasStatus_t r = cublasLtCreate(&lt.h);
    if (r != CUBLAS_STATUS_SUCCESS) return lt_fail(r, "cublasLtCreate");
  }
  if (m == 0 || nn == 0) return NM_OK;
  LtPlan* plan = nullptr;
  for (int i = 0; i < lt.used && !plan; ++i)
    if (lt.plans[i].same(ta, tb, m, nn, k, lda, ldb, ldc, dt, c_f32)) plan = &lt.plans[i];
  if (!plan) {
    LtPlan np;
    np.ta = ta; np.tb = tb; np.c_f32 = c_f32; np.m = m; np.nn = nn; np.k = k;
    np.lda = lda; np.ldb = ldb; np.ldc = ldc; np.dt = dt;
    const cudaDataType_t ty = dt == NM_BF16 ? CUDA_R_16BF : CUDA_R_16F;
    const cudaDataType_t cty = c_f32 ? CUDA_R_32F : ty;
    cublasLtMatmulPreference_t pref = nullptr;
    nm_status st = NM_OK;
    do {
      if (cublasLtMatmulDescCreate(&np.op, CUBLAS_COMPUTE_32F, CUDA_R_32F) != CUBLAS_STATUS_SUCCESS) {
        st = fail(NM_ERR_CUDA, "cublasLtMatmulDescCreate");
        break;
      }
      const cublasOperation_t opa = ta ? CUBLAS_OP_T : CUBLAS_OP_N, opb = tb ? CUBLAS_OP_T : CUBLAS_OP_N;
      cublasLtMatmulDescSetAttribute(np.op, CUBLASLT_MATMUL_DESC_TRANSA, &opa, sizeof(opa));
      cublasLtMatmulDescSetAttribute(np.op, CUBLASLT_MATMUL_DESC_TRANSB, &opb, sizeof(opb));
      if (cublasLtMatrixLayoutCreate(&np.la, ty, ta ? k : m, ta ? m : k, lda) != CUBLAS_STATUS_SUCCESS ||
          cublasLtMatrixLayoutCreate(&np.lb, ty, tb ? nn : k, tb ? k : nn, ldb) != CUBLAS_STATUS_SUCCESS ||
          cublasLtMatrixLayoutCreate(&np.lc, cty, m, nn, ldc) != CUBLAS_STATUS_SUCCESS) {
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
      if (cublasLtMatmulAlgoGetHeuristic(lt.h, np.op, np.la, np.lb, np.lc, np.lc, pref, 1, &heur, &nres) !=
              CUBLAS_STATUS_SUCCESS ||
          nres == 0) {
        st = fail(NM_ERR_CUDA, "cublasLt: no algorithm");
        break;
      }
      np.algo = heur.algo;
    } while (0);
    if (pref) cublasLtMatmulPreferenceDestroy(pref);
    if (st != NM_OK) {
      np.destroy();
      return st;
    }
    // keep it: fill free slots, then replace round-robin
    int slot = lt.used < LtCache::kSlots ? lt.used++ : (lt.next++ % LtCache::kSlots);
    if (slot < lt.used && lt.plans[slot].op) lt.plans[slot].destroy();
    lt.plans[slot] = np;
    plan = &lt.plans[slot];
  }
  const float one = 1.f, zero = 0.f;
  cublasStatus_t r = cublasLtMatmul(lt.h, plan->op, &one, A, plan->la, B, plan->lb, &zero, C, plan->lc, C, plan->lc,
                                    &plan->algo, ws, kLtWorkspace, s);
  if (r != CUBLAS_STATUS_SUCCESS) return lt_fail(r, "cublasLtMatmul");
  return NM_OK;
}

// C[m x nc] = A[m x k] * W[k x nc], all row-major; A, W 16-bit, C 16-bit or fp32: the
// column-major product C^T = W^T A^T (no transposes needed).
nm_status dense_gemm(const void* A, const void* W, void* C, int64_t m, int k, int nc, nm_dtype dt, bool c_f32,
                     void* ws, cudaStream_t s) {
  return lt_gemm(false, false, nc, m, k, W, nc, A, k, C, nc, dt, c_f32, ws, s);
}

// dZ = relu ? dHout * [Hout > 0] : dHout (16-bit in and out, exact), and a 16-bit ones
// vector (the column sums of dZ are a GEMM with it)
__global__ void k_relu_grad(const uint16_t* __restrict__ dHout, const uint16_t* __restrict__ Hout, int64_t total,
                            int relu, uint16_t* __restrict__ dZ) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const uint16_t h = Hout[i];
    // fp16 and bf16 share the sign bit; h > 0 <=> sign clear and not (+0)
    const bool pos = !(h & 0x8000u) && (h & 0x7FFFu);
    dZ[i] = (!relu || pos) ? dHout[i] : (uint16_t)0;
  }
}

__global__ void k_fill16(uint16_t* __restrict__ a, int64_t n, uint16_t v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    a[i] = v;
}

inline int grid_for(int64_t total) {
  int64_t g = (total + 255) / 256;
  if (g > 148 * 16) g = 148 * 16;
  return (int)(g < 1 ? 1 : g);
}

}  // namespace

// row-major C[m x nc] = A[m x k] W[k x nc] (leading dimensions in elements; cuBLASLt, fp32
// accumulation) for the other model layers (models.cu)
nm_status gemm_rm(const void* A, int64_t lda, const void* W, int64_t ldw, void* C, int64_t ldc, int64_t m, int k,
                  int nc, nm_dtype dt, bool c_f32, void* ws, cudaStream_t s) {
  return lt_gemm(false, false, nc, m, k, W, ldw, A, lda, C, ldc, dt, c_f32, ws, s);
}
size_t lt_workspace_bytes() { return kLtWorkspace; }

}  // namespace nm

using namespace nm;

extern "C" size_t nm_gcn_workspace_bytes(int64_t n, int F_in, int F_out) {
  const size_t fmax = (size_t)(F_in > F_out ? F_in : F_out);
  return align256((size_t)n * fmax * 2) + align256((size_t)n * fmax * 4) + align256((size_t)n * F_out * 4) +
         kLtWorkspace;
}

static nm_status gcn_layer_impl(const nm_packed* Ahat, const void* H, const void* W, const float* bias,
                                void* Hout, const DstList* bc, int64_t dst_row0, int F_in, int F_out, int flags,
                                void* ws, size_t ws_bytes, void* stream) {
  if (!Ahat || !H || !W || !(Hout || bc) || !ws) return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer: NULL argument");
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
    if (!bc && Ahat->res_nnz == 0 && Ahat->sptc_format == 1 && (((uintptr_t)Hout) & 3) == 0) {
      // no residual: the tensor-core kernel's epilogue is the last writer of every row, so bias,
      // activation and the 16-bit down-convert run there (no fp32 Y round trip, no extra pass)
      FusedAct fa{Hout, F_out, bias, flags & NM_RELU};
      return launch_spmm_sptc_full(Ahat, buf16, F_out, buf32, F_out, F_out, s, &fa);
    }
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
  if (bc) {
    if (rows > 0) {
      if (bf)
        k_bias_act_bcast<1><<<grid_for(rows * (F_out / 8)), 256, 0, s>>>(pre, rows, F_out, bias, flags & NM_RELU, *bc,
                                                                        dst_row0);
      else
        k_bias_act_bcast<0><<<grid_for(rows * (F_out / 8)), 256, 0, s>>>(pre, rows, F_out, bias, flags & NM_RELU, *bc,
                                                                        dst_row0);
    }
  } else if (bf) {
    k_bias_act<1><<<grid_for(rows * F_out), 256, 0, s>>>(pre, rows, F_out, bias, flags & NM_RELU, (uint16_t*)Hout);
  } else {
    k_bias_act<0><<<grid_for(rows * F_out), 256, 0, s>>>(pre, rows, F_out, bias, flags & NM_RELU, (uint16_t*)Hout);
  }
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

extern "C" nm_status nm_gcn_layer(const nm_packed* Ahat, const void* H, const void* W, const float* bias,
                                  void* Hout, int F_in, int F_out, int flags, void* ws, size_t ws_bytes,
                                  void* stream) {
  return gcn_layer_impl(Ahat, H, W, bias, Hout, nullptr, 0, F_in, F_out, flags, ws, ws_bytes, stream);
}

extern "C" nm_status nm_gcn_layer_bcast(const nm_packed* Ahat, const void* H, const void* W, const float* bias,
                                        void* const* dst, int n_dst, int64_t dst_row0, int F_in, int F_out,
                                        int flags, void* ws, size_t ws_bytes, void* stream) {
  if (!dst || n_dst < 1 || n_dst > kMaxDst)
    return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer_bcast: need 1 <= n_dst <= 16 destination buffers");
  if (dst_row0 < 0) return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer_bcast: dst_row0 < 0");
  DstList bc;
  bc.n = n_dst;
  for (int d = 0; d < n_dst; ++d) {
    if (!dst[d] || ((uintptr_t)dst[d] & 15)) return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer_bcast: NULL or unaligned destination");
    bc.p[d] = (uint16_t*)dst[d];
  }
  for (int d = n_dst; d < kMaxDst; ++d) bc.p[d] = nullptr;
  return gcn_layer_impl(Ahat, H, W, bias, nullptr, &bc, dst_row0, F_in, F_out, flags, ws, ws_bytes, stream);
}

// ---- backward ----------------------------------------------------------
// Z = Ahat (H W) + b, Hout = act(Z).  With dZ = dHout * act'(Z) (act' from Hout > 0 for ReLU):
//   db = 1^T dZ,   dT = Ahat^T dZ = Ahat dZ   (Ahat is symmetric -- the reorder keeps the
//   adjacency symmetric, PAPER.md L69-79 / L725 -- so the same packed matrix serves the
//   backward aggregation),   dW = H^T dT,   dH = dT W^T.
extern "C" size_t nm_gcn_backward_workspace_bytes(int64_t n, int F_in, int F_out) {
  (void)F_in;
  return align256((size_t)n * 2) + 2 * align256((size_t)n * F_out * 2) + align256((size_t)n * F_out * 4) +
         kLtWorkspace;
}

extern "C" nm_status nm_gcn_layer_backward(const nm_packed* Ahat, const void* H, const void* W, const void* Hout,
                                           const void* dHout, void* dH, float* dW, float* db, int F_in, int F_out,
                                           int flags, void* ws, size_t ws_bytes, void* stream) {
  if (!Ahat || !H || !W || !Hout || !dHout || !dW || !ws)
    return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer_backward: NULL argument");
  if (F_in < 1 || F_out < 1 || F_out % 8 != 0 || F_in % 8 != 0)
    return fail(NM_ERR_UNSUPPORTED, "nm_gcn_layer_backward: F_in and F_out must be positive multiples of 8");
  if (flags & ~NM_RELU) return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer_backward: unknown flags");
  if (Ahat->row_map) return fail(NM_ERR_UNSUPPORTED, "nm_gcn_layer_backward: needs a pack in permuted order");
  const int64_t n = Ahat->n;
  if (Ahat->row_begin != 0 || Ahat->row_end != n)
    return fail(NM_ERR_UNSUPPORTED, "nm_gcn_layer_backward: needs the whole matrix (Ahat^T = Ahat), not a row shard");
  if (ws_bytes < nm_gcn_backward_workspace_bytes(n, F_in, F_out))
    return fail(NM_ERR_INVALID_ARG, "nm_gcn_layer_backward: workspace too small");
  if (n == 0) return NM_OK;
  cudaStream_t s = (cudaStream_t)stream;
  const nm_dtype dt = Ahat->dtype;
  uint8_t* w8 = (uint8_t*)ws;
  uint16_t* ones = (uint16_t*)w8;
  uint16_t* dZ = (uint16_t*)(w8 + align256((size_t)n * 2));
  float* dT32 = (float*)((uint8_t*)dZ + align256((size_t)n * F_out * 2));
  uint16_t* dT16 = (uint16_t*)((uint8_t*)dT32 + align256((size_t)n * F_out * 4));
  void* lt_ws = (uint8_t*)dT16 + align256((size_t)n * F_out * 2);
  const int64_t tot = n * F_out;
  k_relu_grad<<<grid_for(tot), 256, 0, s>>>((const uint16_t*)dHout, (const uint16_t*)Hout, tot, flags & NM_RELU, dZ);
  NM_CUDA(cudaGetLastError());
  nm_status st;
  if (db) {  // db[1 x F_out] = ones[1 x n] dZ[n x F_out]
    k_fill16<<<grid_for(n), 256, 0, s>>>(ones, n, dt == NM_BF16 ? (uint16_t)0x3F80u : (uint16_t)0x3C00u);
    NM_CUDA(cudaGetLastError());
    st = dense_gemm(ones, dZ, db, 1, (int)n, F_out, dt, true, lt_ws, s);
    if (st != NM_OK) return st;
  }
  st = nm_spmm(Ahat, dZ, F_out, dT32, F_out, F_out, stream);  // dT = Ahat dZ
  if (st != NM_OK) return st;
  if (dt == NM_BF16) k_to16<1><<<grid_for(tot), 256, 0, s>>>(dT32, tot, dT16);
  else k_to16<0><<<grid_for(tot), 256, 0, s>>>(dT32, tot, dT16);
  NM_CUDA(cudaGetLastError());
  // column-major views: row-major X[r x c] is X^c[c x r].  dW^c[F_out x F_in] = dT^c H^c^T
  st = lt_gemm(false, true, F_out, F_in, n, dT16, F_out, H, F_in, dW, F_out, dt, true, lt_ws, s);
  if (st != NM_OK) return st;
  if (dH) {  // dH^c[F_in x n] = W^c^T dT^c
    st = lt_gemm(true, false, F_in, n, F_out, W, F_out, dT16, F_out, dH, F_in, dt, false, lt_ws, s);
    if (st != NM_OK) return st;
  }
  return NM_OK;
}
