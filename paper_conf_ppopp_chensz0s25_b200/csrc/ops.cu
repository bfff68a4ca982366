// Residual CSR SpMM (keeps the result lossless), X-row permutation / Y-row unpermutation
// (Fig. 1 caption) and the nm_spmm entry points.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "nm_internal.h"

namespace nm {
namespace {

__device__ __forceinline__ float h2f(uint16_t b, int bf) {
  if (bf) return __uint_as_float(((uint32_t)b) << 16);
  __half h;
  *(uint16_t*)&h = b;
  return __half2float(h);
}

// Yp[l][f] += sum_k res_val[k] * PX[res_col[k]][f] -- one warp per row, 4 columns per lane
// per pass (8-byte loads of 4 halves), fp32 accumulation.
template <int BF>
__global__ void __launch_bounds__(256) k_residual(const int64_t* __restrict__ rp, const int32_t* __restrict__ rc,
                                                  const uint16_t* __restrict__ rv, int64_t rows,
                                                  const int32_t* __restrict__ row_map,
                                                  const uint16_t* __restrict__ X, int64_t ldx,
                                                  float* __restrict__ Y, int64_t ldy, int F) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t l = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; l < rows; l += nw) {
    const int64_t b = rp[l], e = rp[l + 1];
    if (b == e) continue;
    for (int f0 = 0; f0 < F; f0 += 128) {
      const int f = f0 + lane * 4;
      float a0 = 0.f, a1 = 0.f, a2 = 0.f, a3 = 0.f;
      for (int64_t k = b; k < e; ++k) {
        const float v = h2f(rv[k], BF);
        const uint16_t* x = X + (int64_t)rc[k] * ldx + f;
        if (f + 3 < F) {
          uint2 q = *(const uint2*)x;
          a0 += v * h2f((uint16_t)(q.x & 0xFFFF), BF);
          a1 += v * h2f((uint16_t)(q.x >> 16), BF);
          a2 += v * h2f((uint16_t)(q.y & 0xFFFF), BF);
          a3 += v * h2f((uint16_t)(q.y >> 16), BF);
        } else {
          if (f < F) a0 += v * h2f(x[0], BF);
          if (f + 1 < F) a1 += v * h2f(x[1], BF);
          if (f + 2 < F) a2 += v * h2f(x[2], BF);
        }
      }
      float* y = Y + (row_map ? (int64_t)row_map[l] : l) * ldy + f;
      if (f < F) y[0] += a0;
      if (f + 1 < F) y[1] += a1;
      if (f + 2 < F) y[2] += a2;
      if (f + 3 < F) y[3] += a3;
    }
  }
}

// dst[p] = src[idx[p]] (gather) or dst[idx[p]] = src[p] (scatter); row bytes copied with
// 16-byte vectors when aligned.  One warp per row.
template <bool SCATTER>
__global__ void __launch_bounds__(256) k_permute(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst,
                                                 const int32_t* __restrict__ idx, int64_t n,
                                                 int64_t row_bytes, int64_t ld_bytes, int vec16) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t p = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; p < n; p += nw) {
    const int64_t q = idx[p];
    const uint8_t* s = src + (SCATTER ? p : q) * ld_bytes;
    uint8_t* d = dst + (SCATTER ? q : p) * ld_bytes;
    if (vec16) {
      for (int64_t o = lane * 16; o < row_bytes; o += 32 * 16)
        *(uint4*)(d + o) = __ldg((const uint4*)(s + o));
    } else {
      for (int64_t o = lane * 2; o < row_bytes; o += 64) *(uint16_t*)(d + o) = *(const uint16_t*)(s + o);
    }
  }
}

int grid_rows(int64_t rows, int warps_per_block) {
  int64_t g = (rows + warps_per_block - 1) / warps_per_block;
  if (g > 148 * 32) g = 148 * 32;
  return (int)(g < 1 ? 1 : g);
}

nm_status permute_impl(const void* src, void* dst, const int32_t* perm, int64_t n, int F, int64_t ld,
                       nm_dtype dt, cudaStream_t s, bool scatter) {
  if (!src || !dst || !perm) return fail(NM_ERR_INVALID_ARG, "permute: NULL pointer");
  if (src == dst) return fail(NM_ERR_INVALID_ARG, "permute: in-place not supported");
  if (n < 0 || F < 0 || ld < F) return fail(NM_ERR_INVALID_ARG, "permute: bad sizes");
  if (n == 0 || F == 0) return NM_OK;
  const int64_t esz = dt == NM_F32 ? 4 : 2;
  const int64_t row_bytes = F * esz, ld_bytes = ld * esz;
  const int vec16 = (row_bytes % 16 == 0) && (ld_bytes % 16 == 0) && (((uintptr_t)src & 15) == 0) &&
                    (((uintptr_t)dst & 15) == 0);
  if (scatter)
    k_permute<true><<<grid_rows(n, 8), 256, 0, s>>>((const uint8_t*)src, (uint8_t*)dst, perm, n, row_bytes,
                                                    ld_bytes, vec16);
  else
    k_permute<false><<<grid_rows(n, 8), 256, 0, s>>>((const uint8_t*)src, (uint8_t*)dst, perm, n, row_bytes,
                                                     ld_bytes, vec16);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

nm_status check_spmm_args(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F) {
  if (!P || !PX || !Yp) return fail(NM_ERR_INVALID_ARG, "nm_spmm: NULL argument");
  if (F < 1 || F > 4096) return fail(NM_ERR_UNSUPPORTED, "nm_spmm: F must be in [1, 4096]");
  if (ldx < F || ldy < F) return fail(NM_ERR_INVALID_ARG, "nm_spmm: leading dimension < F");
  if (ldx % 8 != 0 || ((uintptr_t)PX & 15) != 0)
    return fail(NM_ERR_INVALID_ARG, "nm_spmm: PX rows must be 16-byte aligned (ldx % 8 == 0)");
  return NM_OK;
}

}  // namespace

nm_status launch_spmm_residual(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                               cudaStream_t s) {
  const int64_t rows = P->row_end - P->row_begin;
  if (P->res_nnz == 0 || rows == 0) return NM_OK;
  const int32_t* rcol = P->res_gather ? P->res_gather : P->res_col;
  if (P->dtype == NM_BF16)
    k_residual<1><<<grid_rows(rows, 8), 256, 0, s>>>(P->res_rowptr, rcol, P->res_val, rows, P->row_map,
                                                     (const uint16_t*)PX, ldx, Yp, ldy, F);
  else
    k_residual<0><<<grid_rows(rows, 8), 256, 0, s>>>(P->res_rowptr, rcol, P->res_val, rows, P->row_map,
                                                     (const uint16_t*)PX, ldx, Yp, ldy, F);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

}  // namespace nm

using namespace nm;

extern "C" {

nm_status nm_permute_rows(const void* X, void* PX, const int32_t* perm_dev, int64_t n, int F, int64_t ld,
                          nm_dtype dtype, void* stream) {
  return permute_impl(X, PX, perm_dev, n, F, ld, dtype, (cudaStream_t)stream, false);
}

nm_status nm_unpermute_rows(const void* Yp, void* Y, const int32_t* perm_dev, int64_t n, int F, int64_t ld,
                            nm_dtype dtype, void* stream) {
  return permute_impl(Yp, Y, perm_dev, n, F, ld, dtype, (cudaStream_t)stream, true);
}

nm_status nm_spmm_sptc(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                       void* stream) {
  nm_status st = check_spmm_args(P, PX, ldx, Yp, ldy, F);
  if (st != NM_OK) return st;
  return launch_spmm_sptc(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
}

nm_status nm_spmm_residual(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                           void* stream) {
  nm_status st = check_spmm_args(P, PX, ldx, Yp, ldy, F);
  if (st != NM_OK) return st;
  return launch_spmm_residual(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
}

nm_status nm_spmm(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                  void* stream) {
  nm_status st = check_spmm_args(P, PX, ldx, Yp, ldy, F);
  if (st != NM_OK) return st;
  st = launch_spmm_sptc(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
  if (st != NM_OK) return st;
  return launch_spmm_residual(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
}

}  // extern "C"
