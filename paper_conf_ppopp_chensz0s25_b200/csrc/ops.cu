// Residual CSR SpMM (keeps the result lossless), X-row permutation / Y-row unpermutation
// (Fig. 1 caption) and the nm_spmm entry points.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <algorithm>
#include <mutex>

#include "nm_internal.h"

#ifndef NM_RES_UNROLL
#define NM_RES_UNROLL 2  // X rows in flight per lane in k_residual (measured: 2 >= 4 >> 8)
#endif

namespace nm {
namespace {

// c + a * b with a, b 16-bit (fp16 or bf16 bits) and c fp32: one mixed-precision FMA
// (FHFMA; the product of two 16-bit values is exact in fp32, so this equals converting both
// and using an fp32 FMA)
template <int BF>
__device__ __forceinline__ float fma16(unsigned short a, unsigned short b, float c) {
  float d;
  if (BF)
    asm("fma.rn.f32.bf16 %0, %1, %2, %3;" : "=f"(d) : "h"(a), "h"(b), "f"(c));
  else
    asm("fma.rn.f32.f16 %0, %1, %2, %3;" : "=f"(d) : "h"(a), "h"(b), "f"(c));
  return d;
}

// Yp[l][f] += sum_k res_val[k] * PX[res_col[k]][f]  (the residual CSR, lossless remainder).
// Work items (ResSeg) hold <= kResSeg nonzeros of one row.  A warp is SUB = 32 / LPR
// subgroups of LPR lanes and every subgroup runs its own items (items w*SUB + sub, ...), so a
// warp has SUB independent items -- each a chain of dependent memory round trips -- in
// flight; a lane owns 8 consecutive features of the launch's slab [f_base, f_base + LPR*8)
// and reads them with one 16-byte load per nonzero.  The item's (col, val) pairs are fetched
// LPR at a time with one coalesced load and broadcast within the subgroup by shuffles; the
// loop is unrolled so kUnroll X rows are in flight per lane (2: more costs occupancy).  The next item's descriptor is
// prefetched, and the Y row (addressed by the item's output row, row_map applied at pack
// time) is read next to the first (col, val) batch.  A row with one item adds its sum into Y;
// the items of a split row (hub rows) write partials to their workspace slots and the last
// one to arrive (per-row counter) adds the partials in item order -- deterministic, no float
// atomics.  The workspace and counters are the calling nm_spmm's own (stream-ordered
// allocation, counters zeroed per call), so the packed handle is only read.  F tail: the 16-byte vector at column f < F is inside the row (ldx % 8 == 0), only
// the accumulate/store is masked.
#ifndef NM_RES_CPASYNC
#define NM_RES_CPASYNC 1  // X rows via cp.async into a per-subgroup shared-memory ring (0: registers)
#endif
#ifndef NM_RES_BATCH
#define NM_RES_BATCH 8
#endif
#ifdef NM_RES_MINB  // tuning experiments: minimum resident CTAs per SM for k_residual
#define NM_RES_BOUNDS __launch_bounds__(256, NM_RES_MINB)
#else
#define NM_RES_BOUNDS __launch_bounds__(256)
#endif
constexpr int kResBatch = NM_RES_BATCH;  // entries per cp.async batch (two batches in flight per subgroup)

template <int LPR>
constexpr int res_smem_bytes() {
  return NM_RES_CPASYNC ? 8 * (32 / LPR) * 2 * (LPR < kResBatch ? LPR : kResBatch) * LPR * 16 : 0;
}

__device__ __forceinline__ void cp_async16_z(uint32_t dst, const void* src, uint32_t nbytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(nbytes) : "memory");
}

template <int BF, int LPR>
__global__ void NM_RES_BOUNDS k_residual(const ResSeg* __restrict__ segs, int64_t n_segs,
                                                  const int32_t* __restrict__ rc, const uint16_t* __restrict__ rv,
                                                  const uint16_t* __restrict__ X, int64_t ldx,
                                                  float* __restrict__ Y, int64_t ldy, int F, int f_base,
                                                  float* __restrict__ ws, int32_t* __restrict__ cnt) {
  constexpr int SUB = 32 / LPR;
  constexpr int kUnroll = NM_RES_UNROLL;
  constexpr int KB = LPR < kResBatch ? LPR : kResBatch;
  extern __shared__ __align__(16) uint8_t res_smem[];
  const int lane = threadIdx.x & 31;
  const int sub = lane / LPR, li = lane % LPR;
  const unsigned gmask = LPR == 32 ? 0xffffffffu : (((1u << LPR) - 1u) << (sub * LPR));
  const int f = f_base + li * 8;  // first feature of this lane
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5) * SUB;  // subgroups in the grid
  const bool vec_y = ((ldy & 3) == 0) && ((((uintptr_t)Y) & 15) == 0) && f + 8 <= F;
  // this lane's slots of its subgroup's ring: slot (batch parity b, entry j) at
  // ring + ((b * KB + j) * LPR) * 16 (a lane reads back only the pieces it copied itself, so
  // cp.async.wait_group is all the synchronisation the ring needs)
  const uint32_t ring = (uint32_t)__cvta_generic_to_shared(res_smem) +
                        (uint32_t)((((threadIdx.x >> 5) * SUB + sub) * 2 * KB * LPR + li) * 16);
  const uint32_t xbytes = f < F ? 16u : 0u;
  int64_t w = ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5) * SUB + sub;
  ResSeg gn;
  if (w < n_segs) gn = segs[w];
  for (; w < n_segs; w += nw) {
    const ResSeg g = gn;
    if (w + nw < n_segs) gn = segs[w + nw];  // next item's descriptor, ahead of use
    float* y = Y + (int64_t)g.yrow * ldy + f;
    // single-item rows: the Y row comes in with the first (col, val) batch
    float4 y0 = make_float4(0.f, 0.f, 0.f, 0.f), y1 = y0;
    const bool early_y = g.slot < 0 && vec_y;
    if (early_y) {
      y0 = __ldcs((const float4*)y);
      y1 = __ldcs((const float4*)(y + 4));
    }
    float acc[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[q] = 0.f;
#if NM_RES_CPASYNC
    // two batches of KB entries in flight: batch k+1's X rows are copied (cp.async, no
    // registers held) while batch k is accumulated from shared memory.  Both loops have a fixed
    // trip count (KB): entries past the item's end are zero-filled copies (ignore-src) with a
    // zero value, so the batch needs no per-entry branch and no divergent shuffles.
    const int nb = (g.len + KB - 1) / KB;
    int32_t cn = 0;
    uint32_t vn = 0u, vc = 0u;
    if (li < KB && li < g.len) {
      cn = __ldg(rc + g.kb + li);  // streamed once
      vn = __ldg(rv + g.kb + li);
    }
#pragma unroll
    for (int j = 0; j < KB; ++j) {  // issue batch 0
      const int32_t cc = __shfl_sync(gmask, cn, j, LPR);
      cp_async16_z(ring + j * LPR * 16, X + (int64_t)cc * ldx + (xbytes ? f : 0), j < g.len ? xbytes : 0u);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    for (int k = 0; k < nb; ++k) {
      vc = vn;
      if (k + 1 < nb) {
        const int e1 = (k + 1) * KB;
        cn = 0;
        vn = 0u;
        if (li < KB && e1 + li < g.len) {
          cn = __ldg(rc + g.kb + e1 + li);
          vn = __ldg(rv + g.kb + e1 + li);
        }
        const uint32_t rb = ring + ((k + 1) & 1) * KB * LPR * 16;
#pragma unroll
        for (int j = 0; j < KB; ++j) {
          const int32_t cc = __shfl_sync(gmask, cn, j, LPR);
          cp_async16_z(rb + j * LPR * 16, X + (int64_t)cc * ldx + (xbytes ? f : 0), e1 + j < g.len ? xbytes : 0u);
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 1;" ::: "memory");
      } else {
        asm volatile("cp.async.wait_group 0;" ::: "memory");
      }
      const uint32_t rb = ring + (k & 1) * KB * LPR * 16;
#pragma unroll
      for (int j = 0; j < KB; ++j) {
        const unsigned short a = (unsigned short)__shfl_sync(gmask, vc, j, LPR);
        uint32_t wv[4];
        asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(wv[0]), "=r"(wv[1]), "=r"(wv[2]), "=r"(wv[3])
                     : "r"(rb + j * LPR * 16));
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          acc[2 * q] = fma16<BF>(a, (unsigned short)(wv[q] & 0xFFFFu), acc[2 * q]);
          acc[2 * q + 1] = fma16<BF>(a, (unsigned short)(wv[q] >> 16), acc[2 * q + 1]);
        }
      }
    }
#else
    for (int base = 0; base < g.len; base += LPR) {
      const int cnt_ = min(LPR, g.len - base);
      int32_t c = 0;
      uint32_t v = 0u;  // 16-bit value bits (a zero value adds exact zeros)
      if (li < cnt_) {
        c = __ldg(rc + g.kb + base + li);
        v = __ldg(rv + g.kb + base + li);
      }
      for (int j = 0; j < cnt_; j += kUnroll) {
        uint4 xv[kUnroll];
        uint32_t vv[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const int idx = j + u;
          const int32_t cc = __shfl_sync(gmask, c, idx & (LPR - 1), LPR);
          vv[u] = __shfl_sync(gmask, v, idx & (LPR - 1), LPR);
          if (idx < cnt_ && f < F) {
            xv[u] = __ldg((const uint4*)(X + (int64_t)cc * ldx + f));
          } else {
            xv[u] = make_uint4(0u, 0u, 0u, 0u);
            vv[u] = 0u;
          }
        }
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const uint32_t wv[4] = {xv[u].x, xv[u].y, xv[u].z, xv[u].w};
          const unsigned short a = (unsigned short)vv[u];
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            acc[2 * q] = fma16<BF>(a, (unsigned short)(wv[q] & 0xFFFFu), acc[2 * q]);
            acc[2 * q + 1] = fma16<BF>(a, (unsigned short)(wv[q] >> 16), acc[2 * q + 1]);
          }
        }
      }
    }
#endif
    if (early_y) {
      y0.x += acc[0]; y0.y += acc[1]; y0.z += acc[2]; y0.w += acc[3];
      y1.x += acc[4]; y1.y += acc[5]; y1.z += acc[6]; y1.w += acc[7];
      __stcs((float4*)y, y0);
      __stcs((float4*)(y + 4), y1);
      continue;
    }
    if (g.slot >= 0) {
      // split row: publish this item's partial, the last arrival reduces in item order
      float* part = ws + ((int64_t)(g.slot + g.idx) * (LPR * 8)) + li * 8;
      *(float4*)part = make_float4(acc[0], acc[1], acc[2], acc[3]);
      *(float4*)(part + 4) = make_float4(acc[4], acc[5], acc[6], acc[7]);
      __threadfence();
      __syncwarp(gmask);
      int last = 0;
      if (li == 0) last = atomicAdd(cnt + g.split_id, 1) == g.nseg - 1;
      last = __shfl_sync(gmask, last, 0, LPR);
      if (!last) continue;
      __threadfence();
#pragma unroll
      for (int q = 0; q < 8; ++q) acc[q] = 0.f;
      // the partials in item order, kUnroll loads in flight per lane
      for (int i0 = 0; i0 < g.nseg; i0 += kUnroll) {
        float4 pa[kUnroll], pb[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const int i = i0 + u;
          pa[u] = pb[u] = make_float4(0.f, 0.f, 0.f, 0.f);
          if (i < g.nseg) {
            const float* pi = ws + ((int64_t)(g.slot + i) * (LPR * 8)) + li * 8;
            pa[u] = __ldcg((const float4*)pi);
            pb[u] = __ldcg((const float4*)(pi + 4));
          }
        }
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          acc[0] += pa[u].x; acc[1] += pa[u].y; acc[2] += pa[u].z; acc[3] += pa[u].w;
          acc[4] += pb[u].x; acc[5] += pb[u].y; acc[6] += pb[u].z; acc[7] += pb[u].w;
        }
      }
    }
    if (f < F) {
      if (vec_y) {
        float4 a0 = *(float4*)y, a1 = *(float4*)(y + 4);
        a0.x += acc[0]; a0.y += acc[1]; a0.z += acc[2]; a0.w += acc[3];
        a1.x += acc[4]; a1.y += acc[5]; a1.z += acc[6]; a1.w += acc[7];
        *(float4*)y = a0;
        *(float4*)(y + 4) = a1;
      } else {
#pragma unroll
        for (int q = 0; q < 8; ++q)
          if (f + q < F) y[q] += acc[q];
      }
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
  if (ldx > INT32_MAX) return fail(NM_ERR_UNSUPPORTED, "nm_spmm: ldx must fit in 32 bits");
  if (ldx % 8 != 0 || ((uintptr_t)PX & 15) != 0)
    return fail(NM_ERR_INVALID_ARG, "nm_spmm: PX rows must be 16-byte aligned (ldx % 8 == 0)");
  return NM_OK;
}

}  // namespace

// Tensor-core part: the full-record kernel (spmm_full_sm100.cu) or the compressed-record one
// (spmm_sm100.cu).  format 0 = the pack's choice (nm_packed::sptc_format), 1 = full,
// 2 = compressed.
nm_status launch_spmm_sptc(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                           cudaStream_t s, int format) {
  if (format == 0) format = P->sptc_format;
  if (format == 2) return launch_spmm_sptc_compressed(P, PX, ldx, Yp, ldy, F, s);
  if (format == 3) return launch_spmm_sptc_tm(P, PX, ldx, Yp, ldy, F, s);
  return launch_spmm_sptc_full(P, PX, ldx, Yp, ldy, F, s);
}

// Per-device pool for the per-call residual workspace: allocations are stream-ordered (so calls
// on different streams never share a buffer) and the pool keeps its memory between calls (the
// device's default pool releases at every synchronisation, which made a large workspace cost a
// fresh device allocation per call: C3 at tau = 8 spent 5 ms of its 6.3 ms residual there).
// Library state, not handle state: the packed handle stays immutable.
nm_status workspace_pool(cudaMemPool_t* out) {
  static std::mutex mu;
  static cudaMemPool_t pools[64] = {};
  int dev = 0;
  NM_CUDA(cudaGetDevice(&dev));
  if (dev < 0 || dev >= 64) return fail(NM_ERR_UNSUPPORTED, "workspace_pool: device id >= 64");
  std::lock_guard<std::mutex> lock(mu);
  if (!pools[dev]) {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.handleTypes = cudaMemHandleTypeNone;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    NM_CUDA(cudaMemPoolCreate(&pools[dev], &props));
    uint64_t keep = UINT64_MAX;
    NM_CUDA(cudaMemPoolSetAttribute(pools[dev], cudaMemPoolAttrReleaseThreshold, &keep));
  }
  *out = pools[dev];
  return NM_OK;
}

nm_status launch_spmm_residual(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                               cudaStream_t s) {
  const int64_t rows = P->row_end - P->row_begin;
  if (P->res_nnz == 0 || rows == 0) return NM_OK;
  const int32_t* rcol = P->res_gather ? P->res_gather : P->res_col;
  // lanes per item: 8 features per lane; one launch per slab of LPR * 8 features
  const int lpr = F <= 32 ? 4 : F <= 64 ? 8 : F <= 128 ? 16 : 32;
  const int bf = P->dtype == NM_BF16;
  const int sub_per_warp = 32 / lpr;
  int64_t g = (P->n_res_segs + 8 * sub_per_warp - 1) / (8 * sub_per_warp);
  if (g > 148 * 16) g = 148 * 16;
  // this call's split-row workspace: partial-sum slots + arrival counters (one set per slab
  // launch, so the counters need no reset between the launches of one call)
  const int nslab = (F + lpr * 8 - 1) / (lpr * 8);
  float* ws = nullptr;
  int32_t* cnt = nullptr;
  if (P->n_res_split > 0) {
    cudaMemPool_t pool;
    NM_TRY_STATUS(workspace_pool(&pool));
    NM_CUDA(cudaMallocFromPoolAsync((void**)&ws, sizeof(float) * lpr * 8 * P->n_res_slots, pool, s));
    cudaError_t e = cudaMallocFromPoolAsync((void**)&cnt, sizeof(int32_t) * P->n_res_split * nslab, pool, s);
    if (e != cudaSuccess) {
      cudaFreeAsync(ws, s);
      return cuda_fail(e, "cudaMallocAsync(residual counters)");
    }
    e = cudaMemsetAsync(cnt, 0, sizeof(int32_t) * P->n_res_split * nslab, s);
    if (e != cudaSuccess) {
      cudaFreeAsync(ws, s);
      cudaFreeAsync(cnt, s);
      return cuda_fail(e, "cudaMemsetAsync(residual counters)");
    }
  }
#define NM_RES_LAUNCH(BF, LPR)                                                                              \
  do {                                                                                                      \
    static bool attr_set = false;                                                                           \
    if (!attr_set && res_smem_bytes<LPR>() > 48 * 1024) {                                                   \
      cudaFuncSetAttribute(k_residual<BF, LPR>, cudaFuncAttributeMaxDynamicSharedMemorySize,                \
                           res_smem_bytes<LPR>());                                                          \
      attr_set = true;                                                                                      \
    }                                                                                                       \
    k_residual<BF, LPR><<<(unsigned)g, 256, res_smem_bytes<LPR>(), s>>>(                                    \
        P->res_segs, P->n_res_segs, rcol, P->res_val, (const uint16_t*)PX, ldx, Yp, ldy, F, f_base, ws,     \
        cnt ? cnt + P->n_res_split * (f_base / (lpr * 8)) : nullptr);                                       \
  } while (0)
  for (int f_base = 0; f_base < F; f_base += lpr * 8) {
    switch (lpr * 2 + bf) {
      case 8: NM_RES_LAUNCH(0, 4); break;
      case 9: NM_RES_LAUNCH(1, 4); break;
      case 16: NM_RES_LAUNCH(0, 8); break;
      case 17: NM_RES_LAUNCH(1, 8); break;
      case 32: NM_RES_LAUNCH(0, 16); break;
      case 33: NM_RES_LAUNCH(1, 16); break;
      case 64: NM_RES_LAUNCH(0, 32); break;
      default: NM_RES_LAUNCH(1, 32); break;
    }
  }
#undef NM_RES_LAUNCH
  const cudaError_t le = cudaGetLastError();
  if (ws) cudaFreeAsync(ws, s);
  if (cnt) cudaFreeAsync(cnt, s);
  if (le != cudaSuccess) return cuda_fail(le, "k_residual launch");
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
  return launch_spmm_sptc(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream, 0);
}

nm_status nm_spmm_sptc_format(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                              int format, void* stream) {
  nm_status st = check_spmm_args(P, PX, ldx, Yp, ldy, F);
  if (st != NM_OK) return st;
  if (format < 0 || format > 3) return fail(NM_ERR_INVALID_ARG, "nm_spmm_sptc_format: format must be 0, 1, 2 or 3");
  return launch_spmm_sptc(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream, format);
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
  st = launch_spmm_sptc(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream, 0);
  if (st != NM_OK) return st;
  return launch_spmm_residual(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
}

}  // extern "C"
