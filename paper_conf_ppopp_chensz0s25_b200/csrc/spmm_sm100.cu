// nm_spmm tensor-core part: Yp = B_packed * PX on sm_100a sparse tensor cores.
//
// One work unit = (panel of 128 rows of B, 64..256-column tile of F).  The K dimension of a
// panel is its list of non-empty meta-blocks; 8 meta-blocks (4 selected columns each) form
// one K = 32 chunk, i.e. one tcgen05.mma.sp.cta_group::1.kind::f16 with M = 128, N = BN:
//   record (A values, 2:4 metadata, 32 gather rows; 4736 B) <- one cp.async.bulk (HBM stream)
//   B (32 gathered rows of X x BN, SWIZZLE_128B MN-major)  <- TMA tile::gather4, 4 rows each
//   E (metadata, 128 lanes x 32 b)                          <- tcgen05.st from shared memory
//   D (fp32, 128 x BN)                                      in tensor memory (tcgen05.ld out)
// Warp roles (persistent, one CTA per SM, 11 warps):
//   w0 record TMA | w1 gather4 TMA | w2-5 metadata -> TMEM | w6 MMA issuer (+TMEM alloc)
//   | w7-10 epilogue (TMEM -> registers -> Y).  All hand-offs are mbarriers; the pipeline
//   runs across work units, so consecutive panels overlap.  Layouts measured on B200:
//   tools/probes/probe_umma_sp.b200.txt, tools/probes/probe_gather4.b200.txt.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <mutex>

#include "nm_internal.h"

namespace nm {
namespace {

constexpr int kThreads = 352;
constexpr int kWarpRec = 0, kWarpGather = 1, kWarpMeta0 = 2, kWarpMma = 6;

struct SpmmParams {
  const uint8_t* image;
  const int64_t* panel_chunk_ptr;
  const int32_t* unit_order;
  const int32_t* row_map;  // nullable: output row of Y for packed row l
  float* Y;
  int64_t ldy;
  int F;
  int64_t rows;
  int64_t n_units;
  int n_ftiles;
  uint32_t idesc;
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t a, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count));
}

__device__ __forceinline__ void mbar_wait(uint32_t a, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P;\n"
      "NM_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra NM_WAIT_%=;\n\t}" ::"r"(a),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint32_t a) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(a) : "memory");
}

__device__ __forceinline__ void mbar_arrive_tx(uint32_t a, uint32_t tx) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(tx) : "memory");
}

__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t mbar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
      "l"(src), "r"(bytes), "r"(mbar)
      : "memory");
}

__device__ __forceinline__ void gather4(uint32_t dst, const CUtensorMap* tm, int col, int r0, int r1, int r2, int r3,
                                        uint32_t mbar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(dst),
      "l"(tm), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(mbar)
      : "memory");
}

__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;  // sm_100 descriptor version
  d |= (uint64_t)layout << 61;
  return d;
}

template <int BN>
struct Cfg {
  static constexpr int kRecBytes = kChunkBytes;                 // 4736
  static constexpr int kBBytes = 32 * BN * 2;                   // 32 K-rows x BN halves
  static constexpr int kStageBytes = kRecBytes + kBBytes;
  static constexpr int kStagesRaw = (216 * 1024) / kStageBytes;
  static constexpr int kStages = kStagesRaw > 16 ? 16 : kStagesRaw;
  static constexpr int kNAcc = (2 * BN + kStages <= 512) ? 2 : 1;
  static constexpr int kMeta0 = kNAcc * BN;                     // metadata column of stage s: kMeta0 + s
  static constexpr int kRecRegion = ((kStages * kRecBytes + 1023) / 1024) * 1024;
  static constexpr int kSmem = 1024 + kRecRegion + kStages * kBBytes + 1024;
  static_assert(kMeta0 + kStages <= 512, "TMEM budget");
  static_assert(BN % 64 == 0 && BN >= 64 && BN <= 256, "BN");
  static_assert(kSmem <= 227 * 1024, "smem");
};

template <int BN>
__global__ void __launch_bounds__(kThreads, 1) k_spmm_sptc(const SpmmParams p, const __grid_constant__ CUtensorMap tmX) {
  using C = Cfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sRec = smem;                       // kStages records (16-byte aligned)
  uint8_t* sB = smem + C::kRecRegion;         // kStages B tiles (1024-aligned)
  uint64_t* bars = (uint64_t*)(sB + C::kStages * C::kBBytes);
  uint64_t* full_a = bars;                    // record landed (tx)
  uint64_t* full_b = bars + C::kStages;       // gathers landed (tx)
  uint64_t* meta_ok = bars + 2 * C::kStages;  // metadata in TMEM (128 arrivals)
  uint64_t* empty = bars + 3 * C::kStages;    // MMA done with the stage (tcgen05.commit)
  uint64_t* tfull = bars + 4 * C::kStages;    // accumulator ready (2)
  uint64_t* tempty = tfull + 2;               // accumulator drained (2)
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::kStages; ++s) {
      mbar_init(smem_u32(&full_a[s]), 1);
      mbar_init(smem_u32(&full_b[s]), 1);
      mbar_init(smem_u32(&meta_ok[s]), 128);
      mbar_init(smem_u32(&empty[s]), 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(smem_u32(&tfull[a]), 1);
      mbar_init(smem_u32(&tempty[a]), 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kWarpGather && lane == 0) asm volatile("prefetch.tensormap [%0];" ::"l"(&tmX) : "memory");
  if (warp == kWarpMma) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tmem_slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tbase = *tmem_slot;

  if (warp == kWarpRec) {
    // ------------------------------------------------------------ record producer (HBM stream)
    if (lane == 0) {
      int64_t i = 0;
      for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
        const int32_t panel = p.unit_order[u / p.n_ftiles];
        const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
        for (int64_t c = c0; c < c1; ++c, ++i) {
          const int s = (int)(i % C::kStages);
          const uint32_t ph = (uint32_t)((i / C::kStages) & 1);
          mbar_wait(smem_u32(&empty[s]), ph ^ 1);
          mbar_arrive_tx(smem_u32(&full_a[s]), C::kRecBytes);
          bulk_g2s(smem_u32(sRec + s * C::kRecBytes), p.image + c * kChunkBytes, C::kRecBytes, smem_u32(&full_a[s]));
        }
      }
    }
  } else if (warp == kWarpGather) {
    // ------------------------------------------------------------ X gathers (TMA gather4)
    int64_t i = 0;
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int ft = (int)(u % p.n_ftiles);
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      for (int64_t c = c0; c < c1; ++c, ++i) {
        const int s = (int)(i % C::kStages);
        const uint32_t ph = (uint32_t)((i / C::kStages) & 1);
        mbar_wait(smem_u32(&full_a[s]), ph);
        const int32_t xr = *(const int32_t*)(sRec + s * C::kRecBytes + kChunkXrowOff + 4 * lane);
        const int g = lane & 7;
        const int r0 = __shfl_sync(0xffffffffu, xr, 4 * g + 0);
        const int r1 = __shfl_sync(0xffffffffu, xr, 4 * g + 1);
        const int r2 = __shfl_sync(0xffffffffu, xr, 4 * g + 2);
        const int r3 = __shfl_sync(0xffffffffu, xr, 4 * g + 3);
        if (lane == 0) mbar_arrive_tx(smem_u32(&full_b[s]), C::kBBytes);
        __syncwarp();
        if (lane < 8) {
          const uint32_t dst = smem_u32(sB + s * C::kBBytes) + (g >> 1) * 1024 + (g & 1) * 512;
#pragma unroll
          for (int nc = 0; nc < BN / 64; ++nc)
            gather4(dst + nc * 4096, &tmX, ft * BN + nc * 64, r0, r1, r2, r3, smem_u32(&full_b[s]));
        }
        __syncwarp();
      }
    }
  } else if (warp >= kWarpMeta0 && warp < kWarpMeta0 + 4) {
    // ------------------------------------------------------------ 2:4 metadata -> TMEM
    const int quarter = warp & 3;
    const int L = quarter * 32 + lane;
    int64_t i = 0;
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      for (int64_t c = c0; c < c1; ++c, ++i) {
        const int s = (int)(i % C::kStages);
        const uint32_t ph = (uint32_t)((i / C::kStages) & 1);
        mbar_wait(smem_u32(&full_a[s]), ph);
        const uint32_t w = *(const uint32_t*)(sRec + s * C::kRecBytes + kChunkValBytes + 4 * L);
        const uint32_t taddr = tbase + ((uint32_t)(quarter * 32) << 16) + C::kMeta0 + s;
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(w) : "memory");
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        mbar_arrive(smem_u32(&meta_ok[s]));
      }
    }
  } else if (warp == kWarpMma) {
    // ------------------------------------------------------------ MMA issuer
    int64_t i = 0;
    int acc = 0;
    uint32_t aphase = 0;
    const uint64_t adesc0 = sdesc(smem_u32(sRec), 128, 256, 0);
    const uint64_t bdesc0 = sdesc(smem_u32(sB), 4096, 1024, 2);
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      mbar_wait(smem_u32(&tempty[acc]), aphase ^ 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t dcol = tbase + acc * BN;
      for (int64_t c = c0; c < c1; ++c, ++i) {
        const int s = (int)(i % C::kStages);
        const uint32_t ph = (uint32_t)((i / C::kStages) & 1);
        mbar_wait(smem_u32(&full_b[s]), ph);
        mbar_wait(smem_u32(&meta_ok[s]), ph);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (lane == 0) {
          const uint64_t ad = adesc0 + (uint64_t)((s * C::kRecBytes) >> 4);
          const uint64_t bd = bdesc0 + (uint64_t)((s * C::kBBytes) >> 4);
          const uint32_t mcol = C::kMeta0 + s;
          const uint32_t ecol = tbase + (mcol & ~1u);   // even column address ...
          const uint32_t idesc = p.idesc | (mcol & 1u);  // ... + sparse_id2 selects the odd one
          const uint32_t accum = (c > c0) ? 1u : 0u;
          asm volatile(
              "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %5, 0;\n\t"
              "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t}" ::"r"(dcol),
              "l"(ad), "l"(bd), "r"(ecol), "r"(idesc), "r"(accum)
              : "memory");
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                           smem_u32(&empty[s]))
                       : "memory");
        }
        __syncwarp();
      }
      if (lane == 0) {
        if (c1 > c0)
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                           smem_u32(&tfull[acc]))
                       : "memory");
        else
          mbar_arrive(smem_u32(&tfull[acc]));
      }
      __syncwarp();
      if (++acc == C::kNAcc) { acc = 0; aphase ^= 1; }
    }
  } else {
    // ------------------------------------------------------------ epilogue
    const int quarter = warp & 3;  // TMEM lane quarter this warp may access
    const int r = quarter * 32 + lane;
    int acc = 0;
    uint32_t aphase = 0;
    const bool vec_ok = ((p.ldy & 3) == 0) && ((((uintptr_t)p.Y) & 15) == 0);
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int ft = (int)(u % p.n_ftiles);
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      mbar_wait(smem_u32(&tfull[acc]), aphase);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const int64_t grow = (int64_t)panel * kPanelRows + r;
      const bool row_ok = grow < p.rows;
      const int64_t orow = (row_ok && p.row_map) ? (int64_t)p.row_map[grow] : grow;
      float* yrow = p.Y + orow * p.ldy;
#pragma unroll 1
      for (int cc = 0; cc < BN; cc += 32) {
        uint32_t v[32];
        if (c1 > c0) {
          const uint32_t taddr = tbase + ((uint32_t)(quarter * 32) << 16) + acc * BN + cc;
          asm volatile(
              "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
              "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
              : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
                "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
                "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
                "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
              : "r"(taddr));
          asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        } else {
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] = 0u;
        }
        const int col = ft * BN + cc;
        if (row_ok && col < p.F) {
          if (vec_ok && col + 32 <= p.F) {
#pragma unroll
            for (int j = 0; j < 32; j += 4) {
              float4 f = make_float4(__uint_as_float(v[j]), __uint_as_float(v[j + 1]), __uint_as_float(v[j + 2]),
                                     __uint_as_float(v[j + 3]));
              __stcs((float4*)(yrow + col + j), f);
            }
          } else {
#pragma unroll
            for (int j = 0; j < 32; ++j)
              if (col + j < p.F) yrow[col + j] = __uint_as_float(v[j]);
          }
        }
      }
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      mbar_arrive(smem_u32(&tempty[acc]));
      if (++acc == C::kNAcc) { acc = 0; aphase ^= 1; }
    }
  }

  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == kWarpMma) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
  }
}

uint32_t make_idesc(nm_dtype dt, int BN) {
  uint32_t d = 0;
  d |= 1u << 2;   // sparse
  d |= 1u << 4;   // D = f32
  if (dt == NM_BF16) d |= (1u << 7) | (1u << 10);
  d |= 1u << 16;  // B MN-major (A K-major)
  d |= (uint32_t)(BN >> 3) << 17;
  d |= (uint32_t)(128 >> 4) << 24;
  return d;
}

PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaDriverEntryPointQueryResult q;
    void* f = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)f;
  });
  return fn;
}

// X as a 2-D tensor [n rows x F columns], row pitch ldx; box = 64 columns x 1 row, 128-byte
// swizzle (the UMMA SW128 MN-major atom); rows and columns outside the tensor read as zero.
nm_status make_x_map(CUtensorMap* tm, const void* X, int64_t n, int F, int64_t ldx, nm_dtype dt) {
  auto enc = tensor_map_encoder();
  if (!enc) return fail(NM_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[2] = {(cuuint64_t)F, (cuuint64_t)n};
  cuuint64_t strides[1] = {(cuuint64_t)ldx * 2};
  cuuint32_t box[2] = {64, 1};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(tm, dt == NM_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2,
                   const_cast<void*>(X), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(NM_ERR_CUDA, "cuTensorMapEncodeTiled failed: " + std::to_string((int)r));
  return NM_OK;
}

template <int BN>
nm_status launch_bn(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F, cudaStream_t s) {
  using C = Cfg<BN>;
  static int configured_dev = -1;
  int dev = 0;
  NM_CUDA(cudaGetDevice(&dev));
  if (configured_dev != dev) {
    NM_CUDA(cudaFuncSetAttribute(k_spmm_sptc<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::kSmem));
    configured_dev = dev;
  }
  int sms = 148;
  NM_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  CUtensorMap tm;
  nm_status st = make_x_map(&tm, PX, P->n, F, ldx, P->dtype);
  if (st != NM_OK) return st;
  SpmmParams prm;
  prm.image = P->image;
  prm.panel_chunk_ptr = P->panel_chunk_ptr;
  prm.unit_order = P->unit_order;
  prm.row_map = P->row_map;
  prm.Y = Yp;
  prm.ldy = ldy;
  prm.F = F;
  prm.rows = P->row_end - P->row_begin;
  prm.n_ftiles = (F + BN - 1) / BN;
  prm.n_units = P->n_panels * prm.n_ftiles;
  prm.idesc = make_idesc(P->dtype, BN);
  int64_t grid = prm.n_units < sms ? prm.n_units : sms;
  if (grid < 1) return NM_OK;
  k_spmm_sptc<BN><<<(unsigned)grid, kThreads, C::kSmem, s>>>(prm, tm);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

}  // namespace

nm_status launch_spmm_sptc(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                           cudaStream_t s) {
  if (F <= 64) return launch_bn<64>(P, PX, ldx, Yp, ldy, F, s);
  if (F <= 128) return launch_bn<128>(P, PX, ldx, Yp, ldy, F, s);
  if (F <= 192) return launch_bn<192>(P, PX, ldx, Yp, ldy, F, s);
  return launch_bn<256>(P, PX, ldx, Yp, ldy, F, s);
}

}  // namespace nm
