// nm_spmm tensor-core part: Yp = B_packed * PX on sm_100a sparse tensor cores.
//
// One work unit = (panel of 128 rows of B, 64..256-column tile of F).  The K dimension of a
// panel is its list of non-empty meta-blocks; 8 meta-blocks (4 selected columns each) form
// one K = 32 chunk, i.e. one tcgen05.mma.sp.cta_group::1.kind::f16 with M = 128, N = BN:
//   record (A values, 2:4 metadata, 32 gather rows; 4736 B) <- one cp.async.bulk (HBM stream)
//   B (32 gathered rows of X x BN, SWIZZLE_128B MN-major)  <- cp.async 16-byte gathers
//   E (metadata, 128 lanes x 32 b)                          <- tcgen05.st from shared memory
//   D (fp32, 128 x BN)                                      in tensor memory (tcgen05.ld out)
// Warp roles (persistent, one CTA per SM, 10 warps):
//   w0 record TMA | w1-4 loaders: X gathers + metadata -> TMEM | w5 MMA issuer (+TMEM alloc)
//   | w6-9 epilogue (TMEM -> registers -> smem transpose -> coalesced Y rows).
// All hand-offs are mbarriers; the pipeline runs across work units, so consecutive panels
// overlap.  The X gathers use cp.async rather than TMA tile::gather4: measured on B200 the
// TMA unit spends ~57 cycles per gather4 instruction (4 rows x 128 B), which capped the
// kernel at ~0.9 chunks/us/SM.  Layouts measured on B200:
// tools/probes/probe_umma_sp.b200.txt, tools/probes/probe_gather4.b200.txt.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <cstdlib>

#include "nm_internal.h"

namespace nm {
namespace {

constexpr int kThreads = 320;
constexpr int kWarpRec = 0, kWarpLoad0 = 1, kWarpMma = 5, kWarpEpi0 = 6;
constexpr int kLoaders = 128;
constexpr int kEpiTileFloats = 32 * 33;  // per epilogue warp: 32 rows x 32 cols (+1 pad)

struct SpmmParams {
  const uint8_t* image;
  const int64_t* panel_chunk_ptr;
  const int32_t* unit_order;
  const int32_t* row_map;  // nullable: output row of Y for packed row l
  const uint16_t* X;
  int64_t ldx;
  float* Y;
  int64_t ldy;
  int F;
  int64_t rows;
  int64_t n_units;
  int n_ftiles;
  uint32_t idesc;
  int debug;  // profiling switches (NM_SPMM_DEBUG): 1 = no gathers, 2 = no Y stores, 8 = no metadata
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

__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
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
  static constexpr int kEpiBytes = 4 * kEpiTileFloats * 4;      // 16.5 KB
  static constexpr int kStagesRaw = (214 * 1024 - kEpiBytes) / kStageBytes;
  static constexpr int kStages = kStagesRaw > 16 ? 16 : kStagesRaw;
  static constexpr int kLag = kStages - 4 < 10 ? kStages - 4 : 10;  // chunks in flight per loader
  static constexpr int kNAcc = (2 * BN + kStages <= 512) ? 2 : 1;
  static constexpr int kMeta0 = kNAcc * BN;                     // metadata column of stage s: kMeta0 + s
  static constexpr int kRecRegion = ((kStages * kRecBytes + 1023) / 1024) * 1024;
  static constexpr int kSmem = 1024 + kRecRegion + kStages * kBBytes + kEpiBytes + 1024;
  static_assert(kMeta0 + kStages <= 512, "TMEM budget");
  static_assert(BN % 64 == 0 && BN >= 64 && BN <= 256, "BN");
  static_assert(kSmem <= 227 * 1024, "smem");
  static_assert(kLag >= 2, "pipeline depth");
};

template <int BN>
__global__ void __launch_bounds__(kThreads, 1) k_spmm_sptc(const SpmmParams p) {
  using C = Cfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sRec = smem;                                     // kStages records (16-byte aligned)
  uint8_t* sB = smem + C::kRecRegion;                       // kStages B tiles (1024-aligned)
  float* sEpi = (float*)(sB + C::kStages * C::kBBytes);     // epilogue transpose tiles
  uint64_t* bars = (uint64_t*)((uint8_t*)sEpi + C::kEpiBytes);
  uint64_t* full_a = bars;                  // record landed (tx)
  uint64_t* full_b = bars + C::kStages;     // gathers + metadata ready (128 loader arrivals)
  uint64_t* empty = bars + 2 * C::kStages;  // MMA done with the stage (tcgen05.commit)
  uint64_t* tfull = bars + 3 * C::kStages;  // accumulator ready (2)
  uint64_t* tempty = tfull + 2;             // accumulator drained (2)
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::kStages; ++s) {
      mbar_init(smem_u32(&full_a[s]), 1);
      mbar_init(smem_u32(&full_b[s]), 2 * kLoaders);  // cp.async completions + metadata stores
      mbar_init(smem_u32(&empty[s]), 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(smem_u32(&tfull[a]), 1);
      mbar_init(smem_u32(&tempty[a]), 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
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
  } else if (warp >= kWarpLoad0 && warp < kWarpLoad0 + 4) {
    // ------------------------------------------------------------ loaders: X gathers + metadata
    const int quarter = warp & 3;                 // TMEM lane quarter of this warp
    const int t = threadIdx.x - kWarpLoad0 * 32;  // 0..127
    const int L = quarter * 32 + lane;            // TMEM lane this thread writes
    constexpr int kRowPieces = BN / 8;            // 16-byte pieces per gathered row
    constexpr int kPer = 32 * kRowPieces / kLoaders;
    int64_t i = 0;
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int ft = (int)(u % p.n_ftiles);
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      for (int64_t c = c0; c < c1; ++c, ++i) {
        const int s = (int)(i % C::kStages);
        const uint32_t ph = (uint32_t)((i / C::kStages) & 1);
        mbar_wait(smem_u32(&full_a[s]), ph);
        const uint8_t* rec = sRec + s * C::kRecBytes;
        const uint32_t bst = smem_u32(sB + s * C::kBBytes);
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
          const int idx = t + kLoaders * q;
          const int k = idx / kRowPieces, c16 = idx % kRowPieces;
          int32_t xr = *(const int32_t*)(rec + kChunkXrowOff + 4 * k);
          if (p.debug & 1) xr = -1;
          const int col0 = ft * BN + c16 * 8;
          uint32_t bytes = 0;
          const uint16_t* src = p.X;
          if (xr >= 0 && col0 < p.F) {
            const int rem = p.F - col0;
            bytes = rem >= 8 ? 16u : (uint32_t)(rem * 2);
            src = p.X + (int64_t)xr * p.ldx + col0;
          }
          const uint32_t dst = bst + (c16 >> 3) * 4096 + (k >> 3) * 1024 + (k & 7) * 128 +
                               ((((uint32_t)c16 & 7u) ^ ((uint32_t)k & 7u)) << 4);
          cp_async16(dst, src, bytes);
        }
        // the barrier tracks this thread's gathers asynchronously (arrival when they land)
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(&full_b[s])) : "memory");
        if (!(p.debug & 8)) {
          const uint32_t w = *(const uint32_t*)(rec + kChunkValBytes + 4 * L);
          const uint32_t taddr = tbase + ((uint32_t)(quarter * 32) << 16) + C::kMeta0 + s;
          asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(w) : "memory");
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        }
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        mbar_arrive(smem_u32(&full_b[s]));
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
        // gathers were written through the generic proxy (cp.async); order them before the
        // tensor core's async-proxy reads of the stage
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
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
    float* tile = sEpi + (warp - kWarpEpi0) * kEpiTileFloats;
    int acc = 0;
    uint32_t aphase = 0;
    const bool vec_ok = ((p.ldy & 3) == 0) && ((((uintptr_t)p.Y) & 15) == 0);
    const int rsub = lane >> 3;       // row within a 4-row store group
    const int cq = (lane & 7) * 4;    // column quad within the 32-column slice
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int ft = (int)(u % p.n_ftiles);
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      // this lane's row (as the TMEM lane owner) and its output row in Y
      const int64_t myrow = (int64_t)panel * kPanelRows + quarter * 32 + lane;
      const int64_t myout = myrow < p.rows ? (p.row_map ? (int64_t)p.row_map[myrow] : myrow) : -1;
      mbar_wait(smem_u32(&tfull[acc]), aphase);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
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
        if (col >= p.F || (p.debug & 2)) continue;  // warp-uniform
        // transpose through shared memory: lane = row -> lanes = 4 rows x 8 column quads
#pragma unroll
        for (int j = 0; j < 32; ++j) tile[lane * 33 + j] = __uint_as_float(v[j]);
        __syncwarp();
#pragma unroll
        for (int g = 0; g < 8; ++g) {
          const int rr = g * 4 + rsub;
          const int64_t orow = __shfl_sync(0xffffffffu, myout, rr);
          const float* tr = tile + rr * 33 + cq;
          if (orow >= 0) {
            float* dst = p.Y + orow * p.ldy + col + cq;
            if (vec_ok && col + cq + 4 <= p.F) {
              __stcs((float4*)dst, make_float4(tr[0], tr[1], tr[2], tr[3]));
            } else {
              for (int e = 0; e < 4; ++e)
                if (col + cq + e < p.F) dst[e] = tr[e];
            }
          }
        }
        __syncwarp();
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
  SpmmParams prm;
  prm.image = P->image;
  prm.panel_chunk_ptr = P->panel_chunk_ptr;
  prm.unit_order = P->unit_order;
  prm.row_map = P->row_map;
  prm.X = (const uint16_t*)PX;
  prm.ldx = ldx;
  prm.Y = Yp;
  prm.ldy = ldy;
  prm.F = F;
  prm.rows = P->row_end - P->row_begin;
  prm.n_ftiles = (F + BN - 1) / BN;
  prm.n_units = P->n_panels * prm.n_ftiles;
  prm.idesc = make_idesc(P->dtype, BN);
  const char* dbg = getenv("NM_SPMM_DEBUG");
  prm.debug = dbg ? atoi(dbg) : 0;
  int64_t grid = prm.n_units < sms ? prm.n_units : sms;
  if (grid < 1) return NM_OK;
  k_spmm_sptc<BN><<<(unsigned)grid, kThreads, C::kSmem, s>>>(prm);
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
