// nm_spmm tensor-core part: Yp = B_packed * PX on sm_100a sparse tensor cores.
//
// One work unit = (panel of 128 rows of B, 64..256-column tile of F).  The K dimension of a
// panel is its list of non-empty meta-blocks; 8 meta-blocks (4 selected columns each) form
// one K = 32 chunk, i.e. one tcgen05.mma.sp.cta_group::1.kind::f16 with M = 128, N = BN:
//   A (compressed, 128 x 16 physical)  <- cp.async.bulk of the packed image (HBM stream)
//   E (2:4 metadata, 128 lanes x 32 b) <- tcgen05.st into tensor memory
//   B (32 gathered rows of PX x BN)    <- cp.async 16-byte gathers into the SW128 layout
//   D (fp32, 128 x BN)                 in tensor memory, read back with tcgen05.ld
// Warp roles (persistent CTA per SM, 9 warps): warps 0-3 produce, warp 4 issues MMAs,
// warps 5-8 drain the accumulator (double-buffered when it fits in 512 TMEM columns).
// Layouts were measured on B200: tools/probes/probe_umma_sp.b200.txt.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "nm_internal.h"

namespace nm {
namespace {

constexpr int kThreads = 288;
constexpr int kProducerThreads = 128;
constexpr int kLag = 2;  // producer arrives for chunk i after issuing chunk i + kLag

struct SpmmParams {
  const uint8_t* image;
  const int32_t* xrow;
  const int64_t* panel_chunk_ptr;
  const int32_t* unit_order;
  const uint16_t* X;
  int64_t ldx;
  float* Y;
  int64_t ldy;
  int F;
  int64_t rows;
  int64_t n_units;
  int n_ftiles;
  uint32_t idesc;
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

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
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes)
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
  static constexpr int kStages = 8;
  static constexpr int kABytes = kChunkValBytes;          // 4096
  static constexpr int kBBytes = 32 * BN * 2;             // 32 K-rows x BN halves
  static constexpr int kNAcc = (2 * BN + 4 * kStages <= 512) ? 2 : 1;
  static constexpr int kMeta0 = kNAcc * BN;               // first metadata column (4-aligned)
  static constexpr int kSmem = 1024 + kStages * (kABytes + kBBytes) + 1024;
  static_assert(kMeta0 + 4 * kStages <= 512, "TMEM budget");
  static_assert(BN % 64 == 0 && BN >= 64 && BN <= 256, "BN");
};

template <int BN>
__global__ void __launch_bounds__(kThreads, 1) k_spmm_sptc(const SpmmParams p) {
  using C = Cfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::kStages * C::kABytes;  // 1024-aligned (kStages*4096)
  uint64_t* bars = (uint64_t*)(sB + C::kStages * C::kBBytes);
  uint64_t* full = bars;
  uint64_t* empty = bars + C::kStages;
  uint64_t* tfull = bars + 2 * C::kStages;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::kStages; ++s) {
      mbar_init(smem_u32(&full[s]), kProducerThreads + 1);
      mbar_init(smem_u32(&empty[s]), 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(smem_u32(&tfull[a]), 1);
      mbar_init(smem_u32(&tempty[a]), 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 4) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tmem_slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tbase = *tmem_slot;

  if (warp < 4) {
    // ------------------------------------------------------------------ producers
    const int t = threadIdx.x;
    int64_t issued = 0;  // chunks issued by this CTA so far (stage = issued % kStages)
    constexpr int kPieces = 32 * BN / 8;  // 16-byte pieces of the B tile
    constexpr int kRowPieces = BN / 8;
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int ft = (int)(u % p.n_ftiles);
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      for (int64_t c = c0; c < c1; ++c) {
        const int stage = (int)(issued % C::kStages);
        const uint32_t phase = (uint32_t)((issued / C::kStages) & 1);
        mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
        const uint8_t* img = p.image + c * kChunkBytes;
        if (t == 0) {
          mbar_arrive_tx(smem_u32(&full[stage]), C::kABytes);
          bulk_g2s(smem_u32(sA + stage * C::kABytes), img, C::kABytes, smem_u32(&full[stage]));
        }
        const uint32_t bst = smem_u32(sB + stage * C::kBBytes);
#pragma unroll
        for (int i = t; i < kPieces; i += kProducerThreads) {
          const int k = i / kRowPieces, c16 = i % kRowPieces;
          const int32_t xr = __ldg(p.xrow + c * 32 + k);
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
        asm volatile("cp.async.commit_group;" ::: "memory");
        // 2:4 metadata word of this thread's TMEM lane
        const uint32_t w = __ldg((const uint32_t*)(img + kChunkValBytes) + t);
        const uint32_t taddr = tbase + ((uint32_t)(warp * 32) << 16) + C::kMeta0 + 4 * stage;
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(w) : "memory");
        ++issued;
        if (issued > kLag) {
          // chunk issued-1-kLag is complete in shared memory: publish it to the MMA warp
          asm volatile("cp.async.wait_group %0;" ::"n"(kLag) : "memory");
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
          asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
          mbar_arrive(smem_u32(&full[(issued - 1 - kLag) % C::kStages]));
        }
      }
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    for (int64_t j = (issued > kLag ? issued - kLag : 0); j < issued; ++j)
      mbar_arrive(smem_u32(&full[j % C::kStages]));
  } else if (warp == 4) {
    // ------------------------------------------------------------------ MMA issuer
    int stage = 0;
    uint32_t phase = 0;
    int acc = 0;
    uint32_t aphase = 0;
    const uint64_t adesc0 = sdesc(smem_u32(sA), 128, 256, 0);
    const uint64_t bdesc0 = sdesc(smem_u32(sB), 4096, 1024, 2);
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      mbar_wait(smem_u32(&tempty[acc]), aphase ^ 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t dcol = tbase + acc * BN;
      for (int64_t c = c0; c < c1; ++c) {
        mbar_wait(smem_u32(&full[stage]), phase);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (lane == 0) {
          const uint64_t ad = adesc0 + (uint64_t)((stage * C::kABytes) >> 4);
          const uint64_t bd = bdesc0 + (uint64_t)((stage * C::kBBytes) >> 4);
          const uint32_t ecol = tbase + C::kMeta0 + 4 * stage;
          const uint32_t accum = (c > c0) ? 1u : 0u;
          asm volatile(
              "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %5, 0;\n\t"
              "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t}" ::"r"(dcol),
              "l"(ad), "l"(bd), "r"(ecol), "r"(p.idesc), "r"(accum)
              : "memory");
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                           smem_u32(&empty[stage]))
                       : "memory");
        }
        __syncwarp();
        if (++stage == C::kStages) { stage = 0; phase ^= 1; }
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
    // ------------------------------------------------------------------ epilogue
    const int quarter = warp & 3;  // TMEM lane quarter this warp may access
    const int r = quarter * 32 + lane;
    int acc = 0;
    uint32_t aphase = 0;
    for (int64_t u = blockIdx.x; u < p.n_units; u += gridDim.x) {
      const int32_t panel = p.unit_order[u / p.n_ftiles];
      const int ft = (int)(u % p.n_ftiles);
      const int64_t c0 = p.panel_chunk_ptr[panel], c1 = p.panel_chunk_ptr[panel + 1];
      mbar_wait(smem_u32(&tfull[acc]), aphase);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const int64_t grow = (int64_t)panel * kPanelRows + r;
      float* yrow = p.Y + grow * p.ldy;
      const bool row_ok = grow < p.rows;
      const bool vec_ok = ((p.ldy & 3) == 0) && ((((uintptr_t)p.Y) & 15) == 0);
#pragma unroll 1
      for (int cc = 0; cc < BN; cc += 16) {
        uint32_t v[16];
        if (c1 > c0) {
          const uint32_t taddr = tbase + ((uint32_t)(quarter * 32) << 16) + acc * BN + cc;
          asm volatile(
              "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
              : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
                "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
                "=r"(v[14]), "=r"(v[15])
              : "r"(taddr));
          asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        } else {
#pragma unroll
          for (int j = 0; j < 16; ++j) v[j] = 0u;
        }
        const int col = ft * BN + cc;
        if (row_ok && col < p.F) {
          if (vec_ok && col + 16 <= p.F) {
#pragma unroll
            for (int j = 0; j < 16; j += 4) {
              float4 f = make_float4(__uint_as_float(v[j]), __uint_as_float(v[j + 1]),
                                     __uint_as_float(v[j + 2]), __uint_as_float(v[j + 3]));
              *(float4*)(yrow + col + j) = f;
            }
          } else {
            for (int j = 0; j < 16 && col + j < p.F; ++j) yrow[col + j] = __uint_as_float(v[j]);
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
  if (warp == 4) {
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
nm_status launch_bn(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                    cudaStream_t s) {
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
  prm.xrow = P->xrow;
  prm.panel_chunk_ptr = P->panel_chunk_ptr;
  prm.unit_order = P->unit_order;
  prm.X = (const uint16_t*)PX;
  prm.ldx = ldx;
  prm.Y = Yp;
  prm.ldy = ldy;
  prm.F = F;
  prm.rows = P->row_end - P->row_begin;
  prm.n_ftiles = (F + BN - 1) / BN;
  prm.n_units = P->n_panels * prm.n_ftiles;
  prm.idesc = make_idesc(P->dtype, BN);
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
