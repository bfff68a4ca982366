// nm_spmm tensor-core part, FULL-record form: Yp = B_packed * PX on sm_100a sparse tensor cores.
//
// One work unit = (panel of 128 rows of B, BN-column tile of F).  The K dimension of a panel
// is its list of non-empty meta-blocks; 8 meta-blocks (4 selected columns each) form one
// K = 32 chunk = one tcgen05.mma.sp.cta_group::1.kind::f16 with M = 128, N = BN.  The packed
// image holds every chunk in the operand form the tensor core reads (nm_internal.h, 4736 B:
// A values in the UMMA K-major canonical layout, the metadata in tensor-memory lane order,
// the 32 gather rows), so a chunk costs one bulk copy and no expansion:
//   record (A + metadata + gather rows)   <- one cp.async.bulk per chunk, straight into the
//                                            pipeline stage (HBM stream, L2-prefetched ahead)
//   B (32 gathered rows of X x BN, SWIZZLE_128B MN-major)  <- cp.async 16-byte gathers
//   E (metadata, 128 lanes x 32 b)        <- tcgen05.st of the record's lane words
//   D (fp32, 128 x BN)                    in tensor memory (tcgen05.ld out)
// Warp roles (persistent, one CTA per SM, 22 warps):
//   w0     record producer: waits for a free stage, one bulk copy per chunk, L2 prefetch of
//          the next unit's first records
//   w1-16  four gather groups of 4 warps (one per TMEM lane quarter); group g owns the stages
//          s = g (mod 4): X gathers of the chunk's 32 rows + its metadata column
//   w17    MMA issuer (+ TMEM allocation): warp-uniform loop, one elected lane issues
//   w18-21 epilogue, one warp per TMEM lane quarter: tcgen05.ld 16x256b -> 8-byte stores
// Work distribution: each CTA walks a CONTIGUOUS range of panels (pack time: balanced by chunk
// count, nm_packed::cta_ptr), so the grid has no tail of idle SMs on skewed (power-law) graphs
// and consecutive panels of one CTA share their X neighbourhoods in L2.
// The compressed-record kernel (spmm_sm100.cu) is the alternative for dense chunks; nm_spmm
// picks per pack (launch_spmm_sptc).
#include <cuda.h>
#include <cudaTypedefs.h>

#include "nm_internal.h"

namespace nm {
namespace {

#ifndef NM_FULL_GROUPS
#define NM_FULL_GROUPS 4
#endif
#ifndef NM_FULL_MAX_STAGES
#define NM_FULL_MAX_STAGES 16
#endif
constexpr int kFGroups = NM_FULL_GROUPS;            // gather groups (4 warps each)
#ifdef NM_FULL_MMA_ONLY
#define NM_FULL_MMA_ONLY_ON 1
#else
#define NM_FULL_MMA_ONLY_ON 0
#endif
constexpr int kWProd = 0, kWG0 = 1, kWMma = kWG0 + 4 * kFGroups, kWEpi0 = kWMma + 1;
constexpr int kFThreads = (kWEpi0 + 4) * 32;        // 22 warps (4 groups)
constexpr int kGThreads = 128;                      // threads per gather group
#ifndef NM_FULL_PF
#define NM_FULL_PF 4
#endif
constexpr int kPfChunks = NM_FULL_PF;               // records L2-prefetched ahead (chunks)

struct FullParams {
  const uint8_t* image;            // full records, kChunkBytes each, in chunk order
  const int64_t* panel_chunk_ptr;  // [n_panels + 1]
  const int32_t* cta_ptr;          // [gridDim.x + 1] first panel of each CTA's range
  const int32_t* row_map;          // nullable: output row of Y for packed row l
  const uint16_t* X;
  int64_t ldx;
  float* Y;
  int64_t ldy;
  int F;
  int64_t rows;
  int n_ftiles;
  uint32_t idesc;
  // fused GCN epilogue (nm_gcn_layer on a pack without residual): H16 != nullptr stores
  // act(Y + bias) as 16-bit values (bf16 if bf16_out) instead of Y (F even)
  uint16_t* H16;
  int64_t ldh;
  const float* bias;
  int relu, bf16_out;
};

__device__ __forceinline__ uint32_t pack_act16(float a, float b, const FullParams& p, int col) {
  if (p.bias) {
    a += __ldg(p.bias + col);
    b += __ldg(p.bias + col + 1);
  }
  if (p.relu) {
    a = fmaxf(a, 0.f);
    b = fmaxf(b, 0.f);
  }
  uint32_t r;
  if (p.bf16_out)
    asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(b), "f"(a));
  else
    asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(b), "f"(a));
  return r;  // a in the low half
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}

__device__ __forceinline__ void mbar_init(uint32_t a, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count));
}

__device__ __forceinline__ void mbar_wait(uint32_t a, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P;\n"
      "NMF_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra NMF_WAIT_%=;\n\t}" ::"r"(a),
      "r"(parity)
      : "memory");
}

// long waits (epilogue): suspend-time hint, so the waiting warps take no issue slots
__device__ __forceinline__ void mbar_wait_sleep(uint32_t a, uint32_t parity) {
  uint32_t ok;
  for (;;) {
    asm volatile(
        "{\n\t.reg .pred P;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, P;\n\t}"
        : "=r"(ok)
        : "r"(a), "r"(parity), "r"(1000000)
        : "memory");
    if (ok) return;
  }
}

__device__ __forceinline__ void mbar_arrive(uint32_t a) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(a) : "memory");
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
struct FCfg {
  // chunks per pipeline stage: two K = 32 chunks share one barrier round trip (one record
  // copy of 2 x 4736 B -- consecutive chunks are adjacent in the image -- two gather sets, one
  // tcgen05.st.x2 of the two metadata columns, two MMAs and one commit)
  static constexpr int kCPS = BN <= 128 ? 2 : 1;
  static constexpr int kBBytes = 32 * BN * 2;       // one chunk's 32 gathered rows x BN
  static constexpr int kRecBytes = kChunkBytes;     // A (4096) + metadata (512) + gather rows (128)
  static constexpr int kStageBytes = kCPS * (kBBytes + kRecBytes);
  static constexpr int kStagesRaw = (222 * 1024 - 2048) / kStageBytes;
  static constexpr int kMaxStages = NM_FULL_MAX_STAGES / kCPS;
  static constexpr int kStages = ((kStagesRaw > kMaxStages ? kMaxStages : kStagesRaw) / kFGroups) * kFGroups;
  static constexpr int kMetaCols = kCPS * kStages;
  static constexpr int kNAcc = (3 * BN + kMetaCols <= 512) ? 3 : (2 * BN + kMetaCols <= 512) ? 2 : 1;
  static constexpr int kMeta0 = kNAcc * BN;         // metadata column of (stage s, chunk j): kMeta0 + kCPS*s + j
  static constexpr int kSmem = 1024 + kStages * kStageBytes + 1024;
  static_assert(kMeta0 + kMetaCols <= 512, "TMEM budget");
  static_assert(kRecBytes % 16 == 0, "bulk copy granularity");
  static_assert(kSmem <= 227 * 1024, "smem");
  static_assert(kStages >= 2, "stages");
  static_assert((32 * (BN / 8)) % kGThreads == 0 && kGThreads % (BN / 8) == 0, "gather piece mapping");
};

template <int BN>
__global__ void __launch_bounds__(kFThreads, 1) k_spmm_full(const FullParams p) {
  using C = FCfg<BN>;
  constexpr int CPS = C::kCPS;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const uint32_t sB = smem_u32(smem);                          // stage s: CPS B tiles (SW128)
  const uint32_t sRec = sB + C::kStages * CPS * C::kBBytes;    // stage s: CPS adjacent records
  uint64_t* bars = (uint64_t*)(smem + C::kStages * C::kStageBytes);
  uint64_t* full_rec = bars;                 // records landed (tx)
  uint64_t* full_b = full_rec + C::kStages;  // gathers landed + metadata written
  uint64_t* empty = full_b + C::kStages;     // MMAs done with the stage (tcgen05.commit)
  uint64_t* tfull = empty + C::kStages;      // accumulator ready
  uint64_t* tempty = tfull + 4;              // accumulator drained
  uint32_t* tmem_slot = (uint32_t*)(tempty + 4);
  const uint32_t bRec = smem_u32(full_rec), bFull = smem_u32(full_b), bEmpty = smem_u32(empty);
  const uint32_t bTfull = smem_u32(tfull), bTempty = smem_u32(tempty);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::kStages; ++s) {
      mbar_init(bRec + 8 * s, 1);
      // per-thread cp.async completions (noinc) + one arrival per gather warp (metadata)
      mbar_init(bFull + 8 * s, kGThreads + kGThreads / 32);
      mbar_init(bEmpty + 8 * s, 1);
    }
    for (int a = 0; a < 4; ++a) {
      mbar_init(bTfull + 8 * a, 1);
      mbar_init(bTempty + 8 * a, 4);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kWMma) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tmem_slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tbase = *tmem_slot;
  const int pa = __ldg(p.cta_ptr + blockIdx.x), pz = __ldg(p.cta_ptr + blockIdx.x + 1);
  const int nft = p.n_ftiles;

  if (warp == kWProd) {
    // ------------------------------------------------------------ record producer
    // records are streamed once: L2 evict-first, so they do not push the gathered X rows
    // (evict-last) out of L2 (ncu, C3: DRAM reads 4.08 GB for 2.57 GB of records without it)
    uint64_t pol_stream;
#ifndef NM_FULL_REC_FRAC
#define NM_FULL_REC_FRAC 1.0
#endif
#define NM_STR2(x) #x
#define NM_STR(x) NM_STR2(x)
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, " NM_STR(NM_FULL_REC_FRAC) ";" : "=l"(pol_stream));
    int s = 0;
    uint32_t ph = 0;
    int64_t c0 = pa < pz ? __ldg(p.panel_chunk_ptr + pa) : 0;
    for (int pn = pa; pn < pz; ++pn) {
      const int64_t c1 = __ldg(p.panel_chunk_ptr + pn + 1);
      const int nch = (int)(c1 - c0);
      // the next panel's first records into L2 while this one streams (its F tiles re-read
      // this panel's records from L2)
      if (lane == 0 && pn + 1 < pz) {
        const int64_t n2 = __ldg(p.panel_chunk_ptr + pn + 2) - c1;
        const int64_t k = n2 < kPfChunks ? n2 : kPfChunks;
        if (k > 0)
          asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(p.image + c1 * kChunkBytes),
                       "r"((uint32_t)(k * kChunkBytes)), "l"(pol_stream)
                       : "memory");
      }
      for (int ft = 0; ft < nft; ++ft) {
        for (int c = 0; c < nch; c += CPS) {
          const int sub = min(CPS, nch - c);
          mbar_wait(bEmpty + 8 * s, ph ^ 1);  // the MMAs have finished with stage s
#ifdef NM_FULL_MMA_ONLY  // timing experiment (results invalid): no record copies
          if (lane == 0) mbar_arrive(bRec + 8 * s);
          __syncwarp();
          if (++s == C::kStages) { s = 0; ph ^= 1; }
          continue;
#endif
          if (lane == 0) {
            if (c + kPfChunks < nch && ft == 0)
              asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(
                               p.image + (c0 + c + kPfChunks) * kChunkBytes),
                           "r"((uint32_t)(min(CPS, nch - c - kPfChunks) * kChunkBytes)), "l"(pol_stream)
                           : "memory");
            const uint32_t bytes = (uint32_t)(sub * kChunkBytes);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bRec + 8 * s), "r"(bytes)
                         : "memory");
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
                "%4;" ::"r"(sRec + s * CPS * C::kRecBytes),
                "l"(p.image + (c0 + c) * kChunkBytes), "r"(bytes), "r"(bRec + 8 * s), "l"(pol_stream)
                : "memory");
          }
          __syncwarp();
          if (++s == C::kStages) { s = 0; ph ^= 1; }
        }
      }
      c0 = c1;
    }
  } else if (warp >= kWG0 && warp < kWG0 + 4 * kFGroups) {
    // ------------------------------------------------------------ gathers + metadata
    const int group = (warp - kWG0) >> 2;  // owns the stages s % kFGroups == group
    const int quarter = warp & 3;          // TMEM lane quarter this warp may access
    const int t = threadIdx.x - (kWG0 + 4 * group) * 32;  // 0..127 within the group
    constexpr int kRowPieces = BN / 8;     // 16-byte pieces per gathered row
    constexpr int kPer = 32 * kRowPieces / kGThreads;  // pieces per thread and chunk
    constexpr int kRowsPerPass = kGThreads / kRowPieces;
    const int c16 = t % kRowPieces, kk0 = t / kRowPieces;
    const uint32_t dcol = (uint32_t)(c16 >> 3) * 4096u;  // 64-column slab of the SW128 tile
    const uint32_t ldxb = (uint32_t)p.ldx * 2u;  // row pitch in bytes
    const uint32_t mword = 4u * (uint32_t)(quarter * 32 + lane);  // this lane's metadata word
    uint64_t pol_x;  // gathered X rows stay in L2 (reused by the other panels' meta-blocks)
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_x));
    // this group's stages only: i = group, group + kFGroups, ... (stage s = i mod kStages)
    StageIter<CPS> it;
    it.init(p.panel_chunk_ptr, pa, pz, nft);
    it.advance(group);
    for (int i = group; it.valid(); i += kFGroups, it.advance(kFGroups)) {
      const int s = i % C::kStages;
      const uint32_t ph = (uint32_t)((i / C::kStages) & 1);
      const int col0 = it.ft * BN + c16 * 8;
      const uint32_t colbytes = col0 >= p.F ? 0u : (p.F - col0 >= 8 ? 16u : (uint32_t)(p.F - col0) * 2u);
      const uint16_t* xcol = p.X + (colbytes ? col0 : 0);
      const int sub = min(CPS, it.nch - it.c);
      mbar_wait(bRec + 8 * s, ph);  // records landed (gather rows, metadata, A)
      const uint32_t rec0 = sRec + s * CPS * C::kRecBytes;
      uint32_t mw[CPS];
#pragma unroll
      for (int j = 0; j < CPS; ++j) {
        if (j < sub) {
          const uint32_t rec = rec0 + j * C::kRecBytes;
          const uint32_t sbase = sB + (s * CPS + j) * C::kBBytes + dcol;
#ifdef NM_FULL_MMA_ONLY  // timing experiment (results invalid): no gathers
          if (false) {
#else
          if (colbytes == 16u) {
#endif
#pragma unroll
            for (int q = 0; q < kPer; ++q) {
              const int kk = q * kRowsPerPass + kk0;
              const int32_t xr = (int32_t)lds32(rec + kChunkXrowOff + 4 * kk);
              asm volatile(
                  "{\n\t.reg .pred q;\n\tsetp.lt.s32 q, %2, 0;\n\t"
                  "cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, q, %3;\n\t}" ::"r"(
                      sbase + (kk >> 3) * 1024 + (kk & 7) * 128 + ((((uint32_t)c16 ^ (uint32_t)kk) & 7u) << 4)),
                  "l"((uint64_t)(uint32_t)max(xr, 0) * ldxb + (uint64_t)(uintptr_t)xcol), "r"(xr), "l"(pol_x)
                  : "memory");
            }
          } else if (!NM_FULL_MMA_ONLY_ON) {  // the F tail: partial or empty pieces
#pragma unroll
            for (int q = 0; q < kPer; ++q) {
              const int kk = q * kRowsPerPass + kk0;
              const int32_t xr = (int32_t)lds32(rec + kChunkXrowOff + 4 * kk);
              const uint32_t nb = xr >= 0 ? colbytes : 0u;
              asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2, %3;" ::"r"(
                               sbase + (kk >> 3) * 1024 + (kk & 7) * 128 + ((((uint32_t)c16 ^ (uint32_t)kk) & 7u) << 4)),
                           "l"((uint64_t)(uint32_t)max(xr, 0) * ldxb + (uint64_t)(uintptr_t)xcol), "r"(nb), "l"(pol_x)
                           : "memory");
            }
          }
          mw[j] = lds32(rec + kChunkValBytes + mword);
        } else {
          mw[j] = 0x44444444u;  // unused column (legal no-value nibbles)
        }
      }
      asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bFull + 8 * s) : "memory");
      // metadata: this lane's words of the stage's records into its TMEM columns
      const uint32_t taddr = tbase + ((uint32_t)(quarter * 32) << 16) + C::kMeta0 + CPS * s;
      if constexpr (CPS == 2)
        asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};" ::"r"(taddr), "r"(mw[0]),
                     "r"(mw[CPS - 1])
                     : "memory");
      else
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(mw[0]) : "memory");
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(bFull + 8 * s);
    }
  } else if (warp == kWMma) {
    // ------------------------------------------------------------ MMA issuer
    int s = 0;
    uint32_t ph = 0;
    int acc = 0;
    uint32_t aphase = 0;
    const uint64_t adesc0 = sdesc(sRec, 128, 256, 0);   // A: K-major, no swizzle (LBO 128, SBO 256)
    const uint64_t bdesc0 = sdesc(sB, 4096, 1024, 2);   // B: MN-major, SWIZZLE_128B
    int64_t c0 = pa < pz ? __ldg(p.panel_chunk_ptr + pa) : 0;
    for (int pn = pa; pn < pz; ++pn) {
      const int64_t c1 = __ldg(p.panel_chunk_ptr + pn + 1);
      const int nch = (int)(c1 - c0);
      c0 = c1;
      for (int ft = 0; ft < nft; ++ft) {
        mbar_wait(bTempty + 8 * acc, aphase ^ 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t dcol = tbase + acc * BN;
        for (int c = 0; c < nch; c += CPS) {
          const int sub = min(CPS, nch - c);
          mbar_wait(bFull + 8 * s, ph);
          // the gathers (cp.async) were written through the generic proxy: make them visible
          // to the tensor core's async-proxy operand reads
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
          for (int j = 0; j < CPS; ++j) {
            if (j < sub) {
              const uint64_t ad = adesc0 + (uint64_t)(((s * CPS + j) * C::kRecBytes) >> 4);
              const uint64_t bd = bdesc0 + (uint64_t)(((s * CPS + j) * C::kBBytes) >> 4);
              const uint32_t mcol = C::kMeta0 + CPS * s + j;
              // metadata column: even column address + sparse_id2 selects the odd one
              asm volatile(
                  "{\n\t.reg .pred e, q;\n\t"
                  "elect.sync _|e, 0xffffffff;\n\t"
                  "setp.ne.b32 q, %5, 0;\n\t"
                  "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t}" ::"r"(dcol),
                  "l"(ad), "l"(bd), "r"(tbase + (mcol & ~1u)), "r"(p.idesc | (mcol & 1u)), "r"(c + j)
                  : "memory");
            }
          }
          asm volatile(
              "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
              "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(bEmpty +
                                                                                                            8 * s)
              : "memory");
          if (++s == C::kStages) { s = 0; ph ^= 1; }
        }
        if (nch > 0)
          asm volatile(
              "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
              "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(bTfull +
                                                                                                            8 * acc)
              : "memory");
        else if (lane == 0)
          mbar_arrive(bTfull + 8 * acc);
        __syncwarp();
        if (++acc == C::kNAcc) { acc = 0; aphase ^= 1; }
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue
    // tcgen05.ld 16x256b: thread t holds rows (t/4) and (t/4 + 8) of a 16-lane block, columns
    // 2*(t%4) + {0,1} of every 8-column repetition -> 8-byte stores, four threads complete a
    // 32-byte sector of a Y row
    const int quarter = warp & 3;
    const int cpair = 2 * (lane & 3);
    int acc = 0;
    uint32_t aphase = 0;
    const bool vec_ok = ((p.ldy & 1) == 0) && ((((uintptr_t)p.Y) & 7) == 0);
    int64_t c0 = pa < pz ? __ldg(p.panel_chunk_ptr + pa) : 0;
    for (int pn = pa; pn < pz; ++pn) {
      const int64_t c1 = __ldg(p.panel_chunk_ptr + pn + 1);
      const bool has = c1 > c0;
      c0 = c1;
      int64_t orow[2][2];
#pragma unroll
      for (int b = 0; b < 2; ++b)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int64_t g = (int64_t)pn * kPanelRows + quarter * 32 + b * 16 + (lane >> 2) + 8 * h;
          orow[b][h] = g < p.rows ? (p.row_map ? (int64_t)__ldg(p.row_map + g) : g) : -1;
        }
      for (int ft = 0; ft < nft; ++ft) {
        const bool full_tile = vec_ok && ft * BN + BN <= p.F;
        mbar_wait_sleep(bTfull + 8 * acc, aphase);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
        for (int b = 0; b < 2; ++b) {
          const int64_t olo = orow[b][0], ohi = orow[b][1];
          const uint32_t lane0 = (uint32_t)(quarter * 32 + b * 16);
#pragma unroll 1
          for (int cc = 0; cc < BN; cc += 64) {
            uint32_t v[32];
            if (has) {
              const uint32_t taddr = tbase + (lane0 << 16) + acc * BN + cc;
              asm volatile(
                  "tcgen05.ld.sync.aligned.16x256b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
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
            if (p.H16) {  // fused bias + activation + 16-bit store (F even, 4-byte aligned pairs)
#pragma unroll
              for (int j = 0; j < 8; ++j) {
                const int col = ft * BN + cc + 8 * j + cpair;
                if (col >= p.F) continue;
                if (olo >= 0)
                  *(uint32_t*)(p.H16 + olo * p.ldh + col) =
                      pack_act16(__uint_as_float(v[4 * j]), __uint_as_float(v[4 * j + 1]), p, col);
                if (ohi >= 0)
                  *(uint32_t*)(p.H16 + ohi * p.ldh + col) =
                      pack_act16(__uint_as_float(v[4 * j + 2]), __uint_as_float(v[4 * j + 3]), p, col);
              }
              continue;
            }
            if (full_tile) {
              float* ylo = p.Y + olo * p.ldy + ft * BN + cc + cpair;
              float* yhi = p.Y + ohi * p.ldy + ft * BN + cc + cpair;
#pragma unroll
              for (int j = 0; j < 8; ++j) {
                if (olo >= 0)
                  __stcs((float2*)(ylo + 8 * j), make_float2(__uint_as_float(v[4 * j]), __uint_as_float(v[4 * j + 1])));
                if (ohi >= 0)
                  __stcs((float2*)(yhi + 8 * j),
                         make_float2(__uint_as_float(v[4 * j + 2]), __uint_as_float(v[4 * j + 3])));
              }
              continue;
            }
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              const int col = ft * BN + cc + 8 * j + cpair;
              if (col >= p.F) continue;
              const float2 lo = make_float2(__uint_as_float(v[4 * j]), __uint_as_float(v[4 * j + 1]));
              const float2 hi = make_float2(__uint_as_float(v[4 * j + 2]), __uint_as_float(v[4 * j + 3]));
              if (vec_ok && col + 2 <= p.F) {
                if (olo >= 0) __stcs((float2*)(p.Y + olo * p.ldy + col), lo);
                if (ohi >= 0) __stcs((float2*)(p.Y + ohi * p.ldy + col), hi);
              } else {
                if (olo >= 0) {
                  p.Y[olo * p.ldy + col] = lo.x;
                  if (col + 1 < p.F) p.Y[olo * p.ldy + col + 1] = lo.y;
                }
                if (ohi >= 0) {
                  p.Y[ohi * p.ldy + col] = hi.x;
                  if (col + 1 < p.F) p.Y[ohi * p.ldy + col + 1] = hi.y;
                }
              }
            }
          }
        }
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncwarp();
        if (lane == 0) mbar_arrive(bTempty + 8 * acc);
        if (++acc == C::kNAcc) { acc = 0; aphase ^= 1; }
      }
    }
  }

  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == kWMma) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
  }
}

uint32_t make_idesc_full(nm_dtype dt, int BN) {
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
nm_status launch_full_bn(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                         cudaStream_t s, const FusedAct* fa) {
  using C = FCfg<BN>;
  static int configured_dev = -1;
  int dev = 0;
  NM_CUDA(cudaGetDevice(&dev));
  if (configured_dev != dev) {
    NM_CUDA(cudaFuncSetAttribute(k_spmm_full<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::kSmem));
    configured_dev = dev;
  }
  FullParams prm;
  prm.image = P->image_full;
  prm.panel_chunk_ptr = P->panel_chunk_ptr;
  prm.cta_ptr = P->cta_ptr;
  prm.row_map = P->row_map;
  prm.X = (const uint16_t*)PX;
  prm.ldx = ldx;
  prm.Y = Yp;
  prm.ldy = ldy;
  prm.F = F;
  prm.rows = P->row_end - P->row_begin;
  prm.n_ftiles = (F + BN - 1) / BN;
  prm.idesc = make_idesc_full(P->dtype, BN);
  prm.H16 = fa ? (uint16_t*)fa->out16 : nullptr;
  prm.ldh = fa ? fa->ldo : 0;
  prm.bias = fa ? fa->bias : nullptr;
  prm.relu = fa ? fa->relu : 0;
  prm.bf16_out = P->dtype == NM_BF16;
  if (P->n_ctas < 1 || P->n_panels < 1) return NM_OK;
  k_spmm_full<BN><<<(unsigned)P->n_ctas, kFThreads, C::kSmem, s>>>(prm);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

}  // namespace

nm_status launch_spmm_sptc_full(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                                cudaStream_t s, const FusedAct* fa) {
  if (!P->image_full) return fail(NM_ERR_UNSUPPORTED, "nm_spmm: the pack holds no full-record image");
  if (F <= 64) return launch_full_bn<64>(P, PX, ldx, Yp, ldy, F, s, fa);
  if (F <= 128) return launch_full_bn<128>(P, PX, ldx, Yp, ldy, F, s, fa);
  return launch_full_bn<256>(P, PX, ldx, Yp, ldy, F, s, fa);
}

}  // namespace nm
