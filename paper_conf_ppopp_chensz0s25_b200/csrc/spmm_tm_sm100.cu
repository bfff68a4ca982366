// nm_spmm tensor-core part, COMPRESSED records with the A operand in tensor memory:
// Yp = B_packed * PX on sm_100a sparse tensor cores (nm_spmm_sptc_format 3).
//
// Same work decomposition, warp roles and pipeline as the full-record kernel
// (spmm_full_sm100.cu), but the chunk records are streamed in their compressed HBM form
// (nm_internal.h kRec*: only the non-empty (row, meta-block) value pairs and the nibble words
// of the non-empty rows, ~1.3 KB per C3 chunk instead of 4736 B) and the loader warps expand
// them straight into TENSOR MEMORY: thread r of a gather group owns row r (its TMEM lane),
// rebuilds the row's 8 value words (meta-block g = word g, slots 2g / 2g+1 in its halves) with
// at most 8 shared-memory loads and writes them with one tcgen05.st.32x32b.x8; the metadata
// lane words (two rows' nibbles per lane, nm_internal.h) come from two shuffles of the rows'
// nibble words.  The MMA reads A from TMEM (tcgen05.mma.sp [d], [a], b-desc, [e]), so no
// shared-memory expansion pass and no A tile in shared memory.
// Warp roles (persistent, one CTA per SM, 6 + 4 x NM_TM_GROUPS warps):
//   w0     record producer: one bulk copy of the stage's (1-2 adjacent) compressed records
//   w1..   gather groups of 4 warps (one per TMEM lane quarter): X gathers (cp.async, as the
//          full kernel) + A and metadata expansion into TMEM
//   then   the MMA issuer (+ TMEM allocation) and 4 epilogue warps (as the full kernel)
#include "nm_internal.h"

namespace nm {
namespace {

#ifndef NM_TM_GROUPS
#define NM_TM_GROUPS 4
#endif
constexpr int kTGroups = NM_TM_GROUPS;  // gather + expansion groups (4 warps each)
constexpr int kWProd = 0, kWG0 = 1, kWMma = kWG0 + 4 * kTGroups, kWEpi0 = kWMma + 1;
constexpr int kTThreads = (kWEpi0 + 4) * 32;  // 22 warps at 4 groups
constexpr int kGThreads = 128;
#ifndef NM_TM_PF_KB
#define NM_TM_PF_KB 16
#endif
constexpr int kPfBytes = NM_TM_PF_KB * 1024;  // records L2-prefetched ahead of the stream

struct TmParams {
  const uint8_t* image;            // compressed records, chunk order
  const uint16_t* len16;           // [n_chunks] record size / 16
  const int4* unit_info;           // [2 * n_panels] {panel, #chunks, chunk lo, hi}, {byte off lo, hi, size lo, hi}
  const int64_t* panel_chunk_ptr;  // [n_panels + 1]
  const int32_t* cta_ptr;          // [gridDim.x + 1]
  const int32_t* row_map;
  const uint16_t* X;
  int64_t ldx;
  float* Y;
  int64_t ldy;
  int F;
  int64_t rows;
  int n_ftiles;
  uint32_t idesc;
};

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


__device__ __forceinline__ uint32_t lds8(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}

__device__ __forceinline__ uint32_t lds16(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}

template <int BN>
struct TCfg {
  static constexpr int kCPS = BN <= 128 ? 2 : 1;               // chunks per stage
  static constexpr int kBBytes = 32 * BN * 2;
  static constexpr int kRecSlot = kCPS * kRecMaxBytes;          // worst-case record bytes per stage
  static constexpr int kStageBytes = kCPS * kBBytes + ((kRecSlot + 127) & ~127);
  static constexpr int kStagesRaw = (222 * 1024 - 2048) / kStageBytes;
  static constexpr int kMaxStages = 16 / kCPS;
  static constexpr int kStages = ((kStagesRaw > kMaxStages ? kMaxStages : kStagesRaw) / kTGroups) * kTGroups;
  static constexpr int kACols = 8 * kCPS * kStages;            // A: 8 columns (16 bf16) per chunk
  static constexpr int kMetaCols = kCPS * kStages;
  static constexpr int kNAcc = (3 * BN + kACols + kMetaCols <= 512) ? 3 : (2 * BN + kACols + kMetaCols <= 512) ? 2 : 1;
  static constexpr int kA0 = kNAcc * BN;                       // A column of (stage s, chunk j): kA0 + 8 (kCPS s + j)
  static constexpr int kMeta0 = kA0 + kACols;                  // metadata column: kMeta0 + kCPS s + j
  static constexpr int kSmem = 1024 + kStages * kStageBytes + 1024;
  static_assert(kMeta0 + kMetaCols <= 512, "TMEM budget");
  static_assert(kSmem <= 227 * 1024, "smem");
  static_assert(kStages >= 2, "stages");
};

template <int BN>
__global__ void __launch_bounds__(kTThreads, 1) k_spmm_tm(const TmParams p) {
  using C = TCfg<BN>;
  constexpr int CPS = C::kCPS;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const uint32_t sB = smem_u32(smem);                          // stage s: CPS B tiles (SW128)
  const uint32_t sRec = sB + C::kStages * CPS * C::kBBytes;    // stage s: records at sRec + s * slot
  constexpr uint32_t kSlot = (C::kRecSlot + 127) & ~127;
  uint64_t* bars = (uint64_t*)(smem + C::kStages * C::kStageBytes);
  uint64_t* full_rec = bars;
  uint64_t* full_b = full_rec + C::kStages;
  uint64_t* empty = full_b + C::kStages;
  uint64_t* tfull = empty + C::kStages;
  uint64_t* tempty = tfull + 4;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 4);
  const uint32_t bRec = smem_u32(full_rec), bFull = smem_u32(full_b), bEmpty = smem_u32(empty);
  const uint32_t bTfull = smem_u32(tfull), bTempty = smem_u32(tempty);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::kStages; ++s) {
      mbar_init(bRec + 8 * s, 1);
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
    uint64_t pol_stream;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_stream));
    int s = 0;
    uint32_t ph = 0;
    // L2 prefetch window over the CTA's (contiguous) record bytes
    const int4 ua = pa < pz ? __ldg(p.unit_info + 2 * pa + 1) : make_int4(0, 0, 0, 0);
    const int64_t cta_b0 = (int64_t)(uint32_t)ua.x | ((int64_t)ua.y << 32);
    int64_t cta_b1 = cta_b0;
    if (pa < pz) {
      const int4 uz = __ldg(p.unit_info + 2 * (pz - 1) + 1);
      cta_b1 = ((int64_t)(uint32_t)uz.x | ((int64_t)uz.y << 32)) + ((int64_t)(uint32_t)uz.z | ((int64_t)uz.w << 32));
    }
    int64_t pf = cta_b0;  // prefetched up to here
    int64_t c0 = pa < pz ? __ldg(p.panel_chunk_ptr + pa) : 0;
    for (int pn = pa; pn < pz; ++pn) {
      const int64_t c1 = __ldg(p.panel_chunk_ptr + pn + 1);
      const int nch = (int)(c1 - c0);
      const int4 ub = __ldg(p.unit_info + 2 * pn + 1);
      const int64_t pb0 = (int64_t)(uint32_t)ub.x | ((int64_t)ub.y << 32);
      for (int ft = 0; ft < nft; ++ft) {
        int64_t off = pb0;
        for (int c = 0; c < nch; c += CPS) {
          const int sub = min(CPS, nch - c);
          uint32_t bytes = 16u * __ldg(p.len16 + c0 + c);
          if (sub > 1) bytes += 16u * __ldg(p.len16 + c0 + c + 1);
          mbar_wait(bEmpty + 8 * s, ph ^ 1);
          if (lane == 0) {
            while (pf < cta_b1 && pf < off + kPfBytes) {  // keep the window kPfBytes ahead
              const int64_t k = min((int64_t)32768, cta_b1 - pf);
              asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(p.image + pf),
                           "r"((uint32_t)k), "l"(pol_stream)
                           : "memory");
              pf += k;
            }
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bRec + 8 * s), "r"(bytes)
                         : "memory");
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
                "%4;" ::"r"(sRec + s * kSlot),
                "l"(p.image + off), "r"(bytes), "r"(bRec + 8 * s), "l"(pol_stream)
                : "memory");
          }
          __syncwarp();
          off += bytes;
          if (++s == C::kStages) { s = 0; ph ^= 1; }
        }
      }
      c0 = c1;
    }
  } else if (warp >= kWG0 && warp < kWG0 + 4 * kTGroups) {
    // ------------------------------------------------------------ gathers + A / metadata into TMEM
    const int group = (warp - kWG0) >> 2;
    const int quarter = warp & 3;          // TMEM lane quarter = rows 32 quarter .. +31
    const int t = threadIdx.x - (kWG0 + 4 * group) * 32;
    constexpr int kRowPieces = BN / 8;
    constexpr int kPer = 32 * kRowPieces / kGThreads;
    constexpr int kRowsPerPass = kGThreads / kRowPieces;
    const int c16 = t % kRowPieces, kk0 = t / kRowPieces;
    const uint32_t dcol = (uint32_t)(c16 >> 3) * 4096u;
    const uint32_t ldxb = (uint32_t)p.ldx * 2u;  // row pitch in bytes
    const int row = quarter * 32 + lane;   // the A row (TMEM lane) this thread expands
    // metadata lane word of this lane: rows ra = (lane % 8) + 16 (lane / 16) and ra + 8 of the
    // quarter, K-half k1 = (lane / 8) % 2 (nm_internal.h meta layout)
    const int src_a = (lane & 7) + 16 * (lane >> 4), src_b = src_a + 8, k1 = (lane >> 3) & 1;
    uint64_t pol_x;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_x));
    // this group's stages only: i = group, group + kTGroups, ... (stage s = i mod kStages)
    StageIter<CPS> it;
    it.init(p.panel_chunk_ptr, pa, pz, nft);
    it.advance(group);
    for (int i = group; it.valid(); i += kTGroups, it.advance(kTGroups)) {
      const int s = i % C::kStages;
      const uint32_t ph = (uint32_t)((i / C::kStages) & 1);
      const int col0 = it.ft * BN + c16 * 8;
      const uint32_t colbytes = col0 >= p.F ? 0u : (p.F - col0 >= 8 ? 16u : (uint32_t)(p.F - col0) * 2u);
      const uint16_t* xcol = p.X + (colbytes ? col0 : 0);
      const int sub = min(CPS, it.nch - it.c);
      mbar_wait(bRec + 8 * s, ph);
      uint32_t rec = sRec + s * kSlot;
      uint32_t mw[CPS];
#pragma unroll
      for (int j = 0; j < CPS; ++j) {
        uint32_t w[8];
        if (j < sub) {
          // X gathers of the chunk's 32 rows (gather row list at the record's start)
          const uint32_t sbase = sB + (s * CPS + j) * C::kBBytes + dcol;
#pragma unroll
          for (int q = 0; q < kPer; ++q) {
            const int kk = q * kRowsPerPass + kk0;
            const int32_t xr = (int32_t)lds32(rec + 4 * kk);
            // byte address of row xr: one 32 x 32 -> 64-bit multiply-add (rows, ldx < 2^31)
            const uint64_t src = (uint64_t)(uint32_t)max(xr, 0) * ldxb + (uint64_t)(uintptr_t)xcol;
            const uint32_t dst =
                sbase + (kk >> 3) * 1024 + (kk & 7) * 128 + ((((uint32_t)c16 ^ (uint32_t)kk) & 7u) << 4);
            if (colbytes == 16u)  // full 16-byte piece: ignore-src zero fill for the -1 rows
              asm volatile(
                  "{\n\t.reg .pred q;\n\tsetp.lt.s32 q, %2, 0;\n\t"
                  "cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, q, %3;\n\t}" ::"r"(dst),
                  "l"(src), "r"(xr), "l"(pol_x)
                  : "memory");
            else  // the F tail: partial or empty pieces
              asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2, %3;" ::"r"(dst), "l"(src),
                           "r"(xr >= 0 ? colbytes : 0u), "l"(pol_x)
                           : "memory");
          }
          // A row and nibble word of this thread's row
          const uint32_t mask = lds8(rec + kRecMaskOff + row);
          const uint32_t tot = lds32(rec + kRecTotOff);
          const uint32_t ne = tot & 0xFFFFu;
          const uint32_t cnt = __popc(mask), has = mask ? 1u : 0u;
          // both inclusive warp scans in one register (counts <= 256 per quarter)
          uint32_t sc = cnt | (has << 16);
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const uint32_t a = __shfl_up_sync(0xffffffffu, sc, o);
            if (lane >= o) sc += a;
          }
          const uint32_t pv = sc & 0xFFFFu, pn_ = sc >> 16;
          const uint32_t qv = lds16(rec + kRecQvOff + 2 * quarter), qn = lds16(rec + kRecQnOff + 2 * quarter);
          uint32_t e = qv + pv - cnt;
          const uint32_t vbase = rec + kRecHdrBytes;
#pragma unroll
          for (int g = 0; g < 8; ++g) {
            w[g] = 0u;
            if (mask & (1u << g)) w[g] = lds32(vbase + 4 * e++);
          }
          const uint32_t W = has ? lds32(vbase + 4 * (ne + qn + pn_ - 1)) : kMetaNone;
          const uint32_t Wa = __shfl_sync(0xffffffffu, W, src_a), Wb = __shfl_sync(0xffffffffu, W, src_b);
          mw[j] = ((Wa >> (16 * k1)) & 0xFFFFu) | (((Wb >> (16 * k1)) & 0xFFFFu) << 16);
          rec += 16u * (uint32_t)((kRecHdrBytes + 4 * (ne + (tot >> 16)) + 15) / 16);
        } else {
#pragma unroll
          for (int g = 0; g < 8; ++g) w[g] = 0u;
          mw[j] = kMetaNone;
        }
        const uint32_t ta = tbase + ((uint32_t)(quarter * 32) << 16) + C::kA0 + 8 * (CPS * s + j);
        asm volatile(
            "tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"r"(ta), "r"(w[0]),
            "r"(w[1]), "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7])
            : "memory");
      }
      asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bFull + 8 * s) : "memory");
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
    // ------------------------------------------------------------ MMA issuer (A from TMEM)
    int s = 0;
    uint32_t ph = 0;
    int acc = 0;
    uint32_t aphase = 0;
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
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
          for (int j = 0; j < CPS; ++j) {
            if (j < sub) {
              const uint32_t acol = tbase + C::kA0 + 8 * (CPS * s + j);
              const uint64_t bd = bdesc0 + (uint64_t)(((s * CPS + j) * C::kBBytes) >> 4);
              const uint32_t mcol = C::kMeta0 + CPS * s + j;
              asm volatile(
                  "{\n\t.reg .pred e, q;\n\t"
                  "elect.sync _|e, 0xffffffff;\n\t"
                  "setp.ne.b32 q, %5, 0;\n\t"
                  "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], [%1], %2, [%3], %4, q;\n\t}" ::"r"(dcol),
                  "r"(acol), "l"(bd), "r"(tbase + (mcol & ~1u)), "r"(p.idesc | (mcol & 1u)), "r"(c + j)
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

uint32_t make_idesc_tm(nm_dtype dt, int BN) {
  uint32_t d = 0;
  d |= 1u << 2;   // sparse
  d |= 1u << 4;   // D = f32
  if (dt == NM_BF16) d |= (1u << 7) | (1u << 10);
  d |= 1u << 16;  // B MN-major (A K-major, in TMEM)
  d |= (uint32_t)(BN >> 3) << 17;
  d |= (uint32_t)(128 >> 4) << 24;
  return d;
}

template <int BN>
nm_status launch_tm_bn(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                       cudaStream_t s) {
  using C = TCfg<BN>;
  static int configured_dev = -1;
  int dev = 0;
  NM_CUDA(cudaGetDevice(&dev));
  if (configured_dev != dev) {
    NM_CUDA(cudaFuncSetAttribute(k_spmm_tm<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::kSmem));
    configured_dev = dev;
  }
  TmParams prm;
  prm.image = P->image;
  prm.len16 = P->rec_len16;
  prm.unit_info = P->unit_info;
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
  prm.idesc = make_idesc_tm(P->dtype, BN);
  if (P->n_ctas < 1 || P->n_panels < 1) return NM_OK;
  k_spmm_tm<BN><<<(unsigned)P->n_ctas, kTThreads, C::kSmem, s>>>(prm);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

}  // namespace

nm_status launch_spmm_sptc_tm(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                              cudaStream_t s) {
  if (!P->image || !P->rec_len16 || !P->unit_info)
    return fail(NM_ERR_UNSUPPORTED, "nm_spmm: the pack holds no compressed image");
  if (F <= 64) return launch_tm_bn<64>(P, PX, ldx, Yp, ldy, F, s);
  if (F <= 128) return launch_tm_bn<128>(P, PX, ldx, Yp, ldy, F, s);
  return launch_tm_bn<256>(P, PX, ldx, Yp, ldy, F, s);
}

}  // namespace nm
