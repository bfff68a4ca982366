// nm_spmm tensor-core part: Yp = B_packed * PX on sm_100a sparse tensor cores.
//
// One work unit = (panel of 128 rows of B, 64..256-column tile of F).  The K dimension of a
// panel is its list of non-empty meta-blocks; 8 meta-blocks (4 selected columns each) form
// one K = 32 chunk, i.e. one tcgen05.mma.sp.cta_group::1.kind::f16 with M = 128, N = BN:
//   record (compressed chunk, nm_internal.h kRec*)  <- one cp.async.bulk (HBM stream)
//   A (128 x 16 physical values, K-major)          <- expanded from the record by the loaders
//   B (32 gathered rows of X x BN, SWIZZLE_128B MN-major)  <- cp.async 16-byte gathers
//   E (metadata, 128 lanes x 32 b)                  <- tcgen05.st of the expanded nibbles
//   D (fp32, 128 x BN)                              in tensor memory (tcgen05.ld out)
// The record is the paper's matrix put "into the SPTC required form on the fly" (L492): HBM
// holds only the non-empty (row, meta-block) slots; the dense operand exists only in SMEM.
// Warp roles (persistent, one CTA per SM, 23 warps with the defaults NM_LOAD_GROUPS = 4,
// NM_EPI_WARPS = 4, NM_PRODUCERS = 2):
//   w0      record producer 0 (bulk copies into its half of the byte ring) + L2 prefetch of
//           the next units' records
//   w1-16   loaders, four groups of 4 warps, group g owns the stages s = g (mod 4): X gathers,
//           record expansion into the A tile, metadata into TMEM
//   w17     MMA issuer (+ TMEM allocation)
//   w18-21  epilogue, one warp per TMEM lane quarter: tcgen05.ld 16x256b -> sector-aligned
//           stores of Y rows (no shared-memory staging)
//   w22     record producer 1 (alternate units, the other ring half)
// All hand-offs are mbarriers; the pipeline runs across work units, so consecutive panels
// overlap, and every role prefetches the next unit's schedule entry.  Design evidence
// (DESIGN.md §6): TMA tile::gather4 costs ~57 cycles per instruction on B200, so X rows are
// gathered with cp.async; one loader group spent ~950 cycles per chunk (clock64 timeline,
// tools/trace_spmm.py), so several groups share the stages.  (nm_spmm_sptc_format 2; the
// default tensor-core kernel is spmm_full_sm100.cu.)
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <cstdio>
#include <cstdlib>

#include "nm_internal.h"

namespace nm {
namespace {

#ifndef NM_LOAD_GROUPS
#define NM_LOAD_GROUPS 4
#endif
constexpr int kWarpRec = 0, kWarpLoad0 = 1, kLoadGroups = NM_LOAD_GROUPS;
#ifndef NM_PRODUCERS
#define NM_PRODUCERS 2               // record producer warps (alternate units, own ring halves)
#endif
constexpr int kProducers = NM_PRODUCERS;
constexpr int kSlotsShift = kProducers == 1 ? 6 : kProducers == 2 ? 5 : 4;
constexpr int kSlotsPP = 1 << kSlotsShift;    // record descriptors per producer (power of two)
constexpr int kRecSlots = kSlotsPP * kProducers;
static_assert(kProducers >= 1 && kProducers <= 3, "one to three record producers");
static_assert((1 << kSlotsShift) == kSlotsPP, "descriptor count");
#ifndef NM_EPI_WARPS
#define NM_EPI_WARPS 4
#endif
constexpr int kWarpMma = kWarpLoad0 + 4 * kLoadGroups, kWarpEpi0 = kWarpMma + 1, kEpiWarps = NM_EPI_WARPS;
constexpr int kWarpRec2 = kWarpEpi0 + kEpiWarps;  // producers 1.. (kProducers > 1)
constexpr int kThreads = (kWarpEpi0 + kEpiWarps + kProducers - 1) * 32;
static_assert(kEpiWarps == 4 || kEpiWarps == 8, "epilogue: one or two warps per TMEM lane quarter");
constexpr int kGroupThreads = 128;                     // loader threads per group
constexpr int kPrefetchUnits = 2;                      // record L2-prefetch distance (units)
// compressed records land in byte rings, one per producer (allocated in chunk order; a record
// that runs past the end continues into a kRecMaxBytes pad, so every record is contiguous
// without skipping), each described by kSlotsPP descriptors: a producer's j-th record uses
// descriptor j % kSlotsPP
#ifndef NM_REC_CPASYNC
#define NM_REC_CPASYNC 0             // records by warp-wide cp.async instead of one bulk copy each
#endif
constexpr int kIssueLanes = 8;       // records whose bulk copies are issued together
#ifndef NM_SMEM_BUDGET
#define NM_SMEM_BUDGET (214 * 1024)  // stages + record rings (barriers and alignment on top)
#endif
#ifndef NM_MIN_RING
#define NM_MIN_RING (32 * 1024)      // ring bytes reserved before the stage count is chosen
#endif

struct SpmmParams {
  const uint8_t* image;
  const int4* unit_info;   // 2 per scheduled panel: {panel, #chunks, first chunk lo, hi}, {byte off, bytes}
  const uint16_t* rec_len16;  // compressed record size / 16 per chunk
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
  int debug;                  // profiling switches (NM_SPMM_DEBUG, results invalid): 2 = no Y stores,
                              // 32 = no TMA row tiles, 64 = no record expansion, 128 = no
                              // X gathers, 512 = no record
                              // L2 prefetch, 1024 = no records (with 32|64|128 only)
  unsigned long long* trace;  // NM_SPMM_TRACE: per-chunk clock64 timeline of CTA 0
};

// profiling switches (NM_SPMM_DEBUG, results invalid): compiled in only with
// -DNM_SPMM_DEBUG_BUILD (NM_NVCC_FLAGS); the product kernel reads no switch and skips nothing
#ifdef NM_SPMM_DEBUG_BUILD
#define NM_DBG(p) ((p).debug)
#else
#define NM_DBG(p) 0
#endif

// clock64 timeline of CTA 0 (tools/trace_spmm.py): compiled in only with -DNM_SPMM_TRACE_BUILD
// (NM_NVCC_FLAGS), so the product kernel carries no trace instructions
#ifdef NM_SPMM_TRACE_BUILD
#define NM_TRACE_ON 1
#else
#define NM_TRACE_ON 0
#endif
#define NM_TRACE(slot)                                                                              \
  do {                                                                                              \
    if (NM_TRACE_ON && p.trace && blockIdx.x == 0 && i < 1024) p.trace[i * 8 + (slot)] = clock64(); \
  } while (0)
#define NM_TRACE_U(slot)                                                                            \
  do {                                                                                              \
    if (NM_TRACE_ON && p.trace && blockIdx.x == 0 && lane == 0 && (u / ustep) < 1024)               \
      p.trace[8192 + (u / ustep) * 4 + (slot)] = clock64();                                         \
  } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

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

__device__ __forceinline__ void sts128(uint32_t a, uint32_t x, uint32_t y, uint32_t z, uint32_t w) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(x), "r"(y), "r"(z), "r"(w) : "memory");
}

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
      "NM_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra NM_WAIT_%=;\n\t}" ::"r"(a),
      "r"(parity)
      : "memory");
}

// long waits (the epilogue waiting for a whole unit of MMAs): back off so the spinning warps
// do not take issue slots from the loaders (ncu: 20% of executed instructions were this spin)
__device__ __forceinline__ void mbar_wait_sleep(uint32_t a, uint32_t parity) {
  // try_wait with a suspend-time hint: the warp is descheduled until the phase completes (or
  // ~1 ms passes), so it neither spins nor oversleeps the hand-off
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

// 16-byte cp.async whose source is ignored (destination zero-filled) when ign is true
__device__ __forceinline__ void cp_async16_ign(uint32_t dst, const void* src, bool ign) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t"
      "cp.async.cg.shared.global [%0], [%1], 16, q;\n\t}" ::"r"(dst),
      "l"(src), "r"((int)ign)
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

// unit u = (scheduled panel u / n_ftiles, F tile u % n_ftiles); n_units < 2^31 (host check),
// so 32-bit division -- a 64-bit one is a ~70-instruction sequence on every role's unit step
__device__ __forceinline__ uint32_t unit_panel(const SpmmParams& p, int64_t u) {
  return p.n_ftiles == 1 ? (uint32_t)u : (uint32_t)u / (uint32_t)p.n_ftiles;
}
__device__ __forceinline__ int unit_ft(const SpmmParams& p, int64_t u) {
  return p.n_ftiles == 1 ? 0 : (int)((uint32_t)u % (uint32_t)p.n_ftiles);
}
// schedule entry of unit u (prefetched one unit ahead by every role): {panel, #chunks, c0}
__device__ __forceinline__ int4 unit_entry(const SpmmParams& p, int64_t u) {
  return u < p.n_units ? __ldg(p.unit_info + 2 * unit_panel(p, u)) : make_int4(0, 0, 0, 0);
}
// {record byte offset lo, hi, record bytes lo, hi} of unit u
__device__ __forceinline__ int4 unit_bytes(const SpmmParams& p, int64_t u) {
  return u < p.n_units ? __ldg(p.unit_info + 2 * unit_panel(p, u) + 1) : make_int4(0, 0, 0, 0);
}
__device__ __forceinline__ int64_t entry_c0(int4 e) { return (int64_t)(uint32_t)e.z | ((int64_t)e.w << 32); }
__device__ __forceinline__ int64_t lo_hi(int a, int b) { return (int64_t)(uint32_t)a | ((int64_t)b << 32); }

template <int BN>
struct Cfg {
  static constexpr int kABytes = kChunkValBytes;                // 128 x 16 values (4096)
  static constexpr int kBBytes = 32 * BN * 2;                   // 32 K-rows x BN halves
  static constexpr int kStageBytes = kABytes + kBBytes;
  static constexpr int kStagesRaw = (NM_SMEM_BUDGET - NM_MIN_RING - kRecMaxBytes) / kStageBytes;
  // a multiple of the loader-group count: group g owns stages s % kLoadGroups == g, so every
  // stage has one consumer group that visits it in chunk order (parity waits stay valid)
  static constexpr int kStages = ((kStagesRaw > 16 ? 16 : kStagesRaw) / kLoadGroups) * kLoadGroups;
  // the record ring takes what the stages leave (largest power of two, >= 32 KB)
  static constexpr int kRingAvail = NM_SMEM_BUDGET - kStages * kStageBytes - kProducers * kRecMaxBytes;
  static constexpr int kRingPer = kRingAvail / kProducers;
  static constexpr int kRecRing =  // each producer's ring: the largest power of two that fits
      kRingPer >= 64 * 1024 ? 64 * 1024 : kRingPer >= 32 * 1024 ? 32 * 1024 : 16 * 1024;
  static constexpr int kRingStride = kRecRing + kRecMaxBytes; // ring + wrap pad per producer
  static constexpr int kRecRegion = kProducers * kRingStride;
  // accumulators in TMEM (units in flight between the MMA issuer and the epilogue)
  static constexpr int kNAcc = (3 * BN + kStages <= 512) ? 3 : (2 * BN + kStages <= 512) ? 2 : 1;
  static constexpr int kMeta0 = kNAcc * BN;                     // metadata column of stage s: kMeta0 + s
  static constexpr int kBRegion = kStages * kBBytes;            // 1024-aligned tiles (SW128)
  static constexpr int kSmem = 1024 + kBRegion + kStages * kABytes + kRecRegion + 2048;
  static_assert(kMeta0 + kStages <= 512, "TMEM budget");
  static_assert(BN % 64 == 0 && BN >= 64 && BN <= 256, "BN");
  static_assert(kSmem <= 227 * 1024, "smem");
  static_assert(kRecMaxBytes % 16 == 0 && kRecRing >= 2 * kRecMaxBytes,
                "record ring");
};

template <int BN>
__global__ void __launch_bounds__(kThreads, 1) k_spmm_sptc(const SpmmParams p, const __grid_constant__ CUtensorMap tmX) {
  using C = Cfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const uint32_t sB = smem_u32(smem);                  // kStages B tiles (1024-aligned)
  const uint32_t sA = sB + C::kBRegion;                // kStages A tiles
  const uint32_t sRec = sA + C::kStages * C::kABytes;  // kRecSlots compressed records
  uint64_t* bars = (uint64_t*)(smem + C::kBRegion + C::kStages * C::kABytes + C::kRecRegion);
  uint64_t* rec_full = bars;                // record landed (tx)
  uint64_t* rec_empty = bars + kRecSlots;   // record expanded by its loader group
  uint64_t* full_b = rec_empty + kRecSlots; // A tile + gathers + metadata ready
  uint64_t* empty = full_b + C::kStages;    // MMA done with the stage (tcgen05.commit)
  uint64_t* tfull = empty + C::kStages;     // accumulator ready (2)
  uint64_t* tempty = tfull + 4;             // accumulator drained (kNAcc <= 4)
  uint32_t* tmem_slot = (uint32_t*)(tempty + 4);
  uint32_t* rec_off = tmem_slot + 4;        // [kRecSlots] ring offset of each descriptor's record
  uint32_t* rec_end = rec_off + kRecSlots;  // [kRecSlots] producer-private: cumulative end of each record

  // shared-window addresses of the barrier arrays (index i at base + 8 i)
  const uint32_t bRecFull = smem_u32(rec_full), bRecEmpty = smem_u32(rec_empty);
  const uint32_t bFull = smem_u32(full_b), bEmpty = smem_u32(empty);
  const uint32_t bTfull = smem_u32(tfull), bTempty = smem_u32(tempty);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < kRecSlots; ++s) {
      mbar_init(smem_u32(&rec_full[s]), NM_REC_CPASYNC ? 32 : 1);  // cp.async lanes / one expect_tx
      mbar_init(smem_u32(&rec_empty[s]), kGroupThreads / 32);  // one arrival per loader warp
    }
    for (int s = 0; s < C::kStages; ++s) {
      // per-thread cp.async completions + one arrival per loader warp (A tile / metadata written)
      mbar_init(smem_u32(&full_b[s]), kGroupThreads + kGroupThreads / 32);
      mbar_init(smem_u32(&empty[s]), 1);
    }
    for (int a = 0; a < 4; ++a) {
      mbar_init(smem_u32(&tfull[a]), 1);
      mbar_init(smem_u32(&tempty[a]), kEpiWarps);
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
  const int64_t ustep = gridDim.x;

  if (warp == kWarpRec || (kProducers > 1 && warp >= kWarpRec2)) {
    // ------------------------------------------------------------ record producer (HBM stream)
    // kProducers warps take alternate units of the CTA (producer pw: unit ordinals k with
    // k % kProducers == pw), each with its own half of the ring and its own kSlotsPP
    // descriptors, so record issue is not one warp's serial chain.
    // the warp reads the record sizes of 32 chunks at a time (one unit ahead); lane 0
    // allocates ring space -- waiting, oldest first, for the loader groups to release older
    // records -- and issues the bulk copies.  Lane 0's per-record path is kept short (32-bit
    // wrapping counters, no divisions): it is a serial chain on one thread.
    const int pw = warp == kWarpRec ? 0 : 1 + warp - kWarpRec2;
    const uint32_t sRecP = sRec + pw * C::kRingStride;  // this producer's ring
    const uint32_t bRecFullP = bRecFull + 8 * pw * kSlotsPP, bRecEmptyP = bRecEmpty + 8 * pw * kSlotsPP;
    uint32_t* rec_offP = rec_off + pw * kSlotsPP;
    uint32_t* rec_endP = rec_end + pw * kSlotsPP;
    const int64_t pstep = kProducers * ustep;  // unit stride of this producer
    uint32_t head = 0, tail = 0;       // cumulative ring bytes allocated / released (mod 2^32)
    int ds = 0, os = 0;                // next descriptor to fill / oldest one not yet released
    uint32_t oph = 0;                  // use parity of the oldest descriptor
    int in_flight = 0;                 // records issued and not yet known to be released
    int64_t i = 0;                     // chunk counter (trace only)
    int nsb = 0;                       // sub-batch counter (trace only)
    auto prefetch_unit = [&](int4 b) {  // the records of a panel are contiguous: one L2 prefetch
      const int64_t len = lo_hi(b.z, b.w);
      if (lane == 0 && len > 0 && !(NM_DBG(p) & 512))
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p.image + lo_hi(b.x, b.y)),
                     "r"((uint32_t)len)
                     : "memory");
    };
    auto first_lens = [&](int4 e) -> uint32_t {  // sizes of a unit's first 32 records (lane j)
      return lane < e.y ? 16u * __ldg(p.rec_len16 + entry_c0(e) + lane) : 0u;
    };
    const int64_t u0 = blockIdx.x + pw * ustep;
    for (int k = 0; k < kPrefetchUnits; ++k) prefetch_unit(unit_bytes(p, u0 + k * pstep));
    // schedule lookahead: entries two units ahead, record sizes one unit ahead (from an entry
    // that is already in registers), so no HBM round trip sits between two units' issues
    int4 e1 = unit_entry(p, u0), b1 = unit_bytes(p, u0);
    int4 e2 = unit_entry(p, u0 + pstep), b2 = unit_bytes(p, u0 + pstep);
    int4 pfb = unit_bytes(p, u0 + kPrefetchUnits * pstep);
    uint32_t nlen = first_lens(e1);
    for (int64_t u = u0; u < p.n_units; u += pstep) {
      const int4 cur = e1, curb = b1;
      uint32_t len = nlen;
      e1 = e2;
      b1 = b2;
      e2 = unit_entry(p, u + 2 * pstep);
      b2 = unit_bytes(p, u + 2 * pstep);
      nlen = first_lens(e1);
      prefetch_unit(pfb);
      pfb = unit_bytes(p, u + (kPrefetchUnits + 1) * pstep);
      const int64_t c0 = entry_c0(cur);
      const int nch = cur.y;
      int64_t boff = lo_hi(curb.x, curb.y);
      uint32_t blen = 0;  // sizes of the next batch of 32 records of this unit, one batch ahead
      for (int b0 = 0; b0 < ((NM_DBG(p) & 1024) ? 0 : nch); b0 += 32) {
        const int cnt = min(32, nch - b0);
        if (b0 > 0) len = blen;
        if (b0 + 32 < nch) blen = lane < nch - b0 - 32 ? 16u * __ldg(p.rec_len16 + c0 + b0 + 32 + lane) : 0u;
        uint32_t incl = len;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t a = __shfl_up_sync(0xffffffffu, incl, o);
          if (lane >= o) incl += a;
        }
        // sub-batches of up to kIssueLanes records: lane 0 makes room for all of them, then
        // each lane issues its own record's bulk copy (the issues overlap across lanes)
        const uint32_t excl = incl - len;
        for (int sb = 0, m = 0; sb < cnt; sb += m) {
          // the sub-batch: up to kIssueLanes records totalling at most half the ring
          const uint32_t e0 = __shfl_sync(0xffffffffu, excl, sb);
          m = __popc(__ballot_sync(0xffffffffu, lane >= sb && lane < sb + kIssueLanes && lane < cnt &&
                                                    incl - e0 <= (uint32_t)(C::kRecRing / 2)));
          const uint32_t total = __shfl_sync(0xffffffffu, incl, sb + m - 1) - e0;
          if (NM_TRACE_ON && p.trace && blockIdx.x == 0 && pw == 0 && lane == 0 && nsb < 1024) {
            p.trace[12288 + 4 * nsb] = clock64();
            p.trace[12290 + 4 * nsb] = ((uint64_t)in_flight << 32) | (head - tail);
          }
          if (lane == 0) {
            int nw = 0;
            while (head + total - tail > (uint32_t)C::kRecRing || in_flight + m > kSlotsPP) {
              ++nw;
              mbar_wait(bRecEmptyP + 8 * os, oph);
              tail = rec_endP[os];
              --in_flight;
              if (++os == kSlotsPP) { os = 0; oph ^= 1; }
            }
            if (NM_TRACE_ON && p.trace && blockIdx.x == 0 && pw == 0 && nsb < 1024) {
              p.trace[12289 + 4 * nsb] = clock64();
              p.trace[12291 + 4 * nsb] = ((uint64_t)nw << 32) | (uint32_t)m;
            }
          }
          ++nsb;
          const uint32_t h0 = __shfl_sync(0xffffffffu, head, 0);
          const int d0 = __shfl_sync(0xffffffffu, ds, 0);
#if NM_REC_CPASYNC
          // records through the LSU: the warp copies each record with 16-byte cp.async (512 B
          // per instruction) and every lane's cp.async.mbarrier.arrive.noinc marks it landed
          for (int k = 0; k < m; ++k) {
            int d = d0 + k;
            if (d >= kSlotsPP) d -= kSlotsPP;
            const uint32_t ek = __shfl_sync(0xffffffffu, excl, sb + k);
            const uint32_t lk = __shfl_sync(0xffffffffu, len, sb + k);
            const uint32_t start = h0 + (ek - e0);
            const uint32_t pos = start & (uint32_t)(C::kRecRing - 1);
            if (lane == 0) {
              rec_endP[d] = start + lk;
              rec_offP[d] = pos;
            }
            const uint8_t* src = p.image + boff + ek;
            for (uint32_t o = 16u * lane; o < lk; o += 512u) cp_async16(sRecP + pos + o, src + o, 16u);
            asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bRecFullP + 8 * d) : "memory");
          }
#else
          if (lane >= sb && lane < sb + m) {
            int d = d0 + (lane - sb);
            if (d >= kSlotsPP) d -= kSlotsPP;
            const uint32_t start = h0 + (excl - e0);
            const uint32_t pos = start & (uint32_t)(C::kRecRing - 1);
            rec_endP[d] = start + len;
            rec_offP[d] = pos;
            mbar_arrive_tx(bRecFullP + 8 * d, len);
            bulk_g2s(sRecP + pos, p.image + boff + excl, len, bRecFullP + 8 * d);
          }
#endif
          if (lane == 0) {
            if (NM_TRACE_ON && kProducers == 1 && p.trace && blockIdx.x == 0 && i < 1024) p.trace[i * 8] = clock64();
            head += total;
            in_flight += m;
            ds += m;
            if (ds >= kSlotsPP) ds -= kSlotsPP;
          }
          i += m;
          __syncwarp();
        }
        boff += __shfl_sync(0xffffffffu, incl, cnt - 1);
      }
    }
  } else if (warp >= kWarpLoad0 && warp < kWarpLoad0 + 4 * kLoadGroups) {
    // ------------------------------------------------------------ loaders: X gathers, record
    // expansion (A tile) and metadata
    const int group = (warp - kWarpLoad0) >> 2;  // owns the stages s with s % kLoadGroups == group
    const int quarter = warp & 3;                               // TMEM lane quarter of this warp
    const int t = threadIdx.x - (kWarpLoad0 + 4 * group) * 32;  // 0..127 within the group
    const int r = quarter * 32 + lane;                          // A row (= TMEM lane) this thread expands
    constexpr int kRowPieces = BN / 8;  // 16-byte pieces per gathered row
    constexpr int kPer = kRowPieces / 4;  // pieces per thread (32 rows x kRowPieces / 128 threads)
    constexpr bool kFixedCol = kGroupThreads % kRowPieces == 0;
    constexpr int kRowsPerPass = kGroupThreads / kRowPieces;
    const int c16f = t % kRowPieces, kk0 = t / kRowPieces;
    const uint32_t dcol16 = (uint32_t)(c16f >> 3) * 4096u;
    const int32_t ldx32 = (int32_t)p.ldx;
    // metadata lane word of TMEM lane (quarter*32 + lane): rows r0 and r0 + 8 of the quarter
    const int mr0 = (lane & 7) + 16 * (lane >> 4), mk1 = (lane >> 3) & 1;
    const uint32_t arow = (uint32_t)((r & 7) * 16 + (r >> 3) * 256);
    // the group walks only its own chunks j = group (mod kLoadGroups) of the CTA's chunk
    // sequence; stage j % kStages and record descriptor j % kRecSlots (both multiples of
    // kLoadGroups, so they advance by kLoadGroups with a phase flip on wrap-around)
    // records: unit ordinal k comes from producer k % kProducers; a chunk's descriptor is its
    // index among that producer's chunks (mod kSlotsPP), its use parity the quotient's bit 0
    int64_t i = group, i0 = 0;  // next own chunk, first chunk of the current unit
    int s = group;
    uint32_t ph = 0;
    int64_t pc0 = 0, pc1 = 0, pc2 = 0;  // chunks of producer 0 / 1 / 2 before the current unit
    int pw = 0;                 // producer of the current unit
    int4 nxt = unit_entry(p, blockIdx.x);
    for (int64_t u = blockIdx.x; u < p.n_units; u += ustep, pw = (pw + 1 == kProducers) ? 0 : pw + 1) {
      const int4 cur = nxt;
      nxt = unit_entry(p, u + ustep);
      const int ft = unit_ft(p, u);
      // this thread's gather column piece (kFixedCol): source offset and byte count
      const int col0f = ft * BN + c16f * 8;
      const uint32_t colbytes = col0f >= p.F ? 0u : (p.F - col0f >= 8 ? 16u : (uint32_t)(p.F - col0f) * 2u);
      const uint16_t* xcol = p.X + (colbytes ? col0f : 0);
      const int64_t i_first = i0, i_end = i0 + cur.y;
      i0 = i_end;
      const int64_t lbase = (pw == 0 ? pc0 : pw == 1 ? pc1 : pc2) - i_first;  // producer-local index = lbase + i
      if (pw == 0) pc0 += cur.y; else if (pw == 1) pc1 += cur.y; else pc2 += cur.y;
      for (; i < i_end; i += kLoadGroups) {
        const int64_t li = lbase + i;
        const int rs = pw * kSlotsPP + (int)(li & (kSlotsPP - 1));
        const uint32_t rph = (uint32_t)(li >> kSlotsShift) & 1u;
        mbar_wait(bEmpty + 8 * s, ph ^ 1);       // the MMA has finished with stage s
        if (t == 0) NM_TRACE(7);
        if (!(NM_DBG(p) & 1024)) mbar_wait(bRecFull + 8 * rs, rph);  // the compressed record has landed
        if (t == 0) NM_TRACE(1);
        const uint32_t rec = sRec + pw * C::kRingStride + ((NM_DBG(p) & 1024) ? 0u : rec_off[rs]);
        // 8-row groups of consecutive X rows come in by TMA tile loads (one 8 x 64 box per
        // 64-column slab, written into the SW128 atom); the other rows by cp.async gathers
        const uint32_t cmask = (NM_DBG(p) & 32) ? 0u : lds8(rec + kRecContOff);
        if (t < 32 && cmask) {  // first warp of the group: one TMA tile load per lane
          constexpr int kSlabs = BN / 64;
          if (t == 0)
            asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(bFull + 8 * s),
                         "r"((uint32_t)(__popc(cmask) * kSlabs * 1024))
                         : "memory");
          __syncwarp();
          const int g8 = t / kSlabs, h = t % kSlabs;
          if (g8 < 4 && ((cmask >> g8) & 1u)) {
            const int32_t row0 = (int32_t)lds32(rec + 32 * g8);
            asm volatile(
                "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
                " [%0], [%1, {%2, %3}], [%4];" ::"r"(sB + s * C::kBBytes + h * 4096 + g8 * 1024),
                "l"(&tmX), "r"(ft * BN + 64 * h), "r"(row0), "r"(bFull + 8 * s)
                : "memory");
          }
        }
        // cp.async gathers: 16-byte pieces of the 32 rows x BN columns; piece P = q * 128 + t
        // is row P / kRowPieces, column piece P % kRowPieces, so a warp instruction covers
        // whole 128-byte lines of consecutive pieces of one or more rows
        if constexpr (kFixedCol) {
          // BN = 64 / 128 / 256: the thread's column piece is the same for every q, so the
          // source column, byte count and swizzle term are per-unit constants
          const uint32_t sbase = sB + s * C::kBBytes + dcol16;
          if (NM_DBG(p) & 128) {
            // profiling: no gathers
          } else if (colbytes == 16u) {  // unit-uniform: full pieces, a zero row is an ignore-src zero fill
#pragma unroll
            for (int q = 0; q < kPer; ++q) {
              const int kk = q * kRowsPerPass + kk0;
              if ((cmask >> (kk >> 3)) & 1u) continue;  // this row arrives by TMA
              const int32_t xr = (int32_t)lds32(rec + 4 * kk);
              cp_async16_ign(sbase + (kk >> 3) * 1024 + (kk & 7) * 128 + ((((uint32_t)c16f ^ (uint32_t)kk) & 7u) << 4),
                             xcol + (int64_t)max(xr, 0) * ldx32, xr < 0);
            }
          } else {  // the F tail
#pragma unroll
            for (int q = 0; q < kPer; ++q) {
              const int kk = q * kRowsPerPass + kk0;
              if ((cmask >> (kk >> 3)) & 1u) continue;
              const int32_t xr = (int32_t)lds32(rec + 4 * kk);
              cp_async16(sbase + (kk >> 3) * 1024 + (kk & 7) * 128 + ((((uint32_t)c16f ^ (uint32_t)kk) & 7u) << 4),
                         xcol + (int64_t)max(xr, 0) * ldx32, xr >= 0 ? colbytes : 0u);
            }
          }
        } else {
#pragma unroll
          for (int q = 0; q < kPer; ++q) {
            const int P = q * kGroupThreads + t;
            const int kk = P / kRowPieces, c16 = P % kRowPieces;
            if ((cmask >> (kk >> 3)) & 1u) continue;  // this row arrives by TMA
            const int32_t xr = (int32_t)lds32(rec + 4 * kk);
            const int col0 = ft * BN + c16 * 8;
            uint32_t bytes = 0;
            if (xr >= 0 && col0 < p.F) {
              const int rem = p.F - col0;
              bytes = rem >= 8 ? 16u : (uint32_t)(rem * 2);
            }
            const uint16_t* src = bytes ? p.X + (int64_t)xr * ldx32 + col0 : p.X;
            const uint32_t dst = sB + s * C::kBBytes + (kk >> 3) * 1024 + (kk & 7) * 128 + (c16 >> 3) * 4096 +
                                 ((((uint32_t)c16 & 7u) ^ ((uint32_t)kk & 7u)) << 4);
            cp_async16(dst, src, bytes);
          }
        }
        // the barrier tracks this thread's gathers asynchronously (arrival when they land)
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bFull + 8 * s) : "memory");
        if (t == 0) NM_TRACE(4);
        // expand row r of the record (its non-empty (row, group) value pairs and nibble word)
        // into the A tile and the stage's TMEM metadata column
        const uint32_t mask = (NM_DBG(p) & 64) ? 0u : lds8(rec + kRecMaskOff + r);
        const int ne = __popc(mask), nr = mask != 0u;
        // inclusive prefix sums over the quarter's 32 rows from ballots (no shuffle chain):
        // ne = sum of its bits 2^k, each bit's prefix is a popc of the ballot below this lane
        uint32_t le;
        asm("mov.u32 %0, %%lanemask_le;" : "=r"(le));
        const int ve = __popc(__ballot_sync(0xffffffffu, ne & 1) & le) +
                       2 * __popc(__ballot_sync(0xffffffffu, ne & 2) & le) +
                       4 * __popc(__ballot_sync(0xffffffffu, ne & 4) & le) +
                       8 * __popc(__ballot_sync(0xffffffffu, ne & 8) & le);
        const int vn = __popc(__ballot_sync(0xffffffffu, nr) & le);
        const int NE = (int)lds16(rec + kRecTotOff);
        int e = (int)lds16(rec + kRecQvOff + 2 * quarter) + ve - ne;
        const int wn = (int)lds16(rec + kRecQnOff + 2 * quarter) + vn - 1;
        // entry of (r, g) = e + #set bits of mask below g: independent loads, no serial chain
        uint32_t v[kChunkMB];
        const uint32_t vbase = rec + kRecHdrBytes + 4 * e;
#pragma unroll
        for (int g = 0; g < kChunkMB; ++g) {
          v[g] = 0u;
          if (mask & (1u << g)) v[g] = lds32(vbase + 4 * __popc(mask & ((1u << g) - 1u)));
        }
        const uint32_t W = nr ? lds32(rec + kRecHdrBytes + 4 * (NE + wn)) : kMetaNone;
        __syncwarp();  // every read of the record by this warp is done
        if (lane == 0) mbar_arrive(bRecEmpty + 8 * rs);
        if (t == 0) NM_TRACE(5);
        // metadata word of this thread's TMEM lane: asynchronous store, waited for below
        const uint32_t Wa = __shfl_sync(0xffffffffu, W, mr0), Wb = __shfl_sync(0xffffffffu, W, mr0 + 8);
        const uint32_t word = ((Wa >> (16 * mk1)) & 0xFFFFu) | (((Wb >> (16 * mk1)) & 0xFFFFu) << 16);
        const uint32_t taddr = tbase + ((uint32_t)(quarter * 32) << 16) + C::kMeta0 + s;
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(word) : "memory");
        const uint32_t at = sA + s * C::kABytes + arow;
        sts128(at, v[0], v[1], v[2], v[3]);          // physical k 0..7
        sts128(at + 128, v[4], v[5], v[6], v[7]);    // physical k 8..15 (LBO = 128)
        if (t == 0) NM_TRACE(6);
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncwarp();  // the warp's A-tile rows and metadata lanes are written
        if (lane == 0) mbar_arrive(bFull + 8 * s);
        if (t == 0) NM_TRACE(2);
        s += kLoadGroups;
        if (s >= C::kStages) { s -= C::kStages; ph ^= 1; }
      }
    }
  } else if (warp == kWarpMma) {
    // ------------------------------------------------------------ MMA issuer
    // The loop is warp-uniform (all lanes wait and advance the stage state, so descriptors
    // and TMEM addresses stay in uniform registers) and one elected lane issues the MMA and
    // its commit: the per-chunk issue path is ~20 instructions (a single divergent lane
    // needed ~56 with register moves into the uniform datapath -- the kernel's skeleton was
    // bound by it).  The cp.async gathers are published through
    // cp.async.mbarrier.arrive on full_b.
    int64_t i = 0;  // chunk counter (trace only)
    int s = 0;
    uint32_t ph = 0;
    int acc = 0;
    uint32_t aphase = 0;
    const uint64_t adesc0 = sdesc(sA, 128, 256, 0);
    const uint64_t bdesc0 = sdesc(sB, 4096, 1024, 2);
    uint64_t ad = adesc0, bd = bdesc0;          // descriptors of stage s
    uint32_t mcol = C::kMeta0;                  // metadata column of stage s
    int4 nxt = unit_entry(p, blockIdx.x);
    for (int64_t u = blockIdx.x; u < p.n_units; u += ustep) {
      const int4 cur = nxt;
      nxt = unit_entry(p, u + ustep);
      const int nch = cur.y;
      mbar_wait(bTempty + 8 * acc, aphase ^ 1);
      NM_TRACE_U(1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t dcol = tbase + acc * BN;
      for (int c = 0; c < nch; ++c, ++i) {
        mbar_wait(bFull + 8 * s, ph);
        NM_TRACE(3);
        // the A tile (st.shared) and the gathers (cp.async) were written through the generic
        // proxy: make them visible to the tensor core's async-proxy operand reads (without
        // this fence stale stage contents were observed on B200 -- test_parity_fullsize.py)
        if (!(NM_DBG(p) & 16)) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        // metadata column: even column address + sparse_id2 selects the odd one
        asm volatile(
            "{\n\t.reg .pred e, q;\n\t"
            "elect.sync _|e, 0xffffffff;\n\t"
            "setp.ne.b32 q, %5, 0;\n\t"
            "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%6];\n\t}" ::"r"(dcol),
            "l"(ad), "l"(bd), "r"(tbase + (mcol & ~1u)), "r"(p.idesc | (mcol & 1u)), "r"(c), "r"(bEmpty + 8 * s)
            : "memory");
        if (++s == C::kStages) {
          s = 0;
          ph ^= 1;
          ad = adesc0;
          bd = bdesc0;
          mcol = C::kMeta0;
        } else {
          ad += (uint64_t)(C::kABytes >> 4);
          bd += (uint64_t)(C::kBBytes >> 4);
          ++mcol;
        }
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
  } else {
    // ------------------------------------------------------------ epilogue
    // tcgen05.ld 16x256b: thread t holds rows (t/4) and (t/4 + 8) of a 16-lane block, columns
    // 2*(t%4) + {0,1} of every 8-column repetition -> 8-byte stores, four threads complete a
    // 32-byte sector of a Y row.  kEpiWarps = 8: two warps per TMEM lane quarter, one 16-lane
    // block each; kEpiWarps = 4: one warp per quarter does both blocks.
    constexpr int kBlocks = 8 / kEpiWarps;               // 16-lane blocks per warp
    const int quarter = warp & 3;                        // TMEM lane quarter this warp may access
    const int blk0 = ((warp - kWarpEpi0) >> 2) * kBlocks;
    const int cpair = 2 * (lane & 3);
    int acc = 0;
    uint32_t aphase = 0;
    const bool vec_ok = ((p.ldy & 1) == 0) && ((((uintptr_t)p.Y) & 7) == 0);
    auto out_row = [&](int4 e, int r) -> int64_t {
      const int64_t g = (int64_t)e.x * kPanelRows + r;
      return g < p.rows ? (p.row_map ? (int64_t)__ldg(p.row_map + g) : g) : -1;
    };
    auto row_of = [&](int b, int hi) { return quarter * 32 + (blk0 + b) * 16 + (lane >> 2) + 8 * hi; };
    int4 nxt = unit_entry(p, blockIdx.x);
    int64_t nrow[kBlocks][2];  // output rows of the next unit (prefetched one unit ahead)
#pragma unroll
    for (int b = 0; b < kBlocks; ++b)
#pragma unroll
      for (int h = 0; h < 2; ++h) nrow[b][h] = blockIdx.x < p.n_units ? out_row(nxt, row_of(b, h)) : -1;
    for (int64_t u = blockIdx.x; u < p.n_units; u += ustep) {
      const int4 cur = nxt;
      int64_t orow[kBlocks][2];
#pragma unroll
      for (int b = 0; b < kBlocks; ++b)
#pragma unroll
        for (int h = 0; h < 2; ++h) orow[b][h] = nrow[b][h];
      nxt = unit_entry(p, u + ustep);
      if (u + ustep < p.n_units) {
#pragma unroll
        for (int b = 0; b < kBlocks; ++b)
#pragma unroll
          for (int h = 0; h < 2; ++h) nrow[b][h] = out_row(nxt, row_of(b, h));
      }
      const int ft = unit_ft(p, u);
      const bool has = cur.y > 0;
      const bool full_tile = vec_ok && ft * BN + BN <= p.F;
      mbar_wait_sleep(bTfull + 8 * acc, aphase);
      NM_TRACE_U(2);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
      for (int b = 0; b < kBlocks; ++b) {
        const int64_t olo = orow[b][0], ohi = orow[b][1];
        const uint32_t lane0 = (uint32_t)(quarter * 32 + (blk0 + b) * 16);
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
          if (NM_DBG(p) & 2) continue;
          if (full_tile) {  // unit-uniform fast path: every column in range, 8-byte stores
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
      NM_TRACE_U(3);
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
  prm.unit_info = P->unit_info;
  prm.rec_len16 = P->rec_len16;
  prm.row_map = P->row_map;
  prm.X = (const uint16_t*)PX;
  prm.ldx = ldx;
  prm.Y = Yp;
  prm.ldy = ldy;
  prm.F = F;
  prm.rows = P->row_end - P->row_begin;
  prm.n_ftiles = (F + BN - 1) / BN;
  prm.n_units = P->n_panels * prm.n_ftiles;
  if (prm.n_units + 4 * (int64_t)sms >= ((int64_t)1 << 31))
    return fail(NM_ERR_UNSUPPORTED, "nm_spmm: too many work units for one launch (row-shard the matrix)");
  prm.idesc = make_idesc(P->dtype, BN);
  prm.debug = 0;
  prm.trace = nullptr;
  const char* tr = nullptr;
#ifdef NM_SPMM_DEBUG_BUILD
  const char* dbg = getenv("NM_SPMM_DEBUG");
  prm.debug = dbg ? atoi(dbg) : 0;
#endif
#ifdef NM_SPMM_TRACE_BUILD
  tr = getenv("NM_SPMM_TRACE");
#endif
  if (tr) {
    NM_CUDA(cudaMalloc(&prm.trace, 16384 * 8));
    NM_CUDA(cudaMemset(prm.trace, 0, 16384 * 8));
  }
  int64_t grid = prm.n_units < sms ? prm.n_units : sms;
  if (grid < 1) return NM_OK;
  // X as a 2-D tensor (F columns x n rows, ldx pitch) for the TMA tile loads of consecutive
  // gather rows: 64 x 8 boxes, SWIZZLE_128B (the B tile's atom), out-of-range columns zero
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  if (!encode) {
    cudaDriverEntryPointQueryResult q;
    NM_CUDA(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&encode, cudaEnableDefault, &q));
    if (!encode || q != cudaDriverEntryPointSuccess) return fail(NM_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  }
  CUtensorMap tm;
  const cuuint64_t dims[2] = {(cuuint64_t)F, (cuuint64_t)P->n};
  const cuuint64_t strides[1] = {(cuuint64_t)ldx * 2};
  const cuuint32_t box[2] = {64, 8};
  const cuuint32_t es[2] = {1, 1};
  const CUresult er = encode(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, const_cast<void*>(PX), dims, strides, box, es,
                             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                             CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (er != CUDA_SUCCESS) return fail(NM_ERR_CUDA, "cuTensorMapEncodeTiled failed for X");
  k_spmm_sptc<BN><<<(unsigned)grid, kThreads, C::kSmem, s>>>(prm, tm);
  NM_CUDA(cudaGetLastError());
  if (prm.trace) {  // profiling aid only: synchronous dump of CTA 0's timeline
    NM_CUDA(cudaStreamSynchronize(s));
    static unsigned long long h[16384];
    NM_CUDA(cudaMemcpy(h, prm.trace, sizeof(h), cudaMemcpyDeviceToHost));
    FILE* f = fopen(tr, "wb");
    if (f) {
      fwrite(h, sizeof(h), 1, f);
      fclose(f);
    }
    cudaFree(prm.trace);
  }
  return NM_OK;
}

}  // namespace

nm_status launch_spmm_sptc_compressed(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy,
                                      int F, cudaStream_t s) {
  if (F <= 64) return launch_bn<64>(P, PX, ldx, Yp, ldy, F, s);
  if (F <= 128) return launch_bn<128>(P, PX, ldx, Yp, ldy, F, s);
  if (F <= 192) return launch_bn<192>(P, PX, ldx, Yp, ldy, F, s);
  return launch_bn<256>(P, PX, ldx, Yp, ldy, F, s);
}

}  // namespace nm
