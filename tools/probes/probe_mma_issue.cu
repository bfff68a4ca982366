// Hardware probe (not product code): what sets the ~220-242 cycles per tcgen05.mma that
// probe_sparse_peak.cu measured independent of N?  The B300 notes give a tensor-pipe floor of
// max(M,128)*N/256 cycles per dispatch (64 at M = 128, N = 128), so the probe's figure is an
// issue-side cost.  Variants, each 148 CTAs x one issuing warp, dense kind::f16 K = 16 and
// sparse K = 32, M = 128:
//   unroll u   : u MMAs per elect.sync block (descriptors advanced with immediate adds)
//   a_layout   : A descriptor layout 0 = no swizzle (the product's), 2 = SW128 K-major
//   b_major    : B MN-major SW128 (the product's) or K-major SW128
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_mma_issue probe_mma_issue.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)layout << 61;
  return d;
}

__device__ __forceinline__ uint64_t gtime() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

template <int SPARSE, int U>
__device__ __forceinline__ void issue(uint32_t dcol, uint64_t ad, uint64_t bd, uint32_t mcol, uint32_t idesc,
                                      uint32_t en) {
  if (SPARSE) {
    if (U == 1)
      asm volatile(
          "{\n\t.reg .pred e, q;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 q, %5, 0;\n\t"
          "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t}" ::"r"(dcol),
          "l"(ad), "l"(bd), "r"(mcol), "r"(idesc), "r"(en)
          : "memory");
    else
      asm volatile(
          "{\n\t.reg .pred e, q;\n\t.reg .b64 a1, a2, a3;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 q, %5, 0;\n\t"
          "add.s64 a1, %1, 2;\n\tadd.s64 a2, %1, 4;\n\tadd.s64 a3, %1, 6;\n\t"
          "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t"
          "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a1, %2, [%3], %4, 1;\n\t"
          "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a2, %2, [%3], %4, 1;\n\t"
          "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a3, %2, [%3], %4, 1;\n\t}" ::"r"(dcol),
          "l"(ad), "l"(bd), "r"(mcol), "r"(idesc), "r"(en)
          : "memory");
  } else {
    if (U == 1)
      asm volatile(
          "{\n\t.reg .pred e, q;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 q, %4, 0;\n\t"
          "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, q;\n\t}" ::"r"(dcol),
          "l"(ad), "l"(bd), "r"(idesc), "r"(en)
          : "memory");
    else
      asm volatile(
          "{\n\t.reg .pred e, q;\n\t.reg .b64 a1, a2, a3;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 q, %4, 0;\n\t"
          "add.s64 a1, %1, 2;\n\tadd.s64 a2, %1, 4;\n\tadd.s64 a3, %1, 6;\n\t"
          "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, q;\n\t"
          "@e tcgen05.mma.cta_group::1.kind::f16 [%0], a1, %2, %3, 1;\n\t"
          "@e tcgen05.mma.cta_group::1.kind::f16 [%0], a2, %2, %3, 1;\n\t"
          "@e tcgen05.mma.cta_group::1.kind::f16 [%0], a3, %2, %3, 1;\n\t}" ::"r"(dcol),
          "l"(ad), "l"(bd), "r"(idesc), "r"(en)
          : "memory");
  }
}

template <int SPARSE, int U>
__global__ void __launch_bounds__(128, 1) issue_kernel(int N, int a_layout, int b_kmajor, int iters,
                                                       unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* s = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bar_end;
  const int warp = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 96 * 1024 / 4; i += 128) ((uint32_t*)s)[i] = 0x3c003c00u;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar_end)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tslot;
  const uint32_t mcol = 510;
  {
    const uint32_t taddr = tb + ((uint32_t)(warp * 32) << 16) + mcol;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(0x44444444u));
    asm volatile("tcgen05.wait::st.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  if (warp == 1) {
    const uint32_t A = su32(s), B = su32(s + 32768);
    const uint64_t ad = a_layout == 0 ? sdesc(A, 128, 256, 0) : sdesc(A, 16, 1024, 2);
    const uint64_t bd = b_kmajor ? sdesc(B, 16, 1024, 2) : sdesc(B, 4096, 1024, 2);
    uint32_t idesc = (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    if (!b_kmajor) idesc |= 1u << 16;
    if (SPARSE) idesc |= 1u << 2;
    __syncwarp();
    const uint64_t t0 = gtime();
    const long long c0 = clock64();
    for (int i = 0; i < iters; i += U) issue<SPARSE, U>(tb, ad, bd, tb + mcol, idesc, i > 0);
    asm volatile(
        "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar_end))
        : "memory");
    uint32_t done = 0;
    const uint64_t deadline = gtime() + 2000000000ull;
    while (!done && gtime() < deadline)
      asm volatile(
          "{\n\t.reg .pred q;\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0;\n\tselp.b32 %0, 1, 0, q;\n\t}"
          : "=r"(done)
          : "r"(su32(&bar_end)));
    if (!done && threadIdx.x == 32) printf("CTA %d: watchdog expired\n", blockIdx.x);
    const long long c1 = clock64();
    const uint64_t t1 = gtime();
    if (threadIdx.x == 32) {
      out[4 * blockIdx.x] = t0;
      out[4 * blockIdx.x + 1] = t1;
      out[4 * blockIdx.x + 2] = (unsigned long long)(c1 - c0);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tb));
}

template <int SPARSE, int U>
static void run(int N, int al, int bk, unsigned long long* d, int sms) {
  const int iters = 1 << 16;
  auto k = issue_kernel<SPARSE, U>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  for (int rep = 0; rep < 2; ++rep) {
    k<<<sms, 128, 100 * 1024>>>(N, al, bk, iters, d);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
      printf("error %s\n", cudaGetErrorString(e));
      exit(1);
    }
  }
  unsigned long long h[148 * 4];
  cudaMemcpy(h, d, sms * 4 * 8, cudaMemcpyDeviceToHost);
  unsigned long long tmin = ~0ull, tmax = 0, cmax = 0;
  for (int i = 0; i < sms; ++i) {
    tmin = h[4 * i] < tmin ? h[4 * i] : tmin;
    tmax = h[4 * i + 1] > tmax ? h[4 * i + 1] : tmax;
    cmax = h[4 * i + 2] > cmax ? h[4 * i + 2] : cmax;
  }
  const double ns = (double)(tmax - tmin);
  const double flop = 2.0 * 128 * N * (SPARSE ? 32 : 16) * (double)iters * sms;
  printf("%s N=%3d unroll=%d A=%s B=%s: %7.1f cycles/MMA %7.1f TFLOP/s (logical) SM ~%.0f MHz\n",
         SPARSE ? "sparse" : "dense ", N, U, al ? "sw128K" : "noswzK", bk ? "sw128K " : "sw128MN",
         (double)cmax / iters, flop / ns / 1e3, (double)cmax / ns * 1e3);
}


// what the product kernel adds to the issue loop, one feature at a time (sparse, M = 128, N = 128):
//   bit 0: tcgen05.commit to an mbarrier every 2 MMAs (nobody waits on it)
//   bit 1: metadata TMEM column rotating over 32 columns
//   bit 2: A / B shared-memory descriptors rotating over 8 stages
//   bit 3: fence.proxy.async.shared::cta + tcgen05.fence::after_thread_sync every 2 MMAs
//   bit 4: accumulator rotating over 3 TMEM column ranges every 64 MMAs
__global__ void __launch_bounds__(128, 1) feat_kernel(int feat, int iters, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* s = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bar_end;
  __shared__ __align__(8) uint64_t bar_c;
  const int warp = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 96 * 1024 / 4; i += 128) ((uint32_t*)s)[i] = 0x3c003c00u;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar_end)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar_c)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tslot;
  for (int c = 0; c < 32; ++c) {
    const uint32_t taddr = tb + ((uint32_t)(warp * 32) << 16) + 400 + c;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(0x44444444u));
  }
  asm volatile("tcgen05.wait::st.sync.aligned;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  if (warp == 1) {
    const uint32_t A = su32(s), B = su32(s + 40960);
    const uint64_t ad0 = sdesc(A, 128, 256, 0);
    const uint64_t bd0 = sdesc(B, 4096, 1024, 2);
    const uint32_t idesc = (1u << 2) | (1u << 4) | (1u << 16) | ((uint32_t)(128 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    __syncwarp();
    const uint64_t t0 = gtime();
    const long long c0 = clock64();
    int acc = 0;
    for (int i = 0; i < iters; ++i) {
      const int st = (feat & 4) ? (i & 7) : 0;
      const uint64_t ad = ad0 + (uint64_t)((st * 4736) >> 4);
      const uint64_t bd = bd0 + (uint64_t)((st * 4096) >> 4);
      const uint32_t mc = (feat & 2) ? (uint32_t)(i & 31) : 0u;
      const uint32_t dcol = tb + (uint32_t)(acc * 128);
      if ((feat & 8) && (i & 1) == 0) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      }
      asm volatile(
          "{\n\t.reg .pred e, q;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 q, %5, 0;\n\t"
          "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t}" ::"r"(dcol),
          "l"(ad), "l"(bd), "r"(tb + 400 + (mc & ~1u)), "r"(idesc | (mc & 1u)), "r"(i & 63)
          : "memory");
      if ((feat & 1) && (i & 1))
        asm volatile(
            "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar_c))
            : "memory");
      if ((feat & 16) && (i & 63) == 63) acc = acc == 2 ? 0 : acc + 1;
    }
    asm volatile(
        "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar_end))
        : "memory");
    uint32_t done = 0;
    const uint64_t deadline = gtime() + 2000000000ull;
    while (!done && gtime() < deadline)
      asm volatile(
          "{\n\t.reg .pred q;\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0;\n\tselp.b32 %0, 1, 0, q;\n\t}"
          : "=r"(done)
          : "r"(su32(&bar_end)));
    const long long c1 = clock64();
    const uint64_t t1 = gtime();
    if (threadIdx.x == 32) {
      out[4 * blockIdx.x] = t0;
      out[4 * blockIdx.x + 1] = t1;
      out[4 * blockIdx.x + 2] = (unsigned long long)(c1 - c0);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tb));
}

static void run_feat(int feat, unsigned long long* d, int sms) {
  const int iters = 1 << 16;
  cudaFuncSetAttribute(feat_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  for (int rep = 0; rep < 2; ++rep) {
    feat_kernel<<<sms, 128, 100 * 1024>>>(feat, iters, d);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
      printf("error %s\n", cudaGetErrorString(e));
      exit(1);
    }
  }
  unsigned long long h[148 * 4];
  cudaMemcpy(h, d, sms * 4 * 8, cudaMemcpyDeviceToHost);
  unsigned long long cmax = 0;
  for (int i = 0; i < sms; ++i) cmax = h[4 * i + 2] > cmax ? h[4 * i + 2] : cmax;
  printf("sparse N=128 features %2d [%s%s%s%s%s]: %7.1f cycles/MMA\n", feat, feat & 1 ? " commit/2" : "",
         feat & 2 ? " meta-rot" : "", feat & 4 ? " stage-rot" : "", feat & 8 ? " fences/2" : "",
         feat & 16 ? " acc-rot" : "", (double)cmax / iters);
}

int main() {
  setvbuf(stdout, nullptr, _IONBF, 0);
  unsigned long long* d;
  cudaMalloc(&d, 148 * 4 * 8);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int N : {128})
    for (int al : {0})
      for (int bk : {0}) {
        run<0, 1>(N, al, bk, d, sms);
        run<0, 4>(N, al, bk, d, sms);
        run<1, 1>(N, al, bk, d, sms);
        run<1, 4>(N, al, bk, d, sms);
      }
  for (int f : {0, 1, 2, 4, 8, 16, 3, 5, 9, 31}) run_feat(f, d, sms);
  printf("PROBE DONE\n");
  return 0;
}
