// Hardware probe (not product code): THROUGHPUT of tcgen05.mma.sp.cta_group::1.kind::f16
// (M = 128, K = 32 logical) and of the dense kind::f16 (K = 16) for N in {64, 128, 256} --
// the sparse tensor-pipe peak the roofline needs.
// Unlike probe_mma_rate.cu (one divergent thread issuing a dependent chain: an issue/latency
// figure), the MMAs here are issued the way the product kernel issues them: a warp-uniform loop
// with one elect.sync lane, operands in uniform registers, rotating over `nacc` independent
// TMEM accumulators, a tcgen05.commit every `cgroup` MMAs.  148 CTAs (one per SM) run
// concurrently; time = %globaltimer across the whole grid (first start .. last end), so the
// TFLOP/s figure is at whatever clock the GPU ran (the SM clock is sampled beside it).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_sparse_peak probe_sparse_peak.cu
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

__global__ void __launch_bounds__(128, 1) peak_kernel(int sparse, int N, int nacc, int cgroup, int iters,
                                                      unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* s = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bar;
  __shared__ __align__(8) uint64_t bar_end;
  const int warp = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 48 * 1024 / 4; i += 128) ((uint32_t*)s)[i] = 0x3c003c00u;  // 1.0 halves
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar_end)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tslot;
  const uint32_t mcol = 510;  // metadata column: legal 0x4 nibbles (indices 0,1)
  {
    const uint32_t taddr = tb + ((uint32_t)(warp * 32) << 16) + mcol;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(0x44444444u));
    asm volatile("tcgen05.wait::st.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  if (warp == 1) {
    const uint32_t A = su32(s), B = su32(s + 16384);
    const uint64_t ad = sdesc(A, 128, 256, 0);
    const uint64_t bd = sdesc(B, 4096, 1024, 2);
    uint32_t idesc = (1u << 4) | (1u << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    if (sparse) idesc |= 1u << 2;
    __syncwarp();
    const uint64_t t0 = gtime();
    const long long c0 = clock64();
    int acc = 0;
    for (int i = 0; i < iters; ++i) {
      const uint32_t dcol = tb + (uint32_t)(acc * N);
      const uint32_t en = i >= nacc;
      if (sparse)
        asm volatile(
            "{\n\t.reg .pred e, q;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 q, %5, 0;\n\t"
            "@e tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t}" ::"r"(dcol),
            "l"(ad), "l"(bd), "r"(tb + mcol), "r"(idesc), "r"(en)
            : "memory");
      else
        asm volatile(
            "{\n\t.reg .pred e, q;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 q, %4, 0;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, q;\n\t}" ::"r"(dcol),
            "l"(ad), "l"(bd), "r"(idesc), "r"(en)
            : "memory");
      if ((i + 1) % cgroup == 0)
        asm volatile(
            "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(
                su32(&bar) + 0)
            : "memory");
      if (++acc == nacc) acc = 0;
    }
    // final commit on its own barrier (one phase): completes when every MMA issued by this
    // thread has completed.  (Waiting for the intermediate commits by phase parity can alias
    // phases and hang -- the first version of this probe did.)
    asm volatile(
        "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar_end))
        : "memory");
    uint32_t done = 0;
    const uint64_t deadline = gtime() + 2000000000ull;  // 2 s watchdog
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

int main() {
  setvbuf(stdout, nullptr, _IONBF, 0);
  unsigned long long* d;
  cudaMalloc(&d, 148 * 4 * 8);
  cudaFuncSetAttribute(peak_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int iters = 1 << 16;
  double best_sparse = 0, best_dense = 0;
  for (int sparse = 1; sparse >= 0; --sparse)
    for (int N : {64, 128, 256})
      for (int nacc : {1, 2})
        for (int cg : {1, 8}) {
          if (nacc * N > 500) continue;
          printf("launch sparse=%d N=%d acc=%d cg=%d\n", sparse, N, nacc, cg);
          for (int rep = 0; rep < 2; ++rep) {  // first launch warms clocks up
            peak_kernel<<<sms, 128, 64 * 1024>>>(sparse, N, nacc, cg, iters, d);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
            if (rep == 0) continue;
            unsigned long long h[148 * 4];
            cudaMemcpy(h, d, sms * 4 * 8, cudaMemcpyDeviceToHost);
            unsigned long long tmin = ~0ull, tmax = 0, cmax = 0;
            for (int i = 0; i < sms; ++i) {
              tmin = h[4 * i] < tmin ? h[4 * i] : tmin;
              tmax = h[4 * i + 1] > tmax ? h[4 * i + 1] : tmax;
              cmax = h[4 * i + 2] > cmax ? h[4 * i + 2] : cmax;
            }
            const double ns = (double)(tmax - tmin);
            const double flop = 2.0 * 128 * N * (sparse ? 32 : 16) * (double)iters * sms;  // logical
            const double tf = flop / ns / 1e3;
            const double mhz = (double)cmax / ns * 1e3;
            printf("%s N=%3d acc=%d commit/%d: %7.1f cycles/MMA  %7.1f TFLOP/s (logical)  SM clock ~%.0f MHz\n",
                   sparse ? "sparse K=32" : "dense  K=16", N, nacc, cg, (double)cmax / iters, tf, mhz);
            if (sparse && tf > best_sparse) best_sparse = tf;
            if (!sparse && tf > best_dense) best_dense = tf;
          }
        }
  printf("BEST sparse %.1f TFLOP/s (logical, 2:4), dense %.1f TFLOP/s, ratio %.3f\n", best_sparse, best_dense,
         best_sparse / best_dense);
  printf("PROBE DONE\n");
  return 0;
}
