// Hardware probe (not product code): (1) TMA tile::gather4 of four 64-element fp16 rows into
// a SWIZZLE_128B shared-memory atom, including an out-of-bounds row (must zero-fill and still
// complete the mbarrier transaction count); (2) tcgen05.mma.sp metadata addressing with the
// sparse_id2 selector (even column address + id2 = 1 reads the odd column).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_gather4 probe_gather4.cu
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void g4_kernel(const __grid_constant__ CUtensorMap tm, int r0, int r1, int r2, int r3, int col0,
                          uint8_t* out, uint32_t tx) {
  __shared__ __align__(1024) uint8_t buf[2048];
  __shared__ __align__(8) uint64_t bar;
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) buf[i] = 0xAB;
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar)), "r"(tx));
    // rows 0-3 of the atom at +0, rows 4-7 at +512 (second gather4, same rows shifted)
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(su32(buf)), "l"(&tm), "r"(col0), "r"(r0), "r"(r1),
        "r"(r2), "r"(r3), "r"(su32(&bar))
        : "memory");
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(su32(buf + 512)), "l"(&tm), "r"(col0), "r"(r3),
        "r"(r2), "r"(r1), "r"(r0), "r"(su32(&bar))
        : "memory");
    uint32_t done = 0;
    long spins = 0;
    while (!done && spins < 20000000) {
      asm volatile("{\n\t.reg .pred q;\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0;\n\tselp.b32 %0, 1, 0, q;\n\t}"
                   : "=r"(done) : "r"(su32(&bar)));
      ++spins;
    }
    out[2048] = done ? 1 : 0;
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) out[i] = buf[i];
}

int main() {
  const int n = 100, F = 128, ld = 136;
  std::vector<__half> X((size_t)n * ld);
  for (int r = 0; r < n; ++r)
    for (int c = 0; c < ld; ++c) X[(size_t)r * ld + c] = __float2half((float)((r * 7 + c) % 1000));
  __half* dX;
  CK(cudaMalloc(&dX, X.size() * 2));
  CK(cudaMemcpy(dX, X.data(), X.size() * 2, cudaMemcpyHostToDevice));
  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q));
  CUtensorMap tm;
  cuuint64_t dims[2] = {(cuuint64_t)F, (cuuint64_t)n};
  cuuint64_t strides[1] = {(cuuint64_t)ld * 2};
  cuuint32_t box[2] = {64, 1};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, dX, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode rc=%d\n", (int)r);
  uint8_t* dout;
  CK(cudaMalloc(&dout, 4096));
  int rows[4] = {5, 7, n + 3 /* OOB */, 99};
  for (int col0 : {0, 64}) {
    CK(cudaMemset(dout, 0, 4096));
    g4_kernel<<<1, 128>>>(tm, rows[0], rows[1], rows[2], rows[3], col0, dout, 2 * 4 * 64 * 2);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    std::vector<uint8_t> h(4096);
    CK(cudaMemcpy(h.data(), dout, 4096, cudaMemcpyDeviceToHost));
    int bad = 0;
    int order[8] = {rows[0], rows[1], rows[2], rows[3], rows[3], rows[2], rows[1], rows[0]};
    for (int k = 0; k < 8; ++k) {
      for (int c = 0; c < 64; ++c) {
        int c16 = c / 8;
        size_t off = (size_t)k * 128 + ((c16 ^ k) * 16) + (c % 8) * 2;
        __half v;
        memcpy(&v, &h[off], 2);
        float exp = order[k] < n ? (float)((order[k] * 7 + col0 + c) % 1000) : 0.f;
        if (__half2float(v) != exp) ++bad;
      }
    }
    printf("GATHER4 col0=%d mbar_done=%d mismatches=%d/512 %s\n", col0, h[2048], bad, bad == 0 ? "MATCH" : "");
  }
  printf("PROBE DONE\n");
  return 0;
}
