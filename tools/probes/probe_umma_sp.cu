// Hardware probe (not product code): pins down, on a real B200, the operand layouts the
// sm_100a kernels rely on -- the UMMA shared-memory descriptor LBO/SBO meaning for the
// no-swizzle canonical layouts, and the tensor-memory layout of the 2:4 sparsity metadata
// of tcgen05.mma.sp.kind::f16 (M=128, K=32).  With B = I_32 the sparse MMA returns the
// decompressed logical A, so one run reveals exactly where every compressed value lands.
//
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_umma_sp probe_umma_sp.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <random>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ uint64_t make_sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;  // descriptor version 1 (sm_100)
  return d;                // base_offset 0, lbo_mode 0, layout SWIZZLE_NONE
}

struct Params {
  uint32_t a_lbo, a_sbo, b_lbo, b_sbo;
  uint32_t idesc;
  int sparse;
  uint32_t meta_col;
  uint32_t e_id2;
  int a_bytes, b_bytes;
  uint32_t b_layout;  // 0 = SWIZZLE_NONE, 2 = SWIZZLE_128B
};

template <int N>
__global__ void __launch_bounds__(128, 1)
probe_kernel(const uint8_t* __restrict__ a_img, const uint8_t* __restrict__ b_img,
             const uint32_t* __restrict__ meta, float* __restrict__ D, Params p) {
  __shared__ __align__(1024) uint8_t smA[8192];
  __shared__ __align__(1024) uint8_t smB[16384];
  // (N=128 K=32 16-bit B = 8 KB)
  __shared__ uint32_t tmem_base_sh;
  __shared__ __align__(8) uint64_t mbar;
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int i = tid; i < p.a_bytes / 4; i += 128) ((uint32_t*)smA)[i] = ((const uint32_t*)a_img)[i];
  for (int i = tid; i < p.b_bytes / 4; i += 128) ((uint32_t*)smB)[i] = ((const uint32_t*)b_img)[i];
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;"
                 :: "r"(smem_u32(&tmem_base_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&mbar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tbase = tmem_base_sh;
  if (p.sparse) {
    uint32_t w = meta[tid];
    uint32_t taddr = tbase + ((uint32_t)(32 * warp) << 16) + p.meta_col;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" :: "r"(taddr), "r"(w));
    asm volatile("tcgen05.wait::st.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  if (tid == 0) {
    uint64_t ad = make_sdesc(smem_u32(smA), p.a_lbo, p.a_sbo);
    uint64_t bd = make_sdesc(smem_u32(smB), p.b_lbo, p.b_sbo) | ((uint64_t)p.b_layout << 61);
    uint32_t acc = 0;
    if (p.sparse) {
      uint32_t e = tbase + (p.meta_col & ~1u);  // odd column: even address + sparse_id2 = 1
      uint32_t idesc = p.idesc | (p.e_id2 & 3u);
      asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %5, 0;\n\t"
                   "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t}"
                   :: "r"(tbase), "l"(ad), "l"(bd), "r"(e), "r"(idesc), "r"(acc));
    } else {
      asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %4, 0;\n\t"
                   "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, q;\n\t}"
                   :: "r"(tbase), "l"(ad), "l"(bd), "r"(p.idesc), "r"(acc));
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                 :: "r"(smem_u32(&mbar)));
  }
  {
    uint32_t done = 0;
    while (!done) {
      asm volatile("{\n\t.reg .pred q;\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0;\n\t"
                   "selp.b32 %0, 1, 0, q;\n\t}" : "=r"(done) : "r"(smem_u32(&mbar)));
    }
  }
  asm volatile("tcgen05.fence::after_thread_sync;");
#pragma unroll
  for (int c = 0; c < N; c += 8) {
    uint32_t r[8];
    uint32_t taddr = tbase + ((uint32_t)(32 * warp) << 16) + c;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]),
                   "=r"(r[6]), "=r"(r[7]) : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    for (int j = 0; j < 8; ++j) D[tid * N + c + j] = __uint_as_float(r[j]);
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" :: "r"(tbase));
  }
}

static uint32_t make_idesc(int sparse, int M, int N, int a_major, int b_major) {
  uint32_t d = 0;
  if (sparse) d |= 1u << 2;
  d |= 1u << 4;  // D = f32
  // a_format = b_format = 0 (f16)
  d |= (uint32_t)a_major << 15;
  d |= (uint32_t)b_major << 16;
  d |= (uint32_t)(N >> 3) << 17;
  d |= (uint32_t)(M >> 4) << 24;
  return d;
}

// K-major interleave image of an R x KE (elements) matrix: 8x(16B) core matrices,
// K-chunk stride `cs` bytes, 8-row-group stride `gs` bytes.
static void kmajor_image(std::vector<uint8_t>& img, const std::vector<__half>& m, int R, int KE,
                         int cs, int gs) {
  for (int r = 0; r < R; ++r)
    for (int k = 0; k < KE; ++k) {
      size_t off = (size_t)(r % 8) * 16 + (size_t)(r / 8) * gs + (size_t)(k / 8) * cs + (k % 8) * 2;
      memcpy(&img[off], &m[(size_t)r * KE + k], 2);
    }
}
// MN-major interleave image of a K x N matrix (N contiguous): core matrix 8 K-rows x 16B,
// K-group stride `ks`, N-group stride `ns`.
static void mnmajor_image(std::vector<uint8_t>& img, const std::vector<__half>& b, int K, int N,
                          int ks, int ns) {
  for (int k = 0; k < K; ++k)
    for (int n = 0; n < N; ++n) {
      size_t off = (size_t)(n % 8) * 2 + (size_t)(k % 8) * 16 + (size_t)(k / 8) * ks + (size_t)(n / 8) * ns;
      memcpy(&img[off], &b[(size_t)k * N + n], 2);
    }
}

template <int N>
static void run(const std::vector<uint8_t>& aimg, const std::vector<uint8_t>& bimg,
                const std::vector<uint32_t>& meta, std::vector<float>& out, Params p) {
  uint8_t *da, *db; uint32_t* dm; float* dd;
  CK(cudaMalloc(&da, 8192)); CK(cudaMalloc(&db, 16384)); CK(cudaMalloc(&dm, 512));
  CK(cudaMalloc(&dd, 128 * N * 4));
  CK(cudaMemset(da, 0, 8192)); CK(cudaMemset(db, 0, 16384)); CK(cudaMemset(dd, 0, 128 * N * 4));
  CK(cudaMemcpy(da, aimg.data(), aimg.size(), cudaMemcpyHostToDevice));
  CK(cudaMemcpy(db, bimg.data(), bimg.size(), cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dm, meta.data(), 512, cudaMemcpyHostToDevice));
  p.a_bytes = (int)aimg.size(); p.b_bytes = (int)bimg.size();
  probe_kernel<N><<<1, 128>>>(da, db, dm, dd, p);
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  out.resize(128 * N);
  CK(cudaMemcpy(out.data(), dd, 128 * N * 4, cudaMemcpyDeviceToHost));
  cudaFree(da); cudaFree(db); cudaFree(dm); cudaFree(dd);
}

int main() {
  std::mt19937 rng(7);
  const int M = 128;
  // ---------------- dense: descriptor LBO/SBO semantics ----------------
  {
    const int K = 16, N = 32;
    std::vector<__half> A(M * K), B(K * N);
    std::vector<double> ref(M * N, 0.0);
    for (auto& x : A) x = __float2half((float)((int)(rng() % 9) - 4));
    for (auto& x : B) x = __float2half((float)((int)(rng() % 9) - 4));
    for (int i = 0; i < M; ++i)
      for (int j = 0; j < N; ++j)
        for (int k = 0; k < K; ++k)
          ref[i * N + j] += (double)__half2float(A[i * K + k]) * __half2float(B[k * N + j]);
    // A image: chunk stride 128, group stride 256.  B image (MN-major): K-group stride 128,
    // N-group stride 256 (2 K-groups of 8 for K=16).
    std::vector<uint8_t> aimg(M * K * 2), bimg(K * N * 2);
    kmajor_image(aimg, A, M, K, 128, 256);
    mnmajor_image(bimg, B, K, N, 128, 256);
    std::vector<uint32_t> meta(128, 0);
    for (int va = 0; va < 2; ++va)
      for (int vb = 0; vb < 2; ++vb) {
        Params p{};
        p.a_lbo = va ? 256 : 128; p.a_sbo = va ? 128 : 256;
        p.b_lbo = vb ? 256 : 128; p.b_sbo = vb ? 128 : 256;
        p.idesc = make_idesc(0, M, N, 0, 1);
        p.sparse = 0;
        std::vector<float> out;
        run<32>(aimg, bimg, meta, out, p);
        double err = 0;
        for (int i = 0; i < M * N; ++i) err = fmax(err, fabs(out[i] - ref[i]));
        printf("DENSE a(lbo=%u,sbo=%u) b(lbo=%u,sbo=%u): max_err=%g %s\n", p.a_lbo, p.a_sbo,
               p.b_lbo, p.b_sbo, err, err == 0 ? "MATCH" : "");
      }
    // K-major B (B^T stored N x K, K contiguous): chunk stride 128, group stride 256
    {
      std::vector<__half> BT(N * K);
      for (int k = 0; k < K; ++k) for (int n = 0; n < N; ++n) BT[n * K + k] = B[k * N + n];
      std::vector<uint8_t> btimg(K * N * 2);
      kmajor_image(btimg, BT, N, K, 128, 256);
      for (int va = 0; va < 2; ++va) {
        Params p{};
        p.a_lbo = 128; p.a_sbo = 256;
        p.b_lbo = va ? 256 : 128; p.b_sbo = va ? 128 : 256;
        p.idesc = make_idesc(0, M, N, 0, 0);
        std::vector<float> out;
        run<32>(aimg, btimg, meta, out, p);
        double err = 0;
        for (int i = 0; i < M * N; ++i) err = fmax(err, fabs(out[i] - ref[i]));
        printf("DENSE Kmajor-B b(lbo=%u,sbo=%u): max_err=%g %s\n", p.b_lbo, p.b_sbo, err,
               err == 0 ? "MATCH" : "");
      }
    }
  }
  // ---------------- sparse 2:4, K=32 logical ----------------
  {
    const int K = 32, N = 32, KC = 16;
    static const int pairs[6][2] = {{0, 1}, {0, 2}, {0, 3}, {1, 2}, {1, 3}, {2, 3}};
    std::vector<__half> Ac(M * KC);
    std::vector<int> nib(M * 8);
    std::vector<float> Alog(M * K, 0.f);
    for (int r = 0; r < M; ++r)
      for (int g = 0; g < 8; ++g) {
        int pi = rng() % 6;
        int i0 = pairs[pi][0], i1 = pairs[pi][1];
        nib[r * 8 + g] = i0 | (i1 << 2);
        float v0 = (float)(r * 16 + 2 * g + 0 + 1), v1 = (float)(r * 16 + 2 * g + 1 + 1);
        Ac[r * KC + 2 * g] = __float2half(v0);
        Ac[r * KC + 2 * g + 1] = __float2half(v1);
        Alog[r * K + 4 * g + i0] = v0;
        Alog[r * K + 4 * g + i1] = v1;
      }
    std::vector<__half> B(K * N);
    for (int k = 0; k < K; ++k) for (int n = 0; n < N; ++n) B[k * N + n] = __float2half(k == n ? 1.f : 0.f);
    std::vector<uint8_t> aimg(M * KC * 2), bimg(K * N * 2);
    kmajor_image(aimg, Ac, M, KC, 128, 256);
    mnmajor_image(bimg, B, K, N, 128, 512);  // 4 K-groups at 128, N-groups at 512
    // Hypothesis H1 (from CUTLASS tmem_e_frg FP16 atom): lane L = m0 + 8*k1 + 16*m2 holds
    // rows r0 = m0+16*m2 (low 16 bits) and r0+8 (high 16 bits) for K-half k1.
    std::vector<uint32_t> h1(128, 0), h2(128, 0);
    for (int L = 0; L < 128; ++L) {
      int m0 = L % 8, k1 = (L / 8) % 2, m2 = L / 16;
      int r0 = m0 + 16 * m2, r1 = r0 + 8;
      uint32_t w = 0;
      for (int q = 0; q < 4; ++q) {
        w |= (uint32_t)nib[r0 * 8 + 4 * k1 + q] << (4 * q);
        w |= (uint32_t)nib[r1 * 8 + 4 * k1 + q] << (16 + 4 * q);
      }
      h1[L] = w;
      uint32_t w2 = 0;  // H2: lane = row, 8 nibbles in K order
      for (int g = 0; g < 8; ++g) w2 |= (uint32_t)nib[L * 8 + g] << (4 * g);
      h2[L] = w2;
    }
    const std::vector<uint32_t>* hyps[2] = {&h1, &h2};
    for (int h = 0; h < 2; ++h)
      for (int bv = 0; bv < 2; ++bv) {
        Params p{};
        p.a_lbo = 128; p.a_sbo = 256;
        p.b_lbo = bv ? 512 : 128; p.b_sbo = bv ? 128 : 512;
        p.idesc = make_idesc(1, M, N, 0, 1);
        p.sparse = 1; p.meta_col = 128; p.e_id2 = 0;
        std::vector<float> out;
        run<32>(aimg, bimg, *hyps[h], out, p);
        int bad = 0;
        for (int i = 0; i < M * K; ++i) bad += (out[i] != Alog[i]);
        printf("SPARSE H%d b(lbo=%u,sbo=%u): mismatches=%d/%d %s\n", h + 1, p.b_lbo, p.b_sbo, bad,
               M * K, bad == 0 ? "MATCH" : "");
        if (bad && h == 0 && bv == 0) {
          // decode the first rows to learn the mapping
          for (int r = 0; r < 20; ++r) {
            printf(" row %3d:", r);
            for (int k = 0; k < K; ++k) {
              float v = out[r * N + k];
              if (v != 0.f) {
                int id = (int)v - 1;
                printf(" k%d<-(r%d,s%d)", k, id / 16, id % 16);
              }
            }
            printf("\n  expect:");
            for (int k = 0; k < K; ++k) {
              float v = Alog[r * K + k];
              if (v != 0.f) { int id = (int)v - 1; printf(" k%d<-(r%d,s%d)", k, id / 16, id % 16); }
            }
            printf("\n");
          }
        }
      }
    // id2 / column-offset probe with H1 at meta column 129 (odd) and id2 0/1
    for (int id2 = 0; id2 < 1; ++id2) {
      for (int col = 129; col <= 135; ++col) {
        Params p{};
        p.a_lbo = 128; p.a_sbo = 256; p.b_lbo = 128; p.b_sbo = 512;
        p.idesc = make_idesc(1, M, N, 0, 1);
        p.sparse = 1; p.meta_col = col; p.e_id2 = col & 1;
        std::vector<float> out;
        run<32>(aimg, bimg, h1, out, p);
        int bad = 0;
        for (int i = 0; i < M * K; ++i) bad += (out[i] != Alog[i]);
        printf("SPARSE H1 meta_col=%d id2=%d: mismatches=%d %s\n", col, id2, bad, bad == 0 ? "MATCH" : "");
      }
    }
  }
  // ---------------- sparse, N=128, B MN-major SWIZZLE_128B, f16 and bf16 ----------------
  for (int bf = 0; bf < 2; ++bf) {
    const int K = 32, N = 128, KC = 16;
    static const int pairs[6][2] = {{0, 1}, {0, 2}, {0, 3}, {1, 2}, {1, 3}, {2, 3}};
    std::vector<__half> Ac(M * KC);      // raw 16-bit storage (bf16 bits reinterpret)
    std::vector<int> nib(M * 8);
    std::vector<double> Alog(M * K, 0.0), Bv(K * N);
    auto enc = [&](float v) { __half h; if (bf) { __nv_bfloat16 b = __float2bfloat16(v); memcpy(&h, &b, 2);} else h = __float2half(v); return h; };
    for (int r = 0; r < M; ++r)
      for (int g = 0; g < 8; ++g) {
        int pi = rng() % 6;
        int i0 = pairs[pi][0], i1 = pairs[pi][1];
        nib[r * 8 + g] = i0 | (i1 << 2);
        float v0 = (float)((int)(rng() % 17) - 8) * 0.25f, v1 = (float)((int)(rng() % 17) - 8) * 0.25f;
        Ac[r * KC + 2 * g] = enc(v0); Ac[r * KC + 2 * g + 1] = enc(v1);
        Alog[r * K + 4 * g + i0] = v0; Alog[r * K + 4 * g + i1] = v1;
      }
    std::vector<__half> B(K * N);
    for (int k = 0; k < K; ++k) for (int n = 0; n < N; ++n) { float v = (float)((int)(rng() % 9) - 4); B[k * N + n] = enc(v); Bv[k * N + n] = v; }
    std::vector<uint8_t> aimg(M * KC * 2), bimg(K * N * 2);
    kmajor_image(aimg, Ac, M, KC, 128, 256);
    // SW128 MN-major: atom = 8 K-rows x 128 B (64 elems), 16B chunk c of row r at (c ^ r%8);
    // K-groups at SBO = 1024, 64-element N-chunks at LBO = 4096.
    for (int k = 0; k < K; ++k)
      for (int n = 0; n < N; ++n) {
        int nc = n / 64, c16 = (n % 64) / 8, r = k % 8;
        size_t off = (size_t)nc * 4096 + (size_t)(k / 8) * 1024 + r * 128 + ((c16 ^ r) * 16) + (n % 8) * 2;
        memcpy(&bimg[off], &B[k * N + n], 2);
      }
    std::vector<double> ref(M * N, 0.0);
    for (int i = 0; i < M; ++i) for (int j = 0; j < N; ++j) for (int k = 0; k < K; ++k) ref[i * N + j] += Alog[i * K + k] * Bv[k * N + j];
    std::vector<uint32_t> meta(128);
    for (int L = 0; L < 128; ++L) {
      int m0 = L % 8, k1 = (L / 8) % 2, m2 = L / 16; int r0 = m0 + 16 * m2, r1 = r0 + 8; uint32_t w = 0;
      for (int q = 0; q < 4; ++q) { w |= (uint32_t)nib[r0 * 8 + 4 * k1 + q] << (4 * q); w |= (uint32_t)nib[r1 * 8 + 4 * k1 + q] << (16 + 4 * q); }
      meta[L] = w;
    }
    for (int v = 0; v < 2; ++v) {
      Params p{};
      p.a_lbo = 128; p.a_sbo = 256;
      p.b_lbo = v ? 1024 : 4096; p.b_sbo = v ? 4096 : 1024; p.b_layout = 2;
      p.idesc = make_idesc(1, M, N, 0, 1) | (bf ? ((1u << 7) | (1u << 10)) : 0u);
      p.sparse = 1; p.meta_col = 128;
      std::vector<float> out;
      run<128>(aimg, bimg, meta, out, p);
      double err = 0; for (int i = 0; i < M * N; ++i) err = fmax(err, fabs(out[i] - ref[i]));
      printf("SPARSE N=128 SW128-B %s b(lbo=%u,sbo=%u): max_err=%g %s\n", bf ? "bf16" : "f16", p.b_lbo, p.b_sbo, err, err == 0 ? "MATCH" : "");
    }
  }
  printf("PROBE DONE\n");
  return 0;
}
