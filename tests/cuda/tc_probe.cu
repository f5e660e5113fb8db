// Standalone tcgen05 probe (diagnostic, not part of the product): checks the
// TMEM round trip and single tf32 UMMA instructions with hand-written smem
// descriptors, to validate the encodings dense_tc.cu relies on.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tc_probe tc_probe.cu && ./tc_probe
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstring>

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ uint64_t make_sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout) {
  uint64_t d = 0;
  d |= uint64_t((saddr >> 4) & 0x3FFFu);
  d |= uint64_t((lbo >> 4) & 0x3FFFu) << 16;
  d |= uint64_t((sbo >> 4) & 0x3FFFu) << 32;
  d |= uint64_t(1) << 46;
  d |= uint64_t(layout & 7u) << 61;
  return d;
}
__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N, int bmajor) {
  return (1u << 4) | (2u << 7) | (2u << 10) | (0u << 15) | (uint32_t(bmajor) << 16) | (uint32_t(N >> 3) << 17) |
         (uint32_t(M >> 4) << 24);
}

// mode 0: tmem st/ld roundtrip; 1: A ones, B ones (K-major); 2: A K-major pattern, B MN-major pattern
// out: [128][16]
__global__ void probe(int mode, float* out, uint32_t* info) {
  __shared__ __align__(1024) float sA[128 * 32];
  __shared__ __align__(1024) float sB[32 * 32];
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5, t = threadIdx.x;
  // fill A (128 x 32 tf32, K-major SW128): element (m,k)
  for (int e = t; e < 128 * 32; e += blockDim.x) {
    int m = e / 32, k = e % 32;
    float v = (mode == 2) ? ((k == (m % 8)) ? 1.f : 0.f) : (mode == 5 ? 1.000732421875f : 1.f);
    int chunk = k / 4, w = k % 4;
    sA[(m * 128 + ((chunk ^ (m & 7)) << 4)) / 4 + w] = v;
  }
  // B: 32 (K) x 16 (N)
  for (int e = t; e < 32 * 32; e += blockDim.x) sB[e] = 0.f;
  __syncthreads();
  for (int e = t; e < 32 * 32; e += blockDim.x) {
    int k = e / 32, n = e % 32;
    float v = (mode == 1 || mode == 5) ? 1.f : (mode == 3 ? float(k * 32 + n) : float(k * 16 + n));
    if (mode != 3 && n >= 16) continue;
    if (mode == 5) { int chunk = k / 4, w = k % 4; sB[(n * 128 + ((chunk ^ (n & 7)) << 4)) / 4 + w] = v; } else if (mode == 3) {
      sB[(k * 128 + (((n / 4) ^ (k & 7)) << 4)) / 4 + (n % 4)] = v;
    } else if (mode <= 2) {
      // K-major SW128: row n (128 B = 32 k), chunk swizzle by n%8
      int chunk = k / 4, w = k % 4;
      sB[(n * 128 + ((chunk ^ (n & 7)) << 4)) / 4 + w] = v;
    } else {
      // MN-major SW64 (atom = 16 n-values = 64 B rows, 8 k-rows per 512 B group):
      // row k at k*64 B; 16 B chunk c = n/4 swizzled with bits 7-8 of the address
      uint32_t addr = k * 64 + (n / 4) * 16 + (n % 4) * 4;
      uint32_t sw = addr ^ (((addr >> 7) & 3u) << 4);
      sB[sw / 4] = v;
    }
  }
  if (t == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(smem_u32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tbase = tslot;
  if (t == 0) info[0] = tbase;
  const uint32_t laddr = tbase + (uint32_t(warp * 32) << 16);
  if (mode == 0) {
    uint32_t v[4] = {uint32_t(t), uint32_t(t + 1000), uint32_t(t + 2000), uint32_t(t + 3000)};
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1,%2,%3,%4};" ::"r"(laddr), "r"(v[0]), "r"(v[1]),
                 "r"(v[2]), "r"(v[3]));
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
  } else if (t == 0) {
    uint64_t ad = make_sdesc(smem_u32(sA), 16, 1024, 2);
    uint64_t bd = (mode <= 2 || mode == 5) ? make_sdesc(smem_u32(sB), 16, 1024, 2)
                : (mode == 3 ? make_sdesc(smem_u32(sB), 4096, 1024, 2) : make_sdesc(smem_u32(sB), 2048, 512, 4));
    uint32_t id = idesc_tf32(128, mode == 3 ? 32 : 16, (mode <= 2 || mode == 5) ? 0 : 1);
    asm volatile(
        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(tbase),
        "l"(ad), "l"(bd), "r"(id), "r"(0u));
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar))
                 : "memory");
  }
  if (mode != 0) {
    uint32_t a = smem_u32(&bar);
    asm volatile(
        "{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(a)
        : "memory");
  }
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(laddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
  for (int c = 0; c < 16; ++c) out[t * 16 + c] = mode == 0 ? float(r[c]) : __uint_as_float(r[c]);
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tbase));
}

int main() {
  float* d;
  uint32_t* info;
  cudaMalloc(&d, 128 * 16 * 4);
  cudaMalloc(&info, 16);
  float h[128 * 16];
  for (int mode = 0; mode < 6; ++mode) {
    cudaMemset(d, 0xff, 128 * 16 * 4);
    probe<<<1, 128>>>(mode, d, info);
    cudaError_t e = cudaDeviceSynchronize();
    uint32_t ti = 0;
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    cudaMemcpy(&ti, info, 4, cudaMemcpyDeviceToHost);
    printf("mode %d: err=%s tmem_base=%u\n", mode, cudaGetErrorString(e), ti);
    int bad = 0;
    for (int m = 0; m < 128; ++m)
      for (int c = 0; c < 16; ++c) {
        float exp = mode == 0 ? (c < 4 ? float(m + 1000 * c) : h[m * 16 + c])
                  : mode == 1 ? 8.f : mode == 2 ? float((m % 8) * 16 + c)
                  : mode == 3 ? float(8 * c + 32 * 28) : mode == 5 ? 8.f : float(8 * c + 16 * 28);
        if (h[m * 16 + c] != exp) ++bad;
      }
    printf("  mismatches %d / 2048   D[0][0]=%.10f\n", bad, h[0]);
    for (int m = 0; m < 10; ++m) {
      printf("  row %3d:", m);
      for (int c = 0; c < 8; ++c) printf(" %8.1f", h[m * 16 + c]);
      printf("\n");
    }
  }
  return 0;
}
