// core_bench16c.cu -- candidate-pair cores: the per-candidate f16x2 test (4 ops/pair) vs the per-group
// max of the scores (HFMA2 + 3-input VHMNMX) with a group SLO test.  Design input for DESIGN.md §4.3.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cstdio>
#include <cstdint>
constexpr int ITERS = 8192;
__device__ __forceinline__ uint32_t ha2(uint32_t a, uint32_t b) { uint32_t d; asm volatile("add.rn.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
__device__ __forceinline__ uint32_t hs2(uint32_t a, uint32_t b) { uint32_t d; asm volatile("sub.rn.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
__device__ __forceinline__ uint32_t hf2(uint32_t a, uint32_t b, uint32_t c) { uint32_t d; asm volatile("fma.rn.f16x2 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }
__device__ __forceinline__ uint32_t hmax(uint32_t a, uint32_t b) { uint32_t d; asm volatile("max.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
__device__ __forceinline__ uint32_t imax(uint32_t a, uint32_t b) { uint32_t d; asm volatile("max.s16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
__device__ __forceinline__ uint32_t isub(uint32_t a, uint32_t b, uint32_t z) { uint32_t d; asm volatile("{.reg .u32 t; sub.u32 t, %1, %2; add.u32 %0, t, %3;}" : "=r"(d) : "r"(a), "r"(b), "r"(z)); return d; }

template <int V>
__global__ void kq(uint32_t* out, const uint32_t* tab, uint32_t zero) {
  uint32_t t2[5], cc[5], w3[5], a2[5];
  for (int p = 0; p < 5; ++p) { t2[p] = tab[p]; cc[p] = tab[5 + p]; w3[p] = tab[10 + p]; a2[p] = tab[16 + p]; }
  uint32_t S = 0x3c003c00u ^ threadIdx.x, NL = tab[15], slk = tab[21], acc0 = ~0u, acc1 = ~0u, acc2 = ~0u;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int g = 0; g < 5; ++g) {
      const uint32_t S3 = ha2(S, t2[g]);
      const uint32_t U = hf2(S3, S3, hs2(NL, a2[g]));
      uint32_t a = ~0u;
      if (V == 0) {
#pragma unroll
        for (int p = 0; p < 5; ++p) {
          const uint32_t z = ha2(hf2(S3, t2[p], cc[p]), U);
          a &= z | ~isub(w3[p], S3, zero);
        }
      } else {
        uint32_t y[5];
#pragma unroll
        for (int p = 0; p < 5; ++p) y[p] = hf2(S3, t2[p], cc[p]);
        uint32_t m;
        if (V == 1) m = hmax(hmax(hmax(y[0], y[1]), hmax(y[2], y[3])), y[4]);
        else m = imax(imax(imax(y[0], y[1]), imax(y[2], y[3])), y[4]);
        a = ha2(m, U) | ~isub(slk, S3, zero);
      }
      if (g % 3 == 0) acc0 &= a; else if (g % 3 == 1) acc1 &= a; else acc2 &= a;
    }
    S ^= (acc0 & acc1 & acc2 & 1);
  }
  if ((acc0 ^ acc1 ^ acc2) == 0x1234567) out[0] = 1;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint32_t *o, *tab; cudaMalloc(&o, 4); cudaMalloc(&tab, 64 * 4); cudaMemset(tab, 0, 256);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const char* nm[3] = {"current (4 ops/pair)", "hmax2 + group SLO   ", "imax16 + group SLO  "};
  for (int warps : {8, 12, 16, 24}) {
    int blocks = sms * warps / 4, thr = 128;
    for (int v = 0; v < 3; ++v)
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(a);
        if (v == 0) kq<0><<<blocks, thr>>>(o, tab, 0); else if (v == 1) kq<1><<<blocks, thr>>>(o, tab, 0); else kq<2><<<blocks, thr>>>(o, tab, 0);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        double cands = (double)blocks * thr * ITERS * 25 * 2;
        if (rep) printf("warps/SM=%2d %s: %.3e cand/s (%.2f SMSP-cycles per 32 cand)\n", warps, nm[v],
                        cands / (ms * 1e-3), (double)sms * 4 * 1.965e9 / (cands / (ms * 1e-3)) * 32);
      }
  }
  return 0;
}
