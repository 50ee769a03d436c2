// core_bench16.cu -- candidate-pair cores in packed fp32x2 (current) vs packed f16x2
// (design input for a half-precision pre-filter).  Each body = one
// candidate pair; reports candidates/s over all SMs.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/core_bench16.cu -o tools/core_bench16
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>
typedef unsigned long long f2;
constexpr int ITERS = 16384, CH = 6;

__device__ __forceinline__ f2 fa2(f2 a, f2 b) { f2 d; asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b)); return d; }
__device__ __forceinline__ f2 fs2(f2 a, f2 b) { f2 d; asm volatile("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b)); return d; }
__device__ __forceinline__ f2 ff2(f2 a, f2 b, f2 c) { f2 d; asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c)); return d; }
__device__ __forceinline__ void lo2(f2 v, uint32_t& l, uint32_t& h) { asm("mov.b64 {%0,%1}, %2;" : "=r"(l), "=r"(h) : "l"(v)); }
__device__ __forceinline__ uint32_t ha2(uint32_t a, uint32_t b) { uint32_t d; asm volatile("add.rn.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
__device__ __forceinline__ uint32_t hs2(uint32_t a, uint32_t b) { uint32_t d; asm volatile("sub.rn.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
__device__ __forceinline__ uint32_t hf2(uint32_t a, uint32_t b, uint32_t c) { uint32_t d; asm volatile("fma.rn.f16x2 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }
__device__ __forceinline__ uint32_t bf2(uint32_t a, uint32_t b, uint32_t c) { uint32_t d; asm volatile("fma.rn.bf16x2 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }

// A: FFMA2, FADD2, FADD2(sub), LOP3 x2  (the KS=4 kernel's core)
__global__ void kA(uint32_t* out, f2 t2, f2 cc, f2 U, f2 w3) {
  f2 S[CH]; uint32_t aA[CH], aB[CH];
  for (int i = 0; i < CH; ++i) { S[i] = (f2)(threadIdx.x + i) * 0x100000001ull; aA[i] = aB[i] = ~0u; }
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      f2 z = fa2(ff2(S[i], t2, cc), U);
      f2 d = fs2(w3, S[i]);
      uint32_t zl, zh, dl, dh; lo2(z, zl, zh); lo2(d, dl, dh);
      aA[i] &= zl | dl; aB[i] &= zh | dh;
      S[i] ^= (f2)(aA[i] & 1);
    }
  }
  uint32_t r = 0; for (int i = 0; i < CH; ++i) r ^= aA[i] ^ aB[i];
  if (r == 0x1234567) out[0] = r;
}
// D: HFMA2, HADD2, HADD2(sub), one LOP3 for both halves
__global__ void kD(uint32_t* out, uint32_t t2, uint32_t cc, uint32_t U, uint32_t w3) {
  uint32_t S[CH], a[CH];
  for (int i = 0; i < CH; ++i) { S[i] = 0x3c003c00u ^ (threadIdx.x + i); a[i] = ~0u; }
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      uint32_t z = ha2(hf2(S[i], t2, cc), U);
      uint32_t d = hs2(w3, S[i]);
      a[i] &= z | d;
      S[i] ^= (a[i] & 1);
    }
  }
  uint32_t r = 0; for (int i = 0; i < CH; ++i) r ^= a[i];
  if (r == 0x1234567) out[0] = r;
}
// E: D with bf16x2 FMA
__global__ void kE(uint32_t* out, uint32_t t2, uint32_t cc, uint32_t U, uint32_t w3) {
  uint32_t S[CH], a[CH];
  for (int i = 0; i < CH; ++i) { S[i] = 0x3f803f80u ^ (threadIdx.x + i); a[i] = ~0u; }
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      uint32_t z = bf2(S[i], t2, cc);
      z = bf2(z, 0x3f803f80u, U);
      uint32_t d = bf2(S[i], 0xbf80bf80u, w3);
      a[i] &= z | d;
      S[i] ^= (a[i] & 1);
    }
  }
  uint32_t r = 0; for (int i = 0; i < CH; ++i) r ^= a[i];
  if (r == 0x1234567) out[0] = r;
}
// F: f16x2 with the SLO folded as FMA (d = fma(S, -1, w3)) -- all three on the FMA form
__global__ void kF(uint32_t* out, uint32_t t2, uint32_t cc, uint32_t U, uint32_t w3) {
  uint32_t S[CH], a[CH];
  for (int i = 0; i < CH; ++i) { S[i] = 0x3c003c00u ^ (threadIdx.x + i); a[i] = ~0u; }
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      uint32_t z = hf2(S[i], t2, ha2(cc, U));
      uint32_t d = hs2(w3, S[i]);
      a[i] &= z | d;
      S[i] ^= (a[i] & 1);
    }
  }
  uint32_t r = 0; for (int i = 0; i < CH; ++i) r ^= a[i];
  if (r == 0x1234567) out[0] = r;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint32_t* o; cudaMalloc(&o, 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const char* names[] = {"A f32x2 (current)", "D f16x2", "E bf16x2 (3 fma)", "F f16x2 fma-folded"};
  for (int warps : {8, 16, 32}) {
    int blocks = sms * warps / 8, thr = 256;
    for (int v = 0; v < 4; ++v) {
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(a);
        if (v == 0) kA<<<blocks, thr>>>(o, 0x3f8000003f800000ull, 0, 0, 0);
        if (v == 1) kD<<<blocks, thr>>>(o, 0x3c003c00u, 0, 0, 0);
        if (v == 2) kE<<<blocks, thr>>>(o, 0x3f803f80u, 0, 0, 0);
        if (v == 3) kF<<<blocks, thr>>>(o, 0x3c003c00u, 0, 0, 0);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        double cands = (double)blocks * thr * ITERS * CH * 2;
        if (rep) printf("warps/SM=%2d %-20s: %.3e cand/s  (%.2f SMSP-cycles per 32 cand at 1.965GHz)\n", warps, names[v],
                        cands / (ms * 1e-3), (double)sms * 4 * 1.965e9 / (cands / (ms * 1e-3)) * 32);
      }
    }
  }
  return 0;
}
