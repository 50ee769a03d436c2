// pipe_bench16.cu -- issue rate (warp-instructions per SMSP per clock) of the f16x2 forms
// the KS = 4 body uses: HFMA2 with three registers, HADD2, HFMA2 with an immediate
// multiplicand (a * 1 + b, what ptxas emits for many adds), IADD3, LOP3, and 1:1 mixes.
// Design input for DESIGN.md §4.3.  nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cstdio>
#include <cstdint>
constexpr int ITERS = 16384, CH = 8;

#define KERNEL(name, BODY)                                                                 \
  __global__ void name(uint32_t* out, unsigned long long* cyc, uint32_t a, uint32_t b) { \
    uint32_t r[CH], q[CH];                                                                 \
    _Pragma("unroll") for (int i = 0; i < CH; ++i) { r[i] = 0x3c003c00u + threadIdx.x + i; q[i] = r[i] ^ 0x55; } \
    unsigned long long t0 = clock64();                                                     \
    _Pragma("unroll 1") for (int it = 0; it < ITERS; ++it) {                               \
      _Pragma("unroll") for (int i = 0; i < CH; ++i) { BODY }                              \
    }                                                                                      \
    unsigned long long t1 = clock64();                                                     \
    uint32_t s = 0;                                                                        \
    _Pragma("unroll") for (int i = 0; i < CH; ++i) s ^= r[i] ^ q[i];                       \
    if (s == 0x12345) out[0] = s;                                                          \
    if (threadIdx.x == 0) atomicAdd(cyc, t1 - t0);                                         \
  }

KERNEL(k_hfma_rrr, asm volatile("fma.rn.f16x2 %0, %0, %1, %2;" : "+r"(r[i]) : "r"(a), "r"(b));)
KERNEL(k_hadd, asm volatile("add.rn.f16x2 %0, %0, %1;" : "+r"(r[i]) : "r"(a));)
KERNEL(k_hfma_imm, asm volatile("fma.rn.f16x2 %0, %0, %2, %1;" : "+r"(r[i]) : "r"(a), "r"(0x3c003c00u));)
KERNEL(k_iadd3, asm volatile("{.reg .u32 t; sub.u32 t, %0, %1; add.u32 %0, t, %2;}" : "+r"(r[i]) : "r"(a), "r"(b));)
KERNEL(k_lop3, asm volatile("lop3.b32 %0, %0, %1, %2, 0xEA;" : "+r"(r[i]) : "r"(a), "r"(b));)
KERNEL(k_mix_hfma_lop3, {
  asm volatile("fma.rn.f16x2 %0, %0, %1, %2;" : "+r"(r[i]) : "r"(a), "r"(b));
  asm volatile("lop3.b32 %0, %0, %1, %2, 0xEA;" : "+r"(q[i]) : "r"(a), "r"(b));
})
KERNEL(k_mix_hadd_iadd3, {
  asm volatile("add.rn.f16x2 %0, %0, %1;" : "+r"(r[i]) : "r"(a));
  asm volatile("{.reg .u32 t; sub.u32 t, %0, %1; add.u32 %0, t, %2;}" : "+r"(q[i]) : "r"(a), "r"(b));
})
KERNEL(k_mix_hfmaimm_lop3, {
  asm volatile("fma.rn.f16x2 %0, %0, %2, %1;" : "+r"(r[i]) : "r"(a), "r"(0x3c003c00u));
  asm volatile("lop3.b32 %0, %0, %1, %2, 0xEA;" : "+r"(q[i]) : "r"(a), "r"(b));
})

template <class K>
void run(const char* name, K kern, int ipb, int warps) {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint32_t* out;
  unsigned long long* cyc;
  cudaMalloc(&out, 4);
  cudaMalloc(&cyc, 8);
  int thr = 32 * warps;
  kern<<<sms, thr>>>(out, cyc, 0x3c003c00u, 0x00010001u);
  cudaMemset(cyc, 0, 8);
  kern<<<sms, thr>>>(out, cyc, 0x3c003c00u, 0x00010001u);
  cudaDeviceSynchronize();
  unsigned long long c;
  cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  double avg = (double)c / sms;  // cycles of the block's thread 0
  double wi = (double)warps * ITERS * CH * ipb / avg / 4.0;  // per SMSP per clock
  printf("%-20s warps/SM=%2d  warp-inst/SMSP/clk=%.3f\n", name, warps, wi);
  cudaFree(out);
  cudaFree(cyc);
}

int main() {
  for (int w : {8, 16}) {
    run("hfma2 rrr", k_hfma_rrr, 1, w);
    run("hadd2", k_hadd, 1, w);
    run("hfma2 imm", k_hfma_imm, 1, w);
    run("iadd3", k_iadd3, 1, w);
    run("lop3", k_lop3, 1, w);
    run("hfma2+lop3", k_mix_hfma_lop3, 2, w);
    run("hadd2+iadd3", k_mix_hadd_iadd3, 2, w);
    run("hfma2imm+lop3", k_mix_hfmaimm_lop3, 2, w);
  }
  return 0;
}
