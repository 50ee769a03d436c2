// pipe_bench.cu -- measures warp-instruction throughput per SM per cycle of the
// instruction mixes the search kernel's inner loop can be built from (design input for
// DESIGN.md §5; not part of libffs.so).  nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cstdio>
#include <cstdint>

constexpr int ITERS = 32768, CH = 8;

#define KERNEL(name, BODY)                                                            \
  __global__ void name(float* out, unsigned long long* cyc, float a, float b, int ia, int ib) { \
    float f[CH];                                                                      \
    int r[CH];                                                                        \
    _Pragma("unroll") for (int i = 0; i < CH; ++i) {                                  \
      f[i] = threadIdx.x * 0.001f + i;                                                \
      r[i] = threadIdx.x + i;                                                         \
    }                                                                                 \
    unsigned long long t0 = clock64();                                                \
    _Pragma("unroll 1") for (int it = 0; it < ITERS; ++it) {                          \
      _Pragma("unroll") for (int i = 0; i < CH; ++i) { BODY }                         \
    }                                                                                 \
    unsigned long long t1 = clock64();                                                \
    float s = 0;                                                                      \
    _Pragma("unroll") for (int i = 0; i < CH; ++i) s += f[i] + (float)r[i];           \
    if (s == 1234.5f) out[0] = s;                                                     \
    if (threadIdx.x == 0) atomicAdd(cyc, t1 - t0);                                    \
  }

// 1 instruction per body
KERNEL(k_ffma, asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(f[i]) : "f"(a), "f"(b));)
KERNEL(k_fadd, asm volatile("add.f32 %0, %0, %1;" : "+f"(f[i]) : "f"(a));)
KERNEL(k_fmul, asm volatile("mul.f32 %0, %0, %1;" : "+f"(f[i]) : "f"(a));)
KERNEL(k_iadd, asm volatile("add.s32 %0, %0, %1;" : "+r"(r[i]) : "r"(ia));)
KERNEL(k_lop3, asm volatile("lop3.b32 %0, %0, %1, %2, 0xEA;" : "+r"(r[i]) : "r"(ia), "r"(ib));)
KERNEL(k_fsetp, { int p; asm volatile("{.reg .pred q; setp.gt.f32 q, %1, %2; selp.s32 %0, 1, 0, q;}" : "=r"(p) : "f"(f[i]), "f"(a)); r[i] ^= p; })
KERNEL(k_imad, asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(r[i]) : "r"(ia), "r"(ib));)
// 4-instruction core: FFMA + FADD + IADD + LOP3 (2 per body: fma/add on f, sub/lop on r)
KERNEL(k_core4, {
  asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(f[i]) : "f"(a), "f"(b));
  asm volatile("add.f32 %0, %0, %1;" : "+f"(f[i]) : "f"(a));
  asm volatile("sub.s32 %0, %1, %0;" : "+r"(r[i]) : "r"(ia));
  asm volatile("lop3.b32 %0, %0, %1, %2, 0xA8;" : "+r"(r[i]) : "r"(ib), "r"(__float_as_int(f[i])));
})
// packed fp32x2 (sm_100): two lanes per instruction
KERNEL(k_ffma2, {
  uint64_t v = ((uint64_t)__float_as_uint(f[i]) << 32) | __float_as_uint(f[i] + 1.f);
  uint64_t A = ((uint64_t)__float_as_uint(a) << 32) | __float_as_uint(a);
  uint64_t Bv = ((uint64_t)__float_as_uint(b) << 32) | __float_as_uint(b);
  asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(v) : "l"(A), "l"(Bv));
  f[i] = __uint_as_float((uint32_t)v) + __uint_as_float((uint32_t)(v >> 32));
})
KERNEL(k_fadd2_chain, {
  uint64_t A = ((uint64_t)__float_as_uint(a) << 32) | __float_as_uint(b);
  uint64_t v = ((uint64_t)r[i] << 32) | (uint32_t)r[i];
#pragma unroll
  for (int j = 0; j < 4; ++j) asm volatile("add.rn.f32x2 %0, %0, %1;" : "+l"(v) : "l"(A));
  r[i] = (int)(v ^ (v >> 32));
})
KERNEL(k_fadd_chain4, {
  float x = __int_as_float(r[i]);
#pragma unroll
  for (int j = 0; j < 4; ++j) asm volatile("add.f32 %0, %0, %1;" : "+f"(x) : "f"(a));
  r[i] = __float_as_int(x);
})
// FFMA + IADD alternating
KERNEL(k_ffma_iadd, {
  asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(f[i]) : "f"(a), "f"(b));
  asm volatile("add.s32 %0, %0, %1;" : "+r"(r[i]) : "r"(ia));
})
// FADD + IADD alternating
KERNEL(k_fadd_iadd, {
  asm volatile("add.f32 %0, %0, %1;" : "+f"(f[i]) : "f"(a));
  asm volatile("add.s32 %0, %0, %1;" : "+r"(r[i]) : "r"(ia));
})

template <class K>
void run(const char* name, K kern, int insts_per_body, int blocks_per_sm, int threads) {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float* out;
  unsigned long long* cyc;
  cudaMalloc(&out, 4);
  cudaMalloc(&cyc, 8);
  int blocks = sms * blocks_per_sm;
  kern<<<blocks, threads>>>(out, cyc, 1.0001f, 0.5f, 3, 5);
  cudaMemset(cyc, 0, 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  kern<<<blocks, threads>>>(out, cyc, 1.0001f, 0.5f, 3, 5);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long c;
  cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  double warp_insts = (double)blocks * (threads / 32) * ITERS * CH * insts_per_body;
  double avg_cyc = (double)c / blocks;  // cycles per block (thread 0)
  double per_sm_cycle = warp_insts / sms / avg_cyc * (1.0 / blocks_per_sm) * blocks_per_sm;
  // warp-instructions per SM per cycle, using in-kernel cycle counts (all blocks resident)
  double wi_sm_cyc = (double)(threads / 32) * blocks_per_sm * ITERS * CH * insts_per_body / avg_cyc;
  printf("%-12s warps/SM=%3d  warp-inst/SM/cycle=%.3f  lane-ops/s=%.3e  (%.3f ms)\n", name,
         threads / 32 * blocks_per_sm, wi_sm_cyc, warp_insts * 32 / (ms * 1e-3), ms);
  (void)per_sm_cycle;
  cudaFree(out);
  cudaFree(cyc);
}

int main() {
  for (int occ : {2, 4, 8}) {
    run("ffma", k_ffma, 1, occ, 256);
    run("ffma2", k_ffma2, 1, occ, 256);
    run("fadd", k_fadd, 1, occ, 256);
    run("fmul", k_fmul, 1, occ, 256);
    run("iadd", k_iadd, 1, occ, 256);
    run("lop3", k_lop3, 1, occ, 256);
    run("imad", k_imad, 1, occ, 256);
    run("core4", k_core4, 4, occ, 256);
    run("fadd2x4", k_fadd2_chain, 4, occ, 256);
    run("faddx4", k_fadd_chain4, 4, occ, 256);
    run("ffma+iadd", k_ffma_iadd, 2, occ, 256);
    run("fadd+iadd", k_fadd_iadd, 2, occ, 256);
  }
  return 0;
}
