// issue_bench.cu -- warp-instructions per SMSP per cycle of packed-f16 / integer mixes, to
// choose the roofline denominator's microbenchmark (not part of libffs.so).
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/issue_bench tools/issue_bench.cu
#include <cstdint>
#include <cstdio>

constexpr int ITERS = 16384, CH = 8;

#define KERNEL(name, BODY)                                                                          \
  __global__ void name(uint32_t* out, unsigned long long* cyc, uint32_t a, uint32_t b, uint32_t c) { \
    uint32_t h[CH], r[CH];                                                                          \
    _Pragma("unroll") for (int i = 0; i < CH; ++i) {                                                \
      h[i] = 0x3c003c00u ^ (threadIdx.x + i);                                                       \
      r[i] = threadIdx.x * 3 + i;                                                                   \
    }                                                                                               \
    unsigned long long t0 = clock64();                                                              \
    _Pragma("unroll 1") for (int it = 0; it < ITERS; ++it) {                                        \
      _Pragma("unroll") for (int i = 0; i < CH; ++i) { BODY }                                       \
    }                                                                                               \
    unsigned long long t1 = clock64();                                                              \
    uint32_t s = 0;                                                                                 \
    _Pragma("unroll") for (int i = 0; i < CH; ++i) s ^= h[i] ^ r[i];                                \
    if (s == 0x12345u) out[0] = s;                                                                  \
    if (threadIdx.x == 0) atomicAdd(cyc, t1 - t0);                                                  \
  }

#define HFMA2 asm volatile("fma.rn.f16x2 %0, %0, %1, %2;" : "+r"(h[i]) : "r"(a), "r"(b));
#define HADD2 asm volatile("add.rn.f16x2 %0, %0, %1;" : "+r"(h[i]) : "r"(a));
#define HMNMX2 asm volatile("max.f16x2 %0, %0, %1;" : "+r"(r[i]) : "r"(c));
#define LOP3 asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(r[i]) : "r"(a), "r"(c));
#define IADDI asm volatile("add.u32 %0, %0, 12345;" : "+r"(r[i]));
#define IADD3 asm volatile("{.reg .u32 t; add.u32 t, %0, %1; add.u32 %0, t, %2;}" : "+r"(r[i]) : "r"(a), "r"(c));

KERNEL(k_hfma2, HFMA2)
KERNEL(k_hadd2, HADD2)
KERNEL(k_lop3, LOP3)
KERNEL(k_iaddi, IADDI)
KERNEL(k_hmnmx2, HMNMX2)
KERNEL(k_hfma2_lop3, HFMA2 LOP3)
KERNEL(k_hfma2_iaddi, HFMA2 IADDI)
KERNEL(k_hadd2_iaddi, HADD2 IADDI)
KERNEL(k_hfma2_hmnmx2, HFMA2 HMNMX2)
KERNEL(k_hfma2_iadd3, HFMA2 IADD3)
KERNEL(k_2hfma2_lop3, HFMA2 HFMA2 LOP3)

template <class K>
void run(const char* name, K kern, int per_body, int blocks_per_sm, int threads) {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint32_t* out;
  unsigned long long* cyc;
  cudaMalloc(&out, 4);
  cudaMalloc(&cyc, 8);
  const int blocks = sms * blocks_per_sm;
  for (int w = 0; w < 3; ++w) kern<<<blocks, threads>>>(out, cyc, 0x3bff3bffu, 0x10001000u, 0x12340000u);
  cudaMemset(cyc, 0, 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  kern<<<blocks, threads>>>(out, cyc, 0x3bff3bffu, 0x10001000u, 0x12340000u);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long c;
  cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  const double avg_cyc = (double)c / blocks;  // cycles per block (thread 0)
  const double warps_per_smsp = threads / 32.0 * blocks_per_sm / 4.0;
  const double ipc = warps_per_smsp * ITERS * CH * per_body / avg_cyc;  // warp-instr / SMSP / cycle
  const double lane_per_s = (double)blocks * threads * ITERS * CH * per_body / (ms * 1e-3);
  printf("%-14s warps/SMSP=%4.1f  IPC/SMSP=%.3f  lane-instr/s=%.3e  clock~%.0f MHz\n", name, warps_per_smsp, ipc,
         lane_per_s, avg_cyc / (ms * 1e3));
  cudaFree(out);
  cudaFree(cyc);
}

int main() {
  for (int occ : {4, 8}) {
    run("hfma2", k_hfma2, 1, occ, 256);
    run("hadd2", k_hadd2, 1, occ, 256);
    run("lop3", k_lop3, 1, occ, 256);
    run("iadd-imm", k_iaddi, 1, occ, 256);
    run("hmnmx2", k_hmnmx2, 1, occ, 256);
    run("hfma2+lop3", k_hfma2_lop3, 2, occ, 256);
    run("hfma2+iaddi", k_hfma2_iaddi, 2, occ, 256);
    run("hadd2+iaddi", k_hadd2_iaddi, 2, occ, 256);
    run("hfma2+hmnmx2", k_hfma2_hmnmx2, 2, occ, 256);
    run("hfma2+iadd3", k_hfma2_iadd3, 2, occ, 256);
    run("2hfma2+lop3", k_2hfma2_lop3, 3, occ, 256);
  }
  return 0;
}
