// ffs_kernels.cu -- sm_100a kernels of the batched pipeline-construction search.
//
// K0  k_count_tasks / k_scan_*  per-request task counts C(n-1, k-1) for every stage count
//                               k and their exclusive uint64 prefix (A1)
// K1  k_plan_search<KS>          one launch per stage count KS: unrank cut masks in
//                               registers, enumerate the P^KS profile sequences with
//                               hoisted partial sums, score + check feasibility, reduce
//                               to the per-request minimum packed key (A2-A5)
// K2  k_decode                   key -> plan, recompute figures, bind slices, victims (A6, A8)
// K3  k_evict                    keep-alive state + LRU eviction key per instance (A7)
// K4  k_victim_table/_pick        per-request LRU victim over a tick's instances (A8)
//     (k_victims: warp-per-load scan, used when the per-tick table would be too large)
// K5  k_int_peak                 integer issue-rate microbenchmark (roofline denominator)
//
// Paper: FluidFaaS, HPDC '25.  P:<line> = line of PAPER.md; R<n> = DESIGN.md §3 reading.
#include <algorithm>
#include <cstdio>
#include <type_traits>

#include "ffs_internal.h"

namespace ffsk {

__device__ __forceinline__ uint64_t img_u64(const uint32_t* w, uint32_t o) {
  return (uint64_t)w[o] | ((uint64_t)w[o + 1] << 32);
}
// The prefix-latency table PL is stored as fp32: every prefix is an integer < 2^24 (the
// ffs_stage_tables bound), so values and differences are exact.  Integer uses convert back.
__device__ __forceinline__ float plf(const uint32_t* w, uint32_t o) { return __uint_as_float(w[o]); }
__device__ __forceinline__ uint32_t pl_diff(const uint32_t* w, uint32_t ob, uint32_t oa) {
  return __float2uint_rn(plf(w, ob) - plf(w, oa));
}
// minimum over the (full) warp of a 64-bit value: the minimum high word, then the minimum
// low word among the lanes holding it -- two REDUX.MIN instead of five shuffle rounds
__device__ __forceinline__ uint64_t warp_min_u64(uint64_t x) {
  const uint32_t hi = (uint32_t)(x >> 32), lo = (uint32_t)x;
  const uint32_t mh = __reduce_min_sync(0xffffffffu, hi);
  const uint32_t ml = __reduce_min_sync(0xffffffffu, hi == mh ? lo : 0xffffffffu);
  return (uint64_t)mh << 32 | ml;
}

// profiles whose slice can host function f monolithically within budget B (defined with
// the victim kernels, K4)
__device__ __forceinline__ uint32_t victim_profiles(const uint32_t* img, const ImageLayout& L, uint32_t f, uint32_t B);

__device__ __forceinline__ uint32_t binom(const uint32_t* img, const ImageLayout& L, int c, int i) {
  return img[L.o_binom + c * 8 + i];  // C(c, i), 0 when c < i
}

// ====================================================================================
// K0: task counts and exclusive prefix (A1)
// ====================================================================================
__global__ void k_count_tasks(const ffs_request* __restrict__ req, const uint32_t* __restrict__ img,
                              ImageLayout lay, uint32_t n_nodes, uint32_t n_req, uint32_t K,
                              const uint64_t* __restrict__ node_free, uint32_t skip_full,
                              uint64_t* __restrict__ prefix, int64_t* __restrict__ keys,
                              unsigned long long* __restrict__ checks, unsigned long long* __restrict__ work_ctr,
                              uint32_t k_first, uint32_t k_last) {
  uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r < (uint32_t)kCtrWords) {  // the counters of the segments this call runs (all on k_first = 1)
    const uint32_t ks = r % kCtrBlock;
    if (k_first <= 1 || (ks >= k_first && ks <= k_last)) work_ctr[r] = 0;
  }
  if (r > n_req) return;
  uint32_t n = 0;
  if (r < n_req) {
    ffs_request q = req[r];
    if (q.func < lay.F && q.node < n_nodes) n = img[lay.o_fdesc + 4 * q.func + 1];
    // a node without any free slice admits no candidate: no tasks (INFEASIBLE without
    // enumeration, R37); verify mode enumerates them anyway for the checksums
    if (skip_full && n && node_free[q.node] == 0) n = 0;
    if (keys) keys[r] = (int64_t)kKeyNone;
    if (checks) {
      checks[3ull * r] = 0;
      checks[3ull * r + 1] = 0;
      checks[3ull * r + 2] = 0;
    }
  }
  for (uint32_t k = 1; k <= K; ++k)
    prefix[(uint64_t)(k - 1) * (n_req + 1) + r] = (n >= k) ? binom(img, lay, n - 1, k - 1) : 0ull;
}

constexpr int kScanT = 256, kScanI = 8, kScanChunk = kScanT * kScanI;

__device__ uint64_t block_exclusive_scan(uint64_t v, uint64_t* total) {
  __shared__ uint64_t ws[kScanT / 32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint64_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) ws[w] = x;
  __syncthreads();
  if (w == 0) {
    uint64_t s = lane < kScanT / 32 ? ws[lane] : 0;
#pragma unroll
    for (int o = 1; o < kScanT / 32; o <<= 1) {
      uint64_t y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < kScanT / 32) ws[lane] = s;
  }
  __syncthreads();
  uint64_t out = (w ? ws[w - 1] : 0) + x - v;
  *total = ws[kScanT / 32 - 1];
  __syncthreads();
  return out;
}

// per (segment, chunk) sum
__global__ void __launch_bounds__(kScanT) k_scan_reduce(const uint64_t* __restrict__ prefix, uint64_t len,
                                                         uint64_t* __restrict__ bsum, uint32_t nb) {
  const uint64_t* a = prefix + (uint64_t)blockIdx.y * len;
  uint64_t base = (uint64_t)blockIdx.x * kScanChunk + (uint64_t)threadIdx.x * kScanI, s = 0;
#pragma unroll
  for (int i = 0; i < kScanI; ++i)
    if (base + i < len) s += a[base + i];
  uint64_t tot;
  block_exclusive_scan(s, &tot);
  if (threadIdx.x == 0) bsum[(uint64_t)blockIdx.y * nb + blockIdx.x] = tot;
}

// exclusive scan of the chunk sums, one block per segment
__global__ void __launch_bounds__(kScanT) k_scan_top(uint64_t* __restrict__ bsum, uint32_t nb) {
  uint64_t* a = bsum + (uint64_t)blockIdx.x * nb;
  uint64_t carry = 0;
  for (uint32_t base = 0; base < nb; base += kScanT) {
    uint32_t i = base + threadIdx.x;
    uint64_t v = i < nb ? a[i] : 0, tot;
    uint64_t e = block_exclusive_scan(v, &tot);
    if (i < nb) a[i] = carry + e;
    carry += tot;
  }
}

__global__ void __launch_bounds__(kScanT) k_scan_apply(uint64_t* __restrict__ prefix, uint64_t len,
                                                        const uint64_t* __restrict__ bsum, uint32_t nb) {
  uint64_t* a = prefix + (uint64_t)blockIdx.y * len;
  uint64_t base = (uint64_t)blockIdx.x * kScanChunk + (uint64_t)threadIdx.x * kScanI;
  uint64_t v[kScanI], s = 0;
#pragma unroll
  for (int i = 0; i < kScanI; ++i) {
    v[i] = base + i < len ? a[base + i] : 0;
    s += v[i];
  }
  uint64_t tot;
  uint64_t run = block_exclusive_scan(s, &tot) + bsum[(uint64_t)blockIdx.y * nb + blockIdx.x];
#pragma unroll
  for (int i = 0; i < kScanI; ++i) {
    if (base + i < len) a[base + i] = run;
    run += v[i];
  }
}

cudaError_t launch_count_tasks(const ffs_request* req, const uint32_t* image, const ImageLayout& lay,
                               uint32_t n_nodes, uint32_t n_req, uint32_t k_max, const uint64_t* node_free,
                               bool skip_full, uint64_t* prefix, uint64_t* block_sums, int64_t* keys,
                               unsigned long long* checks, unsigned long long* work_ctr, uint32_t k_first,
                               uint32_t k_last, cudaStream_t st) {
  const uint64_t len = (uint64_t)n_req + 1;
  k_count_tasks<<<(unsigned)((len + 255) / 256), 256, 0, st>>>(req, image, lay, n_nodes, n_req, k_max, node_free,
                                                                skip_full ? 1u : 0u, prefix, keys, checks, work_ctr,
                                                                k_first, k_last);
  const uint32_t nb = (uint32_t)((len + kScanChunk - 1) / kScanChunk);
  dim3 g(nb, k_max);
  k_scan_reduce<<<g, kScanT, 0, st>>>(prefix, len, block_sums, nb);
  k_scan_top<<<k_max, kScanT, 0, st>>>(block_sums, nb);
  k_scan_apply<<<g, kScanT, 0, st>>>(prefix, len, block_sums, nb);
  return cudaGetLastError();
}

// K0b: requests grouped by chain length (exhaustive / verify KS = 4)
__device__ __forceinline__ uint32_t req_chain_len(const ffs_request* req, const uint32_t* img, const ImageLayout& lay,
                                                  uint32_t n_nodes, uint32_t r) {
  const ffs_request q = req[r];
  return (q.func < lay.F && q.node < n_nodes) ? img[lay.o_fdesc + 4 * q.func + 1] : 0u;
}

// Stable counting sort of the request ids by chain length n (0..33): the order must be
// deterministic -- a work unit names (n, group of 32 consecutive requests of the sorted
// order, mask chunk), and the ranks of a candidate-sharded step (separate calls) must agree
// on it.  Tiles of kGrpTile requests: per-tile counts, one exclusive scan over (n, tile),
// then a scatter that keeps the request order within n (the routing sort's pattern).
constexpr int kGrpT = 256, kGrpItems = 8, kGrpTile = kGrpT * kGrpItems, kGrpD = 34;
__global__ void __launch_bounds__(kGrpT) k_group_hist(const ffs_request* __restrict__ req, const uint32_t* __restrict__ img,
                                                      ImageLayout lay, uint32_t n_nodes, uint32_t n_req,
                                                      uint64_t* __restrict__ off, uint32_t nb) {
  __shared__ uint32_t h[kGrpD];
  if (threadIdx.x < kGrpD) h[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t base = blockIdx.x * kGrpTile;
  for (int i = threadIdx.x; i < kGrpTile; i += kGrpT)
    if (base + i < n_req) atomicAdd(&h[req_chain_len(req, img, lay, n_nodes, base + i)], 1u);
  __syncthreads();
  if (threadIdx.x < kGrpD) off[(uint64_t)threadIdx.x * nb + blockIdx.x] = h[threadIdx.x];
}

// one thread: tab[n] = first index of chain length n in perm (tab[33] = requests with
// n <= 32); tab[34 + n] / tab[68 + n] / tab[102 + n] = first work unit of n for KS = 4 / 3 /
// 2 (groups of 32 requests x chunks of masks), [34 + 33] / [68 + 33] / [102 + 33] = the unit
// counts.  Units are
// numbered from the longest chains down (n = 32 first): the warps grab the largest units
// first and the small ones fill the tail.
__global__ void k_group_tab(const uint32_t* __restrict__ img, ImageLayout lay, const uint64_t* __restrict__ off,
                            uint32_t nb, uint32_t s3, uint32_t* __restrict__ tab) {
  for (uint32_t n = 0; n < 34; ++n) tab[n] = (uint32_t)off[(uint64_t)n * nb];
  uint32_t u4 = 0, u3 = 0;
  for (int n = 32; n >= 0; --n) {
    tab[34 + n] = u4;
    tab[68 + n] = u3;
    if (n >= 3) {
      const uint32_t k = tab[n + 1] - tab[n], g = (k + 31) / 32;
      u3 += g * ((binom(img, lay, n - 1, 2) + s3 - 1) / s3);
      if (n >= 4) u4 += g * ((binom(img, lay, n - 1, 3) + kGrpS - 1) / kGrpS);
    }
  }
  tab[34 + 33] = u4;
  tab[68 + 33] = u3;
  uint32_t u2 = 0;  // KS = 2: one unit per group (n - 1 <= 31 masks)
  for (int n = 32; n >= 0; --n) {
    tab[102 + n] = u2;
    if (n >= 2) u2 += (tab[n + 1] - tab[n] + 31) / 32;
  }
  tab[102 + 33] = u2;
}

// stable scatter: warp w owns the contiguous eighth [w * 256, (w + 1) * 256) of the tile
__global__ void __launch_bounds__(kGrpT) k_group_scatter(const ffs_request* __restrict__ req,
                                                         const uint32_t* __restrict__ img, ImageLayout lay,
                                                         uint32_t n_nodes, uint32_t n_req,
                                                         const uint64_t* __restrict__ off, uint32_t nb,
                                                         uint32_t* __restrict__ perm) {
  constexpr int kW = kGrpT / 32;
  __shared__ uint32_t wh[kW][kGrpD];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int d = threadIdx.x; d < kW * kGrpD; d += kGrpT) (&wh[0][0])[d] = 0;
  __syncthreads();
  const uint32_t base = blockIdx.x * kGrpTile + w * (32 * kGrpItems);
  uint32_t dig[kGrpItems];
#pragma unroll
  for (int it = 0; it < kGrpItems; ++it) {  // pass 1: per-warp counts
    const uint32_t i = base + it * 32 + lane;
    const bool in = i < n_req;
    dig[it] = in ? req_chain_len(req, img, lay, n_nodes, i) : 64u + lane;
    const uint32_t m = __match_any_sync(0xffffffffu, dig[it]);
    if (in && lane == __ffs(m) - 1) wh[w][dig[it]] += __popc(m);
    __syncwarp();
  }
  __syncthreads();
  if (threadIdx.x < kGrpD) {  // exclusive prefix over warps per n, plus the (n, tile) offset
    const uint32_t d = threadIdx.x;
    uint32_t run = (uint32_t)off[(uint64_t)d * nb + blockIdx.x];
    for (int ww = 0; ww < kW; ++ww) {
      const uint32_t c = wh[ww][d];
      wh[ww][d] = run;
      run += c;
    }
  }
  __syncthreads();
#pragma unroll
  for (int it = 0; it < kGrpItems; ++it) {  // pass 2: scatter in request order
    const uint32_t i = base + it * 32 + lane;
    const bool in = i < n_req;
    const uint32_t m = __match_any_sync(0xffffffffu, dig[it]);
    if (in) perm[wh[w][dig[it]] + __popc(m & ((1u << lane) - 1))] = i;
    __syncwarp();
    if (in && lane == __ffs(m) - 1) wh[w][dig[it]] += __popc(m);
    __syncwarp();
  }
}

cudaError_t launch_group_n(const ffs_request* req, const uint32_t* image, const ImageLayout& lay, uint32_t n_nodes,
                           uint32_t n_req, uint32_t s3, uint64_t* off, uint64_t* bsum, uint32_t* tab, uint32_t* perm,
                           cudaStream_t st) {
  const uint32_t nb = (n_req + kGrpTile - 1) / kGrpTile;
  const uint64_t len = (uint64_t)kGrpD * nb + 1;  // the last entry (0) becomes the total
  const uint32_t sb = (uint32_t)((len + kScanChunk - 1) / kScanChunk);
  cudaMemsetAsync(off + len - 1, 0, 8, st);
  k_group_hist<<<nb, kGrpT, 0, st>>>(req, image, lay, n_nodes, n_req, off, nb);
  k_scan_reduce<<<dim3(sb, 1), kScanT, 0, st>>>(off, len, bsum, sb);
  k_scan_top<<<1, kScanT, 0, st>>>(bsum, sb);
  k_scan_apply<<<dim3(sb, 1), kScanT, 0, st>>>(off, len, bsum, sb);
  k_group_tab<<<1, 1, 0, st>>>(image, lay, off, nb, s3, tab);
  k_group_scatter<<<nb, kGrpT, 0, st>>>(req, image, lay, n_nodes, n_req, off, nb, perm);
  return cudaGetLastError();
}

// ====================================================================================
// K1: the search (A2-A5)
// ====================================================================================
// Per-thread state.  Everything indexed by a compile-time index stays in registers.
template <int KS>
struct SearchState {
  const uint32_t* sm;  // table image in shared memory
  uint32_t o_pl, o_pm, o_xf, o_cap, o_gpcs;
  // request
  uint32_t row0, n, B;
  uint32_t thr_u;     // throughput floor: max stage time (R38), 0xffffffff = none
  float thr;          // the same as an exact fp32 (clamped to 2^24 > every stage time)
  uint64_t freeb;     // 8 x u8 free counts (clamped to 8) of the request's node
  uint32_t free_w;    // 5-bit SWAR lanes 16 + free[p]
  uint64_t idx_base;  // offk[n][KS] + rank * P^KS
  int64_t best;
  float alpha;        // scale of sum t^2 in the balance filter
  float alpha_h;      // the same with the wider margin of the f16x2 pre-filter (KS = 4)
  uint64_t n_scored;  // candidates whose own score this thread computed (measurement)
  float tmin, tmax;   // KS = 4: sum over the chain of the min / max component latency over
                      // all profiles (bounds of every candidate's T, for the f16 scale)
  bool none_can_win;  // best's cvq/k already unbeatable by any KS-stage candidate
  // mask
  int bnd[KS + 1];
  uint32_t memst[KS];
  uint32_t X;         // transfer cost of the cuts
  float blim_raw, blim;
  // register tables of the last two stages: q = stage KS-2, p = stage KS-1
  float tq[kP], sqq[kP], aq[kP], tp[kP], sqp[kP], ap[kP];
  int pd[KS];         // digits of the outer levels
  // verify mode
  uint64_t nfeas, ksum;
};

template <int KS>
__device__ __forceinline__ void set_threshold(SearchState<KS>& c) {
  float ap = 0.f;  // alpha' = 1024 KS / (1025 + c*), rounded down; 0 while nothing is known
  if ((uint64_t)c.best == kKeyNone) {
    c.alpha = 0.f;
    c.none_can_win = false;
  } else {
    const int cb = (int)((uint64_t)c.best >> 50);
    const int kb = (int)(((uint64_t)c.best >> 47) & 7) + 1;
    const int cthr = (kb >= KS) ? cb : cb - 1;  // equal cvq wins only on fewer stages (R1)
    c.none_can_win = cthr < 0;
    // can-win: cvq <= cthr  <=>  1024*KS*sum t^2 < (1025 + cthr) * (sum t)^2
    // filter: (sum t)^2 > alpha * sum t^2 with alpha rounded down by a 2^-16 margin
    // 1024*KS*(1 - 2^-16) = KS*65535/64 is exact in fp32; the quotient is rounded down
    c.alpha = __fdiv_rd((float)(KS * 65535) * (1.f / 64.f), (float)(1025 + cthr));
    if constexpr (KS == 3 || KS == 4) ap = __fdiv_rd((float)(1024 * KS), (float)(1025 + cthr));
  }
  if constexpr (KS == 3 || KS == 4) {
    // f16x2 pre-filter (ks3_pair_h, ks4_pair_h): alpha_h = alpha' - 2^-6 (KS + 1 + alpha'),
    // every step rounded down; the margin covers the f16 rounding (DESIGN.md §4.3 "f16x2
    // pre-filter"; KS = 3 sums fewer terms, so the KS = 4 bound covers it)
    c.alpha_h = __fsub_rd(__fmul_rd(ap, 1.f - 1.f / 64.f), (float)(KS + 1) * (1.f / 64.f));
  }
  c.blim = c.none_can_win ? -1.f : c.blim_raw;
#pragma unroll
  for (int p = 0; p < kP; ++p) {
    c.aq[p] = c.alpha * c.sqq[p];
    c.ap[p] = c.alpha * c.sqp[p];
  }
}

// Exact integer evaluation of one candidate (the rare path): digits pd[0..KS-3], q, p.
template <int KS, bool VERIFY>
__device__ __forceinline__ void exact_eval(SearchState<KS>& c, int q, int p, bool fast_pass,
                                           unsigned long long* misses) {
  int prof[KS];
#pragma unroll
  for (int i = 0; i < KS; ++i) prof[i] = (i < KS - 2) ? c.pd[i] : (i == KS - 2 ? q : p);
  uint64_t St = 0, Sq = 0, seq = 0;
  uint32_t used = 0, g = 0;
  bool ok = true;
#pragma unroll
  for (int i = 0; i < KS; ++i) {
    const int pr = prof[i];
    const uint32_t a = (c.row0 + c.bnd[i]) * kRowW, b = (c.row0 + c.bnd[i + 1]) * kRowW;
    const uint32_t t = pl_diff(c.sm, c.o_pl + b + pr, c.o_pl + a + pr);
    ok &= c.memst[i] <= c.sm[c.o_cap + pr];
    ok &= t <= c.thr_u;  // R38 throughput floor
    St += t;
    Sq += (uint64_t)t * t;
    used += 1u << (4 * pr);
    g += c.sm[c.o_gpcs + pr];
    seq = seq * kP + (uint64_t)pr;
  }
#pragma unroll
  for (int pp = 0; pp < kP; ++pp) ok &= ((used >> (4 * pp)) & 15u) <= ((c.freeb >> (8 * pp)) & 255u);
  ok &= St + c.X <= (uint64_t)c.B;
  if (!ok) return;
  const uint64_t D = St * St;
  const uint64_t N = (uint64_t)KS * Sq - D;
  const uint64_t cvq = (N << 10) / D;  // floor(1024 * CV^2), exact (R4)
  const int64_t key =
      (int64_t)((cvq << 50) | ((uint64_t)(KS - 1) << 47) | ((uint64_t)g << 41) | (c.idx_base + seq));
  if (VERIFY) {
    c.nfeas++;
    c.ksum += (uint64_t)key;
    if (key < c.best && !fast_pass) atomicAdd(misses, 1ull);
  }
  if (key < c.best) {
    c.best = key;
    set_threshold(c);
  }
}

template <int KS, bool VERIFY>
__device__ __forceinline__ void handle_hits(SearchState<KS>& c, uint32_t all, uint32_t fast,
                                            unsigned long long* misses) {
  while (all) {
    const int bit = __ffs(all) - 1;
    all &= all - 1;
    const int q = bit / kP, p = bit - kP * (bit / kP);
    exact_eval<KS, VERIFY>(c, q, p, (fast >> bit) & 1u, misses);
  }
}

constexpr uint32_t kOne5 = 0x0108421u;  // 1 in each of the five 5-bit lanes
constexpr uint32_t kBit4 = kOne5 << 4;

// The innermost two levels, fully unrolled: P*P candidates with the stage-(KS-2)
// profile q and the stage-(KS-1) profile p.  Per candidate: one FADD (sum of stage
// times), one FFMA ((sum t)^2 - scaled prefix), two compares and a predicated OR.
template <int KS, bool VERIFY>
__device__ __forceinline__ void inner_block(SearchState<KS>& c, float S, float Q, uint32_t cw,
                                            unsigned long long* misses) {
  const uint32_t e1 = (cw - kOne5) & kBit4;      // profiles with >= 1 free slice left
  const uint32_t e2 = (cw - 2 * kOne5) & kBit4;  // ... with >= 2 left (p == q)
  const float INF = __int_as_float(0x7f800000);
  const float L0 = c.alpha * Q;
  float tq2[kP], tp2[kP], tpd[kP];
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t bit = 1u << (5 * x + 4);
    tq2[x] = (e1 & bit) ? c.tq[x] : INF;
    tp2[x] = (e1 & bit) ? c.tp[x] : INF;
    tpd[x] = (e2 & bit) ? c.tp[x] : INF;
  }
  uint32_t hits = 0;
#pragma unroll
  for (int q = 0; q < kP; ++q) {
    const float S2 = S + tq2[q];
    const float L2 = L0 + c.aq[q];
#pragma unroll
    for (int p = 0; p < kP; ++p) {
      const float St = S2 + (p == q ? tpd[p] : tp2[p]);
      const float r = fmaf(St, St, -L2);
      const bool pass = (St <= c.blim) & (r > c.ap[p]);
      hits |= (uint32_t)pass << (kP * q + p);
    }
  }
  if (VERIFY) {
    handle_hits<KS, VERIFY>(c, (1u << (kP * kP)) - 1, hits, misses);
  } else if (hits) {
    handle_hits<KS, VERIFY>(c, hits, hits, misses);
  }
}

template <int L, int KS, bool VERIFY>
__device__ __forceinline__ void outer_level(SearchState<KS>& c, float S, float Q, uint32_t cw,
                                            unsigned long long* misses) {
  if constexpr (L >= KS - 2) {
    inner_block<KS, VERIFY>(c, S, Q, cw, misses);
  } else {
    const float INF = __int_as_float(0x7f800000);
    const uint32_t a = c.o_pl + (c.row0 + c.bnd[L]) * kRowW, b = c.o_pl + (c.row0 + c.bnd[L + 1]) * kRowW;
#pragma unroll 1
    for (int p = 0; p < kP; ++p) {
      const uint32_t t = pl_diff(c.sm, b + p, a + p);
      const uint32_t cw2 = cw - (1u << (5 * p));
      const bool ok = (c.memst[L] <= c.sm[c.o_cap + p]) && t <= c.thr_u && ((cw2 >> (5 * p + 4)) & 1u);
      const float tf = ok ? __uint2float_rn(t) : INF;
      c.pd[L] = p;
      outer_level<L + 1, KS, VERIFY>(c, S + tf, fmaf(tf, tf, Q), cw2, misses);
    }
  }
}

// Load the register tables of stage s (its P latencies and squares).
template <int KS>
__device__ __forceinline__ void load_stage(const SearchState<KS>& c, int s, float (&tf)[kP], float (&sq)[kP]) {
  const float INF = __int_as_float(0x7f800000);
  const uint32_t a = c.o_pl + (c.row0 + c.bnd[s]) * kRowW, b = c.o_pl + (c.row0 + c.bnd[s + 1]) * kRowW;
  const float4 la = *reinterpret_cast<const float4*>(c.sm + a);
  const float4 lb = *reinterpret_cast<const float4*>(c.sm + b);
  const float t[kP] = {lb.x - la.x, lb.y - la.y, lb.z - la.z, lb.w - la.w, plf(c.sm, b + 4) - plf(c.sm, a + 4)};
#pragma unroll
  for (int p = 0; p < kP; ++p) {
    const float f = t[p];
    tf[p] = (c.memst[s] <= c.sm[c.o_cap + p] && f <= c.thr) ? f : INF;
    sq[p] = f * f;
  }
}

// ---- unrolled path for KS = 2, 3 ------------------------------------
// All levels are compile-time loops, so the multiplicity m of a profile within the
// sequence is a constant and the free-slice check is folded into variant tables:
// vf[s][m][x] = t (stage s on profile x fits in memory and the node has more than m free
// slices of x) else +INF for the leading stages, and for the last stage the score
// constant ccv[m][x] = (1 - alpha) t^2 under the same condition else -INF (t2 = 2t, 0 for a
// stage that fits no slice).  Per group (S, L = the prefix's sum of stage times and
// alpha * sum t^2, v = the q stage) and its five last-stage profiles p:
//   y_p = fma(S + v, t2_p, ccv_p)        -INF for an inadmissible last stage
//   z   = max_p y_p + ((S+v)^2 - L - alpha v^2)
//                                  sign set <=> no (S+v+t_p)^2 > alpha (sum t^2): no
//                                  candidate of the group can beat the running minimum
//                                  (conservative, §4.3; max is exact and rounding monotone)
//   d2  = (B - vmin) - v           sign set <=> even the fastest admissible last stage
//                                  misses the SLO (exact: integers < 2^25 or INF)
//   acc &= bits(z) | bits(d2)      sign of acc clear <=> some candidate may win
// Five FFMA and two 3-input FMNMX3 per five candidates plus a few group operations.
template <int KS>
struct Tables {
  float vf[KS - 1][KS - 1][kP];  // [stage][multiplicity][profile], +INF folded (stages 0..KS-2)
  float a[KS][kP];               // alpha * t^2   (stages 0..KS-2)
  float t2[kP];                  // last stage: 2t (0 if it fits no slice)
  float ccv[KS][kP];             // last stage: (1 - alpha) t^2 by multiplicity, -INF folded
  float vmin;                    // fastest admissible last stage (>= 1 free slice), else INF
};

template <int KS>
__device__ __forceinline__ void stage_lat(const SearchState<KS>& c, int s, float (&f)[kP]) {
  const uint32_t ra = c.o_pl + (c.row0 + c.bnd[s]) * kRowW, rb = c.o_pl + (c.row0 + c.bnd[s + 1]) * kRowW;
  const float4 la = *reinterpret_cast<const float4*>(c.sm + ra);
  const float4 lb = *reinterpret_cast<const float4*>(c.sm + rb);
  f[0] = lb.x - la.x;
  f[1] = lb.y - la.y;
  f[2] = lb.z - la.z;
  f[3] = lb.w - la.w;
  f[4] = plf(c.sm, rb + 4) - plf(c.sm, ra + 4);
}

template <int KS>
__device__ __forceinline__ void build_tables(const SearchState<KS>& c, Tables<KS>& T) {
  const float INF = __int_as_float(0x7f800000);
  const float one_m_a = 1.f - c.alpha;
  T.vmin = INF;
#pragma unroll
  for (int s = 0; s < KS; ++s) {
    float f[kP];
    stage_lat(c, s, f);
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      const bool mem_ok = c.memst[s] <= c.sm[c.o_cap + x] && f[x] <= c.thr;
      const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
      if (s < KS - 1) {
#pragma unroll
        for (int m = 0; m <= s; ++m) T.vf[s][m][x] = (mem_ok && fr > (uint32_t)m) ? f[x] : INF;
        T.a[s][x] = c.alpha * (f[x] * f[x]);
      } else {
        const float cc = one_m_a * (f[x] * f[x]);
        T.t2[x] = mem_ok ? f[x] + f[x] : 0.f;
#pragma unroll
        for (int m = 0; m <= s; ++m) T.ccv[m][x] = (mem_ok && fr > (uint32_t)m) ? cc : -INF;
        if (mem_ok && fr > 0) T.vmin = fminf(T.vmin, f[x]);
      }
    }
  }
}

// one block = the last two levels (q, p): P*P candidates.  vq selects the q stage's
// variant table and cp the last stage's score constant by compile-time multiplicity;
// Bm = Blim - S - vmin.
template <class VQ, class CP>
__device__ __forceinline__ uint32_t block_qp(const float (&aq)[kP], const float (&t2)[kP], float S, float L,
                                             float Bm, VQ vq, CP cp) {
  uint32_t acc = ~0u;
#pragma unroll
  for (int q = 0; q < kP; ++q) {
    const float v = vq(q);
    const float S3 = S + v;
    const float d2 = Bm - v;
    const float U = fmaf(S3, S3, -(L + aq[q]));
    float y[kP];
#pragma unroll
    for (int p = 0; p < kP; ++p) y[p] = fmaf(S3, t2[p], cp(q, p));
    const float z = fmaxf(fmaxf(fmaxf(y[0], y[1]), y[2]), fmaxf(y[3], y[4])) + U;
    acc &= __float_as_uint(z) | __float_as_uint(d2);
  }
  return (acc >> 31) ^ 1u;  // 1 if some candidate of the block may win
}

// ---- KS = 4, two cut masks per thread in the two fp32 lanes of FFMA2/FADD2 -----------
// Mask A (lane lo) and the next mask B of the same request (lane hi) share every
// control decision (loops, multiplicities) and differ only in data, so one packed
// instruction scores a candidate of each: per candidate pair FFMA2 + FADD2 + FADD2 on
// the FMA pipe and two LOP3 on the ALU pipe.
// stage-0 SLO bound of the KS = 3 / KS = 4 cores; 0 = only the +INF skip (KS = 4)
#ifndef FFS_D0_BOUND
#define FFS_D0_BOUND 1
#endif
typedef unsigned long long f2;
__device__ __forceinline__ f2 f2pack(float lo, float hi) {
  f2 r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
  return r;
}
__device__ __forceinline__ void f2bits(f2 v, uint32_t& lo, uint32_t& hi) {
  asm("mov.b64 {%0, %1}, %2;" : "=r"(lo), "=r"(hi) : "l"(v));
}
__device__ __forceinline__ f2 f2add(f2 a, f2 b) {
  f2 d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ f2 f2sub(f2 a, f2 b) {
  f2 d;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ f2 f2fma(f2 a, f2 b, f2 c) {
  f2 d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}

template <int KS>
struct Geo {
  int bnd[KS + 1];
  uint32_t memst[KS];
  uint32_t X;
  float blim;
};
typedef Geo<4> Geo4;

template <int KS>
__device__ __forceinline__ void geo(const SearchState<KS>& c, uint32_t mask, Geo<KS>& g) {
  g.bnd[0] = 0;
  uint32_t m = mask, X = 0;
#pragma unroll
  for (int i = 0; i < KS - 1; ++i) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    g.bnd[i + 1] = j + 1;
    X += c.sm[c.o_xf + c.row0 + j];
  }
  g.bnd[KS] = c.n;
  g.X = X;
#pragma unroll
  for (int i = 0; i < KS; ++i) g.memst[i] = c.sm[c.o_pm + c.row0 + g.bnd[i + 1]] - c.sm[c.o_pm + c.row0 + g.bnd[i]];
  g.blim = (X <= c.B && !c.none_can_win) ? (float)min(c.B - X, 1u << 24) : -1.f;
}
__device__ __forceinline__ void geo4(const SearchState<4>& c, uint32_t mask, Geo4& g) { geo<4>(c, mask, g); }

template <int KS>
__device__ __forceinline__ void geo_lat(const SearchState<KS>& c, const Geo<KS>& g, int s, float (&f)[kP]) {
  const uint32_t ra = c.o_pl + (c.row0 + g.bnd[s]) * kRowW, rb = c.o_pl + (c.row0 + g.bnd[s + 1]) * kRowW;
  const float4 la = *reinterpret_cast<const float4*>(c.sm + ra);
  const float4 lb = *reinterpret_cast<const float4*>(c.sm + rb);
  f[0] = lb.x - la.x;
  f[1] = lb.y - la.y;
  f[2] = lb.z - la.z;
  f[3] = lb.w - la.w;
  f[4] = plf(c.sm, rb + 4) - plf(c.sm, ra + 4);
}

// Copy half h's geometry into the state and run the exact path over the flagged blocks.
template <int KS, bool VERIFY>
__device__ __forceinline__ void pair_rescan(SearchState<KS>& c, const Geo<KS>& G, uint32_t pend, uint32_t all,
                                            uint64_t idx_shift, unsigned long long* misses) {
  constexpr uint32_t kAll = (1u << (kP * kP)) - 1;
#pragma unroll
  for (int i = 0; i <= KS; ++i) c.bnd[i] = G.bnd[i];
#pragma unroll
  for (int i = 0; i < KS; ++i) c.memst[i] = G.memst[i];
  c.X = G.X;
  c.idx_base += idx_shift;
  for (uint32_t todo = all; todo;) {
    const int b = __ffs(todo) - 1;
    todo &= todo - 1;
    if constexpr (KS == 3) c.pd[0] = b;
    if constexpr (KS == 4) {
      c.pd[0] = b / kP;
      c.pd[1] = b - kP * (b / kP);
    }
    const uint32_t fast = ((pend >> b) & 1u) ? kAll : 0u;
    handle_hits<KS, VERIFY>(c, kAll, fast, misses);
  }
  c.idx_base -= idx_shift;
}

// KS = 3, two consecutive masks per thread in f32x2 lanes, every level unrolled (125
// candidates per mask, ~8 KB of SASS) and every table in registers.  Per group (d0, q)
// the group maximum of §4.3: y_p = fma(S2, 2t_p, ccw_p) (ccw = -INF for an inadmissible
// last stage), z = max_p y_p + U, and one exact SLO test against the fastest admissible
// last stage (blim - v2min - S2, integers < 2^25).
template <bool VERIFY>
__device__ __forceinline__ void ks3_pair(SearchState<3>& c, uint32_t maskA, uint32_t maskB, bool haveB,
                                         unsigned long long* misses, bool exh, uint64_t shiftB,
                                         uint32_t* defer = nullptr) {
  const float INF = __int_as_float(0x7f800000);
  Geo<3> G[2];
  geo<3>(c, maskA, G[0]);
  geo<3>(c, maskB, G[1]);
  if (!haveB) G[1].blim = -1.f;
  const float al = c.alpha, one_m_a = 1.f - c.alpha;
  f2 v0[kP], v1[2][kP], ccw[3][kP], na0[kP], a1[kP], t2[kP], slm;
  {
    float f[2][3][kP], vmin[2] = {INF, INF};
#pragma unroll
    for (int h = 0; h < 2; ++h)
#pragma unroll
      for (int s = 0; s < 3; ++s) geo_lat<3>(c, G[h], s, f[h][s]);
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
      const uint32_t cap = c.sm[c.o_cap + x];
      float v[2][2][2], cw[2][3], tw[2];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
#pragma unroll
        for (int s = 0; s < 2; ++s)
#pragma unroll
          for (int m = 0; m <= s; ++m)
            v[h][s][m] = (G[h].memst[s] <= cap && f[h][s][x] <= c.thr && fr > (uint32_t)m) ? f[h][s][x] : INF;
        const bool ad = G[h].memst[2] <= cap && f[h][2][x] <= c.thr;  // the last stage fits x
        const float ccx = one_m_a * (f[h][2][x] * f[h][2][x]);
        tw[h] = ad ? f[h][2][x] + f[h][2][x] : 0.f;
#pragma unroll
        for (int m = 0; m < 3; ++m) cw[h][m] = (ad && fr > (uint32_t)m) ? ccx : -INF;
        if (ad && fr > 0) vmin[h] = fminf(vmin[h], f[h][2][x]);
      }
      v0[x] = f2pack(v[0][0][0], v[1][0][0]);
      v1[0][x] = f2pack(v[0][1][0], v[1][1][0]);
      v1[1][x] = f2pack(v[0][1][1], v[1][1][1]);
#pragma unroll
      for (int m = 0; m < 3; ++m) ccw[m][x] = f2pack(cw[0][m], cw[1][m]);
      na0[x] = f2pack(-al * (f[0][0][x] * f[0][0][x]), -al * (f[1][0][x] * f[1][0][x]));
      a1[x] = f2pack(al * (f[0][1][x] * f[0][1][x]), al * (f[1][1][x] * f[1][1][x]));
      t2[x] = f2pack(tw[0], tw[1]);
    }
    slm = f2pack(G[0].blim - vmin[0], G[1].blim - vmin[1]);  // exact (integers < 2^25 or -INF)
  }
  // fastest admissible stage 1 per half (the unshifted window; a shifted entry is the same
  // value or +INF), for the stage-0 bound below
  float v1lo = INF, v1hi = INF;
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    uint32_t l, h;
    f2bits(v1[0][x], l, h);
    v1lo = fminf(v1lo, __uint_as_float(l));
    v1hi = fminf(v1hi, __uint_as_float(h));
  }
  const f2 v1min = f2pack(v1lo, v1hi);
  uint32_t pendA = 0, pendB = 0;
#pragma unroll
  for (int d0 = 0; d0 < kP; ++d0) {
    const f2 S1 = v0[d0], NL1 = na0[d0];
#if FFS_D0_BOUND
    {  // stage-0 bound: every group has S2 >= S1 + v1min (monotone fp32
       // rounding) and its SLO test d2 = slm - S2 is monotone in S2, so when slm -
       // (S1 + v1min) < 0 in every live half the iteration can flag nothing
      uint32_t bl, bh;
      f2bits(f2sub(slm, f2add(S1, v1min)), bl, bh);
      if (!exh && (bl >> 31) && (!haveB || (bh >> 31))) continue;
    }
#endif
    c.n_scored += haveB ? 2 * kP * kP : kP * kP;  // 25 candidates per mask of this d0
    uint32_t accA = ~0u, accB = ~0u;
#pragma unroll
    for (int q = 0; q < kP; ++q) {
      const f2 S2 = f2add(S1, v1[q == d0][q]);
      const f2 U = f2fma(S2, S2, f2sub(NL1, a1[q]));
      float ylo[kP], yhi[kP];
#pragma unroll
      for (int p = 0; p < kP; ++p) {
        uint32_t l, h;
        f2bits(f2fma(S2, t2[p], ccw[(p == d0) + (p == q)][p]), l, h);
        ylo[p] = __uint_as_float(l);
        yhi[p] = __uint_as_float(h);
      }
      const float mlo = fmaxf(fmaxf(fmaxf(ylo[0], ylo[1]), ylo[2]), fmaxf(ylo[3], ylo[4]));
      const float mhi = fmaxf(fmaxf(fmaxf(yhi[0], yhi[1]), yhi[2]), fmaxf(yhi[3], yhi[4]));
      const f2 z = f2add(f2pack(mlo, mhi), U);
      const f2 d2 = f2sub(slm, S2);  // sign set <=> S2 + v2min > blim: no candidate meets the SLO
      uint32_t zl, zh, dl, dh;
      f2bits(z, zl, zh);
      f2bits(d2, dl, dh);
      accA &= zl | dl;
      accB &= zh | dh;
    }
    pendA |= ((accA >> 31) ^ 1u) << d0;
    pendB |= ((accB >> 31) ^ 1u) << d0;
  }
  constexpr uint32_t kAllB = (1u << kP) - 1;
  if (!VERIFY && defer) {  // the caller rescans the flagged blocks warp-cooperatively
    defer[0] = pendA;
    defer[1] = haveB ? pendB : 0u;
    return;
  }
  pair_rescan<3, VERIFY>(c, G[0], pendA, VERIFY ? kAllB : pendA, 0, misses);
  if (haveB) pair_rescan<3, VERIFY>(c, G[1], pendB, VERIFY ? kAllB : pendB, shiftB, misses);
}

// ---- KS = 4, f16x2 pre-filter ---------------------------------------
// The same candidate-pair core in packed half precision: mask A in the low and mask B in
// the high f16 of one 32-bit register, so one HFMA2/HADD2 scores a candidate of each and
// one LOP3 folds both sign bits (4 instructions per candidate pair instead of 3 f32x2 +
// 2 LOP3).  Each half is scaled by its own power of two sigma (exact) so that every
// feasible candidate's T sigma <= 32: no overflow (T^2, alpha Sigma t^2 < 2^13) and, with
// T sigma >= 1/8 checked per half, negligible underflow.  The filter is conservative by
// construction: alpha_h (set_threshold) leaves a 2^-6 (KS + 1 + alpha') Sigma t^2 margin
// for the f16 rounding and the SLO slack is widened by 2^-7 Blim; a block with a possible
// winner is always flagged, flagged blocks are re-evaluated exactly (pair_rescan), so the
// pre-filter decides only how much exact work runs, never a result.
typedef uint32_t h2;
__device__ __forceinline__ h2 h2pack(float lo, float hi) {
  h2 r;
  asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ h2 h2add(h2 a, h2 b) {
  h2 d;
  asm("add.rn.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
__device__ __forceinline__ h2 h2mul(h2 a, h2 b) {
  h2 d;
  asm("mul.rn.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
__device__ __forceinline__ h2 h2sub(h2 a, h2 b) {
  h2 d;
  asm("sub.rn.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
__device__ __forceinline__ h2 h2fma(h2 a, h2 b, h2 c) {
  h2 d;
  asm("fma.rn.f16x2 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}
// IEEE maxNum per half (a NaN operand loses); ptxas fuses pairs into 3-input VHMNMX
__device__ __forceinline__ h2 h2max(h2 a, h2 b) {
  h2 d;
  asm("max.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}

__device__ __forceinline__ h2 h2min(h2 a, h2 b) {
  h2 d;
  asm("min.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}

// SLO slack in "guarded" form for the integer SWAR test of the inner loop: per f16 half,
// bit 15 (guard) | the magnitude bits of slack - v3 when it is >= 0, else the guard alone
// (magnitude 0).  For S3 >= 0 (a sum of non-negative f16, never NaN), the 32-bit integer
// difference guarded - bits(S3) keeps the halves apart (every half's minuend >= 2^15 >
// S3's bits) and its bit 15 / 31 is set iff slack - v3 >= S3 in f16: the same decision as
// the sign of an f16 subtraction, moved from the FMA pipe to one IADD3 on the ALU pipe.
__device__ __forceinline__ uint32_t h2guard(h2 w) {
  const uint32_t neg = w & 0x80008000u;
  const uint32_t m = neg - (neg >> 15);  // 0x7fff in every half whose sign bit is set
  return (w & ~m) | 0x80008000u;
}

// a - b + zero with an opaque zero register: a three-operand add, which only IADD3 (ALU
// pipe) encodes, so ptxas cannot move the test to an IMAD.IADD on the busier FMA pipe
__device__ __forceinline__ uint32_t isub(uint32_t a, uint32_t b, uint32_t zero) {
  uint32_t d;
  asm("{.reg .u32 t; sub.u32 t, %1, %2; add.u32 %0, t, %3;}" : "=r"(d) : "r"(a), "r"(b), "r"(zero));
  return d;
}

struct WinH {
  h2 s1, s2[2], c3[3];
};

// Per-thread shared-memory windows of the KS = 4 kernel, [slot][thread] (4-byte,
// conflict-free, immediate offsets: the stride is the compile-time CTA size): x * 11 + k,
// x = profile, k = 0-1 s1 (stage 1 gated by > 0 / > 1 free slices), 2-4 s2 (> 0, > 1, > 2),
// 5-8 cc3 (> 0 .. > 3), 9 v0 (> 0), 10 -alpha t0^2; window e (e = 1 when x is the stage-0
// profile: every multiplicity shifted by one) is read at offset e.  (A per-thread cache of
// the stage-2/3 tables across the masks of a row measured 4 % slower: SIMT rebuilds it
// whenever any lane of the warp leaves its row.)

__device__ __forceinline__ void ks4_cuts(uint32_t m, int& j1, int& j2, int& j3) {
  j1 = __ffs(m) - 1;
  m &= m - 1;
  j2 = __ffs(m) - 1;
  m &= m - 1;
  j3 = __ffs(m) - 1;
}

template <bool VERIFY>
__device__ __forceinline__ void ks4_pair_h(SearchState<4>& c, uint32_t maskA, uint32_t maskB, bool haveB, h2* rows,
                                           unsigned long long* misses, uint32_t zero, bool exh, uint64_t shiftB,
                                           uint32_t* defer = nullptr) {
  const float INF = __int_as_float(0x7f800000);
  constexpr int nb = search_block(4);  // slot stride: the CTA size, fixed at compile time
  h2* slot = rows + threadIdx.x;
  constexpr h2 kInf2 = 0x7c007c00u, kNegInf2 = 0xfc00fc00u, kGuard = 0x80008000u;
  const float al = c.alpha_h, one_m_a = 1.f - c.alpha_h;
  const h2 al2 = h2pack(al, al), nal2 = h2pack(-al, -al), oma2 = h2pack(one_m_a, one_m_a);
  const uint32_t* PL = c.sm + c.o_pl + c.row0 * kRowW;  // prefix rows of the request's chain
  const uint32_t* PM = c.sm + c.o_pm + c.row0;
  const uint32_t* XF = c.sm + c.o_xf + c.row0;          // XF[j]: cut after component j
  // per half: the stage times of its four stages from the five prefix rows 0 (= 0), b1,
  // b2, b3, n (shared by adjacent stages), the stage memories, the budget
  float f[2][4][kP], sig[2], slack[2];
  uint32_t ms[2][4];
  bool wide[2];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    int j1, j2, j3;
    ks4_cuts(h ? maskB : maskA, j1, j2, j3);
    const uint32_t b[5] = {0u, (uint32_t)j1 + 1, (uint32_t)j2 + 1, (uint32_t)j3 + 1, c.n};
    float pr[5][kP];
#pragma unroll
    for (int i = 0; i < 5; ++i) {
      if (i == 0) {
#pragma unroll
        for (int x = 0; x < kP; ++x) pr[0][x] = 0.f;
        continue;
      }
      const float4 l = *reinterpret_cast<const float4*>(PL + b[i] * kRowW);
      pr[i][0] = l.x;
      pr[i][1] = l.y;
      pr[i][2] = l.z;
      pr[i][3] = l.w;
      pr[i][4] = __uint_as_float(PL[b[i] * kRowW + 4]);
    }
#pragma unroll
    for (int s = 0; s < 4; ++s) {
#pragma unroll
      for (int x = 0; x < kP; ++x) f[h][s][x] = pr[s + 1][x] - pr[s][x];
      ms[h][s] = PM[b[s + 1]] - PM[b[s]];
    }
    const uint32_t X = XF[j1] + XF[j2] + XF[j3];
    const bool live_h = h == 0 || haveB;  // the B half of a single mask is a dummy: nothing passes
    const float bl = (live_h && X <= c.B && !c.none_can_win) ? (float)min(c.B - X, 1u << 24) : -1.f;
    // scale sigma = 2^(5 - E) with M = min(Blim, tmax) <= 2^E, so every feasible candidate
    // (T <= M) has T sigma <= 32; the SLO slack is M sigma (1 + 2^-7) (clamping Blim to tmax
    // changes no candidate's SLO outcome: T <= tmax always)
    const float M = fmaxf(fminf(bl, c.tmax), 1.f);
    const uint32_t mb = __float_as_uint(M);
    const int E = (int)((mb >> 23) & 255u) - 127 + ((mb & 0x7fffffu) != 0u);  // M <= 2^E
    sig[h] = __int_as_float((127 + 5 - E) << 23);
    wide[h] = bl >= 0.f && c.tmin * sig[h] < 0.125f;  // f16 underflow could matter: exact path
    slack[h] = bl >= 0.f ? M * sig[h] * (1.f + 1.f / 128.f) : -INF;
  }
  // the scaled stage times with memory and the throughput floor (R38) folded: +INF where
  // the stage does not fit the profile; a function without a floor (the common case) skips
  // the floor compare (uniform per request)
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t cap = c.sm[c.o_cap + x];
    if (c.thr_u == 0xffffffffu) {
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int s = 0; s < 4; ++s) f[h][s][x] = ms[h][s] <= cap ? f[h][s][x] * sig[h] : INF;
    } else {
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int s = 0; s < 4; ++s)
          f[h][s][x] = (ms[h][s] <= cap && f[h][s][x] <= c.thr) ? f[h][s][x] * sig[h] : INF;
    }
  }
  // the packed stage tables and the per-half minima the stage-0 bound needs
  h2 P0[kP], P1[kP], P2[kP], P3[kP];
  float v3m[2] = {INF, INF};  // fastest admissible last stage per half (>= 1 free slice)
  h2 v1min = kInf2, v2min = kInf2;
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
    float vm[2][4];
#pragma unroll
    for (int h = 0; h < 2; ++h)
#pragma unroll
      for (int s = 0; s < 4; ++s) vm[h][s] = f[h][s][x];
    P0[x] = h2pack(vm[0][0], vm[1][0]);
    P1[x] = h2pack(vm[0][1], vm[1][1]);
    P2[x] = h2pack(vm[0][2], vm[1][2]);
    // a last stage longer than the (widened) SLO slack on its own is inadmissible too: no
    // candidate holding it is feasible, and the bound keeps t3 and t3^2 far from overflow
    // (an admissible t3 sigma <= slack < 33 never packs to the f16 INF pattern)
    const float u0 = vm[0][3] <= slack[0] ? vm[0][3] : INF, u1 = vm[1][3] <= slack[1] ? vm[1][3] : INF;
    P3[x] = h2pack(u0, u1);
    if (fr > 0) {
      v3m[0] = fminf(v3m[0], u0);
      v3m[1] = fminf(v3m[1], u1);
      if (!exh) {  // only the stage-0 bound needs them
        v1min = h2min(v1min, P1[x]);
        v2min = h2min(v2min, P2[x]);
      }
    }
  }
  // guarded SLO slack of the fastest admissible last stage (h2guard): S3 <= slack - v3min
  const uint32_t slk = h2guard(h2pack(slack[0] - v3m[0], slack[1] - v3m[1]));
  // d0 bound: every group of stage-0 iteration d0 has S3 = (S1 + w1) + w2 >= (S1 + v1min)
  // + v2min (f16 addition rounds monotonically, and a window entry is its profile's value
  // or +INF), and the group SLO test is monotone in S3, so when the bound already fails it
  // in every live half the iteration can flag nothing: it is skipped.  This covers a
  // stage-0 profile with no free slice on the node (S1 = +INF) and stage-0 prefixes that
  // leave too little budget.
  uint32_t live = (1u << kP) - 1;  // exhaustive mode: every stage-0 iteration is scored
  if (!exh) {  // (uniform: a kernel argument)
    live = 0;
#pragma unroll
    for (int d0 = 0; d0 < kP; ++d0) {
      const h2 S1 = ((c.freeb >> (8 * d0)) & 255u) ? P0[d0] : kInf2;
      const uint32_t okb = isub(slk, h2add(h2add(S1, v1min), v2min), zero);
      const bool on = (okb & 0x8000u) || (haveB && (okb & 0x80000000u));
      live |= (on ? 1u : 0u) << d0;
    }
  }
  uint32_t pendA = 0, pendB = 0;
  // no live iteration (the common case in bounded mode): nothing else to set up
  if (VERIFY || live != 0) {
    // the per-thread windows and the register tables of the scoring core
    h2 a1[kP], a2[kP], t2[kP];
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
      const h2 p0 = P0[x], p1 = P1[x], p2 = P2[x], p3 = P3[x];
      a1[x] = h2mul(h2mul(p1, p1), al2);
      a2[x] = h2mul(h2mul(p2, p2), al2);
      // last stage as (2 t3, (1 - alpha_h) t3^2); an inadmissible one (INF) as (0, -INF), so
      // its score y = S3 * 2t3 + cc is -INF for every finite S3 (no INF * 0, no INF - INF)
      const uint32_t inf3 = ((p3 & 0xffffu) == 0x7c00u ? 0x0000ffffu : 0u) | ((p3 >> 16) == 0x7c00u ? 0xffff0000u : 0u);
      t2[x] = h2add(p3, p3) & ~inf3;
      const h2 cc = (h2mul(h2mul(p3, p3), oma2) & ~inf3) | (kNegInf2 & inf3);
      h2* r = slot + (x * 11) * nb;
      r[0 * nb] = fr > 0 ? p1 : kInf2;
      r[1 * nb] = fr > 1 ? p1 : kInf2;
      r[2 * nb] = fr > 0 ? p2 : kInf2;
      r[3 * nb] = fr > 1 ? p2 : kInf2;
      r[4 * nb] = fr > 2 ? p2 : kInf2;
      r[5 * nb] = fr > 0 ? cc : kNegInf2;
      r[6 * nb] = fr > 1 ? cc : kNegInf2;
      r[7 * nb] = fr > 2 ? cc : kNegInf2;
      r[8 * nb] = fr > 3 ? cc : kNegInf2;
      r[9 * nb] = fr > 0 ? p0 : kInf2;
      r[10 * nb] = h2mul(h2mul(p0, p0), nal2);
    }
    // each lane walks its own live stage-0 profiles: a warp runs max(popcount) iterations,
    // not the union of its lanes' sets (records of the bounded list mode differ per lane)
#pragma unroll 1
    for (uint32_t todo = live; todo; todo &= todo - 1) {
      const int d0 = __ffs(todo) - 1;
      const h2 S1 = slot[(d0 * 11 + 9) * nb];
      c.n_scored += haveB ? 250 : 125;  // 125 candidates per mask of this d0, each y_p computed
      WinH W[kP];
      const h2* shifted = slot + nb;  // the d0 profile's windows are read one slot later
#pragma unroll
      for (int x = 0; x < kP; ++x) {
        const h2* r = (x == d0 ? shifted : slot) + x * 11 * nb;  // a select + immediate offsets
        W[x].s1 = r[0];
        W[x].s2[0] = r[2 * nb];
        W[x].s2[1] = r[3 * nb];
        W[x].c3[0] = r[5 * nb];
        W[x].c3[1] = r[6 * nb];
        W[x].c3[2] = r[7 * nb];
      }
      const h2 NL1 = slot[(d0 * 11 + 10) * nb];  // -alpha t0^2
      uint32_t mm[kP];  // per d1: sign bits 15 / 31 clear <=> the (d0, d1) block may hold a winner
#pragma unroll
      for (int d1 = 0; d1 < kP; ++d1) {
        const h2 S2 = h2add(S1, W[d1].s1), NL2 = h2sub(NL1, a1[d1]);
        uint32_t acc = ~0u;
#pragma unroll
        for (int q = 0; q < kP; ++q) {
          const h2 S3 = h2add(S2, W[q].s2[q == d1]);
          const h2 U = h2fma(S3, S3, h2sub(NL2, a2[q]));
          // y_p = S3 * 2t3 + (1 - alpha_h) t3^2 (-INF for an inadmissible last stage); the
          // group's best z = max_p y_p + U (rounding is monotone: the same decision as testing
          // every candidate's own z), two 3-input packed maxima (VHMNMX) per 5 candidates
          h2 y[kP];
#pragma unroll
          for (int p = 0; p < kP; ++p) y[p] = h2fma(S3, t2[p], W[p].c3[(p == d1) + (p == q)]);
          const h2 z = h2add(h2max(h2max(h2max(y[0], y[1]), y[2]), h2max(y[3], y[4])), U);
          // group SLO test: bit 15/31 clear <=> S3 + (fastest admissible t3) > slack
          const uint32_t ok = isub(slk, S3, zero);
          acc &= z | ~ok;  // one 3-input LOP3 per group
        }
        mm[d1] = acc;
      }
      // flagged blocks are rare: the per-block bookkeeping runs only when some block is
      if ((mm[0] & mm[1] & mm[2] & mm[3] & mm[4] & kGuard) != kGuard) {
        uint32_t bA = 0, bB = 0;
#pragma unroll
        for (int d1 = 0; d1 < kP; ++d1) {
          bA |= ((mm[d1] >> 15) & 1u) << d1;
          bB |= (mm[d1] >> 31) << d1;
        }
        pendA |= (bA ^ 31u) << (kP * d0);
        pendB |= (bB ^ 31u) << (kP * d0);
      }
    }
  }
  constexpr uint32_t kAll = (1u << (kP * kP)) - 1;
  if (wide[0]) pendA = kAll;  // dynamic range too wide for f16: every block exactly
  if (wide[1]) pendB = kAll;
  if (!VERIFY && defer) {  // the caller rescans the flagged blocks warp-cooperatively
    defer[0] = pendA;
    defer[1] = haveB ? pendB : 0u;
    return;
  }
  if (VERIFY || pendA) {
    Geo4 G;
    geo4(c, maskA, G);
    pair_rescan<4, VERIFY>(c, G, pendA, VERIFY ? kAll : pendA, 0, misses);
  }
  if (haveB && (VERIFY || pendB)) {
    Geo4 G;
    geo4(c, maskB, G);
    pair_rescan<4, VERIFY>(c, G, pendB, VERIFY ? kAll : pendB, shiftB, misses);
  }
}

// ---- KS = 4 over requests grouped by chain length (exhaustive / verify) ----------------
// The warp's lanes hold 32 requests with the same n and walk the same masks in lockstep, so
// a pair's two highest cuts (its "row": stages 2 and 3) change for all lanes at once, at
// row boundaries: the stage-2/3 half of ks4_pair_h's setup (prefix rows, memory / floor
// fold, scaled packing, the s2 / c3 windows, a2, t2) runs once per row pair instead of once
// per mask pair.  Scale sigma and the last stage's admissibility are taken per row (from
// B - X(j2, j3) >= B - X(mask)): sigma is no larger and the admissibility test no
// stricter than per mask, so the filter stays conservative; the group SLO test keeps the
// mask's own slack.  The core (stage-0 loop) is ks4_pair_h's.
struct Row4 {
  uint32_t keyA, keyB;  // rows (mask & (mask - 1)) the state was built for; ~0u = none
  uint32_t Xr[2];       // transfer cost of the two highest cuts per half
  float sig[2], v3m[2];
  bool wide[2];
  h2 a2[kP], t2[kP];
};

template <bool VERIFY>
__device__ __forceinline__ void ks4_pair_rows(SearchState<4>& c, Row4& R, uint32_t maskA, uint32_t maskB, bool haveB,
                                              bool lane_live, h2* rows, unsigned long long* misses, uint32_t zero,
                                              uint64_t shiftB, uint32_t* defer) {
  const float INF = __int_as_float(0x7f800000);
  constexpr int nb = search_block(4);
  h2* slot = rows + threadIdx.x;
  constexpr h2 kInf2 = 0x7c007c00u, kNegInf2 = 0xfc00fc00u, kGuard = 0x80008000u;
  const float al = c.alpha_h, one_m_a = 1.f - c.alpha_h;
  const h2 al2 = h2pack(al, al), nal2 = h2pack(-al, -al), oma2 = h2pack(one_m_a, one_m_a);
  const uint32_t* PL = c.sm + c.o_pl + c.row0 * kRowW;
  const uint32_t* PM = c.sm + c.o_pm + c.row0;
  const uint32_t* XF = c.sm + c.o_xf + c.row0;
  const uint32_t kA = maskA & (maskA - 1), kB = maskB & (maskB - 1);
  if (kA != R.keyA || kB != R.keyB) {  // warp-uniform (the lanes walk the same masks)
    R.keyA = kA;
    R.keyB = kB;
    float f[2][2][kP], slr[2];
    uint32_t ms[2][2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      uint32_t m = h ? kB : kA;
      const int j2 = __ffs(m) - 1;
      m &= m - 1;
      const int j3 = __ffs(m) - 1;
      const uint32_t b[3] = {(uint32_t)j2 + 1, (uint32_t)j3 + 1, c.n};
      float pr[3][kP];
#pragma unroll
      for (int i = 0; i < 3; ++i) {
        const float4 l = *reinterpret_cast<const float4*>(PL + b[i] * kRowW);
        pr[i][0] = l.x;
        pr[i][1] = l.y;
        pr[i][2] = l.z;
        pr[i][3] = l.w;
        pr[i][4] = __uint_as_float(PL[b[i] * kRowW + 4]);
      }
#pragma unroll
      for (int s = 0; s < 2; ++s) {
#pragma unroll
        for (int x = 0; x < kP; ++x) f[h][s][x] = pr[s + 1][x] - pr[s][x];
        ms[h][s] = PM[b[s + 1]] - PM[b[s]];
      }
      R.Xr[h] = XF[j2] + XF[j3];
      const float bl = (lane_live && R.Xr[h] <= c.B && !c.none_can_win) ? (float)min(c.B - R.Xr[h], 1u << 24) : -1.f;
      const float M = fmaxf(fminf(bl, c.tmax), 1.f);
      const uint32_t mb = __float_as_uint(M);
      const int E = (int)((mb >> 23) & 255u) - 127 + ((mb & 0x7fffffu) != 0u);  // M <= 2^E
      R.sig[h] = __int_as_float((127 + 5 - E) << 23);
      R.wide[h] = bl >= 0.f && c.tmin * R.sig[h] < 0.125f;
      slr[h] = bl >= 0.f ? M * R.sig[h] * (1.f + 1.f / 128.f) : -INF;
    }
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      const uint32_t cap = c.sm[c.o_cap + x];
      if (c.thr_u == 0xffffffffu) {
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
          for (int s = 0; s < 2; ++s) f[h][s][x] = ms[h][s] <= cap ? f[h][s][x] * R.sig[h] : INF;
      } else {
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
          for (int s = 0; s < 2; ++s)
            f[h][s][x] = (ms[h][s] <= cap && f[h][s][x] <= c.thr) ? f[h][s][x] * R.sig[h] : INF;
      }
    }
    R.v3m[0] = INF;
    R.v3m[1] = INF;
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
      const h2 p2 = h2pack(f[0][0][x], f[1][0][x]);
      const float u0 = f[0][1][x] <= slr[0] ? f[0][1][x] : INF, u1 = f[1][1][x] <= slr[1] ? f[1][1][x] : INF;
      const h2 p3 = h2pack(u0, u1);
      if (fr > 0) {
        R.v3m[0] = fminf(R.v3m[0], u0);
        R.v3m[1] = fminf(R.v3m[1], u1);
      }
      R.a2[x] = h2mul(h2mul(p2, p2), al2);
      const uint32_t inf3 = ((p3 & 0xffffu) == 0x7c00u ? 0x0000ffffu : 0u) | ((p3 >> 16) == 0x7c00u ? 0xffff0000u : 0u);
      R.t2[x] = h2add(p3, p3) & ~inf3;
      const h2 cc = (h2mul(h2mul(p3, p3), oma2) & ~inf3) | (kNegInf2 & inf3);
      h2* r = slot + (x * 11) * nb;
      r[2 * nb] = fr > 0 ? p2 : kInf2;
      r[3 * nb] = fr > 1 ? p2 : kInf2;
      r[4 * nb] = fr > 2 ? p2 : kInf2;
      r[5 * nb] = fr > 0 ? cc : kNegInf2;
      r[6 * nb] = fr > 1 ? cc : kNegInf2;
      r[7 * nb] = fr > 2 ? cc : kNegInf2;
      r[8 * nb] = fr > 3 ? cc : kNegInf2;
    }
  }
  // per mask pair: stages 0 and 1, the mask's own SLO slack
  float f[2][2][kP], sl[2];
  uint32_t ms[2][2];
  bool wide[2];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    uint32_t m = h ? maskB : maskA;
    const int j1 = __ffs(m) - 1;
    m &= m - 1;
    const int j2 = __ffs(m) - 1;
    const uint32_t b1 = (uint32_t)j1 + 1, b2 = (uint32_t)j2 + 1;
    const float4 l1 = *reinterpret_cast<const float4*>(PL + b1 * kRowW);
    const float4 l2 = *reinterpret_cast<const float4*>(PL + b2 * kRowW);
    const float p1[kP] = {l1.x, l1.y, l1.z, l1.w, __uint_as_float(PL[b1 * kRowW + 4])};
    const float p2[kP] = {l2.x, l2.y, l2.z, l2.w, __uint_as_float(PL[b2 * kRowW + 4])};
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      f[h][0][x] = p1[x];  // prefix row 0 is zero
      f[h][1][x] = p2[x] - p1[x];
    }
    ms[h][0] = PM[b1] - PM[0];
    ms[h][1] = PM[b2] - PM[b1];
    const uint32_t X = XF[j1] + R.Xr[h];
    const bool live_h = lane_live && (h == 0 || haveB);  // a single mask's B half is a dummy
    const float bl = (live_h && X <= c.B && !c.none_can_win) ? (float)min(c.B - X, 1u << 24) : -1.f;
    const float M = fmaxf(fminf(bl, c.tmax), 1.f);
    sl[h] = bl >= 0.f ? M * R.sig[h] * (1.f + 1.f / 128.f) - R.v3m[h] : -INF;
    wide[h] = bl >= 0.f && R.wide[h];
  }
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t cap = c.sm[c.o_cap + x];
    if (c.thr_u == 0xffffffffu) {  // no throughput floor (the common case; uniform per request)
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int s = 0; s < 2; ++s) f[h][s][x] = ms[h][s] <= cap ? f[h][s][x] * R.sig[h] : INF;
    } else {
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int s = 0; s < 2; ++s)
          f[h][s][x] = (ms[h][s] <= cap && f[h][s][x] <= c.thr) ? f[h][s][x] * R.sig[h] : INF;
    }
  }
  h2 a1[kP];
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
    const h2 p0 = h2pack(f[0][0][x], f[1][0][x]), p1 = h2pack(f[0][1][x], f[1][1][x]);
    a1[x] = h2mul(h2mul(p1, p1), al2);
    h2* r = slot + (x * 11) * nb;
    r[0 * nb] = fr > 0 ? p1 : kInf2;
    r[1 * nb] = fr > 1 ? p1 : kInf2;
    r[9 * nb] = fr > 0 ? p0 : kInf2;
    r[10 * nb] = h2mul(h2mul(p0, p0), nal2);
  }
  const uint32_t slk = h2guard(h2pack(sl[0], sl[1]));
  uint32_t pendA = 0, pendB = 0;
#pragma unroll 1
  for (int d0 = 0; d0 < kP; ++d0) {  // every stage-0 profile (exhaustive / verify)
    const h2 S1 = slot[(d0 * 11 + 9) * nb];
    if (lane_live) c.n_scored += haveB ? 250 : 125;  // 125 candidates per mask of this d0, each y_p computed
    WinH W[kP];
    const h2* shifted = slot + nb;  // the d0 profile's windows are read one slot later
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      const h2* r = (x == d0 ? shifted : slot) + x * 11 * nb;  // a select + immediate offsets
      W[x].s1 = r[0];
      W[x].s2[0] = r[2 * nb];
      W[x].s2[1] = r[3 * nb];
      W[x].c3[0] = r[5 * nb];
      W[x].c3[1] = r[6 * nb];
      W[x].c3[2] = r[7 * nb];
    }
    const h2 NL1 = slot[(d0 * 11 + 10) * nb];  // -alpha t0^2
    uint32_t mm[kP];
#pragma unroll
    for (int d1 = 0; d1 < kP; ++d1) {
      const h2 S2 = h2add(S1, W[d1].s1), NL2 = h2sub(NL1, a1[d1]);
      uint32_t acc = ~0u;
#pragma unroll
      for (int q = 0; q < kP; ++q) {
        const h2 S3 = h2add(S2, W[q].s2[q == d1]);
        const h2 U = h2fma(S3, S3, h2sub(NL2, R.a2[q]));
        h2 y[kP];
#pragma unroll
        for (int p = 0; p < kP; ++p) y[p] = h2fma(S3, R.t2[p], W[p].c3[(p == d1) + (p == q)]);
        const h2 z = h2add(h2max(h2max(h2max(y[0], y[1]), y[2]), h2max(y[3], y[4])), U);
        const uint32_t ok = isub(slk, S3, zero);
        acc &= z | ~ok;
      }
      mm[d1] = acc;
    }
    if ((mm[0] & mm[1] & mm[2] & mm[3] & mm[4] & kGuard) != kGuard) {
      uint32_t bA = 0, bB = 0;
#pragma unroll
      for (int d1 = 0; d1 < kP; ++d1) {
        bA |= ((mm[d1] >> 15) & 1u) << d1;
        bB |= (mm[d1] >> 31) << d1;
      }
      pendA |= (bA ^ 31u) << (kP * d0);
      pendB |= (bB ^ 31u) << (kP * d0);
    }
  }
  constexpr uint32_t kAll = (1u << (kP * kP)) - 1;
  if (wide[0]) pendA = kAll;  // dynamic range too wide for f16: every block exactly
  if (wide[1]) pendB = kAll;
  if (!VERIFY && defer) {  // the caller rescans the flagged blocks warp-cooperatively
    defer[0] = lane_live ? pendA : 0u;
    defer[1] = (lane_live && haveB) ? pendB : 0u;
    return;
  }
  if (!lane_live) return;
  if (VERIFY || pendA) {
    Geo4 G;
    geo4(c, maskA, G);
    pair_rescan<4, VERIFY>(c, G, pendA, VERIFY ? kAll : pendA, 0, misses);
  }
  if (haveB && (VERIFY || pendB)) {
    Geo4 G;
    geo4(c, maskB, G);
    pair_rescan<4, VERIFY>(c, G, pendB, VERIFY ? kAll : pendB, shiftB, misses);
  }
}

// ---- KS = 3, f16x2 pre-filter ---------------------------------------------------------
// ks4_pair_h with one stage fewer: masks A / B in the low / high f16 halves, each half
// scaled by its own power of two sigma, memory / floor / an over-long last stage folded in
// as +INF, group maximum over the last stage (p) per (d0, q): 13 instructions per 10
// candidates.  Every table fits in registers (no windows in shared memory): stage 1 by
// multiplicity {> 0, > 1}, the last stage's cc by {> 0, > 1, > 2}; d0 is unrolled so the
// multiplicity selects are compile-time.  Conservative as ks4_pair_h (same alpha_h margin,
// same guarded SLO test); flagged blocks (one per d0) are rescanned exactly.
template <bool VERIFY>
__device__ __forceinline__ void ks3_pair_h(SearchState<3>& c, uint32_t maskA, uint32_t maskB, bool haveB,
                                           unsigned long long* misses, uint32_t zero, bool exh, uint64_t shiftB,
                                           uint32_t* defer = nullptr) {
  const float INF = __int_as_float(0x7f800000);
  constexpr h2 kInf2 = 0x7c007c00u, kNegInf2 = 0xfc00fc00u;
  const float al = c.alpha_h, one_m_a = 1.f - c.alpha_h;
  const h2 al2 = h2pack(al, al), nal2 = h2pack(-al, -al), oma2 = h2pack(one_m_a, one_m_a);
  const uint32_t* PL = c.sm + c.o_pl + c.row0 * kRowW;
  const uint32_t* PM = c.sm + c.o_pm + c.row0;
  const uint32_t* XF = c.sm + c.o_xf + c.row0;
  float f[2][3][kP], sig[2], slack[2];
  uint32_t ms[2][3];
  bool wide[2];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    uint32_t m = h ? maskB : maskA;
    const int j1 = __ffs(m) - 1;
    m &= m - 1;
    const int j2 = __ffs(m) - 1;
    const uint32_t b[4] = {0u, (uint32_t)j1 + 1, (uint32_t)j2 + 1, c.n};
    float pr[4][kP];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      if (i == 0) {
#pragma unroll
        for (int x = 0; x < kP; ++x) pr[0][x] = 0.f;
        continue;
      }
      const float4 l = *reinterpret_cast<const float4*>(PL + b[i] * kRowW);
      pr[i][0] = l.x;
      pr[i][1] = l.y;
      pr[i][2] = l.z;
      pr[i][3] = l.w;
      pr[i][4] = __uint_as_float(PL[b[i] * kRowW + 4]);
    }
#pragma unroll
    for (int st = 0; st < 3; ++st) {
#pragma unroll
      for (int x = 0; x < kP; ++x) f[h][st][x] = pr[st + 1][x] - pr[st][x];
      ms[h][st] = PM[b[st + 1]] - PM[b[st]];
    }
    const uint32_t X = XF[j1] + XF[j2];
    const bool live_h = h == 0 || haveB;  // the B half of a single mask is a dummy: nothing passes
    const float bl = (live_h && X <= c.B && !c.none_can_win) ? (float)min(c.B - X, 1u << 24) : -1.f;
    // sigma = 2^(5 - E) with M = min(Blim, tmax) <= 2^E (as ks4_pair_h)
    const float M = fmaxf(fminf(bl, c.tmax), 1.f);
    const uint32_t mb = __float_as_uint(M);
    const int E = (int)((mb >> 23) & 255u) - 127 + ((mb & 0x7fffffu) != 0u);
    sig[h] = __int_as_float((127 + 5 - E) << 23);
    wide[h] = bl >= 0.f && c.tmin * sig[h] < 0.125f;
    slack[h] = bl >= 0.f ? M * sig[h] * (1.f + 1.f / 128.f) : -INF;
  }
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t cap = c.sm[c.o_cap + x];
    if (c.thr_u == 0xffffffffu) {
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int st = 0; st < 3; ++st) f[h][st][x] = ms[h][st] <= cap ? f[h][st][x] * sig[h] : INF;
    } else {
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int st = 0; st < 3; ++st)
          f[h][st][x] = (ms[h][st] <= cap && f[h][st][x] <= c.thr) ? f[h][st][x] * sig[h] : INF;
    }
  }
  h2 v0[kP], nl0[kP], s1w[2][kP], a1[kP], t2[kP], c2w[3][kP];
  float v2m[2] = {INF, INF};  // fastest admissible last stage per half (>= 1 free slice)
  h2 v1min = kInf2;
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
    const h2 p0 = h2pack(f[0][0][x], f[1][0][x]), p1 = h2pack(f[0][1][x], f[1][1][x]);
    // an over-long last stage is inadmissible (keeps t2 and t2^2 far from overflow)
    const float u0 = f[0][2][x] <= slack[0] ? f[0][2][x] : INF, u1 = f[1][2][x] <= slack[1] ? f[1][2][x] : INF;
    const h2 p2 = h2pack(u0, u1);
    if (fr > 0) {
      v2m[0] = fminf(v2m[0], u0);
      v2m[1] = fminf(v2m[1], u1);
      v1min = h2min(v1min, p1);
    }
    v0[x] = fr > 0 ? p0 : kInf2;
    nl0[x] = h2mul(h2mul(p0, p0), nal2);
    s1w[0][x] = fr > 0 ? p1 : kInf2;
    s1w[1][x] = fr > 1 ? p1 : kInf2;
    a1[x] = h2mul(h2mul(p1, p1), al2);
    const uint32_t inf2 = ((p2 & 0xffffu) == 0x7c00u ? 0x0000ffffu : 0u) | ((p2 >> 16) == 0x7c00u ? 0xffff0000u : 0u);
    t2[x] = h2add(p2, p2) & ~inf2;
    const h2 cc = (h2mul(h2mul(p2, p2), oma2) & ~inf2) | (kNegInf2 & inf2);
    c2w[0][x] = fr > 0 ? cc : kNegInf2;
    c2w[1][x] = fr > 1 ? cc : kNegInf2;
    c2w[2][x] = fr > 2 ? cc : kNegInf2;
  }
  const uint32_t slk = h2guard(h2pack(slack[0] - v2m[0], slack[1] - v2m[1]));
  uint32_t pendA = 0, pendB = 0;
#pragma unroll
  for (int d0 = 0; d0 < kP; ++d0) {
    const h2 S1 = v0[d0], NL1 = nl0[d0];
    if (!exh) {  // stage-0 bound (bounded mode): every group has S2 >= S1 + v1min
      const uint32_t okb = isub(slk, h2add(S1, v1min), zero);
      if (!((okb & 0x8000u) || (haveB && (okb & 0x80000000u)))) continue;
    }
    c.n_scored += haveB ? 2 * kP * kP : kP * kP;  // 25 candidates per mask of this d0
    uint32_t acc = ~0u;
#pragma unroll
    for (int q = 0; q < kP; ++q) {
      const h2 S2 = h2add(S1, s1w[q == d0][q]);
      const h2 U = h2fma(S2, S2, h2sub(NL1, a1[q]));
      h2 y[kP];
#pragma unroll
      for (int p = 0; p < kP; ++p) y[p] = h2fma(S2, t2[p], c2w[(p == d0) + (p == q)][p]);
      const h2 z = h2add(h2max(h2max(h2max(y[0], y[1]), y[2]), h2max(y[3], y[4])), U);
      const uint32_t ok = isub(slk, S2, zero);
      acc &= z | ~ok;
    }
    pendA |= (((acc >> 15) & 1u) ^ 1u) << d0;
    pendB |= ((acc >> 31) ^ 1u) << d0;
  }
  constexpr uint32_t kAllB = (1u << kP) - 1;
  if (wide[0]) pendA = kAllB;  // dynamic range too wide for f16: every block exactly
  if (wide[1]) pendB = kAllB;
  if (!VERIFY && defer) {  // the caller rescans the flagged blocks warp-cooperatively
    defer[0] = pendA;
    defer[1] = haveB ? pendB : 0u;
    return;
  }
  if (VERIFY || pendA) {
    Geo<3> G;
    geo<3>(c, maskA, G);
    pair_rescan<3, VERIFY>(c, G, pendA, VERIFY ? kAllB : pendA, 0, misses);
  }
  if (haveB && (VERIFY || pendB)) {
    Geo<3> G;
    geo<3>(c, maskB, G);
    pair_rescan<3, VERIFY>(c, G, pendB, VERIFY ? kAllB : pendB, shiftB, misses);
  }
}

// KS = 3 over requests grouped by chain length (exhaustive / verify): ks3_pair_h with the
// last stage's tables (its "row" = the highest cut) rebuilt only when a half's row changes,
// warp-uniformly (the lanes walk the same masks), as ks4_pair_rows does for KS = 4.
struct Row3 {
  uint32_t keyA, keyB;  // rows (mask & (mask - 1)) the state was built for; ~0u = none
  uint32_t Xr[2];
  float sig[2], v2m[2];
  bool wide[2];
  h2 t2[kP], c2w[3][kP];
};

template <bool VERIFY>
__device__ __forceinline__ void ks3_pair_rows(SearchState<3>& c, Row3& R, uint32_t maskA, uint32_t maskB, bool haveB,
                                              bool lane_live, unsigned long long* misses, uint32_t zero,
                                              uint64_t shiftB, uint32_t* defer) {
  const float INF = __int_as_float(0x7f800000);
  constexpr h2 kInf2 = 0x7c007c00u, kNegInf2 = 0xfc00fc00u;
  const float al = c.alpha_h, one_m_a = 1.f - c.alpha_h;
  const h2 al2 = h2pack(al, al), nal2 = h2pack(-al, -al), oma2 = h2pack(one_m_a, one_m_a);
  const uint32_t* PL = c.sm + c.o_pl + c.row0 * kRowW;
  const uint32_t* PM = c.sm + c.o_pm + c.row0;
  const uint32_t* XF = c.sm + c.o_xf + c.row0;
  const uint32_t kA = maskA & (maskA - 1), kB = maskB & (maskB - 1);
  if (kA != R.keyA || kB != R.keyB) {  // warp-uniform
    R.keyA = kA;
    R.keyB = kB;
    float f2[2][kP], slr[2];
    uint32_t ms2[2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int j2 = __ffs(h ? kB : kA) - 1;
      const uint32_t b2 = (uint32_t)j2 + 1;
      const float4 la = *reinterpret_cast<const float4*>(PL + b2 * kRowW);
      const float4 lb = *reinterpret_cast<const float4*>(PL + c.n * kRowW);
      f2[h][0] = lb.x - la.x;
      f2[h][1] = lb.y - la.y;
      f2[h][2] = lb.z - la.z;
      f2[h][3] = lb.w - la.w;
      f2[h][4] = __uint_as_float(PL[c.n * kRowW + 4]) - __uint_as_float(PL[b2 * kRowW + 4]);
      ms2[h] = PM[c.n] - PM[b2];
      R.Xr[h] = XF[j2];
      const float bl = (lane_live && R.Xr[h] <= c.B && !c.none_can_win) ? (float)min(c.B - R.Xr[h], 1u << 24) : -1.f;
      const float M = fmaxf(fminf(bl, c.tmax), 1.f);
      const uint32_t mb = __float_as_uint(M);
      const int E = (int)((mb >> 23) & 255u) - 127 + ((mb & 0x7fffffu) != 0u);
      R.sig[h] = __int_as_float((127 + 5 - E) << 23);
      R.wide[h] = bl >= 0.f && c.tmin * R.sig[h] < 0.125f;
      slr[h] = bl >= 0.f ? M * R.sig[h] * (1.f + 1.f / 128.f) : -INF;
    }
    R.v2m[0] = INF;
    R.v2m[1] = INF;
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
      const uint32_t cap = c.sm[c.o_cap + x];
      float u[2];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const float v = (ms2[h] <= cap && f2[h][x] <= c.thr) ? f2[h][x] * R.sig[h] : INF;
        u[h] = v <= slr[h] ? v : INF;  // an over-long last stage is inadmissible
        if (fr > 0) R.v2m[h] = fminf(R.v2m[h], u[h]);
      }
      const h2 p2 = h2pack(u[0], u[1]);
      const uint32_t inf2 = ((p2 & 0xffffu) == 0x7c00u ? 0x0000ffffu : 0u) | ((p2 >> 16) == 0x7c00u ? 0xffff0000u : 0u);
      R.t2[x] = h2add(p2, p2) & ~inf2;
      const h2 cc = (h2mul(h2mul(p2, p2), oma2) & ~inf2) | (kNegInf2 & inf2);
      R.c2w[0][x] = fr > 0 ? cc : kNegInf2;
      R.c2w[1][x] = fr > 1 ? cc : kNegInf2;
      R.c2w[2][x] = fr > 2 ? cc : kNegInf2;
    }
  }
  // per mask pair: stages 0 and 1, the mask's own SLO slack
  float f[2][2][kP], sl[2];
  uint32_t ms[2][2];
  bool wide[2];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    uint32_t m = h ? maskB : maskA;
    const int j1 = __ffs(m) - 1;
    m &= m - 1;
    const int j2 = __ffs(m) - 1;
    const uint32_t b1 = (uint32_t)j1 + 1, b2 = (uint32_t)j2 + 1;
    const float4 l1 = *reinterpret_cast<const float4*>(PL + b1 * kRowW);
    const float4 l2 = *reinterpret_cast<const float4*>(PL + b2 * kRowW);
    const float p1[kP] = {l1.x, l1.y, l1.z, l1.w, __uint_as_float(PL[b1 * kRowW + 4])};
    const float p2[kP] = {l2.x, l2.y, l2.z, l2.w, __uint_as_float(PL[b2 * kRowW + 4])};
#pragma unroll
    for (int x = 0; x < kP; ++x) {
      f[h][0][x] = p1[x];  // prefix row 0 is zero
      f[h][1][x] = p2[x] - p1[x];
    }
    ms[h][0] = PM[b1] - PM[0];
    ms[h][1] = PM[b2] - PM[b1];
    const uint32_t X = XF[j1] + R.Xr[h];
    const bool live_h = lane_live && (h == 0 || haveB);
    const float bl = (live_h && X <= c.B && !c.none_can_win) ? (float)min(c.B - X, 1u << 24) : -1.f;
    const float M = fmaxf(fminf(bl, c.tmax), 1.f);
    sl[h] = bl >= 0.f ? M * R.sig[h] * (1.f + 1.f / 128.f) - R.v2m[h] : -INF;
    wide[h] = bl >= 0.f && R.wide[h];
  }
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t cap = c.sm[c.o_cap + x];
    if (c.thr_u == 0xffffffffu) {  // no throughput floor (the common case; uniform per request)
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int s = 0; s < 2; ++s) f[h][s][x] = ms[h][s] <= cap ? f[h][s][x] * R.sig[h] : INF;
    } else {
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int s = 0; s < 2; ++s)
          f[h][s][x] = (ms[h][s] <= cap && f[h][s][x] <= c.thr) ? f[h][s][x] * R.sig[h] : INF;
    }
  }
  h2 v0[kP], nl0[kP], s1w[2][kP], a1[kP];
#pragma unroll
  for (int x = 0; x < kP; ++x) {
    const uint32_t fr = (uint32_t)(c.freeb >> (8 * x)) & 255u;
    const h2 p0 = h2pack(f[0][0][x], f[1][0][x]), p1 = h2pack(f[0][1][x], f[1][1][x]);
    v0[x] = fr > 0 ? p0 : kInf2;
    nl0[x] = h2mul(h2mul(p0, p0), nal2);
    s1w[0][x] = fr > 0 ? p1 : kInf2;
    s1w[1][x] = fr > 1 ? p1 : kInf2;
    a1[x] = h2mul(h2mul(p1, p1), al2);
  }
  const uint32_t slk = h2guard(h2pack(sl[0], sl[1]));
  uint32_t pendA = 0, pendB = 0;
#pragma unroll
  for (int d0 = 0; d0 < kP; ++d0) {
    const h2 S1 = v0[d0], NL1 = nl0[d0];
    if (lane_live) c.n_scored += haveB ? 2 * kP * kP : kP * kP;  // 25 candidates per mask of this d0
    uint32_t acc = ~0u;
#pragma unroll
    for (int q = 0; q < kP; ++q) {
      const h2 S2 = h2add(S1, s1w[q == d0][q]);
      const h2 U = h2fma(S2, S2, h2sub(NL1, a1[q]));
      h2 y[kP];
#pragma unroll
      for (int p = 0; p < kP; ++p) y[p] = h2fma(S2, R.t2[p], R.c2w[(p == d0) + (p == q)][p]);
      const h2 z = h2add(h2max(h2max(h2max(y[0], y[1]), y[2]), h2max(y[3], y[4])), U);
      const uint32_t ok = isub(slk, S2, zero);
      acc &= z | ~ok;
    }
    pendA |= (((acc >> 15) & 1u) ^ 1u) << d0;
    pendB |= ((acc >> 31) ^ 1u) << d0;
  }
  constexpr uint32_t kAllB = (1u << kP) - 1;
  if (wide[0]) pendA = kAllB;
  if (wide[1]) pendB = kAllB;
  if (!VERIFY && defer) {
    defer[0] = lane_live ? pendA : 0u;
    defer[1] = (lane_live && haveB) ? pendB : 0u;
    return;
  }
  if (!lane_live) return;
  if (VERIFY || pendA) {
    Geo<3> G;
    geo<3>(c, maskA, G);
    pair_rescan<3, VERIFY>(c, G, pendA, VERIFY ? kAllB : pendA, 0, misses);
  }
  if (haveB && (VERIFY || pendB)) {
    Geo<3> G;
    geo<3>(c, maskB, G);
    pair_rescan<3, VERIFY>(c, G, pendB, VERIFY ? kAllB : pendB, shiftB, misses);
  }
}

template <int KS, bool VERIFY>
__device__ __forceinline__ void unrolled_mask(SearchState<KS>& c, float* rows, unsigned long long* misses,
                                              uint32_t* defer = nullptr) {
  uint32_t pend = 0;  // one bit per block of P*P candidates
  if constexpr (KS == 4) {
    __trap();  // KS = 4 uses ks4_pair
  } else {
    Tables<KS> T;
    build_tables<KS>(c, T);
    const float Bl = c.blim;
    if constexpr (KS == 2) {
      pend = block_qp(T.a[0], T.t2, 0.f, 0.f, Bl - T.vmin, [&](int q) { return T.vf[0][0][q]; },
                      [&](int q, int p) { return T.ccv[p == q][p]; });
    } else {
#pragma unroll
      for (int d0 = 0; d0 < kP; ++d0) {
        const float v0 = T.vf[0][0][d0];
        pend |= block_qp(T.a[1], T.t2, v0, T.a[0][d0], (Bl - v0) - T.vmin,
                         [&](int q) { return T.vf[1][q == d0][q]; },
                         [&](int q, int p) { return T.ccv[(p == d0) + (p == q)][p]; })
                << d0;
      }
    }
  }
  constexpr int NB = KS == 2 ? 1 : (KS == 3 ? kP : kP * kP);
  c.n_scored += (KS == 2 ? kP * kP : KS == 3 ? kP * kP * kP : kP * kP * kP * kP);
  if (!VERIFY && defer) {  // the caller rescans the flagged block warp-cooperatively (KS = 2)
    *defer = pend;
    return;
  }
  const uint32_t all = VERIFY ? ((1u << NB) - 1) : pend;
  for (uint32_t todo = all; todo;) {
    const int b = __ffs(todo) - 1;
    todo &= todo - 1;
    if constexpr (KS == 3) c.pd[0] = b;
    if constexpr (KS == 4) {
      c.pd[0] = b / kP;
      c.pd[1] = b - kP * (b / kP);
    }
    const uint32_t fast = ((pend >> b) & 1u) ? ((1u << (kP * kP)) - 1) : 0u;
    handle_hits<KS, VERIFY>(c, (1u << (kP * kP)) - 1, fast, misses);
  }
}

template <int KS, bool VERIFY>
__device__ __forceinline__ void process_mask(SearchState<KS>& c, uint32_t mask, float* rows,
                                             unsigned long long* misses, uint32_t* defer = nullptr) {
  // stage boundaries: a cut after component j iff bit j is set
  c.bnd[0] = 0;
  uint32_t m = mask, X = 0;
#pragma unroll
  for (int i = 0; i < KS - 1; ++i) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    c.bnd[i + 1] = j + 1;
    X += c.sm[c.o_xf + c.row0 + j];
  }
  c.bnd[KS] = c.n;
  c.X = X;
#pragma unroll
  for (int i = 0; i < KS; ++i) c.memst[i] = c.sm[c.o_pm + c.row0 + c.bnd[i + 1]] - c.sm[c.o_pm + c.row0 + c.bnd[i]];
  // e2e <= B  <=>  sum t <= B - X; exact in float because sum t < 2^24 (R4 bound)
  c.blim_raw = (X <= c.B) ? __uint2float_rd(c.B - X) : -1.f;
  if constexpr (KS >= 2 && KS <= 4) {
    // exact in fp32: min(B - X, 2^24) is an integer <= 2^24 and every stage sum is < 2^24
    c.blim_raw = (X <= c.B) ? (float)min(c.B - X, 1u << 24) : -1.f;
    c.blim = c.none_can_win ? -1.f : c.blim_raw;
    unrolled_mask<KS, VERIFY>(c, rows, misses, defer);
  } else if constexpr (KS == 1) {
    c.blim = c.blim_raw;
    // 5 candidates per request: evaluate them exactly
    c.pd[0] = 0;
    c.n_scored += kP;
#pragma unroll
    for (int p = 0; p < kP; ++p) exact_eval<KS, VERIFY>(c, 0, p, true, misses);
  } else {
    load_stage<KS>(c, KS - 2, c.tq, c.sqq);
    load_stage<KS>(c, KS - 1, c.tp, c.sqp);
    set_threshold(c);
    uint64_t pk = 1;
#pragma unroll
    for (int i = 0; i < KS; ++i) pk *= kP;
    c.n_scored += pk;  // the generic path scores every candidate of the mask
    outer_level<0, KS, VERIFY>(c, 0.f, 0.f, c.free_w, misses);
  }
}

__device__ __forceinline__ uint32_t gosper_next(uint32_t x) {
  const uint32_t t = x | (x - 1);
  return (t + 1) | (((~t & (0u - ~t)) - 1) >> __ffs(x));
}

// largest r with prefix[r] <= t (prefix non-decreasing, prefix[0] = 0 <= t)
__device__ __forceinline__ uint32_t find_request(const uint64_t* __restrict__ pre, uint32_t n_req, uint64_t t) {
  uint32_t lo = 0, hi = n_req;  // invariant: pre[lo] <= t < pre[hi] (pre[n_req] = total > t)
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (pre[mid] <= t) lo = mid; else hi = mid;
  }
  return lo;
}

// Exact key of one candidate (as exact_eval): request state broadcast from the lane that
// owns the block, cut mask, profile digits; FFS_KEY_NONE when infeasible.
template <int KS>
__device__ __forceinline__ int64_t exact_key(const SearchState<KS>& c, uint32_t row0, uint32_t n, uint32_t B,
                                             uint32_t thr_u, uint64_t freeb, uint32_t mask, uint64_t idx,
                                             const int (&prof)[KS]) {
  uint32_t bnd[KS + 1];
  bnd[0] = 0;
  uint32_t m = mask, X = 0;
#pragma unroll
  for (int i = 1; i < KS; ++i) {
    const uint32_t j = __ffs(m) - 1;
    m &= m - 1;
    bnd[i] = j + 1;
    X += c.sm[c.o_xf + row0 + j];
  }
  bnd[KS] = n;
  uint64_t St = 0, Sq = 0;
  uint32_t used = 0, g = 0;
  bool ok = true;
#pragma unroll
  for (int i = 0; i < KS; ++i) {
    const int pr = prof[i];
    const uint32_t a = (row0 + bnd[i]) * kRowW, b = (row0 + bnd[i + 1]) * kRowW;
    const uint32_t t = pl_diff(c.sm, c.o_pl + b + pr, c.o_pl + a + pr);
    ok &= c.sm[c.o_pm + row0 + bnd[i + 1]] - c.sm[c.o_pm + row0 + bnd[i]] <= c.sm[c.o_cap + pr];
    ok &= t <= thr_u;  // R38 throughput floor
    St += t;
    Sq += (uint64_t)t * t;
    used += 1u << (4 * pr);
    g += c.sm[c.o_gpcs + pr];
  }
#pragma unroll
  for (int pp = 0; pp < kP; ++pp) ok &= ((used >> (4 * pp)) & 15u) <= ((freeb >> (8 * pp)) & 255u);
  ok &= St + X <= (uint64_t)B;
  if (!ok) return (int64_t)kKeyNone;
  const uint64_t D = St * St, N = (uint64_t)KS * Sq - D;
  const uint64_t cvq = (N << 10) / D;  // floor(1024 * CV^2), exact (R4)
  return (int64_t)((cvq << 50) | ((uint64_t)(KS - 1) << 47) | ((uint64_t)g << 41) | idx);
}

// Warp-cooperative exact rescan of the flagged blocks (KS = 4: block = stage-0/1 profiles
// (d0, d1); KS = 3: block = d0; KS = 2: the mask), each a block of 25 candidates (the last
// two stages' q, p):
// the block's owner lane broadcasts its request state, 25 lanes evaluate one candidate
// each, the warp minimum goes back to the owner.  In the bounded list mode the flags are
// frequent and sparse across lanes -- rescanned lane by lane they ran at ~2 active threads
// per instruction.  All 32 lanes must call it.
template <int KS>
__device__ __forceinline__ void coop_rescan(SearchState<KS>& c, uint32_t mask, uint32_t pend, uint64_t idx0) {
  const uint32_t lane = threadIdx.x & 31;
  for (;;) {
    const uint32_t who = __ballot_sync(0xffffffffu, pend != 0u);
    if (!who) break;
    const int L = __ffs(who) - 1;
    const int b = __shfl_sync(0xffffffffu, __ffs(pend) - 1, L);
    if ((int)lane == L) pend &= pend - 1;
    const uint32_t row0 = __shfl_sync(0xffffffffu, c.row0, L), n = __shfl_sync(0xffffffffu, c.n, L);
    const uint32_t B = __shfl_sync(0xffffffffu, c.B, L), thr = __shfl_sync(0xffffffffu, c.thr_u, L);
    const uint32_t mk = __shfl_sync(0xffffffffu, mask, L);
    const uint64_t freeb = __shfl_sync(0xffffffffu, c.freeb, L);
    const uint64_t i0 = __shfl_sync(0xffffffffu, idx0, L);
    int64_t key = (int64_t)kKeyNone;
    if (lane < (uint32_t)(kP * kP)) {
      const int q = (int)lane / kP, p = (int)lane - kP * q;
      int prof[KS];
      uint64_t seq;
      if constexpr (KS == 4) {
        prof[0] = b / kP;
        prof[1] = b - kP * (b / kP);
        prof[2] = q;
        prof[3] = p;
        seq = (uint64_t)b * (kP * kP) + lane;
      } else if constexpr (KS == 2) {  // one block per mask (b = 0)
        prof[0] = q;
        prof[1] = p;
        seq = lane;
      } else {
        prof[0] = b;
        prof[1] = q;
        prof[2] = p;
        seq = (uint64_t)b * (kP * kP) + lane;
      }
      key = exact_key<KS>(c, row0, n, B, thr, freeb, mk, i0 + seq, prof);
    }
    const int64_t kmin = (int64_t)warp_min_u64((uint64_t)key);
    if ((int)lane == L && kmin < c.best) {
      c.best = kmin;
      set_threshold(c);
    }
  }
}

// colex rank of a cut mask among the (KS-1)-subsets of the cut positions: sum C(j_i, i)
template <int KS>
__device__ __forceinline__ uint64_t colex_rank(const uint32_t* img, const ImageLayout& L, uint32_t mask) {
  uint64_t rk = 0;
#pragma unroll
  for (int i = 1; i < KS; ++i) {
    const int j = __ffs(mask) - 1;
    mask &= mask - 1;
    rk += binom(img, L, j, i);
  }
  return rk;
}

// LIST: the bounded mode's kernel (walks k_live's records, task ranges only as the
// overflow fallback); !LIST: task ranges only (exhaustive and verify modes, or no lists)
template <int KS, bool VERIFY, bool TG, bool LIST>
__global__ void __launch_bounds__(search_block(KS, LIST), KS <= 4 ? FFS_MINB4 : 1) k_plan_search(const __grid_constant__ SearchArgs A) {
  extern __shared__ __align__(16) uint32_t smem[];
  // A0: stage the table image into shared memory (16-byte copies); an image too large
  // for shared memory is read from global memory through L1 instead (A.tables_global)
  // (TG is a template parameter so that the shared-memory variant keeps LDS accesses)
  const uint32_t* tbl = smem;
  uint32_t img_words = A.lay.words;
  if constexpr (TG) {
    tbl = A.image;
    img_words = 0;
  } else {
    const uint4* src = reinterpret_cast<const uint4*>(A.image);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    for (uint32_t i = threadIdx.x; i < A.lay.words / 4; i += blockDim.x) dst[i] = src[i];
  }
  __syncthreads();
  // KS = 4: per-thread windows of the shifted variant tables after the image (ks4_pair_h)
  float* rows = reinterpret_cast<float*>(smem + img_words);

  const uint64_t* pre = A.prefix + (uint64_t)(KS - 1) * (A.n_req + 1);
  const uint32_t lane = threadIdx.x & 31;
  uint64_t PK = 1;
#pragma unroll
  for (int i = 0; i < KS; ++i) PK *= kP;

  SearchState<KS> c;
  c.n_scored = 0;
  c.sm = tbl;
  c.o_pl = A.lay.o_pl;
  c.o_pm = A.lay.o_pm;
  c.o_xf = A.lay.o_xf;
  c.o_cap = A.lay.o_cap;
  c.o_gpcs = A.lay.o_gpcs;
  uint32_t r = 0;
  int64_t best0 = 0;

  // request r's state; idx_base = the index of the rank0-th mask's first candidate
  auto load_request = [&](uint64_t rank0) {
    const ffs_request q = A.req[r];
    const uint32_t* fd = tbl + A.lay.o_fdesc + 4 * q.func;
    c.row0 = fd[0];
    c.n = fd[1];
    c.B = A.slo[r];
    c.freeb = A.node_free[q.node];
    c.thr_u = tbl[A.lay.o_thr + q.func];
    c.thr = (float)min(c.thr_u, 1u << 24);
    uint32_t w = 0;
#pragma unroll
    for (int p = 0; p < kP; ++p) w |= (16u + (uint32_t)((c.freeb >> (8 * p)) & 255u)) << (5 * p);
    c.free_w = w;
    c.idx_base = img_u64(tbl, A.lay.o_offk + 2 * (c.n * 10 + KS)) + rank0 * PK;
    c.best = *reinterpret_cast<volatile const int64_t*>(A.keys + r);  // earlier segments' minimum
    best0 = c.best;
    if constexpr (KS >= 2) set_threshold(c);
    if constexpr (KS == 3 || KS == 4) {  // f16 scale bounds; fp32 rounding above 2^24 is covered by the 2^-7 slack margin
      c.tmin = __uint_as_float(tbl[A.lay.o_tmm + 2 * q.func]);
      c.tmax = __uint_as_float(tbl[A.lay.o_tmm + 2 * q.func + 1]);
    }
    c.nfeas = 0;
    c.ksum = 0;
  };
  auto flush = [&](uint64_t done) {
    if (c.best < best0) atomicMin(reinterpret_cast<long long*>(A.keys + r), (long long)c.best);
    if (VERIFY) {
      atomicAdd(A.checks + 3ull * r, (unsigned long long)(done * PK));
      atomicAdd(A.checks + 3ull * r + 1, (unsigned long long)c.nfeas);
      atomicAdd(A.checks + 3ull * r + 2, (unsigned long long)c.ksum);
    }
  };

  uint64_t n_list = ~0ull;
  if (LIST && !VERIFY && KS >= 2 && KS <= 4 && A.list != nullptr)
    n_list = *reinterpret_cast<volatile const unsigned long long*>(A.work_ctr + kCtrListCount + KS);
  if (LIST && n_list <= A.list_cap) {
    // ---- bounded mode: the live (request, mask pair) records of k_live ----------------
    // A warp takes 32 consecutive records (one per lane) at a time; every record carries
    // its request, so a lane loads the request's state per record.
    // The loop stays warp-converged (a lane without a record idles) so the flagged blocks
    // of all lanes are rescanned cooperatively (coop_rescan).
    unsigned long long* lctr = A.work_ctr + kCtrListGrab + KS;
    for (;;) {
      unsigned long long jg = 0;
      if (lane == 0) jg = atomicAdd(lctr, 1ull);
      jg = __shfl_sync(0xffffffffu, jg, 0);
      if (jg * 32 >= n_list) break;
      const uint64_t i = jg * 32 + lane;
      const bool has = i < n_list;
      uint32_t maskA = 0, maskB = 0, pend[2] = {0u, 0u};
      uint64_t shiftB = 0;
      if (has) {
        const uint4 rec = A.list[i];
        r = rec.x;
        maskA = rec.y;
        maskB = rec.z;
        const bool haveB = maskB != 0u;
        const uint64_t rkA = colex_rank<KS>(tbl, A.lay, maskA);
        shiftB = haveB ? (colex_rank<KS>(tbl, A.lay, maskB) - rkA) * PK : 0ull;
        load_request(rkA);
        if constexpr (KS == 4) {
          ks4_pair_h<false>(c, maskA, haveB ? maskB : maskA, haveB, reinterpret_cast<h2*>(rows), A.misses, A.zero,
                            false, shiftB, pend);
        } else if constexpr (KS == 3) {
          ks3_pair<false>(c, maskA, haveB ? maskB : maskA, haveB, A.misses, false, shiftB, pend);
        } else if constexpr (KS == 2) {
          // (flags are dense among live records: each lane rescans its own, in parallel)
          process_mask<KS, false>(c, maskA, rows, A.misses);
          if (haveB) {
            c.idx_base += shiftB;
            process_mask<KS, false>(c, maskB, rows, A.misses);
          }
        }
      }
      if constexpr (KS == 3 || KS == 4) {
        __syncwarp();
        coop_rescan<KS>(c, maskA, pend[0], c.idx_base);
        coop_rescan<KS>(c, maskB, pend[1], c.idx_base + shiftB);
      }
      if (has) flush(0);
    }
  } else if (KS >= 2 && KS <= 4 && !LIST && A.g_perm != nullptr) {
    if constexpr (KS >= 2 && KS <= 4 && !LIST) {
      // ---- exhaustive / verify KS = 2..4: 32 requests of equal n per warp, lockstep masks -
      // Work unit = (n, group of 32 requests of g_perm, chunk of kGrpS masks in colex
      // order); rank `rank` owns units j * world + rank; warps grab them dynamically.  Every
      // lane walks the same masks (Gosper), so ks4_pair_rows rebuilds its stage-2/3 tables
      // warp-uniformly, only when a half's row changes.  A lane past the group's last
      // request mirrors the first one's state but scores, flags and flushes nothing.
      const uint32_t* gt = A.g_tab;
      const uint32_t* gu = gt + (KS == 4 ? 34 : KS == 3 ? 68 : 102);  // unit prefix per n of this segment
      const uint32_t U = gu[33];
      unsigned long long* ctr = A.work_ctr + KS;
      for (;;) {
        unsigned long long jg = 0;
        if (lane == 0) jg = atomicAdd(ctr, 1ull);
        jg = __shfl_sync(0xffffffffu, jg, 0);
        const uint64_t u = (uint64_t)jg * A.world + A.rank;
        if (u >= U) break;
        uint32_t n = 32;  // units of n: [gu[n], gu[n - 1]) (longest chains first), n = KS: up to gu[33]
        while (n > KS && gu[n - 1] <= u) --n;
        const uint32_t S = KS == 4 ? kGrpS : KS == 3 ? A.g_s3 : 32u;  // KS = 2: a request's n - 1 <= 31 masks
        const uint32_t Mn = binom(tbl, A.lay, (int)n - 1, KS - 1), Cn = (Mn + S - 1) / S;
        const uint32_t loc = (uint32_t)(u - gu[n]), g = loc / Cn, ch = loc - g * Cn;
        const uint32_t ii = 32 * g + lane;
        const bool has = ii < gt[n + 1] - gt[n];
        r = A.g_perm[gt[n] + (has ? ii : 32 * g)];
        const uint32_t m0 = ch * S, m1 = min(m0 + S, Mn);
        load_request(m0);
        uint32_t mask = 0;
        {  // colex unrank of m0 among the (KS-1)-subsets of the n - 1 cut positions (uniform)
          uint32_t mm = m0;
          int cc = (int)n - 2;
#pragma unroll
          for (int i = KS - 1; i >= 1; --i) {
            while (binom(tbl, A.lay, cc, i) > mm) --cc;
            mask |= 1u << cc;
            mm -= binom(tbl, A.lay, cc, i);
            --cc;
          }
        }
        if constexpr (KS == 2) {  // one mask per step (25 candidates, fp32 block_qp)
          for (uint32_t m = m0; m < m1; ++m) {
            uint32_t pend[2] = {0u, 0u};
            const uint64_t i0 = c.idx_base;
            if (has) process_mask<KS, VERIFY>(c, mask, rows, A.misses, VERIFY ? nullptr : pend);
            if constexpr (!VERIFY) {
              __syncwarp();
              coop_rescan<KS>(c, mask, pend[0], i0);
            }
            mask = gosper_next(mask);
            c.idx_base += PK;
          }
          if (has) flush(m1 - m0);
          continue;
        }
        std::conditional_t<KS == 4, Row4, Row3> R;
        R.keyA = R.keyB = ~0u;
        for (uint32_t m = m0; m < m1; m += 2) {
          const bool haveB = m + 1 < m1;
          const uint32_t maskB = haveB ? gosper_next(mask) : mask;
          uint32_t pend[2] = {0u, 0u};
          const uint64_t i0 = c.idx_base;
          if constexpr (KS == 4)
            ks4_pair_rows<VERIFY>(c, R, mask, maskB, haveB, has, reinterpret_cast<h2*>(rows), A.misses, A.zero, PK,
                                  VERIFY ? nullptr : pend);
          else if constexpr (KS == 3)
            ks3_pair_rows<VERIFY>(c, R, mask, maskB, haveB, has, A.misses, A.zero, PK, VERIFY ? nullptr : pend);
          if constexpr (!VERIFY) {
            __syncwarp();
            coop_rescan<KS>(c, mask, pend[0], i0);
            coop_rescan<KS>(c, maskB, pend[1], i0 + PK);
          }
          if (haveB) mask = gosper_next(maskB);
          c.idx_base += 2 * PK;
        }
        if (has) flush(m1 - m0);
      }
    }
  } else {
    // ---- task ranges (exhaustive and verify modes; bounded mode's fallback) -------------
    const uint64_t T = pre[A.n_req];
    // bounded mode whose live list overflowed: k_live partitioned the masks over the ranks
    // by row, not by these chunks, so this rank covers the whole segment (redundant with
    // the other ranks but complete; the MIN of the keys is idempotent)
    const bool whole = A.list != nullptr;
    const uint32_t world = whole ? 1u : A.world, rank = whole ? 0u : A.rank;
    // Work split: the segment's task list is cut into NC = world x (nthr/32) x kdyn(KS) chunks
    // of 32 equal contiguous pieces (one per lane).  Rank `rank` owns chunks
    // j * world + rank; its warps grab them dynamically (atomic counter, zeroed by the count
    // kernel), so a warp whose pieces are cheap (skipped stage-0 profiles, no rescans) takes
    // more of them and the launch ends when the work does, not with the slowest static
    // share.  Ranks interleave at the grain of one chunk, so each samples the whole batch
    // (contiguous 1/world ranges measured up to 1.2x apart on C5).  Exact cover needs the
    // same nthr on every rank (same kernel and device type).  DESIGN.md §4.3, §7.
    const uint64_t nthr = (uint64_t)gridDim.x * blockDim.x;
    // at most warps x kdyn chunks per rank, pieces of at least kMinPiece(KS) tasks (short
    // segments -- a request shard's -- would otherwise pay a request lookup per task)
    uint64_t NC = (nthr >> 5) * kdyn(KS) * world;
    const uint64_t want = T / (32ull * kMinPiece(KS));
    if (want < NC) NC = max((uint64_t)world, (want + world - 1) / world * world);
    const uint64_t NT = NC * 32;
    const uint64_t Tq = T / NT, Tr = T % NT;  // piece u = [Tq u + Tr u / NT, ...): no overflow
    auto piece = [&](uint64_t u) { return Tq * u + Tr * u / NT; };
    unsigned long long* ctr = A.work_ctr + KS;
    for (;;) {
      unsigned long long jg = 0;
      if (lane == 0) jg = atomicAdd(ctr, 1ull);
      jg = __shfl_sync(0xffffffffu, jg, 0);
      const uint64_t chunk = (uint64_t)jg * world + rank;
      if (chunk >= NC) break;
      const uint64_t t0 = piece(chunk * 32 + lane), t1 = piece(chunk * 32 + lane + 1);
      // the lanes walk their pieces in lockstep (pieces differ by at most one task), so the
      // flagged blocks of KS = 3/4 pairs are rescanned warp-cooperatively (coop_rescan);
      // verify mode rescans every block per lane
      bool active = t0 < t1;
      uint64_t task = t0, m = 0, cnt = 0, done = 0;
      uint32_t mask = 0;
      // colex unrank of rank0 among the (KS-1)-subsets of the n-1 cut positions.  Rank 0
      // (a request entered at its first task) is the lowest KS-1 bits: a shortcut worth it
      // where requests are short (KS <= 3); for KS = 4 the extra branch measured 1% slower.
      auto unrank = [&](uint64_t rank0) {
        uint32_t mk = (1u << (KS - 1)) - 1;
        if (KS >= 4 || rank0 != 0) {
          mk = 0;
          uint64_t mm = rank0;
          int cc = (int)c.n - 2;
#pragma unroll
          for (int i = KS - 1; i >= 1; --i) {
            while (binom(tbl, A.lay, cc, i) > mm) --cc;
            mk |= 1u << cc;
            mm -= binom(tbl, A.lay, cc, i);
            --cc;
          }
        }
        mask = mk;
      };
      if (active) {
        r = find_request(pre, A.n_req, task);
        m = task - pre[r];
        cnt = pre[r + 1] - pre[r];
        load_request(m);
        unrank(m);
      }
      while (__any_sync(0xffffffffu, active)) {
        uint32_t step = 1, pend[2] = {0u, 0u}, mA = 0, mB = 0;
        const uint64_t i0 = c.idx_base;
        if (active) {
          if constexpr (KS == 3 || KS == 4) {
            // two consecutive masks of the same request per iteration (ks3_pair / ks4_pair_h)
            const bool haveB = (m + 1 < cnt) && (task + 1 < t1);
            const uint32_t maskB = haveB ? gosper_next(mask) : mask;
            if constexpr (KS == 4)
              ks4_pair_h<VERIFY>(c, mask, maskB, haveB, reinterpret_cast<h2*>(rows), A.misses, A.zero,
                                 A.exhaustive != 0, PK, VERIFY ? nullptr : pend);
            else if constexpr (LIST)
              ks3_pair<VERIFY>(c, mask, maskB, haveB, A.misses, A.exhaustive != 0, PK, VERIFY ? nullptr : pend);
            else
              ks3_pair_h<VERIFY>(c, mask, maskB, haveB, A.misses, A.zero, A.exhaustive != 0, PK,
                                 VERIFY ? nullptr : pend);
            mA = mask;
            mB = maskB;
            if (haveB) step = 2;
          } else {
            process_mask<KS, VERIFY>(c, mask, rows, A.misses, (KS == 2 && !VERIFY) ? pend : nullptr);
            mA = mask;
          }
        }
        if constexpr (!VERIFY && (KS == 3 || KS == 4)) {
          __syncwarp();
          coop_rescan<KS>(c, mA, pend[0], i0);  // before the lane moves on to another request
          coop_rescan<KS>(c, mB, pend[1], i0 + PK);
        } else if constexpr (!VERIFY && KS == 2) {
          __syncwarp();  // (flags are sparse over task ranges: cooperative, ~2x over per lane)
          coop_rescan<KS>(c, mA, pend[0], i0);
        }
        if (active) {
          if (step == 2) mask = mB;
          done += step;
          task += step;
          if (task >= t1) {
            flush(done);
            active = false;
          } else {
            m += step;
            if (m == cnt) {
              flush(done);
              done = 0;
              // tasks are consecutive: the next one belongs to the next request with tasks
              // (requests without tasks of this KS have pre[r + 1] == pre[r]); no binary search
              do ++r; while (pre[r + 1] <= task);
              m = 0;
              cnt = pre[r + 1] - pre[r];
              load_request(0);
              unrank(0);
            } else {
              mask = gosper_next(mask);
              c.idx_base += step * PK;
            }
          }
        }
      }
    }  // grab loop
  }
  {  // measurement: candidates scored by this warp (ffs_search_scored)
    uint64_t e = c.n_scored;
#pragma unroll
    for (int o = 16; o; o >>= 1) e += __shfl_xor_sync(0xffffffffu, e, o);
    if ((threadIdx.x & 31) == 0 && e) atomicAdd(A.work_ctr + kCtrScored + KS, (unsigned long long)e);
  }
}

template <int KS, bool V, bool TG, bool L>
static cudaError_t set_attr() {
  return cudaFuncSetAttribute(k_plan_search<KS, V, TG, L>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMaxSmem);
}

// (ks, verify, list) -> instantiation; list kernels exist for KS = 2..4 without verify.
#define FFS_KS_SWITCH(ks, verify, list, CALL)                                        \
  switch ((ks) * 2 + ((verify) ? 1 : 0) + ((list) && !(verify) && (ks) >= 2 && (ks) <= 4 ? 100 : 0)) { \
    case 2: CALL(1, false, false); break;                                          \
    case 3: CALL(1, true, false); break;                                           \
    case 4: CALL(2, false, false); break;                                          \
    case 5: CALL(2, true, false); break;                                           \
    case 6: CALL(3, false, false); break;                                          \
    case 7: CALL(3, true, false); break;                                           \
    case 8: CALL(4, false, false); break;                                          \
    case 9: CALL(4, true, false); break;                                           \
    case 10: CALL(5, false, false); break;                                         \
    case 11: CALL(5, true, false); break;                                          \
    case 12: CALL(6, false, false); break;                                         \
    case 13: CALL(6, true, false); break;                                          \
    case 14: CALL(7, false, false); break;                                         \
    case 15: CALL(7, true, false); break;                                          \
    case 16: CALL(8, false, false); break;                                         \
    case 17: CALL(8, true, false); break;                                          \
    case 104: CALL(2, false, true); break;                                         \
    case 106: CALL(3, false, true); break;                                         \
    case 108: CALL(4, false, true); break;                                         \
    default: return cudaErrorInvalidValue;                                         \
  }

template <bool TG>
static cudaError_t search_config_t(int ks, bool verify, bool list, int block, size_t smem, int* blocks_per_sm) {
  cudaError_t e = cudaSuccess;
#define CFG(K, V, L)                                                                                        \
  do {                                                                                                    \
    e = set_attr<K, V, TG, L>();                                                                          \
    if (e == cudaSuccess)                                                                                 \
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k_plan_search<K, V, TG, L>, block, smem); \
  } while (0)
  FFS_KS_SWITCH(ks, verify, list, CFG)
#undef CFG
  return e;
}

template <bool TG>
static cudaError_t launch_search_t(int ks, bool verify, bool list, const SearchArgs& a, int grid, int block,
                                   size_t smem, cudaStream_t st) {
#define LAUNCH(K, V, L) k_plan_search<K, V, TG, L><<<grid, block, smem, st>>>(a)
  FFS_KS_SWITCH(ks, verify, list, LAUNCH)
#undef LAUNCH
  return cudaGetLastError();
}

cudaError_t search_kernel_config(int ks, bool verify, bool list, bool tables_global, int block, size_t smem,
                                 int* blocks_per_sm) {
  return tables_global ? search_config_t<true>(ks, verify, list, block, smem, blocks_per_sm)
                       : search_config_t<false>(ks, verify, list, block, smem, blocks_per_sm);
}

cudaError_t launch_search(int ks, bool verify, bool list, const SearchArgs& a, int grid, int block, size_t smem,
                          cudaStream_t st) {
  return a.tables_global ? launch_search_t<true>(ks, verify, list, a, grid, block, smem, st)
                         : launch_search_t<false>(ks, verify, list, a, grid, block, smem, st);
}

// ====================================================================================
// K1b: bounded mode -- group tables and live-mask compaction
// ====================================================================================
// One CTA per (function, availability pattern).  W(i, j) = the fastest admissible time of
// stage [i, j): over the profiles p of the pattern with stage memory <= cap_p and time <=
// the throughput floor (R38); a candidate's stage on p needs p admissible, so every
// candidate's stage time is >= W (the multiplicity of p is ignored: still a lower bound).
__global__ void __launch_bounds__(128) k_group_tables(const uint32_t* __restrict__ img, ImageLayout L,
                                                      const uint32_t* __restrict__ gofs, uint32_t* __restrict__ grp) {
  __shared__ uint32_t Wm[33 * 33];  // W(i, j) at [j * 33 + i]
  __shared__ uint32_t h0[33], r2[33];
  const uint32_t f = blockIdx.x, a = blockIdx.y;
  const uint32_t row0 = img[L.o_fdesc + 4 * f], n = img[L.o_fdesc + 4 * f + 1], N1 = n + 1;
  const uint32_t thr = img[L.o_thr + f];
  uint32_t* g = grp + gofs[f] + a * grp_stride(n);
  uint32_t *H0 = g, *T3 = g + N1, *R2 = g + 2 * N1, *R3 = g + 3 * N1, *Mt = g + 4 * N1;
  auto X = [&](uint32_t j) { return img[L.o_xf + row0 + j - 1]; };  // cut at boundary j (after component j-1)
  auto sat = [](uint64_t v) { return (uint32_t)(v < kGInf ? v : kGInf); };
  for (uint32_t idx = threadIdx.x; idx < N1 * N1; idx += blockDim.x) {
    const uint32_t i = idx % N1, j = idx / N1;
    uint32_t w = kGInf;
    if (i < j) {
      const uint32_t mem = img[L.o_pm + row0 + j] - img[L.o_pm + row0 + i];
      for (int p = 0; p < kP; ++p) {
        if (!((a >> p) & 1u) || mem > img[L.o_cap + p]) continue;
        const uint32_t t = pl_diff(img, L.o_pl + (row0 + j) * kRowW + p, L.o_pl + (row0 + i) * kRowW + p);
        if (t <= thr) w = min(w, t);
      }
    }
    Wm[j * 33 + i] = w;
  }
  __syncthreads();
  for (uint32_t idx = threadIdx.x; idx < N1 * N1; idx += blockDim.x) {
    const uint32_t i = idx % N1, j = idx / N1;
    Mt[j * N1 + i] = (i < j && j < n && i >= 1) ? sat((uint64_t)Wm[j * 33 + i] + X(j)) : kGInf;
  }
  for (uint32_t j = threadIdx.x; j < N1; j += blockDim.x) {
    const uint32_t h = (j >= 1 && j < n) ? sat((uint64_t)Wm[j * 33] + X(j)) : kGInf;
    H0[j] = h;
    h0[j] = h;
    T3[j] = (j >= 1 && j < n) ? Wm[n * 33 + j] : kGInf;
  }
  __syncthreads();
  for (uint32_t j = threadIdx.x; j < N1; j += blockDim.x) {
    uint32_t m = kGInf;
    if (j < n)
      for (uint32_t i = 1; i < j; ++i) m = min(m, sat((uint64_t)h0[i] + Wm[j * 33 + i] + X(j)));
    R2[j] = m;
    r2[j] = m;
  }
  __syncthreads();
  for (uint32_t j = threadIdx.x; j < N1; j += blockDim.x) {
    uint32_t m = kGInf;
    if (j < n)
      for (uint32_t i = 2; i < j; ++i) m = min(m, sat((uint64_t)r2[i] + Wm[j * 33 + i] + X(j)));
    R3[j] = m;
  }
}

cudaError_t launch_group_tables(const uint32_t* image, const ImageLayout& lay, const uint32_t* gofs, uint32_t* grp,
                                cudaStream_t st) {
  k_group_tables<<<dim3(lay.F, 32), 128, 0, st>>>(image, lay, gofs, grp);
  return cudaGetLastError();
}

// K1b: live-mask compaction of segment KS (2..4), launched right before its search.  A
// mask (j1 < j2 < j3: cut positions) is kept iff its exact e2e lower bound
//   LB = W(0,b1) + X(b1) + W(b1,b2) + X(b2) + ... + W(b_{KS-1}, n) <= B   (b = j + 1)
// -- a mask with LB > B holds no feasible candidate, so dropping it is exact.  A warp takes
// per_grab (<= 32) requests at a time, one per lane: each lane loads its request's header (task counts,
// best key, function, budget, node availability) in parallel, and the requests that still
// have work are visited one after another by the whole warp (n <= 32, so each colex level
// fits the lanes): KS = 4 tests the blocks (fixed highest cut j3: R3[b3] + T3[b3], lanes over
// j3), the rows of every live block (fixed j2, j3: R2[b2] + Mt[b3][b2] + T3[b3], lanes over
// j2) and the masks of every live row (H0[b1] + Mt[b2][b1] + row constant, lanes over j1);
// KS = 3 and 2 are the same with one and two levels fewer.  A request is skipped for a
// segment when it has no tasks there (short chain, full node, bad request) or when its best
// key so far has cvq = 0 with fewer stages (no KS-stage candidate can beat it, R1 -- every
// 1-stage plan has CV = 0: 71 % of C5 after KS = 1, and many 2- and 3-stage winners).
// Live masks of a request are paired in order into records {r, maskA, maskB (0 = single), 0},
// staged per warp and segment in shared memory and appended 32 at a time (one atomic per
// 32 records).  Candidate shards (world > 1): rank g keeps the rows whose (request, j3, j2)
// hash is g mod world -- a partition of the masks.
__device__ __forceinline__ bool live_owned(uint32_t r, uint32_t j3, uint32_t j2, uint32_t rank, uint32_t world) {
  if (world == 1) return true;
  const uint32_t h = (r * 0x9E3779B1u) ^ ((j3 << 5 | j2) * 0x85EBCA6Bu);
  return (h ^ (h >> 15)) % world == rank;
}

// one segment's record stream of a warp: shared staging, flushed 32 records at a time
struct LiveStage {
  uint4* stage;                 // this warp's 64 staging slots
  uint4* list;
  unsigned long long* lcount;   // records appended so far (the segment's list length)
  uint32_t cap, cnt, pend;      // warp-uniform: staged records, unpaired live mask

  __device__ __forceinline__ void flush(uint32_t upto, uint32_t lane) {  // stage[0, upto) -> list
    uint32_t base = 0;
    if (lane == 0) base = (uint32_t)atomicAdd(lcount, (unsigned long long)upto);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (lane < upto && base + lane < cap) list[base + lane] = stage[lane];
  }
  __device__ __forceinline__ void push(bool has, uint4 rec, uint32_t lane) {  // one record per lane with `has`
    const uint32_t bal = __ballot_sync(0xffffffffu, has);
    if (has) stage[cnt + __popc(bal & ((1u << lane) - 1u))] = rec;
    cnt += __popc(bal);
    __syncwarp();
    if (cnt >= 32) {
      flush(32, lane);
      __syncwarp();
      if (lane < cnt - 32) stage[lane] = stage[32 + lane];
      __syncwarp();
      cnt -= 32;
    }
  }
  // the live masks of one row of request r (bit j1 of `bal`, the row's other cuts in `hi`)
  // continue the request's sequence after `pend`: consecutive masks are paired, an unpaired
  // last one stays in `pend`.  Every lane of the warp calls it.
  __device__ __forceinline__ void row(uint32_t bal, uint32_t hi, uint32_t r, uint32_t lane) {
    if (!bal) return;
    const uint32_t lt = (1u << lane) - 1u, hp = pend ? 1u : 0u;
    const uint32_t i = __popc(bal & lt) + hp;  // index of this lane's mask in the sequence
    bool has = false;
    uint4 rec = make_uint4(r, 0u, 0u, 0u);
    if (((bal >> lane) & 1u) && (i & 1u)) {  // second of a pair: the previous mask is pend or the bit below
      const uint32_t below = bal & lt;
      rec.y = below ? ((1u << (31 - __clz(below))) | hi) : pend;
      rec.z = (1u << lane) | hi;
      has = true;
    }
    pend = ((__popc(bal) + hp) & 1u) ? ((1u << (31 - __clz(bal))) | hi) : 0u;
    push(has, rec, lane);
  }
  // the same for live masks held one per lane (lane order = colex order): `bal` = lanes
  // with a live mask, `mk` = this lane's mask.  Every lane of the warp calls it.
  __device__ __forceinline__ void masks(uint32_t bal, uint32_t mk, uint32_t r, uint32_t lane) {
    if (!bal) return;
    const uint32_t lt = (1u << lane) - 1u, hp = pend ? 1u : 0u;
    const uint32_t below = bal & lt;
    const uint32_t prev = __shfl_sync(0xffffffffu, mk, below ? 31 - __clz(below) : lane);
    const uint32_t i = __popc(below) + hp;
    const bool has = ((bal >> lane) & 1u) && (i & 1u);  // second of a pair
    const uint4 rec = make_uint4(r, below ? prev : pend, mk, 0u);
    const uint32_t last = __shfl_sync(0xffffffffu, mk, 31 - __clz(bal));
    pend = ((__popc(bal) + hp) & 1u) ? last : 0u;
    push(has, rec, lane);
  }
  __device__ __forceinline__ void end_request(uint32_t r, uint32_t lane) {
    if (pend) push(lane == 0, make_uint4(r, pend, 0u, 0u), lane);
    pend = 0;
  }
};

template <int KS>
__global__ void __launch_bounds__(256) k_live(const __grid_constant__ LiveArgs A) {
  static_assert(KS >= 2 && KS <= 4, "k_live: KS = 2..4");
  constexpr uint32_t kTabWords = 4 * 33 + 33 * 33;  // grp_stride(32)
  const uint32_t* img = A.image;
  const ImageLayout& L = A.lay;
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t NR = A.n_req;
  __shared__ uint4 stage_all[8][64];
  // KS = 3, 4: the visited request's group tables, copied once per request -- the row and
  // mask tests are a dependent chain per row (ballot -> row constant -> mask loads), so
  // they run at shared-memory rather than L2 latency
  __shared__ uint32_t tab_all[KS >= 3 ? 8 : 1][KS >= 3 ? kTabWords : 1];
  // colex order of the pairs j1 < j2 (< 32): tri[C(j2, 2) + j1] = j2 << 8 | j1
  __shared__ uint16_t tri[KS >= 3 ? 496 : 1];
  if constexpr (KS >= 3) {
    for (uint32_t t = threadIdx.x; t < 496; t += blockDim.x) {
      uint32_t j2 = 1;
      while ((j2 + 1) * j2 / 2 <= t) ++j2;
      tri[t] = (uint16_t)(j2 << 8 | (t - j2 * (j2 - 1) / 2));
    }
    __syncthreads();
  }
  LiveStage sg{stage_all[warp], A.list[KS - 2], A.work_ctr + kCtrListCount + KS, A.list_cap, 0u, 0u};
  const uint64_t* pre = A.prefix + (uint64_t)(KS - 1) * (NR + 1);
  unsigned long long* ctr = A.work_ctr + kCtrLiveGrab + KS;
  for (;;) {
    unsigned long long jg = 0;
    if (lane == 0) jg = atomicAdd(ctr, 1ull);
    jg = __shfl_sync(0xffffffffu, jg, 0);
    const uint64_t r0 = jg * A.per_grab;
    if (r0 >= NR) break;
    // this lane's request: does the segment need it, its chain length, budget, group tables
    const uint32_t rl = (uint32_t)r0 + lane;
    uint32_t n = 0, B = 0, go = 0;
    bool need = false;
    if (lane < A.per_grab && rl < NR && pre[rl + 1] != pre[rl]) {
      const uint64_t bk = (uint64_t)A.keys[rl];
      need = !(bk != kKeyNone && (bk >> 50) == 0 && (uint32_t)((bk >> 47) & 7) + 1u < (uint32_t)KS);
      if (need) {
        const ffs_request q = A.req[rl];
        n = img[L.o_fdesc + 4 * q.func + 1];
        B = A.slo[rl];
        const uint64_t fb = A.node_free[q.node];
        uint32_t av = 0;
#pragma unroll
        for (int p = 0; p < kP; ++p) av |= (((fb >> (8 * p)) & 255u) != 0u ? 1u : 0u) << p;
        go = A.gofs[q.func] + av * grp_stride(n);
      }
    }
    uint32_t todo = __ballot_sync(0xffffffffu, need);
    while (todo) {
      const int Lr = __ffs(todo) - 1;
      todo &= todo - 1;
      const uint32_t r = (uint32_t)r0 + Lr;
      const uint32_t nr = __shfl_sync(0xffffffffu, n, Lr), N1 = nr + 1;
      const uint32_t Br = __shfl_sync(0xffffffffu, B, Lr);
      const uint32_t* gp = A.grp + __shfl_sync(0xffffffffu, go, Lr);
      if constexpr (KS >= 3) {
        uint32_t* t = tab_all[warp];
        const uint32_t words = grp_stride(nr);
        __syncwarp();  // the previous request's readers are done
        for (uint32_t i = lane; i < words; i += 32) t[i] = gp[i];
        __syncwarp();
        gp = t;
      }
      const uint32_t* H0 = gp;
      const uint32_t* T3 = gp + N1;
      const uint32_t* R2 = gp + 2 * N1;
      const uint32_t* R3 = gp + 3 * N1;
      const uint32_t* Mt = gp + 4 * N1;
      const uint32_t h0 = lane + 1 < N1 ? H0[lane + 1] : 0u;  // W(0, b1) + X(b1) of j1 = lane
      if constexpr (KS == 2) {  // one row, masks j1 (b1 = j1 + 1): H0[b1] + T3[b1]
        const uint32_t j1 = lane;
        const bool live = j1 + 2 <= nr && live_owned(r, 0, j1, A.rank, A.world) &&
                          (uint64_t)h0 + T3[j1 + 1] <= Br;
        sg.row(__ballot_sync(0xffffffffu, live), 0u, r, lane);
      } else if constexpr (KS == 3) {
        // rows j2 (R2[b2] + T3[b2] <= B, lanes over j2), then the masks (j2, j1) of all
        // rows flattened over the lanes in colex order, 32 per step (a row-by-row walk
        // was a serial chain of up to 30 short steps per request)
        const uint32_t j2 = lane + 1;
        const bool valid = j2 + 2 <= nr && live_owned(r, 0, j2, A.rank, A.world);
        const uint32_t rc = valid ? T3[j2 + 1] : 0u;
        const uint32_t rows = __ballot_sync(0xffffffffu, valid && (uint64_t)R2[j2 + 1] + rc <= Br);
        if (rows) {
          // masks of the live rows' span j2 = jlo..jtop (rows bit b = j2 - 1)
          const uint32_t jlo = __ffs(rows), jtop = 32 - __clz(rows);
          const uint32_t tot = jtop * (jtop + 1) / 2;
          for (uint32_t t0 = jlo * (jlo - 1) / 2; t0 < tot; t0 += 32) {
            const uint32_t t = t0 + lane;
            const uint32_t tj = t < tot ? tri[t] : 0x0100u;
            const uint32_t m2 = tj >> 8, m1 = tj & 255u;  // (j2, j1), j1 < j2
            const uint32_t rcm = __shfl_sync(0xffffffffu, rc, (m2 - 1) & 31);
            const bool live = t < tot && ((rows >> (m2 - 1)) & 1u) &&
                              (uint64_t)H0[m1 + 1] + Mt[(m2 + 1) * N1 + m1 + 1] + rcm <= Br;
            sg.masks(__ballot_sync(0xffffffffu, live), (1u << m1) | (1u << m2), r, lane);
          }
        }
      } else {
        // blocks j3 (R3[b3] + T3[b3] <= B, lanes over j3); per live block its rows j2
        // (R2[b2] + Mt[b3][b2] + T3[b3] <= B, lanes over j2), then the block's masks
        // (j2, j1) flattened over the lanes in colex order, 32 per step
        const uint32_t j3 = lane + 2;
        uint32_t blocks = __ballot_sync(0xffffffffu, j3 + 2 <= nr && (uint64_t)R3[j3 + 1] + T3[j3 + 1] <= Br);
        const uint32_t r2 = lane + 2 < N1 ? R2[lane + 2] : 0u;  // R2[b2] of j2 = lane + 1
        while (blocks) {
          const uint32_t jb = __ffs(blocks) - 1 + 2;
          blocks &= blocks - 1;
          const uint32_t b3 = jb + 1, t3 = T3[b3];
          const uint32_t j2 = lane + 1;
          const bool valid = j2 < jb && live_owned(r, jb, j2, A.rank, A.world);
          const uint32_t rc = valid ? Mt[b3 * N1 + j2 + 1] + t3 : 0u;
          const uint32_t rows = __ballot_sync(0xffffffffu, valid && (uint64_t)r2 + rc <= Br);
          if (!rows) continue;
          const uint32_t jlo = __ffs(rows), jtop = 32 - __clz(rows);
          const uint32_t tot = jtop * (jtop + 1) / 2;
          for (uint32_t t0 = jlo * (jlo - 1) / 2; t0 < tot; t0 += 32) {
            const uint32_t t = t0 + lane;
            const uint32_t tj = t < tot ? tri[t] : 0x0100u;
            const uint32_t m2 = tj >> 8, m1 = tj & 255u;
            const uint32_t rcm = __shfl_sync(0xffffffffu, rc, (m2 - 1) & 31);
            const bool live = t < tot && ((rows >> (m2 - 1)) & 1u) &&
                              (uint64_t)H0[m1 + 1] + Mt[(m2 + 1) * N1 + m1 + 1] + rcm <= Br;
            sg.masks(__ballot_sync(0xffffffffu, live), (1u << m1) | (1u << m2) | (1u << jb), r, lane);
          }
        }
      }
      sg.end_request(r, lane);
    }
  }
  if (sg.cnt) sg.flush(sg.cnt, lane);
}

cudaError_t launch_live(const LiveArgs& a, int grid, cudaStream_t st) {
  if (a.per_grab < 1 || a.per_grab > 32) return cudaErrorInvalidValue;
  if (a.ks == 2) k_live<2><<<grid, 256, 0, st>>>(a);
  else if (a.ks == 3) k_live<3><<<grid, 256, 0, st>>>(a);
  else if (a.ks == 4) k_live<4><<<grid, 256, 0, st>>>(a);
  else return cudaErrorInvalidValue;
  return cudaGetLastError();
}

// ====================================================================================
// K2: decode + bind (A6) and time-share victim (A8)
// ====================================================================================
// per-(node, slice profile) minimum LRU score of one snapshot (A8 in ffs_plan_decode):
// a flat grid over the instances, 64-bit atomicMin into the table (~0 = empty)
__global__ void __launch_bounds__(256) k_vtab_snapshot(const ffs_instance* __restrict__ inst,
                                                       const int64_t* __restrict__ score, uint32_t n,
                                                       const uint16_t* __restrict__ slice_node,
                                                       const uint8_t* __restrict__ slice_prof, uint32_t n_slices,
                                                       unsigned long long* __restrict__ tab) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int64_t s = score[i];
    if ((uint64_t)s == kKeyNone) continue;
    const int32_t sl = inst[i].slice;
    if (sl < 0 || (uint32_t)sl >= n_slices) continue;
    atomicMin(tab + (uint32_t)slice_node[sl] * kP + slice_prof[sl], (unsigned long long)s);
  }
}

__device__ __forceinline__ void plan_init(ffs_plan& pl) {
  pl.key = (int64_t)kKeyNone;
  pl.status = FFS_PLAN_BAD_REQ;
  pl.k = pl.cut_mask = pl.e2e_us = pl.bottleneck_us = pl.gpcs = pl.cvq = 0;
#pragma unroll
  for (int i = 0; i < kMaxK; ++i) {
    pl.prof[i] = 0xFF;
    pl.slice[i] = -1;
  }
  pl.victim = -1;
}

// key -> (k, cut mask, profile digits) -> plan figures; slices are left to the caller.
__device__ __forceinline__ void plan_from_key(const uint32_t* img, const ImageLayout& L, uint32_t func,
                                              uint32_t k_max, int64_t key, ffs_plan& pl) {
  const uint32_t* fd = img + L.o_fdesc + 4 * func;
  const uint32_t row0 = fd[0], n = fd[1];
  pl.status = FFS_PLAN_OK;
  pl.key = key;
  const uint64_t idx = (uint64_t)key & ((1ull << kIdxBits) - 1);
  const uint32_t kmax = k_max < n ? k_max : n;
  uint32_t k = 1;
  while (k < kmax && img_u64(img, L.o_offk + 2 * (n * 10 + k + 1)) <= idx) ++k;
  uint64_t PK = 1;
  for (uint32_t i = 0; i < k; ++i) PK *= kP;
  const uint64_t rem = idx - img_u64(img, L.o_offk + 2 * (n * 10 + k));
  uint64_t rank = rem / PK, seq = rem % PK;
  uint32_t mask = 0;
  int cc = (int)n - 2;
  for (int i = (int)k - 1; i >= 1; --i) {
    while (img[L.o_binom + cc * 8 + i] > rank) --cc;
    mask |= 1u << cc;
    rank -= img[L.o_binom + cc * 8 + i];
    --cc;
  }
  for (int i = (int)k - 1; i >= 0; --i) {
    pl.prof[i] = (uint8_t)(seq % kP);
    seq /= kP;
  }
  uint32_t a = 0, e2e = 0, bott = 0, g = 0, m = mask;
  for (uint32_t i = 0; i < k; ++i) {
    uint32_t b = n;
    if (i + 1 < k) {
      const int j = __ffs(m) - 1;
      m &= m - 1;
      b = j + 1;
      e2e += img[L.o_xf + row0 + j];
    }
    const int p = pl.prof[i];
    const uint32_t t = pl_diff(img, L.o_pl + (row0 + b) * kRowW + p, L.o_pl + (row0 + a) * kRowW + p);
    e2e += t;
    bott = t > bott ? t : bott;
    g += img[L.o_gpcs + p];
    a = b;
  }
  pl.k = k;
  pl.cut_mask = mask;
  pl.e2e_us = e2e;
  pl.bottleneck_us = bott;  // throughput = 1e6 / bottleneck (R17)
  pl.gpcs = g;
  pl.cvq = (uint32_t)((uint64_t)key >> 50);
}

__global__ void k_decode(const __grid_constant__ DecodeArgs A) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= A.n_req) return;
  const uint32_t* img = A.image;
  const ImageLayout& L = A.lay;
  ffs_plan pl;
  plan_init(pl);
  const ffs_request q = A.req[r];
  if (q.func < L.F && q.node < A.n_nodes) {
    const int64_t key = A.keys[r];
    if ((uint64_t)key == kKeyNone) {
      pl.status = FFS_PLAN_INFEASIBLE;
      if (A.inst) {
        // A8: the least recently used evictable instance on the node whose slice can
        // host the function monolithically within the budget: the minimum over the request's
        // admissible profiles of the per-(node, profile) minima (k_vtab_snapshot; the score's
        // low 20 bits are the instance index)
        const uint32_t okp = victim_profiles(img, L, q.func, A.slo[r]);
        unsigned long long bs = ~0ull;
#pragma unroll
        for (int p = 0; p < kP; ++p)
          if ((okp >> p) & 1u) bs = min(bs, A.vtab[(uint64_t)q.node * kP + p]);
        pl.victim = bs == ~0ull ? -1 : (int32_t)(bs & 0xFFFFFull);
      }
    } else {
      plan_from_key(img, L, q.func, A.k_max, key, pl);
      uint32_t used[kP] = {0, 0, 0, 0, 0};
      for (uint32_t i = 0; i < pl.k; ++i) {
        const int p = pl.prof[i];
        uint32_t u = 0;
#pragma unroll
        for (int x = 0; x < kP; ++x)
          if (x == p) u = used[x]++;
        pl.slice[i] = A.free_list[((uint64_t)q.node * 8 + p) * 8 + u];  // R11 binding
      }
    }
  }
  A.out[r] = pl;
}

// ====================================================================================
// K7 (NEXT-2): joint commit in monotone rounds
// ====================================================================================
// state: 0 pending (key valid for the current free state), 1 dirty (re-plan), 2 final
__device__ __forceinline__ uint64_t joint_order(const uint32_t* img, const ImageLayout& L, const ffs_request& q,
                                                uint32_t B, uint32_t r) {
  // adjusted deadline = B - load - fastest 1-stage latency (R28), biased to be >= 0, then index
  const uint32_t* fd = img + L.o_fdesc + 4 * q.func;
  const uint32_t row0 = fd[0], n = fd[1];
  uint32_t fast = 0xFFFFFFFFu;
#pragma unroll
  for (int p = 0; p < kP; ++p) {
    const uint32_t t = pl_diff(img, L.o_pl + (row0 + n) * kRowW + p, L.o_pl + row0 * kRowW + p);
    fast = t < fast ? t : fast;
  }
  const int64_t adj = (int64_t)B - (int64_t)fd[2] - (int64_t)fast + (1ll << 26);  // >= 0: load, fast < 2^26
  return ((uint64_t)adj << 31) | r;
}

__global__ void k_joint_init(const __grid_constant__ JointArgs A) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= A.n_req) return;
  const ffs_request q = A.req[r];
  if (q.func < A.lay.F && q.node < A.n_nodes) {
    A.state[r] = 1;  // plan in round 0
    A.dirty[r] = r;
  } else {
    ffs_plan pl;
    plan_init(pl);
    A.out[r] = pl;
    A.state[r] = 2;
    A.dirty[r] = r;  // planned harmlessly in round 0 (BAD_REQ keys are ignored)
  }
}

__global__ void k_joint_gather(const __grid_constant__ JointArgs A, uint32_t n) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t r = A.dirty[i];
  A.sub_req[i] = A.req[r];
  A.sub_slo[i] = A.slo[r];
}

__global__ void k_joint_scatter(const __grid_constant__ JointArgs A, uint32_t n_sub) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n_sub) A.keys[A.dirty[i]] = A.sub_keys[i];  // re-planned keys back to their requests
}

__global__ void k_joint_pick(const __grid_constant__ JointArgs A) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= A.n_req || A.state[r] == 2) return;
  if ((uint64_t)A.keys[r] == kKeyNone) return;
  const ffs_request q = A.req[r];
  atomicMin(reinterpret_cast<unsigned long long*>(A.node_win + q.node),
            (unsigned long long)joint_order(A.image, A.lay, q, A.slo[r], r));
}

// one thread per node: commit the earliest-deadline feasible request, bind its slices to
// the lowest-index free slices of its profiles in stage order, take them
__global__ void k_joint_commit(const __grid_constant__ JointArgs A) {
  const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
  if (v >= A.n_nodes) return;
  const uint64_t w = A.node_win[v];
  if (w == ~0ull) return;
  const uint32_t r = (uint32_t)(w & 0x7FFFFFFFu);
  const ffs_request q = A.req[r];
  ffs_plan pl;
  plan_init(pl);
  plan_from_key(A.image, A.lay, q.func, A.k_max, A.keys[r], pl);
  uint8_t* cnt = A.cnt + (uint64_t)v * 8;
  for (uint32_t i = 0; i < pl.k; ++i) {
    const uint32_t p = pl.prof[i];
    for (uint32_t s = A.node_off[v]; s < A.node_off[v + 1]; ++s)
      if (!A.busy[s] && A.slice_prof[s] == p) {
        A.busy[s] = 1;
        pl.slice[i] = (int32_t)s;
        cnt[p]--;
        break;
      }
  }
  uint64_t nf = 0;
  for (int p = 0; p < 8; ++p) nf |= (uint64_t)(cnt[p] < 8 ? cnt[p] : 8) << (8 * p);
  A.node_free[v] = nf;
  A.out[r] = pl;
  A.state[r] = 2;
}

// per request: infeasible -> final; a pending plan that no longer fits the node's counts
// -> dirty (appended to the re-plan list); counts the requests still open
__global__ void k_joint_finalize(const __grid_constant__ JointArgs A) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= A.n_req || A.state[r] == 2) return;
  const ffs_request q = A.req[r];
  const int64_t key = A.keys[r];
  if ((uint64_t)key == kKeyNone) {  // the free state only shrinks: stays infeasible
    ffs_plan pl;
    plan_init(pl);
    pl.status = FFS_PLAN_INFEASIBLE;
    A.out[r] = pl;
    A.state[r] = 2;
    return;
  }
  uint8_t st = 0;
  if (A.node_win[q.node] != ~0ull) {  // the node committed this round: does the plan still fit?
    ffs_plan pl;
    plan_from_key(A.image, A.lay, q.func, A.k_max, key, pl);
    uint32_t used[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (uint32_t i = 0; i < pl.k; ++i) used[pl.prof[i] & 7]++;
    const uint8_t* cnt = A.cnt + (uint64_t)q.node * 8;
    for (int p = 0; p < 8; ++p)
      if (used[p] > cnt[p]) st = 1;
  }
  A.state[r] = st;
  atomicAdd(A.n_open, 1u);
  if (st == 1) A.dirty[atomicAdd(A.n_dirty, 1u)] = r;
}

cudaError_t launch_joint(int phase, const JointArgs& a, uint32_t n, cudaStream_t st) {
  const uint32_t T = 256;
  switch (phase) {
    case 0: k_joint_init<<<(a.n_req + T - 1) / T, T, 0, st>>>(a); break;
    case 1: if (n) k_joint_gather<<<(n + T - 1) / T, T, 0, st>>>(a, n); break;
    case 2: if (n) k_joint_scatter<<<(n + T - 1) / T, T, 0, st>>>(a, n); break;
    case 3: k_joint_pick<<<(a.n_req + T - 1) / T, T, 0, st>>>(a); break;
    case 4: k_joint_commit<<<(a.n_nodes + T - 1) / T, T, 0, st>>>(a); break;
    case 5: k_joint_finalize<<<(a.n_req + T - 1) / T, T, 0, st>>>(a); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_decode(const DecodeArgs& a, unsigned long long* vtab, cudaStream_t st) {
  if (a.n_req == 0) return cudaSuccess;
  DecodeArgs b = a;
  if (a.inst) {  // victims: the snapshot's per-(node, profile) minima first (O(n_inst + n_req))
    cudaError_t e = cudaMemsetAsync(vtab, 0xFF, (size_t)a.n_nodes * kP * 8, st);
    if (e != cudaSuccess) return e;
    if (a.n_inst)
      k_vtab_snapshot<<<(a.n_inst + 255) / 256, 256, 0, st>>>(a.inst, a.score, a.n_inst, a.slice_node, a.slice_prof,
                                                             a.n_slices, vtab);
    b.vtab = vtab;
  }
  k_decode<<<(a.n_req + 127) / 128, 128, 0, st>>>(b);
  return cudaGetLastError();
}

// ====================================================================================
// K3: hotness-aware eviction score (A7)
// ====================================================================================
__device__ __forceinline__ int64_t evict_one(const ffs_instance& in, uint32_t i, uint64_t now,
                                             const ffs_evict_params& p, int64_t* score, uint8_t* state, uint64_t gi) {
  const uint64_t idle = now >= in.last_used_us ? now - in.last_used_us : 0;
  uint8_t st;
  if (idle >= p.cold_after_us) st = FFS_ST_COLD;
  else if (in.slice < 0) st = FFS_ST_WARM;
  else if ((in.flags & FFS_INST_PIPELINE) || (uint64_t)in.busy_us * 100u >= (uint64_t)p.util_thr_pct * p.window_us)
    st = FFS_ST_EXCL_HOT;
  else st = FFS_ST_TIME_SHARING;
  // LRU key (R20c): the least recently used instance has the largest idle time;
  // a time-sharing instance has idle < cold_after_us < 2^43 (host-checked), so
  // (cold_after - idle) packs into 43 bits whatever the timestamps' epoch
  const bool evictable = st == FFS_ST_TIME_SHARING && !(in.flags & FFS_INST_BUSY) && i < (1u << 20);
  const int64_t sc = evictable ? (int64_t)(((p.cold_after_us - idle) << 20) | i) : (int64_t)kKeyNone;
  score[gi] = sc;
  state[gi] = st;
  return sc;
}

// one CTA per tick; kEvU records in flight per thread (memory-level parallelism).  (A flat
// persistent grid with a per-record binary search of the tick measured 1.7x slower.)
#ifndef FFS_EVT
#define FFS_EVT 128
#endif
#ifndef FFS_EVU
#define FFS_EVU 5  // 640 >= the ~582 instances of a C4 tick: one round of loads per CTA (0.545 -> 0.567 of the copy peak)
#endif
constexpr int kEvT = FFS_EVT, kEvU = FFS_EVU;
// TAB (ffs_evict_step): the CTA also folds every scored instance into the tick's
// (node, slice profile) minima in shared memory (64-bit atomicMin) and writes that row of
// the victim table once -- the victim pass then reads <= 5 cells per load instead of
// re-reading the tick's scores and records.  ~0 marks an empty cell.

// PICK (loads grouped by tick, d_load_off): the tick's loads take their victims from the
// shared-memory minima right away -- no table in device memory, one launch for the step.
struct EvictPick {
  const uint32_t* image;
  ImageLayout lay;
  const ffs_request* req;
  const uint32_t* slo;
  const uint32_t* load_off;  // [n_ticks + 1] loads of tick t: [load_off[t], load_off[t+1])
  int32_t* victim;
};

template <bool TAB, bool PICK = false>
__global__ void __launch_bounds__(kEvT) k_evict_ticks(const ffs_instance* __restrict__ inst,
                                                       const uint32_t* __restrict__ tick_off,
                                                       const uint64_t* __restrict__ now_us, ffs_evict_params prm,
                                                       int64_t* __restrict__ score, uint8_t* __restrict__ state,
                                                       const uint16_t* __restrict__ slice_node,
                                                       const uint8_t* __restrict__ slice_prof, uint32_t n_slices,
                                                       uint32_t n_nodes, unsigned long long* __restrict__ tab,
                                                       EvictPick pk = EvictPick{}) {
  extern __shared__ unsigned long long cell[];
  const uint32_t t = blockIdx.x;
  const uint32_t b = tick_off[t], e = tick_off[t + 1];
  const uint64_t now = now_us[t];
  const uint32_t ncell = n_nodes * kP;
  if constexpr (TAB) {
    for (uint32_t i = threadIdx.x; i < ncell; i += kEvT) cell[i] = ~0ull;
    __syncthreads();
  }
  // PICK: the first kEvT loads of the tick (one per thread) resolve their request, node and
  // monolithic profiles before the scoring pass, so those dependent loads overlap it; only
  // the minimum over the finished cells waits for the barrier
  uint32_t p_okp = 0, p_node = 0;
  if constexpr (TAB && PICK) {
    const uint32_t r = pk.load_off[t] + threadIdx.x;
    if (r < pk.load_off[t + 1]) {
      const ffs_request q = pk.req[r];
      if (q.func < pk.lay.F && q.node < n_nodes) {
        p_okp = victim_profiles(pk.image, pk.lay, q.func, pk.slo[r]);
        p_node = q.node;
      }
    }
  }
  for (uint32_t g0 = b + threadIdx.x; g0 < e; g0 += kEvT * kEvU) {
    ffs_instance in[kEvU];
#pragma unroll
    for (int u = 0; u < kEvU; ++u)
      if (g0 + u * kEvT < e) in[u] = inst[g0 + u * kEvT];
#pragma unroll
    for (int u = 0; u < kEvU; ++u) {
      const uint32_t gi = g0 + u * kEvT;
      if (gi < e) {
        const int64_t sc = evict_one(in[u], gi - b, now, prm, score, state, gi);
        if (TAB && (uint64_t)sc != kKeyNone) {
          const int32_t sl = in[u].slice;
          if (sl >= 0 && (uint32_t)sl < n_slices)
            atomicMin(cell + (uint32_t)slice_node[sl] * kP + slice_prof[sl], (unsigned long long)sc);
        }
      }
    }
  }
  if constexpr (TAB && !PICK) {
    __syncthreads();
    unsigned long long* row = tab + (uint64_t)t * ncell;
    for (uint32_t i = threadIdx.x; i < ncell; i += kEvT) row[i] = cell[i];
  }
  if constexpr (TAB && PICK) {  // this tick's loads: the minimum over their monolithic profiles' cells
    __syncthreads();
    const uint32_t lb = pk.load_off[t], le = pk.load_off[t + 1];
    if (lb + threadIdx.x < le) {
      unsigned long long bs = ~0ull;
#pragma unroll
      for (int p = 0; p < kP; ++p)
        if ((p_okp >> p) & 1u) bs = min(bs, cell[p_node * kP + p]);
      pk.victim[lb + threadIdx.x] = bs == ~0ull ? -1 : (int32_t)(bs & 0xFFFFFull);
    }
    for (uint32_t r = lb + kEvT + threadIdx.x; r < le; r += kEvT) {
      const ffs_request q = pk.req[r];
      unsigned long long bs = ~0ull;
      if (q.func < pk.lay.F && q.node < n_nodes) {
        const uint32_t okp = victim_profiles(pk.image, pk.lay, q.func, pk.slo[r]);
#pragma unroll
        for (int p = 0; p < kP; ++p)
          if ((okp >> p) & 1u) bs = min(bs, cell[q.node * kP + p]);
      }
      pk.victim[r] = bs == ~0ull ? -1 : (int32_t)(bs & 0xFFFFFull);
    }
  }
}

__global__ void __launch_bounds__(256) k_evict_one(const ffs_instance* __restrict__ inst, uint32_t n, uint64_t now,
                                                    ffs_evict_params prm, int64_t* __restrict__ score,
                                                    uint8_t* __restrict__ state) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const ffs_instance in = inst[i];
    evict_one(in, i, now, prm, score, state, i);
  }
}

cudaError_t launch_evict(const ffs_instance* inst, uint32_t n_inst, const uint32_t* tick_off, const uint64_t* now_us,
                         uint32_t n_ticks, uint64_t now_single, ffs_evict_params prm, int64_t* score, uint8_t* state,
                         cudaStream_t st) {
  if (tick_off) {
    if (n_ticks)
      k_evict_ticks<false><<<n_ticks, kEvT, 0, st>>>(inst, tick_off, now_us, prm, score, state, nullptr, nullptr, 0,
                                                     0, nullptr);
  } else if (n_inst) {
    int blocks = (int)((n_inst + 255) / 256);
    k_evict_one<<<blocks, 256, 0, st>>>(inst, n_inst, now_single, prm, score, state);
  }
  return cudaGetLastError();
}

// ====================================================================================
// K4: victims per request over its tick's instances (A8)
// ====================================================================================
// Profiles whose slice can host request (f, B) monolithically: the whole function fits
// the slice memory and latency alone + reload <= B (R19).
__device__ __forceinline__ uint32_t victim_profiles(const uint32_t* img, const ImageLayout& L, uint32_t f,
                                                    uint32_t B) {  // (declared above k_evict_ticks)
  const uint32_t* fd = img + L.o_fdesc + 4 * f;
  const uint32_t row0 = fd[0], n = fd[1];
  uint32_t ok = 0;
#pragma unroll
  for (int p = 0; p < kP; ++p) {
    const uint64_t lat = pl_diff(img, L.o_pl + (row0 + n) * kRowW + p, L.o_pl + row0 * kRowW + p);
    if (fd[3] <= img[L.o_cap + p] && lat + fd[2] <= B && lat <= img[L.o_thr + f]) ok |= 1u << p;
  }
  return ok;
}

// one warp per load: lanes scan the tick's instances, warp min of the packed score
constexpr int kViT = 256;
__global__ void __launch_bounds__(kViT) k_victims(const uint32_t* __restrict__ img, ImageLayout L,
                                                   const ffs_request* __restrict__ req, const uint32_t* __restrict__ slo,
                                                   const uint32_t* __restrict__ req_tick, uint32_t n_req,
                                                   uint32_t n_ticks, const ffs_instance* __restrict__ inst,
                                                   const uint32_t* __restrict__ tick_off,
                                                   const int64_t* __restrict__ score, const uint16_t* slice_node,
                                                   const uint8_t* slice_prof, uint32_t n_slices,
                                                   int32_t* __restrict__ victim) {
  const uint32_t r = (blockIdx.x * kViT + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (r >= n_req) return;
  const ffs_request q = req[r];
  int64_t bs = (int64_t)kKeyNone;
  uint32_t b = 0, e = 0;
  const uint32_t t = req_tick[r];
  if (q.func < L.F && t < n_ticks) {
    const uint32_t okp = victim_profiles(img, L, q.func, slo[r]);
    b = tick_off[t];
    e = tick_off[t + 1];
    for (uint32_t i = b + lane; i < e; i += 32) {
      const int64_t s = score[i];
      if ((uint64_t)s == kKeyNone || s >= bs) continue;
      const int32_t sl = inst[i].slice;
      if (sl < 0 || (uint32_t)sl >= n_slices || slice_node[sl] != q.node || !((okp >> slice_prof[sl]) & 1u)) continue;
      bs = s;
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const int64_t y = __shfl_xor_sync(0xffffffffu, bs, o);
    bs = y < bs ? y : bs;
  }
  // the packed score's low 20 bits are the index within the tick (R20b)
  if (lane == 0) victim[r] = (uint64_t)bs == kKeyNone ? -1 : (int32_t)((uint64_t)bs & 0xFFFFFu);
}

// Table variant: the minimum packed score per (tick, node, slice profile) is built once
// per tick (one CTA per tick, 64-bit atomicMin), then each load takes the minimum over its
// monolithic profiles -- at most 5 reads instead of a scan of the whole tick.  Scores are
// unique within a tick (low 20 bits = index), so the minimum of the per-profile minima is
// the same victim.  UINT64_MAX marks an empty cell (FFS_KEY_NONE scores are skipped).
__global__ void __launch_bounds__(256) k_victim_table(const ffs_instance* __restrict__ inst,
                                                      const uint32_t* __restrict__ tick_off,
                                                      const int64_t* __restrict__ score,
                                                      const uint16_t* __restrict__ slice_node,
                                                      const uint8_t* __restrict__ slice_prof, uint32_t n_slices,
                                                      uint32_t n_nodes, unsigned long long* __restrict__ tab) {
  const uint32_t t = blockIdx.x, b = tick_off[t], e = tick_off[t + 1];
  unsigned long long* row = tab + (uint64_t)t * n_nodes * kP;
  for (uint32_t i = b + threadIdx.x; i < e; i += blockDim.x) {
    const int64_t s = score[i];
    if ((uint64_t)s == kKeyNone) continue;
    const int32_t sl = inst[i].slice;
    if (sl < 0 || (uint32_t)sl >= n_slices) continue;
    atomicMin(row + (uint32_t)slice_node[sl] * kP + slice_prof[sl], (unsigned long long)s);
  }
}

__global__ void __launch_bounds__(256) k_victim_pick(const uint32_t* __restrict__ img, ImageLayout L,
                                                     const ffs_request* __restrict__ req,
                                                     const uint32_t* __restrict__ slo,
                                                     const uint32_t* __restrict__ req_tick, uint32_t n_req,
                                                     uint32_t n_ticks, uint32_t n_nodes,
                                                     const unsigned long long* __restrict__ tab,
                                                     int32_t* __restrict__ victim) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= n_req) return;
  const ffs_request q = req[r];
  const uint32_t t = req_tick[r];
  unsigned long long bs = ~0ull;
  if (q.func < L.F && q.node < n_nodes && t < n_ticks) {
    const uint32_t okp = victim_profiles(img, L, q.func, slo[r]);
    const unsigned long long* cell = tab + ((uint64_t)t * n_nodes + q.node) * kP;
#pragma unroll
    for (int p = 0; p < kP; ++p)
      if ((okp >> p) & 1u) bs = min(bs, cell[p]);
  }
  victim[r] = bs == ~0ull ? -1 : (int32_t)(bs & 0xFFFFFull);
}

// ffs_evict_step: scores + states + the per-tick victim table in one pass, then the picks
cudaError_t launch_evict_step(const uint32_t* image, const ImageLayout& lay, const ffs_instance* inst,
                              const uint32_t* tick_off, const uint64_t* now_us, uint32_t n_ticks, ffs_evict_params prm,
                              int64_t* score, uint8_t* state, const uint16_t* slice_node, const uint8_t* slice_prof,
                              uint32_t n_slices, uint32_t n_nodes, unsigned long long* tab, const ffs_request* req,
                              const uint32_t* slo, const uint32_t* req_tick, const uint32_t* load_off, uint32_t n_req,
                              int32_t* victim, cudaStream_t st) {
  const size_t sm = (size_t)n_nodes * kP * 8;
  if (load_off && n_ticks) {  // loads grouped by tick: picks inside the tick's CTA, one launch
    if (sm > 48 * 1024) {
      cudaError_t e = cudaFuncSetAttribute(k_evict_ticks<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           (int)sm);
      if (e != cudaSuccess) return e;
    }
    EvictPick pk{image, lay, req, slo, load_off, victim};
    k_evict_ticks<true, true><<<n_ticks, kEvT, sm, st>>>(inst, tick_off, now_us, prm, score, state, slice_node,
                                                         slice_prof, n_slices, n_nodes, nullptr, pk);
    return cudaGetLastError();
  }
  if (n_ticks) {
    if (sm > 48 * 1024) {
      cudaError_t e = cudaFuncSetAttribute(k_evict_ticks<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
      if (e != cudaSuccess) return e;
    }
    k_evict_ticks<true><<<n_ticks, kEvT, sm, st>>>(inst, tick_off, now_us, prm, score, state, slice_node, slice_prof,
                                                   n_slices, n_nodes, tab);
  }
  if (n_req)
    k_victim_pick<<<(n_req + 255) / 256, 256, 0, st>>>(image, lay, req, slo, req_tick, n_req, n_ticks, n_nodes, tab,
                                                       victim);
  return cudaGetLastError();
}

cudaError_t launch_victims(const uint32_t* image, const ImageLayout& lay, const ffs_request* req, const uint32_t* slo,
                           const uint32_t* req_tick, uint32_t n_req, const ffs_instance* inst,
                           const uint32_t* tick_off, const int64_t* score, uint32_t n_ticks,
                           const uint16_t* slice_node, const uint8_t* slice_prof, uint32_t n_slices,
                           uint32_t n_nodes, unsigned long long* tab, int32_t* victim, cudaStream_t st) {
  if (n_req == 0) return cudaSuccess;
  if (tab && n_ticks > 0) {
    cudaError_t e = cudaMemsetAsync(tab, 0xFF, (size_t)n_ticks * n_nodes * kP * 8, st);
    if (e != cudaSuccess) return e;
    k_victim_table<<<n_ticks, 256, 0, st>>>(inst, tick_off, score, slice_node, slice_prof, n_slices, n_nodes, tab);
    k_victim_pick<<<(n_req + 255) / 256, 256, 0, st>>>(image, lay, req, slo, req_tick, n_req, n_ticks, n_nodes, tab,
                                                       victim);
    return cudaGetLastError();
  }
  const uint64_t threads = (uint64_t)n_req * 32;
  k_victims<<<(unsigned)((threads + kViT - 1) / kViT), kViT, 0, st>>>(image, lay, req, slo, req_tick, n_req, n_ticks,
                                                                       inst, tick_off, score, slice_node, slice_prof,
                                                                       n_slices, victim);
  return cudaGetLastError();
}

// ====================================================================================
// K6 (NEXT-1): the paper's ranked first-fit walk, one warp per request
// ====================================================================================
// Lanes test 32 consecutive ranked partitions at once; the warp stops at the first
// chunk with a supported partition and takes its lowest rank (ballot + ffs), which is
// exactly the sequential first fit.
struct RankedEval {
  uint32_t k, e2e, bott, gpcs, cvq;
  int prof[kMaxK];
};

__device__ __forceinline__ bool ranked_eval(const RankedArgs& A, uint32_t row0, uint32_t n, uint32_t mask,
                                            uint64_t freeb, uint32_t B, uint32_t thr, RankedEval& out) {
  const uint32_t* img = A.image;
  const ImageLayout& L = A.lay;
  const uint32_t k = __popc(mask) + 1;
  uint32_t bnd[kMaxK + 1], mem[kMaxK];
  bnd[0] = 0;
  uint32_t m = mask, X = 0;
  for (uint32_t i = 1; i < k; ++i) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    bnd[i] = j + 1;
    X += img[L.o_xf + row0 + j];
  }
  bnd[k] = n;
  for (uint32_t i = 0; i < k; ++i) mem[i] = img[L.o_pm + row0 + bnd[i + 1]] - img[L.o_pm + row0 + bnd[i]];
  // min-resource greedy: stages by descending memory (ties: lower stage), each takes the
  // first profile in (capacity, gpcs, id) order with a free slice left that holds it and
  // runs it within the throughput floor (R38)
  uint32_t left[kP];
#pragma unroll
  for (int p = 0; p < kP; ++p) left[p] = (uint32_t)(freeb >> (8 * p)) & 255u;
  uint32_t done = 0;
  for (uint32_t step = 0; step < k; ++step) {
    int s = -1;
    for (uint32_t i = 0; i < k; ++i)
      if (!((done >> i) & 1u) && (s < 0 || mem[i] > mem[s])) s = (int)i;
    done |= 1u << s;
    int got = -1;
#pragma unroll
    for (int oi = 0; oi < kP; ++oi) {
      const int p = (int)((A.prof_order >> (4 * oi)) & 15u);
      bool ok = false;
#pragma unroll
      for (int q = 0; q < kP; ++q)
        if (q == p) ok = left[q] > 0;
      if (got < 0 && ok && mem[s] <= img[L.o_cap + p] &&
          pl_diff(img, L.o_pl + (row0 + bnd[s + 1]) * kRowW + p, L.o_pl + (row0 + bnd[s]) * kRowW + p) <= thr) {
        got = p;
#pragma unroll
        for (int q = 0; q < kP; ++q)
          if (q == p) left[q]--;
      }
    }
    if (got < 0) return false;
    out.prof[s] = got;
  }
  uint64_t St = 0, Sq = 0;
  uint32_t bott = 0, g = 0;
  for (uint32_t i = 0; i < k; ++i) {
    const int p = out.prof[i];
    const uint32_t t = pl_diff(img, L.o_pl + (row0 + bnd[i + 1]) * kRowW + p, L.o_pl + (row0 + bnd[i]) * kRowW + p);
    St += t;
    Sq += (uint64_t)t * t;
    bott = t > bott ? t : bott;
    g += img[L.o_gpcs + p];
  }
  if (St + X > (uint64_t)B) return false;
  out.k = k;
  out.e2e = (uint32_t)(St + X);
  out.bott = bott;
  out.gpcs = g;
  const uint64_t D = St * St, N = (uint64_t)k * Sq - D;
  out.cvq = (uint32_t)((N << 10) / D);
  return true;
}

constexpr int kRkT = 128;
// 12 CTAs of 128 threads per SM (40 registers): one warp per request walking its ranked
// list is latency-bound, more warps win (C5: 10.4 / 7.9 / 7.6 / 7.5 ms at 1 / 8 / 12 / 16)
#ifndef FFS_RANKED_MINB
#define FFS_RANKED_MINB 12
#endif
__global__ void __launch_bounds__(kRkT, FFS_RANKED_MINB) k_plan_ranked(const __grid_constant__ RankedArgs A) {
  const uint32_t r = (blockIdx.x * kRkT + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (r >= A.n_req) return;
  const uint32_t* img = A.image;
  const ImageLayout& L = A.lay;
  const ffs_request q = A.req[r];
  ffs_plan pl;
  pl.key = (int64_t)kKeyNone;
  pl.status = FFS_PLAN_BAD_REQ;
  pl.k = pl.cut_mask = pl.e2e_us = pl.bottleneck_us = pl.gpcs = pl.cvq = 0;
#pragma unroll
  for (int i = 0; i < kMaxK; ++i) {
    pl.prof[i] = 0xFF;
    pl.slice[i] = -1;
  }
  pl.victim = -1;
  if (q.func < L.F && q.node < A.n_nodes) {
    pl.status = FFS_PLAN_INFEASIBLE;
    const uint32_t* fd = img + L.o_fdesc + 4 * q.func;
    const uint32_t row0 = fd[0], n = fd[1], B = A.slo[r];
    const uint64_t freeb = A.node_free[q.node];
    const uint32_t off = A.rank_off[q.func], cnt = A.rank_off[q.func + 1] - off;
    for (uint32_t base = 0; base < cnt; base += 32) {
      const uint32_t j = base + lane;
      RankedEval ev;
      uint32_t mask = 0;
      bool ok = false;
      if (j < cnt) {
        mask = A.rank_mask[off + j];
        ok = ranked_eval(A, row0, n, mask, freeb, B, img[L.o_thr + q.func], ev);
      }
      const uint32_t bal = __ballot_sync(0xffffffffu, ok);
      if (bal) {
        const uint32_t w = __ffs(bal) - 1;
        if (lane == w) {
          pl.status = FFS_PLAN_OK;
          pl.key = (int64_t)(base + w);
          pl.k = ev.k;
          pl.cut_mask = mask;
          pl.e2e_us = ev.e2e;
          pl.bottleneck_us = ev.bott;
          pl.gpcs = ev.gpcs;
          pl.cvq = ev.cvq;
          uint32_t used[kP] = {0, 0, 0, 0, 0};
          for (uint32_t i = 0; i < ev.k; ++i) {
            const int p = ev.prof[i];
            pl.prof[i] = (uint8_t)p;
            uint32_t u = 0;
#pragma unroll
            for (int x = 0; x < kP; ++x)
              if (x == p) u = used[x]++;
            pl.slice[i] = A.free_list[((uint64_t)q.node * 8 + p) * 8 + u];  // R11 binding
          }
          A.out[r] = pl;
        }
        return;
      }
    }
  }
  if (lane == 0) A.out[r] = pl;
}

cudaError_t launch_ranked(const RankedArgs& a, cudaStream_t st) {
  const uint64_t threads = (uint64_t)a.n_req * 32;
  k_plan_ranked<<<(unsigned)((threads + kRkT - 1) / kRkT), kRkT, 0, st>>>(a);
  return cudaGetLastError();
}

// ====================================================================================
// K8 (NEXT-3): frontier build (peeling rounds) and frontier queries
// ====================================================================================
// synthetic requests of the active groups: function g / n_fv on a node with free-vector
// g % n_fv (a representative node), budget = the group's current budget
__global__ void k_front_gather(const __grid_constant__ FrontierArgs A, uint32_t n_active,
                               const uint32_t* __restrict__ fv_node, uint32_t* __restrict__ gslo) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n_active) return;
  const uint32_t g = A.active[i];
  ffs_request q;
  q.func = g / A.n_fv;
  q.node = fv_node[g % A.n_fv];
  A.greq[i] = q;
  gslo[i] = A.budget[g];
}

// record this round's frontier point of every active group; groups with a point stay
// active with budget e2e - 1
__global__ void k_front_record(const __grid_constant__ FrontierArgs A, uint32_t n_active) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n_active) return;
  const uint32_t g = A.active[i];
  const int64_t key = A.keys[i];
  if ((uint64_t)key == kKeyNone) return;
  ffs_plan pl;
  plan_from_key(A.image, A.lay, g / A.n_fv, A.k_max, key, pl);
  const uint64_t at = (uint64_t)A.round * A.n_groups + g;
  A.fr_key[at] = key;
  A.fr_e2e[at] = pl.e2e_us;
  A.fr_cnt[g] = A.round + 1;
  if (pl.e2e_us > 0) {
    A.budget[g] = pl.e2e_us - 1;
    A.next_active[atomicAdd(A.n_next, 1u)] = g;
  }
}

// one thread per request: the first frontier point (lowest key) with e2e <= B; the
// points of a group have increasing keys and strictly decreasing e2e
__global__ void k_front_query(const __grid_constant__ FrontierArgs A) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= A.n_req) return;
  ffs_plan pl;
  plan_init(pl);
  const ffs_request q = A.req[r];
  if (q.func < A.lay.F && q.node < A.n_nodes) {
    const uint32_t g = q.func * A.n_fv + A.node_fv[q.node];
    const uint32_t B = A.slo[r];
    uint32_t lo = 0, hi = A.fr_cnt[g];  // first i in [lo, hi) with e2e_i <= B
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (A.fr_e2e[(uint64_t)mid * A.n_groups + g] <= B) hi = mid; else lo = mid + 1;
    }
    if (lo == A.fr_cnt[g]) {
      pl.status = FFS_PLAN_INFEASIBLE;
    } else {
      plan_from_key(A.image, A.lay, q.func, A.k_max, A.fr_key[(uint64_t)lo * A.n_groups + g], pl);
      uint32_t used[kP] = {0, 0, 0, 0, 0};
      for (uint32_t i = 0; i < pl.k; ++i) {
        const int p = pl.prof[i];
        uint32_t u = 0;
#pragma unroll
        for (int x = 0; x < kP; ++x)
          if (x == p) u = used[x]++;
        pl.slice[i] = A.free_list[((uint64_t)q.node * 8 + p) * 8 + u];
      }
    }
  }
  A.out[r] = pl;
}

// first frontier point of group g with e2e <= B (the argmin for budget B), or KEY_NONE
__device__ __forceinline__ int64_t front_lookup(const FrontierArgs& A, uint32_t g, uint32_t B) {
  uint32_t lo = 0, hi = A.fr_cnt[g];
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (A.fr_e2e[(uint64_t)mid * A.n_groups + g] <= B) hi = mid; else lo = mid + 1;
  }
  return lo == A.fr_cnt[g] ? (int64_t)kKeyNone : A.fr_key[(uint64_t)lo * A.n_groups + g];
}

// NEXT-2 any-invoker query (R39): one warp per request, lanes over the function's
// free-vector classes; min of (key, class != home class, lowest node of the class)
__global__ void __launch_bounds__(256) k_front_query_any(const __grid_constant__ FrontierArgs A) {
  const uint32_t r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (r >= A.n_req) return;
  const ffs_request q = A.req[r];
  const bool valid = q.func < A.lay.F && q.node < A.n_nodes;
  int64_t bk = (int64_t)kKeyNone;
  uint32_t bt = 0xffffffffu;  // tiebreak: (class != home class) << 31 | node
  if (valid) {
    const uint32_t home = A.node_fv[q.node], B = A.slo[r];
    for (uint32_t c = lane; c < A.n_fv; c += 32) {
      const int64_t k = front_lookup(A, q.func * A.n_fv + c, B);
      const uint32_t t = (c == home) ? q.node : (0x80000000u | A.fv_node[c]);
      if (k < bk || (k == bk && t < bt)) {
        bk = k;
        bt = t;
      }
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const int64_t k2 = __shfl_xor_sync(0xffffffffu, bk, o);
    const uint32_t t2 = __shfl_xor_sync(0xffffffffu, bt, o);
    if (k2 < bk || (k2 == bk && t2 < bt)) {
      bk = k2;
      bt = t2;
    }
  }
  if (lane) return;
  ffs_plan pl;
  plan_init(pl);
  int32_t node = -1;
  if (valid) {
    if ((uint64_t)bk == kKeyNone) {
      pl.status = FFS_PLAN_INFEASIBLE;
    } else {
      node = (int32_t)(bt & 0x7fffffffu);
      plan_from_key(A.image, A.lay, q.func, A.k_max, bk, pl);
      uint32_t used[kP] = {0, 0, 0, 0, 0};
      for (uint32_t i = 0; i < pl.k; ++i) {
        const int p = pl.prof[i];
        uint32_t u = 0;
#pragma unroll
        for (int x = 0; x < kP; ++x)
          if (x == p) u = used[x]++;
        pl.slice[i] = A.free_list[((uint64_t)node * 8 + p) * 8 + u];
      }
    }
  }
  A.out[r] = pl;
  if (A.node_out) A.node_out[r] = node;
}

cudaError_t launch_frontier(int phase, const FrontierArgs& a, uint32_t n, cudaStream_t st) {
  const uint32_t T = 256;
  if (phase == 1 && n) k_front_record<<<(n + T - 1) / T, T, 0, st>>>(a, n);
  if (phase == 2 && a.n_req) k_front_query<<<(a.n_req + T - 1) / T, T, 0, st>>>(a);
  if (phase == 3 && a.n_req) k_front_query_any<<<(uint32_t)(((uint64_t)a.n_req * 32 + T - 1) / T), T, 0, st>>>(a);
  return cudaGetLastError();
}
cudaError_t launch_front_gather(const FrontierArgs& a, uint32_t n, const uint32_t* fv_node, uint32_t* gslo,
                                cudaStream_t st) {
  if (n) k_front_gather<<<(n + 255) / 256, 256, 0, st>>>(a, n, fv_node, gslo);
  return cudaGetLastError();
}

// ====================================================================================
// Stable LSD radix sort of (u64 key, u32 value) pairs, 8-bit digits (NEXT-2 routing)
// ====================================================================================
constexpr int kRsT = 256, kRsWarps = kRsT / 32, kRsItems = 8, kRsTile = kRsT * kRsItems;  // 2048

// per (digit, block) counts, digit-major so that one exclusive scan gives stable offsets
__global__ void __launch_bounds__(kRsT) k_rs_hist(const uint64_t* __restrict__ key, uint32_t n, int shift,
                                                   uint64_t* __restrict__ hist, uint32_t nb) {
  __shared__ uint32_t h[256];
  h[threadIdx.x] = 0;
  __syncthreads();
  const uint64_t base = (uint64_t)blockIdx.x * kRsTile;
  for (int i = threadIdx.x; i < kRsTile; i += kRsT)
    if (base + i < n) atomicAdd(&h[(key[base + i] >> shift) & 255u], 1u);
  __syncthreads();
  hist[(uint64_t)threadIdx.x * nb + blockIdx.x] = h[threadIdx.x];
}

// stable scatter: warp w owns the contiguous quarter-chunk [w*256, (w+1)*256) of the tile
__global__ void __launch_bounds__(kRsT) k_rs_scatter(const uint64_t* __restrict__ key, const uint32_t* __restrict__ val,
                                                      uint32_t n, int shift, const uint64_t* __restrict__ off,
                                                      uint32_t nb, uint64_t* __restrict__ key_out,
                                                      uint32_t* __restrict__ val_out) {
  __shared__ uint32_t wh[kRsWarps][256];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int d = threadIdx.x; d < kRsWarps * 256; d += kRsT) (&wh[0][0])[d] = 0;
  __syncthreads();
  const uint64_t base = (uint64_t)blockIdx.x * kRsTile + (uint64_t)w * (32 * kRsItems);
  // pass 1: per-warp digit counts
  for (int it = 0; it < kRsItems; ++it) {
    const uint64_t i = base + it * 32 + lane;
    const bool in = i < n;
    const uint32_t d = in ? (uint32_t)((key[i] >> shift) & 255u) : 256u + lane;
    const uint32_t m = __match_any_sync(0xffffffffu, d);
    if (in && lane == __ffs(m) - 1) wh[w][d] += __popc(m);
    __syncwarp();  // the next iteration's leader of the same digit may be another lane
  }
  __syncthreads();
  // exclusive prefix over warps per digit, plus the global offset of (digit, block)
  {
    const uint32_t d = threadIdx.x;  // kRsT == 256 digits
    uint32_t run = (uint32_t)off[(uint64_t)d * nb + blockIdx.x];
    for (int ww = 0; ww < kRsWarps; ++ww) {
      const uint32_t c = wh[ww][d];
      wh[ww][d] = run;
      run += c;
    }
  }
  __syncthreads();
  // pass 2: scatter in order
  for (int it = 0; it < kRsItems; ++it) {
    const uint64_t i = base + it * 32 + lane;
    const bool in = i < n;
    const uint64_t k = in ? key[i] : 0;
    const uint32_t d = in ? (uint32_t)((k >> shift) & 255u) : 256u + lane;
    const uint32_t m = __match_any_sync(0xffffffffu, d);
    if (in) {
      const uint32_t pos = wh[w][d] + __popc(m & ((1u << lane) - 1));
      key_out[pos] = k;
      val_out[pos] = val[i];
    }
    __syncwarp();
    if (in && lane == __ffs(m) - 1) wh[w][d] += __popc(m);
    __syncwarp();
  }
}

// sorts (key, val) by the low `bits` bits of key, stably; result in key/val (ping-pong
// through key2/val2); hist needs 256 * ceil(n / 2048) + 1 entries, bsum scan scratch
cudaError_t radix_sort_pairs(uint64_t* key, uint32_t* val, uint64_t* key2, uint32_t* val2, uint32_t n, int bits,
                             uint64_t* hist, uint64_t* bsum, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const uint32_t nb = (n + kRsTile - 1) / kRsTile;
  const uint64_t len = (uint64_t)256 * nb;
  const uint32_t sb = (uint32_t)((len + kScanChunk - 1) / kScanChunk);
  for (int shift = 0; shift < bits; shift += 8) {
    k_rs_hist<<<nb, kRsT, 0, st>>>(key, n, shift, hist, nb);
    k_scan_reduce<<<dim3(sb, 1), kScanT, 0, st>>>(hist, len, bsum, sb);
    k_scan_top<<<1, kScanT, 0, st>>>(bsum, sb);
    k_scan_apply<<<dim3(sb, 1), kScanT, 0, st>>>(hist, len, bsum, sb);
    k_rs_scatter<<<nb, kRsT, 0, st>>>(key, val, n, shift, hist, nb, key2, val2);
    uint64_t* tk = key; key = key2; key2 = tk;
    uint32_t* tv = val; val = val2; val2 = tv;
  }
  // an odd number of passes leaves the result in the second buffers: copy back
  if (((bits + 7) / 8) & 1) {
    cudaMemcpyAsync(key2, key, (size_t)n * 8, cudaMemcpyDeviceToDevice, st);
    cudaMemcpyAsync(val2, val, (size_t)n * 4, cudaMemcpyDeviceToDevice, st);
  }
  return cudaGetLastError();
}

// ====================================================================================
// K9 (NEXT-2 routing)
// ====================================================================================
__global__ void k_route_keys(const __grid_constant__ RouteArgs A) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < A.n_req) {
    const ffs_request q = A.req[i];
    const uint32_t f = q.func < A.lay.F ? q.func : A.lay.F;  // invalid functions sort last
    const uint64_t adj = q.func < A.lay.F ? (joint_order(A.image, A.lay, q, A.slo[i], 0) >> 31) : 0;
    A.rkey[i] = ((uint64_t)f << 34) | adj;  // adj < 2^34 (joint_order biases it non-negative)
    A.rval[i] = i;
    A.route[i] = -1;
  }
  if (i < A.n_inst) {
    const uint32_t f = A.inst[i].func < A.lay.F ? A.inst[i].func : A.lay.F;
    const bool hot = A.state[i] == FFS_ST_EXCL_HOT;
    // non-hot instances sort after every hot one of their function
    A.ikey[i] = ((uint64_t)f << 33) | ((uint64_t)(hot ? 0u : 1u) << 32) | A.lat[i];
    A.ival[i] = i;
  }
  if (i <= A.lay.F) {
    A.first_req[i] = 0xFFFFFFFFu;
    A.first_hot[i] = 0xFFFFFFFFu;
    A.n_hot[i] = 0;
    A.ts[i] = 0x7FFFFFFF;
  }
}

__global__ void k_route_marks(const __grid_constant__ RouteArgs A) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < A.n_req) atomicMin(A.first_req + (uint32_t)(A.rkey[i] >> 34), i);
  if (i < A.n_inst) {
    const uint32_t j = A.ival[i];  // sorted position i holds instance j
    const uint32_t f = (uint32_t)(A.ikey[i] >> 33);
    if (f < A.lay.F) {
      if (A.state[j] == FFS_ST_EXCL_HOT) {
        atomicMin(A.first_hot + f, i);
        atomicAdd(A.n_hot + f, 1u);
        A.icap[i] = A.cap[j];
      } else {
        A.icap[i] = 0;
        if (A.state[j] == FFS_ST_TIME_SHARING || A.state[j] == FFS_ST_WARM) atomicMin(A.ts + f, (int32_t)j);
      }
    } else {
      A.icap[i] = 0;
    }
  }
}

// request at sorted position i with rank j within its function: the instance whose
// cumulative capacity range covers j, else the time-sharing instance
__global__ void k_route_assign(const __grid_constant__ RouteArgs A) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= A.n_req) return;
  const uint32_t f = (uint32_t)(A.rkey[i] >> 34);
  const uint32_t r = A.rval[i];
  if (f >= A.lay.F) return;
  const uint64_t j = i - A.first_req[f];
  int32_t out = A.ts[f] == 0x7FFFFFFF ? -1 : A.ts[f];
  const uint32_t h0 = A.first_hot[f], nh = A.n_hot[f];
  if (nh) {
    const uint64_t c0 = A.icum[h0];
    if (j < A.icum[h0 + nh] - c0) {
      uint32_t lo = 0, hi = nh;  // first l with icum[h0 + l + 1] - c0 > j
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (A.icum[h0 + mid + 1] - c0 > j) hi = mid; else lo = mid + 1;
      }
      out = (int32_t)A.ival[h0 + lo];
    }
  }
  A.route[r] = out;
}

cudaError_t launch_route(int phase, const RouteArgs& a, cudaStream_t st) {
  const uint32_t n = std::max(std::max(a.n_req, a.n_inst), a.lay.F + 1);
  const uint32_t T = 256;
  if (phase == 0) k_route_keys<<<(n + T - 1) / T, T, 0, st>>>(a);
  if (phase == 1) k_route_marks<<<(n + T - 1) / T, T, 0, st>>>(a);
  if (phase == 2 && a.n_req) k_route_assign<<<(a.n_req + T - 1) / T, T, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t scan_u64(uint64_t* a, uint64_t len, uint64_t* bsum, cudaStream_t st) {
  const uint32_t sb = (uint32_t)((len + kScanChunk - 1) / kScanChunk);
  k_scan_reduce<<<dim3(sb, 1), kScanT, 0, st>>>(a, len, bsum, sb);
  k_scan_top<<<1, kScanT, 0, st>>>(bsum, sb);
  k_scan_apply<<<dim3(sb, 1), kScanT, 0, st>>>(a, len, bsum, sb);
  return cudaGetLastError();
}

// ====================================================================================
// K10 (NEXT-4): time-sharing simulator, one warp per node
// ====================================================================================

// Warp-wide exact argmin of function f's candidates against free counts `freeb` (8 x u8)
// and budget B (R44: the pipeline a new instance is built as): the masks walked in colex
// order by the whole warp, the lanes over the profile sequences; exact integer scoring as
// exact_eval (memory, floor, free slices, SLO, cvq), packed key (R1).  Returns the key.
__device__ int64_t warp_plan_argmin(const uint32_t* img, const ImageLayout& L, uint32_t f, uint64_t freeb,
                                    uint32_t B, uint32_t K, uint32_t lane) {
  const uint32_t* fd = img + L.o_fdesc + 4 * f;
  const uint32_t row0 = fd[0], n = fd[1];
  const uint32_t thr = img[L.o_thr + f];
  int64_t best = (int64_t)kKeyNone;
  const uint32_t kk = min(K, n);
  for (uint32_t k = 1; k <= kk; ++k) {
    uint32_t pk = 1;
    for (uint32_t i = 0; i < k; ++i) pk *= kP;
    const uint64_t off = img_u64(img, L.o_offk + 2 * (n * 10 + k));
    const uint32_t nm = binom(img, L, n - 1, k - 1);
    uint32_t mask = (1u << (k - 1)) - 1;
    for (uint32_t rk = 0; rk < nm; ++rk, mask = (k > 1 ? gosper_next(mask) : 0u)) {
      // stage bounds of the mask (warp-uniform)
      uint32_t bnd[kMaxK + 1];
      bnd[0] = 0;
      uint32_t m = mask, X = 0;
      for (uint32_t i = 1; i < k; ++i) {
        const uint32_t j = __ffs(m) - 1;
        m &= m - 1;
        bnd[i] = j + 1;
        X += img[L.o_xf + row0 + j];
      }
      bnd[k] = n;
      if (X > B) continue;
      for (uint32_t seq = lane; seq < pk; seq += 32) {
        uint32_t rest = seq, used = 0, g = 0;
        uint64_t St = 0, Sq = 0;
        bool ok = true;
        for (int i = (int)k - 1; i >= 0; --i) {  // digits, stage 0 most significant
          const uint32_t pr = rest % kP;
          rest /= kP;
          const uint32_t t = pl_diff(img, L.o_pl + (row0 + bnd[i + 1]) * kRowW + pr, L.o_pl + (row0 + bnd[i]) * kRowW + pr);
          ok &= img[L.o_pm + row0 + bnd[i + 1]] - img[L.o_pm + row0 + bnd[i]] <= img[L.o_cap + pr];
          ok &= t <= thr;
          St += t;
          Sq += (uint64_t)t * t;
          used += 1u << (4 * pr);
          g += img[L.o_gpcs + pr];
        }
#pragma unroll
        for (int pp = 0; pp < kP; ++pp) ok &= ((used >> (4 * pp)) & 15u) <= ((freeb >> (8 * pp)) & 255u);
        ok &= St + X <= (uint64_t)B;
        if (!ok) continue;
        const uint64_t D = St * St, N = (uint64_t)k * Sq - D;
        const uint64_t cvq = (N << 10) / D;  // floor(1024 CV^2), exact (R4)
        const int64_t key = (int64_t)((cvq << 50) | ((uint64_t)(k - 1) << 47) | ((uint64_t)g << 41) | (off + rk * pk + seq));
        best = key < best ? key : best;
      }
    }
  }
  return (int64_t)warp_min_u64((uint64_t)best);
}

__global__ void __launch_bounds__(128) k_simulate(const __grid_constant__ SimArgs A) {
  const uint32_t v = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (v >= A.n_nodes) return;
  const uint32_t* img = A.image;
  const ImageLayout& L = A.lay;
  const uint32_t F = L.F, s0 = A.node_off[v], s1 = A.node_off[v + 1];
  int32_t* sl = A.slice + (uint64_t)v * F;
  uint64_t* last = A.last + (uint64_t)v * F;
  uint32_t* busy = A.busy + (uint64_t)v * F;
  uint8_t* fl = A.flags + (uint64_t)v * F;
  uint8_t* pk = A.pk + (uint64_t)v * F;
  int32_t* psl = A.psl + (uint64_t)v * F * 8;
  uint32_t* pe2e = A.pe2e + (uint64_t)v * F;
  for (uint32_t f = lane; f < F; f += 32) {
    sl[f] = -1;
    last[f] = 0;
    busy[f] = 0;
    fl[f] = 0;
    pk[f] = 0;
  }
  for (uint32_t s = s0 + lane; s < s1; s += 32) A.res[s] = -1;
  uint64_t c_req = 0, c_srv = 0, c_hit = 0, c_uns = 0, c_rel = 0, c_evi = 0, c_ter = 0, c_occ = 0;
  uint64_t c_pip = 0, c_mig = 0, c_psrv = 0, c_pocc = 0;
  const uint64_t window_us = (uint64_t)A.window_ticks * A.tick_us;
  __syncwarp();
  // smallest (capacity, gpcs, id) free slice of the node holding memt MiB, ~0 if none
  auto free_fit = [&](uint32_t memt) {
    uint64_t best = ~0ull;
    for (uint32_t s = s0 + lane; s < s1; s += 32) {
      const uint32_t p = A.slice_prof[s];
      if (!A.slice_busy[s] && A.res[s] < 0 && memt <= img[L.o_cap + p])
        best = min(best, ((uint64_t)img[L.o_cap + p] << 40) | ((uint64_t)img[L.o_gpcs + p] << 32) | s);
    }
    return warp_min_u64(best);
  };
  for (uint32_t t = 0; t < A.n_ticks; ++t) {
    const uint64_t now = A.t0_us + (uint64_t)t * A.tick_us;
    const uint32_t j0 = A.req_off[(uint64_t)v * A.n_ticks + t], j1 = A.req_off[(uint64_t)v * A.n_ticks + t + 1];
    for (uint32_t j = j0; j < j1; ++j) {
      const uint32_t f = A.req_func[j];
      const uint64_t B = A.req_budget[j];
      const uint32_t* fd = img + L.o_fdesc + 4 * f;
      const uint32_t row0 = fd[0], n = fd[1], load = fd[2], memt = fd[3];
      ++c_req;
      if (lane == 0 && !(fl[f] & 1u)) {  // created on its first request, warm
        fl[f] = 1;
        sl[f] = -1;
        busy[f] = 0;
        last[f] = now;
      }
      __syncwarp();
      int32_t at = sl[f];
      uint64_t latency = 0, ex = 0;
      bool served = false;
      if (at < 0 && pk[f] >= 2) {  // resident pipeline (R45)
        ex = pe2e[f];
        latency = ex;
        served = true;
        ++c_psrv;
      } else if (at < 0) {
        uint64_t best = free_fit(memt);
        if (best == ~0ull && A.k_max >= 2) {
          // a pipeline over the node's free slices: the argmin plan for this budget (R44)
          uint32_t cnt[kP] = {0, 0, 0, 0, 0};
          for (uint32_t s = s0; s < s1; ++s)
            if (!A.slice_busy[s] && A.res[s] < 0) ++cnt[A.slice_prof[s]];
          uint64_t freeb = 0;
#pragma unroll
          for (int p = 0; p < kP; ++p) freeb |= (uint64_t)min(cnt[p], 8u) << (8 * p);
          if (freeb) {
            const int64_t key = warp_plan_argmin(img, L, f, freeb, (uint32_t)min(B, (uint64_t)0xffffffffull), A.k_max, lane);
            if ((uint64_t)key != kKeyNone) {
              // decode (as k_decode): k, mask rank, profile digits; bind stage i to the
              // lowest-index free slice of its profile not taken by an earlier stage (R11)
              const uint64_t idx = (uint64_t)key & ((1ull << kIdxBits) - 1);
              const uint32_t k = (uint32_t)(((uint64_t)key >> 47) & 7) + 1;
              uint32_t pkk = 1;
              for (uint32_t i = 0; i < k; ++i) pkk *= kP;
              const uint64_t rel = idx - img_u64(img, L.o_offk + 2 * (n * 10 + k));
              uint64_t rk = rel / pkk;
              uint32_t seq = (uint32_t)(rel % pkk);
              uint32_t mask = 0;
              int cc = (int)n - 2;
              for (int i = (int)k - 1; i >= 1; --i) {  // colex unrank
                while (binom(img, L, cc, i) > rk) --cc;
                mask |= 1u << cc;
                rk -= binom(img, L, cc, i);
                --cc;
              }
              uint32_t prof[kMaxK];
              for (int i = (int)k - 1; i >= 0; --i) {
                prof[i] = seq % kP;
                seq /= kP;
              }
              uint32_t e2e = 0, a0 = 0;
              uint32_t mm = mask;
              for (uint32_t i = 0; i < k; ++i) {
                uint32_t b1 = n;
                if (i + 1 < k) {
                  const uint32_t jj = __ffs(mm) - 1;
                  mm &= mm - 1;
                  b1 = jj + 1;
                  e2e += img[L.o_xf + row0 + jj];
                }
                e2e += pl_diff(img, L.o_pl + (row0 + b1) * kRowW + prof[i], L.o_pl + (row0 + a0) * kRowW + prof[i]);
                a0 = b1;
              }
              if (lane == 0) {
                for (uint32_t i = 0; i < k; ++i) {
                  for (uint32_t s = s0; s < s1; ++s) {
                    if (A.slice_busy[s] || A.res[s] >= 0 || A.slice_prof[s] != prof[i]) continue;
                    A.res[s] = (int32_t)f;  // taken: later stages skip it
                    psl[f * 8 + i] = (int32_t)s;
                    break;
                  }
                }
                pk[f] = (uint8_t)k;
                pe2e[f] = e2e;
              }
              __syncwarp();
              ++c_pip;
              ++c_rel;
              ++c_psrv;
              ex = e2e;
              latency = (uint64_t)load + e2e;
              served = true;
            }
          }
        }
        if (!served && best == ~0ull) {  // LRU time-sharing victim not used in this tick
          for (uint32_t s = s0 + lane; s < s1; s += 32) {
            const int32_t g = A.res[s];
            if (g < 0 || (uint32_t)g == f || pk[g] >= 2 || (fl[g] & 2u) || last[g] >= now) continue;
            if (memt > img[L.o_cap + A.slice_prof[s]]) continue;
            best = min(best, (last[g] << 20) | (s - s0));
          }
          best = warp_min_u64(best);
          if (best != ~0ull) {
            const uint32_t s = s0 + (uint32_t)(best & 0xFFFFFu);
            if (lane == 0) {
              sl[A.res[s]] = -1;  // evicted to CPU memory: warm
              A.res[s] = -1;
            }
            ++c_evi;
            best = s;
          }
        } else if (!served) {
          best &= 0xFFFFFFFFull;
        }
        if (!served && best != ~0ull) {
          at = (int32_t)best;
          if (lane == 0) {
            A.res[at] = (int32_t)f;
            sl[f] = at;
          }
          ++c_rel;
          latency = load;
        }
      }
      if (!served && at >= 0) {
        const uint32_t p = A.slice_prof[at];
        ex = pl_diff(img, L.o_pl + (row0 + n) * kRowW + p, L.o_pl + row0 * kRowW + p);
        latency += ex;
        served = true;
      }
      if (served) {
        ++c_srv;
        c_hit += latency <= B;
        if (lane == 0) {
          busy[f] += (uint32_t)ex;
          last[f] = now;
        }
      } else {
        ++c_uns;
      }
      __syncwarp();
    }
    // end of tick: occupied slices, utilisation windows, cold terminations, migrations
    uint32_t occ = 0, pocc = 0;
    for (uint32_t s = s0 + lane; s < s1; s += 32) {
      const int32_t g = A.res[s];
      occ += g >= 0;
      pocc += g >= 0 && pk[g] >= 2;
    }
    uint32_t ter = 0;
    const bool roll = (t + 1) % A.window_ticks == 0;
    for (uint32_t f = lane; f < F; f += 32) {
      uint8_t x = fl[f];
      if (roll) {
        x = (uint8_t)((x & 1u) | (((uint64_t)busy[f] * 100u >= (uint64_t)A.thr_pct * window_us) ? 2u : 0u));
        busy[f] = 0;
      }
      if ((x & 1u) && now - last[f] >= A.cold_after_us) {
        if (sl[f] >= 0) A.res[sl[f]] = -1;
        for (uint32_t i = 0; i < pk[f]; ++i) A.res[psl[f * 8 + i]] = -1;
        pk[f] = 0;
        sl[f] = -1;
        busy[f] = 0;
        x = 0;
        ++ter;
      }
      fl[f] = x;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      occ += __shfl_xor_sync(0xffffffffu, occ, o);
      pocc += __shfl_xor_sync(0xffffffffu, pocc, o);
      ter += __shfl_xor_sync(0xffffffffu, ter, o);
    }
    c_occ += occ;
    c_pocc += pocc;
    c_ter += ter;
    __syncwarp();
    // pipeline migration (R46), function order
    for (uint32_t f0 = 0; f0 < F; f0 += 32) {
      uint32_t has = __ballot_sync(0xffffffffu, f0 + lane < F && pk[f0 + lane] >= 2);
      while (has) {
        const uint32_t f = f0 + __ffs(has) - 1;
        has &= has - 1;
        const uint64_t best = free_fit(img[L.o_fdesc + 4 * f + 3]);
        if (best == ~0ull) continue;
        if (lane == 0) {
          for (uint32_t i = 0; i < pk[f]; ++i) A.res[psl[f * 8 + i]] = -1;
          pk[f] = 0;
          A.res[(uint32_t)best] = (int32_t)f;
          sl[f] = (int32_t)(uint32_t)best;
        }
        __syncwarp();
        ++c_mig;
        ++c_rel;
      }
    }
  }
  for (uint32_t f = lane; f < F; f += 32) {
    const uint8_t x = fl[f];
    const bool pipe = pk[f] >= 2;
    A.state[(uint64_t)v * F + f] = !(x & 1u) ? FFS_ST_COLD
                                   : pipe ? FFS_ST_EXCL_HOT
                                   : (sl[f] < 0 ? FFS_ST_WARM : ((x & 2u) ? FFS_ST_EXCL_HOT : FFS_ST_TIME_SHARING));
    A.stages[(uint64_t)v * F + f] = pipe ? pk[f] : (sl[f] >= 0 ? 1 : 0);
    if (pipe) sl[f] = psl[f * 8];
  }
  if (lane == 0) {
    uint64_t* C = A.ctr + (uint64_t)v * 12;
    C[0] = c_req; C[1] = c_srv; C[2] = c_hit; C[3] = c_uns;
    C[4] = c_rel; C[5] = c_evi; C[6] = c_ter; C[7] = c_occ;
    C[8] = c_pip; C[9] = c_mig; C[10] = c_psrv; C[11] = c_pocc;
  }
}

cudaError_t launch_sim(const SimArgs& a, cudaStream_t st) {
  const uint64_t threads = (uint64_t)a.n_nodes * 32;
  k_simulate<<<(unsigned)((threads + 127) / 128), 128, 0, st>>>(a);
  return cudaGetLastError();
}

// ====================================================================================
// K5: integer issue-rate microbenchmark (roofline denominator)
// ====================================================================================
constexpr int kPeakIters = 4096, kPeakReps = 16;
__global__ void __launch_bounds__(256) k_int_peak(uint32_t seed, uint32_t* out) {
  // 8 independent chains of IADD3 / LOP3 / IMAD: 3 integer lane-ops per chain step.
  uint32_t a[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) a[i] = seed + threadIdx.x * 7 + i * 13;
  const uint32_t k1 = seed | 1, k2 = seed ^ 0x5bd1e995u;
#pragma unroll 1
  for (int it = 0; it < kPeakIters; ++it) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        a[i] = a[i] + k1 + (uint32_t)u;         // IADD3
        a[i] = (a[i] ^ k2) & (a[i] | 0x1234u);  // LOP3
        a[i] = a[i] * 0x9E3779B1u + k1;          // IMAD
      }
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s ^= a[i];
  if (s == 0x12345678u) out[0] = s;  // keep the work alive
}

cudaError_t run_int_peak(int sms, double* ops, double* seconds) {
  uint32_t* d = nullptr;
  cudaError_t e = cudaMalloc(&d, 4);
  if (e != cudaSuccess) return e;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int blocks = sms * 8;  // 2048 threads per SM
  // ~100 ms of warm-up so the SM clock has ramped from idle, then 16 timed launches
  for (int i = 0; i < 32; ++i) k_int_peak<<<blocks, 256>>>(1u, d);
  cudaEventRecord(a);
  for (int i = 0; i < kPeakReps; ++i) k_int_peak<<<blocks, 256>>>(2u, d);
  cudaEventRecord(b);
  e = cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(d);
  if (e != cudaSuccess) return e;
  // 3 ops per chain step; IADD3 with an immediate counts 1, LOP3 1, IMAD 1
  *ops = (double)kPeakReps * blocks * 256.0 * kPeakIters * 4 * 8 * 3 / (ms * 1e-3);
  *seconds = ms * 1e-3;
  return cudaGetLastError();
}

// Packed f16x2 issue-rate microbenchmark (roofline denominator of the KS = 4 pre-filter,
// DESIGN.md §5).  mode 0: eight independent HFMA2 chains (the FMA-pipe rate of the packed
// datapath); mode 1: eight HFMA2 chains interleaved with eight independent LOP3 chains (ALU
// pipe); mode 2: the same with packed max (HMNMX2) on the ALU side -- modes 1 and 2 measure
// the issue-limited rate, one warp-instruction per SMSP per clock at best.
template <int MODE>
__global__ void __launch_bounds__(256) k_packed_peak(uint32_t seed, uint32_t* out) {
  uint32_t h[8], m[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    h[i] = 0x3c003c00u ^ ((seed + threadIdx.x + i) & 0x00ff00ffu);
    m[i] = h[i] ^ 0x04000400u;
  }
  const uint32_t a = 0x3bff3bffu ^ (seed & 1u), b = 0x10001000u | (seed & 2u), c = 0x12340000u ^ seed;
#pragma unroll 1
  for (int it = 0; it < kPeakIters; ++it) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        asm volatile("fma.rn.f16x2 %0, %0, %1, %2;" : "+r"(h[i]) : "r"(a), "r"(b));
        if (MODE == 1) asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(m[i]) : "r"(a), "r"(c));
        if (MODE == 2) asm volatile("max.f16x2 %0, %0, %1;" : "+r"(m[i]) : "r"(c));
      }
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s ^= h[i] ^ m[i];
  if (s == 0x12345678u) out[0] = s;
}

cudaError_t run_packed_peak(int sms, int mode, double* lane_instr_per_s, double* seconds) {
  uint32_t* d = nullptr;
  cudaError_t e = cudaMalloc(&d, 4);
  if (e != cudaSuccess) return e;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int blocks = sms * 8;  // 2048 threads per SM
  auto launch = [&](uint32_t seed) {
    if (mode == 0) k_packed_peak<0><<<blocks, 256>>>(seed, d);
    else if (mode == 1) k_packed_peak<1><<<blocks, 256>>>(seed, d);
    else k_packed_peak<2><<<blocks, 256>>>(seed, d);
  };
  for (int i = 0; i < 32; ++i) launch(1u);  // ~100 ms warm-up: clocks ramped from idle
  cudaEventRecord(a);
  for (int i = 0; i < kPeakReps; ++i) launch(2u);
  cudaEventRecord(b);
  e = cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(d);
  if (e != cudaSuccess) return e;
  const double per_step = mode == 0 ? 1.0 : 2.0;  // lane-instructions per chain step
  *lane_instr_per_s = (double)kPeakReps * blocks * 256.0 * kPeakIters * 4 * 8 * per_step / (ms * 1e-3);
  *seconds = ms * 1e-3;
  return cudaGetLastError();
}

// ====================================================================================
// K11 (NEXT-1): DAG stages (R40-R43)
// ====================================================================================
// One warp per request; lane l takes the function's mask-table entries l, l+32, ...
// (unit-cut masks in candidate order with their first candidate index) and scores every
// stage-option combination of its mask exactly in integers: stage times from the prefix
// rows of the table image (one slice: the run's component range; split: per branch, max),
// memory per slice, the throughput floor, free slices as a SWAR byte compare against the
// node's clamped counts (a plan holds <= 8 slices, so the clamp at 8 is exact), SLO,
// cvq = floor(1024 (k Q - T^2) / T^2) in u64 (T < 2^24: every stage is at most its
// one-slice sum).  Warp argmin of the packed keys; the winning lane writes and binds.
constexpr int kDagT = 128;

__device__ __forceinline__ uint32_t dag_lat(const DagArgs& A, const uint32_t* img, uint32_t row0, uint32_t a,
                                            uint32_t b, uint32_t p) {
  return __float2uint_rn(plf(img, A.lay.o_pl + (row0 + b) * kRowW + p) - plf(img, A.lay.o_pl + (row0 + a) * kRowW + p));
}

// options of the stage made of units [u0, u1]: P, plus P^nb splits when it is one
// fork/join block (a conditional unit's alternatives never split, R48; uo[6u] = nb |
// cond << 8)
__device__ __forceinline__ uint32_t dag_nopt(const uint32_t* uo, uint32_t u0, uint32_t u1) {
  const uint32_t nb = uo[6 * u0] & 0xffu;
  if (u0 != u1 || nb < 2 || (uo[6 * u0] >> 8)) return kP;
  uint32_t q = 1;
  for (uint32_t j = 0; j < nb; ++j) q *= kP;
  return kP + q;
}

// Score option o of the stage [u0, u1] (uo = the function's units): adds its time t,
// GPCs and per-profile slice counts, clears ok on a memory / floor miss; returns t.
// A split's branch profiles are the base-P digits of o - P, branch 0 most significant
// (sums and max are order-free, so the digits are taken least significant first).
__device__ __forceinline__ uint32_t dag_stage(const DagArgs& A, const uint32_t* img, uint32_t row0, const uint32_t* uo,
                                              uint32_t u0, uint32_t u1, uint32_t o, uint32_t thr, uint32_t& gp,
                                              uint64_t& use, bool& ok, const uint32_t* sv) {
  const uint32_t* U0 = uo + 6 * u0;
  uint32_t t;
  if (o < (uint32_t)kP) {
    const uint32_t* U1 = uo + 6 * u1;
    const uint32_t c0 = U0[1], c1 = U1[1 + (U1[0] & 0xffu)];  // end of the last branch of unit u1
    // every component in sequence, minus the conditional units' sum - max (R48)
    t = dag_lat(A, img, row0, c0, c1, o) - (sv[8 * (u1 + 1) + o] - sv[8 * u0 + o]);
    ok &= img[A.lay.o_pm + row0 + c1] - img[A.lay.o_pm + row0 + c0] <= img[A.lay.o_cap + o];
    gp += img[A.lay.o_gpcs + o];
    use += 1ull << (8 * o);
  } else {
    const uint32_t nb = U0[0] & 0xffu;
    uint32_t w = o - kP;
    t = 0;
    for (uint32_t jj = nb; jj > 0; --jj) {
      const uint32_t j = jj - 1, p = w % kP;
      w /= kP;
      const uint32_t c = U0[1 + j], e = U0[2 + j];  // branch j = [end of branch j-1 (or c0), e)
      t = max(t, dag_lat(A, img, row0, c, e, p));
      ok &= img[A.lay.o_pm + row0 + e] - img[A.lay.o_pm + row0 + c] <= img[A.lay.o_cap + p];
      gp += img[A.lay.o_gpcs + p];
      use += 1ull << (8 * p);
    }
  }
  ok &= t <= thr;
  return t;
}

// stage s of a mask: units [u0, u1] from the packed last units (4 bits per stage)
__device__ __forceinline__ void dag_bounds(uint32_t ends, uint32_t s, uint32_t& u0, uint32_t& u1) {
  u1 = (ends >> (4 * s)) & 15u;
  u0 = s ? ((ends >> (4 * (s - 1))) & 15u) + 1 : 0;
}

// one request, the whole warp (img: the table image, staged in shared memory)
template <bool VERIFY>
__device__ __forceinline__ void dag_request(const DagArgs& A, const uint32_t* img, uint32_t r) {
  const uint32_t lane = threadIdx.x & 31;
  const ffs_request q = A.req[r];
  ffs_dag_plan* out = A.out + r;
  const bool bad = q.func >= A.lay.F || q.node >= A.n_nodes;
  const uint32_t f = bad ? 0 : q.func, v = bad ? 0 : q.node;
  const uint32_t row0 = img[A.lay.o_fdesc + 4 * f];
  const uint32_t thr = img[A.lay.o_thr + f];
  const uint32_t B = A.slo[r];
  const uint64_t nf = A.node_free[v];
  const uint32_t* uo = A.units + 6 * A.fu[2 * f];
  const uint32_t m = A.fu[2 * f + 1];
  const uint32_t* xc = A.xcut + A.fu[2 * f];
  const uint32_t* sv = A.sv + 8 * (A.fu[2 * f] + f);
  uint64_t best = kKeyNone, scored = 0, nfeas = 0, ksum = 0;
  uint32_t best_mk = 0, best_c = 0;
  uint32_t gpc[kP];
#pragma unroll
  for (int x = 0; x < kP; ++x) gpc[x] = img[A.lay.o_gpcs + x];
  // The warp walks the function's masks together (uniform control flow: k, the stage
  // bounds and option counts are the same on every lane); within a mask the lanes split
  // the outer combinations (stages 0 .. k-2), and each lane scores the last stage's
  // options for its outer combination from per-mask tables.
  const uint32_t e0 = A.mt_off[f], e1 = bad ? e0 : A.mt_off[f + 1];
  for (uint32_t e = e0; e < e1; ++e) {
    const uint32_t mk = A.mt_mk[e], mask = mk & 0xffffu, k = mk >> 16;
    const uint64_t idx0 = A.mt_cand[e];
    // last unit of every stage (4 bits each), cut costs, option counts
    uint32_t ends = 0, X = 0, st = 0, total = 1;
    for (uint32_t u = 0; u < m; ++u) {
      const bool cut = u + 1 < m && ((mask >> u) & 1u);
      if (cut) X += xc[u];
      if (u + 1 == m || cut) {
        ends |= u << (4 * st);
        ++st;
      }
    }
    for (uint32_t s = 0; s < k; ++s) {
      uint32_t u0, u1;
      dag_bounds(ends, s, u0, u1);
      total *= dag_nopt(uo, u0, u1);  // <= (5 + 5^4)^2 or 30^4: 32 bits (R43 limits)
    }
    if (lane == 0) scored += total;
    uint32_t lu0, lu1;
    dag_bounds(ends, k - 1, lu0, lu1);
    const uint32_t nl = dag_nopt(uo, lu0, lu1), nouter = total / nl;
    // the last stage's one-slice options, and for a two-branch last block each branch's
    // time and memory fit per profile (a split option is then a max of two table reads)
    uint32_t lt[kP], lg[kP];
    bool lok[kP];
#pragma unroll
    for (int o = 0; o < kP; ++o) {
      uint64_t us = 0;
      lg[o] = 0;
      lok[o] = true;
      lt[o] = dag_stage(A, img, row0, uo, lu0, lu1, (uint32_t)o, thr, lg[o], us, lok[o], sv);
    }
    const bool split2 = nl == kP + kP * kP;
    uint32_t bt[2][kP], bok = 0;
    if (split2) {
      const uint32_t* U = uo + 6 * lu0;
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int x = 0; x < kP; ++x) {
          const uint32_t cb0 = U[1 + j], ce0 = U[2 + j];
          bt[j][x] = dag_lat(A, img, row0, cb0, ce0, x);
          if (img[A.lay.o_pm + row0 + ce0] - img[A.lay.o_pm + row0 + cb0] <= img[A.lay.o_cap + x])
            bok |= 1u << (5 * j + x);
        }
    }
    for (uint32_t co = lane; co < nouter; co += 32) {
      uint64_t T0 = 0, Q0 = 0, use0 = 0;
      uint32_t gp0 = 0, rest = co;
      bool ok0 = true;
      for (uint32_t ss = k - 1; ss > 0; --ss) {  // digits of co: stage k-2 fastest
        uint32_t u0, u1;
        dag_bounds(ends, ss - 1, u0, u1);
        const uint32_t no = dag_nopt(uo, u0, u1), os = rest % no;
        rest /= no;
        const uint64_t t = dag_stage(A, img, row0, uo, u0, u1, os, thr, gp0, use0, ok0, sv);
        T0 += t;
        Q0 += t * t;
      }
      // the outer stages alone already miss memory, the floor, the free slices or the SLO:
      // no last stage can repair that (times and slice counts only grow)
      ok0 &= (((nf | 0x8080808080808080ull) - use0) & 0x8080808080808080ull) == 0x8080808080808080ull;
      if (!ok0 || T0 + X > B) continue;
      const uint32_t cbase = co * nl;  // the combination's index, last stage fastest
      auto score = [&](uint64_t t, uint32_t gp, uint64_t use, bool ok, uint32_t ol) {
        const uint64_t T = T0 + t, Q = Q0 + t * t;
        // every byte: use <= free (both <= 8), SLO inclusive (R8)
        ok &= (((nf | 0x8080808080808080ull) - use) & 0x8080808080808080ull) == 0x8080808080808080ull;
        ok &= T + X <= B;
        if (ok) {
          const uint64_t D = T * T, N = (uint64_t)k * Q - D;
          // production: a candidate whose cvq exceeds the running best's cannot win --
          // decided by one multiply (cvq >= c + 1 <=> 1024 N >= (c + 1) D, < 2^62) before
          // the 64-bit division (verify mode sums every feasible key)
          if (!VERIFY && best != kKeyNone && (N << 10) >= ((best >> 50) + 1) * D) return;
          const uint64_t key =
              (((N << 10) / D) << 50) | ((uint64_t)(k - 1) << 47) | ((uint64_t)gp << 41) | (idx0 + cbase + ol);
          if (VERIFY) {
            ++nfeas;
            ksum += key;
          }
          if (key < best) {
            best = key;
            best_mk = mk;
            best_c = cbase + ol;
          }
        }
      };
#pragma unroll
      for (int o = 0; o < kP; ++o) score(lt[o], gp0 + lg[o], use0 + (1ull << (8 * o)), lok[o], (uint32_t)o);
      if (split2) {  // splits of a two-branch last block (option kP + 5 p0 + p1)
#pragma unroll
        for (int p0 = 0; p0 < kP; ++p0)
#pragma unroll
          for (int p1 = 0; p1 < kP; ++p1) {
            const uint32_t t = max(bt[0][p0], bt[1][p1]);
            const bool ok = ((bok >> p0) & (bok >> (5 + p1)) & 1u) && t <= thr;
            score(t, gp0 + gpc[p0] + gpc[p1], use0 + (1ull << (8 * p0)) + (1ull << (8 * p1)), ok,
                  (uint32_t)(kP + kP * p0 + p1));
          }
      } else {
        for (uint32_t ol = kP; ol < nl; ++ol) {  // splits of a one-block last stage (3-4 branches)
          uint64_t use = use0;
          uint32_t gp = gp0;
          bool ok = true;
          const uint64_t t = dag_stage(A, img, row0, uo, lu0, lu1, ol, thr, gp, use, ok, sv);
          score(t, gp, use, ok, ol);
        }
      }
    }
  }
  // warp argmin (keys are unique: idx is embedded) and checksum sums
  uint64_t wbest = best;
#pragma unroll
  for (int d = 16; d; d >>= 1) wbest = min(wbest, (uint64_t)__shfl_xor_sync(0xffffffffu, (unsigned long long)wbest, d));
  if (VERIFY) {
#pragma unroll
    for (int d = 16; d; d >>= 1) {
      scored += __shfl_xor_sync(0xffffffffu, (unsigned long long)scored, d);
      nfeas += __shfl_xor_sync(0xffffffffu, (unsigned long long)nfeas, d);
      ksum += __shfl_xor_sync(0xffffffffu, (unsigned long long)ksum, d);
    }
    if (lane == 0) {
      A.checks[3 * (size_t)r] = scored;
      A.checks[3 * (size_t)r + 1] = nfeas;
      A.checks[3 * (size_t)r + 2] = ksum;
    }
  }
  const bool writer = wbest == kKeyNone ? lane == 0 : best == wbest;
  if (!writer) return;
  ffs_dag_plan P;
  P.key = (int64_t)wbest;
  P.status = bad ? FFS_PLAN_BAD_REQ : (wbest == kKeyNone ? FFS_PLAN_INFEASIBLE : FFS_PLAN_OK);
  P.k = P.cut_mask = P.split_mask = P.e2e_us = P.bottleneck_us = P.gpcs = P.cvq = P.n_slots = P.pad = 0;
  for (int i = 0; i < FFS_DAG_MAX_SLOTS; ++i) {
    P.prof[i] = 0xff;
    P.slice[i] = -1;
  }
  if (P.status == FFS_PLAN_OK) {
    const uint32_t mask = best_mk & 0xffffu, k = best_mk >> 16;
    P.k = k;
    P.cut_mask = mask;
    P.cvq = (uint32_t)(wbest >> 50);
    uint32_t ends = 0, X = 0, st = 0;
    for (uint32_t u = 0; u < m; ++u) {
      const bool cut = u + 1 < m && ((mask >> u) & 1u);
      if (cut) X += xc[u];
      if (u + 1 == m || cut) {
        ends |= u << (4 * st);
        ++st;
      }
    }
    // the winner's option of every stage: digits of best_c, stage 0 most significant
    uint32_t div = 1;
    for (uint32_t s = 1; s < k; ++s) {
      uint32_t u0, u1;
      dag_bounds(ends, s, u0, u1);
      div *= dag_nopt(uo, u0, u1);
    }
    uint32_t rest = best_c, e2e = X, bott = 0, g = 0, ns = 0, taken = 0;  // taken: 4-bit count per profile
    uint64_t use = 0;
    bool ok = true;
    for (uint32_t s = 0; s < k; ++s) {
      uint32_t u0, u1;
      dag_bounds(ends, s, u0, u1);
      const uint32_t os = rest / div;
      rest -= os * div;
      if (s + 1 < k) {
        uint32_t a0, a1;
        dag_bounds(ends, s + 1, a0, a1);
        div /= dag_nopt(uo, a0, a1);
      }
      const uint32_t t = dag_stage(A, img, row0, uo, u0, u1, os, 0xffffffffu, g, use, ok, sv);
      e2e += t;
      bott = max(bott, t);
      // slots: one slice, or the branches in order (branch 0 = most significant digit)
      uint32_t nb = 1, w = os, pw = 1;
      if (os >= (uint32_t)kP) {
        P.split_mask |= 1u << s;
        nb = uo[6 * u0] & 0xffu;
        w = os - kP;
        for (uint32_t j = 1; j < nb; ++j) pw *= kP;
      }
      for (uint32_t j = 0; j < nb; ++j, ++ns) {
        const uint32_t p = os >= (uint32_t)kP ? (w / pw) % kP : os;
        pw = pw > 1 ? pw / kP : 1;
        const uint32_t cnt = (taken >> (4 * p)) & 15u;
        P.prof[ns] = (uint8_t)p;
        P.slice[ns] = A.free_list[((size_t)v * 8 + p) * 8 + cnt];
        taken += 1u << (4 * p);
      }
    }
    P.e2e_us = e2e;
    P.bottleneck_us = bott;
    P.gpcs = g;
    P.n_slots = ns;
  }
  *out = P;
}


// Persistent CTAs: the table image is staged into shared memory once per CTA (as the search
// kernel does), then the CTA's warps take requests r = warp, warp + all warps, ...; an image
// too large for shared memory is read from global memory (A.tables_global).
// 6 CTAs of 128 threads per SM (80 registers, a few spills): the kernel is latency-bound
// (dependent integer chains, wait stalls), more warps win (CD: 18.4 / 17.6 / 14.6 / 15.6 ms
// at 1 / 4 / 6 / 8)
#ifndef FFS_DAG_MINB
#define FFS_DAG_MINB 6
#endif
template <bool VERIFY>
__global__ void __launch_bounds__(kDagT, FFS_DAG_MINB) k_plan_dag(const __grid_constant__ DagArgs A) {
  extern __shared__ __align__(16) uint32_t dag_smem[];
  const uint32_t* img = A.image;
  if (!A.tables_global) {
    const uint4* src = reinterpret_cast<const uint4*>(A.image);
    uint4* dst = reinterpret_cast<uint4*>(dag_smem);
    for (uint32_t i = threadIdx.x; i < A.lay.words / 4; i += blockDim.x) dst[i] = src[i];
    __syncthreads();
    img = dag_smem;
  }
  const uint32_t nw = gridDim.x * (kDagT / 32);
  for (uint32_t r = blockIdx.x * (kDagT / 32) + (threadIdx.x >> 5); r < A.n_req; r += nw) dag_request<VERIFY>(A, img, r);
}

cudaError_t launch_dag(const DagArgs& a, cudaStream_t st) {
  int dev = 0, sms = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const size_t smem = a.tables_global ? 0 : (size_t)a.lay.words * 4;
  cudaError_t e = a.checks ? cudaFuncSetAttribute(k_plan_dag<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMaxSmem)
                           : cudaFuncSetAttribute(k_plan_dag<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMaxSmem);
  if (e != cudaSuccess) return e;
  e = a.checks ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_plan_dag<true>, kDagT, smem)
               : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_plan_dag<false>, kDagT, smem);
  if (e != cudaSuccess) return e;
  const uint64_t need = ((uint64_t)a.n_req + kDagT / 32 - 1) / (kDagT / 32);
  const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(need, (uint64_t)sms * std::max(per, 1)));
  if (a.checks)
    k_plan_dag<true><<<grid, kDagT, smem, st>>>(a);
  else
    k_plan_dag<false><<<grid, kDagT, smem, st>>>(a);
  return cudaGetLastError();
}

}  // namespace ffsk
