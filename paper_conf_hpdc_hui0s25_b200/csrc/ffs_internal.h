// ffs_internal.h -- shared between the host side (ffs_host.cu) and the kernels
// (ffs_kernels.cu) of libffs.so.  Not part of the ABI.  Nothing here is shared with the
// CPU oracle (oracle/), which is independent test infrastructure.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "ffs.h"

namespace ffsk {

constexpr int kP = 5;          // profiles this build is compiled for (Table 2)
constexpr int kRowW = 8;       // words per prefix-latency row (P padded to 8 -> 2 x LDS.128)
constexpr int kMaxN = 32;      // max components per chain (cut masks fit in uint32)
constexpr int kMaxK = 8;       // max stages
constexpr int kIdxBits = 41;   // canonical index field of the key
constexpr uint64_t kKeyNone = 0x7FFFFFFFFFFFFFFFull;
#ifndef FFS_BLOCK
#define FFS_BLOCK 256
#endif
#ifndef FFS_MINB4
#define FFS_MINB4 1
#endif
constexpr int kBlock = FFS_BLOCK;  // threads per CTA of the search kernel
// The f16x2 KS = 4 kernel uses 128 registers at 16 warps per SM (round 2, C5: 42.6 ms;
// 8 / 12 / 14 / 18 / 20 warps measured 52.0 / 45.4 / 43.9 / 44.3 / 44.5 ms).
#ifndef FFS_BLOCK4
#define FFS_BLOCK4 512
#endif
// KS = 3: the f16x2 core of the task-range kernel (exhaustive / verify modes, 127-136
// registers) runs 16 warps per SM; the list kernel of the bounded mode keeps the fp32 core
// (tighter filter margin: fewer rescans of its near-winning records, 168 registers, 12 warps)
#ifndef FFS_BLOCK3
#define FFS_BLOCK3 512
#endif
__host__ __device__ constexpr int search_block(int ks, bool list = false) {
  return ks == 3 ? (list ? 384 : FFS_BLOCK3) : ks == 4 ? FFS_BLOCK4 : kBlock;
}
constexpr size_t kMaxSmem = 227 * 1024;  // dynamic shared memory per CTA on sm_100
#ifndef FFS_HOST_SLICES
#define FFS_HOST_SLICES 2
#endif
constexpr uint32_t kHostSlices = FFS_HOST_SLICES;  // request slices of ffs_plan_batch_host (>= 2^20 requests)
// bytes of per-thread shared memory of the KS = 4 kernel: 5 profiles x 11 packed f16x2
// windows (ks4_pair_h)
constexpr size_t kWin4 = 55 * 4;

// Layout of the staged "table image" (32-bit words).  The search kernel copies the whole
// image into shared memory once per CTA (A0 of DESIGN.md §4); every other kernel reads
// it from global memory.
struct ImageLayout {
  uint32_t words;     // total size in words, multiple of 4 (16-byte copies)
  uint32_t F;         // functions
  uint32_t o_gpcs;    // [8] u32
  uint32_t o_cap;     // [8] u32 slice memory (MiB)
  uint32_t o_binom;   // [33][8] u32 C(c, i), c <= 32, i <= 7
  uint32_t o_offk;    // [33][10] u64 (word pairs) offk[n][k] = sum_{k'<k} C(n-1,k'-1) P^k'
  uint32_t o_fdesc;   // [F][4] u32 {row0, n, load_us, mem_total}
  uint32_t o_pl;      // [rows][8] fp32 bits: PL[row0+i][p] = sum_{c<i} lat[c][p], exact (< 2^24), 16-B aligned
  uint32_t o_pm;      // [rows] u32 PM[row0+i] = sum_{c<i} mem[c]
  uint32_t o_xf;      // [rows] u32 xfer cost of a cut after component i (row0+i)
  uint32_t o_thr;     // [F] u32 throughput floor: max stage time (R38); 0xffffffff = none
  uint32_t o_tmm;     // [F][2] fp32 {tmin, tmax}: sum over the chain of the min / max component
                      // latency over all profiles (KS = 4 f16 scale bounds), fp32 in chain order
};

struct SearchArgs {
  const uint32_t* image;        // device copy of the table image
  ImageLayout lay;
  const ffs_request* req;
  const uint32_t* slo;
  const uint64_t* node_free;    // [n_nodes] 8 x u8 free counts clamped to 8
  const uint64_t* prefix;       // [K][n_req+1] exclusive task prefix of segment k
  uint32_t n_req;
  uint32_t rank, world;
  int64_t* keys;
  unsigned long long* checks;   // [n_req][3] or null
  unsigned long long* misses;   // debug counter (verify mode)
  uint32_t tables_global;       // 1: read the image from global memory (too large for smem)
  unsigned long long* work_ctr; // [kCtrWords] chunk counters [KS] and scored-candidate
                                // counters [kCtrScored + KS], zeroed by the count kernel
  uint32_t zero;                // always 0: an operand ptxas cannot fold (ks4_pair_h's IADD3)
  uint32_t exhaustive;          // FFS_SEARCH_EXHAUSTIVE: no stage-0 SLO bound, every
                                // candidate of every enumerated mask is scored
  // bounded mode, KS = 2..4: the live (request, mask pair) records k_live wrote; when set
  // and the segment's record count fits list_cap, the search walks the list instead of
  // the task ranges (DESIGN.md §4.3 "live-mask compaction")
  const uint4* list;            // {request, maskA, maskB (0 = none), 0}
  uint32_t list_cap;
  // exhaustive / verify, KS = 2..4: the requests grouped by chain length (k_group_*); a
  // warp's lanes walk the same masks of 32 requests with equal n, so the tables of the
  // stages after the second-highest cut change only at row boundaries, warp-uniformly
  // (DESIGN.md §4.3).  Null: plain task ranges.
  const uint32_t* g_perm;       // [n_req] request ids ordered by n (n >= 4 only)
  const uint32_t* g_tab;        // [4 x 34]: first index in g_perm of each n, unit prefix per n (KS = 4, 3, 2)
  uint32_t g_s3;                // masks per KS = 3 unit (grp_unit3(n_req)); KS = 4: kGrpS
};
#ifndef FFS_GRP_S
#define FFS_GRP_S 128
#endif
constexpr uint32_t kGrpS = FFS_GRP_S;  // masks per work unit of the grouped KS = 4 path
// masks per work unit of the grouped KS = 3 path: a request shard of C5 has too few KS = 3
// units of 128 masks for 16 warps per SM (measured per shard size 1, 1/2, 1/4, 1/8, 1/16 of
// C5 with 128 / 64 / 32: 1.80 / 0.93 / 0.54 / 0.41 / 0.30 ms, 1.82 / 0.94 / 0.52 / 0.33 /
// 0.24, 1.87 / 0.96 / 0.51 / 0.29 / 0.20), so it shrinks with the batch
__host__ __device__ constexpr uint32_t grp_unit3(uint32_t n_req) {
  return n_req >= (1u << 19) ? 128u : n_req >= (1u << 18) ? 64u : 32u;
}
// work_ctr layout: blocks of kCtrBlock words indexed by KS: [KS] task-chunk grab
// counters; [kCtrScored + KS] candidates the segment's kernel scored (every candidate whose
// own score it computed); [kCtrListGrab + KS] record-chunk grab counters, [kCtrListCount +
// KS] live records written by k_live and [kCtrLiveGrab + KS] k_live's own task-chunk grab
// counters (bounded mode).  A search call zeroes the slots of the segments it runs (all of
// them when k_first = 1), so a caller running the segments range by range (candidate
// shards) still reads every segment's counters after the last range.
constexpr int kCtrBlock = 12, kCtrScored = 12, kCtrListGrab = 24, kCtrListCount = 36, kCtrLiveGrab = 48,
              kCtrWords = 60;

// Group tables of the bounded mode: per function f and availability
// pattern a (bit p = the node has >= 1 free slice of profile p), with W(i, j) = the fastest
// admissible time of stage [i, j) (profile in a, stage memory <= capacity, time <= floor;
// kGInf if none) and X(j) the cost of the cut at boundary j:
//   H0[j] = W(0, j) + X(j), T3[i] = W(i, n), Mt[j][i] = W(i, j) + X(j) (i < j < n),
//   R2[j] = min_i H0[i] + Mt[j][i], R3[j] = min_i R2[i] + Mt[j][i]
// every value clamped to kGInf.  An e2e lower bound of a KS-stage mask is then a sum of
// <= 4 table entries, exact in u32.
constexpr uint32_t kGInf = 1u << 29;
__host__ __device__ constexpr uint32_t grp_stride(uint32_t n) { return 4 * (n + 1) + (n + 1) * (n + 1); }

struct LiveArgs {
  const uint32_t* image;        // global copy (read through L1)
  ImageLayout lay;
  const ffs_request* req;
  const uint32_t* slo;
  const uint64_t* node_free;
  const uint64_t* prefix;
  uint32_t n_req, rank, world;
  const int64_t* keys;          // best keys of the earlier segments (request-level CV test)
  const uint32_t* gofs;         // [F] word offset of function f's group tables
  const uint32_t* grp;
  uint4* list[3];               // record lists of KS = 2, 3, 4 (list_cap records each)
  uint32_t list_cap, ks;        // the segment this launch compacts (2..4)
  uint32_t per_grab;            // requests a warp takes per grab (1..32, one per lane)
  unsigned long long* work_ctr;
};

struct DecodeArgs {
  const uint32_t* image;
  ImageLayout lay;
  const ffs_request* req;
  const uint32_t* slo;
  const int64_t* keys;
  uint32_t n_req, k_max, n_nodes, n_slices;
  const int32_t* free_list;     // [n_nodes][8][8] slice index of the j-th free slice
  const uint16_t* slice_node;   // [n_slices]
  const uint8_t* slice_prof;    // [n_slices]
  const ffs_instance* inst;     // nullable
  const int64_t* score;
  uint32_t n_inst;
  ffs_plan* out;
  const unsigned long long* vtab;  // [n_nodes][kP] minimum LRU score per (node, slice profile), ~0 empty
};

// launchers (ffs_kernels.cu)
// search chunks per warp and rank (dynamic grab, k_plan_search), per stage count: more
// chunks shorten the tail of the grab, each costs a request lookup.  Measured on C5 (ms of
// the KS = 1 / 2 / 3 / 4 segments): 1: 0.04 / 1.01 / - / -, 8: 0.06 / 0.92 / 3.14 / 41.8,
// 16: - / - / 3.04 / -, 32: 0.18 / 0.88 / 3.14 / 40.6, 64: - / - / - / 40.45.
__host__ __device__ constexpr int kdyn(int ks) { return ks == 1 ? 1 : ks == 2 ? 32 : ks == 3 ? 16 : ks == 4 ? 64 : 32; }
// minimum tasks per lane piece of the search's task ranges (a piece costs a request
// lookup; a KS = 1/2 task is ~5 / ~100 instructions, a KS = 4 mask pair ~3000)
// (measured on C5 slices of 1/1 .. 1/16 of the batch: shorter pieces leave more of the
// per-piece lookups, longer ones more imbalance)
__host__ __device__ constexpr int kMinPiece(int ks) { return ks == 1 ? 4 : ks == 2 ? 8 : ks == 3 ? 2 : 1; }
cudaError_t launch_count_tasks(const ffs_request* req, const uint32_t* image, const ImageLayout& lay,
                               uint32_t n_nodes, uint32_t n_req, uint32_t k_max, const uint64_t* node_free,
                               bool skip_full, uint64_t* prefix, uint64_t* block_sums, int64_t* keys,
                               unsigned long long* checks, unsigned long long* work_ctr, uint32_t k_first,
                               uint32_t k_last, cudaStream_t st);
// requests grouped by chain length (stable) for the exhaustive / verify KS = 4 segment:
// off [34 * ceil(n_req / 2048) + 1], bsum (scan scratch, like the task prefix's), tab [68],
// perm [n_req]; tab [136]
cudaError_t launch_group_n(const ffs_request* req, const uint32_t* image, const ImageLayout& lay, uint32_t n_nodes,
                           uint32_t n_req, uint32_t s3, uint64_t* off, uint64_t* bsum, uint32_t* tab, uint32_t* perm,
                           cudaStream_t st);
cudaError_t launch_search(int ks, bool verify, bool list, const SearchArgs& a, int grid, int block, size_t smem,
                          cudaStream_t st);
cudaError_t search_kernel_config(int ks, bool verify, bool list, bool tables_global, int block, size_t smem,
                                 int* blocks_per_sm);
cudaError_t launch_decode(const DecodeArgs& a, unsigned long long* vtab, cudaStream_t st);
cudaError_t launch_evict(const ffs_instance* inst, uint32_t n_inst, const uint32_t* tick_off,
                         const uint64_t* now_us, uint32_t n_ticks, uint64_t now_single,
                         ffs_evict_params prm, int64_t* score, uint8_t* state, cudaStream_t st);
cudaError_t launch_victims(const uint32_t* image, const ImageLayout& lay, const ffs_request* req,
                           const uint32_t* slo, const uint32_t* req_tick, uint32_t n_req,
                           const ffs_instance* inst, const uint32_t* tick_off, const int64_t* score,
                           uint32_t n_ticks, const uint16_t* slice_node, const uint8_t* slice_prof,
                           uint32_t n_slices, uint32_t n_nodes, unsigned long long* tab, int32_t* victim,
                           cudaStream_t st);
cudaError_t launch_evict_step(const uint32_t* image, const ImageLayout& lay, const ffs_instance* inst,
                              const uint32_t* tick_off, const uint64_t* now_us, uint32_t n_ticks, ffs_evict_params prm,
                              int64_t* score, uint8_t* state, const uint16_t* slice_node, const uint8_t* slice_prof,
                              uint32_t n_slices, uint32_t n_nodes, unsigned long long* tab, const ffs_request* req,
                              const uint32_t* slo, const uint32_t* req_tick, const uint32_t* load_off, uint32_t n_req,
                              int32_t* victim, cudaStream_t st);
cudaError_t run_int_peak(int sms, double* ops, double* seconds);
cudaError_t run_packed_peak(int sms, int mode, double* lane_instr_per_s, double* seconds);
cudaError_t launch_group_tables(const uint32_t* image, const ImageLayout& lay, const uint32_t* gofs, uint32_t* grp,
                                cudaStream_t st);
cudaError_t launch_live(const LiveArgs& a, int grid, cudaStream_t st);

struct RankedArgs {
  const uint32_t* image;
  ImageLayout lay;
  const ffs_request* req;
  const uint32_t* slo;
  uint32_t n_req, n_nodes;
  const uint64_t* node_free;
  const int32_t* free_list;
  const uint32_t* rank_off;   // [F+1]
  const uint32_t* rank_mask;  // ranked cut masks, per function contiguous
  uint32_t prof_order;        // profiles by (capacity, gpcs, id): 4 bits each, first = low nibble
  ffs_plan* out;
};
cudaError_t launch_ranked(const RankedArgs& a, cudaStream_t st);

// NEXT-1 DAG stages
struct DagArgs {
  const uint32_t* image;
  ImageLayout lay;
  const ffs_request* req;
  const uint32_t* slo;
  uint32_t n_req, n_nodes;
  const uint64_t* node_free;
  const int32_t* free_list;
  const uint32_t* fu;         // [F][2] {first unit, units}
  const uint32_t* units;      // [U][6] {nb, c0, e0, e1, e2, e3} function-relative components
  const uint32_t* xcut;       // [U] cost of a cut after the unit (R42, R48)
  const uint32_t* sv;         // [U + F][8] per function (rows fu[2f] + f ..): prefix over its units
                              // of the conditional units' one-slice saving sum - max (R48)
  const uint32_t* mt_off;     // [F+1] mask-table entries of f
  const uint32_t* mt_mk;      // unit-cut mask | k << 16
  const unsigned long long* mt_cand;  // first candidate index of the entry
  ffs_dag_plan* out;
  unsigned long long* checks; // [n_req][3] or null
  uint32_t tables_global;     // 1: the image is too large for shared memory, read it from global
};
cudaError_t launch_dag(const DagArgs& a, cudaStream_t st);

struct JointArgs {
  const uint32_t* image;
  ImageLayout lay;
  const ffs_request* req;
  const uint32_t* slo;
  uint32_t n_req, n_nodes, k_max;
  int64_t* keys;               // [n_req] current argmin key of every open request
  uint8_t* state;              // [n_req] 0 pending, 1 re-plan, 2 final
  uint32_t* dirty;             // [n_req] requests to (re-)plan next round
  ffs_request* sub_req;        // gathered dirty requests
  uint32_t* sub_slo;
  int64_t* sub_keys;
  uint64_t* node_win;          // [n_nodes] min (adjusted deadline, index) of feasible open requests
  uint8_t* busy;               // [n_slices] mutable copy of the slice states
  uint8_t* cnt;                // [n_nodes][8] free slices per profile (true counts, <= 255)
  uint64_t* node_free;         // [n_nodes] counts clamped to 8 (search input)
  const uint32_t* node_off;    // [n_nodes+1] slices of node v
  const uint8_t* slice_prof;
  ffs_plan* out;
  uint32_t* n_open;
  uint32_t* n_dirty;
};
cudaError_t launch_joint(int phase, const JointArgs& a, uint32_t n, cudaStream_t st);

struct FrontierArgs {
  const uint32_t* image;
  ImageLayout lay;
  uint32_t k_max, n_groups, n_fv, n_nodes, cap;  // cap = rounds allocated
  const uint32_t* node_fv;      // [n_nodes] free-vector id of each node
  // build
  const uint32_t* active;       // [n_active] group ids searched this round
  const int64_t* keys;          // [n_active] argmin keys of this round
  uint32_t* next_active;
  uint32_t* n_next;
  uint32_t* budget;             // [n_groups] budget of the group's next search (e2e of last point - 1)
  ffs_request* greq;            // [n_active] synthetic requests of this round
  uint32_t round;
  // frontier storage, round-major: point i of group g at [i * n_groups + g]
  int64_t* fr_key;
  uint32_t* fr_e2e;
  uint32_t* fr_cnt;             // [n_groups]
  // query
  const ffs_request* req;
  const uint32_t* slo;
  uint32_t n_req;
  const int32_t* free_list;
  ffs_plan* out;
  const uint32_t* fv_node;      // [n_fv] lowest node id of each free-vector class (any-invoker)
  int32_t* node_out;            // [n_req] serving node (any-invoker), nullable
};
cudaError_t launch_frontier(int phase, const FrontierArgs& a, uint32_t n, cudaStream_t st);

struct RouteArgs {
  const uint32_t* image;
  ImageLayout lay;
  const ffs_request* req;
  const uint32_t* slo;
  uint32_t n_req, n_inst;
  const ffs_instance* inst;
  const uint8_t* state;
  const uint32_t* lat;
  const uint32_t* cap;
  uint64_t* rkey; uint32_t* rval;   // requests: (func, adjusted deadline) -> index, sorted
  uint64_t* ikey; uint32_t* ival;   // instances: (func, not-hot, latency) -> index, sorted
  uint64_t* icum;                   // [n_inst+1] exclusive prefix of hot capacities (sorted order)
  uint64_t* icap;                   // alias of icum before the scan
  uint32_t* first_req;              // [F+1]
  uint32_t* first_hot;              // [F+1]
  uint32_t* n_hot;                  // [F+1]
  int32_t* ts;                      // [F+1]
  int32_t* route;
};
cudaError_t launch_route(int phase, const RouteArgs& a, cudaStream_t st);

struct SimArgs {
  const uint32_t* image;
  ImageLayout lay;
  uint32_t n_nodes, n_ticks, window_ticks, thr_pct, tick_us;
  uint64_t t0_us, cold_after_us;
  const uint32_t* node_off;     // [n_nodes+1]
  const uint8_t* slice_prof;
  const uint8_t* slice_busy;    // staged states (other tenants)
  const uint32_t* req_off;
  const uint32_t* req_func;
  const uint32_t* req_budget;
  int32_t* res;                 // [n_slices] resident function or -1 (scratch)
  uint8_t* flags;               // [n_nodes][F] bit0 exists, bit1 hot (scratch)
  uint64_t* ctr;                // [n_nodes][12]
  int32_t* slice;
  uint8_t* state;
  uint64_t* last;
  uint32_t* busy;
  uint8_t* stages;              // [n_nodes][F] 0 none, 1 monolithic, k pipeline
  uint32_t k_max;               // pipeline search depth (0: monolithic instances only)
  int32_t* psl;                 // [n_nodes][F][8] pipeline slices (scratch)
  uint32_t* pe2e;               // [n_nodes][F] pipeline e2e (scratch)
  uint8_t* pk;                  // [n_nodes][F] pipeline stages (scratch)
};
cudaError_t launch_sim(const SimArgs& a, cudaStream_t st);
cudaError_t radix_sort_pairs(uint64_t* key, uint32_t* val, uint64_t* key2, uint32_t* val2, uint32_t n, int bits,
                             uint64_t* hist, uint64_t* bsum, cudaStream_t st);
cudaError_t scan_u64(uint64_t* a, uint64_t len, uint64_t* bsum, cudaStream_t st);
cudaError_t launch_front_gather(const FrontierArgs& a, uint32_t n, const uint32_t* fv_node, uint32_t* gslo,
                                cudaStream_t st);

}  // namespace ffsk
