/*
 * ffs.h -- C ABI of libffs.so, the B200 (sm_100a) batched pipeline-construction search of
 * FluidFaaS (Hui, Xu, Shen, HPDC '25).  Citations "P:<line>" are lines of the paper text
 * (PAPER.md); "R<n>" are the readings fixed in DESIGN.md §3.
 *
 * What the library computes:
 *   For every pending invocation (request) the invoker picks "the appropriate assignment
 *   of MIG slices to the components in the DAG" by evaluating "all possible
 *   partitions" of the component chain (§5.2.2) against "the available MIGs
 *   within the invoker", ranking by the coefficient of variation of stage times
 *   (Eq. 1), under the SLO and each slice's memory.
 *   Candidate = (k stages <= k_max, cut mask, ordered profile sequence); the plan is the
 *   feasible argmin of the packed key
 *        key = cvq << 50 | (k-1) << 47 | gpcs << 41 | idx          (R1, R4)
 *   cvq = floor(1024 * CV^2) with population std (R3), gpcs = sum of the stage profiles'
 *   GPCs (ESG's "most resource-efficient option"), idx = canonical candidate index
 *   (k ascending, cut masks in ascending numeric order, profile digits p_1 most
 *   significant).  A feasible key is < 2^63 - 1, so INT64_MAX (FFS_KEY_NONE) = infeasible.
 *   The hotness-aware eviction score is the second entry point.
 *
 * Conventions
 *   - Every call returns ffs_status; no exception or abort crosses the ABI.  On a non-OK
 *     status ffs_last_error() describes it.
 *   - Integers are little-endian, fixed width; times in microseconds, memory in MiB (R14).
 *   - Pointers prefixed d_ are DEVICE pointers on the context's device, caller-owned, read
 *     or written only by stream work enqueued by the call (the call returns before that
 *     work finishes unless stated).  h_ pointers are host memory (pinned recommended).
 *     Tables passed to ffs_stage_tables are host memory copied during the call.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *   - The library allocates only context-owned scratch; it never frees caller memory.
 *   - There is no CPU fallback: a context can only be created on a CUDA device with
 *     compute capability 10.0 (sm_100a).
 */
#ifndef FFS_H
#define FFS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    FFS_OK = 0,
    FFS_ERR_ARG = -1,   /* null/ill-formed argument: lat = 0, non-monotone comp_off, unsorted slices ... */
    FFS_ERR_RANGE = -2, /* a bound of the exact integer encoding is exceeded (see each call)  */
    FFS_ERR_CUDA = -3,  /* a CUDA runtime call failed (message has the CUDA error string)       */
    FFS_ERR_STATE = -4  /* tables not staged, or staged for a different shape                   */
} ffs_status;

#define FFS_MAX_PROFILES 8
#define FFS_MAX_STAGES 8
#define FFS_MAX_CHAIN 32
#define FFS_KEY_NONE INT64_MAX

/* search modes (ffs_set_search_mode) */
#define FFS_SEARCH_BOUNDED 0u    /* default: exact SLO lower bounds skip candidates that cannot be feasible */
#define FFS_SEARCH_EXHAUSTIVE 1u /* every candidate of every request is scored ("all possible partitions") */

/* per-plan status (an infeasible request is not an error) */
#define FFS_PLAN_OK 0u
#define FFS_PLAN_INFEASIBLE 1u
#define FFS_PLAN_BAD_REQ 2u /* func >= n_funcs or node >= n_nodes */

/* keep-alive states (Fig. 8) */
#define FFS_ST_EXCL_HOT 0u
#define FFS_ST_TIME_SHARING 1u
#define FFS_ST_WARM 2u
#define FFS_ST_COLD 3u
/* ffs_instance.flags */
#define FFS_INST_PIPELINE 1u /* pipeline instances are exclusive hot */
#define FFS_INST_BUSY 2u     /* currently serving a request: never evicted   */

typedef struct ffs_ctx ffs_ctx; /* opaque; one per device; owns staged tables and scratch */

/* MIG profile table (Table 2).  gpcs[p] in 1..7, mem_mib[p] = slice memory. */
typedef struct {
    uint32_t n_profiles; /* P; this build is compiled for P = 5 (FFS_ERR_RANGE otherwise) */
    uint32_t gpcs[FFS_MAX_PROFILES];
    uint32_t mem_mib[FFS_MAX_PROFILES];
} ffs_profiles;

/* Per-component profile of every function ("the size of the required memory and
 * the running speeds of the component on each size of MIG").  Function f's chain is
 * components comp_off[f] .. comp_off[f+1]-1 (1 <= n_f <= 32).  Host pointers. */
typedef struct {
    uint32_t n_funcs;
    const uint32_t *comp_off; /* [F+1], comp_off[0] = 0, strictly increasing          */
    const uint32_t *lat_us;   /* [C][P] latency of component c alone on profile p, >= 1 */
    const uint32_t *mem_mib;  /* [C] memory of component c                            */
    const uint32_t *xfer_us;  /* [C] cost of a stage cut after component c (R7); the
                                 last component's entry is ignored                     */
    const uint32_t *load_us;  /* [F] warm -> MIG reload time (victim rule)     */
    /* [F] throughput floor (NEXT-2, R38), nullable: every stage of a plan of f
     * -- and the monolithic instance on a time-share victim's slice -- must run in at most
     * max_stage_us[f] us, i.e. serve >= 10^6 / max_stage_us[f] requests/s (an instance
     * sized for the function's load); 0 = no floor.  NULL = no floors. */
    const uint32_t *max_stage_us;
} ffs_profile_table;

/* One MIG slice of the cluster (12 bytes). */
typedef struct {
    uint16_t node;    /* invoker / node id (R10)           */
    uint8_t gpu;      /* GPU within the node                */
    uint8_t slice;    /* slice within the GPU               */
    uint8_t profile;  /* index into ffs_profiles            */
    uint8_t busy;     /* 1 = occupied (not free)            */
    uint16_t pad;
    int32_t instance; /* occupying instance or -1 (informational) */
} ffs_slice;

/* Cluster free-slice state.  Slices sorted by (node, gpu, slice) ascending; the free
 * count of (node, profile) is derived from them.  Host pointer. */
typedef struct {
    uint32_t n_nodes;
    uint32_t n_slices;
    const ffs_slice *slices;
} ffs_cluster;

/* A pending invocation: function and home node.  Its latency budget B_r (remaining SLO,
 * R9) is passed in a parallel uint32 array. */
typedef struct {
    uint32_t func, node;
} ffs_request;

/* The plan of one request (80 bytes) -- the "configuration layer" content: stages
 * (cut_mask) and the MIG slice of every stage (Listing 1). */
typedef struct {
    int64_t key;            /* FFS_KEY_NONE when not OK                                  */
    uint32_t status;        /* FFS_PLAN_*                                                 */
    uint32_t k;             /* number of stages                                           */
    uint32_t cut_mask;      /* bit j = stage boundary after component j                   */
    uint32_t e2e_us;        /* sum of stage latencies + transfers of the cuts             */
    uint32_t bottleneck_us; /* max stage latency; throughput = 1e6 / bottleneck_us rps    */
    uint32_t gpcs;          /* sum of GPCs of the stages' profiles                        */
    uint32_t cvq;           /* floor(1024 * CV^2) of the stage latencies (Eq. 1)          */
    uint8_t prof[FFS_MAX_STAGES];  /* profile of stage i (0xFF unused)                    */
    int32_t slice[FFS_MAX_STAGES]; /* bound slice index into ffs_cluster.slices (-1 unused) */
    int32_t victim;         /* time-share victim instance (INFEASIBLE only) or -1          */
} ffs_plan;

/* A function instance as seen by the invoker's keep-alive manager (24 bytes). */
typedef struct {
    uint32_t func;
    int32_t slice; /* resident on this slice, -1 = not resident (warm/cold) */
    uint8_t flags; /* FFS_INST_* */
    uint8_t pad[3];
    uint32_t busy_us;      /* busy time within the utilisation window          */
    uint64_t last_used_us; /* time of the last request (< 2^43)                */
} ffs_instance;

typedef struct {
    uint32_t util_thr_pct;  /* 30                                    */
    uint32_t window_us;     /* utilisation window (R18; default 10 s)        */
    uint64_t cold_after_us; /* 600e6 = 10 minutes             */
} ffs_evict_params;

/* ---- context --------------------------------------------------------------------- */
/* Create a context on `cuda_device`.  FFS_ERR_CUDA if the device is not sm_100. */
ffs_status ffs_create(int cuda_device, ffs_ctx **out);
void ffs_destroy(ffs_ctx *ctx);
/* Message for the last non-OK status returned on this context (never NULL). */
const char *ffs_last_error(const ffs_ctx *ctx);

/* ---- A0: stage tables --------------------------------------------------------------
 * Validate, prefix-sum and upload the profile table and the cluster free-slice state
 * (P:217).  Synchronous; host memory is only read during the call.
 * FFS_ERR_ARG   : null pointers, lat = 0, comp_off not strictly increasing, slices not
 *                 sorted by (node, gpu, slice), node >= n_nodes, profile >= P, gpcs not
 *                 in 1..7.
 * FFS_ERR_RANGE : P != 5, n_f > 32, sum_c max_p lat >= 2^24, sum xfer >= 2^24,
 *                 sum mem >= 2^31, n_nodes >= 2^16. */
ffs_status ffs_stage_tables(ffs_ctx *ctx, const ffs_profiles *profiles, const ffs_profile_table *table,
                            const ffs_cluster *cluster);

/* ---- search mode ------------------------------------------------------------------------
 * FFS_SEARCH_BOUNDED (default): the search skips candidates that an exact integer lower
 * bound of their end-to-end latency proves infeasible (SLO) -- identical keys,
 * much less work.  FFS_SEARCH_EXHAUSTIVE: every candidate of every request (including
 * requests on a node without a free slice, R37) has its own score computed, "all
 * possible partitions"; the measured throughput of this mode is the benchmark's
 * candidates-scored/s.  Both modes return bit-identical keys and plans.  FFS_ERR_ARG for
 * another value.  Applies to every later search call on the context. */
ffs_status ffs_set_search_mode(ffs_ctx *ctx, uint32_t mode);

/* ---- A1-A5: keys ---------------------------------------------------------------------
 * Partial argmin keys of shard `rank` of `world` (0 <= rank < world).  For every k the
 * flattened (request, cut mask) task list is cut into world x (search warps) x c chunks
 * of 32 equal contiguous pieces; shard `rank` owns the chunks j with j mod world = rank
 * (chunk interleave, DESIGN.md §4.3/§7) and decides every candidate of its chunks
 * (scored, or in bounded mode possibly proved infeasible by the exact SLO bound).  In
 * exhaustive and verify modes the segments k = 3, 4 (and k = 2 on batches of >= 2^19
 * requests) instead order the requests by chain length (a stable sort, identical on every
 * rank) and deal work units (32 consecutive requests of that order x a run of consecutive
 * masks) to the shards by unit index mod world.
 * In bounded mode the segments k = 2..4 are partitioned by a hash of (request, two
 * highest cut positions) -- in every case the shards partition the candidates.  Bounded mode
 * keeps three device lists of live (request, mask pair) records, 16 B each, capacity
 * 16 n_req + 2^20 records per list (0.85 GB at n_req = 2^20; the environment variable
 * FFS_LIST_CAP lowers it); a segment whose records exceed it runs on the task ranges
 * instead, with the same result.  d_keys[r] receives the minimum
 * feasible key of request r within the shard, FFS_KEY_NONE where none (overwritten, not
 * combined with its previous content).  Combine shards with an element-wise MIN
 * (torch.distributed.all_reduce(keys, MIN) over NCCL) before ffs_plan_decode.
 * d_checksums (nullable; verify mode, slower): uint64[3*n_req] = per request {candidates
 * scored, feasible candidates, sum of feasible keys mod 2^64} of this shard; combine
 * with SUM.  Asynchronous on `stream`.
 * FFS_ERR_RANGE: k_max not in 1..8, S(n, k_max) >= 2^41 for a staged function,
 * k_max * max gpcs >= 64.  FFS_ERR_STATE: tables not staged. */
ffs_status ffs_plan_keys(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                         uint32_t k_max, uint32_t rank, uint32_t world, int64_t *d_keys, uint64_t *d_checksums,
                         void *stream);

/* Segments k_first..k_last (1 <= k_first <= k_last <= k_max) of ffs_plan_keys, same shard
 * rule.  k_first == 1 initialises d_keys (FFS_KEY_NONE) and d_checksums (0) like
 * ffs_plan_keys; k_first > 1 leaves both as given and min-combines / adds into them, so a
 * caller can all_reduce(MIN) the keys between ranges: every rank then prunes the later
 * (heavier) segments against the best key of ALL shards of the earlier ones, exactly as
 * one GPU does, which keeps the shards equal in work.  The result after
 * the last range and a final MIN is the same as ffs_plan_keys.  Checksums stay per-shard
 * sums; reduce them with SUM once at the end.  Every call recomputes its task prefix from
 * d_req (no state is carried between calls besides d_keys / d_checksums).  FFS_ERR_RANGE:
 * bad segment range, or as ffs_plan_keys.  Asynchronous on `stream`. */
ffs_status ffs_plan_keys_range(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                               uint32_t k_max, uint32_t k_first, uint32_t k_last, uint32_t rank, uint32_t world,
                               int64_t *d_keys, uint64_t *d_checksums, void *stream);

/* ---- A6 (+A8): decode and bind ---------------------------------------------------------
 * Decode the combined keys into plans and bind every stage, in stage order, to the
 * lowest-index free slice of its profile in the request's node not taken by an earlier
 * stage (R11).  When d_inst and d_evict_scores are non-null, an INFEASIBLE request gets
 * the time-share victim of A8: the instance with the smallest eviction score
 * (from ffs_evict_scores on the same snapshot) resident in the request's node on a slice
 * that holds the whole function and meets lat + load <= budget; -1 if none.  The victims
 * cost O(n_inst + n_req): one pass folds the scores into per-(node, slice profile) minima
 * (context scratch), each INFEASIBLE request reads at most 5 of them.
 * Asynchronous on `stream`.  k_max must equal the one given to ffs_plan_keys.
 * FFS_ERR_RANGE: n_inst > 2^20 (the scores' index field). */
ffs_status ffs_plan_decode(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, const int64_t *d_keys,
                           uint32_t n_req, uint32_t k_max, const ffs_instance *d_inst,
                           const int64_t *d_evict_scores, uint32_t n_inst, ffs_plan *d_out, void *stream);

/* ---- one-GPU convenience: keys + decode (no victims) ---------------------------------
 * Uses context scratch for the keys.  Asynchronous on `stream`. */
ffs_status ffs_plan_batch(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                          uint32_t k_max, ffs_plan *d_out, void *stream);

/* Same with HOST buffers: copies the requests and budgets host->device, plans, copies
 * the plans device->host and synchronises `stream` before returning (the end-to-end
 * call of a user holding host data).  A batch of >= 2^20 requests is planned in two
 * request slices whose copies run on two context-owned non-blocking streams (ordered
 * after the work already queued on `stream`): the upload of the second and the download
 * of the first overlap the planning of the other (pinned host buffers are needed for the
 * overlap; pageable ones work, serialised).  The plans equal ffs_plan_batch's on the whole
 * batch (requests are planned independently). */
ffs_status ffs_plan_batch_host(ffs_ctx *ctx, const ffs_request *h_req, const uint32_t *h_slo_us, uint32_t n_req,
                               uint32_t k_max, ffs_plan *h_out, void *stream);

/* ---- A7: hotness-aware eviction scores -------------------------------------------------
 * One snapshot of n_inst instances at time now_us.  State, in order:
 *   idle = now - last_used (0 if negative) >= cold_after   -> COLD
 *   slice < 0 (not resident)                               -> WARM
 *   PIPELINE flag, or busy_us*100 >= util_thr_pct*window_us -> EXCL_HOT
 *   otherwise                                              -> TIME_SHARING
 * d_score[i] = ((cold_after_us - idle) << 20) | i for a TIME_SHARING instance without the
 * BUSY flag, FFS_KEY_NONE otherwise: the LRU key -- the smallest score is the
 * instance with the largest idle time (least recently used), ties to the lower index
 * (R20c).  A time-sharing instance has idle < cold_after_us, so the key is exact for any
 * timestamp epoch (e.g. Unix microseconds).  d_state[i] = FFS_ST_*.
 * FFS_ERR_RANGE: n_inst > 2^20, params->cold_after_us >= 2^43.  Async. */
ffs_status ffs_evict_scores(ffs_ctx *ctx, const ffs_instance *d_inst, uint32_t n_inst, uint64_t now_us,
                            const ffs_evict_params *params, int64_t *d_score, uint8_t *d_state, void *stream);

/* Batched over n_ticks snapshots: tick t owns instances d_tick_off[t] .. d_tick_off[t+1]-1
 * (device array, n_ticks+1 entries, non-decreasing) at time d_now_us[t]; the index in the
 * score is the index within the tick.  An instance at index >= 2^20 within its tick
 * scores FFS_KEY_NONE (ticks are device data; the caller keeps ticks below 2^20
 * instances).  FFS_ERR_RANGE: params->cold_after_us >= 2^43.  Async. */
ffs_status ffs_evict_scores_ticks(ffs_ctx *ctx, const ffs_instance *d_inst, const uint32_t *d_tick_off,
                                  const uint64_t *d_now_us, uint32_t n_ticks, const ffs_evict_params *params,
                                  int64_t *d_score, uint8_t *d_state, void *stream);

/* A8 batched over ticks: for every request r (tick d_req_tick[r]) the victim among the
 * instances of that tick, by the rule of ffs_plan_decode, regardless of the request's
 * plan (the caller passes the loads that need one).  d_victim[r] = index within the tick
 * or -1 (also when d_req_tick[r] >= n_ticks or the request's function/node is out of
 * range).  Scratch: a per-(tick, node, profile) table of n_ticks x nodes x 5 x 8 bytes when
 * that is <= 256 MiB, else a warp scan of the tick per request.  Async. */
ffs_status ffs_evict_victims(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us,
                             const uint32_t *d_req_tick, uint32_t n_req, const ffs_instance *d_inst,
                             const uint32_t *d_tick_off, const int64_t *d_score, uint32_t n_ticks,
                             int32_t *d_victim, void *stream);

/* A7 + A8 fused over ticks: the scores and states of ffs_evict_scores_ticks and the victims
 * of ffs_evict_victims for the n_req loads, in one pass over the instances: each tick's
 * CTA folds its scored instances into per-(node, slice profile) minima in shared memory.
 * Loads given per tick (d_req_tick[r], any order): the minima go to a table in device
 * memory and a second kernel picks (<= 5 cells per load).  Loads grouped by tick
 * (d_load_off non-null: uint32[n_ticks + 1], the loads of tick t are rows d_load_off[t] ..
 * d_load_off[t+1]-1 of d_req/d_slo_us/d_victim; d_req_tick may then be null): the tick's
 * CTA picks its loads' victims from shared memory -- one launch, no table.  Same outputs,
 * same rules and errors as the two calls (which it falls back to when a tick's minima
 * exceed 160 KiB of shared memory, or the table 256 MiB with per-load ticks).  n_req may
 * be 0 (scores only).  Async. */
ffs_status ffs_evict_step(ffs_ctx *ctx, const ffs_instance *d_inst, const uint32_t *d_tick_off,
                          const uint64_t *d_now_us, uint32_t n_ticks, const ffs_evict_params *params,
                          int64_t *d_score, uint8_t *d_state, const ffs_request *d_req, const uint32_t *d_slo_us,
                          const uint32_t *d_req_tick, const uint32_t *d_load_off, uint32_t n_req, int32_t *d_victim,
                          void *stream);

/* ---- NEXT-1: the paper's literal ranked first-fit ---------------------------
 * "After calculating and sorting the CVs for all possible pipeline configurations, which
 * is done once and offline for each application ... The pipelines are then evaluated in
 * order with the profiles, against the available MIG resources".
 * ffs_rank_partitions: offline step.  For every staged function, every contiguous
 * partition with k <= k_max stages ranked by (cvq of the stage times on the reference
 * profile p_ref, k, cut mask) ascending (R24, R25).  Host computation +
 * upload, synchronous.  FFS_ERR_RANGE: p_ref >= P, k_max not in 1..8, or more than 2^24
 * ranked partitions in total.  FFS_ERR_STATE: tables not staged.
 * ffs_plan_ranked: per request, walk its function's ranked list and take the first
 * partition "supported by the available resources" (R26): stages in descending memory
 * each take a distinct free slice of the smallest-capacity (then fewest-GPC, then
 * lowest-id) profile of the request's node that holds the stage, and the resulting
 * e2e <= budget.  d_out fields as ffs_plan_decode (computed on the assigned profiles,
 * slices bound in stage order); key = position in the ranked list (R27); INFEASIBLE
 * when no partition is supported.  Asynchronous on `stream`. */
ffs_status ffs_rank_partitions(ffs_ctx *ctx, uint32_t k_max, uint32_t p_ref);
ffs_status ffs_plan_ranked(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                           ffs_plan *d_out, void *stream);

/* ---- NEXT-1: DAG stages (R40-R43) -----------------------
 * The FFS DAG of a function is read as a series of UNITS: one component, or a fork/join
 * block of 2..4 parallel branches, each branch a chain of components (an app "is
 * extended with two branches to form a DAG").  The staged profile table numbers each
 * function's components unit by unit, branch by branch.  Stages are runs of consecutive
 * units (cuts only at unit boundaries -- the dominators, "dominator-based method
 * from ESG").  A stage runs on one slice (t = sum of all its components' latencies,
 * memory = sum), or, when the stage is exactly one block, SPLIT: branch j on its own slice
 * of profile p_j and t = max_j branch time ("If a stage involves multiple MIGs
 * running in parallel, we use the maximum execution time among them as the stage's
 * execution time"), memory checked per branch slice.  A cut after a unit costs the sum of
 * xfer_us of its branches' last components (R42).  Candidate order (R43): k ascending,
 * unit-cut masks ascending, stage options in mixed radix with stage 0 most significant,
 * option o < P = one slice of profile o, o = P + w = split with branch profiles the base-P
 * digits of w (branch 0 most significant); key, feasibility and binding as ffs_plan_keys /
 * ffs_plan_decode with every slice of the plan counted (gpcs, free slices).
 * Conditional units (unit_cond, R48) contribute their slowest alternative to a one-slice
 * stage and offer no split.  A table of one-component units reproduces ffs_plan_batch's
 * keys exactly. */
#define FFS_DAG_MAX_UNITS 16
#define FFS_DAG_MAX_BRANCHES 4
#define FFS_DAG_MAX_SLOTS 8

/* Unit structure of every staged function.  Host pointers, copied by ffs_dag_stage. */
typedef struct {
    uint32_t n_funcs;          /* = n_funcs of the staged profile table                       */
    const uint32_t *unit_off;  /* [F+1] function f has units unit_off[f] .. unit_off[f+1]-1  */
    const uint8_t *unit_nb;    /* [U] branches of the unit, 1..4 (1 = exactly one component) */
    const uint8_t *unit_bend;  /* [U][4] function-relative exclusive end component of branch j
                                  (branch j starts where branch j-1, or the previous unit,
                                  ends); entries j >= nb are ignored                         */
    const uint8_t *unit_cond;  /* [U] nullable: 1 = CONDITIONAL unit (R48, App 3): 2..4
                                  alternative branches, exactly one runs per request, an empty
                                  branch is "pass"; the slice hosts every branch, the unit's
                                  time is its slowest branch, it never splits, a cut after it
                                  costs the largest branch output (an empty branch: the
                                  previous component's)                                      */
} ffs_dag_table;

/* The plan of one request of a DAG function (88 bytes).  Slots: the plan's slices in
 * stage order, a split stage's branches in branch order. */
typedef struct {
    int64_t key;            /* FFS_KEY_NONE when not OK                                  */
    uint32_t status;        /* FFS_PLAN_*                                                 */
    uint32_t k;             /* stages                                                     */
    uint32_t cut_mask;      /* bit u = stage boundary after unit u                        */
    uint32_t split_mask;    /* bit s = stage s runs its branches on separate slices       */
    uint32_t e2e_us;        /* sum of stage times + cut transfers                         */
    uint32_t bottleneck_us; /* max stage time; throughput = 1e6 / bottleneck_us rps       */
    uint32_t gpcs;          /* sum of GPCs of every slice of the plan                     */
    uint32_t cvq;           /* floor(1024 * CV^2) of the k stage times (Eq. 1)            */
    uint32_t n_slots;       /* slices of the plan                                         */
    uint32_t pad;
    uint8_t prof[FFS_DAG_MAX_SLOTS];  /* profile of slot i (0xFF unused)                  */
    int32_t slice[FFS_DAG_MAX_SLOTS]; /* bound slice (lowest free index of the profile not
                                         taken by an earlier slot, R11), -1 unused        */
} ffs_dag_plan;

/* Validate and upload the unit structure for plans with up to k_max stages (host work:
 * the per-function list of unit-cut masks with candidate offsets).  Synchronous.
 * FFS_ERR_ARG: n_funcs differs from the staged table, units not covering a chain, a
 * branch count outside 1..4 (2..4 for a conditional unit), an empty branch outside a
 * conditional unit, a unit without components, a one-branch unit of more than one
 * component.  FFS_ERR_RANGE: > 16 units, k_max not in 1..8, k_max * max branches > 8,
 * k_max * max branches * max gpcs >= 64, >= 2^41 candidates for a function.
 * FFS_ERR_STATE: tables not staged (staging new tables drops the DAG). */
ffs_status ffs_dag_stage(ffs_ctx *ctx, const ffs_dag_table *dag, uint32_t k_max);
/* Plan every request against its home node's free slices: one warp per request walking
 * the function's unit-cut masks together, lanes over each mask's stage-option
 * combinations, every candidate scored exactly in integers, warp argmin; the winning lane
 * writes the plan and binds its slices (R11).  d_checksums (nullable; verify mode):
 * uint64[3*n_req] = candidates scored, feasible, sum of feasible keys mod 2^64.
 * Asynchronous on `stream`.  FFS_ERR_STATE: no DAG staged. */
ffs_status ffs_plan_dag(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                        ffs_dag_plan *d_out, uint64_t *d_checksums, void *stream);

/* ---- NEXT-2: joint commit of the batch ---------------------------------
 * The requests of each node are served one at a time in ascending adjusted deadline
 * (budget - reload time - fastest 1-stage latency, ties by index; R28), each
 * planned as ffs_plan_batch would against the slices still free and taking the slices
 * its plan binds (R29), so the batch's plans are jointly feasible.  Computed in monotone
 * rounds on the GPU (§4.6).  Uses context scratch; synchronous on `stream` (one host
 * read of two counters per round).  Errors as ffs_plan_keys. */
ffs_status ffs_plan_joint(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                          uint32_t k_max, ffs_plan *d_out, uint32_t *rounds, void *stream);

/* ---- NEXT-2 (routing): heterogeneity-aware request routing ---------------------
 * Per function, requests in ascending adjusted deadline (R28) are directed to the
 * function's exclusive-hot instances (d_state[i] == FFS_ST_EXCL_HOT, e.g. from
 * ffs_evict_scores) in ascending (latency d_lat_us[i], index), each taking up to
 * d_capacity[i] requests; the remaining requests go to the function's time-sharing
 * instance (lowest index in state TIME_SHARING or WARM), -1 if none (R30).
 * d_route[r] = instance index or -1 (also for func >= n_funcs).  Uses context scratch
 * (stable radix sorts); asynchronous.  FFS_ERR_RANGE: n_req or n_inst >= 2^31,
 * n_funcs >= 2^22. */
ffs_status ffs_route(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                     const ffs_instance *d_inst, const uint8_t *d_state, const uint32_t *d_lat_us,
                     const uint32_t *d_capacity, uint32_t n_inst, int32_t *d_route, void *stream);

/* ---- NEXT-4: time-sharing simulator (Fig. 8) --------------------------------
 * Simulates n_ticks ticks of tick_us on the staged cluster (slices busy in the staged
 * state belong to other tenants).  Per node every function has at most one instance;
 * the requests of node v and tick t are d_req_func/d_req_budget[d_req_off[v*n_ticks+t] ..
 * d_req_off[v*n_ticks+t+1]) and are served in that order: a resident instance serves
 * (latency = its execution time on its slice, or its plan's e2e for a pipeline);
 * otherwise the instance is built "adaptive based on available resources": on the
 * free slice of smallest (capacity, gpcs, id) that holds the function; else, when k_max >=
 * 2, as a PIPELINE over the node's free slices -- the argmin plan of ffs_plan_keys for the
 * request's budget, slices bound as ffs_plan_decode, exclusive hot and never evicted
 * (P:358); else on the slice of the least-recently-used time-sharing instance of another
 * function not used in this tick (evicted to warm); latency = reload + execution
 * (e2e); otherwise the request is unserved.  Every window_ticks an instance becomes
 * exclusive hot (not evictable) iff its busy time reached thr_pct % of the window;
 * instances idle >= cold_after_us terminate; then every pipeline for which a free slice
 * holds the whole function migrates to a non-pipeline instance on the smallest such slice
 * (a reload) and releases its slices (R31-R36, R44-R46).  k_max = 0
 * simulates monolithic instances only.  Outputs (device): d_ctr uint64[n_nodes][12] =
 * requests, served, SLO hits, unserved, reloads, evictions, terminations, occupied
 * slice-ticks, pipelines placed, migrations, requests served by pipelines, pipeline
 * slice-ticks; final per (node, function): d_slice int32 (a pipeline's stage-0 slice),
 * d_state uint8 (FFS_ST_*), d_last uint64, d_busy uint32, d_stages uint8 (0 none, 1
 * monolithic, k pipeline; all [n_nodes][n_funcs]).  FFS_ERR_RANGE: k_max > 8 or as
 * ffs_plan_keys for k_max >= 2.  Asynchronous. */
ffs_status ffs_simulate(ffs_ctx *ctx, const uint32_t *d_req_off, const uint32_t *d_req_func,
                        const uint32_t *d_req_budget, uint32_t n_ticks, uint64_t t0_us, uint32_t tick_us,
                        uint32_t window_ticks, uint32_t thr_pct, uint64_t cold_after_us, uint32_t k_max,
                        uint64_t *d_ctr, int32_t *d_slice, uint8_t *d_state, uint64_t *d_last, uint32_t *d_busy,
                        uint8_t *d_stages, void *stream);

/* ---- NEXT-3: frontier precompute ------------------------------------------------------
 * For a fixed (function, node free-vector) the feasible set depends on the budget only
 * through e2e <= B, so the argmin for any B is the lowest-key point of the Pareto
 * frontier of (key, e2e) with e2e <= B.  ffs_frontier_build computes every frontier of
 * the staged tables by peeling with the search kernels: point i+1 = the minimum key among
 * candidates with e2e < e2e(point i).  Synchronous; *n_groups and
 * *rounds report the work (nullable).  ffs_plan_frontier answers a batch from the
 * frontiers (binary search by budget + decode/bind): its plans are identical to
 * ffs_plan_batch's.  Asynchronous.  FFS_ERR_STATE: frontiers not built for these
 * tables / k_max. */
ffs_status ffs_frontier_build(ffs_ctx *ctx, uint32_t k_max, uint32_t *n_groups, uint32_t *rounds, void *stream);
ffs_status ffs_plan_frontier(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                             ffs_plan *d_out, void *stream);
/* NEXT-2 any-invoker (cross-node) planning from the same frontiers (R39): a
 * request may be served by any invoker's node -- the controller's load balancer sees every
 * invoker -- so its plan is the argmin over nodes of the per-node argmin (a
 * pipeline still never spans nodes, R10); key ties prefer the home node (req.node), then
 * the lowest node id.  One warp per request scans the function's frontier groups (one per
 * distinct node free-vector).  d_out: plans bound to the chosen node's slices; d_node
 * (nullable): int32 serving node per request, -1 when not OK.  An out-of-range func or home
 * node is FFS_PLAN_BAD_REQ.  Asynchronous.  FFS_ERR_STATE: frontiers not built. */
ffs_status ffs_plan_frontier_any(ffs_ctx *ctx, const ffs_request *d_req, const uint32_t *d_slo_us, uint32_t n_req,
                                 ffs_plan *d_out, int32_t *d_node, void *stream);

/* ---- measurement / debug helpers ------------------------------------------------------
 * K5: integer issue-rate microbenchmark over all SMs; *ops_per_s = measured lane-ops/s of
 * an IADD3/LOP3/IMAD mix (8 independent chains, 2048 threads per SM), *seconds = the
 * timed launch's duration.  Synchronous. */
ffs_status ffs_bench_int_peak(ffs_ctx *ctx, double *ops_per_s, double *seconds);
/* Packed f16x2 microbenchmark over all SMs (roofline denominator of the KS = 4 pre-filter):
 * mode 0 = HFMA2 chains only (FMA-pipe rate), mode 1 = HFMA2 chains interleaved 1:1 with
 * independent LOP3 chains, mode 2 = the same with packed max (HMNMX2): the issue-limited
 * rate.  *lane_instr_per_s = measured lane-instructions per second (each acts on two 16-bit
 * halves).  FFS_ERR_ARG for mode > 2.  Synchronous. */
ffs_status ffs_bench_packed_peak(ffs_ctx *ctx, uint32_t mode, double *lane_instr_per_s, double *seconds);
/* Device time (ms, CUDA events recorded on the launch stream around each launch) of each
 * search-kernel segment run since the last ffs_plan_keys / ffs_plan_keys_range call with
 * k_first = 1 on this context: ms[ks-1] for ks = 1..8 stages, 0 where no segment ran.
 * Waits for those events.  */
ffs_status ffs_segment_times(ffs_ctx *ctx, float *ms /* [8] */);
/* Number of candidates, since the context was created, that the fast float filter
 * rejected although their exact key would have beaten the running minimum (verify mode
 * only; must be 0).  Synchronous. */
ffs_status ffs_debug_filter_misses(ffs_ctx *ctx, uint64_t *out);
/* Candidates whose own score the search kernels computed in the last ffs_plan_keys /
 * ffs_plan_keys_range call on this context, per stage count: per_ks[ks-1], ks = 1..8
 * (device counters; in FFS_SEARCH_EXHAUSTIVE mode the sum over ks equals
 * sum_r S(n_r, k_max) of the shard; candidates the bounded mode proves infeasible without
 * scoring are not counted).  Synchronises the device.  Zeros before the first call. */
ffs_status ffs_search_scored(ffs_ctx *ctx, uint64_t *per_ks /* [8] */);
/* Live (request, mask pair) records the bounded mode's compaction kernel wrote per stage
 * count in the last search call (per_ks[ks-1]; 0 for segments that did not compact:
 * ks = 1, ks > 4, exhaustive / verify modes).  A count above the context's list capacity
 * means that segment ran on the task ranges instead.  Synchronises the device. */
ffs_status ffs_search_live_records(ffs_ctx *ctx, uint64_t *per_ks /* [8] */);

#ifdef __cplusplus
}
#endif
#endif /* FFS_H */
