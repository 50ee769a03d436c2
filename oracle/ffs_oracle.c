/*
 * ffs_oracle.c -- CPU ORACLE for the FluidFaaS batched pipeline-construction search.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_hpdc_hui0s25_b200/csrc, libffs.so) never links, includes or calls it,
 * and this file includes nothing from the product tree.
 *
 * It is the plain, slow definition of what the hot path computes, written from the
 * paper (P:<line> = line of /root/reference/PAPER.md) and the readings fixed in
 * DESIGN.md §3 (R1..R21, which restate SURVEY.md §8(c)):
 *
 *   plan  (oracle_plan)   : for every request, brute force over every contiguous split
 *                           of the component chain into k <= k_max stages (P:339,
 *                           §5.2.2, "2^4 possible consecutive partitions") and every
 *                           assignment of a MIG profile to each stage,
 *                           feasibility = SLO + memory + free slices (P:217, P:343,
 *                           P:392-394), balance = CV of stage times (Eq. 1),
 *                           selection = argmin of the packed key (R1).  Stage sums are
 *                           DIRECT sums over components ("Run all components in
 *                           stage"), no prefix tables; masks are enumerated by nested
 *                           choice of cut positions, not by the GPU's Gosper/unranking.
 *   bind                  : lowest (gpu, slice) free slice of the stage's profile in the
 *                           request's node, stages in order (R11, "available MIGs
 *                           within the invoker").
 *   evict (oracle_evict)  : multi-level keep-alive state + LRU key (§5.3).
 *   victim(oracle_victim) : LRU time-sharing victim for a request with no free-slice
 *                           plan.
 *
 * Arithmetic is exact integer arithmetic; the CV^2 quotient is taken with 128-bit
 * integers so no bound has to be argued for the oracle itself.
 *
 * Parity status: every function here is pinned by tests/test_oracle_*.py against hand
 * enumerations, the paper's worked scenarios (Fig. 1, Fig. 4, Table 5), closed forms,
 * an independent Python brute force and the north_star invariants (a)-(d).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#define ORACLE_MAX_STAGES 8
#define ORACLE_MAX_P 8
#define ORACLE_MAX_N 32
#define KEY_NONE INT64_MAX

/* per-plan status codes (R: "an infeasible request is not an error") */
#define PLAN_OK 0
#define PLAN_INFEASIBLE 1
#define PLAN_BAD_REQ 2

typedef struct {
    /* profiles, Table 2 */
    int P;
    const uint32_t *gpcs, *cap_mib;
    /* profile table, one chain per function */
    int F;
    const uint32_t *comp_off, *lat_us /* [C][P] */, *mem_mib, *xfer_us, *load_us;
    /* throughput floor (R38, NEXT-2): every stage of a plan of f runs in <= max_stage_us[f]
     * (= 10^6 / lambda_f: an instance sized for the function's load); 0 = none;
     * nullable */
    const uint32_t *max_stage_us;
    /* cluster: slices sorted by (node, gpu, slice) */
    int n_nodes, n_slices;
    const uint16_t *sl_node;
    const uint8_t *sl_gpu, *sl_slice, *sl_prof, *sl_busy;
    /* requests */
    int R;
    const uint32_t *req_func, *req_node, *req_slo_us;
    int k_max;
    /* outputs, one row per request */
    int64_t *key;
    int32_t *status, *k, *slice /* [R][8] */;
    uint32_t *cut_mask, *e2e_us, *bottleneck_us, *gpcs_out, *cvq;
    uint8_t *prof /* [R][8] */;
    uint64_t *checks /* [R][3] = scored, feasible, sum of feasible keys mod 2^64; nullable */;
} oracle_plan_args;

/* ---- state of one request's search ---------------------------------------------- */
typedef struct {
    const oracle_plan_args *a;
    int f, v, n, k;
    uint32_t B;
    uint32_t free_cnt[ORACLE_MAX_P];
    uint64_t idx; /* canonical candidate index (R1, R11) */
    int64_t best;
    int best_k;
    uint32_t best_mask;
    int best_prof[ORACLE_MAX_STAGES];
    uint64_t nfeas, ksum;
} req_state;

static uint32_t lat_of(const oracle_plan_args *a, int f, int c, int p) {
    return a->lat_us[(size_t)(a->comp_off[f] + c) * a->P + p];
}

/* R38: does a stage time t meet function f's throughput floor? */
static int within_floor(const oracle_plan_args *a, int f, uint64_t t) {
    if (a->max_stage_us == NULL || a->max_stage_us[f] == 0) return 1;
    return t <= a->max_stage_us[f];
}

/* Score every profile sequence for one cut mask (stages = maximal runs of components,
 * a cut after component j iff bit j is set; "consecutive partitions"). */
static void score_mask(req_state *s, uint32_t mask) {
    const oracle_plan_args *a = s->a;
    const int k = s->k, n = s->n, P = a->P;
    /* stage boundaries: stage i covers components [first[i], last[i]] */
    int first[ORACLE_MAX_STAGES], last[ORACLE_MAX_STAGES];
    int st = 0;
    first[0] = 0;
    for (int c = 0; c < n; c++) {
        int cut_after = (c < n - 1) && ((mask >> c) & 1u);
        if (c == n - 1 || cut_after) {
            last[st] = c;
            st++;
            if (st < k) first[st] = c + 1;
        }
    }
    /* transfer cost of the cuts (R7): one xfer per cut position, counted in e2e only */
    uint64_t xfer = 0;
    for (int j = 0; j < n - 1; j++)
        if ((mask >> j) & 1u) xfer += a->xfer_us[a->comp_off[s->f] + j];

    uint64_t nseq = 1;
    for (int i = 0; i < k; i++) nseq *= (uint64_t)P;

    for (uint64_t seq = 0; seq < nseq; seq++) {
        /* digits, p_1 most significant (R11) */
        int p[ORACLE_MAX_STAGES];
        uint64_t rest = seq;
        for (int i = k - 1; i >= 0; i--) {
            p[i] = (int)(rest % (uint64_t)P);
            rest /= (uint64_t)P;
        }
        uint64_t t[ORACLE_MAX_STAGES], m[ORACLE_MAX_STAGES];
        uint64_t sum_t = 0;
        for (int i = 0; i < k; i++) {
            t[i] = 0;
            m[i] = 0;
            for (int c = first[i]; c <= last[i]; c++) {
                t[i] += lat_of(a, s->f, c, p[i]);            /* R5: sequential stage */
                m[i] += a->mem_mib[a->comp_off[s->f] + c];    /* R6: all models loaded */
            }
            sum_t += t[i];
        }
        uint64_t e2e = sum_t + xfer;
        /* feasibility (A4): memory per slice, free slices per profile, SLO (R8 inclusive) */
        int feasible = 1;
        for (int i = 0; i < k; i++)
            if (m[i] > a->cap_mib[p[i]]) feasible = 0;
        for (int i = 0; i < k; i++)
            if (!within_floor(a, s->f, t[i])) feasible = 0; /* R38 throughput floor */
        for (int q = 0; q < P; q++) {
            uint32_t used = 0;
            for (int i = 0; i < k; i++)
                if (p[i] == q) used++;
            if (used > s->free_cnt[q]) feasible = 0;
        }
        if (e2e > s->B) feasible = 0;

        if (feasible) {
            /* Eq. 1 squared, population std (R3): CV^2 = (k*sum t^2 - (sum t)^2)/(sum t)^2 */
            unsigned __int128 sum_sq = 0;
            for (int i = 0; i < k; i++) sum_sq += (unsigned __int128)t[i] * t[i];
            unsigned __int128 D = (unsigned __int128)sum_t * sum_t;
            unsigned __int128 N = (unsigned __int128)k * sum_sq - D;
            uint64_t cvq = (uint64_t)(((unsigned __int128)1024 * N) / D); /* R4: Q10 floor */
            uint64_t g = 0;
            for (int i = 0; i < k; i++) g += a->gpcs[p[i]];
            int64_t key = (int64_t)((cvq << 50) | ((uint64_t)(k - 1) << 47) | (g << 41) | s->idx);
            if (key < s->best) {
                s->best = key;
                s->best_k = k;
                s->best_mask = mask;
                for (int i = 0; i < k; i++) s->best_prof[i] = p[i];
            }
            s->nfeas++;
            s->ksum += (uint64_t)key;
        }
        s->idx++;
    }
}

/* All masks over cut positions 0..limit-1 with `remaining` more bits, in ascending
 * numeric order: the highest cut is chosen first, ascending, then the next lower one. */
static void enum_masks(req_state *s, int remaining, int limit, uint32_t mask) {
    if (remaining == 0) {
        score_mask(s, mask);
        return;
    }
    for (int j = remaining - 1; j < limit; j++) enum_masks(s, remaining - 1, j, mask | (1u << j));
}

static uint64_t binom(int n, int r) {
    if (r < 0 || r > n) return 0;
    uint64_t c = 1;
    for (int i = 1; i <= r; i++) c = c * (uint64_t)(n - r + i) / (uint64_t)i;
    return c;
}

static void plan_one_busy(const oracle_plan_args *a, int r, const uint8_t *busy);
static void plan_one(const oracle_plan_args *a, int r) { plan_one_busy(a, r, a->sl_busy); }

/* plan request r against the slice states `busy` (free = !busy) */
static void plan_one_busy(const oracle_plan_args *a, int r, const uint8_t *busy) {
    int64_t *key = &a->key[r];
    a->status[r] = PLAN_BAD_REQ;
    *key = KEY_NONE;
    a->k[r] = 0;
    a->cut_mask[r] = 0;
    a->e2e_us[r] = 0;
    a->bottleneck_us[r] = 0;
    a->gpcs_out[r] = 0;
    a->cvq[r] = 0;
    for (int i = 0; i < ORACLE_MAX_STAGES; i++) {
        a->prof[(size_t)r * 8 + i] = 0xFF;
        a->slice[(size_t)r * 8 + i] = -1;
    }
    if (a->checks) {
        a->checks[(size_t)r * 3 + 0] = 0;
        a->checks[(size_t)r * 3 + 1] = 0;
        a->checks[(size_t)r * 3 + 2] = 0;
    }
    if (a->req_func[r] >= (uint32_t)a->F || a->req_node[r] >= (uint32_t)a->n_nodes) return;

    req_state s;
    memset(&s, 0, sizeof s);
    s.a = a;
    s.f = (int)a->req_func[r];
    s.v = (int)a->req_node[r];
    s.n = (int)(a->comp_off[s.f + 1] - a->comp_off[s.f]);
    s.B = a->req_slo_us[r];
    s.best = KEY_NONE;
    /* free slices of each profile in the request's node (R10) */
    for (int i = 0; i < a->n_slices; i++)
        if (a->sl_node[i] == s.v && !busy[i]) s.free_cnt[a->sl_prof[i]]++;

    int kmax = a->k_max < s.n ? a->k_max : s.n;
    for (int k = 1; k <= kmax; k++) {
        s.k = k;
        enum_masks(&s, k - 1, s.n - 1, 0u);
    }
    /* coverage: idx must equal S(n, K) = sum_k C(n-1, k-1) P^k */
    uint64_t S = 0;
    for (int k = 1; k <= kmax; k++) {
        uint64_t pk = 1;
        for (int i = 0; i < k; i++) pk *= (uint64_t)a->P;
        S += binom(s.n - 1, k - 1) * pk;
    }
    if (s.idx != S) abort();
    if (a->checks) {
        a->checks[(size_t)r * 3 + 0] = s.idx;
        a->checks[(size_t)r * 3 + 1] = s.nfeas;
        a->checks[(size_t)r * 3 + 2] = s.ksum;
    }
    if (s.best == KEY_NONE) {
        a->status[r] = PLAN_INFEASIBLE;
        return;
    }
    /* the plan (A6): recompute the winner's figures from the table */
    a->status[r] = PLAN_OK;
    *key = s.best;
    a->k[r] = s.best_k;
    a->cut_mask[r] = s.best_mask;
    a->cvq[r] = (uint32_t)((uint64_t)s.best >> 50);
    uint64_t e2e = 0, bott = 0, g = 0;
    int stage = 0;
    uint64_t t = 0;
    for (int c = 0; c < s.n; c++) {
        t += lat_of(a, s.f, c, s.best_prof[stage]);
        int cut_after = (c < s.n - 1) && ((s.best_mask >> c) & 1u);
        if (cut_after) e2e += a->xfer_us[a->comp_off[s.f] + c];
        if (c == s.n - 1 || cut_after) {
            e2e += t;
            if (t > bott) bott = t;
            t = 0;
            stage++;
        }
    }
    for (int i = 0; i < s.best_k; i++) g += a->gpcs[s.best_prof[i]];
    a->e2e_us[r] = (uint32_t)e2e;
    a->bottleneck_us[r] = (uint32_t)bott; /* throughput = 1e6 / bottleneck_us (R17) */
    a->gpcs_out[r] = (uint32_t)g;
    /* bind: stage i takes the lowest-index free slice of its profile in node v that no
     * earlier stage took (slices are sorted by (node, gpu, slice)) */
    for (int i = 0; i < s.best_k; i++) {
        a->prof[(size_t)r * 8 + i] = (uint8_t)s.best_prof[i];
        for (int x = 0; x < a->n_slices; x++) {
            if (a->sl_node[x] != s.v || busy[x] || a->sl_prof[x] != s.best_prof[i]) continue;
            int taken = 0;
            for (int j = 0; j < i; j++)
                if (a->slice[(size_t)r * 8 + j] == x) taken = 1;
            if (taken) continue;
            a->slice[(size_t)r * 8 + i] = x;
            break;
        }
    }
}

typedef struct {
    const oracle_plan_args *a;
    int tid, nthreads;
} worker_arg;

static void *worker(void *p) {
    worker_arg *w = (worker_arg *)p;
    for (int r = w->tid; r < w->a->R; r += w->nthreads) plan_one(w->a, r); /* interleaved */
    return NULL;
}

/* Returns 0 on success, -1 on bad arguments. */
int oracle_plan(const oracle_plan_args *a, int n_threads) {
    if (!a || a->P < 1 || a->P > ORACLE_MAX_P || a->k_max < 1 || a->k_max > ORACLE_MAX_STAGES) return -1;
    for (int f = 0; f < a->F; f++) {
        int n = (int)(a->comp_off[f + 1] - a->comp_off[f]);
        if (n < 1 || n > ORACLE_MAX_N) return -1;
    }
    if (n_threads < 1) n_threads = 1;
    if (n_threads == 1) {
        for (int r = 0; r < a->R; r++) plan_one(a, r);
        return 0;
    }
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)n_threads);
    worker_arg *wa = (worker_arg *)malloc(sizeof(worker_arg) * (size_t)n_threads);
    for (int i = 0; i < n_threads; i++) {
        wa[i].a = a;
        wa[i].tid = i;
        wa[i].nthreads = n_threads;
        pthread_create(&th[i], NULL, worker, &wa[i]);
    }
    for (int i = 0; i < n_threads; i++) pthread_join(th[i], NULL);
    free(th);
    free(wa);
    return 0;
}

/* ---- hotness-aware eviction ------------------------------------------ */
#define ST_EXCL_HOT 0
#define ST_TIME_SHARING 1
#define ST_WARM 2
#define ST_COLD 3
#define FL_PIPELINE 1u
#define FL_BUSY 2u

/* One snapshot (tick).  Rules, in order (R18-R20):
 *   idle >= cold_after                 -> COLD  ("no requests ... for 10 minutes")
 *   not resident (slice < 0)           -> WARM  (evicted to CPU memory)
 *   pipeline, or busy*100 >= thr*window -> EXCL_HOT (P:358 pipelines; P:370 threshold)
 *   otherwise                          -> TIME_SHARING (utilization below 30%)
 * evictable[i] = 1 for a resident, idle (not BUSY) time-sharing instance (LRU
 * eviction among time-sharing instances; exclusive-hot ones are exempt), idle[i] =
 * now - last_used (0 when last_used is in the future, R20b).  The least recently used
 * evictable instance is the one with the largest idle time (R20c); no packed key, so any
 * 64-bit timestamp is representable. */
void oracle_evict(int n_inst, const int32_t *inst_slice, const uint8_t *inst_flags, const uint32_t *inst_busy_us,
                  const uint64_t *inst_last_used_us, uint64_t now_us, uint32_t util_thr_pct, uint32_t window_us,
                  uint64_t cold_after_us, uint8_t *state, uint8_t *evictable, uint64_t *idle_out) {
    for (int i = 0; i < n_inst; i++) {
        uint64_t last = inst_last_used_us[i];
        uint64_t idle = now_us >= last ? now_us - last : 0;
        uint8_t st;
        if (idle >= cold_after_us)
            st = ST_COLD;
        else if (inst_slice[i] < 0)
            st = ST_WARM;
        else if ((inst_flags[i] & FL_PIPELINE) ||
                 (uint64_t)inst_busy_us[i] * 100u >= (uint64_t)util_thr_pct * window_us)
            st = ST_EXCL_HOT;
        else
            st = ST_TIME_SHARING;
        state[i] = st;
        evictable[i] = (st == ST_TIME_SHARING && !(inst_flags[i] & FL_BUSY)) ? 1 : 0;
        idle_out[i] = idle;
    }
}

/* Time-share victim for each request whose status is INFEASIBLE: among the
 * evictable instances whose slice is in the request's node, whose slice profile holds
 * the whole function (time-sharing instances are non-pipeline) and whose monolithic
 * latency plus the reload time meets the budget ("deadlines subtracted by estimated
 * execution and instance load times"), the least recently used one: the largest
 * idle time, ties to the lower instance index.  -1 when there is none or when the
 * request is not INFEASIBLE. */
void oracle_victim(const oracle_plan_args *a, const int32_t *status, int n_inst, const int32_t *inst_slice,
                   const uint8_t *evictable, const uint64_t *idle, int32_t *victim) {
    for (int r = 0; r < a->R; r++) {
        victim[r] = -1;
        if (status[r] != PLAN_INFEASIBLE) continue;
        int f = (int)a->req_func[r], v = (int)a->req_node[r];
        int n = (int)(a->comp_off[f + 1] - a->comp_off[f]);
        uint64_t mem = 0;
        for (int c = 0; c < n; c++) mem += a->mem_mib[a->comp_off[f] + c];
        int have = 0;
        uint64_t best = 0;
        for (int i = 0; i < n_inst; i++) {
            if (!evictable[i]) continue;
            int s = inst_slice[i];
            if (s < 0 || s >= a->n_slices || a->sl_node[s] != v) continue;
            int p = a->sl_prof[s];
            if (mem > a->cap_mib[p]) continue;
            uint64_t lat = 0;
            for (int c = 0; c < n; c++) lat += lat_of(a, f, c, p);
            if (lat + a->load_us[f] > a->req_slo_us[r]) continue;
            if (!within_floor(a, f, lat)) continue; /* R38: the monolithic instance meets the floor */
            if (!have || idle[i] > best) { /* strictly larger: ties keep the lower index */
                have = 1;
                best = idle[i];
                victim[r] = i;
            }
        }
    }
}

/* ---- NEXT-1: the paper's literal offline CV ranking + first-fit walk ------
 * Offline (per function): every contiguous partition with k <= k_max stages, ranked by
 * (cvq_ref, k, mask) ascending where cvq_ref = floor(1024 * CV^2) of the stage times on
 * the reference profile p_ref (R24, R25; "calculating and sorting the CVs for all possible
 * pipeline configurations ... once and offline").  Online (per request): walk the ranked
 * list and take the first partition "supported by the available resources":
 * stages in descending memory (ties: lower stage) each take a distinct free slice of the
 * smallest-capacity (then fewest-GPC, then lowest-id) profile that holds the stage; the
 * partition is supported when every stage gets one and the resulting e2e <= B (R26).
 * Plan fields as in oracle_plan, computed on the assigned profiles; key = position in the
 * ranked list (R27). */
typedef struct {
    uint64_t cvq;
    int k;
    uint32_t mask;
} ranked_entry;

static int cmp_ranked(const void *x, const void *y) {
    const ranked_entry *a = (const ranked_entry *)x, *b = (const ranked_entry *)y;
    if (a->cvq != b->cvq) return a->cvq < b->cvq ? -1 : 1;
    if (a->k != b->k) return a->k < b->k ? -1 : 1;
    if (a->mask != b->mask) return a->mask < b->mask ? -1 : 1;
    return 0;
}

typedef struct {
    ranked_entry *e;
    int n, cap;
    const oracle_plan_args *a;
    int f, nc, k, p_ref;
} rank_builder;

static void rank_add(rank_builder *b, uint32_t mask) {
    const oracle_plan_args *a = b->a;
    uint64_t t[ORACLE_MAX_STAGES] = {0}, sum = 0;
    int st = 0;
    for (int c = 0; c < b->nc; c++) {
        t[st] += lat_of(a, b->f, c, b->p_ref);
        if (c < b->nc - 1 && ((mask >> c) & 1u)) st++;
    }
    unsigned __int128 sq = 0;
    for (int i = 0; i < b->k; i++) {
        sum += t[i];
        sq += (unsigned __int128)t[i] * t[i];
    }
    unsigned __int128 D = (unsigned __int128)sum * sum;
    unsigned __int128 N = (unsigned __int128)b->k * sq - D;
    if (b->n == b->cap) {
        b->cap = b->cap ? 2 * b->cap : 64;
        b->e = (ranked_entry *)realloc(b->e, sizeof(ranked_entry) * (size_t)b->cap);
    }
    b->e[b->n].cvq = (uint64_t)(((unsigned __int128)1024 * N) / D);
    b->e[b->n].k = b->k;
    b->e[b->n].mask = mask;
    b->n++;
}

static void rank_masks(rank_builder *b, int remaining, int limit, uint32_t mask) {
    if (remaining == 0) {
        rank_add(b, mask);
        return;
    }
    for (int j = remaining - 1; j < limit; j++) rank_masks(b, remaining - 1, j, mask | (1u << j));
}

static void ranked_one(const oracle_plan_args *a, int p_ref, int r) {
    a->status[r] = PLAN_BAD_REQ;
    a->key[r] = KEY_NONE;
    a->k[r] = 0;
    a->cut_mask[r] = 0;
    a->e2e_us[r] = 0;
    a->bottleneck_us[r] = 0;
    a->gpcs_out[r] = 0;
    a->cvq[r] = 0;
    for (int i = 0; i < ORACLE_MAX_STAGES; i++) {
        a->prof[(size_t)r * 8 + i] = 0xFF;
        a->slice[(size_t)r * 8 + i] = -1;
    }
    if (a->req_func[r] >= (uint32_t)a->F || a->req_node[r] >= (uint32_t)a->n_nodes) return;
    int f = (int)a->req_func[r], v = (int)a->req_node[r];
    int n = (int)(a->comp_off[f + 1] - a->comp_off[f]);
    uint32_t free_cnt[ORACLE_MAX_P] = {0};
    for (int i = 0; i < a->n_slices; i++)
        if (a->sl_node[i] == v && !a->sl_busy[i]) free_cnt[a->sl_prof[i]]++;
    /* offline ranking of this function's partitions (recomputed here for plainness) */
    rank_builder b = {0};
    b.a = a;
    b.f = f;
    b.nc = n;
    b.p_ref = p_ref;
    int kmax = a->k_max < n ? a->k_max : n;
    for (int k = 1; k <= kmax; k++) {
        b.k = k;
        rank_masks(&b, k - 1, n - 1, 0u);
    }
    qsort(b.e, (size_t)b.n, sizeof(ranked_entry), cmp_ranked);
    /* profiles in (capacity, gpcs, id) order */
    int order[ORACLE_MAX_P];
    for (int p = 0; p < a->P; p++) order[p] = p;
    for (int i = 0; i < a->P; i++)
        for (int j = i + 1; j < a->P; j++) {
            int x = order[i], y = order[j];
            int swap = a->cap_mib[y] < a->cap_mib[x] ||
                       (a->cap_mib[y] == a->cap_mib[x] && (a->gpcs[y] < a->gpcs[x] || (a->gpcs[y] == a->gpcs[x] && y < x)));
            if (swap) {
                order[i] = y;
                order[j] = x;
            }
        }
    a->status[r] = PLAN_INFEASIBLE;
    for (int e = 0; e < b.n; e++) {
        int k = b.e[e].k;
        uint32_t mask = b.e[e].mask;
        int first[ORACLE_MAX_STAGES], last[ORACLE_MAX_STAGES], st = 0;
        first[0] = 0;
        for (int c = 0; c < n; c++) {
            int cut = (c < n - 1) && ((mask >> c) & 1u);
            if (c == n - 1 || cut) {
                last[st] = c;
                st++;
                if (st < k) first[st] = c + 1;
            }
        }
        uint64_t m[ORACLE_MAX_STAGES];
        for (int i = 0; i < k; i++) {
            m[i] = 0;
            for (int c = first[i]; c <= last[i]; c++) m[i] += a->mem_mib[a->comp_off[f] + c];
        }
        /* min-resource greedy: stages by descending memory, smallest fitting free profile */
        uint32_t left[ORACLE_MAX_P];
        for (int p = 0; p < a->P; p++) left[p] = free_cnt[p];
        int prof[ORACLE_MAX_STAGES], done[ORACLE_MAX_STAGES] = {0}, ok = 1;
        for (int step = 0; step < k && ok; step++) {
            int s = -1;
            for (int i = 0; i < k; i++)
                if (!done[i] && (s < 0 || m[i] > m[s])) s = i;
            done[s] = 1;
            prof[s] = -1;
            for (int oi = 0; oi < a->P; oi++) {
                int p = order[oi];
                uint64_t ts = 0; /* the stage's time on p, for the throughput floor (R38) */
                for (int c = first[s]; c <= last[s]; c++) ts += lat_of(a, f, c, p);
                if (left[p] > 0 && m[s] <= a->cap_mib[p] && within_floor(a, f, ts)) {
                    prof[s] = p;
                    left[p]--;
                    break;
                }
            }
            if (prof[s] < 0) ok = 0;
        }
        if (!ok) continue;
        uint64_t t[ORACLE_MAX_STAGES], e2e = 0, bott = 0, g = 0;
        unsigned __int128 sq = 0;
        uint64_t sum = 0;
        for (int i = 0; i < k; i++) {
            t[i] = 0;
            for (int c = first[i]; c <= last[i]; c++) t[i] += lat_of(a, f, c, prof[i]);
            sum += t[i];
            sq += (unsigned __int128)t[i] * t[i];
            if (t[i] > bott) bott = t[i];
            g += a->gpcs[prof[i]];
        }
        e2e = sum;
        for (int j = 0; j < n - 1; j++)
            if ((mask >> j) & 1u) e2e += a->xfer_us[a->comp_off[f] + j];
        if (e2e > a->req_slo_us[r]) continue;
        unsigned __int128 D = (unsigned __int128)sum * sum;
        unsigned __int128 N = (unsigned __int128)k * sq - D;
        a->status[r] = PLAN_OK;
        a->key[r] = e;
        a->k[r] = k;
        a->cut_mask[r] = mask;
        a->e2e_us[r] = (uint32_t)e2e;
        a->bottleneck_us[r] = (uint32_t)bott;
        a->gpcs_out[r] = (uint32_t)g;
        a->cvq[r] = (uint32_t)(((unsigned __int128)1024 * N) / D);
        for (int i = 0; i < k; i++) {
            a->prof[(size_t)r * 8 + i] = (uint8_t)prof[i];
            for (int x = 0; x < a->n_slices; x++) {
                if (a->sl_node[x] != v || a->sl_busy[x] || a->sl_prof[x] != prof[i]) continue;
                int taken = 0;
                for (int j = 0; j < i; j++)
                    if (a->slice[(size_t)r * 8 + j] == x) taken = 1;
                if (taken) continue;
                a->slice[(size_t)r * 8 + i] = x;
                break;
            }
        }
        break;
    }
    free(b.e);
}

typedef struct {
    const oracle_plan_args *a;
    int p_ref, tid, nthreads;
} ranked_worker_arg;

static void *ranked_worker(void *p) {
    ranked_worker_arg *w = (ranked_worker_arg *)p;
    for (int r = w->tid; r < w->a->R; r += w->nthreads) ranked_one(w->a, w->p_ref, r);
    return NULL;
}

int oracle_plan_ranked(const oracle_plan_args *a, int p_ref, int n_threads) {
    if (!a || a->P < 1 || a->P > ORACLE_MAX_P || a->k_max < 1 || a->k_max > ORACLE_MAX_STAGES) return -1;
    if (p_ref < 0 || p_ref >= a->P) return -1;
    if (n_threads < 1) n_threads = 1;
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)n_threads);
    ranked_worker_arg *wa = (ranked_worker_arg *)malloc(sizeof(ranked_worker_arg) * (size_t)n_threads);
    for (int i = 0; i < n_threads; i++) {
        wa[i].a = a;
        wa[i].p_ref = p_ref;
        wa[i].tid = i;
        wa[i].nthreads = n_threads;
        pthread_create(&th[i], NULL, ranked_worker, &wa[i]);
    }
    for (int i = 0; i < n_threads; i++) pthread_join(th[i], NULL);
    free(th);
    free(wa);
    return 0;
}

/* ---- NEXT-2: joint commit of a batch ----------------------------------
 * Requests of a node are served one at a time in ascending adjusted deadline
 * ("deadlines subtracted by estimated execution and instance load times"):
 * adj_r = B_r - load_f - t_exec_f, t_exec_f = the function's fastest 1-stage latency
 * (min over profiles of the sum of its component latencies) -- DESIGN.md R28; ties by
 * request index.  Each request is planned exactly as oracle_plan against the slices
 * still free, and a plan takes its bound slices (R29).  Sequential, plain. */
typedef struct {
    int64_t adj;
    int node, r;
} joint_item;

static int cmp_joint(const void *x, const void *y) {
    const joint_item *a = (const joint_item *)x, *b = (const joint_item *)y;
    if (a->node != b->node) return a->node < b->node ? -1 : 1;
    if (a->adj != b->adj) return a->adj < b->adj ? -1 : 1;
    return a->r < b->r ? -1 : (a->r > b->r);
}

int oracle_plan_joint(const oracle_plan_args *a) {
    if (!a || a->P < 1 || a->P > ORACLE_MAX_P || a->k_max < 1 || a->k_max > ORACLE_MAX_STAGES) return -1;
    uint8_t *busy = (uint8_t *)malloc((size_t)(a->n_slices > 0 ? a->n_slices : 1));
    for (int i = 0; i < a->n_slices; i++) busy[i] = a->sl_busy[i];
    joint_item *it = (joint_item *)malloc(sizeof(joint_item) * (size_t)(a->R > 0 ? a->R : 1));
    for (int r = 0; r < a->R; r++) {
        int f = (int)a->req_func[r];
        int64_t adj = (int64_t)a->req_slo_us[r];
        if (f < a->F) {
            int n = (int)(a->comp_off[f + 1] - a->comp_off[f]);
            uint64_t fast = UINT64_MAX;
            for (int p = 0; p < a->P; p++) {
                uint64_t t = 0;
                for (int c = 0; c < n; c++) t += lat_of(a, f, c, p);
                if (t < fast) fast = t;
            }
            adj -= (int64_t)a->load_us[f] + (int64_t)fast;
        }
        it[r].adj = adj;
        it[r].node = (int)a->req_node[r];
        it[r].r = r;
    }
    qsort(it, (size_t)a->R, sizeof(joint_item), cmp_joint);
    for (int i = 0; i < a->R; i++) {
        int r = it[i].r;
        plan_one_busy(a, r, busy);
        if (a->status[r] == PLAN_OK)
            for (int j = 0; j < a->k[r]; j++) busy[a->slice[(size_t)r * 8 + j]] = 1;
    }
    free(it);
    free(busy);
    return 0;
}

/* ---- NEXT-2 (routing): heterogeneity-aware request routing -------------------
 * "urgent requests are directed to the instance with the lowest latency until its
 * serving capacity is reached.  Subsequent requests are routed to the next lowest
 * latency instance, and so forth.  Then the remaining requests are routed to the time
 * sharing state instance."  Per function (R30): requests in ascending adjusted
 * deadline (R28: budget - load - fastest 1-stage latency, ties by index); exclusive-hot
 * instances of the function (state EXCL_HOT) in ascending (latency, index), each taking
 * `capacity` requests; every further request goes to the function's time-sharing
 * instance (the lowest-index instance in state TIME_SHARING or WARM), or -1 if it has
 * none.  route[r] = instance index; BAD_REQ requests (func >= F) get -1. */
typedef struct {
    int64_t a;
    uint32_t b;
    int i;
} route_item;

static int cmp_route(const void *x, const void *y) {
    const route_item *p = (const route_item *)x, *q = (const route_item *)y;
    if (p->a != q->a) return p->a < q->a ? -1 : 1;
    if (p->b != q->b) return p->b < q->b ? -1 : 1;
    return p->i < q->i ? -1 : (p->i > q->i);
}

int oracle_route(const oracle_plan_args *a, int n_inst, const uint32_t *inst_func, const uint8_t *inst_state,
                 const uint32_t *inst_lat, const uint32_t *inst_cap, int32_t *route) {
    for (int f = 0; f < a->F; f++) {
        /* requests of f in adjusted-deadline order */
        int nr = 0;
        route_item *rq = (route_item *)malloc(sizeof(route_item) * (size_t)(a->R > 0 ? a->R : 1));
        int n = (int)(a->comp_off[f + 1] - a->comp_off[f]);
        uint64_t fast = UINT64_MAX;
        for (int p = 0; p < a->P; p++) {
            uint64_t t = 0;
            for (int c = 0; c < n; c++) t += lat_of(a, f, c, p);
            if (t < fast) fast = t;
        }
        for (int r = 0; r < a->R; r++)
            if ((int)a->req_func[r] == f) {
                rq[nr].a = (int64_t)a->req_slo_us[r] - (int64_t)a->load_us[f] - (int64_t)fast;
                rq[nr].b = (uint32_t)r;
                rq[nr].i = r;
                nr++;
            }
        qsort(rq, (size_t)nr, sizeof(route_item), cmp_route);
        /* exclusive-hot instances of f by (latency, index); the time-sharing instance */
        int nh = 0, ts = -1;
        route_item *hot = (route_item *)malloc(sizeof(route_item) * (size_t)(n_inst > 0 ? n_inst : 1));
        for (int i = 0; i < n_inst; i++) {
            if ((int)inst_func[i] != f) continue;
            if (inst_state[i] == ST_EXCL_HOT) {
                hot[nh].a = inst_lat[i];
                hot[nh].b = (uint32_t)i;
                hot[nh].i = i;
                nh++;
            } else if ((inst_state[i] == ST_TIME_SHARING || inst_state[i] == ST_WARM) && ts < 0) {
                ts = i;
            }
        }
        qsort(hot, (size_t)nh, sizeof(route_item), cmp_route);
        int h = 0;
        uint64_t used = 0;
        for (int j = 0; j < nr; j++) {
            while (h < nh && used >= inst_cap[hot[h].i]) {
                h++;
                used = 0;
            }
            if (h < nh) {
                route[rq[j].i] = hot[h].i;
                used++;
            } else {
                route[rq[j].i] = ts;
            }
        }
        free(rq);
        free(hot);
    }
    for (int r = 0; r < a->R; r++)
        if (a->req_func[r] >= (uint32_t)a->F) route[r] = -1;
    return 0;
}

/* ---- NEXT-4: time-sharing simulator (Fig. 8) -------------------------------
 * DESIGN.md R31-R36, R44-R46.  Each node (invoker) is simulated independently; per node
 * every function has at most one instance (created on its first request there).  Ticks of
 * tick_us; the requests of a tick are served in trace order:
 *   resident monolithic instance -> served, latency = exec on its slice's profile;
 *   resident pipeline instance   -> served, latency = the plan's e2e (R45);
 *   otherwise (warm / new): "the construction of that instance should be flexible and
 *     adaptive based on available resources ... a two-stage or three-stage pipeline, or ...
 *     a non-pipeline process":
 *     (1) the free slice with the smallest (capacity, gpcs, id) that holds the function
 *         (monolithic, time-sharing), latency = load + exec (R33);
 *     (2) else a PIPELINE over the node's free slices: the argmin plan of the search
 *         (oracle_plan, R1) with the request's budget, slices bound per R11; pipeline
 *         instances are exclusive hot and never evicted ("All pipeline instances are in the
 *         exclusive hot state"), latency = load + e2e (R44);
 *     (3) else the slice of the least recently used (ties: lower slice) time-sharing
 *         instance of another function not used in this tick whose slice holds the
 *         function (the victim goes warm: P:364), latency = load + exec (R33);
 *     otherwise unserved.  A served request is an SLO hit when its latency <= its budget.
 *   A served request adds its service time (exec, or e2e for a pipeline) to the instance's
 *   busy time and sets its last use to now.
 * At the end of every tick the occupied slices are counted; every window_ticks the
 * instances whose busy time reached thr% of the window become exclusive hot (exempt from
 * eviction) for the next window, the others time-sharing, busy resets;
 * instances idle >= cold_after are terminated, releasing their slices; then
 * every pipeline instance (function order) for which a free slice now holds the whole
 * function migrates to a new non-pipeline instance on the smallest such slice and releases
 * its slices ("migrates pipeline instances to non-pipeline instances when large MIG
 * slices become available"); the new instance loads its model (a reload) and keeps the
 * function's hotness (R46).
 * Slices busy in the staged cluster belong to other tenants and are never used.
 * ctr[v][12] = requests, served, SLO hits, unserved, reloads, evictions, terminations,
 * occupied slice-ticks, pipelines placed, migrations, requests served by a pipeline
 * (including the one that placed it), pipeline slice-ticks.  Final per (node, function): slice (a pipeline: its stage-0
 * slice), state, last use, busy, stages (0 none, 1 monolithic, k >= 2 pipeline). */
#define SIM_CTR 12
int oracle_sim(const oracle_plan_args *a, int T, const uint32_t *req_off, const uint32_t *req_func,
               const uint32_t *req_budget, uint64_t t0_us, uint32_t tick_us, uint32_t window_ticks,
               uint32_t thr_pct, uint64_t cold_after_us, uint64_t *ctr, int32_t *fin_slice, uint8_t *fin_state,
               uint64_t *fin_last, uint32_t *fin_busy, uint8_t *fin_k) {
    const int F = a->F, P = a->P;
    /* per function: exec on each profile, total memory, reload */
    uint64_t *exec = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)F * (size_t)P);
    uint64_t *memt = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)F);
    for (int f = 0; f < F; f++) {
        int n = (int)(a->comp_off[f + 1] - a->comp_off[f]);
        memt[f] = 0;
        for (int c = 0; c < n; c++) memt[f] += a->mem_mib[a->comp_off[f] + c];
        for (int p = 0; p < P; p++) {
            uint64_t t = 0;
            for (int c = 0; c < n; c++) t += lat_of(a, f, c, p);
            exec[(size_t)f * P + p] = t;
        }
    }
    const int NS = a->n_slices > 0 ? a->n_slices : 1;
    int *res = (int *)malloc(sizeof(int) * (size_t)NS);
    uint8_t *occ = (uint8_t *)malloc((size_t)NS);
    /* one-request plan arguments for the pipeline search (R44): the staged tables, the
     * simulated slice occupancy as "busy" */
    oracle_plan_args b = *a;
    uint32_t q_func = 0, q_node = 0, q_slo = 0;
    int64_t o_key;
    int32_t o_status, o_k, o_slice[8];
    uint32_t o_cut, o_e2e, o_bott, o_g, o_cvq;
    uint8_t o_prof[8];
    b.R = 1;
    b.req_func = &q_func;
    b.req_node = &q_node;
    b.req_slo_us = &q_slo;
    b.key = &o_key;
    b.status = &o_status;
    b.k = &o_k;
    b.slice = o_slice;
    b.cut_mask = &o_cut;
    b.e2e_us = &o_e2e;
    b.bottleneck_us = &o_bott;
    b.gpcs_out = &o_g;
    b.cvq = &o_cvq;
    b.prof = o_prof;
    b.checks = NULL;
    for (int v = 0; v < a->n_nodes; v++) {
        uint64_t *C = ctr + (size_t)v * SIM_CTR;
        for (int i = 0; i < SIM_CTR; i++) C[i] = 0;
        int32_t *sl = fin_slice + (size_t)v * F;
        uint8_t *st = fin_state + (size_t)v * F;
        uint64_t *last = fin_last + (size_t)v * F;
        uint32_t *busy = fin_busy + (size_t)v * F;
        uint8_t *exists = (uint8_t *)calloc((size_t)F, 1), *hot = (uint8_t *)calloc((size_t)F, 1);
        uint8_t *pk = (uint8_t *)calloc((size_t)F, 1); /* pipeline stages, 0 = no pipeline */
        int32_t *psl = (int32_t *)malloc(sizeof(int32_t) * (size_t)F * 8);
        uint64_t *pe2e = (uint64_t *)calloc((size_t)F, sizeof(uint64_t));
        for (int f = 0; f < F; f++) {
            sl[f] = -1;
            last[f] = 0;
            busy[f] = 0;
        }
        for (int s = 0; s < a->n_slices; s++) res[s] = -1;
        for (int t = 0; t < T; t++) {
            uint64_t now = t0_us + (uint64_t)t * tick_us;
            for (uint32_t j = req_off[(size_t)v * T + t]; j < req_off[(size_t)v * T + t + 1]; j++) {
                int f = (int)req_func[j];
                uint64_t B = req_budget[j];
                C[0]++;
                if (!exists[f]) {
                    exists[f] = 1;
                    sl[f] = -1;
                    hot[f] = 0;
                    busy[f] = 0;
                    last[f] = now;
                }
                uint64_t latency = 0, ex = 0;
                int ok = 0;
                if (sl[f] >= 0) {
                    ex = exec[(size_t)f * P + a->sl_prof[sl[f]]];
                    latency = ex;
                    ok = 1;
                } else if (pk[f] >= 2) {
                    ex = pe2e[f];
                    latency = ex;
                    ok = 1;
                    C[10]++;
                } else {
                    /* (1) smallest free slice that holds the function */
                    int best = -1;
                    for (int s = 0; s < a->n_slices; s++) {
                        if (a->sl_node[s] != v || a->sl_busy[s] || res[s] >= 0) continue;
                        int p = a->sl_prof[s];
                        if (memt[f] > a->cap_mib[p]) continue;
                        if (best < 0) {
                            best = s;
                            continue;
                        }
                        int q = a->sl_prof[best];
                        if (a->cap_mib[p] < a->cap_mib[q] || (a->cap_mib[p] == a->cap_mib[q] && a->gpcs[p] < a->gpcs[q]))
                            best = s;
                    }
                    if (best < 0) {
                        /* (2) a pipeline over the free slices: the plan search's argmin */
                        int any_free = 0;
                        for (int s = 0; s < a->n_slices; s++) {
                            occ[s] = (uint8_t)(a->sl_busy[s] || res[s] >= 0);
                            if (a->sl_node[s] == v && !occ[s]) any_free = 1;
                        }
                        if (any_free) {
                            q_func = (uint32_t)f;
                            q_node = (uint32_t)v;
                            q_slo = (uint32_t)(B > 0xffffffffull ? 0xffffffffull : B);
                            plan_one_busy(&b, 0, occ);
                            if (o_status == PLAN_OK) {
                                pk[f] = (uint8_t)o_k;
                                for (int i = 0; i < o_k; i++) {
                                    psl[(size_t)f * 8 + i] = o_slice[i];
                                    res[o_slice[i]] = f;
                                }
                                pe2e[f] = o_e2e;
                                C[8]++;
                                C[4]++;
                                C[10]++;
                                ex = o_e2e;
                                latency = a->load_us[f] + ex;
                                ok = 1;
                            }
                        }
                    }
                    if (!ok && best < 0) {
                        /* (3) evict the LRU time-sharing instance of another function */
                        for (int s = 0; s < a->n_slices; s++) {
                            if (a->sl_node[s] != v || res[s] < 0 || res[s] == f) continue;
                            int g = res[s], p = a->sl_prof[s];
                            if (pk[g] >= 2 || hot[g] || last[g] >= now) continue;
                            if (memt[f] > a->cap_mib[p]) continue;
                            if (best < 0 || last[g] < last[res[best]]) best = s;
                        }
                        if (best >= 0) {
                            sl[res[best]] = -1; /* evicted to CPU memory: warm */
                            res[best] = -1;
                            C[5]++;
                        }
                    }
                    if (!ok && best >= 0) {
                        res[best] = f;
                        sl[f] = best;
                        C[4]++;
                        ex = exec[(size_t)f * P + a->sl_prof[best]];
                        latency = a->load_us[f] + ex;
                        ok = 1;
                    }
                }
                if (ok) {
                    C[1]++;
                    if (latency <= B) C[2]++;
                    busy[f] += (uint32_t)ex;
                    last[f] = now;
                } else {
                    C[3]++;
                }
            }
            for (int s = 0; s < a->n_slices; s++)
                if (a->sl_node[s] == v && res[s] >= 0) {
                    C[7]++;
                    if (pk[res[s]] >= 2) C[11]++;
                }
            if ((uint32_t)(t + 1) % window_ticks == 0) {
                uint64_t window_us = (uint64_t)window_ticks * tick_us;
                for (int f = 0; f < F; f++) {
                    hot[f] = (uint64_t)busy[f] * 100u >= (uint64_t)thr_pct * window_us;
                    busy[f] = 0;
                }
            }
            for (int f = 0; f < F; f++) {
                if (exists[f] && now - last[f] >= cold_after_us) {
                    if (sl[f] >= 0) res[sl[f]] = -1;
                    for (int i = 0; i < pk[f]; i++) res[psl[(size_t)f * 8 + i]] = -1;
                    pk[f] = 0;
                    exists[f] = 0;
                    sl[f] = -1;
                    hot[f] = 0;
                    busy[f] = 0;
                    C[6]++;
                }
            }
            /* pipeline migration (R46) */
            for (int f = 0; f < F; f++) {
                if (pk[f] < 2) continue;
                int best = -1;
                for (int s = 0; s < a->n_slices; s++) {
                    if (a->sl_node[s] != v || a->sl_busy[s] || res[s] >= 0) continue;
                    int p = a->sl_prof[s];
                    if (memt[f] > a->cap_mib[p]) continue;
                    if (best < 0) {
                        best = s;
                        continue;
                    }
                    int q = a->sl_prof[best];
                    if (a->cap_mib[p] < a->cap_mib[q] || (a->cap_mib[p] == a->cap_mib[q] && a->gpcs[p] < a->gpcs[q]))
                        best = s;
                }
                if (best < 0) continue;
                for (int i = 0; i < pk[f]; i++) res[psl[(size_t)f * 8 + i]] = -1;
                pk[f] = 0;
                res[best] = f;
                sl[f] = best;
                C[9]++;
                C[4]++;
            }
        }
        for (int f = 0; f < F; f++) {
            st[f] = !exists[f] ? ST_COLD
                               : (pk[f] >= 2 ? ST_EXCL_HOT : (sl[f] < 0 ? ST_WARM : (hot[f] ? ST_EXCL_HOT : ST_TIME_SHARING)));
            fin_k[(size_t)v * F + f] = pk[f] >= 2 ? pk[f] : (sl[f] >= 0 ? 1 : 0);
            if (pk[f] >= 2) sl[f] = psl[(size_t)f * 8];
        }
        free(exists);
        free(hot);
        free(pk);
        free(psl);
        free(pe2e);
    }
    free(res);
    free(occ);
    free(exec);
    free(memt);
    return 0;
}

/* ==== NEXT-1 DAG stages (oracle_plan_dag; R40-R43) ======================
 * The FFS DAG of a function ("represents the components in the function as nodes
 * and dataflows among them as edges") is read as a series of UNITS: a unit is one
 * component or a parallel block of 2..4 branches (fork/join), each branch a chain of
 * components (the expanded image classification app "is extended with two
 * branches to form a DAG").  Components are numbered unit by unit, branch by branch.
 *   R40 cuts: only between units -- the dominators of a series-parallel DAG ("based
 *       on the dominator-based method from ESG"); a stage is a run of consecutive units.
 *   R41 a stage runs on ONE slice (all its components in sequence: t = sum of their
 *       latencies, memory = sum), or -- only when the stage is exactly one parallel block --
 *       SPLIT: branch j on its own slice of profile p_j, t = max_j (branch time) ("If a
 *       stage involves multiple MIGs running in parallel, we use the maximum execution time
 *       among them as the stage's execution time"), memory checked per branch slice.
 *   R42 a cut after a unit moves every branch output: cost = sum over its branches of the
 *       xfer_us of the branch's last component (one component: its xfer_us, as R7).
 *   R43 candidate order: k ascending, unit-cut masks ascending, stage options in mixed
 *       radix (stage 0 most significant); option o < P = one slice of profile o, o = P + w
 *       = split with branch profiles the base-P digits of w (branch 0 most significant).
 *       idx = the candidate's position; key, feasibility and binding as R1-R11 with every
 *       slice of the plan counted (gpcs, free slices), slots in stage then branch order;
 *       k_max * (max branches) <= 8, so a plan holds at most 8 slices.
 *   R48 a CONDITIONAL unit (App 3, Table 4: "Deblur -> (if low resolution: -> Super
 *       resolution; else: pass) -> ...") holds 2..4 alternative branches of which exactly
 *       one runs per request (a branch may be empty: "pass"): the instance hosts all of
 *       them (memory = every branch's components), the unit's time on a slice is its
 *       slowest branch (the SLO must hold whichever branch a request takes; the profile
 *       table carries no branch probabilities), alternatives are never split over slices,
 *       and a cut after the unit moves the output of the branch that ran: the largest of
 *       the branches' last-component xfer_us (an empty branch passes the previous
 *       component's output; nothing before the first component).
 * A DAG of one-component units is the chain of oracle_plan, candidate for candidate. */
#define DAG_MAX_UNITS 16
#define DAG_MAX_BR 4
#define DAG_MAX_SLOTS 8

typedef struct {
    const uint32_t *unit_off; /* [F+1] */
    const uint8_t *unit_nb;   /* [U] branches, 1..4 */
    const uint8_t *unit_bend; /* [U][4] function-relative exclusive end component of branch j */
    const uint8_t *unit_cond; /* [U] nullable: 1 = conditional unit (R48) */
    int64_t *key;
    int32_t *status, *k, *slice /* [R][8] */;
    uint32_t *cut_mask, *split_mask, *e2e_us, *bottleneck_us, *gpcs_out, *cvq, *n_slots;
    uint8_t *prof /* [R][8] */;
    uint64_t *checks /* [R][3], nullable */;
} oracle_dag_args;

typedef struct {
    int nb, c0, cond;         /* branches, first component (function-relative), R48 */
    int bc0[DAG_MAX_BR], bc1[DAG_MAX_BR]; /* branch j = components [bc0, bc1) */
} dag_unit;

/* cost of a cut right after unit un (R42; R48 for a conditional unit) */
static uint64_t dag_cut_cost(const oracle_plan_args *a, uint32_t base, const dag_unit *un) {
    uint64_t x = 0;
    for (int j = 0; j < un->nb; j++) {
        uint64_t xb = 0;
        if (un->bc1[j] > un->bc0[j]) xb = a->xfer_us[base + (uint32_t)un->bc1[j] - 1];
        else if (un->c0 > 0) xb = a->xfer_us[base + (uint32_t)un->c0 - 1]; /* "pass" */
        if (un->cond) x = xb > x ? xb : x;
        else x += xb;
    }
    return x;
}

static void plan_dag_one(const oracle_plan_args *a, const oracle_dag_args *d, int r) {
    const int P = a->P;
    d->status[r] = PLAN_BAD_REQ;
    d->key[r] = KEY_NONE;
    d->k[r] = 0;
    d->cut_mask[r] = d->split_mask[r] = d->e2e_us[r] = d->bottleneck_us[r] = 0;
    d->gpcs_out[r] = d->cvq[r] = d->n_slots[r] = 0;
    for (int i = 0; i < DAG_MAX_SLOTS; i++) {
        d->prof[(size_t)r * DAG_MAX_SLOTS + i] = 0xFF;
        d->slice[(size_t)r * DAG_MAX_SLOTS + i] = -1;
    }
    if (d->checks)
        for (int i = 0; i < 3; i++) d->checks[(size_t)r * 3 + i] = 0;
    if (a->req_func[r] >= (uint32_t)a->F || a->req_node[r] >= (uint32_t)a->n_nodes) return;
    const int f = (int)a->req_func[r], v = (int)a->req_node[r];
    const uint32_t base = a->comp_off[f], B = a->req_slo_us[r];
    const int m = (int)(d->unit_off[f + 1] - d->unit_off[f]);
    dag_unit U[DAG_MAX_UNITS];
    int c = 0;
    for (int u = 0; u < m; u++) {
        const uint32_t gu = d->unit_off[f] + (uint32_t)u;
        U[u].nb = d->unit_nb[gu];
        U[u].c0 = c;
        U[u].cond = d->unit_cond ? d->unit_cond[gu] : 0;
        for (int j = 0; j < U[u].nb; j++) {
            U[u].bc0[j] = c;
            U[u].bc1[j] = d->unit_bend[(size_t)gu * DAG_MAX_BR + j];
            c = U[u].bc1[j];
        }
    }
    uint32_t free_cnt[ORACLE_MAX_P] = {0};
    for (int i = 0; i < a->n_slices; i++)
        if (a->sl_node[i] == v && !a->sl_busy[i]) free_cnt[a->sl_prof[i]]++;

    int64_t best = KEY_NONE;
    int best_k = 0, best_nsl = 0;
    uint32_t best_mask = 0, best_split = 0;
    int best_prof[DAG_MAX_SLOTS];
    uint64_t idx = 0, nfeas = 0, ksum = 0;
    const int kmax = a->k_max < m ? a->k_max : m;
    for (int k = 1; k <= kmax; k++) {
        for (uint32_t mask = 0; mask < (1u << (m - 1)); mask++) {
            if (__builtin_popcount(mask) != k - 1) continue;
            /* stages: runs of units; stage s = units [su0[s], su1[s]] */
            int su0[ORACLE_MAX_STAGES], su1[ORACLE_MAX_STAGES], st = 0;
            su0[0] = 0;
            uint64_t xfer = 0;
            for (int u = 0; u < m; u++) {
                const int cut = u < m - 1 && ((mask >> u) & 1u);
                if (cut) xfer += dag_cut_cost(a, base, &U[u]);
                if (u == m - 1 || cut) {
                    su1[st] = u;
                    st++;
                    if (st < k) su0[st] = u + 1;
                }
            }
            uint64_t nopt[ORACLE_MAX_STAGES], total = 1;
            for (int s = 0; s < k; s++) {
                const int blk = su0[s] == su1[s] && U[su0[s]].nb >= 2 && !U[su0[s]].cond;
                uint64_t pb = 1;
                if (blk)
                    for (int j = 0; j < U[su0[s]].nb; j++) pb *= (uint64_t)P;
                nopt[s] = (uint64_t)P + (blk ? pb : 0);
                total *= nopt[s];
            }
            for (uint64_t o = 0; o < total; o++, idx++) {
                uint64_t opt[ORACLE_MAX_STAGES], rest = o;
                for (int s = k - 1; s >= 0; s--) {
                    opt[s] = rest % nopt[s];
                    rest /= nopt[s];
                }
                uint64_t t[ORACLE_MAX_STAGES], sum_t = 0, g = 0;
                int prof[DAG_MAX_SLOTS], nsl = 0, feasible = 1;
                uint32_t split = 0;
                for (int s = 0; s < k; s++) {
                    if (opt[s] < (uint64_t)P) { /* one slice: every component of the stage */
                        const int p = (int)opt[s];
                        uint64_t ts = 0, ms = 0;
                        for (int u = su0[s]; u <= su1[s]; u++) {
                            uint64_t tu = 0; /* the unit's time: sum, or the slowest alternative (R48) */
                            for (int j = 0; j < U[u].nb; j++) {
                                uint64_t tb = 0;
                                for (int cc = U[u].bc0[j]; cc < U[u].bc1[j]; cc++) {
                                    tb += lat_of(a, f, cc, p);
                                    ms += a->mem_mib[base + (uint32_t)cc];
                                }
                                if (U[u].cond) tu = tb > tu ? tb : tu;
                                else tu += tb;
                            }
                            ts += tu;
                        }
                        if (ms > a->cap_mib[p]) feasible = 0;
                        t[s] = ts;
                        prof[nsl++] = p;
                    } else { /* split: branch j on its own slice, the stage takes the max */
                        const dag_unit *un = &U[su0[s]];
                        int pj[DAG_MAX_BR];
                        uint64_t w = opt[s] - (uint64_t)P;
                        for (int j = un->nb - 1; j >= 0; j--) {
                            pj[j] = (int)(w % (uint64_t)P);
                            w /= (uint64_t)P;
                        }
                        uint64_t ts = 0;
                        for (int j = 0; j < un->nb; j++) {
                            uint64_t tb = 0, mb = 0;
                            for (int cc = un->bc0[j]; cc < un->bc1[j]; cc++) {
                                tb += lat_of(a, f, cc, pj[j]);
                                mb += a->mem_mib[base + (uint32_t)cc];
                            }
                            if (mb > a->cap_mib[pj[j]]) feasible = 0;
                            if (tb > ts) ts = tb;
                            prof[nsl++] = pj[j];
                        }
                        t[s] = ts;
                        split |= 1u << s;
                    }
                    if (!within_floor(a, f, t[s])) feasible = 0;
                    sum_t += t[s];
                }
                for (int i = 0; i < nsl; i++) g += a->gpcs[prof[i]];
                for (int q = 0; q < P; q++) {
                    uint32_t used = 0;
                    for (int i = 0; i < nsl; i++) used += prof[i] == q;
                    if (used > free_cnt[q]) feasible = 0;
                }
                if (sum_t + xfer > B) feasible = 0;
                if (!feasible) continue;
                unsigned __int128 sum_sq = 0;
                for (int s = 0; s < k; s++) sum_sq += (unsigned __int128)t[s] * t[s];
                unsigned __int128 D = (unsigned __int128)sum_t * sum_t;
                unsigned __int128 N = (unsigned __int128)k * sum_sq - D;
                uint64_t cvq = (uint64_t)(((unsigned __int128)1024 * N) / D); /* Eq. 1, R3, R4 */
                int64_t key = (int64_t)((cvq << 50) | ((uint64_t)(k - 1) << 47) | (g << 41) | idx);
                nfeas++;
                ksum += (uint64_t)key;
                if (key < best) {
                    best = key;
                    best_k = k;
                    best_mask = mask;
                    best_split = split;
                    best_nsl = nsl;
                    for (int i = 0; i < nsl; i++) best_prof[i] = prof[i];
                }
            }
        }
    }
    if (d->checks) {
        d->checks[(size_t)r * 3 + 0] = idx;
        d->checks[(size_t)r * 3 + 1] = nfeas;
        d->checks[(size_t)r * 3 + 2] = ksum;
    }
    if (best == KEY_NONE) {
        d->status[r] = PLAN_INFEASIBLE;
        return;
    }
    d->status[r] = PLAN_OK;
    d->key[r] = best;
    d->k[r] = best_k;
    d->cut_mask[r] = best_mask;
    d->split_mask[r] = best_split;
    d->cvq[r] = (uint32_t)((uint64_t)best >> 50);
    d->n_slots[r] = (uint32_t)best_nsl;
    /* the plan's figures, recomputed from the winner (stage times as in the search) */
    uint64_t e2e = 0, bott = 0, g = 0;
    int s = 0, slot = 0;
    uint64_t tcur = 0;
    for (int u = 0; u < m; u++) {
        const int cut = u < m - 1 && ((best_mask >> u) & 1u);
        if ((best_split >> s) & 1u) {
            for (int j = 0; j < U[u].nb; j++) {
                uint64_t tb = 0;
                for (int cc = U[u].bc0[j]; cc < U[u].bc1[j]; cc++) tb += lat_of(a, f, cc, best_prof[slot + j]);
                if (tb > tcur) tcur = tb;
            }
        } else {
            uint64_t tu = 0;
            for (int j = 0; j < U[u].nb; j++) {
                uint64_t tb = 0;
                for (int cc = U[u].bc0[j]; cc < U[u].bc1[j]; cc++) tb += lat_of(a, f, cc, best_prof[slot]);
                if (U[u].cond) tu = tb > tu ? tb : tu;
                else tu += tb;
            }
            tcur += tu;
        }
        if (cut) e2e += dag_cut_cost(a, base, &U[u]);
        if (u == m - 1 || cut) {
            e2e += tcur;
            if (tcur > bott) bott = tcur;
            slot += ((best_split >> s) & 1u) ? U[u].nb : 1;
            tcur = 0;
            s++;
        }
    }
    for (int i = 0; i < best_nsl; i++) g += a->gpcs[best_prof[i]];
    d->e2e_us[r] = (uint32_t)e2e;
    d->bottleneck_us[r] = (uint32_t)bott;
    d->gpcs_out[r] = (uint32_t)g;
    /* bind (R11): slot i takes the lowest-index free slice of its profile in node v that
     * no earlier slot took */
    for (int i = 0; i < best_nsl; i++) {
        d->prof[(size_t)r * DAG_MAX_SLOTS + i] = (uint8_t)best_prof[i];
        for (int x = 0; x < a->n_slices; x++) {
            if (a->sl_node[x] != v || a->sl_busy[x] || a->sl_prof[x] != best_prof[i]) continue;
            int taken = 0;
            for (int j = 0; j < i; j++)
                if (d->slice[(size_t)r * DAG_MAX_SLOTS + j] == x) taken = 1;
            if (taken) continue;
            d->slice[(size_t)r * DAG_MAX_SLOTS + i] = x;
            break;
        }
    }
}

typedef struct {
    const oracle_plan_args *a;
    const oracle_dag_args *d;
    int tid, nthreads;
} dag_worker_arg;

static void *dag_worker(void *p) {
    dag_worker_arg *w = (dag_worker_arg *)p;
    for (int r = w->tid; r < w->a->R; r += w->nthreads) plan_dag_one(w->a, w->d, r);
    return NULL;
}

/* Returns 0, or -1 for a malformed DAG table (units not covering the chain, a branch
 * count outside 1..4, > 16 units, an empty branch, a one-branch unit of more than one
 * component), k_max * (max branches) > 8 (slices per plan) or k_max * (max branches) *
 * max gpcs >= 64 (the 6-bit key field). */
int oracle_plan_dag(const oracle_plan_args *a, const oracle_dag_args *d, int n_threads) {
    if (a->P < 1 || a->P > ORACLE_MAX_P || a->k_max < 1 || a->k_max > ORACLE_MAX_STAGES) return -1;
    uint32_t maxg = 0, maxnb = 1;
    for (int p = 0; p < a->P; p++)
        if (a->gpcs[p] > maxg) maxg = a->gpcs[p];
    for (int f = 0; f < a->F; f++) {
        const int n = (int)(a->comp_off[f + 1] - a->comp_off[f]);
        const int m = (int)(d->unit_off[f + 1] - d->unit_off[f]);
        if (m < 1 || m > DAG_MAX_UNITS) return -1;
        int c = 0;
        for (int u = 0; u < m; u++) {
            const uint32_t gu = d->unit_off[f] + (uint32_t)u;
            const int nb = d->unit_nb[gu];
            const int cond = d->unit_cond ? d->unit_cond[gu] : 0;
            if (nb < 1 || nb > DAG_MAX_BR || (cond && nb < 2)) return -1;
            if (!cond && (uint32_t)nb > maxnb) maxnb = (uint32_t)nb; /* alternatives never split */
            const int start = c;
            for (int j = 0; j < nb; j++) {
                const int e = d->unit_bend[(size_t)gu * DAG_MAX_BR + j];
                if (cond ? e < c : e <= c) return -1; /* an alternative may be empty ("pass") */
                c = e;
            }
            if (c == start) return -1; /* a unit holds at least one component */
        }
        if (c != n) return -1;
        for (int u = 0; u < m; u++) { /* a one-branch unit is one component */
            const uint32_t gu = d->unit_off[f] + (uint32_t)u;
            const int start = u == 0 ? 0 : (int)d->unit_bend[(size_t)(gu - 1) * DAG_MAX_BR + d->unit_nb[gu - 1] - 1];
            if (d->unit_nb[gu] == 1 && d->unit_bend[(size_t)gu * DAG_MAX_BR] != start + 1) return -1;
        }
    }
    if ((uint64_t)a->k_max * maxnb > DAG_MAX_SLOTS || (uint64_t)a->k_max * maxnb * maxg >= 64) return -1;
    if (n_threads < 1) n_threads = 1;
    pthread_t th[256];
    dag_worker_arg w[256];
    if (n_threads > 256) n_threads = 256;
    for (int i = 0; i < n_threads; i++) {
        w[i].a = a;
        w[i].d = d;
        w[i].tid = i;
        w[i].nthreads = n_threads;
        pthread_create(&th[i], NULL, dag_worker, &w[i]);
    }
    for (int i = 0; i < n_threads; i++) pthread_join(th[i], NULL);
    return 0;
}
