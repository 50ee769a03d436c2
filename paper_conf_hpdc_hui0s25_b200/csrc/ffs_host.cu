// ffs_host.cu -- host side of libffs.so: context, validation and staging of the tables
// (A0), scratch management and the C-ABI entry points declared in include/ffs.h.
#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "ffs_internal.h"

using namespace ffsk;

namespace {

struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  cudaError_t ensure(size_t n) {
    if (n <= bytes) return cudaSuccess;
    if (p) cudaFree(p);
    p = nullptr;
    bytes = 0;
    cudaError_t e = cudaMalloc(&p, n);
    if (e == cudaSuccess) bytes = n;
    return e;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    bytes = 0;
  }
  template <class T>
  T* as() const { return reinterpret_cast<T*>(p); }
};

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

}  // namespace

static_assert(sizeof(ffs_dag_plan) == 88, "ffs_dag_plan layout");

struct ffs_ctx {
  int device = 0;
  int sms = 0;
  std::string err;
  // staged tables
  bool staged = false;
  ImageLayout lay{};
  uint32_t P = 0, F = 0, n_nodes = 0, n_slices = 0, max_n = 0, max_gpcs = 0;
  std::vector<uint32_t> fn_len;
  DevBuf image, node_free, free_list, slice_node, slice_prof;
  std::vector<uint32_t> h_image;  // host copy of the table image (offline ranking)
  ImageLayout h_lay{};
  // NEXT-2 joint commit: staged slice states and per-node slice ranges
  std::vector<uint8_t> h_busy, h_cnt;
  std::vector<uint64_t> h_node_free;
  DevBuf node_off, j_keys, j_state, j_dirty, j_sreq, j_sslo, j_skeys, j_win, j_busy, j_cnt, j_free, j_ctr;
  // NEXT-2 routing scratch
  DevBuf r_k, r_k2, r_v, r_v2, i_k, i_k2, i_v, i_v2, i_cum, r_f, r_h, r_n, r_ts, r_hist, r_bsum;
  // NEXT-4 simulator scratch
  DevBuf s_res, s_flags, s_busy, s_psl, s_pe2e, s_pk;
  // NEXT-3 frontiers
  DevBuf f_nodefv, f_fvnode, f_act, f_next, f_budget, f_greq, f_gslo, f_gkeys, f_cnt, f_key, f_e2e, f_ctr;
  bool front_built = false;
  uint32_t front_kmax = 0, front_groups = 0, front_nfv = 0, front_cap = 0;
  // NEXT-1 ranked partitions
  DevBuf rank_off, rank_mask;
  // NEXT-1 DAG stages
  DevBuf dag_fu, dag_units, dag_xcut, dag_mt_off, dag_mt_mk, dag_mt_cand, dag_sv;
  bool dag_staged = false;
  bool ranked = false;
  uint32_t rank_kmax = 0, prof_order = 0;
  // scratch
  DevBuf prefix, block_sums, keys, req_dev, slo_dev, plans_dev, misses, v_tab, work_ctr;
  // cached occupancy per (ks, verify, smem)
  size_t occ_smem = 0;
  int occ[3][kMaxK + 1] = {};  // [task ranges | verify | bounded list kernel][KS]
  // per-segment timing of the last plan_keys call
  cudaEvent_t ev[kMaxK + 1] = {}, evs[kMaxK + 1] = {};  // per segment: end, start
  uint32_t seg_mask = 0;                                 // segments timed since the last k_first = 1
  // search mode (ffs_set_search_mode)
  uint32_t search_mode = FFS_SEARCH_BOUNDED;
  // bounded mode: group tables (per function x availability pattern) and live-record lists
  DevBuf gofs, grp, live_list, d_vtab;
  // exhaustive / verify KS = 4: requests grouped by chain length (launch_group_n)
  DevBuf g_perm, g_cnt, g_tab;
  bool grp_ok = false;
  uint32_t list_cap = 0;
  uint64_t list_cap_max = 1ull << 28;  // FFS_LIST_CAP (tests: force the task-range fallback)
  // ffs_plan_batch_host: copy streams (non-blocking) and the pipeline's events
  cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
  cudaEvent_t h_ev[2 * kHostSlices + 2] = {};
};

static ffs_status fail(ffs_ctx* c, ffs_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  if (c) c->err = buf;
  return s;
}

static ffs_status cuda_fail(ffs_ctx* c, cudaError_t e, const char* what) {
  return fail(c, FFS_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define CK(expr, what)                              \
  do {                                              \
    cudaError_t _e = (expr);                        \
    if (_e != cudaSuccess) return cuda_fail(c, _e, what); \
  } while (0)

static uint64_t binom64(int n, int r) {
  if (r < 0 || n < 0 || r > n) return 0;
  uint64_t v = 1;
  for (int i = 1; i <= r; ++i) v = v * (uint64_t)(n - r + i) / (uint64_t)i;
  return v;
}

extern "C" {

ffs_status ffs_create(int cuda_device, ffs_ctx** out) {
  if (!out) return FFS_ERR_ARG;
  *out = nullptr;
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess || cuda_device < 0 || cuda_device >= n) return FFS_ERR_CUDA;
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, cuda_device) != cudaSuccess) return FFS_ERR_CUDA;
  if (prop.major != 10 || prop.minor != 0) return FFS_ERR_CUDA;  // built for sm_100a only
  ffs_ctx* c = new ffs_ctx;
  c->device = cuda_device;
  c->sms = prop.multiProcessorCount;
  if (const char* e = std::getenv("FFS_LIST_CAP")) c->list_cap_max = std::strtoull(e, nullptr, 10);
  {
    DeviceGuard g(c->device);
    if (c->misses.ensure(8) != cudaSuccess || cudaMemset(c->misses.p, 0, 8) != cudaSuccess) {
      delete c;
      return FFS_ERR_CUDA;
    }
    for (auto& e : c->ev) cudaEventCreate(&e);
    for (auto& e : c->evs) cudaEventCreate(&e);
  }
  *out = c;
  return FFS_OK;
}

void ffs_destroy(ffs_ctx* c) {
  if (!c) return;
  {
    DeviceGuard g(c->device);
    for (auto& e : c->ev)
      if (e) cudaEventDestroy(e);
    for (auto& e : c->evs)
      if (e) cudaEventDestroy(e);
    for (auto& e : c->h_ev)
      if (e) cudaEventDestroy(e);
    if (c->s_h2d) cudaStreamDestroy(c->s_h2d);
    if (c->s_d2h) cudaStreamDestroy(c->s_d2h);
    for (DevBuf* b : {&c->s_res, &c->s_flags, &c->s_busy, &c->s_psl, &c->s_pe2e, &c->s_pk}) b->release();
    for (DevBuf* b : {&c->r_k, &c->r_k2, &c->r_v, &c->r_v2, &c->i_k, &c->i_k2, &c->i_v, &c->i_v2, &c->i_cum, &c->r_f,
                      &c->r_h, &c->r_n, &c->r_ts, &c->r_hist, &c->r_bsum})
      b->release();
    for (DevBuf* b : {&c->f_nodefv, &c->f_fvnode, &c->f_act, &c->f_next, &c->f_budget, &c->f_greq, &c->f_gslo,
                      &c->f_gkeys, &c->f_cnt, &c->f_key, &c->f_e2e, &c->f_ctr})
      b->release();
    for (DevBuf* b : {&c->node_off, &c->j_keys, &c->j_state, &c->j_dirty, &c->j_sreq, &c->j_sslo, &c->j_skeys,
                      &c->j_win, &c->j_busy, &c->j_cnt, &c->j_free, &c->j_ctr})
      b->release();
    for (DevBuf* b : {&c->dag_fu, &c->dag_units, &c->dag_xcut, &c->dag_mt_off, &c->dag_mt_mk, &c->dag_mt_cand, &c->dag_sv,
                      &c->rank_off, &c->rank_mask, &c->image, &c->node_free, &c->free_list, &c->slice_node, &c->slice_prof, &c->prefix,
                      &c->block_sums, &c->keys, &c->req_dev, &c->slo_dev, &c->plans_dev, &c->misses, &c->v_tab, &c->work_ctr,
                      &c->gofs, &c->grp, &c->live_list, &c->d_vtab, &c->g_perm, &c->g_cnt, &c->g_tab})
      b->release();
  }
  delete c;
}

const char* ffs_last_error(const ffs_ctx* c) { return c ? c->err.c_str() : "null context"; }

ffs_status ffs_stage_tables(ffs_ctx* c, const ffs_profiles* pr, const ffs_profile_table* tb, const ffs_cluster* cl) {
  if (!c) return FFS_ERR_ARG;
  c->staged = false;
  if (!pr || !tb || !cl) return fail(c, FFS_ERR_ARG, "null table pointer");
  if (pr->n_profiles != (uint32_t)kP)
    return fail(c, FFS_ERR_RANGE, "this build is compiled for P=%d profiles (got %u)", kP, pr->n_profiles);
  const uint32_t P = pr->n_profiles, F = tb->n_funcs;
  if (F == 0 || !tb->comp_off || !tb->lat_us || !tb->mem_mib || !tb->xfer_us || !tb->load_us)
    return fail(c, FFS_ERR_ARG, "empty or null profile table");
  uint32_t max_g = 0;
  for (uint32_t p = 0; p < P; ++p) {
    if (pr->gpcs[p] < 1 || pr->gpcs[p] > 7) return fail(c, FFS_ERR_ARG, "gpcs[%u]=%u not in 1..7", p, pr->gpcs[p]);
    max_g = std::max(max_g, pr->gpcs[p]);
  }
  if (tb->comp_off[0] != 0) return fail(c, FFS_ERR_ARG, "comp_off[0] != 0");
  uint32_t max_n = 0;
  std::vector<uint32_t> len(F);
  for (uint32_t f = 0; f < F; ++f) {
    if (tb->comp_off[f + 1] <= tb->comp_off[f]) return fail(c, FFS_ERR_ARG, "comp_off not strictly increasing at %u", f);
    len[f] = tb->comp_off[f + 1] - tb->comp_off[f];
    if (len[f] > (uint32_t)kMaxN) return fail(c, FFS_ERR_RANGE, "function %u has %u > 32 components", f, len[f]);
    max_n = std::max(max_n, len[f]);
  }
  const uint32_t C = tb->comp_off[F];
  // exact-encoding bounds (DESIGN.md §3 R4): sum_c max_p lat < 2^24, sum xfer < 2^24, sum mem < 2^31
  for (uint32_t f = 0; f < F; ++f) {
    uint64_t smax = 0, sx = 0, sm = 0;
    for (uint32_t i = tb->comp_off[f]; i < tb->comp_off[f + 1]; ++i) {
      uint32_t mx = 0;
      for (uint32_t p = 0; p < P; ++p) {
        const uint32_t l = tb->lat_us[(uint64_t)i * P + p];
        if (l == 0) return fail(c, FFS_ERR_ARG, "lat[%u][%u] = 0", i, p);
        mx = std::max(mx, l);
      }
      smax += mx;
      if (i + 1 < tb->comp_off[f + 1]) sx += tb->xfer_us[i];
      sm += tb->mem_mib[i];
    }
    if (smax >= (1u << 24)) return fail(c, FFS_ERR_RANGE, "function %u: sum of latencies >= 2^24 us", f);
    if (sx >= (1u << 24)) return fail(c, FFS_ERR_RANGE, "function %u: sum of transfer costs >= 2^24 us", f);
    if (sm >= (1ull << 31)) return fail(c, FFS_ERR_RANGE, "function %u: memory >= 2^31 MiB", f);
  }
  if (cl->n_nodes == 0 || cl->n_nodes >= (1u << 16)) return fail(c, FFS_ERR_RANGE, "n_nodes must be in 1..65535");
  if (cl->n_slices && !cl->slices) return fail(c, FFS_ERR_ARG, "null slices");
  for (uint32_t s = 0; s < cl->n_slices; ++s) {
    const ffs_slice& x = cl->slices[s];
    if (x.node >= cl->n_nodes) return fail(c, FFS_ERR_ARG, "slice %u: node %u >= n_nodes", s, x.node);
    if (x.profile >= P) return fail(c, FFS_ERR_ARG, "slice %u: profile %u >= P", s, x.profile);
    if (s) {
      const ffs_slice& y = cl->slices[s - 1];
      const uint64_t ky = ((uint64_t)y.node << 16) | ((uint64_t)y.gpu << 8) | y.slice;
      const uint64_t kx = ((uint64_t)x.node << 16) | ((uint64_t)x.gpu << 8) | x.slice;
      if (kx <= ky) return fail(c, FFS_ERR_ARG, "slices not sorted by (node, gpu, slice) at %u", s);
    }
  }

  // ---- build the table image (ImageLayout) ----
  ImageLayout L{};
  uint32_t w = 0;
  auto take = [&](uint32_t n, uint32_t align) {
    w = (w + align - 1) / align * align;
    uint32_t o = w;
    w += n;
    return o;
  };
  L.F = F;
  L.o_gpcs = take(8, 4);
  L.o_cap = take(8, 4);
  L.o_binom = take(33 * 8, 4);
  L.o_offk = take(33 * 10 * 2, 4);
  L.o_fdesc = take(4 * F, 4);
  const uint32_t rows = C + F;  // n_f + 1 boundaries per function
  L.o_pl = take(rows * kRowW, 4);
  L.o_pm = take(rows, 4);
  L.o_xf = take(rows, 4);
  L.o_thr = take(F, 4);
  L.o_tmm = take(2 * F, 4);
  L.words = (w + 3) / 4 * 4;
  std::vector<uint32_t> img(L.words, 0);
  for (uint32_t p = 0; p < 8; ++p) {
    img[L.o_gpcs + p] = p < P ? pr->gpcs[p] : 0;
    img[L.o_cap + p] = p < P ? pr->mem_mib[p] : 0;
  }
  for (int n = 0; n <= 32; ++n)
    for (int i = 0; i < 8; ++i) img[L.o_binom + n * 8 + i] = (uint32_t)binom64(n, i);
  for (int n = 1; n <= 32; ++n) {
    uint64_t acc = 0, pk = 1;
    for (int k = 1; k <= 9; ++k) {
      img[L.o_offk + 2 * (n * 10 + k)] = (uint32_t)acc;
      img[L.o_offk + 2 * (n * 10 + k) + 1] = (uint32_t)(acc >> 32);
      pk *= P;
      if (k <= 8) acc += binom64(n - 1, k - 1) * pk;
    }
  }
  uint32_t row = 0;
  for (uint32_t f = 0; f < F; ++f) {
    const uint32_t c0 = tb->comp_off[f], n = len[f];
    uint64_t mtot = 0;
    for (uint32_t i = 0; i < n; ++i) mtot += tb->mem_mib[c0 + i];
    img[L.o_fdesc + 4 * f + 0] = row;
    img[L.o_fdesc + 4 * f + 1] = n;
    img[L.o_fdesc + 4 * f + 2] = tb->load_us[f];
    img[L.o_fdesc + 4 * f + 3] = (uint32_t)mtot;
    const uint32_t fl = tb->max_stage_us ? tb->max_stage_us[f] : 0u;
    img[L.o_thr + f] = fl ? fl : 0xffffffffu;  // R38: 0 = no floor
    {  // KS = 4 f16 scale bounds, fp32 in chain order (as the kernel used to sum them)
      float tmin = 0.f, tmax = 0.f;
      for (uint32_t i = 0; i < n; ++i) {
        float lo = 0.f, hi = 0.f;
        for (uint32_t p = 0; p < P; ++p) {
          const float l = (float)tb->lat_us[(uint64_t)(c0 + i) * P + p];
          lo = p ? std::min(lo, l) : l;
          hi = p ? std::max(hi, l) : l;
        }
        tmin += lo;
        tmax += hi;
      }
      std::memcpy(&img[L.o_tmm + 2 * f], &tmin, 4);
      std::memcpy(&img[L.o_tmm + 2 * f + 1], &tmax, 4);
    }
    for (uint32_t p = 0; p < 8; ++p) img[L.o_pl + row * kRowW + p] = 0;
    img[L.o_pm + row] = 0;
    for (uint32_t i = 0; i < n; ++i) {
      for (uint32_t p = 0; p < 8; ++p)
        img[L.o_pl + (row + i + 1) * kRowW + p] =
            img[L.o_pl + (row + i) * kRowW + p] + (p < P ? tb->lat_us[(uint64_t)(c0 + i) * P + p] : 0);
      img[L.o_pm + row + i + 1] = img[L.o_pm + row + i] + tb->mem_mib[c0 + i];
      img[L.o_xf + row + i] = (i + 1 < n) ? tb->xfer_us[c0 + i] : 0;
    }
    row += n + 1;
  }

  // ---- per node: free counts (clamped to 8) and the first 8 free slices per profile ----
  const uint32_t NN = cl->n_nodes;
  std::vector<uint64_t> node_free(NN, 0);
  std::vector<int32_t> free_list((size_t)NN * 64, -1);
  std::vector<uint16_t> snode(std::max(1u, cl->n_slices));
  std::vector<uint8_t> sprof(std::max(1u, cl->n_slices));
  std::vector<uint8_t> cnt((size_t)NN * 8, 0);
  for (uint32_t s = 0; s < cl->n_slices; ++s) {
    const ffs_slice& x = cl->slices[s];
    snode[s] = x.node;
    sprof[s] = x.profile;
    if (x.busy) continue;
    uint8_t& k = cnt[(size_t)x.node * 8 + x.profile];
    if (k < 8) free_list[((size_t)x.node * 8 + x.profile) * 8 + k] = (int32_t)s;
    if (k < 255) ++k;
  }
  for (uint32_t v = 0; v < NN; ++v)
    for (uint32_t p = 0; p < 8; ++p)
      node_free[v] |= (uint64_t)std::min<uint32_t>(cnt[(size_t)v * 8 + p], 8) << (8 * p);
  std::vector<uint32_t> noff(NN + 1, 0);
  std::vector<uint8_t> hbusy(cl->n_slices);
  for (uint32_t s = 0; s < cl->n_slices; ++s) {
    noff[cl->slices[s].node + 1]++;
    hbusy[s] = cl->slices[s].busy ? 1 : 0;
  }
  for (uint32_t v = 0; v < NN; ++v) noff[v + 1] += noff[v];

  DeviceGuard g(c->device);
  CK(c->image.ensure((size_t)L.words * 4), "cudaMalloc(image)");
  {  // device copy: the prefix-latency rows as exact fp32 (every prefix < 2^24, checked above)
    std::vector<uint32_t> up(img);
    for (uint32_t i = L.o_pl; i < L.o_pl + rows * kRowW; ++i) {
      const float f = (float)img[i];
      std::memcpy(&up[i], &f, 4);
    }
    CK(cudaMemcpy(c->image.p, up.data(), (size_t)L.words * 4, cudaMemcpyHostToDevice), "upload image");
  }
  CK(c->node_free.ensure(NN * 8), "cudaMalloc(node_free)");
  CK(cudaMemcpy(c->node_free.p, node_free.data(), NN * 8, cudaMemcpyHostToDevice), "upload node_free");
  CK(c->free_list.ensure(free_list.size() * 4), "cudaMalloc(free_list)");
  CK(cudaMemcpy(c->free_list.p, free_list.data(), free_list.size() * 4, cudaMemcpyHostToDevice), "upload free_list");
  CK(c->slice_node.ensure(snode.size() * 2), "cudaMalloc(slice_node)");
  CK(cudaMemcpy(c->slice_node.p, snode.data(), snode.size() * 2, cudaMemcpyHostToDevice), "upload slice_node");
  CK(c->node_off.ensure(noff.size() * 4), "cudaMalloc(node_off)");
  CK(cudaMemcpy(c->node_off.p, noff.data(), noff.size() * 4, cudaMemcpyHostToDevice), "upload node_off");
  c->h_busy = hbusy;
  c->h_cnt = cnt;
  c->h_node_free = node_free;
  CK(c->slice_prof.ensure(sprof.size()), "cudaMalloc(slice_prof)");
  CK(cudaMemcpy(c->slice_prof.p, sprof.data(), sprof.size(), cudaMemcpyHostToDevice), "upload slice_prof");
  // bounded-mode group tables: 32 availability patterns per function,
  // built on the device from the image; skipped (task-range search only) above 1 GiB
  {
    std::vector<uint32_t> gofs(F);
    uint64_t tot = 0;
    for (uint32_t f = 0; f < F; ++f) {
      gofs[f] = (uint32_t)tot;
      tot += 32ull * grp_stride(len[f]);
    }
    c->grp_ok = tot * 4 <= (1ull << 30);
    if (c->grp_ok) {
      CK(c->gofs.ensure((size_t)F * 4), "cudaMalloc(gofs)");
      CK(cudaMemcpy(c->gofs.p, gofs.data(), (size_t)F * 4, cudaMemcpyHostToDevice), "upload gofs");
      CK(c->grp.ensure((size_t)tot * 4), "cudaMalloc(group tables)");
      CK(launch_group_tables(c->image.as<uint32_t>(), L, c->gofs.as<uint32_t>(), c->grp.as<uint32_t>(), 0),
         "group tables kernel");
      CK(cudaDeviceSynchronize(), "group tables");
    }
  }
  c->lay = L;
  c->h_image = img;
  c->ranked = false;
  c->dag_staged = false;
  c->front_built = false;
  c->P = P;
  c->F = F;
  c->n_nodes = NN;
  c->n_slices = cl->n_slices;
  c->max_n = max_n;
  c->max_gpcs = max_g;
  c->fn_len = len;
  c->staged = true;
  c->occ_smem = 0;
  return FFS_OK;
}

static ffs_status check_kmax(ffs_ctx* c, uint32_t k_max) {
  if (!c->staged) return fail(c, FFS_ERR_STATE, "tables not staged");
  if (k_max < 1 || k_max > (uint32_t)kMaxK) return fail(c, FFS_ERR_RANGE, "k_max %u not in 1..8", k_max);
  if (k_max * c->max_gpcs >= 64) return fail(c, FFS_ERR_RANGE, "k_max * max gpcs >= 64 (6-bit key field)");
  // S(n, K) < 2^41 for every staged function (idx field)
  uint64_t pk = 1, S = 0;
  for (uint32_t k = 1; k <= std::min(k_max, c->max_n); ++k) {
    pk *= c->P;
    S += binom64((int)c->max_n - 1, (int)k - 1) * pk;
  }
  if (S >= (1ull << kIdxBits)) return fail(c, FFS_ERR_RANGE, "S(n=%u, K=%u) >= 2^41", c->max_n, k_max);
  return FFS_OK;
}

static ffs_status search_keys(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req,
                              uint32_t k_max, uint32_t rank, uint32_t world, int64_t* d_keys, uint64_t* d_checks,
                              const uint64_t* node_free, void* stream, uint32_t k_first = 1, uint32_t k_last = 0);

ffs_status ffs_plan_keys(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req, uint32_t k_max,
                         uint32_t rank, uint32_t world, int64_t* d_keys, uint64_t* d_checks, void* stream) {
  if (!c) return FFS_ERR_ARG;
  return search_keys(c, d_req, d_slo, n_req, k_max, rank, world, d_keys, d_checks, nullptr, stream);
}

ffs_status ffs_plan_keys_range(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req,
                               uint32_t k_max, uint32_t k_first, uint32_t k_last, uint32_t rank, uint32_t world,
                               int64_t* d_keys, uint64_t* d_checks, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (k_first < 1 || k_first > k_last || k_last > k_max)
    return fail(c, FFS_ERR_RANGE, "segment range %u..%u not within 1..k_max=%u", k_first, k_last, k_max);
  return search_keys(c, d_req, d_slo, n_req, k_max, rank, world, d_keys, d_checks, nullptr, stream, k_first, k_last);
}

static ffs_status search_keys(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req,
                              uint32_t k_max, uint32_t rank, uint32_t world, int64_t* d_keys, uint64_t* d_checks,
                              const uint64_t* node_free, void* stream, uint32_t k_first, uint32_t k_last) {
  ffs_status s = check_kmax(c, k_max);
  if (s != FFS_OK) return s;
  if (k_last == 0) k_last = k_max;
  if (world == 0 || rank >= world) return fail(c, FFS_ERR_ARG, "rank %u / world %u", rank, world);
  if (n_req == 0) return FFS_OK;
  if (!d_req || !d_slo || !d_keys) return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  const uint64_t len = (uint64_t)n_req + 1;
  CK(c->prefix.ensure(len * k_max * 8), "cudaMalloc(prefix)");
  const uint64_t nb = (len + 2047) / 2048;
  CK(c->block_sums.ensure(nb * k_max * 8 + 8), "cudaMalloc(block_sums)");
  // keys and checksums are initialised by the first segment only; later ranges continue
  // from (and prune against) whatever the caller combined into d_keys in between
  const bool init = k_first == 1;
  CK(c->work_ctr.ensure(kCtrWords * 8), "cudaMalloc(work_ctr)");
  const uint64_t* nf = node_free ? node_free : c->node_free.as<uint64_t>();
  const bool exhaustive = c->search_mode == FFS_SEARCH_EXHAUSTIVE;
  // verify and exhaustive modes enumerate every request, including those whose node has
  // no free slice (R37); the task prefix is recomputed on every call (a continuation range
  // k_first > 1 therefore never sees a stale prefix, whatever the caller did to d_req)
  const bool skip_full = d_checks == nullptr && !exhaustive;
  nvtxRangePushA("ffs count+scan");
  CK(launch_count_tasks(d_req, c->image.as<uint32_t>(), c->lay, c->n_nodes, n_req, k_max, nf, skip_full,
                        c->prefix.as<uint64_t>(), c->block_sums.as<uint64_t>(), init ? d_keys : nullptr,
                        init ? reinterpret_cast<unsigned long long*>(d_checks) : nullptr,
                        c->work_ctr.as<unsigned long long>(), k_first, k_last, st),
     "count/scan kernels");
  nvtxRangePop();
  // dynamic shared memory: the table image (every KS) + the per-thread variant windows
  // of the KS = 4 kernel (kWin4 B per thread).  The f16x2 kernel's window stride is the
  // compile-time CTA size (immediate LDS/STS offsets); an image that does not fit next to
  // its windows is read from global memory instead (tables_global).
  const size_t min_win = kWin4 * search_block(4);
  const bool tables_global = (size_t)c->lay.words * 4 + min_win > kMaxSmem;
  const size_t smem = tables_global ? 0 : (size_t)c->lay.words * 4;
  const int block4 = search_block(4);
  // kernel variants: v = 0 task ranges, 1 verify, 2 the bounded mode's list kernel (KS = 2..4)
  auto blk = [&](int k, int v) { return k == 4 ? block4 : search_block(k, v == 2); };
  auto shm = [&](int k) { return smem + (k == 4 ? kWin4 * block4 : 0); };
  if (c->occ_smem != smem + 1) {  // (smem = 0 <=> tables in global memory)
    for (int v = 0; v < 3; ++v)
      for (int k = 1; k <= kMaxK; ++k) {
        if (v == 2 && (k < 2 || k > 4)) continue;
        int b = 0;
        CK(search_kernel_config(k, v == 1, v == 2, tables_global, blk(k, v), shm(k), &b), "search kernel occupancy");
        c->occ[v][k] = std::max(1, b);
      }
    c->occ_smem = smem + 1;
  }
  SearchArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.req = d_req;
  a.slo = d_slo;
  a.node_free = node_free ? node_free : c->node_free.as<uint64_t>();
  a.prefix = c->prefix.as<uint64_t>();
  a.n_req = n_req;
  a.rank = rank;
  a.world = world;
  a.keys = d_keys;
  a.checks = reinterpret_cast<unsigned long long*>(d_checks);
  a.misses = c->misses.as<unsigned long long>();
  a.tables_global = tables_global ? 1u : 0u;
  a.work_ctr = c->work_ctr.as<unsigned long long>();
  a.exhaustive = exhaustive ? 1u : 0u;
  const bool verify = d_checks != nullptr;
  const uint32_t kk = std::min(k_last, c->max_n);
  // bounded mode, KS = 2..4: live-mask compaction (k_live) before the search, which then
  // walks the compacted records.  The list holds up to list_cap records;
  // a segment with more live records falls back to the task ranges inside the search
  // kernel (same result), so the capacity only bounds memory, never correctness.
  const bool use_live = !verify && !exhaustive && c->grp_ok;
  LiveArgs la{};
  if (use_live) {
    const uint64_t want = std::min<uint64_t>(16ull * n_req + (1ull << 20), c->list_cap_max);
    if (c->list_cap != want) {  // one list per segment KS = 2..4
      CK(c->live_list.ensure(std::max<uint64_t>(want, 1) * 16 * 3), "cudaMalloc(live lists)");
      c->list_cap = (uint32_t)want;
    }
    la.image = c->image.as<uint32_t>();
    la.lay = c->lay;
    la.req = d_req;
    la.slo = d_slo;
    la.node_free = a.node_free;
    la.prefix = a.prefix;
    la.n_req = n_req;
    la.rank = rank;
    la.world = world;
    la.keys = d_keys;
    la.gofs = c->gofs.as<uint32_t>();
    la.grp = c->grp.as<uint32_t>();
    for (int j = 0; j < 3; ++j) la.list[j] = c->live_list.as<uint4>() + (size_t)j * c->list_cap;
    la.list_cap = c->list_cap;
    la.work_ctr = a.work_ctr;
  }
  if (init) c->seg_mask = 0;
  bool grouped = false;
  for (uint32_t k = k_first; k <= kk; ++k) {
    const bool list = use_live && k >= 2 && k <= 4;
    const int var = verify ? 1 : list ? 2 : 0;
    const int grid = c->sms * c->occ[var][k];
    static const char* kSegName[kMaxK + 1] = {"", "ffs search KS=1", "ffs search KS=2", "ffs search KS=3",
                                              "ffs search KS=4", "ffs search KS=5", "ffs search KS=6",
                                              "ffs search KS=7", "ffs search KS=8"};
    nvtxRangePushA(kSegName[k]);
    CK(cudaEventRecord(c->evs[k], st), "event");
    a.list = nullptr;
    a.list_cap = 0;
    a.g_perm = nullptr;
    a.g_tab = nullptr;
    // KS = 2 walks the groups only on large batches: a request's n - 1 masks form one unit,
    // and a request shard has too few of them (1/8 of C5: 0.09 ms on the task ranges, 0.18
    // grouped); at full C5 0.48 -> 0.34 ms
    const bool grp_k = k == 3 || k == 4 || (k == 2 && n_req >= (1u << 19));
    if (grp_k && !list && (verify || exhaustive)) {
      // lanes of a warp = 32 requests of equal chain length walking the same masks; the
      // grouping is built once per call, before the first grouped segment
      if (!grouped) {
        const uint64_t glen = 34ull * ((n_req + 2047) / 2048) + 1;
        CK(c->g_perm.ensure((size_t)n_req * 4), "cudaMalloc(group perm)");
        CK(c->g_cnt.ensure(glen * 8 + (glen / 2048 + 2) * 8), "cudaMalloc(group offsets)");
        CK(c->g_tab.ensure(136 * 4), "cudaMalloc(group table)");
        CK(launch_group_n(d_req, c->image.as<uint32_t>(), c->lay, c->n_nodes, n_req, grp_unit3(n_req),
                          c->g_cnt.as<uint64_t>(),
                          c->g_cnt.as<uint64_t>() + glen, c->g_tab.as<uint32_t>(), c->g_perm.as<uint32_t>(), st),
           "group kernels");
        grouped = true;
      }
      a.g_perm = c->g_perm.as<uint32_t>();
      a.g_tab = c->g_tab.as<uint32_t>();
      a.g_s3 = grp_unit3(n_req);
    }
    if (list) {
      // compaction right before the segment: the keys of all earlier segments drop the
      // requests already settled with cvq = 0 (a 2- or 3-stage winner with CV^2 < 1/1024
      // is common; one pass for KS = 2..4 after KS = 1 measured 6x the records at KS = 4)
      la.ks = k;
      // requests per warp grab: 32 (one header per lane, loaded in parallel) for the light
      // KS = 2 pass; fewer for the heavy segments, whose per-request mask work would
      // otherwise leave the last grabs of a small batch (a request shard) on a few warps
      const uint64_t warps = (uint64_t)c->sms * 8 * 8, div = k == 2 ? 1 : k == 3 ? 4 : 16;
      la.per_grab = k == 2 ? 32u : (uint32_t)std::min<uint64_t>(32, std::max<uint64_t>(1, n_req / (warps * div)));
      CK(launch_live(la, c->sms * 8, st), "live-mask kernel");
      a.list = la.list[k - 2];
      a.list_cap = c->list_cap;
    }
    CK(launch_search((int)k, verify, list, a, grid, blk((int)k, var), shm((int)k), st), "search kernel");
    CK(cudaEventRecord(c->ev[k], st), "event");
    nvtxRangePop();
    c->seg_mask |= 1u << k;
  }
  return FFS_OK;
}

ffs_status ffs_plan_decode(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, const int64_t* d_keys,
                           uint32_t n_req, uint32_t k_max, const ffs_instance* d_inst, const int64_t* d_scores,
                           uint32_t n_inst, ffs_plan* d_out, void* stream) {
  if (!c) return FFS_ERR_ARG;
  ffs_status s = check_kmax(c, k_max);
  if (s != FFS_OK) return s;
  if (n_req == 0) return FFS_OK;
  if (!d_req || !d_slo || !d_keys || !d_out) return fail(c, FFS_ERR_ARG, "null device pointer");
  if ((d_inst == nullptr) != (d_scores == nullptr)) return fail(c, FFS_ERR_ARG, "d_inst and d_evict_scores must both be set");
  if (d_inst && n_inst > (1u << 20)) return fail(c, FFS_ERR_RANGE, "n_inst %u > 2^20", n_inst);
  DeviceGuard g(c->device);
  DecodeArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.req = d_req;
  a.slo = d_slo;
  a.keys = d_keys;
  a.n_req = n_req;
  a.k_max = k_max;
  a.n_nodes = c->n_nodes;
  a.n_slices = c->n_slices;
  a.free_list = c->free_list.as<int32_t>();
  a.slice_node = c->slice_node.as<uint16_t>();
  a.slice_prof = c->slice_prof.as<uint8_t>();
  a.inst = d_inst;
  a.score = d_scores;
  a.n_inst = d_inst ? n_inst : 0;
  a.out = d_out;
  if (d_inst) CK(c->d_vtab.ensure((size_t)c->n_nodes * c->P * 8), "cudaMalloc(decode victim table)");
  CK(launch_decode(a, c->d_vtab.as<unsigned long long>(), (cudaStream_t)stream), "decode kernel");
  return FFS_OK;
}

ffs_status ffs_plan_batch(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req, uint32_t k_max,
                          ffs_plan* d_out, void* stream) {
  if (!c) return FFS_ERR_ARG;
  {
    DeviceGuard g(c->device);
    CK(c->keys.ensure((size_t)std::max(1u, n_req) * 8), "cudaMalloc(keys)");
  }
  ffs_status s = ffs_plan_keys(c, d_req, d_slo, n_req, k_max, 0, 1, c->keys.as<int64_t>(), nullptr, stream);
  if (s != FFS_OK) return s;
  return ffs_plan_decode(c, d_req, d_slo, c->keys.as<int64_t>(), n_req, k_max, nullptr, nullptr, 0, d_out, stream);
}

ffs_status ffs_plan_batch_host(ffs_ctx* c, const ffs_request* h_req, const uint32_t* h_slo, uint32_t n_req,
                               uint32_t k_max, ffs_plan* h_out, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (n_req == 0) return FFS_OK;
  if (!h_req || !h_slo || !h_out) return fail(c, FFS_ERR_ARG, "null host pointer");
  cudaStream_t st = (cudaStream_t)stream;
  // Large batches are planned in kHostSlices request slices (requests are independent,
  // R13: a slice plans exactly as within the batch): the upload of slice i+1 and the
  // download of the plans of slice i-1 run on two copy streams while slice i is planned on
  // `stream`, so only the first upload and the last download are exposed.  Each slice pays
  // the per-call fixed costs once more, so the slices stay few and large.
  const uint32_t nch = n_req >= (1u << 20) ? kHostSlices : 1u;
  {
    DeviceGuard g(c->device);
    CK(c->req_dev.ensure((size_t)n_req * sizeof(ffs_request)), "cudaMalloc(req)");
    CK(c->slo_dev.ensure((size_t)n_req * 4), "cudaMalloc(slo)");
    CK(c->plans_dev.ensure((size_t)n_req * sizeof(ffs_plan)), "cudaMalloc(plans)");
    if (!c->s_h2d) CK(cudaStreamCreateWithFlags(&c->s_h2d, cudaStreamNonBlocking), "copy stream");
    if (!c->s_d2h) CK(cudaStreamCreateWithFlags(&c->s_d2h, cudaStreamNonBlocking), "copy stream");
    for (auto& e : c->h_ev)
      if (!e) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event");
    // the copies start after the work already queued on `stream` (its buffers may be in use)
    CK(cudaEventRecord(c->h_ev[2 * kHostSlices], st), "event");
    CK(cudaStreamWaitEvent(c->s_h2d, c->h_ev[2 * kHostSlices], 0), "wait");
    CK(cudaStreamWaitEvent(c->s_d2h, c->h_ev[2 * kHostSlices], 0), "wait");
    for (uint32_t i = 0; i < nch; ++i) {
      const size_t lo = (size_t)n_req * i / nch, hi = (size_t)n_req * (i + 1) / nch;
      CK(cudaMemcpyAsync(c->req_dev.as<ffs_request>() + lo, h_req + lo, (hi - lo) * sizeof(ffs_request),
                         cudaMemcpyHostToDevice, c->s_h2d), "H2D req");
      CK(cudaMemcpyAsync(c->slo_dev.as<uint32_t>() + lo, h_slo + lo, (hi - lo) * 4, cudaMemcpyHostToDevice, c->s_h2d),
         "H2D slo");
      CK(cudaEventRecord(c->h_ev[i], c->s_h2d), "event");
    }
  }
  for (uint32_t i = 0; i < nch; ++i) {
    const size_t lo = (size_t)n_req * i / nch, hi = (size_t)n_req * (i + 1) / nch;
    {
      DeviceGuard g(c->device);
      CK(cudaStreamWaitEvent(st, c->h_ev[i], 0), "wait");
    }
    ffs_status s = ffs_plan_batch(c, c->req_dev.as<ffs_request>() + lo, c->slo_dev.as<uint32_t>() + lo,
                                  (uint32_t)(hi - lo), k_max, c->plans_dev.as<ffs_plan>() + lo, stream);
    if (s != FFS_OK) return s;
    DeviceGuard g(c->device);
    CK(cudaEventRecord(c->h_ev[kHostSlices + i], st), "event");
    CK(cudaStreamWaitEvent(c->s_d2h, c->h_ev[kHostSlices + i], 0), "wait");
    CK(cudaMemcpyAsync(h_out + lo, c->plans_dev.as<ffs_plan>() + lo, (hi - lo) * sizeof(ffs_plan),
                       cudaMemcpyDeviceToHost, c->s_d2h), "D2H plans");
  }
  DeviceGuard g(c->device);
  CK(cudaEventRecord(c->h_ev[2 * kHostSlices + 1], c->s_d2h), "event");
  CK(cudaStreamWaitEvent(st, c->h_ev[2 * kHostSlices + 1], 0), "wait");
  CK(cudaStreamSynchronize(st), "stream sync");
  return FFS_OK;
}

ffs_status ffs_evict_scores(ffs_ctx* c, const ffs_instance* d_inst, uint32_t n_inst, uint64_t now_us,
                            const ffs_evict_params* prm, int64_t* d_score, uint8_t* d_state, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!prm) return fail(c, FFS_ERR_ARG, "null params");
  if (n_inst > (1u << 20)) return fail(c, FFS_ERR_RANGE, "n_inst %u > 2^20", n_inst);
  if (prm->cold_after_us >= (1ull << 43)) return fail(c, FFS_ERR_RANGE, "cold_after_us >= 2^43");
  if (n_inst == 0) return FFS_OK;
  if (!d_inst || !d_score || !d_state) return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  CK(launch_evict(d_inst, n_inst, nullptr, nullptr, 0, now_us, *prm, d_score, d_state, (cudaStream_t)stream),
     "evict kernel");
  return FFS_OK;
}

ffs_status ffs_evict_scores_ticks(ffs_ctx* c, const ffs_instance* d_inst, const uint32_t* d_tick_off,
                                  const uint64_t* d_now_us, uint32_t n_ticks, const ffs_evict_params* prm,
                                  int64_t* d_score, uint8_t* d_state, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!prm) return fail(c, FFS_ERR_ARG, "null params");
  if (prm->cold_after_us >= (1ull << 43)) return fail(c, FFS_ERR_RANGE, "cold_after_us >= 2^43");
  if (n_ticks == 0) return FFS_OK;
  if (!d_inst || !d_tick_off || !d_now_us || !d_score || !d_state) return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  CK(launch_evict(d_inst, 0, d_tick_off, d_now_us, n_ticks, 0, *prm, d_score, d_state, (cudaStream_t)stream),
     "evict kernel");
  return FFS_OK;
}

ffs_status ffs_evict_step(ffs_ctx* c, const ffs_instance* d_inst, const uint32_t* d_tick_off, const uint64_t* d_now_us,
                          uint32_t n_ticks, const ffs_evict_params* prm, int64_t* d_score, uint8_t* d_state,
                          const ffs_request* d_req, const uint32_t* d_slo, const uint32_t* d_req_tick,
                          const uint32_t* d_load_off, uint32_t n_req, int32_t* d_victim, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged) return fail(c, FFS_ERR_STATE, "tables not staged");
  if (!prm) return fail(c, FFS_ERR_ARG, "null params");
  if (prm->cold_after_us >= (1ull << 43)) return fail(c, FFS_ERR_RANGE, "cold_after_us >= 2^43");
  if (n_ticks == 0 && n_req == 0) return FFS_OK;
  if (!d_inst || !d_tick_off || !d_now_us || !d_score || !d_state) return fail(c, FFS_ERR_ARG, "null device pointer");
  if (n_req && (!d_req || !d_slo || (!d_req_tick && !d_load_off) || !d_victim))
    return fail(c, FFS_ERR_ARG, "null device pointer");
  const uint64_t tab_bytes = (uint64_t)n_ticks * c->n_nodes * c->P * 8;
  // the fused pass needs the tick's (node, profile) minima in shared memory and the whole
  // table in device memory; otherwise: the two calls it fuses
  const bool grouped = d_load_off != nullptr && n_req > 0;
  if (c->n_nodes * c->P * 8 > 160 * 1024 || (!grouped && tab_bytes > (256ull << 20))) {
    if (!d_req_tick && n_req) return fail(c, FFS_ERR_ARG, "d_req_tick needed for this cluster size");
    ffs_status s = ffs_evict_scores_ticks(c, d_inst, d_tick_off, d_now_us, n_ticks, prm, d_score, d_state, stream);
    if (s != FFS_OK || n_req == 0) return s;
    return ffs_evict_victims(c, d_req, d_slo, d_req_tick, n_req, d_inst, d_tick_off, d_score, n_ticks, d_victim,
                             stream);
  }
  DeviceGuard g(c->device);
  if (!grouped) CK(c->v_tab.ensure(std::max<uint64_t>(tab_bytes, 8)), "cudaMalloc(victim table)");
  CK(launch_evict_step(c->image.as<uint32_t>(), c->lay, d_inst, d_tick_off, d_now_us, n_ticks, *prm, d_score, d_state,
                       c->slice_node.as<uint16_t>(), c->slice_prof.as<uint8_t>(), c->n_slices, c->n_nodes,
                       c->v_tab.as<unsigned long long>(), d_req, d_slo, d_req_tick, grouped ? d_load_off : nullptr,
                       n_req, d_victim, (cudaStream_t)stream),
     "evict step kernels");
  return FFS_OK;
}

ffs_status ffs_evict_victims(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, const uint32_t* d_req_tick,
                             uint32_t n_req, const ffs_instance* d_inst, const uint32_t* d_tick_off,
                             const int64_t* d_score, uint32_t n_ticks, int32_t* d_victim, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged) return fail(c, FFS_ERR_STATE, "tables not staged");
  if (n_req == 0) return FFS_OK;
  if (!d_req || !d_slo || !d_req_tick || !d_inst || !d_tick_off || !d_score || !d_victim)
    return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  // per-(tick, node, profile) minimum table when it stays small, else the warp scan
  const uint64_t tab_bytes = (uint64_t)n_ticks * c->n_nodes * c->P * 8;
  unsigned long long* tab = nullptr;
  if (tab_bytes > 0 && tab_bytes <= (256ull << 20) && c->v_tab.ensure(tab_bytes) == cudaSuccess)
    tab = c->v_tab.as<unsigned long long>();
  CK(launch_victims(c->image.as<uint32_t>(), c->lay, d_req, d_slo, d_req_tick, n_req, d_inst, d_tick_off, d_score,
                    n_ticks, c->slice_node.as<uint16_t>(), c->slice_prof.as<uint8_t>(), c->n_slices, c->n_nodes, tab,
                    d_victim, (cudaStream_t)stream),
     "victims kernel");
  return FFS_OK;
}

ffs_status ffs_rank_partitions(ffs_ctx* c, uint32_t k_max, uint32_t p_ref) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged) return fail(c, FFS_ERR_STATE, "tables not staged");
  if (k_max < 1 || k_max > (uint32_t)kMaxK) return fail(c, FFS_ERR_RANGE, "k_max %u not in 1..8", k_max);
  if (p_ref >= c->P) return fail(c, FFS_ERR_RANGE, "p_ref %u >= P", p_ref);
  const ImageLayout& L = c->lay;
  const std::vector<uint32_t>& img = c->h_image;
  uint64_t total = 0;
  for (uint32_t f = 0; f < c->F; ++f)
    for (uint32_t k = 1; k <= std::min(k_max, c->fn_len[f]); ++k) total += binom64((int)c->fn_len[f] - 1, (int)k - 1);
  if (total >= (1ull << 24)) return fail(c, FFS_ERR_RANGE, "%llu ranked partitions > 2^24", (unsigned long long)total);
  std::vector<uint32_t> off(c->F + 1, 0), masks;
  masks.reserve((size_t)total);
  struct E { uint64_t cvq; uint32_t k, mask; };
  for (uint32_t f = 0; f < c->F; ++f) {
    const uint32_t row0 = img[L.o_fdesc + 4 * f], n = img[L.o_fdesc + 4 * f + 1];
    std::vector<E> es;
    for (uint32_t k = 1; k <= std::min(k_max, n); ++k) {
      // every (k-1)-subset of the n-1 cut positions in ascending numeric order (Gosper)
      if (k == 1) {
        es.push_back({0, 1, 0});
        continue;
      }
      const uint32_t lim = 1u << (n - 1);
      for (uint32_t m = (1u << (k - 1)) - 1; m < lim;) {
        uint64_t s = 0, sq = 0;
        uint32_t a = 0, mm = m;
        for (uint32_t i = 0; i < k; ++i) {
          uint32_t b = n;
          if (i + 1 < k) {
            b = (uint32_t)__builtin_ctz(mm) + 1;
            mm &= mm - 1;
          }
          const uint64_t t = (uint64_t)img[L.o_pl + (row0 + b) * kRowW + p_ref] - img[L.o_pl + (row0 + a) * kRowW + p_ref];
          s += t;
          sq += t * t;
          a = b;
        }
        const uint64_t D = s * s, N = (uint64_t)k * sq - D;  // exact under the R4 bounds
        es.push_back({(N << 10) / D, k, m});
        const uint32_t t = m | (m - 1);
        const uint32_t nm = (uint32_t)((uint64_t)t + 1) | (uint32_t)((((~t & (0u - ~t)) - 1)) >> (__builtin_ctz(m) + 1));
        if (nm <= m) break;
        m = nm;
      }
    }
    std::stable_sort(es.begin(), es.end(), [](const E& x, const E& y) {
      if (x.cvq != y.cvq) return x.cvq < y.cvq;
      if (x.k != y.k) return x.k < y.k;
      return x.mask < y.mask;
    });
    for (const E& e : es) masks.push_back(e.mask);
    off[f + 1] = (uint32_t)masks.size();
  }
  // profiles ordered by (capacity, gpcs, id) for the min-resource assignment
  std::vector<uint32_t> ord(c->P);
  for (uint32_t p = 0; p < c->P; ++p) ord[p] = p;
  std::sort(ord.begin(), ord.end(), [&](uint32_t x, uint32_t y) {
    const uint32_t cx = img[L.o_cap + x], cy = img[L.o_cap + y], gx = img[L.o_gpcs + x], gy = img[L.o_gpcs + y];
    if (cx != cy) return cx < cy;
    if (gx != gy) return gx < gy;
    return x < y;
  });
  uint32_t po = 0;
  for (uint32_t i = 0; i < c->P; ++i) po |= ord[i] << (4 * i);
  DeviceGuard g(c->device);
  CK(c->rank_off.ensure(off.size() * 4), "cudaMalloc(rank_off)");
  CK(cudaMemcpy(c->rank_off.p, off.data(), off.size() * 4, cudaMemcpyHostToDevice), "upload rank_off");
  CK(c->rank_mask.ensure(std::max<size_t>(1, masks.size()) * 4), "cudaMalloc(rank_mask)");
  if (!masks.empty())
    CK(cudaMemcpy(c->rank_mask.p, masks.data(), masks.size() * 4, cudaMemcpyHostToDevice), "upload rank_mask");
  c->prof_order = po;
  c->rank_kmax = k_max;
  c->ranked = true;
  return FFS_OK;
}

ffs_status ffs_plan_ranked(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req,
                           ffs_plan* d_out, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged || !c->ranked) return fail(c, FFS_ERR_STATE, "call ffs_rank_partitions after staging");
  if (n_req == 0) return FFS_OK;
  if (!d_req || !d_slo || !d_out) return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  RankedArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.req = d_req;
  a.slo = d_slo;
  a.n_req = n_req;
  a.n_nodes = c->n_nodes;
  a.node_free = c->node_free.as<uint64_t>();
  a.free_list = c->free_list.as<int32_t>();
  a.rank_off = c->rank_off.as<uint32_t>();
  a.rank_mask = c->rank_mask.as<uint32_t>();
  a.prof_order = c->prof_order;
  a.out = d_out;
  CK(launch_ranked(a, (cudaStream_t)stream), "ranked kernel");
  return FFS_OK;
}

// ---- NEXT-1 DAG stages (R40-R43) ------------------------------------
ffs_status ffs_dag_stage(ffs_ctx* c, const ffs_dag_table* d, uint32_t k_max) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged) return fail(c, FFS_ERR_STATE, "tables not staged");
  c->dag_staged = false;
  if (!d || !d->unit_off || !d->unit_nb || !d->unit_bend) return fail(c, FFS_ERR_ARG, "null DAG table pointer");
  if (d->n_funcs != c->F) return fail(c, FFS_ERR_ARG, "DAG n_funcs %u != staged %u", d->n_funcs, c->F);
  if (k_max < 1 || k_max > (uint32_t)kMaxK) return fail(c, FFS_ERR_RANGE, "k_max %u not in 1..8", k_max);
  if (d->unit_off[0] != 0) return fail(c, FFS_ERR_ARG, "unit_off[0] != 0");
  const ImageLayout& L = c->lay;
  const std::vector<uint32_t>& img = c->h_image;
  const uint32_t F = c->F, U = d->unit_off[F];
  std::vector<uint32_t> fu(2 * (size_t)F), units(6 * (size_t)std::max(U, 1u), 0), xcut(std::max(U, 1u), 0);
  // per function m + 1 rows of 8: prefix over its units of the conditional units'
  // one-slice saving (sum of the alternatives' times - the slowest), R48
  std::vector<uint32_t> sv(8 * ((size_t)U + F), 0);
  auto plat = [&](uint32_t row, uint32_t p) { return img[L.o_pl + row * kRowW + p]; };  // host copy: integers
  uint32_t maxnb = 1;
  for (uint32_t f = 0; f < F; ++f) {
    if (d->unit_off[f + 1] < d->unit_off[f]) return fail(c, FFS_ERR_ARG, "unit_off decreasing at %u", f);
    const uint32_t m = d->unit_off[f + 1] - d->unit_off[f];
    if (m < 1) return fail(c, FFS_ERR_ARG, "function %u has no units", f);
    if (m > FFS_DAG_MAX_UNITS) return fail(c, FFS_ERR_RANGE, "function %u has %u > 16 units", f, m);
    const uint32_t row0 = img[L.o_fdesc + 4 * f], n = img[L.o_fdesc + 4 * f + 1];
    fu[2 * f] = d->unit_off[f];
    fu[2 * f + 1] = m;
    uint32_t cc = 0;
    uint32_t* svf = sv.data() + 8 * ((size_t)d->unit_off[f] + f);
    for (uint32_t u = d->unit_off[f]; u < d->unit_off[f + 1]; ++u) {
      const uint32_t nb = d->unit_nb[u];
      const bool cond = d->unit_cond && d->unit_cond[u];
      if (nb < 1 || nb > FFS_DAG_MAX_BRANCHES) return fail(c, FFS_ERR_ARG, "unit %u: %u branches not in 1..4", u, nb);
      if (cond && nb < 2) return fail(c, FFS_ERR_ARG, "conditional unit %u: %u alternatives", u, nb);
      if (!cond) maxnb = std::max(maxnb, nb);  // alternatives never split (R48)
      units[6 * (size_t)u] = nb | (cond ? 1u << 8 : 0u);
      units[6 * (size_t)u + 1] = cc;
      const uint32_t start = cc;
      uint32_t x = 0, tsum[kP] = {0, 0, 0, 0, 0}, tmax[kP] = {0, 0, 0, 0, 0};
      for (uint32_t j = 0; j < nb; ++j) {
        const uint32_t e = d->unit_bend[4 * (size_t)u + j];
        if ((cond ? e < cc : e <= cc) || e > n)
          return fail(c, FFS_ERR_ARG, "unit %u branch %u: end %u not in (%u, %u]", u, j, e, cc, n);
        units[6 * (size_t)u + 2 + j] = e;
        // R42: every branch output moves at a cut; R48: the alternative that ran (worst
        // case), an empty one passing the previous component's output
        const uint32_t xb = e > cc ? img[L.o_xf + row0 + e - 1] : (start > 0 ? img[L.o_xf + row0 + start - 1] : 0u);
        x = cond ? std::max(x, xb) : x + xb;
        for (uint32_t p = 0; p < (uint32_t)kP; ++p) {
          const uint32_t tb = plat(row0 + e, p) - plat(row0 + cc, p);
          tsum[p] += tb;
          tmax[p] = std::max(tmax[p], tb);
        }
        cc = e;
      }
      if (cc == start) return fail(c, FFS_ERR_ARG, "unit %u has no components", u);
      if (nb == 1 && cc != start + 1) return fail(c, FFS_ERR_ARG, "unit %u: one branch of %u components", u, cc - start);
      xcut[u] = x;
      const uint32_t lu = u - d->unit_off[f];
      for (uint32_t p = 0; p < 8; ++p)
        svf[8 * (lu + 1) + p] = svf[8 * lu + p] + (cond && p < (uint32_t)kP ? tsum[p] - tmax[p] : 0u);
    }
    if (cc != n) return fail(c, FFS_ERR_ARG, "function %u: units cover %u of %u components", f, cc, n);
  }
  if (k_max * maxnb > FFS_DAG_MAX_SLOTS)
    return fail(c, FFS_ERR_RANGE, "k_max %u x %u branches > %d slices per plan", k_max, maxnb, FFS_DAG_MAX_SLOTS);
  if (k_max * maxnb * c->max_gpcs >= 64) return fail(c, FFS_ERR_RANGE, "k_max x branches x max gpcs >= 64");
  // per function: unit-cut masks in candidate order (k ascending, masks ascending) with
  // the first candidate index of each (R43)
  std::vector<uint32_t> mt_off(F + 1, 0), mt_mk;
  std::vector<unsigned long long> mt_cand;
  for (uint32_t f = 0; f < F; ++f) {
    const uint32_t m = fu[2 * f + 1], ub = fu[2 * f];
    uint64_t cand = 0;
    for (uint32_t k = 1; k <= std::min(k_max, m); ++k)
      for (uint32_t mask = 0; mask < (1u << (m - 1)); ++mask) {
        if ((uint32_t)__builtin_popcount(mask) != k - 1) continue;
        mt_mk.push_back(mask | (k << 16));
        mt_cand.push_back(cand);
        uint64_t tot = 1;
        uint32_t u0 = 0;
        for (uint32_t u = 0; u < m; ++u)
          if (u + 1 == m || ((mask >> u) & 1u)) {
            const uint32_t nb = units[6 * (size_t)(ub + u0)] & 0xffu;
            const bool cond = (units[6 * (size_t)(ub + u0)] >> 8) != 0;
            uint64_t q = kP;
            if (u0 == u && nb >= 2 && !cond) {
              uint64_t pw = 1;
              for (uint32_t j = 0; j < nb; ++j) pw *= kP;
              q += pw;
            }
            tot *= q;
            u0 = u + 1;
          }
        cand += tot;
        if (cand >= (1ull << kIdxBits)) return fail(c, FFS_ERR_RANGE, "function %u: >= 2^41 DAG candidates", f);
      }
    mt_off[f + 1] = (uint32_t)mt_mk.size();
  }
  DeviceGuard g(c->device);
  auto up = [&](DevBuf& b, const void* src, size_t bytes) -> cudaError_t {
    cudaError_t e = b.ensure(std::max<size_t>(bytes, 8));
    if (e != cudaSuccess || bytes == 0) return e;
    return cudaMemcpy(b.p, src, bytes, cudaMemcpyHostToDevice);
  };
  CK(up(c->dag_fu, fu.data(), fu.size() * 4), "upload dag_fu");
  CK(up(c->dag_units, units.data(), units.size() * 4), "upload dag_units");
  CK(up(c->dag_xcut, xcut.data(), xcut.size() * 4), "upload dag_xcut");
  CK(up(c->dag_sv, sv.data(), sv.size() * 4), "upload dag_sv");
  CK(up(c->dag_mt_off, mt_off.data(), mt_off.size() * 4), "upload dag_mt_off");
  CK(up(c->dag_mt_mk, mt_mk.data(), mt_mk.size() * 4), "upload dag_mt_mk");
  CK(up(c->dag_mt_cand, mt_cand.data(), mt_cand.size() * 8), "upload dag_mt_cand");
  c->dag_staged = true;
  return FFS_OK;
}

ffs_status ffs_plan_dag(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req,
                        ffs_dag_plan* d_out, uint64_t* d_checksums, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged || !c->dag_staged) return fail(c, FFS_ERR_STATE, "call ffs_dag_stage after staging");
  if (n_req == 0) return FFS_OK;
  if (!d_req || !d_slo || !d_out) return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  DagArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.req = d_req;
  a.slo = d_slo;
  a.n_req = n_req;
  a.n_nodes = c->n_nodes;
  a.node_free = c->node_free.as<uint64_t>();
  a.free_list = c->free_list.as<int32_t>();
  a.fu = c->dag_fu.as<uint32_t>();
  a.units = c->dag_units.as<uint32_t>();
  a.xcut = c->dag_xcut.as<uint32_t>();
  a.sv = c->dag_sv.as<uint32_t>();
  a.mt_off = c->dag_mt_off.as<uint32_t>();
  a.mt_mk = c->dag_mt_mk.as<uint32_t>();
  a.mt_cand = c->dag_mt_cand.as<unsigned long long>();
  a.out = d_out;
  a.checks = reinterpret_cast<unsigned long long*>(d_checksums);
  a.tables_global = (size_t)c->lay.words * 4 > kMaxSmem ? 1u : 0u;
  CK(launch_dag(a, (cudaStream_t)stream), "dag kernel");
  return FFS_OK;
}

ffs_status ffs_plan_joint(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req, uint32_t k_max,
                          ffs_plan* d_out, uint32_t* rounds, void* stream) {
  if (!c) return FFS_ERR_ARG;
  ffs_status s0 = check_kmax(c, k_max);
  if (s0 != FFS_OK) return s0;
  if (rounds) *rounds = 0;
  if (n_req == 0) return FFS_OK;
  if (!d_req || !d_slo || !d_out) return fail(c, FFS_ERR_ARG, "null device pointer");
  if (n_req >= (1u << 31)) return fail(c, FFS_ERR_RANGE, "n_req >= 2^31");
  DeviceGuard g(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  const size_t R = n_req, NN = c->n_nodes, S = std::max(1u, c->n_slices);
  CK(c->j_keys.ensure(R * 8), "cudaMalloc");
  CK(c->j_state.ensure(R), "cudaMalloc");
  CK(c->j_dirty.ensure(R * 4), "cudaMalloc");
  CK(c->j_sreq.ensure(R * sizeof(ffs_request)), "cudaMalloc");
  CK(c->j_sslo.ensure(R * 4), "cudaMalloc");
  CK(c->j_skeys.ensure(R * 8), "cudaMalloc");
  CK(c->j_win.ensure(NN * 8), "cudaMalloc");
  CK(c->j_busy.ensure(S), "cudaMalloc");
  CK(c->j_cnt.ensure(NN * 8), "cudaMalloc");
  CK(c->j_free.ensure(NN * 8), "cudaMalloc");
  CK(c->j_ctr.ensure(8), "cudaMalloc");
  if (c->n_slices)
    CK(cudaMemcpyAsync(c->j_busy.p, c->h_busy.data(), c->n_slices, cudaMemcpyHostToDevice, st), "H2D busy");
  CK(cudaMemcpyAsync(c->j_cnt.p, c->h_cnt.data(), NN * 8, cudaMemcpyHostToDevice, st), "H2D counts");
  CK(cudaMemcpyAsync(c->j_free.p, c->h_node_free.data(), NN * 8, cudaMemcpyHostToDevice, st), "H2D free");
  JointArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.req = d_req;
  a.slo = d_slo;
  a.n_req = n_req;
  a.n_nodes = c->n_nodes;
  a.k_max = k_max;
  a.keys = c->j_keys.as<int64_t>();
  a.state = c->j_state.as<uint8_t>();
  a.dirty = c->j_dirty.as<uint32_t>();
  a.sub_req = c->j_sreq.as<ffs_request>();
  a.sub_slo = c->j_sslo.as<uint32_t>();
  a.sub_keys = c->j_skeys.as<int64_t>();
  a.node_win = c->j_win.as<uint64_t>();
  a.busy = c->j_busy.as<uint8_t>();
  a.cnt = c->j_cnt.as<uint8_t>();
  a.node_free = c->j_free.as<uint64_t>();
  a.node_off = c->node_off.as<uint32_t>();
  a.slice_prof = c->slice_prof.as<uint8_t>();
  a.out = d_out;
  a.n_open = c->j_ctr.as<uint32_t>();
  a.n_dirty = c->j_ctr.as<uint32_t>() + 1;
  CK(launch_joint(0, a, 0, st), "joint init");
  uint32_t n_sub = n_req, nr = 0;
  for (;;) {
    ++nr;
    if (n_sub) {
      CK(launch_joint(1, a, n_sub, st), "joint gather");
      ffs_status s = search_keys(c, a.sub_req, a.sub_slo, n_sub, k_max, 0, 1, a.sub_keys, nullptr, a.node_free, stream);
      if (s != FFS_OK) return s;
      CK(launch_joint(2, a, n_sub, st), "joint scatter");
    }
    CK(cudaMemsetAsync(a.node_win, 0xFF, NN * 8, st), "memset");
    CK(cudaMemsetAsync(a.n_open, 0, 8, st), "memset");
    CK(launch_joint(3, a, 0, st), "joint pick");
    CK(launch_joint(4, a, 0, st), "joint commit");
    CK(launch_joint(5, a, 0, st), "joint finalize");
    uint32_t ctr[2];
    CK(cudaMemcpyAsync(ctr, a.n_open, 8, cudaMemcpyDeviceToHost, st), "D2H counters");
    CK(cudaStreamSynchronize(st), "sync");
    if (ctr[0] == 0) break;
    n_sub = ctr[1];
  }
  if (rounds) *rounds = nr;
  return FFS_OK;
}

ffs_status ffs_route(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req,
                     const ffs_instance* d_inst, const uint8_t* d_state, const uint32_t* d_lat, const uint32_t* d_cap,
                     uint32_t n_inst, int32_t* d_route, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged) return fail(c, FFS_ERR_STATE, "tables not staged");
  if (n_req == 0) return FFS_OK;
  if (n_req >= (1u << 31) || n_inst >= (1u << 31)) return fail(c, FFS_ERR_RANGE, "n_req/n_inst >= 2^31");
  if (c->F >= (1u << 22)) return fail(c, FFS_ERR_RANGE, "n_funcs >= 2^22");
  if (!d_req || !d_slo || !d_route || (n_inst && (!d_inst || !d_state || !d_lat || !d_cap)))
    return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  const size_t R = n_req, I = std::max(1u, n_inst), F1 = c->F + 1;
  for (DevBuf* b : {&c->r_k, &c->r_k2}) CK(b->ensure(R * 8), "cudaMalloc");
  for (DevBuf* b : {&c->r_v, &c->r_v2}) CK(b->ensure(R * 4), "cudaMalloc");
  for (DevBuf* b : {&c->i_k, &c->i_k2}) CK(b->ensure(I * 8), "cudaMalloc");
  for (DevBuf* b : {&c->i_v, &c->i_v2}) CK(b->ensure(I * 4), "cudaMalloc");
  CK(c->i_cum.ensure((I + 1) * 8), "cudaMalloc");
  for (DevBuf* b : {&c->r_f, &c->r_h, &c->r_n, &c->r_ts}) CK(b->ensure(F1 * 4), "cudaMalloc");
  const size_t nmax = std::max<size_t>(R, I);
  const size_t hist = 256 * ((nmax + 2047) / 2048) + 1;
  CK(c->r_hist.ensure(hist * 8), "cudaMalloc");
  CK(c->r_bsum.ensure(((hist + 2047) / 2048 + 1) * 8), "cudaMalloc");
  RouteArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.req = d_req;
  a.slo = d_slo;
  a.n_req = n_req;
  a.n_inst = n_inst;
  a.inst = d_inst;
  a.state = d_state;
  a.lat = d_lat;
  a.cap = d_cap;
  a.rkey = c->r_k.as<uint64_t>();
  a.rval = c->r_v.as<uint32_t>();
  a.ikey = c->i_k.as<uint64_t>();
  a.ival = c->i_v.as<uint32_t>();
  a.icum = a.icap = c->i_cum.as<uint64_t>();
  a.first_req = c->r_f.as<uint32_t>();
  a.first_hot = c->r_h.as<uint32_t>();
  a.n_hot = c->r_n.as<uint32_t>();
  a.ts = c->r_ts.as<int32_t>();
  a.route = d_route;
  int fb = 1;
  while ((1u << fb) <= c->F) ++fb;  // bits of the function id (F means "invalid")
  CK(launch_route(0, a, st), "route keys");
  CK(radix_sort_pairs(a.rkey, a.rval, c->r_k2.as<uint64_t>(), c->r_v2.as<uint32_t>(), n_req, 34 + fb,
                      c->r_hist.as<uint64_t>(), c->r_bsum.as<uint64_t>(), st), "sort requests");
  if (n_inst)
    CK(radix_sort_pairs(a.ikey, a.ival, c->i_k2.as<uint64_t>(), c->i_v2.as<uint32_t>(), n_inst, 33 + fb,
                        c->r_hist.as<uint64_t>(), c->r_bsum.as<uint64_t>(), st), "sort instances");
  CK(cudaMemsetAsync(a.icum + n_inst, 0, 8, st), "memset");
  CK(launch_route(1, a, st), "route marks");
  CK(scan_u64(a.icum, (uint64_t)n_inst + 1, c->r_bsum.as<uint64_t>(), st), "capacity scan");
  CK(launch_route(2, a, st), "route assign");
  return FFS_OK;
}

ffs_status ffs_simulate(ffs_ctx* c, const uint32_t* d_req_off, const uint32_t* d_req_func,
                        const uint32_t* d_req_budget, uint32_t n_ticks, uint64_t t0_us, uint32_t tick_us,
                        uint32_t window_ticks, uint32_t thr_pct, uint64_t cold_after_us, uint32_t k_max,
                        uint64_t* d_ctr, int32_t* d_slice, uint8_t* d_state, uint64_t* d_last, uint32_t* d_busy,
                        uint8_t* d_stages, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged) return fail(c, FFS_ERR_STATE, "tables not staged");
  if (k_max > (uint32_t)kMaxK) return fail(c, FFS_ERR_RANGE, "k_max %u > 8", k_max);
  if (k_max >= 2) {
    ffs_status s = check_kmax(c, k_max);
    if (s != FFS_OK) return s;
  }
  if (n_ticks == 0) return FFS_OK;
  if (!d_req_off || !d_req_func || !d_req_budget || !d_ctr || !d_slice || !d_state || !d_last || !d_busy ||
      !d_stages)
    return fail(c, FFS_ERR_ARG, "null device pointer");
  if (window_ticks == 0 || tick_us == 0) return fail(c, FFS_ERR_ARG, "window_ticks and tick_us must be > 0");
  if (c->n_slices >= (1u << 20)) return fail(c, FFS_ERR_RANGE, "n_slices >= 2^20");
  DeviceGuard g(c->device);
  CK(c->s_res.ensure((size_t)std::max(1u, c->n_slices) * 4), "cudaMalloc");
  CK(c->s_flags.ensure((size_t)c->n_nodes * c->F), "cudaMalloc");
  CK(c->s_busy.ensure(std::max<size_t>(1, c->n_slices)), "cudaMalloc");
  CK(c->s_psl.ensure((size_t)c->n_nodes * c->F * 8 * 4), "cudaMalloc");
  CK(c->s_pe2e.ensure((size_t)c->n_nodes * c->F * 4), "cudaMalloc");
  CK(c->s_pk.ensure((size_t)c->n_nodes * c->F), "cudaMalloc");
  if (c->n_slices)
    CK(cudaMemcpyAsync(c->s_busy.p, c->h_busy.data(), c->n_slices, cudaMemcpyHostToDevice, (cudaStream_t)stream),
       "H2D busy");
  SimArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.n_nodes = c->n_nodes;
  a.n_ticks = n_ticks;
  a.window_ticks = window_ticks;
  a.thr_pct = thr_pct;
  a.tick_us = tick_us;
  a.t0_us = t0_us;
  a.cold_after_us = cold_after_us;
  a.node_off = c->node_off.as<uint32_t>();
  a.slice_prof = c->slice_prof.as<uint8_t>();
  a.slice_busy = c->s_busy.as<uint8_t>();
  a.req_off = d_req_off;
  a.req_func = d_req_func;
  a.req_budget = d_req_budget;
  a.res = c->s_res.as<int32_t>();
  a.flags = c->s_flags.as<uint8_t>();
  a.ctr = d_ctr;
  a.slice = d_slice;
  a.state = d_state;
  a.last = d_last;
  a.busy = d_busy;
  a.stages = d_stages;
  a.k_max = k_max;
  a.psl = c->s_psl.as<int32_t>();
  a.pe2e = c->s_pe2e.as<uint32_t>();
  a.pk = c->s_pk.as<uint8_t>();
  CK(launch_sim(a, (cudaStream_t)stream), "simulator kernel");
  return FFS_OK;
}

ffs_status ffs_frontier_build(ffs_ctx* c, uint32_t k_max, uint32_t* n_groups, uint32_t* rounds, void* stream) {
  if (!c) return FFS_ERR_ARG;
  ffs_status s0 = check_kmax(c, k_max);
  if (s0 != FFS_OK) return s0;
  DeviceGuard g(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  c->front_built = false;
  // groups = (function, distinct clamped free vector of a node)
  std::vector<uint32_t> node_fv(c->n_nodes), fv_node;
  {
    std::vector<std::pair<uint64_t, uint32_t>> seen;
    for (uint32_t v = 0; v < c->n_nodes; ++v) {
      uint32_t id = (uint32_t)seen.size();
      for (auto& e : seen)
        if (e.first == c->h_node_free[v]) id = e.second;
      if (id == seen.size()) {
        seen.push_back({c->h_node_free[v], id});
        fv_node.push_back(v);
      }
      node_fv[v] = id;
    }
  }
  const uint32_t nfv = (uint32_t)fv_node.size();
  const uint64_t G64 = (uint64_t)c->F * nfv;
  if (G64 >= (1ull << 31)) return fail(c, FFS_ERR_RANGE, "too many frontier groups");
  const uint32_t G = (uint32_t)G64;
  CK(c->f_nodefv.ensure(node_fv.size() * 4), "cudaMalloc");
  CK(cudaMemcpy(c->f_nodefv.p, node_fv.data(), node_fv.size() * 4, cudaMemcpyHostToDevice), "H2D");
  CK(c->f_fvnode.ensure(fv_node.size() * 4), "cudaMalloc");
  CK(cudaMemcpy(c->f_fvnode.p, fv_node.data(), fv_node.size() * 4, cudaMemcpyHostToDevice), "H2D");
  for (DevBuf* b : {&c->f_act, &c->f_next, &c->f_budget, &c->f_gslo, &c->f_cnt}) CK(b->ensure((size_t)G * 4), "cudaMalloc");
  CK(c->f_greq.ensure((size_t)G * sizeof(ffs_request)), "cudaMalloc");
  CK(c->f_gkeys.ensure((size_t)G * 8), "cudaMalloc");
  CK(c->f_ctr.ensure(8), "cudaMalloc");
  std::vector<uint32_t> iota(G);
  for (uint32_t i = 0; i < G; ++i) iota[i] = i;
  CK(cudaMemcpyAsync(c->f_act.p, iota.data(), (size_t)G * 4, cudaMemcpyHostToDevice, st), "H2D");
  CK(cudaMemsetAsync(c->f_budget.p, 0xFF, (size_t)G * 4, st), "memset");
  CK(cudaMemsetAsync(c->f_cnt.p, 0, (size_t)G * 4, st), "memset");
  uint32_t cap = 64;
  CK(c->f_key.ensure((size_t)cap * G * 8), "cudaMalloc");
  CK(c->f_e2e.ensure((size_t)cap * G * 4), "cudaMalloc");
  FrontierArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.k_max = k_max;
  a.n_groups = G;
  a.n_fv = nfv;
  a.n_nodes = c->n_nodes;
  a.node_fv = c->f_nodefv.as<uint32_t>();
  a.budget = c->f_budget.as<uint32_t>();
  a.greq = c->f_greq.as<ffs_request>();
  a.n_next = c->f_ctr.as<uint32_t>();
  a.fr_cnt = c->f_cnt.as<uint32_t>();
  uint32_t n_active = G, round = 0;
  uint32_t *act = c->f_act.as<uint32_t>(), *nxt = c->f_next.as<uint32_t>();
  while (n_active) {
    if (round == cap) {  // grow the round-major point arrays
      DevBuf nk, ne;
      CK(nk.ensure((size_t)2 * cap * G * 8), "cudaMalloc");
      CK(ne.ensure((size_t)2 * cap * G * 4), "cudaMalloc");
      CK(cudaMemcpyAsync(nk.p, c->f_key.p, (size_t)cap * G * 8, cudaMemcpyDeviceToDevice, st), "D2D");
      CK(cudaMemcpyAsync(ne.p, c->f_e2e.p, (size_t)cap * G * 4, cudaMemcpyDeviceToDevice, st), "D2D");
      CK(cudaStreamSynchronize(st), "sync");
      c->f_key.release();
      c->f_e2e.release();
      c->f_key = nk;
      c->f_e2e = ne;
      nk.p = ne.p = nullptr;
      cap *= 2;
    }
    a.cap = cap;
    a.fr_key = c->f_key.as<int64_t>();
    a.fr_e2e = c->f_e2e.as<uint32_t>();
    a.active = act;
    a.next_active = nxt;
    a.keys = c->f_gkeys.as<int64_t>();
    a.round = round;
    CK(launch_front_gather(a, n_active, c->f_fvnode.as<uint32_t>(), c->f_gslo.as<uint32_t>(), st), "gather");
    ffs_status s = search_keys(c, a.greq, c->f_gslo.as<uint32_t>(), n_active, k_max, 0, 1, c->f_gkeys.as<int64_t>(),
                               nullptr, nullptr, stream);
    if (s != FFS_OK) return s;
    CK(cudaMemsetAsync(a.n_next, 0, 4, st), "memset");
    CK(launch_frontier(1, a, n_active, st), "record");
    CK(cudaMemcpyAsync(&n_active, a.n_next, 4, cudaMemcpyDeviceToHost, st), "D2H");
    CK(cudaStreamSynchronize(st), "sync");
    std::swap(act, nxt);
    ++round;
  }
  c->front_built = true;
  c->front_kmax = k_max;
  c->front_groups = G;
  c->front_nfv = nfv;
  c->front_cap = cap;
  if (n_groups) *n_groups = G;
  if (rounds) *rounds = round;
  return FFS_OK;
}

ffs_status ffs_plan_frontier(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req,
                             ffs_plan* d_out, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged || !c->front_built) return fail(c, FFS_ERR_STATE, "call ffs_frontier_build after staging");
  if (n_req == 0) return FFS_OK;
  if (!d_req || !d_slo || !d_out) return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  FrontierArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.k_max = c->front_kmax;
  a.n_groups = c->front_groups;
  a.n_fv = c->front_nfv;
  a.n_nodes = c->n_nodes;
  a.cap = c->front_cap;
  a.node_fv = c->f_nodefv.as<uint32_t>();
  a.fr_key = c->f_key.as<int64_t>();
  a.fr_e2e = c->f_e2e.as<uint32_t>();
  a.fr_cnt = c->f_cnt.as<uint32_t>();
  a.req = d_req;
  a.slo = d_slo;
  a.n_req = n_req;
  a.free_list = c->free_list.as<int32_t>();
  a.out = d_out;
  CK(launch_frontier(2, a, 0, (cudaStream_t)stream), "frontier query");
  return FFS_OK;
}

ffs_status ffs_plan_frontier_any(ffs_ctx* c, const ffs_request* d_req, const uint32_t* d_slo, uint32_t n_req,
                                 ffs_plan* d_out, int32_t* d_node, void* stream) {
  if (!c) return FFS_ERR_ARG;
  if (!c->staged || !c->front_built) return fail(c, FFS_ERR_STATE, "call ffs_frontier_build after staging");
  if (n_req == 0) return FFS_OK;
  if (!d_req || !d_slo || !d_out) return fail(c, FFS_ERR_ARG, "null device pointer");
  DeviceGuard g(c->device);
  FrontierArgs a{};
  a.image = c->image.as<uint32_t>();
  a.lay = c->lay;
  a.k_max = c->front_kmax;
  a.n_groups = c->front_groups;
  a.n_fv = c->front_nfv;
  a.n_nodes = c->n_nodes;
  a.cap = c->front_cap;
  a.node_fv = c->f_nodefv.as<uint32_t>();
  a.fv_node = c->f_fvnode.as<uint32_t>();
  a.fr_key = c->f_key.as<int64_t>();
  a.fr_e2e = c->f_e2e.as<uint32_t>();
  a.fr_cnt = c->f_cnt.as<uint32_t>();
  a.req = d_req;
  a.slo = d_slo;
  a.n_req = n_req;
  a.free_list = c->free_list.as<int32_t>();
  a.out = d_out;
  a.node_out = d_node;
  CK(launch_frontier(3, a, 0, (cudaStream_t)stream), "frontier any-invoker query");
  return FFS_OK;
}

ffs_status ffs_bench_int_peak(ffs_ctx* c, double* ops, double* seconds) {
  if (!c || !ops || !seconds) return FFS_ERR_ARG;
  DeviceGuard g(c->device);
  CK(run_int_peak(c->sms, ops, seconds), "int peak kernel");
  return FFS_OK;
}

ffs_status ffs_segment_times(ffs_ctx* c, float* ms) {
  if (!c || !ms) return FFS_ERR_ARG;
  for (int k = 0; k < kMaxK; ++k) ms[k] = 0.f;
  DeviceGuard g(c->device);
  for (int k = 1; k <= kMaxK; ++k) {
    if (!((c->seg_mask >> k) & 1u)) continue;
    CK(cudaEventSynchronize(c->ev[k]), "event sync");
    CK(cudaEventElapsedTime(&ms[k - 1], c->evs[k], c->ev[k]), "event time");
  }
  return FFS_OK;
}

ffs_status ffs_set_search_mode(ffs_ctx* c, uint32_t mode) {
  if (!c) return FFS_ERR_ARG;
  if (mode != FFS_SEARCH_BOUNDED && mode != FFS_SEARCH_EXHAUSTIVE) return fail(c, FFS_ERR_ARG, "search mode %u", mode);
  c->search_mode = mode;
  return FFS_OK;
}

ffs_status ffs_search_scored(ffs_ctx* c, uint64_t* per_ks) {
  if (!c || !per_ks) return FFS_ERR_ARG;
  for (int k = 0; k < kMaxK; ++k) per_ks[k] = 0;
  if (!c->work_ctr.p) return FFS_OK;
  DeviceGuard g(c->device);
  CK(cudaDeviceSynchronize(), "sync");
  unsigned long long w[kCtrWords];
  CK(cudaMemcpy(w, c->work_ctr.p, sizeof w, cudaMemcpyDeviceToHost), "read counters");
  for (int k = 1; k <= kMaxK; ++k) per_ks[k - 1] = w[kCtrScored + k];
  return FFS_OK;
}

ffs_status ffs_search_live_records(ffs_ctx* c, uint64_t* per_ks) {
  if (!c || !per_ks) return FFS_ERR_ARG;
  for (int k = 0; k < kMaxK; ++k) per_ks[k] = 0;
  if (!c->work_ctr.p) return FFS_OK;
  DeviceGuard g(c->device);
  CK(cudaDeviceSynchronize(), "sync");
  unsigned long long w[kCtrWords];
  CK(cudaMemcpy(w, c->work_ctr.p, sizeof w, cudaMemcpyDeviceToHost), "read counters");
  for (int k = 1; k <= kMaxK; ++k) per_ks[k - 1] = w[kCtrListCount + k];
  return FFS_OK;
}

ffs_status ffs_bench_packed_peak(ffs_ctx* c, uint32_t mode, double* lane_instr_per_s, double* seconds) {
  if (!c || !lane_instr_per_s || !seconds || mode > 2) return FFS_ERR_ARG;
  DeviceGuard g(c->device);
  CK(run_packed_peak(c->sms, (int)mode, lane_instr_per_s, seconds), "packed peak kernel");
  return FFS_OK;
}

ffs_status ffs_debug_filter_misses(ffs_ctx* c, uint64_t* out) {
  if (!c || !out) return FFS_ERR_ARG;
  DeviceGuard g(c->device);
  CK(cudaDeviceSynchronize(), "sync");
  CK(cudaMemcpy(out, c->misses.p, 8, cudaMemcpyDeviceToHost), "read misses");
  return FFS_OK;
}

}  // extern "C"
