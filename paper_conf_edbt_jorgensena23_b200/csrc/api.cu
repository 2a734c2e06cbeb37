// api.cu -- C ABI (include/eggsync.h), workspace and the host loop of
// Algorithm 4.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "common.cuh"

namespace egg {

template <int D>
int run_update(Workspace&, int64_t, int64_t, int32_t*);
template <int D>
int run_second_term(Workspace&, int64_t, int64_t);
size_t cub_temp_bytes(int64_t n);

static thread_local std::string g_err;

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
}

bool make_consts(int64_t n, int d, float eps, Consts* c, std::string* why, double cw_factor) {
  if (!(eps > 0.f) || !std::isfinite(eps)) {
    *why = "eps must be finite and > 0";
    return false;
  }
  if (!(cw_factor > 0.0 && cw_factor <= 1.0)) {
    *why = "cw_factor must be in (0, 1] (c_w <= eps/(2 sqrt d), L252)";
    return false;
  }
  c->n = n;
  c->d = d;
  c->e = (double)eps;
  c->e2 = c->e * c->e;
  c->cw = cw_factor * (c->e / (2.0 * std::sqrt((double)d)));  // L252: cell diagonal <= eps/2
  c->inv_cw = 1.0 / c->cw;
  const double wd = std::ceil(1.0 / c->cw);     // Eq.4
  if (wd > 2147483647.0) {
    *why = "grid too fine (ceil(1/c_w) > 2^31)";
    return false;
  }
  c->w = (int64_t)wd;
  int bits = 0;
  while ((int64_t(1) << bits) < c->w) ++bits;
  c->bits = std::max(bits, 1);
  if (d * c->bits > 64 * kMaxKeyWords) {
    *why = "grid too fine: d*ceil(log2 w) > 512 key bits";
    return false;
  }
  // Update units: each cell split into 2^(sub*d) sub-cells (F2).  In low d a cell holds
  // many points and a ball boundary cuts through cells; finer units shrink the
  // point-by-point boundary scan.  In high d cells are (near) singletons already.
  // (measured on C2-C5, T1: finer is faster until units are ~single points)
  static const int kSubByDim[21] = {0, 8, 8, 7, 6, 5, 5, 4, 3, 3, 2, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  int sub = d <= 20 ? kSubByDim[d] : 0;
  if (const char* s = getenv("EGGSYNC_SUBBITS")) sub = std::max(0, std::min(8, atoi(s)));
  while (sub > 0 && d * (c->bits + sub) > 64 * kMaxKeyWords) --sub;
  c->sub = sub;
  c->keybits = d * (c->bits + sub);
  c->nw = (c->keybits + 63) / 64;
  c->delta = c->e - c->e * std::sqrt(15.0 / 16.0) + c->e / 2.0 - std::sin(c->e / 2.0);  // L110
  c->ed = c->e + c->delta;
  c->ed2 = c->ed * c->ed;
  c->ef = eps;
  c->e2f = (float)c->e2;
  c->edf = (float)c->ed;
  c->ed2f = (float)c->ed2;
  c->rel = (float)(4 * d + 16) * kU;
  return true;
}

// ------------------------------------------------------------------ workspace cache
// One released workspace arena (+ its pinned flag mirror) is kept per device and
// reused by the next call that fits in it -- a caching allocator, so repeated
// eggsync_cluster() calls do not pay cudaMalloc/cudaFree (eggsync_release_cache()).
struct CachedArena {
  int device;
  char* p;
  size_t bytes;
  int32_t* hflags;
};
static std::mutex g_cache_mu;
static std::vector<CachedArena> g_cache;

static bool cache_take(int device, size_t need, char** p, size_t* bytes, int32_t** hflags) {
  std::lock_guard<std::mutex> lk(g_cache_mu);
  for (size_t k = 0; k < g_cache.size(); ++k) {
    if (g_cache[k].device == device && g_cache[k].bytes >= need) {
      *p = g_cache[k].p;
      *bytes = g_cache[k].bytes;
      *hflags = g_cache[k].hflags;
      g_cache.erase(g_cache.begin() + k);
      return true;
    }
  }
  return false;
}

static void cache_give(int device, char* p, size_t bytes, int32_t* hflags) {
  std::lock_guard<std::mutex> lk(g_cache_mu);
  for (size_t k = 0; k < g_cache.size(); ++k) {
    if (g_cache[k].device == device) {
      if (g_cache[k].bytes >= bytes) {  // keep the larger one
        cudaFree(p);
        cudaFreeHost(hflags);
        return;
      }
      cudaFree(g_cache[k].p);
      cudaFreeHost(g_cache[k].hflags);
      g_cache.erase(g_cache.begin() + k);
      break;
    }
  }
  g_cache.push_back({device, p, bytes, hflags});
}

// grow-only buffers of the tensor-core update (range lists, entry lists), cached per
// (device, tag) across calls like the arenas
struct CachedBuf {
  int device;
  int tag;
  void* p;
  size_t bytes;
};
static std::vector<CachedBuf> g_rcache;

static int buf_reserve(Workspace& ws, int tag, void** p, size_t* cap_bytes, size_t need_bytes) {
  if (*cap_bytes >= need_bytes) return EGGSYNC_OK;
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    for (size_t k = 0; k < g_rcache.size(); ++k) {
      if (g_rcache[k].device == ws.cur_device && g_rcache[k].tag == tag && g_rcache[k].bytes >= need_bytes) {
        if (*p) {
          cudaStreamSynchronize(ws.stream);
          cudaFree(*p);
        }
        *p = g_rcache[k].p;
        *cap_bytes = g_rcache[k].bytes;
        g_rcache.erase(g_rcache.begin() + k);
        return EGGSYNC_OK;
      }
    }
  }
  if (*p) {
    EGG_CUDA(cudaStreamSynchronize(ws.stream));
    EGG_CUDA(cudaFree(*p));
    *p = nullptr;
    *cap_bytes = 0;
  }
  const size_t cap = need_bytes + need_bytes / 4 + 4096;
  EGG_CUDA(cudaMalloc(p, cap));
  *cap_bytes = cap;
  return EGGSYNC_OK;
}

static void buf_give(int device, int tag, void* p, size_t bytes) {
  if (!p) return;
  std::lock_guard<std::mutex> lk(g_cache_mu);
  for (size_t k = 0; k < g_rcache.size(); ++k) {
    if (g_rcache[k].device == device && g_rcache[k].tag == tag) {
      if (g_rcache[k].bytes >= bytes) {
        cudaFree(p);
        return;
      }
      cudaFree(g_rcache[k].p);
      g_rcache.erase(g_rcache.begin() + k);
      break;
    }
  }
  g_rcache.push_back({device, tag, p, bytes});
}

int tc_ranges_reserve(Workspace& ws, size_t need) {
  size_t cb = ws.tc_rcap * sizeof(int2);
  const int rc = buf_reserve(ws, 0, (void**)&ws.tc_ranges, &cb, need * sizeof(int2));
  ws.tc_rcap = cb / sizeof(int2);
  return rc;
}

int dense_reserve(Workspace& ws, size_t cells) {
  return buf_reserve(ws, 2, (void**)&ws.dense, &ws.dense_bytes, cells * sizeof(int32_t));
}

int tc_ent_reserve(Workspace& ws, size_t need) {
  size_t cb = ws.tc_ecap * sizeof(int32_t);
  const int rc = buf_reserve(ws, 1, (void**)&ws.tc_ent, &cb, need * sizeof(int32_t));
  ws.tc_ecap = cb / sizeof(int32_t);
  return rc;
}

static void cache_clear() {
  std::lock_guard<std::mutex> lk(g_cache_mu);
  int prev = -1;
  cudaGetDevice(&prev);
  for (auto& c : g_cache) {
    cudaSetDevice(c.device);
    cudaFree(c.p);
    cudaFreeHost(c.hflags);
  }
  g_cache.clear();
  for (auto& c : g_rcache) {
    cudaSetDevice(c.device);
    cudaFree(c.p);
  }
  g_rcache.clear();
  if (prev >= 0) cudaSetDevice(prev);
}

int Workspace::alloc(int64_t n_, int d_, float eps, int dev, cudaStream_t st, double cw_factor) {
  std::string why;
  if (!make_consts(n_, d_, eps, &k, &why, cw_factor)) {
    set_error("%s", why.c_str());
    return EGGSYNC_EINVAL;
  }
  n = n_;
  d = d_;
  cap = n_;
  device = dev;
  const int nw = k.nw;
  const int CREC = ceil4(3 * d + 3), BS = ceil4(2 * d);
  cub_bytes = cub_temp_bytes(n);
  struct Item {
    void** p;
    size_t bytes;
  };
  Item items[] = {
      {(void**)&xs[0], sizeof(float) * d * n},
      {(void**)&xs[1], sizeof(float) * d * n},
      {(void**)&orig[0], sizeof(uint32_t) * n},
      {(void**)&orig[1], sizeof(uint32_t) * n},
      {(void**)&keys, sizeof(uint64_t) * nw * n},
      {(void**)&keys_tmp, sizeof(uint64_t) * nw * n},
      {(void**)&kb[0], sizeof(uint64_t) * n},
      {(void**)&kb[1], sizeof(uint64_t) * n},
      {(void**)&pb[0], sizeof(uint32_t) * n},
      {(void**)&pb[1], sizeof(uint32_t) * n},
      {(void**)&cub_tmp, cub_bytes},
      {(void**)&sn, sizeof(float) * d * n},
      {(void**)&cs, sizeof(float) * d * n},
      {(void**)&cell_of, sizeof(int32_t) * n},
      {(void**)&iscan, sizeof(int32_t) * n},
      {(void**)&cell_start, sizeof(int32_t) * (cap + 1)},
      {(void**)&c_fix, sizeof(uint64_t) * 2 * d * cap},
      {(void**)&c_lo, sizeof(uint32_t) * d * cap},
      {(void**)&c_hi, sizeof(uint32_t) * d * cap},
      {(void**)&c_cnt, sizeof(int32_t) * cap},
      {(void**)&c_rec, sizeof(float) * CREC * cap},
      {(void**)&c_dig, d <= kTcMaxD ? (size_t)(((kDigMax * (2 * d + 1)) + 15) / 16 * 16) * cap : 0},
      {(void**)&c_head, d <= kTcMaxD ? sizeof(float) * ceil4(d + 3) * cap : 0},
      {(void**)&c_key, sizeof(uint64_t) * nw * cap},
      {(void**)&t_meta, sizeof(int4) * cap},
      {(void**)&t_parent, sizeof(int32_t) * cap},
      {(void**)&l_parent, sizeof(int32_t) * cap},
      {(void**)&t_visit, sizeof(uint32_t) * cap},
      {(void**)&t_fix, sizeof(uint64_t) * 3 * d * cap},  // k_tree_agg rows: exact sums [2d], (hi<<32|lo) [d]
      {(void**)&t_cnt, sizeof(int32_t) * cap},
      {(void**)&t_box, sizeof(float) * BS * cap},
      {(void**)&t_sum, sizeof(float) * BS * cap},
      {(void**)&flags, sizeof(int32_t) * 8},
      {(void**)&io, sizeof(float) * d * n},
      {(void**)&i_lab, sizeof(int32_t) * n},
      {(void**)&c_minorig, sizeof(uint32_t) * cap},
      {(void**)&nbr, sizeof(int32_t) * n},
      {(void**)&lab_final, sizeof(int32_t) * n},
      {(void**)&second_need, sizeof(uint8_t) * cap},
      {(void**)&work, sizeof(unsigned long long) * 8},
      {(void**)&co_of, sizeof(int32_t) * n},
      {(void**)&full_S, d <= 16 ? sizeof(double) * 2 * d * n : 0},
      {(void**)&full_N, sizeof(int32_t) * n},
      {(void**)&tc_nr, sizeof(int32_t) * (n / 128 + 2)},
      {(void**)&tc_ne, sizeof(int32_t) * (n / 128 + 2)},
      {(void**)&tc_chunks, d <= 16 ? sizeof(int32_t) * (n / 128 + 2) * kChunkMax : 0},
      {(void**)&tc_ctr, sizeof(int32_t) * 8},
      {(void**)&tc_epad, sizeof(int32_t) * (n / 128 + 2)},
      {(void**)&tc_eoff, sizeof(int32_t) * (n / 128 + 2)},
      {(void**)&tc_pv, sizeof(int32_t) * (n / 128 + 2)},
      {(void**)&tc_pk, sizeof(int32_t) * (n / 128 + 2)},
      {(void**)&tc_perm, sizeof(int32_t) * (n / 128 + 2)},
      {(void**)&co_start, sizeof(int32_t) * (cap + 1)},
      {(void**)&co_cnt, sizeof(int32_t) * cap},
      {(void**)&co_lo, sizeof(uint32_t) * d * cap},
      {(void**)&co_hi, sizeof(uint32_t) * d * cap},
      {(void**)&u2co, sizeof(int32_t) * cap},
  };
  size_t total = 0;
  for (auto& it : items) total += (it.bytes + 255) & ~size_t(255);
  char* base = nullptr;
  EGG_CUDA(cudaGetDevice(&cur_device));
  size_t got = 0;
  if (cache_take(cur_device, total, &base, &got, &h_flags)) {
    total = got;
  } else {
    cudaError_t e = cudaMalloc((void**)&base, total);
    if (e != cudaSuccess) {
      set_error("cudaMalloc(%zu bytes) failed: %s", total, cudaGetErrorString(e));
      cudaGetLastError();
      return e == cudaErrorMemoryAllocation ? EGGSYNC_ENOMEM : EGGSYNC_ECUDA;
    }
    e = cudaMallocHost((void**)&h_flags, 16 * sizeof(int32_t));
    if (e != cudaSuccess) {
      cudaFree(base);
      set_error("cudaMallocHost failed: %s", cudaGetErrorString(e));
      return EGGSYNC_ENOMEM;
    }
  }
  arena = base;
  size_t off = 0;
  for (auto& it : items) {
    *it.p = base + off;
    off += (it.bytes + 255) & ~size_t(255);
  }
  bytes = (int64_t)total;
  if (st) {
    stream = st;
    own_stream = false;
  } else {
    EGG_CUDA(cudaStreamCreateWithFlags(&stream, cudaStreamNonBlocking));
    own_stream = true;
  }
  for (auto& v : ev) EGG_CUDA(cudaEventCreate(&v));
  ev_ok = true;
  EGG_CUDA(cudaMemsetAsync(flags, 0, 8 * sizeof(int32_t), stream));
  return EGGSYNC_OK;
}

void Workspace::release() {
  if (arena) {
    if (stream) cudaStreamSynchronize(stream);  // no pending work may touch a cached arena
    cache_give(cur_device, arena, (size_t)bytes, h_flags);
  }
  buf_give(cur_device, 0, tc_ranges, tc_rcap * sizeof(int2));
  buf_give(cur_device, 1, tc_ent, tc_ecap * sizeof(int32_t));
  buf_give(cur_device, 2, dense, dense_bytes);
  dense = nullptr;
  dense_bytes = 0;
  tc_ent = nullptr;
  tc_ecap = 0;
  tc_ranges = nullptr;
  tc_rcap = 0;
  for (auto& e : tc_ev)
    if (e) {
      cudaEventDestroy(e);
      e = nullptr;
    }
  tc_pending = false;
  arena = nullptr;
  h_flags = nullptr;
  if (own_stream && stream) cudaStreamDestroy(stream);
  stream = nullptr;
  own_stream = false;
  if (ev_ok)
    for (auto& v : ev) cudaEventDestroy(v);
  ev_ok = false;
}


int stage_update(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr) {
  EGG_DISPATCH(ws.d, run_update, ws, lo, hi, nbr);
}
int stage_second_term(Workspace& ws, int64_t lo, int64_t hi) {
  EGG_DISPATCH(ws.d, run_second_term, ws, lo, hi);
}

__global__ void k_set_flags(int32_t* f, int32_t a, int32_t b) {
  f[0] = a;
  f[1] = b;
}
__global__ void k_pack(const float* __restrict__ xs, int64_t n, int d, int64_t lo, int64_t cnt,
                       float* __restrict__ buf) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= cnt * d) return;
  int i = (int)(t / cnt);
  int64_t k = t - (int64_t)i * cnt;
  int64_t pos = lo + k;
  buf[t] = pos < n ? xs[(int64_t)i * n + pos] : 0.f;
}
__global__ void k_unpack(const float* __restrict__ g, int64_t n, int d, int32_t ranks, int64_t cnt,
                         float* __restrict__ xs) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= (int64_t)ranks * d * cnt) return;
  int64_t per_rank = (int64_t)d * cnt;
  int64_t r = t / per_rank;
  int64_t rem = t - r * per_rank;
  int i = (int)(rem / cnt);
  int64_t k = rem - (int64_t)i * cnt;
  int64_t pos = r * cnt + k;
  if (pos < n) xs[(int64_t)i * n + pos] = g[t];
}

// Block-interleaved ownership: rank r of R owns the update blocks b (B points each) with
// b % R == r; its send buffer is [d][cnt], cnt = ceil(nblocks / R) * B (zero padded).
__global__ void k_pack_owned(const float* __restrict__ xs, int64_t n, int d, int64_t B, int32_t r, int32_t R,
                             int64_t cnt, float* __restrict__ buf) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= cnt * d) return;
  const int i = (int)(t / cnt);
  const int64_t k = t - (int64_t)i * cnt;
  const int64_t pos = ((k / B) * R + r) * B + (k % B);
  buf[t] = pos < n ? xs[(int64_t)i * n + pos] : 0.f;
}
__global__ void k_unpack_owned(const float* __restrict__ g, int64_t n, int d, int64_t B, int32_t R, int64_t cnt,
                               float* __restrict__ xs) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= (int64_t)R * d * cnt) return;
  const int64_t per_rank = (int64_t)d * cnt;
  const int32_t r = (int32_t)(t / per_rank);
  const int64_t rem = t - r * per_rank;
  const int i = (int)(rem / cnt);
  const int64_t k = rem - (int64_t)i * cnt;
  const int64_t pos = ((k / B) * R + r) * B + (k % B);
  if (pos < n) xs[(int64_t)i * n + pos] = g[t];
}

static int64_t owned_block_points(const Workspace&) { return kOwnBlock; }
static int64_t owned_count(const Workspace& ws, int32_t R) {
  const int64_t B = owned_block_points(ws);
  const int64_t nb = (ws.n + B - 1) / B;
  return (nb + R - 1) / R * B;
}

static int read_flags(Workspace& ws, int32_t* f1, int32_t* f2, int32_t* err) {
  EGG_CUDA(cudaMemcpyAsync(ws.h_flags, ws.flags, 4 * sizeof(int32_t), cudaMemcpyDeviceToHost, ws.stream));
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  if (f1) *f1 = ws.h_flags[0];
  if (f2) *f2 = ws.h_flags[1];
  if (err) *err = ws.h_flags[3];
  if (ws.h_flags[3]) {
    set_error("traversal stack overflow (internal error)");
    return EGGSYNC_ECUDA;
  }
  return EGGSYNC_OK;
}

static double ev_ms(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0.f;
  cudaEventElapsedTime(&ms, a, b);
  return ms * 1e-3;
}

// One pass of Alg 4's loop body: build, update, first term, (second term).
// Returns synced through *synced; labels of the verified state into lab (device) when synced.
static int iterate(Workspace& ws, int32_t* synced, int32_t* f1o, int32_t* f2o, int32_t* nbr_sorted,
                   eggsync_stats* stats) {
  if (stats) EGG_CUDA(cudaEventRecord(ws.ev[0], ws.stream));
  if (!ws.built) EGG_TRY(stage_build(ws));
  if (stats) EGG_CUDA(cudaEventRecord(ws.ev[1], ws.stream));
  k_set_flags<<<1, 1, 0, ws.stream>>>(ws.flags, 1, 1);
  ws.launches++;
  EGG_CUDA(cudaGetLastError());
  EGG_TRY(stage_update(ws, 0, ws.n, nbr_sorted));
  if (stats) EGG_CUDA(cudaEventRecord(ws.ev[2], ws.stream));
  int32_t f1 = 0, f2 = -1, err = 0;
  EGG_TRY(read_flags(ws, &f1, nullptr, &err));
  if (stats) {
    stats->t_build += ev_ms(ws.ev[0], ws.ev[1]);
    stats->t_update += ev_ms(ws.ev[1], ws.ev[2]);
  }
  if (f1) {
    if (stats) EGG_CUDA(cudaEventRecord(ws.ev[3], ws.stream));
    EGG_TRY(stage_second_term(ws, 0, ws.n));
    if (stats) EGG_CUDA(cudaEventRecord(ws.ev[4], ws.stream));
    EGG_TRY(read_flags(ws, nullptr, &f2, &err));
    if (stats) stats->t_extra_check += ev_ms(ws.ev[3], ws.ev[4]);
  }
  *synced = (f1 && f2 == 1) ? 1 : 0;
  if (f1o) *f1o = f1;
  if (f2o) *f2o = f1 ? f2 : -1;
  return EGGSYNC_OK;
}

static void advance(Workspace& ws) {
  ws.xcur ^= 1;
  ws.built = false;
}

// Algorithm 4: iterate until the criterion holds on the state the update read
// (reading R6/R7), labels = cells of that state (gatherCluster, L256).
static int run_loop(Workspace& ws, int32_t max_iters, int32_t* iters_out, eggsync_stats* stats) {
  int32_t t = 0, synced = 0;
  ws.have_final = false;
  for (;;) {
    EGG_TRY(iterate(ws, &synced, nullptr, nullptr, nullptr, stats));
    if (stats) {
      if (t == 0) stats->n_cells_first = ws.n_grid;
      stats->n_cells_last = ws.n_grid;
    }
    if (synced) {
      if (stats) EGG_CUDA(cudaEventRecord(ws.ev[5], ws.stream));
      EGG_TRY(stage_labels(ws, ws.lab_final));
      if (stats) EGG_CUDA(cudaEventRecord(ws.ev[6], ws.stream));
      ws.have_final = true;
    }
    advance(ws);
    ++t;
    if (synced || t >= max_iters) break;
  }
  if (!synced) {
    EGG_TRY(stage_build(ws));
    EGG_TRY(stage_labels(ws, ws.lab_final));
    ws.have_final = true;
  }
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  if (stats && synced) stats->t_cluster += ev_ms(ws.ev[5], ws.ev[6]);
  if (stats) {
    stats->iters = t;
    stats->sort_skipped = ws.sort_skipped;
  }
  *iters_out = t;
  return synced ? EGGSYNC_OK : EGGSYNC_NOT_CONVERGED;
}

// Algorithm 4 with Def 4.2 literally (term_mode = EGGSYNC_TERM_DEF42, F3): the same grid
// update; term (i), MBR(N_{eps/2}) and term (ii) on the grid structure of D^t (def42_grid.cu);
// labels = eps-graph components of the returned state (as the oracle's DEF42 mode).
static int run_loop_def42(Workspace& ws, int32_t max_iters, int32_t* iters_out) {
  struct Scratch {
    void* p = nullptr;
    ~Scratch() {
      if (p) cudaFree(p);
    }
  } sc;
  const size_t fb = sizeof(float) * (size_t)ws.n * ws.d;
  EGG_CUDA(cudaMalloc(&sc.p, 2 * fb + 4 * sizeof(int32_t) * (size_t)ws.n));
  float* mlo = reinterpret_cast<float*>(sc.p);
  float* mhi = mlo + (size_t)ws.n * ws.d;
  int32_t* lab_scratch = reinterpret_cast<int32_t*>(mhi + (size_t)ws.n * ws.d);
  int32_t t = 0, synced = 0;
  ws.have_final = false;
  for (;;) {
    if (!ws.built) EGG_TRY(stage_build(ws));
    k_set_flags<<<1, 1, 0, ws.stream>>>(ws.flags, 1, 1);
    EGG_CUDA(cudaGetLastError());
    EGG_TRY(stage_update(ws, 0, ws.n, nullptr));
    k_set_flags<<<1, 1, 0, ws.stream>>>(ws.flags, 1, 1);  // the update's grid first term is not used
    EGG_CUDA(cudaGetLastError());
    ws.launches += 2;
    EGG_TRY(def42_grid_first(ws));
    int32_t f1 = 0, f2 = 0;
    EGG_TRY(read_flags(ws, &f1, nullptr, nullptr));
    if (f1) {
      EGG_TRY(def42_grid_second(ws, mlo, mhi));
      EGG_TRY(read_flags(ws, nullptr, &f2, nullptr));
    }
    synced = f1 && f2;
    advance(ws);
    ++t;
    if (synced || t >= max_iters) break;
  }
  EGG_TRY(stage_build(ws));  // the returned state D^t
  EGG_TRY(def42_grid_labels(ws, lab_scratch, ws.lab_final));
  ws.have_final = true;
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  *iters_out = t;
  return synced ? EGGSYNC_OK : EGGSYNC_NOT_CONVERGED;
}

struct DeviceGuard {
  int prev = -1;
  bool changed = false;
  int set(int dev) {
    if (dev < 0) return EGGSYNC_OK;
    EGG_CUDA(cudaGetDevice(&prev));
    if (prev != dev) {
      EGG_CUDA(cudaSetDevice(dev));
      changed = true;
    }
    return EGGSYNC_OK;
  }
  ~DeviceGuard() {
    if (changed) cudaSetDevice(prev);
  }
};

static int validate(const void* points, int64_t n, int32_t d, float eps) {
  if (!points) {
    set_error("points is NULL");
    return EGGSYNC_EINVAL;
  }
  if (n < 1 || n > INT32_MAX) {
    set_error("n=%lld out of range [1, 2^31-1]", (long long)n);
    return EGGSYNC_EINVAL;
  }
  if (d < 1 || d > EGGSYNC_MAX_D) {
    set_error("d=%d out of range [1, %d]", d, EGGSYNC_MAX_D);
    return EGGSYNC_EINVAL;
  }
  Consts c;
  std::string why;
  if (!make_consts(n, d, eps, &c, &why)) {
    set_error("%s", why.c_str());
    return EGGSYNC_EINVAL;
  }
  return EGGSYNC_OK;
}

static int check_device() {
  int cnt = 0;
  cudaError_t e = cudaGetDeviceCount(&cnt);
  if (e != cudaSuccess || cnt < 1) {
    cudaGetLastError();
    set_error("no CUDA device available (%s); there is no CPU fallback",
              e != cudaSuccess ? cudaGetErrorString(e) : "0 devices");
    return EGGSYNC_ECUDA;
  }
  return EGGSYNC_OK;
}

}  // namespace egg

using namespace egg;

struct eggsync_ctx {
  Workspace ws;
};

// every context entry point runs on the context's device and restores the caller's
#define CTX_DEVICE(ctx)  \
  DeviceGuard _ctx_dg; \
  EGG_TRY(_ctx_dg.set((ctx)->ws.cur_device))

extern "C" {

const char* eggsync_last_error(void) { return g_err.c_str(); }
const char* eggsync_version(void) { return "eggsync-b200 0.1 (sm_100a)"; }

static void small_release();  // the one-launch path's scratch (below)
void eggsync_release_cache(void) {
  cache_clear();
  small_release();
}

void eggsync_default_opts(eggsync_opts* o) {
  if (!o) return;
  memset(o, 0, sizeof *o);
  o->struct_size = (int32_t)sizeof(eggsync_opts);
  o->max_iters = 10000;
  o->device = -1;
  o->term_mode = EGGSYNC_TERM_GRID;
  o->cw_factor = 1.0;
}

static int get_opts(const eggsync_opts* in, eggsync_opts* o) {
  eggsync_default_opts(o);
  if (!in) return EGGSYNC_OK;
  if (in->struct_size != (int32_t)sizeof(eggsync_opts)) {
    set_error("eggsync_opts.struct_size mismatch (%d != %d)", in->struct_size, (int)sizeof(eggsync_opts));
    return EGGSYNC_EINVAL;
  }
  *o = *in;
  if (o->max_iters < 1) {
    set_error("max_iters must be >= 1");
    return EGGSYNC_EINVAL;
  }
  if (!(o->cw_factor > 0.0 && o->cw_factor <= 1.0)) {
    set_error("cw_factor=%g must be in (0, 1] (c_w <= eps/(2 sqrt d), L252)", o->cw_factor);
    return EGGSYNC_EINVAL;
  }
  if (o->term_mode != EGGSYNC_TERM_GRID && o->term_mode != EGGSYNC_TERM_DEF42 &&
      o->term_mode != EGGSYNC_TERM_DEF42_DIRECT) {
    set_error("term_mode %d unknown (EGGSYNC_TERM_GRID, _DEF42 or _DEF42_DIRECT)", o->term_mode);
    return EGGSYNC_EINVAL;
  }
  return EGGSYNC_OK;
}

// ------------------------------------------------------------------ small inputs (F1)
// Scratch of the one-launch path, cached per device (grow-only): input, labels, coordinates,
// [iterations, converged] -- so that a small clustering costs one H2D, one launch, one D2H.
struct SmallScratch {
  int device = -1;
  char* dev = nullptr;
  size_t bytes = 0;
  char* host = nullptr;  // pinned mirror of the outputs
  size_t hbytes = 0;
};
static std::mutex g_small_mu;
static std::vector<SmallScratch> g_small;

static void small_release() {
  std::lock_guard<std::mutex> lk(g_small_mu);
  for (auto& c : g_small) {
    cudaSetDevice(c.device);
    if (c.dev) cudaFree(c.dev);
    if (c.host) cudaFreeHost(c.host);
  }
  g_small.clear();
}

static int small_path(const float* points, int64_t n, int32_t d, const Consts& k, const eggsync_opts& o,
                      int32_t* labels_out, int32_t* iters_out, int* rc_out) {
  int dev = 0;
  EGG_CUDA(cudaGetDevice(&dev));
  const size_t nx = (size_t)n * d * sizeof(float), nl = (size_t)n * sizeof(int32_t);
  const size_t need = 2 * nx + nl + 64;
  std::lock_guard<std::mutex> lk(g_small_mu);
  SmallScratch* sc = nullptr;
  for (auto& c : g_small)
    if (c.device == dev) sc = &c;
  if (!sc) {
    g_small.push_back(SmallScratch{});
    sc = &g_small.back();
    sc->device = dev;
  }
  if (sc->bytes < need) {
    if (sc->dev) cudaFree(sc->dev);
    sc->bytes = 0;
    EGG_CUDA(cudaMalloc((void**)&sc->dev, need));
    sc->bytes = need;
  }
  if (sc->hbytes < need) {
    if (sc->host) cudaFreeHost(sc->host);
    sc->hbytes = 0;
    EGG_CUDA(cudaMallocHost((void**)&sc->host, need));
    sc->hbytes = need;
  }
  cudaStream_t st = (cudaStream_t)o.stream;
  float* x = reinterpret_cast<float*>(sc->dev);
  float* co = reinterpret_cast<float*>(sc->dev + nx);
  int32_t* lab = reinterpret_cast<int32_t*>(sc->dev + 2 * nx);
  int32_t* out = reinterpret_cast<int32_t*>(sc->dev + 2 * nx + nl);
  const float* src = points;
  if (!o.device_pointers) {
    EGG_CUDA(cudaMemcpyAsync(x, points, nx, cudaMemcpyHostToDevice, st));
    src = x;
  }
  EGG_TRY(small_cluster(src, n, d, k, o.max_iters, o.device_pointers ? labels_out : lab,
                        o.device_pointers && o.coords_out ? o.coords_out : co, out, st));
  EGG_CUDA(cudaGetLastError());
  int32_t* hout = reinterpret_cast<int32_t*>(sc->host);
  EGG_CUDA(cudaMemcpyAsync(hout, out, 2 * sizeof(int32_t), cudaMemcpyDeviceToHost, st));
  if (!o.device_pointers) {
    EGG_CUDA(cudaMemcpyAsync(labels_out, lab, nl, cudaMemcpyDeviceToHost, st));
    if (o.coords_out) EGG_CUDA(cudaMemcpyAsync(o.coords_out, co, nx, cudaMemcpyDeviceToHost, st));
  }
  EGG_CUDA(cudaStreamSynchronize(st));
  *iters_out = hout[0];
  *rc_out = hout[1] ? EGGSYNC_OK : EGGSYNC_NOT_CONVERGED;
  return EGGSYNC_OK;
}

int eggsync_cluster_ex(const float* points, int64_t n, int32_t d, float eps, const eggsync_opts* opts,
                       int32_t* labels_out, int32_t* iters_out) {
  eggsync_opts o;
  EGG_TRY(get_opts(opts, &o));
  EGG_TRY(validate(points, n, d, eps));
  if (!labels_out || !iters_out) {
    set_error("labels_out / iters_out is NULL");
    return EGGSYNC_EINVAL;
  }
  EGG_TRY(check_device());
  DeviceGuard g;
  EGG_TRY(g.set(o.device));
  if (o.term_mode == EGGSYNC_TERM_DEF42_DIRECT) return def42_cluster(points, n, d, eps, o, labels_out, iters_out);
  if (o.term_mode == EGGSYNC_TERM_GRID) {
    // F1: small inputs run Algorithm 4 in one kernel launch (no per-iteration host round trip);
    // validation of the domain happens inside (a point outside [0,1] is rejected below first)
    Consts kc;
    std::string why;
    if (!o.stats && make_consts(n, d, eps, &kc, &why, o.cw_factor) && small_eligible(n, d, kc)) {
      if (!o.device_pointers) {  // EDOMAIN before any output is written (host input)
        for (int64_t t = 0; t < n * d; ++t)
          if (!(points[t] >= 0.f && points[t] <= 1.f)) {
            set_error("a coordinate is NaN/Inf or outside [0,1] (PAPER.md L70: data must be normalised)");
            return EGGSYNC_EDOMAIN;
          }
        int rc = EGGSYNC_OK;
        EGG_TRY(small_path(points, n, d, kc, o, labels_out, iters_out, &rc));
        return rc;
      }
    }
  }
  eggsync_stats local{};
  eggsync_stats* stats = o.stats ? &local : nullptr;
  auto t0 = std::chrono::steady_clock::now();
  Workspace ws;
  EGG_TRY(ws.alloc(n, d, eps, o.device, (cudaStream_t)o.stream, o.cw_factor));
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  auto t1 = std::chrono::steady_clock::now();
  if (stats) stats->t_alloc = std::chrono::duration<double>(t1 - t0).count();
  EGG_TRY(stage_ingest(ws, points, o.device_pointers != 0));
  auto t2 = std::chrono::steady_clock::now();
  int32_t iters = 0;
  int rc = o.term_mode == EGGSYNC_TERM_DEF42 ? run_loop_def42(ws, o.max_iters, &iters)
                                              : run_loop(ws, o.max_iters, &iters, stats);
  if (rc < 0) return rc;
  // outputs
  auto t3 = std::chrono::steady_clock::now();
  if (o.device_pointers) {
    EGG_CUDA(cudaMemcpyAsync(labels_out, ws.lab_final, sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, ws.stream));
    if (o.coords_out) EGG_TRY(stage_coords(ws, ws.xcur, o.coords_out));
  } else {
    EGG_CUDA(cudaMemcpyAsync(labels_out, ws.lab_final, sizeof(int32_t) * n, cudaMemcpyDeviceToHost, ws.stream));
    if (o.coords_out) {
      EGG_TRY(stage_coords(ws, ws.xcur, ws.io));
      EGG_CUDA(cudaMemcpyAsync(o.coords_out, ws.io, sizeof(float) * n * d, cudaMemcpyDeviceToHost, ws.stream));
    }
  }
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  auto t4 = std::chrono::steady_clock::now();
  *iters_out = iters;
  if (stats) {
    local.t_transfer = std::chrono::duration<double>(t2 - t1).count() +
                       std::chrono::duration<double>(t4 - t3).count();
    local.device_bytes = ws.bytes;
    ws.release();
    local.t_free = std::chrono::duration<double>(std::chrono::steady_clock::now() - t4).count();
    *o.stats = local;
  }
  return rc;
}

int eggsync_cluster(const float* points, int64_t n, int32_t d, float eps, int32_t* labels_out,
                    int32_t* iters_out) {
  return eggsync_cluster_ex(points, n, d, eps, nullptr, labels_out, iters_out);
}

int eggsync_step_ex(float* points, int64_t n, int32_t d, float eps, const eggsync_opts* opts,
                    int32_t* first_term_out, int32_t* second_term_out) {
  eggsync_opts o;
  EGG_TRY(get_opts(opts, &o));
  if (o.term_mode != EGGSYNC_TERM_GRID) {
    set_error("eggsync_step_ex evaluates the grid criterion only (term_mode must be EGGSYNC_TERM_GRID)");
    return EGGSYNC_EINVAL;
  }
  EGG_TRY(validate(points, n, d, eps));
  EGG_TRY(check_device());
  DeviceGuard g;
  EGG_TRY(g.set(o.device));
  Workspace ws;
  EGG_TRY(ws.alloc(n, d, eps, o.device, (cudaStream_t)o.stream, o.cw_factor));
  EGG_TRY(stage_ingest(ws, points, o.device_pointers != 0));
  int32_t synced = 0, f1 = 0, f2 = -1;
  EGG_TRY(iterate(ws, &synced, &f1, &f2, o.nbr_count_out ? ws.nbr : nullptr, nullptr));
  // nbr counts refer to D^t's sorted order -> original order
  if (o.nbr_count_out) {
    EGG_TRY(stage_scatter_i32(ws, ws.nbr, ws.i_lab));
    EGG_CUDA(cudaMemcpyAsync(o.nbr_count_out, ws.i_lab, sizeof(int32_t) * n,
                             o.device_pointers ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, ws.stream));
  }
  advance(ws);
  if (o.device_pointers) {
    EGG_TRY(stage_coords(ws, ws.xcur, points));
  } else {
    EGG_TRY(stage_coords(ws, ws.xcur, ws.io));
    EGG_CUDA(cudaMemcpyAsync(points, ws.io, sizeof(float) * n * d, cudaMemcpyDeviceToHost, ws.stream));
  }
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  if (first_term_out) *first_term_out = f1;
  if (second_term_out) *second_term_out = f2;
  return EGGSYNC_OK;
}

int eggsync_step(float* points, int64_t n, int32_t d, float eps, int32_t* synced_out) {
  int32_t f1 = 0, f2 = -1;
  int rc = eggsync_step_ex(points, n, d, eps, nullptr, &f1, &f2);
  if (rc == EGGSYNC_OK && synced_out) *synced_out = (f1 && f2 == 1) ? 1 : 0;
  return rc;
}

// ------------------------------------------------------------------ context
int eggsync_ctx_create(int64_t n, int32_t d, float eps, int32_t device, void* stream, eggsync_ctx** out) {
  if (!out) {
    set_error("out is NULL");
    return EGGSYNC_EINVAL;
  }
  static const float dummy = 0.f;
  EGG_TRY(validate(&dummy, n, d, eps));
  EGG_TRY(check_device());
  DeviceGuard g;  // the caller's current device is restored on return
  EGG_TRY(g.set(device));
  eggsync_ctx* c = new eggsync_ctx();
  int rc = c->ws.alloc(n, d, eps, device, (cudaStream_t)stream);
  if (rc != EGGSYNC_OK) {
    delete c;
    return rc;
  }
  *out = c;
  return EGGSYNC_OK;
}

void eggsync_ctx_destroy(eggsync_ctx* ctx) {
  if (!ctx) return;
  DeviceGuard g;
  g.set(ctx->ws.cur_device);
  delete ctx;
}

int eggsync_ctx_load(eggsync_ctx* ctx, const float* points, int32_t on_device) {
  if (!ctx || !points) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  return stage_ingest(ctx->ws, points, on_device != 0);
}

int eggsync_ctx_build(eggsync_ctx* ctx, int32_t* n_cells_out) {
  if (!ctx) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  EGG_TRY(stage_build(ws));
  k_set_flags<<<1, 1, 0, ws.stream>>>(ws.flags, 1, 1);
  ws.launches++;
  EGG_CUDA(cudaGetLastError());
  ws.second_checked = false;
  if (n_cells_out) *n_cells_out = ws.n_grid;
  return EGGSYNC_OK;
}

int eggsync_ctx_update(eggsync_ctx* ctx, int64_t lo, int64_t hi) {
  if (!ctx || lo < 0 || hi > ctx->ws.n || lo > hi) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  if (!ctx->ws.built) {
    set_error("eggsync_ctx_update before eggsync_ctx_build");
    return EGGSYNC_EINVAL;
  }
  return stage_update(ctx->ws, lo, hi, nullptr);
}

int eggsync_ctx_second_term(eggsync_ctx* ctx, int64_t lo, int64_t hi) {
  if (!ctx || lo < 0 || hi > ctx->ws.n || lo > hi) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  if (!ctx->ws.built) return EGGSYNC_EINVAL;
  ctx->ws.second_checked = true;
  return stage_second_term(ctx->ws, lo, hi);
}

int eggsync_ctx_flags(eggsync_ctx* ctx, int32_t* first_out, int32_t* second_out) {
  if (!ctx) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  int32_t f1 = 0, f2 = 0;
  EGG_TRY(read_flags(ctx->ws, &f1, &f2, nullptr));
  if (first_out) *first_out = f1;
  if (second_out) *second_out = ctx->ws.second_checked ? f2 : -1;
  return EGGSYNC_OK;
}

float* eggsync_ctx_cur_coords(eggsync_ctx* ctx) { return ctx ? ctx->ws.xs[ctx->ws.xcur] : nullptr; }
float* eggsync_ctx_next_coords(eggsync_ctx* ctx) { return ctx ? ctx->ws.xs[ctx->ws.xcur ^ 1] : nullptr; }

int eggsync_ctx_pack(eggsync_ctx* ctx, int64_t lo, int64_t cnt, float* buf) {
  if (!ctx || !buf || lo < 0 || cnt < 0) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  const int64_t tot = cnt * ws.d;
  if (tot == 0) return EGGSYNC_OK;
  k_pack<<<(unsigned)((tot + 255) / 256), 256, 0, ws.stream>>>(ws.xs[ws.xcur ^ 1], ws.n, ws.d, lo, cnt, buf);
  ws.launches++;
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

int eggsync_ctx_unpack(eggsync_ctx* ctx, const float* gathered, int32_t ranks, int64_t cnt) {
  if (!ctx || !gathered || ranks < 1 || cnt < 0) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  const int64_t tot = (int64_t)ranks * ws.d * cnt;
  if (tot == 0) return EGGSYNC_OK;
  k_unpack<<<(unsigned)((tot + 255) / 256), 256, 0, ws.stream>>>(gathered, ws.n, ws.d, ranks, cnt,
                                                                  ws.xs[ws.xcur ^ 1]);
  ws.launches++;
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

int eggsync_ctx_advance(eggsync_ctx* ctx) {
  if (!ctx) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  advance(ctx->ws);
  ctx->ws.have_final = false;
  return EGGSYNC_OK;
}

int eggsync_ctx_labels(eggsync_ctx* ctx, int32_t* labels, int32_t on_device) {
  if (!ctx || !labels) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  const int32_t* src = ws.lab_final;
  if (!ws.have_final) {
    if (!ws.built) EGG_TRY(stage_build(ws));
    EGG_TRY(stage_labels(ws, ws.i_lab));
    src = ws.i_lab;
  }
  EGG_CUDA(cudaMemcpyAsync(labels, src, sizeof(int32_t) * ws.n,
                           on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, ws.stream));
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  return EGGSYNC_OK;
}

int eggsync_ctx_coords(eggsync_ctx* ctx, float* coords, int32_t on_device) {
  if (!ctx || !coords) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  if (on_device) {
    EGG_TRY(stage_coords(ws, ws.xcur, coords));
  } else {
    EGG_TRY(stage_coords(ws, ws.xcur, ws.io));
    EGG_CUDA(cudaMemcpyAsync(coords, ws.io, sizeof(float) * ws.n * ws.d, cudaMemcpyDeviceToHost, ws.stream));
  }
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  return EGGSYNC_OK;
}

int eggsync_ctx_run(eggsync_ctx* ctx, int32_t max_iters, int32_t* iters_out) {
  if (!ctx || !iters_out || max_iters < 1) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  return run_loop(ctx->ws, max_iters, iters_out, nullptr);
}

void* eggsync_ctx_stream(eggsync_ctx* ctx) { return ctx ? (void*)ctx->ws.stream : nullptr; }

int eggsync_ctx_work(eggsync_ctx* ctx, int32_t enable, int64_t* totals_out) {
  if (!ctx) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  if (totals_out) {
    EGG_CUDA(cudaMemcpyAsync(totals_out, ws.work, 8 * sizeof(int64_t), cudaMemcpyDeviceToHost, ws.stream));
    EGG_CUDA(cudaStreamSynchronize(ws.stream));
  }
  if (enable == 1) {
    EGG_CUDA(cudaMemsetAsync(ws.work, 0, 8 * sizeof(int64_t), ws.stream));
    ws.count_work = true;
  } else if (enable == 0) {
    ws.count_work = false;
  }
  return EGGSYNC_OK;
}

int64_t eggsync_ctx_launches(eggsync_ctx* ctx) { return ctx ? ctx->ws.launches : -1; }

namespace egg {
int Workspace::tc_flush() {
  if (!tc_pending) return EGGSYNC_OK;
  EGG_CUDA(cudaEventSynchronize(tc_ev[1]));
  float ms = 0.f;
  EGG_CUDA(cudaEventElapsedTime(&ms, tc_ev[0], tc_ev[1]));
  tc_acc[4] += (long long)((double)ms * 1e6);
  tc_pending = false;
  return EGGSYNC_OK;
}
}  // namespace egg

int eggsync_ctx_tc_work(eggsync_ctx* ctx, int32_t enable, int64_t* out) {
  if (!ctx) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  EGG_TRY(ws.tc_flush());
  if (out)
    for (int k = 0; k < 5; ++k) out[k] = ws.tc_acc[k];
  if (enable == 1) {
    if (!ws.tc_ev[0]) {
      EGG_CUDA(cudaEventCreate(&ws.tc_ev[0]));
      EGG_CUDA(cudaEventCreate(&ws.tc_ev[1]));
    }
    for (int k = 0; k < 5; ++k) ws.tc_acc[k] = 0;
    ws.tc_timing = true;
  } else if (enable == 0) {
    ws.tc_timing = false;
  }
  return EGGSYNC_OK;
}

int eggsync_ctx_update_owned(eggsync_ctx* ctx, int32_t rank, int32_t ranks) {
  if (!ctx || ranks < 1 || rank < 0 || rank >= ranks) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  if (!ctx->ws.built) {
    set_error("eggsync_ctx_update_owned before eggsync_ctx_build");
    return EGGSYNC_EINVAL;
  }
  ctx->ws.own_stride = ranks;
  ctx->ws.own_offset = rank;
  const int rc = stage_update(ctx->ws, 0, ctx->ws.n, nullptr);
  ctx->ws.own_stride = 1;
  ctx->ws.own_offset = 0;
  return rc;
}

int eggsync_ctx_plan_owned(eggsync_ctx* ctx, int32_t rank, int32_t ranks, int64_t* stats_out) {
  if (!ctx || !stats_out || ranks < 1 || rank < 0 || rank >= ranks) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  if (!ws.built) {
    set_error("eggsync_ctx_plan_owned before eggsync_ctx_build");
    return EGGSYNC_EINVAL;
  }
  ws.own_stride = ranks;
  ws.own_offset = rank;
  ws.tc_mode = 1;
  const int rc = stage_update(ws, 0, ws.n, nullptr);
  ws.tc_mode = 0;
  ws.own_stride = 1;
  ws.own_offset = 0;
  if (rc != EGGSYNC_OK) return rc;
  for (int k = 0; k < 6; ++k) stats_out[k] = ws.tc_local[k];
  return EGGSYNC_OK;
}

int eggsync_ctx_update_planned(eggsync_ctx* ctx, int32_t rank, int32_t ranks, const int64_t* global_stats) {
  if (!ctx || !global_stats || ranks < 1 || rank < 0 || rank >= ranks) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  if (!ws.built) {
    set_error("eggsync_ctx_update_planned before eggsync_ctx_build");
    return EGGSYNC_EINVAL;
  }
  for (int k = 0; k < 6; ++k) ws.tc_global[k] = global_stats[k];
  ws.own_stride = ranks;
  ws.own_offset = rank;
  ws.tc_mode = 2;
  const int rc = stage_update(ws, 0, ws.n, nullptr);
  ws.tc_mode = 0;
  ws.own_stride = 1;
  ws.own_offset = 0;
  return rc;
}

int eggsync_ctx_set_own(eggsync_ctx* ctx, int64_t n_own) {
  if (!ctx || n_own < 0) return EGGSYNC_EINVAL;
  ctx->ws.n_own = n_own >= ctx->ws.n ? INT64_MAX : n_own;
  return EGGSYNC_OK;
}

int64_t eggsync_ctx_owned_count(eggsync_ctx* ctx, int32_t ranks) {
  if (!ctx || ranks < 1) return -1;
  return owned_count(ctx->ws, ranks);
}

int eggsync_ctx_pack_owned(eggsync_ctx* ctx, int32_t rank, int32_t ranks, float* buf) {
  if (!ctx || !buf || ranks < 1 || rank < 0 || rank >= ranks) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  const int64_t cnt = owned_count(ws, ranks), tot = cnt * ws.d;
  k_pack_owned<<<(unsigned)((tot + 255) / 256), 256, 0, ws.stream>>>(ws.xs[ws.xcur ^ 1], ws.n, ws.d,
                                                                      owned_block_points(ws), rank, ranks, cnt, buf);
  ws.launches++;
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

int eggsync_ctx_unpack_owned(eggsync_ctx* ctx, const float* gathered, int32_t ranks) {
  if (!ctx || !gathered || ranks < 1) return EGGSYNC_EINVAL;
  CTX_DEVICE(ctx);
  Workspace& ws = ctx->ws;
  const int64_t cnt = owned_count(ws, ranks), tot = (int64_t)ranks * ws.d * cnt;
  k_unpack_owned<<<(unsigned)((tot + 255) / 256), 256, 0, ws.stream>>>(gathered, ws.n, ws.d, owned_block_points(ws),
                                                                        ranks, cnt, ws.xs[ws.xcur ^ 1]);
  ws.launches++;
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}


}  // extern "C"
