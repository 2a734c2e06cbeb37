// sync_brute.cu -- direct SynC update (Eq.1) and cluster order parameter (Eq.2)
// on the GPU, GPU-SynC style (L284): every point against every point, no grid.
//
// an internal cross-check of the grid path (a second, independent
// GPU implementation of Eq.1) and its speed floor, plus SynC's lambda-termination
// (Algorithm 1, L46-56) for the Fig 1 failure case (L89, L95).
//
// Layout: points row-major [n][d] (the ABI layout; no transpose needed: a 128-point
// tile of q is one contiguous 128*d-float block, staged coalesced in shared memory and
// read by broadcast).  One thread per p; p's coordinates and fp64 sums live in registers.
// Bound: plain FP32 ALU (2d+1 instructions per pair + sinf/expf per neighbour pair).
#include <cmath>

#include "common.cuh"

namespace egg {
namespace {

constexpr int kSyncT = 128;  // threads per CTA = points per CTA = q-tile length

struct SyncArgs {
  const float* x;  // D^t [n][d]
  float* xn;       // D^{t+1} [n][d]
  int32_t* nbr;    // |N_eps(p)| or nullptr
  double* rcp;     // per-point inner mean of Eq.2
  int64_t n;
  float e2_lo, e2_hi;  // fp32 band around eps^2: below lo -> in, above hi -> out
  double e2;           // exact test (fp64 of the fp32 eps, squared)
  int32_t* f1_def;     // Def 4.2 term (i) flag (cleared on a pair eps/2 < ||p-q|| <= eps) or nullptr
  float e2h_lo, e2h_hi;
  double e2h;          // (eps/2)^2 = e2 / 4 (as the oracle)
  int64_t qchunk;      // q points per slice (blockIdx.y); slices > 1 write partial sums to part
  double* part;        // [slice][n][D+2]: sum sin, sum exp, count (nullptr when one slice)
};

// Exact fp64 squared distance: the oracle's predicate (R4), dimension order, no FMA.
template <int D>
__device__ __forceinline__ double exact_d2(const float* q, const float* x) {
  double dd = 0.0;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const double t = (double)q[i] - (double)x[i];
    dd = __dadd_rn(dd, __dmul_rn(t, t));
  }
  return dd;
}

template <int D>
__global__ void __launch_bounds__(kSyncT) k_sync_brute(SyncArgs a) {
  constexpr int DP = ceil4(D);  // tile rows padded to whole float4s (pads are 0 in q and p)
  __shared__ float4 tile4[kSyncT * DP / 4];
  __shared__ uint8_t hq[kSyncT * kSyncT];  // [slot k][thread]: neighbour queue of the current tile
  float* tile = reinterpret_cast<float*>(tile4);
  const int64_t p = (int64_t)blockIdx.x * kSyncT + threadIdx.x;
  const bool act = p < a.n;
  float x[DP];
#pragma unroll
  for (int i = 0; i < DP; ++i) x[i] = (act && i < D) ? a.x[p * D + i] : 0.f;
  double S[D];
#pragma unroll
  for (int i = 0; i < D; ++i) S[i] = 0.0;
  double R = 0.0;
  int32_t cnt = 0;
  const int64_t q0 = (int64_t)blockIdx.y * a.qchunk;
  const int64_t q1 = q0 + a.qchunk < a.n ? q0 + a.qchunk : a.n;
  for (int64_t t0 = q0; t0 < q1; t0 += kSyncT) {
    const int64_t rem = q1 - t0;
    const int m = rem < kSyncT ? (int)rem : kSyncT;
    __syncthreads();
    for (int k = threadIdx.x; k < m * D; k += kSyncT) tile[(k / D) * DP + (k % D)] = a.x[t0 * D + k];
    if constexpr (DP != D)
      for (int k = threadIdx.x; k < m * (DP - D); k += kSyncT) tile[(k / (DP - D)) * DP + D + k % (DP - D)] = 0.f;
    __syncthreads();
    // pass 1: the pair test (float4 shared loads, broadcast); each thread queues the tile
    // slots of its neighbours in ascending order
    int nh = 0;
    for (int j = 0; j < m; ++j) {
      const float4* q4 = tile4 + j * (DP / 4);
      float d2 = 0.f;
#pragma unroll
      for (int c = 0; c < DP / 4; ++c) {
        const float4 v = q4[c];
        float t = v.x - x[4 * c];
        d2 = fmaf(t, t, d2);
        t = v.y - x[4 * c + 1];
        d2 = fmaf(t, t, d2);
        t = v.z - x[4 * c + 2];
        d2 = fmaf(t, t, d2);
        t = v.w - x[4 * c + 3];
        d2 = fmaf(t, t, d2);
      }
      if (d2 > a.e2_hi) continue;
      const float* q = tile + j * DP;
      bool in = d2 <= a.e2_lo;
      if (!in) in = exact_d2<D>(q, x) <= a.e2;  // inside the band: the oracle's exact decision
      if (in) {
        hq[nh++ * kSyncT + threadIdx.x] = (uint8_t)j;
        if (a.f1_def && act && d2 > a.e2h_lo && (d2 > a.e2h_hi || exact_d2<D>(q, x) > a.e2h))
          *a.f1_def = 0;  // eps/2 < ||p - q|| <= eps: Def 4.2 term (i) fails (L108)
      }
    }
    // pass 2: q in N_eps(p): Eq.1 terms sin(q_i - p_i), Eq.2 term exp(-||q - p||).  The warp
    // runs max(nh) iterations over its lanes instead of one sinf branch per slot any lane hits.
    cnt += nh;
    float s[D];
#pragma unroll
    for (int i = 0; i < D; ++i) s[i] = 0.f;
    float r = 0.f;
    for (int k = 0; k < nh; ++k) {
      const float* q = tile + (int)hq[k * kSyncT + threadIdx.x] * DP;
      float d2 = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float t = q[i] - x[i];
        d2 = fmaf(t, t, d2);
        s[i] += sinf(t);
      }
      r += expf(-sqrtf(d2));
    }
#pragma unroll
    for (int i = 0; i < D; ++i) S[i] += (double)s[i];
    R += (double)r;
  }
  if (!act) return;
  if (a.part) {  // one slice of the q range: partial sums, combined in slice order by k_sync_reduce
    double* o = a.part + ((int64_t)blockIdx.y * a.n + p) * (D + 2);
#pragma unroll
    for (int i = 0; i < D; ++i) o[i] = S[i];
    o[D] = R;
    o[D + 1] = (double)cnt;
    return;
  }
  const double inv = 1.0 / (double)cnt;  // cnt >= 1: p in N_eps(p)
#pragma unroll
  for (int i = 0; i < D; ++i) a.xn[p * D + i] = (float)((double)x[i] + inv * S[i]);
  if (a.nbr) a.nbr[p] = cnt;
  a.rcp[p] = R * inv;
}

// Sum of the slices' partial sums in slice order (deterministic) + Eq.1 / Eq.2 epilogue.
template <int D>
__global__ void k_sync_reduce(SyncArgs a, int slices) {
  const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= a.n) return;
  double S[D + 2];
#pragma unroll
  for (int i = 0; i < D + 2; ++i) S[i] = 0.0;
  for (int sl = 0; sl < slices; ++sl) {
    const double* o = a.part + ((int64_t)sl * a.n + p) * (D + 2);
#pragma unroll
    for (int i = 0; i < D + 2; ++i) S[i] += o[i];
  }
  const int32_t cnt = (int32_t)S[D + 1];
  const double inv = 1.0 / (double)cnt;
#pragma unroll
  for (int i = 0; i < D; ++i) a.xn[p * D + i] = (float)((double)a.x[p * D + i] + inv * S[i]);
  if (a.nbr) a.nbr[p] = cnt;
  a.rcp[p] = S[D] * inv;
}

// Deterministic mean of the per-point inner means (one CTA, fixed order).
__global__ void __launch_bounds__(1024) k_mean(const double* __restrict__ v, int64_t n, double* __restrict__ out) {
  __shared__ double sh[1024];
  double s = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += 1024) s += v[i];
  sh[threadIdx.x] = s;
  __syncthreads();
  for (int w = 512; w > 0; w >>= 1) {
    if ((int)threadIdx.x < w) sh[threadIdx.x] += sh[threadIdx.x + w];
    __syncthreads();
  }
  if (threadIdx.x == 0) *out = sh[0] / (double)n;
}

// Slices of the q range: one thread per p gives only ceil(n/128) CTAs, too few to fill 148 SMs
// below n ~ 100k; split the q range so about 6 CTAs per SM run (each slice >= 1 tile).
int64_t sync_slices(int64_t n) {
  const int64_t nb = (n + kSyncT - 1) / kSyncT;
  int64_t sl = (148 * 6 + nb - 1) / nb;
  if (sl > nb) sl = nb;
  if (sl > 64) sl = 64;
  return sl < 1 ? 1 : sl;
}

template <int D>
int launch_sync(SyncArgs a, cudaStream_t st) {
  const int64_t blocks = (a.n + kSyncT - 1) / kSyncT;
  const int64_t sl = sync_slices(a.n);
  a.qchunk = ((a.n + sl - 1) / sl + kSyncT - 1) / kSyncT * kSyncT;
  const int64_t used = (a.n + a.qchunk - 1) / a.qchunk;
  a.part = nullptr;
  if (used > 1) EGG_CUDA(cudaMallocAsync(&a.part, sizeof(double) * used * a.n * (D + 2), st));
  k_sync_brute<D><<<dim3((unsigned)blocks, (unsigned)used), kSyncT, 0, st>>>(a);
  EGG_CUDA(cudaGetLastError());
  if (used > 1) {
    k_sync_reduce<D><<<(unsigned)((a.n + 255) / 256), 256, 0, st>>>(a, (int)used);
    EGG_CUDA(cudaGetLastError());
    EGG_CUDA(cudaFreeAsync(a.part, st));
  }
  return EGGSYNC_OK;
}

int check_args(const float* points, int64_t n, int32_t d, float eps) {
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
  if (!std::isfinite(eps) || eps <= 0.f) {
    set_error("eps=%g must be finite and > 0", (double)eps);
    return EGGSYNC_EINVAL;
  }
  int cnt = 0;
  cudaError_t e = cudaGetDeviceCount(&cnt);
  if (e != cudaSuccess || cnt < 1) {
    cudaGetLastError();
    set_error("no CUDA device available; there is no CPU fallback");
    return EGGSYNC_ECUDA;
  }
  return EGGSYNC_OK;
}

// Device state of a direct-SynC run: two coordinate buffers, per-point r_c terms, r_c.
struct SyncBufs {
  float* x[2] = {nullptr, nullptr};
  int32_t* nbr = nullptr;
  double* rcp = nullptr;
  double* rc = nullptr;
  ~SyncBufs() {
    cudaFree(x[0]);
    cudaFree(x[1]);
    cudaFree(nbr);
    cudaFree(rcp);
    cudaFree(rc);
  }
  int alloc(int64_t n, int d, bool want_nbr) {
    EGG_CUDA(cudaMalloc(&x[0], sizeof(float) * n * d));
    EGG_CUDA(cudaMalloc(&x[1], sizeof(float) * n * d));
    if (want_nbr) EGG_CUDA(cudaMalloc(&nbr, sizeof(int32_t) * n));
    EGG_CUDA(cudaMalloc(&rcp, sizeof(double) * n));
    EGG_CUDA(cudaMalloc(&rc, sizeof(double)));
    return EGGSYNC_OK;
  }
};

// One Alg 1 iteration on device buffers: xn = Eq.1(x), *rc_dev = Eq.2(x).
int sync_iter(const float* x, float* xn, int32_t* nbr, double* rcp, int64_t n, int d, float eps,
              int32_t* f1_def = nullptr, cudaStream_t st = 0) {
  const double e = (double)eps;
  const double e2 = e * e, e2h = e2 / 4.0;
  const float e2f = (float)e2, e2hf = (float)e2h;
  const float rel = (float)(4 * d + 16) * kU;
  SyncArgs a{x, xn, nbr, rcp, n, e2f * (1.f - rel), e2f * (1.f + rel), e2,
             f1_def, e2hf * (1.f - rel), e2hf * (1.f + rel), e2h, n, nullptr};
  EGG_DISPATCH(d, launch_sync, a, st);
}

int sync_run(const float* x, float* xn, int32_t* nbr, double* rcp, double* rc_dev, int64_t n, int d, float eps) {
  EGG_TRY(sync_iter(x, xn, nbr, rcp, n, d, eps));
  k_mean<<<1, 1024>>>(rcp, n, rc_dev);
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}


// ============================================================================
// term_mode = EGGSYNC_TERM_DEF42: Def 4.2 literally (L106-110) on the
// direct path -- term (i) "no pair with eps/2 < ||p-q|| <= eps" (flag of k_sync_brute),
// term (ii) with MBR(N_{eps/2}(q)) per point, labels = connected components of the eps-graph
// (Theorem 4.7: at the criterion they are the clusters).  O(n^2 d) per iteration.
// ============================================================================

// MBR(N_{eps/2}(q)) of every q: lo/hi [n][D] (min/max of fp32 coordinates: exact).
template <int D>
__global__ void __launch_bounds__(kSyncT) k_half_mbr(const float* __restrict__ X, int64_t n, float lo_f, float hi_f,
                                                     double e2h, float* __restrict__ lo, float* __restrict__ hi) {
  __shared__ float tile[kSyncT * D];
  const int64_t p = (int64_t)blockIdx.x * kSyncT + threadIdx.x;
  const bool act = p < n;
  float x[D], l[D], h[D];
#pragma unroll
  for (int i = 0; i < D; ++i) l[i] = h[i] = x[i] = act ? X[p * D + i] : 0.f;
  for (int64_t t0 = 0; t0 < n; t0 += kSyncT) {
    const int64_t rem = n - t0;
    const int m = rem < kSyncT ? (int)rem : kSyncT;
    __syncthreads();
    for (int k = threadIdx.x; k < m * D; k += kSyncT) tile[k] = X[t0 * D + k];
    __syncthreads();
    for (int j = 0; j < m; ++j) {
      const float* q = tile + j * D;
      float d2 = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float t = q[i] - x[i];
        d2 = fmaf(t, t, d2);
      }
      if (d2 > hi_f) continue;
      if (d2 > lo_f && exact_d2<D>(q, x) > e2h) continue;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        l[i] = fminf(l[i], q[i]);
        h[i] = fmaxf(h[i], q[i]);
      }
    }
  }
  if (!act) return;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    lo[p * D + i] = l[i];
    hi[p * D + i] = h[i];
  }
}

// Def 4.2 term (ii) (L108-110): clear *f2 if some p, q have eps < ||p-q|| <= eps+delta and
// dist(MBR(N_{eps/2}(q)), p) <= eps (per-dimension clamp distance, R10), all in fp64 as the oracle.
template <int D>
__global__ void __launch_bounds__(kSyncT) k_second_def(const float* __restrict__ X, int64_t n,
                                                       const float* __restrict__ lo, const float* __restrict__ hi,
                                                       float in_lo, float out_hi, double e2, double ed2,
                                                       int32_t* __restrict__ f2) {
  __shared__ float tile[kSyncT * D];
  const int64_t p = (int64_t)blockIdx.x * kSyncT + threadIdx.x;
  const bool act = p < n;
  float x[D];
#pragma unroll
  for (int i = 0; i < D; ++i) x[i] = act ? X[p * D + i] : 0.f;
  bool viol = false;
  for (int64_t t0 = 0; t0 < n; t0 += kSyncT) {
    const int64_t rem = n - t0;
    const int m = rem < kSyncT ? (int)rem : kSyncT;
    __syncthreads();
    for (int k = threadIdx.x; k < m * D; k += kSyncT) tile[k] = X[t0 * D + k];
    __syncthreads();
    if (!act || viol) continue;
    for (int j = 0; j < m; ++j) {
      const float* q = tile + j * D;
      float d2 = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float t = q[i] - x[i];
        d2 = fmaf(t, t, d2);
      }
      if (d2 < in_lo || d2 > out_hi) continue;  // surely inside eps or outside eps + delta
      const double dd = exact_d2<D>(q, x);
      if (!(dd > e2 && dd <= ed2)) continue;
      const int64_t qi = t0 + j;
      double mm = 0.0;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const double v = (double)x[i], L = (double)lo[qi * D + i], H = (double)hi[qi * D + i];
        double t = 0.0;
        if (v < L) t = __dsub_rn(L, v);
        else if (v > H) t = __dsub_rn(v, H);
        mm = __dadd_rn(mm, __dmul_rn(t, t));
      }
      if (mm <= e2) {
        viol = true;
        break;
      }
    }
  }
  if (viol) *f2 = 0;
}

// One min-label propagation round over the eps-graph: out[p] = min(in[p], in[q] : ||p-q|| <= eps).
template <int D>
__global__ void __launch_bounds__(kSyncT) k_cc_round(const float* __restrict__ X, int64_t n, float lo_f, float hi_f,
                                                     double e2, const int32_t* __restrict__ in,
                                                     int32_t* __restrict__ out, int32_t* __restrict__ changed) {
  __shared__ float tile[kSyncT * D];
  __shared__ int32_t tl[kSyncT];
  const int64_t p = (int64_t)blockIdx.x * kSyncT + threadIdx.x;
  const bool act = p < n;
  float x[D];
#pragma unroll
  for (int i = 0; i < D; ++i) x[i] = act ? X[p * D + i] : 0.f;
  int32_t m = act ? in[p] : 0;
  for (int64_t t0 = 0; t0 < n; t0 += kSyncT) {
    const int64_t rem = n - t0;
    const int mm = rem < kSyncT ? (int)rem : kSyncT;
    __syncthreads();
    for (int k = threadIdx.x; k < mm * D; k += kSyncT) tile[k] = X[t0 * D + k];
    if ((int)threadIdx.x < mm) tl[threadIdx.x] = in[t0 + threadIdx.x];
    __syncthreads();
    for (int j = 0; j < mm; ++j) {
      if (tl[j] >= m) continue;
      const float* q = tile + j * D;
      float d2 = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float t = q[i] - x[i];
        d2 = fmaf(t, t, d2);
      }
      if (d2 > hi_f) continue;
      if (d2 > lo_f && exact_d2<D>(q, x) > e2) continue;
      m = tl[j];
    }
  }
  if (!act) return;
  out[p] = m;
  if (m != in[p]) *changed = 1;
}

__global__ void k_jump(const int32_t* __restrict__ in, int64_t n, int32_t* __restrict__ out) {
  const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p < n) out[p] = in[in[p]];
}

// Canonical numbering (R14): component label = its smallest index m (lab[m] == m); ids are
// the ranks of those roots in index order.  One CTA: chunked counts, block scan, scatter.
__global__ void __launch_bounds__(1024) k_canon(const int32_t* __restrict__ lab, int64_t n, int32_t* __restrict__ ids,
                                                int32_t* __restrict__ labels) {
  __shared__ int32_t sc[1024];
  const int64_t chunk = (n + 1023) / 1024;
  const int64_t b = threadIdx.x * chunk, e = b + chunk < n ? b + chunk : n;
  int32_t c = 0;
  for (int64_t p = b; p < e; ++p) c += lab[p] == p;
  sc[threadIdx.x] = c;
  __syncthreads();
  for (int off = 1; off < 1024; off <<= 1) {
    const int32_t v = (int)threadIdx.x >= off ? sc[threadIdx.x - off] : 0;
    __syncthreads();
    sc[threadIdx.x] += v;
    __syncthreads();
  }
  int32_t id = sc[threadIdx.x] - c;
  for (int64_t p = b; p < e; ++p)
    if (lab[p] == p) ids[p] = id++;
  __syncthreads();
  for (int64_t p = threadIdx.x; p < n; p += 1024) labels[p] = ids[lab[p]];
}

__global__ void k_domain(const float* __restrict__ X, int64_t m, int32_t* __restrict__ bad) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k < m && !(X[k] >= 0.f && X[k] <= 1.f)) *bad = 1;  // NaN fails both comparisons
}
__global__ void k_iota(int32_t* __restrict__ v, int64_t n) {
  const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p < n) v[p] = (int32_t)p;
}

template <int D>
int launch_def42_second(const float* x, int64_t n, float eps, float* lo, float* hi, int32_t* f2, cudaStream_t st) {
  const double e = (double)eps, e2 = e * e, e2h = e2 / 4.0;
  const double delta = e - e * std::sqrt(15.0 / 16.0) + e / 2.0 - std::sin(e / 2.0);  // L110 (R11)
  const double ed2 = (e + delta) * (e + delta);
  const float rel = (float)(4 * D + 16) * kU;
  const unsigned blocks = (unsigned)((n + kSyncT - 1) / kSyncT);
  k_half_mbr<D><<<blocks, kSyncT, 0, st>>>(x, n, (float)e2h * (1.f - rel), (float)e2h * (1.f + rel), e2h, lo, hi);
  k_second_def<D><<<blocks, kSyncT, 0, st>>>(x, n, lo, hi, (float)e2 * (1.f - rel), (float)ed2 * (1.f + rel), e2, ed2,
                                             f2);
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

template <int D>
int launch_cc_round(const float* x, int64_t n, float eps, const int32_t* in, int32_t* out, int32_t* changed,
                    cudaStream_t st) {
  const double e = (double)eps, e2 = e * e;
  const float rel = (float)(4 * D + 16) * kU;
  const unsigned blocks = (unsigned)((n + kSyncT - 1) / kSyncT);
  k_cc_round<D><<<blocks, kSyncT, 0, st>>>(x, n, (float)e2 * (1.f - rel), (float)e2 * (1.f + rel), e2, in, out,
                                           changed);
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

int def42_second(const float* x, int64_t n, int d, float eps, float* lo, float* hi, int32_t* f2, cudaStream_t st) {
  EGG_DISPATCH(d, launch_def42_second, x, n, eps, lo, hi, f2, st);
}
int cc_round(const float* x, int64_t n, int d, float eps, const int32_t* in, int32_t* out, int32_t* changed,
             cudaStream_t st) {
  EGG_DISPATCH(d, launch_cc_round, x, n, eps, in, out, changed, st);
}

struct Def42Bufs {
  float* x[2] = {nullptr, nullptr};
  float *lo = nullptr, *hi = nullptr;
  int32_t *lab[2] = {nullptr, nullptr}, *ids = nullptr, *out = nullptr, *flags = nullptr;
  double* rcp = nullptr;
  ~Def42Bufs() {
    for (void* p : {(void*)x[0], (void*)x[1], (void*)lo, (void*)hi, (void*)lab[0], (void*)lab[1], (void*)ids,
                    (void*)out, (void*)flags, (void*)rcp})
      cudaFree(p);
  }
};

int set_flag(int32_t* f, int32_t v, cudaStream_t st) {
  EGG_CUDA(cudaMemsetAsync(f, 0, sizeof(int32_t), st));
  if (v) EGG_CUDA(cudaMemsetAsync(f, 1, 1, st));  // little-endian int32 1
  return EGGSYNC_OK;
}
int get_flag(const int32_t* f, int32_t* v, cudaStream_t st) {
  EGG_CUDA(cudaMemcpyAsync(v, f, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
  EGG_CUDA(cudaStreamSynchronize(st));
  return EGGSYNC_OK;
}

}  // namespace

// Algorithm 4 (R6/R7) with Def 4.2's literal first term; called by eggsync_cluster_ex for
// term_mode == EGGSYNC_TERM_DEF42 after argument validation.  Labels: eps-components of the
// returned state, canonical (as oracle_cluster's DEF42 mode).
int def42_cluster(const float* points, int64_t n, int d, float eps, const eggsync_opts& o, int32_t* labels_out,
                  int32_t* iters_out) {
  cudaStream_t st = (cudaStream_t)o.stream;
  const bool dev = o.device_pointers != 0;
  const size_t bytes = sizeof(float) * n * d;
  Def42Bufs b;
  EGG_CUDA(cudaMalloc(&b.x[0], bytes));
  EGG_CUDA(cudaMalloc(&b.x[1], bytes));
  EGG_CUDA(cudaMalloc(&b.lo, bytes));
  EGG_CUDA(cudaMalloc(&b.hi, bytes));
  for (int k = 0; k < 2; ++k) EGG_CUDA(cudaMalloc(&b.lab[k], sizeof(int32_t) * n));
  EGG_CUDA(cudaMalloc(&b.ids, sizeof(int32_t) * n));
  EGG_CUDA(cudaMalloc(&b.out, sizeof(int32_t) * n));
  EGG_CUDA(cudaMalloc(&b.flags, sizeof(int32_t) * 4));
  EGG_CUDA(cudaMalloc(&b.rcp, sizeof(double) * n));
  EGG_CUDA(cudaMemcpyAsync(b.x[0], points, bytes, dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, st));
  // domain (L70, L290): every coordinate finite and in [0,1]
  EGG_TRY(set_flag(b.flags + 3, 0, st));
  k_domain<<<(unsigned)((n * d + 255) / 256), 256, 0, st>>>(b.x[0], n * d, b.flags + 3);
  int32_t bad = 0;
  EGG_TRY(get_flag(b.flags + 3, &bad, st));
  if (bad) {
    set_error("a coordinate is NaN/Inf or outside [0,1]");
    return EGGSYNC_EDOMAIN;
  }
  int32_t t = 0, cur = 0, synced = 0;
  for (;;) {
    EGG_TRY(set_flag(b.flags, 1, st));
    EGG_TRY(sync_iter(b.x[cur], b.x[cur ^ 1], nullptr, b.rcp, n, d, eps, b.flags, st));
    int32_t f1 = 0, f2 = 0;
    EGG_TRY(get_flag(b.flags, &f1, st));
    if (f1) {
      EGG_TRY(set_flag(b.flags + 1, 1, st));
      EGG_TRY(def42_second(b.x[cur], n, d, eps, b.lo, b.hi, b.flags + 1, st));
      EGG_TRY(get_flag(b.flags + 1, &f2, st));
    }
    synced = f1 && f2;
    cur ^= 1;
    ++t;
    if (synced || t >= o.max_iters) break;
  }
  // eps-components of the returned state: min-label propagation + pointer jumping
  const unsigned nb = (unsigned)((n + 255) / 256);
  k_iota<<<nb, 256, 0, st>>>(b.lab[0], n);
  for (;;) {
    EGG_TRY(set_flag(b.flags + 2, 0, st));
    EGG_TRY(cc_round(b.x[cur], n, d, eps, b.lab[0], b.lab[1], b.flags + 2, st));
    k_jump<<<nb, 256, 0, st>>>(b.lab[1], n, b.lab[0]);
    EGG_CUDA(cudaGetLastError());
    int32_t ch = 0;
    EGG_TRY(get_flag(b.flags + 2, &ch, st));
    if (!ch) break;
  }
  k_canon<<<1, 1024, 0, st>>>(b.lab[0], n, b.ids, b.out);
  EGG_CUDA(cudaGetLastError());
  EGG_CUDA(cudaMemcpyAsync(labels_out, b.out, sizeof(int32_t) * n, dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                           st));
  if (o.coords_out)
    EGG_CUDA(cudaMemcpyAsync(o.coords_out, b.x[cur], bytes, dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, st));
  EGG_CUDA(cudaStreamSynchronize(st));
  if (o.stats) {
    memset(o.stats, 0, sizeof(eggsync_stats));
    o.stats->iters = t;
  }
  *iters_out = t;
  return synced ? EGGSYNC_OK : EGGSYNC_NOT_CONVERGED;
}

}  // namespace egg

using namespace egg;

extern "C" {

int eggsync_sync_step(float* points, int64_t n, int32_t d, float eps, int32_t on_device, double* rc_out,
                      int32_t* nbr_out) {
  EGG_TRY(check_args(points, n, d, eps));
  SyncBufs b;
  EGG_TRY(b.alloc(n, d, nbr_out && !on_device));
  const size_t bytes = sizeof(float) * n * d;
  const float* x = points;
  float* xn = b.x[1];
  if (!on_device) {
    EGG_CUDA(cudaMemcpy(b.x[0], points, bytes, cudaMemcpyHostToDevice));
    x = b.x[0];
  }
  int32_t* nbr = nbr_out ? (on_device ? nbr_out : b.nbr) : nullptr;
  EGG_TRY(sync_run(x, xn, nbr, b.rcp, b.rc, n, d, eps));
  EGG_CUDA(cudaMemcpy(points, xn, bytes, on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost));
  if (nbr_out && !on_device) EGG_CUDA(cudaMemcpy(nbr_out, b.nbr, sizeof(int32_t) * n, cudaMemcpyDeviceToHost));
  double rc = 0.0;
  EGG_CUDA(cudaMemcpy(&rc, b.rc, sizeof(double), cudaMemcpyDeviceToHost));
  if (rc_out) *rc_out = rc;
  return EGGSYNC_OK;
}

int eggsync_sync_lambda(float* points, int64_t n, int32_t d, float eps, double lambda, int32_t max_iters,
                        int32_t on_device, int32_t* iters_out, double* rc_out) {
  EGG_TRY(check_args(points, n, d, eps));
  if (max_iters < 1 || !std::isfinite(lambda)) {
    set_error("max_iters must be >= 1 and lambda finite");
    return EGGSYNC_EINVAL;
  }
  SyncBufs b;
  EGG_TRY(b.alloc(n, d, false));
  const size_t bytes = sizeof(float) * n * d;
  EGG_CUDA(cudaMemcpy(b.x[0], points, bytes, on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice));
  // Alg 1: t = 0, r_c = 0; while r_c < lambda: update (l.5), r_c on D^t (l.6), t += 1
  int32_t t = 0, cur = 0;
  double rc = 0.0;
  while (rc < lambda && t < max_iters) {
    EGG_TRY(sync_run(b.x[cur], b.x[cur ^ 1], nullptr, b.rcp, b.rc, n, d, eps));
    EGG_CUDA(cudaMemcpy(&rc, b.rc, sizeof(double), cudaMemcpyDeviceToHost));
    cur ^= 1;
    ++t;
  }
  EGG_CUDA(cudaMemcpy(points, b.x[cur], bytes, on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost));
  if (iters_out) *iters_out = t;
  if (rc_out) *rc_out = rc;
  return rc >= lambda ? EGGSYNC_OK : EGGSYNC_NOT_CONVERGED;
}

}  // extern "C"
