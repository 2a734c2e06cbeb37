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
};

template <int D>
__global__ void __launch_bounds__(kSyncT) k_sync_brute(SyncArgs a) {
  __shared__ float tile[kSyncT * D];
  const int64_t p = (int64_t)blockIdx.x * kSyncT + threadIdx.x;
  const bool act = p < a.n;
  float x[D];
#pragma unroll
  for (int i = 0; i < D; ++i) x[i] = act ? a.x[p * D + i] : 0.f;
  double S[D];
#pragma unroll
  for (int i = 0; i < D; ++i) S[i] = 0.0;
  double R = 0.0;
  int32_t cnt = 0;
  for (int64_t t0 = 0; t0 < a.n; t0 += kSyncT) {
    const int64_t rem = a.n - t0;
    const int m = rem < kSyncT ? (int)rem : kSyncT;
    __syncthreads();
    for (int k = threadIdx.x; k < m * D; k += kSyncT) tile[k] = a.x[t0 * D + k];
    __syncthreads();
    float s[D];
#pragma unroll
    for (int i = 0; i < D; ++i) s[i] = 0.f;
    float r = 0.f;
    for (int j = 0; j < m; ++j) {
      const float* q = tile + j * D;
      float d2 = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float t = q[i] - x[i];
        d2 = fmaf(t, t, d2);
      }
      if (d2 > a.e2_hi) continue;
      bool in = d2 <= a.e2_lo;
      if (!in) {  // inside the band: the oracle's exact fp64 decision (dimension order, no FMA)
        double dd = 0.0;
#pragma unroll
        for (int i = 0; i < D; ++i) {
          const double t = (double)q[i] - (double)x[i];
          dd = __dadd_rn(dd, __dmul_rn(t, t));
        }
        in = dd <= a.e2;
      }
      if (in) {  // q in N_eps(p): Eq.1 term sin(q_i - p_i), Eq.2 term exp(-||q - p||)
        ++cnt;
#pragma unroll
        for (int i = 0; i < D; ++i) s[i] += sinf(q[i] - x[i]);
        r += expf(-sqrtf(d2));
      }
    }
#pragma unroll
    for (int i = 0; i < D; ++i) S[i] += (double)s[i];
    R += (double)r;
  }
  if (!act) return;
  const double inv = 1.0 / (double)cnt;  // cnt >= 1: p in N_eps(p)
#pragma unroll
  for (int i = 0; i < D; ++i) a.xn[p * D + i] = (float)((double)x[i] + inv * S[i]);
  if (a.nbr) a.nbr[p] = cnt;
  a.rcp[p] = R * inv;
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

template <int D>
int launch_sync(const SyncArgs& a) {
  const int64_t blocks = (a.n + kSyncT - 1) / kSyncT;
  k_sync_brute<D><<<(unsigned)blocks, kSyncT>>>(a);
  EGG_CUDA(cudaGetLastError());
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
int sync_iter(const float* x, float* xn, int32_t* nbr, double* rcp, double* rc_dev, int64_t n, int d, float eps) {
  const double e = (double)eps;
  const float e2f = (float)(e * e);
  const float rel = (float)(4 * d + 16) * kU;
  SyncArgs a{x, xn, nbr, rcp, n, e2f * (1.f - rel), e2f * (1.f + rel), e * e};
  EGG_DISPATCH(d, launch_sync, a);
}

int sync_run(const float* x, float* xn, int32_t* nbr, double* rcp, double* rc_dev, int64_t n, int d, float eps) {
  EGG_TRY(sync_iter(x, xn, nbr, rcp, rc_dev, n, d, eps));
  k_mean<<<1, 1024>>>(rcp, n, rc_dev);
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

}  // namespace
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
