// small.cu -- SURVEY.md §8(f) F1: the whole of Algorithm 4 for small
// inputs in ONE kernel launch, with no per-iteration host round trip.
//
// A thread-block cluster of kSmCtas CTAs keeps the state D^t (and D^{t+1}) of all n points in
// the shared memory of every CTA.  Per iteration, on the device:
//   keys     c_i = min(floor(x_i * (1/c_w)), w-1) in fp64 (Eq.4, c_w L252), packed
//   update   Eq.1 (L68) for the CTA's own points: q-range slices over the 16 lanes of a
//            half-warp, fp32 pair test with the fp64 re-decision inside the error band (the
//            oracle's predicate, R4), sinf(q_i - p_i) terms summed in fp32 chunks into fp64;
//            D^{t+1} written to every CTA's buffer through distributed shared memory
//   term 1   every neighbour in p's grid cell (Alg 3 l.14-15 L248; L252)
//   term 2   (only when term 1 holds) no q with eps < ||p-q|| <= eps+delta whose cell MBR
//            (= MBR(N_eps/2(q)) under term 1, R9) lies within eps of p (L108-110), fp64; the
//            MBRs come with the update (under term 1 a point's neighbours are its cell)
//   labels   cells of the verified state, numbered by their smallest point index (L256, R14)
// with cluster barriers (~0.2 us) between the phases.  The same readings (R1-R16) as the
// grid path; one launch replaces ~25 launches and 2-3 host synchronisations per iteration,
// which dominate inputs of a few thousand points (C1) and many-iteration inputs (the Fig 1
// bridge, L298: up to 343 iterations).
#include <cooperative_groups.h>

#include <cmath>
#include <cstdlib>

#include "common.cuh"

namespace cg = cooperative_groups;

namespace egg {
namespace {

constexpr int kSmCtas = 16;           // CTAs per cluster (non-portable cluster size)
constexpr int kSmThreads = 1024;
constexpr int kSmSlices = 16;         // q-range slices per point: a half-warp
constexpr int kSmMaxN = 4096;
constexpr int kSmMaxFloats = 8192;    // n * d of one state buffer in shared memory
constexpr int kSmMaxD = 8;            // (registers: 64 per thread at 1024 threads)

struct SmallArgs {
  const float* x0;  // n*d row-major input (device)
  int32_t n;
  double inv_cw;
  int64_t w;
  int32_t bits;
  float e2_lo, e2_hi, ed2_lo, ed2_hi;  // fp32 bands around eps^2 and (eps+delta)^2
  double e2, ed2;                      // exact tests (fp64, as the oracle)
  int32_t max_iters;
  int32_t* labels;   // n, original order (= input order)
  float* coords;     // n*d row-major, D^{t+1} at exit
  int32_t* out;      // [0] iterations, [1] converged
};

template <int D>
__device__ __forceinline__ double exact_d2s(const float* q, const float* p) {
  double s = 0.0;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const double t = __dsub_rn((double)q[i], (double)p[i]);
    s = __dadd_rn(s, __dmul_rn(t, t));
  }
  return s;
}

template <int D>
__global__ void __launch_bounds__(kSmThreads, 1) k_cluster_small(const SmallArgs a) {
  cg::cluster_group cl = cg::this_cluster();
  const int rank = (int)cl.block_rank();
  const int n = a.n;
  extern __shared__ __align__(16) unsigned char sm[];
  float* xb[2] = {reinterpret_cast<float*>(sm), reinterpret_cast<float*>(sm) + (size_t)n * D};  // [n][D]
  unsigned long long* key = reinterpret_cast<unsigned long long*>(sm + (size_t)2 * n * D * 4);
  float* lo = reinterpret_cast<float*>(key + n);  // [n][D] MBR of each point's cell (term 2)
  float* hi = lo + (size_t)n * D;
  int32_t* scan = reinterpret_cast<int32_t*>(hi + (size_t)n * D);  // [n] labels scratch (CTA 0)
  __shared__ int32_t flag[2];  // cluster-wide AND of term 1 / term 2 (every CTA holds the result)
  const int tid = threadIdx.x;

  for (int k = tid; k < n * D; k += kSmThreads) xb[0][k] = a.x0[k];
  __syncthreads();  // D^0 complete before the first keys read it (racecheck)
  const int per = (n + kSmCtas - 1) / kSmCtas;  // own points [rank*per, rank*per + per)
  const int p0 = rank * per, p1 = min(n, p0 + per);
  int cur = 0, t = 0;
  bool synced = false;
  for (;;) {
    const float* X = xb[cur];
    // ---- keys of D^t (every CTA, all points)
    for (int p = tid; p < n; p += kSmThreads) {
      unsigned long long kk = 0;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const double tt = __dmul_rn((double)X[p * D + i], a.inv_cw);  // one rounding, as the oracle
        long long c = (long long)floor(tt);
        c = c > a.w - 1 ? a.w - 1 : (c < 0 ? 0 : c);
        kk = (kk << a.bits) | (unsigned long long)c;
      }
      key[p] = kk;
    }
    if (tid < 2) flag[tid] = 1;
    cl.sync();  // keys ready; every CTA reset its flags before any remote AND below
    // ---- update + term 1 for the own points: half-warp h = point, lane s = q slice
    const int s = tid & (kSmSlices - 1);
    const int rounds = p1 > p0 ? (p1 - p0 + (kSmThreads >> 4) - 1) / (kSmThreads >> 4) : 0;  // uniform in the CTA
    for (int rr = 0; rr < rounds; ++rr) {
      const int p = p0 + rr * (kSmThreads >> 4) + (tid >> 4);
      const bool act = p < p1;
      float x[D];
#pragma unroll
      for (int i = 0; i < D; ++i) x[i] = act ? X[p * D + i] : 0.f;
      const unsigned long long kp = act ? key[p] : 0ull;
      double S[D];
#pragma unroll
      for (int i = 0; i < D; ++i) S[i] = 0.0;
      float sf[D], l[D], h[D];  // l, h: MBR of N_eps(p) (= MBR of cell(p) when term 1 holds)
#pragma unroll
      for (int i = 0; i < D; ++i) {
        sf[i] = 0.f;
        l[i] = h[i] = x[i];
      }
      int cnt = 0, chunk = 0;
      bool f1 = true;
      if (act) {
        for (int q = s; q < n; q += kSmSlices) {
          const float* xq = X + q * D;
          float d2 = 0.f;
#pragma unroll
          for (int i = 0; i < D; ++i) {
            const float u = xq[i] - x[i];
            d2 = fmaf(u, u, d2);
          }
          if (d2 > a.e2_hi) continue;
          bool in = d2 <= a.e2_lo;
          if (!in) in = exact_d2s<D>(xq, x) <= a.e2;  // the oracle's exact decision (R4)
          if (!in) continue;
          ++cnt;
          if (key[q] != kp) f1 = false;
#pragma unroll
          for (int i = 0; i < D; ++i) {
            sf[i] += sinf(xq[i] - x[i]);
            l[i] = fminf(l[i], xq[i]);
            h[i] = fmaxf(h[i], xq[i]);
          }
          if (++chunk == 64) {
#pragma unroll
            for (int i = 0; i < D; ++i) {
              S[i] += (double)sf[i];
              sf[i] = 0.f;
            }
            chunk = 0;
          }
        }
      }
#pragma unroll
      for (int i = 0; i < D; ++i) S[i] += (double)sf[i];
      // reduce over the 16 slices of the half-warp (fixed order: deterministic)
#pragma unroll
      for (int o = 8; o > 0; o >>= 1) {
        cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
#pragma unroll
        for (int i = 0; i < D; ++i) {
          S[i] += __shfl_xor_sync(0xffffffffu, S[i], o);
          l[i] = fminf(l[i], __shfl_xor_sync(0xffffffffu, l[i], o));
          h[i] = fmaxf(h[i], __shfl_xor_sync(0xffffffffu, h[i], o));
        }
      }
      const bool f1all = __all_sync(0xffffffffu, f1 || !act);
      if (!f1all && (tid & 31) == 0) {
        for (int r = 0; r < kSmCtas; ++r) atomicAnd(cl.map_shared_rank(&flag[0], r), 0);
      }
      if (act && s < D) {  // lane s writes coordinate s of p' to every CTA (Eq.1 in fp64)
        const double xd = (double)x[s];
        double Ss = 0.0;
        float ls = 0.f, hs = 0.f;
#pragma unroll
        for (int i = 0; i < D; ++i)
          if (i == s) {
            Ss = S[i];
            ls = l[i];
            hs = h[i];
          }
        const float xn = (float)(xd + Ss / (double)cnt);
        for (int r = 0; r < kSmCtas; ++r) {
          cl.map_shared_rank(xb[cur ^ 1], r)[p * D + s] = xn;
          cl.map_shared_rank(lo, r)[p * D + s] = ls;
          cl.map_shared_rank(hi, r)[p * D + s] = hs;
        }
      }
    }
    cl.sync();  // D^{t+1} complete in every CTA; flag[0] = term 1
    bool f1 = flag[0] != 0, f2 = false;
    if (f1) {
      // ---- term 2 for the own points; lo / hi hold MBR(N_eps(q)) from the update, which is
      // the MBR of cell(q) when term 1 holds (N_eps(q) = cell(q): the cell diagonal is eps/2)
      bool ok = true;
      for (int p = p0 + (tid >> 4); p < p1; p += kSmThreads >> 4) {
        const float* xp = X + p * D;
        for (int q = s; q < n; q += kSmSlices) {
          const float* xq = X + q * D;
          float d2 = 0.f;
#pragma unroll
          for (int i = 0; i < D; ++i) {
            const float u = xq[i] - xp[i];
            d2 = fmaf(u, u, d2);
          }
          if (d2 < a.e2_lo || d2 > a.ed2_hi) continue;
          const double dd = exact_d2s<D>(xq, xp);
          if (!(dd > a.e2 && dd <= a.ed2)) continue;  // eps < ||p-q|| <= eps + delta (L108)
          double m = 0.0;                              // dist(MBR(cell(q)), p)^2 (L110), fp64
#pragma unroll
          for (int i = 0; i < D; ++i) {
            const double v = (double)xp[i], L = (double)lo[q * D + i], H = (double)hi[q * D + i];
            double tt = 0.0;
            if (v < L) tt = L - v;
            else if (v > H) tt = v - H;
            m = __dadd_rn(m, __dmul_rn(tt, tt));
          }
          if (m <= a.e2) ok = false;
        }
      }
      if (!__all_sync(0xffffffffu, ok) && (tid & 31) == 0)
        for (int r = 0; r < kSmCtas; ++r) atomicAnd(cl.map_shared_rank(&flag[1], r), 0);
      cl.sync();
      f2 = flag[1] != 0;
    }
    synced = f1 && f2;
    ++t;
    if (synced || t >= a.max_iters) {
      // labels: cells of the verified state (D^t) or, at max_iters, of the last state (R15)
      const float* XL = synced ? X : xb[cur ^ 1];
      if (!synced) {  // keys of the last state
        for (int p = tid; p < n; p += kSmThreads) {
          unsigned long long kk = 0;
#pragma unroll
          for (int i = 0; i < D; ++i) {
            const double tt = __dmul_rn((double)XL[p * D + i], a.inv_cw);
            long long c = (long long)floor(tt);
            c = c > a.w - 1 ? a.w - 1 : (c < 0 ? 0 : c);
            kk = (kk << a.bits) | (unsigned long long)c;
          }
          key[p] = kk;
        }
        __syncthreads();
      }
      if (rank == 0) {
        for (int p = tid; p < n; p += kSmThreads) {  // representative: the smallest index in the cell
          int r = p;
          for (int q = 0; q < p; ++q)
            if (key[q] == key[p]) {
              r = q;
              break;
            }
          scan[p] = r;
        }
        __syncthreads();
        if (tid == 0) {  // canonical numbering by first occurrence (R14)
          int next = 0;
          for (int p = 0; p < n; ++p) {
            const int r = scan[p];
            a.labels[p] = r == p ? next++ : a.labels[r];
          }
          a.out[0] = t;
          a.out[1] = synced ? 1 : 0;
        }
        const float* XN = xb[cur ^ 1];  // D^{t+1}: the state after the last update
        for (int k = tid; k < n * D; k += kSmThreads) a.coords[k] = XN[k];
      }
      break;
    }
    cur ^= 1;
    cl.sync();  // everyone done reading D^t before it is overwritten next iteration
  }
}

template <int D>
int launch_small(const SmallArgs& a, cudaStream_t st) {
  const size_t smem = (size_t)4 * a.n * D * 4 + (size_t)a.n * 8 + (size_t)a.n * 4;
  EGG_CUDA(cudaFuncSetAttribute(k_cluster_small<D>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  EGG_CUDA(cudaFuncSetAttribute(k_cluster_small<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(kSmCtas, 1, 1);
  cfg.blockDim = dim3(kSmThreads, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = kSmCtas;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  EGG_CUDA(cudaLaunchKernelEx(&cfg, k_cluster_small<D>, a));
  return EGGSYNC_OK;
}

}  // namespace

// Eligibility of the one-launch path: n points of d dims fit the shared memory of a CTA twice
// over, and a cell's coordinates pack into one 64-bit key.
bool small_eligible(int64_t n, int d, const Consts& k) {
  if (const char* e = getenv("EGGSYNC_SMALL"))
    if (atoi(e) == 0) return false;
  return n >= 1 && n <= kSmMaxN && d <= kSmMaxD && n * d <= kSmMaxFloats && d * k.bits <= 64;
}

// Algorithm 4 on the device in one launch (see the header).  x_dev: n*d row-major device
// input; labels / coords: device outputs; out_host[0] = iterations, [1] = converged.
int small_cluster(const float* x_dev, int64_t n, int d, const Consts& k, int32_t max_iters, int32_t* labels_dev,
                  float* coords_dev, int32_t* out_dev, cudaStream_t st) {
  SmallArgs a;
  a.x0 = x_dev;
  a.n = (int32_t)n;
  a.inv_cw = k.inv_cw;
  a.w = k.w;
  a.bits = k.bits;
  a.e2_lo = k.e2f * (1.f - k.rel);
  a.e2_hi = k.e2f * (1.f + k.rel);
  a.ed2_lo = k.ed2f * (1.f - k.rel);
  a.ed2_hi = k.ed2f * (1.f + k.rel);
  a.e2 = k.e2;
  a.ed2 = k.ed2;
  a.max_iters = max_iters;
  a.labels = labels_dev;
  a.coords = coords_dev;
  a.out = out_dev;
  switch (d) {
    case 1: return launch_small<1>(a, st);
    case 2: return launch_small<2>(a, st);
    case 3: return launch_small<3>(a, st);
    case 4: return launch_small<4>(a, st);
    case 5: return launch_small<5>(a, st);
    case 6: return launch_small<6>(a, st);
    case 7: return launch_small<7>(a, st);
    case 8: return launch_small<8>(a, st);
    default: set_error("small path: unsupported d=%d", d); return EGGSYNC_EINVAL;
  }
}

}  // namespace egg
