// update_dense.cu -- F3: the random-access grid of PAPER.md §4.2.2 (L165-169) for d <= 4, as an
// alternative neighbour enumeration for A6 (the EGG-update, Alg 3; Eq.5-6).
//
// All w^d grid cells are enumerated (Eq.4: c_i = min(floor(x_i / c_w), w-1), the cell
// coordinates of the keys, fp64 as k_keys); a dense table maps the cell index sum c_i w^i to the
// non-empty grid cell of the current build (-1: empty), rebuilt every iteration.  A point p looks
// at every cell of the v^d window around its own cell, v = 2 ceil(eps / c_w) + 1 (L167), and
// within each non-empty cell at its update units (the F2 sub-cells, contiguous in key order):
// a unit entirely inside the eps-ball (MAXDIST of its exact MBR, fp32 with the (4d+16)u margin)
// contributes its exact summary (c_fix, Eq.6's full part), a unit entirely outside is skipped,
// any other unit is scanned point by point (fp32 distance, fp64 re-decision inside the margin,
// exactly the oracle's predicate; Eq.6's partial part, the per-point Eq.5 terms).  Sums are
// 64-bit fixed point (2^-32), so the result does not depend on the enumeration order; the
// epilogue is Eq.5 in fp64 and the first-term flag (Alg 3 l.14-15, L252).
// One thread per point: consecutive sorted points share most of their window.
#include "update.cuh"

namespace egg {

namespace {

template <int D>
struct DenseArgs {
  const uint32_t* __restrict__ orig;  // sharded runs: original local index (own iff < n_own), else nullptr
  int64_t n_own;
  const float* __restrict__ xs;
  float* __restrict__ xs_next;
  const float* __restrict__ sn;
  const float* __restrict__ cs;
  const int32_t* __restrict__ g_of;
  const int32_t* __restrict__ g_cnt;
  const int32_t* __restrict__ g_start;  // grid cell point ranges
  const int32_t* __restrict__ cell_of;  // unit of each sorted point
  const int32_t* __restrict__ cell_start;
  const uint64_t* __restrict__ c_fix;   // [2D][cap] exact unit sums (2^-32)
  const uint32_t* __restrict__ c_lo;
  const uint32_t* __restrict__ c_hi;
  const int32_t* __restrict__ c_cnt;
  const int32_t* __restrict__ dense;    // [w^D] grid cell of each cell index, -1 = empty
  int64_t n, cap, lo, hi, w;
  int32_t r;                            // window half-width ceil(eps / c_w)
  double inv_cw;
  float cwf, e2f, rel;
  double e2d;
  int32_t* flags;
  int32_t* nbr;
};

template <int D>
__device__ __forceinline__ int64_t cell_coord(float x, double inv_cw, int64_t w) {
  int64_t c = (int64_t)floor((double)x * inv_cw);  // as k_keys (R2): one fp64 product, floor, clamp
  return c < 0 ? 0 : (c >= w ? w - 1 : c);
}

template <int D>
__global__ void k_dense_fill(const float* __restrict__ xs, int64_t n, const int32_t* __restrict__ g_start,
                             int32_t n_grid, double inv_cw, int64_t w, int32_t* __restrict__ dense) {
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g >= n_grid) return;
  const int64_t j = g_start[g];  // every point of a grid cell has the cell's coordinates
  int64_t idx = 0, mul = 1;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    idx += cell_coord<D>(xs[(int64_t)i * n + j], inv_cw, w) * mul;
    mul *= w;
  }
  dense[idx] = (int32_t)g;
}

template <int D>
__global__ void __launch_bounds__(128) k_update_dense(const DenseArgs<D> a) {
  const int64_t j = a.lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= a.hi) return;
  float p[D];
  int64_t pc[D];
#pragma unroll
  for (int i = 0; i < D; ++i) {
    p[i] = a.xs[(int64_t)i * a.n + j];
    pc[i] = cell_coord<D>(p[i], a.inv_cw, a.w);
  }
  const float lim_in = a.e2f * (1.f - a.rel), lim_out = a.e2f * (1.f + a.rel);
  // window cells: a cell whose box lies beyond eps (+ a margin of 2^-20, far above the fp32
  // rounding of the box bounds) is skipped without a table look-up
  const float lim_cell = (sqrtf(a.e2f) + 9.5367431640625e-07f) * (sqrtf(a.e2f) + 9.5367431640625e-07f);
  unsigned long long fs[2 * D];
#pragma unroll
  for (int i = 0; i < 2 * D; ++i) fs[i] = 0ull;
  int64_t N = 0;
  int64_t off[D];
#pragma unroll
  for (int i = 0; i < D; ++i) off[i] = -a.r;
  for (;;) {
    int64_t idx = 0, mul = 1;
    bool inside = true;
    float m = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const int64_t c = pc[i] + off[i];
      inside = inside && c >= 0 && c < a.w;
      const float clo = (float)c * a.cwf, chi = (float)(c + 1) * a.cwf;
      const float dd = fmaxf(fmaxf(clo - p[i], p[i] - chi), 0.f);
      m = fmaf(dd, dd, m);
      idx += c * mul;
      mul *= a.w;
    }
    const int32_t g = (inside && m <= lim_cell) ? a.dense[idx] : -1;
    if (g >= 0) {
      const int32_t s0 = a.g_start[g], s1 = a.g_start[g + 1];
      const int32_t u0 = a.cell_of[s0], u1 = a.cell_of[s1 - 1];
      for (int32_t u = u0; u <= u1; ++u) {
        float mind = 0.f, maxd = 0.f;
#pragma unroll
        for (int i = 0; i < D; ++i) {
          const float l = ordf(a.c_lo[(int64_t)i * a.cap + u]), h = ordf(a.c_hi[(int64_t)i * a.cap + u]);
          const float dl = l - p[i], dh = p[i] - h;
          const float mn = fmaxf(fmaxf(dl, dh), 0.f), mx = fmaxf(-dl, -dh);
          mind = fmaf(mn, mn, mind);
          maxd = fmaf(mx, mx, maxd);
        }
        if (mind > lim_out) continue;
        if (maxd <= lim_in) {  // the whole unit is in N_eps(p): its exact summary
#pragma unroll
          for (int i = 0; i < 2 * D; ++i) fs[i] += a.c_fix[(int64_t)i * a.cap + u];
          N += a.c_cnt[u];
          continue;
        }
        const int32_t q0 = a.cell_start[u], q1 = a.cell_start[u + 1];
        for (int32_t q = q0; q < q1; ++q) {
          float qv[D];
          float d2 = 0.f;
#pragma unroll
          for (int i = 0; i < D; ++i) {
            qv[i] = a.xs[(int64_t)i * a.n + q];
            const float t = qv[i] - p[i];
            d2 = fmaf(t, t, d2);
          }
          bool in = d2 <= lim_in;
          if (!in && d2 <= lim_out) in = exact_d2<D>(qv, p) <= a.e2d;
          if (in) {
#pragma unroll
            for (int i = 0; i < D; ++i) {
              fs[i] += (unsigned long long)__double2ll_rn((double)a.sn[(int64_t)i * a.n + q] * kFix);
              fs[D + i] += (unsigned long long)__double2ll_rn((double)a.cs[(int64_t)i * a.n + q] * kFix);
            }
            ++N;
          }
        }
      }
    }
    // next window cell (odometer over D offsets in [-r, r])
    int k = 0;
    for (; k < D; ++k) {
      if (++off[k] <= a.r) break;
      off[k] = -a.r;
    }
    if (k == D) break;
  }
  // Eq.5 (L233-235) in fp64 from the exact sums
  const double inv = 1.0 / (double)N;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const double S = (double)(long long)fs[i] * kInvFix, C = (double)(long long)fs[D + i] * kInvFix;
    double sx, cx;
    const double x = (double)p[i];
    sincos(x, &sx, &cx);
    const double xn = x + (cx * S - sx * C) * inv;
    // x' lies in the range of N(p) (L104) and so in [0,1]; the clamp removes rounding only
    a.xs_next[(int64_t)i * a.n + j] = fminf(fmaxf((float)xn, 0.f), 1.f);
  }
  const bool f1 = N == (int64_t)a.g_cnt[a.g_of[j]];  // Alg 3 l.14-15 (L248)
  if (!f1 && (!a.orig || a.orig[j] < (uint32_t)a.n_own)) atomicAnd(&a.flags[0], 0);
  if (a.nbr) a.nbr[j] = (int32_t)N;
}

template <int D>
int dense_d(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr) {
  if constexpr (D > 4) {
    return EGGSYNC_EINVAL;
  } else {
    const Consts& K = ws.k;
    const int64_t cells = dense_cells(ws);
    EGG_TRY(dense_reserve(ws, (size_t)cells));
    cudaStream_t st = ws.stream;
    const int32_t* g_start = K.sub > 0 ? ws.co_start : ws.cell_start;
    EGG_CUDA(cudaMemsetAsync(ws.dense, 0xff, sizeof(int32_t) * (size_t)cells, st));
    k_dense_fill<D><<<(unsigned)((ws.n_grid + 255) / 256), 256, 0, st>>>(ws.xs[ws.xcur], ws.n, g_start, ws.n_grid,
                                                                         K.inv_cw, K.w, ws.dense);
    EGG_CUDA(cudaGetLastError());
    ws.launches += 2;
    if (hi <= lo) return EGGSYNC_OK;
    DenseArgs<D> a;
    a.orig = ws.own_orig();
    a.n_own = ws.n_own;
    a.xs = ws.xs[ws.xcur];
    a.xs_next = ws.xs[ws.xcur ^ 1];
    a.sn = ws.sn;
    a.cs = ws.cs;
    a.g_of = ws.g_of;
    a.g_cnt = ws.g_cnt;
    a.g_start = g_start;
    a.cell_of = ws.cell_of;
    a.cell_start = ws.cell_start;
    a.c_fix = ws.c_fix;
    a.c_lo = ws.c_lo;
    a.c_hi = ws.c_hi;
    a.c_cnt = ws.c_cnt;
    a.dense = ws.dense;
    a.n = ws.n;
    a.cap = ws.cap;
    a.lo = lo;
    a.hi = hi;
    a.w = K.w;
    a.r = (int32_t)std::ceil(K.e * K.inv_cw);  // v = 2 ceil(eps / c_w) + 1 (L167)
    a.inv_cw = K.inv_cw;
    a.cwf = (float)K.cw;
    a.e2f = K.e2f;
    a.rel = K.rel;
    a.e2d = K.e2;
    a.flags = ws.flags;
    a.nbr = nbr;
    k_update_dense<D><<<(unsigned)((hi - lo + 127) / 128), 128, 0, st>>>(a);
    EGG_CUDA(cudaGetLastError());
    ws.launches += 1;
    return EGGSYNC_OK;
  }
}

}  // namespace

// cells of the dense table (w^d), 0 when the table does not apply (d > 4 or more than 2^26 cells)
int64_t dense_cells(const Workspace& ws) {
  if (ws.d > 4) return 0;
  int64_t c = 1;
  for (int i = 0; i < ws.d; ++i) {
    c *= ws.k.w;
    if (c > (int64_t(1) << 26)) return 0;
  }
  return c;
}

// F3 random-access grid: EGGSYNC_DENSE=1 uses it wherever it applies (d <= 4, w^d <= 2^26),
// EGGSYNC_DENSE=0 never; default: never (the radix tree is faster on the measured configs)
bool dense_choose(const Workspace& ws) {
  static const int env = [] {
    const char* e = getenv("EGGSYNC_DENSE");
    return e ? atoi(e) : 0;
  }();
  return env == 1 && dense_cells(ws) > 0;
}

int run_update_dense(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr) {
  switch (ws.d) {
    case 1: return dense_d<1>(ws, lo, hi, nbr);
    case 2: return dense_d<2>(ws, lo, hi, nbr);
    case 3: return dense_d<3>(ws, lo, hi, nbr);
    case 4: return dense_d<4>(ws, lo, hi, nbr);
    default: return EGGSYNC_EINVAL;
  }
}

}  // namespace egg
