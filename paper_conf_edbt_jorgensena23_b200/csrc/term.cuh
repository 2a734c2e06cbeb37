// term.cuh -- A7b: second term of the synchronization criterion (Def 4.2,
// PAPER.md L106-110; its grid check L254), evaluated only when the first term
// holds (Alg 4 l.9-10, L273-275).
//
// Violation iff for some p there is q with eps < ||p-q|| <= eps + delta and
// dist(MBR(N_{eps/2}(q)), p) <= eps.  When the first term holds in its grid
// form every neighbourhood is exactly a cell (diagonal <= eps/2, L252), so
// N_{eps/2}(q) = cell(q) and its MBR is the cell MBR computed in A4.  The
// search uses the same subtree hierarchy as the update with radius eps+delta.
#pragma once
#include "update.cuh"

namespace egg {

template <int D>
struct TermArgs {
  const uint32_t* __restrict__ orig;  // sharded runs: original local index (own iff < n_own), else nullptr
  int64_t n_own;
  const float* __restrict__ xs;
  const int32_t* __restrict__ g_of;    // grid cell of each sorted point
  const int32_t* __restrict__ u2co;    // unit -> grid cell (nullptr: identity)
  const int32_t* __restrict__ cell_start;  // unit point ranges
  const uint32_t* __restrict__ c_lo;   // unit MBR (candidate pruning)
  const uint32_t* __restrict__ c_hi;
  const uint32_t* __restrict__ g_lo;   // grid cell MBR = MBR(N_{eps/2}(q)) under the first term
  const uint32_t* __restrict__ g_hi;
  const int4* __restrict__ t_meta;
  const float* __restrict__ t_box;
  const float* __restrict__ c_rec;  // unit centre + radius (cheap sphere pre-test)
  int64_t n, cap, lo, hi;
  int32_t nc, stack_len, bucket;
  float e2f, ed2f, edf, rel;
  double e2d, ed2d;
  int32_t* flags;  // [1] second term AND, [3] error
  const uint8_t* __restrict__ need;  // per grid cell: its points need the point-level test (nullptr: all)
  int32_t n_grid;
};

// dist(MBR, p)^2 exactly as the oracle evaluates it (L110; fp64, dimension order)
template <int D>
__device__ __forceinline__ double exact_mindist2(const float* lo, const float* hi, const float* p) {
  double m = 0.0;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const double v = (double)p[i], l = (double)lo[i], h = (double)hi[i];
    double t = 0.0;
    if (v < l) t = __dsub_rn(l, v);
    else if (v > h) t = __dsub_rn(v, h);
    m = __dadd_rn(m, __dmul_rn(t, t));
  }
  return m;
}

template <int D>
__global__ void __launch_bounds__(kWarpsPerCta * 32) k_second(const TermArgs<D> a) {
  constexpr int BS = ceil4(2 * D);
  extern __shared__ __align__(16) float smem[];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  int2* stk = reinterpret_cast<int2*>(smem) + wid * a.stack_len;
  const int64_t j = a.lo + ((int64_t)blockIdx.x * kWarpsPerCta + wid) * 32 + lane;
  bool valid = j < a.hi && (!a.orig || a.orig[j] < (uint32_t)a.n_own);  // halo points do not test
  if (valid && a.need) valid = a.need[a.g_of[j]] != 0;  // cells cleared by the cell-level pass
  const unsigned amask = __ballot_sync(FULLMASK, valid);
  if (amask == 0u) return;
  float p[D];
#pragma unroll
  for (int i = 0; i < D; ++i) p[i] = valid ? a.xs[(int64_t)i * a.n + j] : 0.f;
  const int32_t own = valid ? a.g_of[j] : -1;
  const float lim_ed = a.ed2f * (1.f + a.rel);
  const float e_in = a.e2f * (1.f - a.rel), e_out = a.e2f * (1.f + a.rel);
  const float ed_in = a.ed2f * (1.f - a.rel);
  bool viol = false;
  int sp = 1;
  if (lane == 0) stk[0] = make_int2(a.nc > 1 ? 0 : (int)kLeafBit, (int)amask);
  __syncwarp();
  int pops = 0;
  while (sp > 0) {
    // early exit once any warp found a violation (polled every 64 pops: an L2 round trip)
    if ((++pops & 63) == 0 && *(volatile int32_t*)&a.flags[1] == 0) break;
    --sp;
    const int2 ent = stk[sp];
    __syncwarp();
    const unsigned m = (unsigned)ent.y;
    const bool act = (m >> lane) & 1u;
    int32_t first, last;
    unsigned pm;
    if (ent.x & (int)kLeafBit) {
      first = last = ent.x & 0x7fffffff;
      pm = m;
    } else {
      const float* __restrict__ bx = a.t_box + (int64_t)ent.x * BS;
      float mind = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float mn = fmaxf(fmaxf(bx[i] - p[i], p[i] - bx[D + i]), 0.f);
        mind = fmaf(mn, mn, mind);
      }
      pm = __ballot_sync(FULLMASK, act && mind <= lim_ed);
      if (pm == 0u) continue;
      const int4 meta = a.t_meta[ent.x];
      if (meta.y - meta.x + 1 > a.bucket) {
        if (sp + 2 > a.stack_len) {
          if (lane == 0) atomicExch(&a.flags[3], 1);
          break;
        }
        if (lane == 0) {
          stk[sp] = make_int2(meta.w, (int)pm);
          stk[sp + 1] = make_int2(meta.z, (int)pm);
        }
        sp += 2;
        __syncwarp();
        continue;
      }
      first = meta.x;
      last = meta.y;
    }
    const bool pact = (pm >> lane) & 1u;
    for (int32_t c = first; c <= last; ++c) {
      {  // sphere pre-test on the unit record: skip when |p - centre| - r > eps + delta
        const float* __restrict__ rc = a.c_rec + (int64_t)c * CellRec<D>::kFloats;
        float dc = 0.f;
#pragma unroll
        for (int i = 0; i < D; ++i) {
          const float t = rc[i] - p[i];
          dc = fmaf(t, t, dc);
        }
        const float reach = (a.edf + rc[D]) * (1.f + 4.f * kU);
        if (!__any_sync(FULLMASK, pact && dc <= reach * reach * (1.f + a.rel))) continue;
      }
      const int32_t gc = a.u2co ? a.u2co[c] : c;
      // prune the unit by its own MBR (no point of it within eps + delta)
      float umin = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float l = ordf(a.c_lo[(int64_t)i * a.cap + c]), h = ordf(a.c_hi[(int64_t)i * a.cap + c]);
        const float mn = fmaxf(fmaxf(l - p[i], p[i] - h), 0.f);
        umin = fmaf(mn, mn, umin);
      }
      float lo[D], hi[D];
      float mind = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        lo[i] = ordf(a.g_lo[(int64_t)i * a.cap + gc]);
        hi[i] = ordf(a.g_hi[(int64_t)i * a.cap + gc]);
        const float mn = fmaxf(fmaxf(lo[i] - p[i], p[i] - hi[i]), 0.f);
        mind = fmaf(mn, mn, mind);
      }
      // condition on q's MBR: dist(MBR(cell(q)), p) <= eps (L108), decided exactly near the margin
      bool cand = pact && gc != own && umin <= lim_ed && mind <= e_out;
      const bool amb = cand && mind > e_in;
      if (__any_sync(FULLMASK, amb)) {
        if (amb) cand = exact_mindist2<D>(lo, hi, p) <= a.e2d;
      }
      if (!__any_sync(FULLMASK, cand)) continue;
      const int32_t s0 = a.cell_start[c], s1 = a.cell_start[c + 1];
      for (int32_t q = s0; q < s1; ++q) {
        float qv[D];
        float d2 = 0.f;
#pragma unroll
        for (int i = 0; i < D; ++i) {
          qv[i] = a.xs[(int64_t)i * a.n + q];
          const float t = qv[i] - p[i];
          d2 = fmaf(t, t, d2);
        }
        // eps < ||p-q|| <= eps + delta   (L108)
        bool shell = cand && d2 > e_out && d2 <= ed_in;
        const bool amb2 = cand && !shell && d2 > e_in && d2 <= lim_ed;
        if (__any_sync(FULLMASK, amb2)) {
          if (amb2) {
            const double x = exact_d2<D>(qv, p);
            shell = x > a.e2d && x <= a.ed2d;
          }
        }
        viol = viol || shell;
      }
      if (__any_sync(FULLMASK, viol)) break;
    }
    if (__any_sync(FULLMASK, viol)) break;
  }
  if (__any_sync(FULLMASK, viol) && lane == 0) atomicAnd(&a.flags[1], 0);
}

// Cell-level pre-pass of the second term (one thread per grid cell A, its MBR standing for
// its points): a unit u of another cell B can host a violating pair (p in A, q in u) only if
//   MINDIST(MBR_u, MBR_A) <= eps + delta  (some pair within eps + delta),
//   MINDIST(MBR_B, MBR_A) <= eps          (some p of A with dist(MBR_B, p) <= eps, L108-110), and
//   MAXDIST(MBR_u, MBR_A) >  eps          (some pair beyond eps: a shell pair is possible),
// all tested in fp32 with the rel margins (conservative: an undecided case needs the point test).
// Cells for which no unit passes need no point-level test; near convergence that is almost all
// of them (collapsed clusters are single cells), so the point pass runs on a few points only.
template <int D>
__global__ void __launch_bounds__(128) k_second_cells(const TermArgs<D> a, int32_t ng, const int32_t* __restrict__ u2co,
                                                      uint8_t* __restrict__ need) {
  constexpr int BS = ceil4(2 * D);
  const int32_t A = (int32_t)((int64_t)blockIdx.x * blockDim.x + threadIdx.x);
  if (A >= ng) return;
  float lo[D], hi[D];
#pragma unroll
  for (int i = 0; i < D; ++i) {
    lo[i] = ordf(a.g_lo[(int64_t)i * a.cap + A]);
    hi[i] = ordf(a.g_hi[(int64_t)i * a.cap + A]);
  }
  const float lim_ed = a.ed2f * (1.f + a.rel), e_out = a.e2f * (1.f + a.rel), e_in = a.e2f * (1.f - a.rel);
  // box-box distances: min over the boxes' gap, max over their farthest corners
  auto mind_box = [&](const float* bl, const float* bh) {
    float m = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const float g = fmaxf(fmaxf(bl[i] - hi[i], lo[i] - bh[i]), 0.f);
      m = fmaf(g, g, m);
    }
    return m;
  };
  int stk[96];
  int sp = 0;
  stk[sp++] = a.nc > 1 ? 0 : (int)kLeafBit;
  bool needed = false;
  while (sp > 0 && !needed) {
    const int node = stk[--sp];
    if (node & (int)kLeafBit) {
      const int32_t u = node & 0x7fffffff;
      const int32_t B = u2co ? u2co[u] : u;
      if (B == A) continue;
      float ul[D], uh[D], bl[D], bh[D];
#pragma unroll
      for (int i = 0; i < D; ++i) {
        ul[i] = ordf(a.c_lo[(int64_t)i * a.cap + u]);
        uh[i] = ordf(a.c_hi[(int64_t)i * a.cap + u]);
        bl[i] = ordf(a.g_lo[(int64_t)i * a.cap + B]);
        bh[i] = ordf(a.g_hi[(int64_t)i * a.cap + B]);
      }
      if (mind_box(ul, uh) > lim_ed) continue;
      if (mind_box(bl, bh) > e_out) continue;
      float mx = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float g = fmaxf(uh[i] - lo[i], hi[i] - ul[i]);
        mx = fmaf(g, g, mx);
      }
      if (mx <= e_in) continue;
      needed = true;
      continue;
    }
    const float* __restrict__ bx = a.t_box + (int64_t)node * BS;
    float bl[D], bh[D];
#pragma unroll
    for (int i = 0; i < D; ++i) {
      bl[i] = bx[i];
      bh[i] = bx[D + i];
    }
    if (mind_box(bl, bh) > lim_ed) continue;
    if (sp + 2 > 96) {
      needed = true;  // too deep for the private stack: leave it to the point pass
      break;
    }
    const int4 meta = a.t_meta[node];
    stk[sp++] = meta.w;
    stk[sp++] = meta.z;
  }
  need[A] = needed ? 1 : 0;
}

template <int D>
int run_second_term(Workspace& ws, int64_t lo, int64_t hi) {
  if (hi <= lo) return EGGSYNC_OK;
  TermArgs<D> a;
  a.orig = ws.own_orig();
  a.n_own = ws.n_own;
  a.xs = ws.xs[ws.xcur];
  a.g_of = ws.g_of;
  a.u2co = ws.g_u2co;
  a.cell_start = ws.cell_start;
  a.c_lo = ws.c_lo;
  a.c_hi = ws.c_hi;
  a.g_lo = ws.g_lo;
  a.g_hi = ws.g_hi;
  a.t_meta = ws.t_meta;
  a.t_box = ws.t_box;
  a.c_rec = ws.c_rec;
  a.n = ws.n;
  a.cap = ws.cap;
  a.lo = lo;
  a.hi = hi;
  a.nc = ws.n_cells;
  a.stack_len = ws.k.keybits + 4;
  // as in the update: mostly-singleton units make subtree boxes useless for pruning
  a.bucket = (int64_t)ws.n_cells * 2 > ws.n ? 256 : kBucket;
  a.e2f = ws.k.e2f;
  a.ed2f = ws.k.ed2f;
  a.edf = ws.k.edf;
  a.rel = ws.k.rel;
  a.e2d = ws.k.e2;
  a.ed2d = ws.k.ed2;
  a.flags = ws.flags;
  a.need = nullptr;
  a.n_grid = ws.n_grid;
  if (ws.n_grid >= 2 && ws.second_need) {  // cell-level pass first: which cells need the point test
    k_second_cells<D><<<(unsigned)((ws.n_grid + 127) / 128), 128, 0, ws.stream>>>(a, ws.n_grid, ws.g_u2co,
                                                                                ws.second_need);
    ws.launches += 1;
    EGG_CUDA(cudaGetLastError());
    a.need = ws.second_need;
  }
  const size_t smem = (size_t)kWarpsPerCta * a.stack_len * sizeof(int2);
  EGG_CUDA(cudaFuncSetAttribute(k_second<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int64_t per = 32 * kWarpsPerCta;
  k_second<D><<<(unsigned)((hi - lo + per - 1) / per), kWarpsPerCta * 32, smem, ws.stream>>>(a);
  ws.launches += 1;
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

}  // namespace egg
