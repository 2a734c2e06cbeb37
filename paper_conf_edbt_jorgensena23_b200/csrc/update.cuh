// update.cuh -- A6 EGG-update (Algorithm 3; §4.3.2) and
// A7a first-term flag (Alg 3 l.14-15, L252), templated on the dimension D.
//
// For every point p (one lane each, 32 consecutive sorted points per warp):
//   sum_{q in N_eps(p)} sin(q_i)  and  sum cos(q_i)   (Eq.5)
// split into full and partial pieces (Eq.6):
//   * subtree of the cell hierarchy entirely inside the eps-ball of p
//     -> its summary (count, sum sin, sum cos)           [full fast path]
//   * subtree entirely outside -> skipped
//   * otherwise descend; at <= kBucket cells the cells are staged in shared
//     memory (origin-shifted to the warp's MBR centre) and classified per lane:
//     full cell -> cell summary; partial cell -> exact point scan  [boundary scan]
// then p_i <- p_i + (cos p_i * S_i - sin p_i * C_i) / |N|   (fp64 epilogue)
// and the first term |N_eps(p)| == |cell(p)| is AND-reduced into flags[0].
//
// The traversal is a warp "packet": one shared stack of (node, lane mask); a
// node is visited iff some lane still needs it, and every lane classifies it
// against its own point, so noise points and cluster points in one warp do
// not inflate each other's work.
//
// Exactness: every "full"/"out" decision carries a proven fp32 error margin;
// point pairs inside the margin are re-decided in fp64 exactly as the oracle's
// sum_i (q_i - p_i)^2 <= eps^2 (dimension order, no FMA).
#pragma once
#include "common.cuh"

namespace egg {

#define FULLMASK 0xffffffffu

template <int D>
struct UpdArgs {
  const float* __restrict__ xs;  // D^t, SoA [D][n], sorted
  float* __restrict__ xs_next;   // D^{t+1}, SoA [D][n], sorted
  const float* __restrict__ sn;  // sin(x), SoA [D][n]
  const float* __restrict__ cs;  // cos(x)
  const int32_t* __restrict__ cell_of;
  const int32_t* __restrict__ c_cnt;
  const float* __restrict__ c_rec;  // [nc][CellRec<D>::kFloats]
  const uint32_t* __restrict__ c_lo;  // [D][cap] ordered bits
  const uint32_t* __restrict__ c_hi;
  const int4* __restrict__ t_meta;
  const float* __restrict__ t_box;  // [nc-1][ceil4(2D)]
  const float* __restrict__ t_sum;
  const int32_t* __restrict__ t_cnt;
  int64_t n, cap, lo, hi;
  int32_t nc, stack_len;
  float e, e2f, rel;
  double e2d;
  int32_t* flags;  // [0] first term AND, [3] error
  int32_t* nbr;    // optional |N(p)| (sorted order)
  unsigned long long* work;  // optional work counters (CNT variant), see WorkCnt
};

// Work counters of the instrumented variant (lane-level events, summed per warp).
struct WorkCnt {
  long long cls = 0;     // (point, staged cell) classifications
  long long acc = 0;     // summary / point accumulations (2D adds each)
  long long scan = 0;    // (point, point) distance tests in partial-cell scans
  long long node = 0;    // (point, subtree box) tests
  long long exact = 0;   // fp64 re-decisions inside the error band
  long long part = 0;    // (point, partial cell) pairs
  long long nfull = 0;   // full-subtree summary uses
  long long staged = 0;  // cells staged into shared memory (per warp)
};

__device__ __forceinline__ float ordf(uint32_t o) {
  uint32_t b = (o & 0x80000000u) ? (o & 0x7fffffffu) : ~o;
  return __uint_as_float(b);
}

// squared distance exactly as the oracle evaluates it (fp64, dimension order, no contraction)
template <int D>
__device__ __forceinline__ double exact_d2(const float* q, const float* p) {
  double s = 0.0;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    double t = __dsub_rn((double)q[i], (double)p[i]);
    s = __dadd_rn(s, __dmul_rn(t, t));
  }
  return s;
}

template <int D>
struct UpdState {
  float p[D];    // the point
  float m2p[D];  // -2 (p - o)
  float pp;      // |p - o|^2
  float S[D], C[D];    // fp32 chunk accumulators
  double Sd[D], Cd[D]; // fp64 masters
  int N;               // |N_eps(p)|

  __device__ __forceinline__ void flush() {
#pragma unroll
    for (int i = 0; i < D; ++i) {
      Sd[i] += (double)S[i];
      Cd[i] += (double)C[i];
      S[i] = 0.f;
      C[i] = 0.f;
    }
  }
};

// Exact point scan of one partial cell for lanes with `pa` (warp-uniform call).
template <int D, bool CNT>
__device__ __forceinline__ void scan_cell(const UpdArgs<D>& a, UpdState<D>& s, bool pa, int32_t c,
                                          const float* __restrict__ sg, WorkCnt& wc) {
  constexpr int KA = Stage<D>::kA, KB = Stage<D>::kB;
  const int32_t cnt = __float_as_int(sg[KA + KB]);
  const int32_t start = __float_as_int(sg[KA + KB + 1]);
  // refine with the exact MBR of the cell (fp32 + margin)
  float mind = 0.f, maxd = 0.f;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const float l = ordf(a.c_lo[(int64_t)i * a.cap + c]), h = ordf(a.c_hi[(int64_t)i * a.cap + c]);
    const float dl = l - s.p[i], dh = s.p[i] - h;
    const float mn = fmaxf(fmaxf(dl, dh), 0.f), mx = fmaxf(-dl, -dh);
    mind = fmaf(mn, mn, mind);
    maxd = fmaf(mx, mx, maxd);
  }
  const bool full = pa && maxd <= a.e2f * (1.f - a.rel);
  pa = pa && !full && mind <= a.e2f * (1.f + a.rel);
  if constexpr (CNT) wc.acc += __popc(__ballot_sync(FULLMASK, full));
  if (__any_sync(FULLMASK, full)) {
    const float f = full ? 1.f : 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      s.S[i] = fmaf(f, sg[KA + i], s.S[i]);
      s.C[i] = fmaf(f, sg[KA + D + i], s.C[i]);
    }
    s.N += full ? cnt : 0;
  }
  if (!__any_sync(FULLMASK, pa)) return;
  s.flush();
  const float lim_in = a.e2f * (1.f - a.rel), lim_out = a.e2f * (1.f + a.rel);
  for (int32_t k = 0; k < cnt; ++k) {
    const int64_t q = start + k;
    float qv[D];
    float d2 = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      qv[i] = a.xs[(int64_t)i * a.n + q];
      const float t = qv[i] - s.p[i];
      d2 = fmaf(t, t, d2);
    }
    bool in = pa && d2 <= lim_in;
    const bool amb = pa && !in && d2 <= lim_out;
    if (__any_sync(FULLMASK, amb)) {
      if (amb) in = exact_d2<D>(qv, s.p) <= a.e2d;
    }
    if constexpr (CNT) {
      wc.scan += __popc(__ballot_sync(FULLMASK, pa));
      wc.exact += __popc(__ballot_sync(FULLMASK, amb));
      wc.acc += __popc(__ballot_sync(FULLMASK, in));
    }
    if (__any_sync(FULLMASK, in)) {
      const float f = in ? 1.f : 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        s.S[i] = fmaf(f, a.sn[(int64_t)i * a.n + q], s.S[i]);
        s.C[i] = fmaf(f, a.cs[(int64_t)i * a.n + q], s.C[i]);
      }
      s.N += in ? 1 : 0;
    }
    if ((k & 31) == 31) s.flush();
  }
  s.flush();
}

// Stage cells [first, first+cnt) (cnt <= 32) into the warp's shared buffer and
// accumulate them for the lanes in `pm`.
template <int D, bool CNT>
__device__ __forceinline__ void process_cells(const UpdArgs<D>& a, UpdState<D>& s, int32_t first, int32_t cntc,
                                              unsigned pm, float* __restrict__ st,
                                              const float* __restrict__ ov, int lane, WorkCnt& wc) {
  constexpr int SF = Stage<D>::kFloats, KA = Stage<D>::kA, KB = Stage<D>::kB;
  constexpr int R = CellRec<D>::kFloats;
  __syncwarp();
  if (lane < cntc) {
    const float* __restrict__ r = a.c_rec + (int64_t)(first + lane) * R;
    float* dst = st + lane * SF;
    const float Bw = ov[D];
    float cc = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const float t = r[i] - ov[i];
      dst[i] = t;
      cc = fmaf(t, t, cc);
    }
    const float rad = r[D];
    const float gerr = (float)(4 * D + 16) * kU * (Bw + cc + a.e2f);
    const float em = a.e - rad;
    const float emr = em * (1.f - 4.f * kU);
    const float ep = (a.e + rad) * (1.f + 4.f * kU);
    dst[D] = cc;
    dst[D + 1] = em > 0.f ? emr * emr - gerr : -1.f;
    dst[D + 2] = ep * ep + gerr;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      dst[KA + i] = r[D + 3 + i];
      dst[KA + D + i] = r[2 * D + 3 + i];
    }
    dst[KA + KB] = r[D + 1];      // count bits
    dst[KA + KB + 1] = r[D + 2];  // start bits
  }
  __syncwarp();
  const bool act = (pm >> lane) & 1u;
  if constexpr (CNT) {
    wc.staged += cntc;
    wc.cls += (long long)cntc * __popc(pm);
  }
  for (int g = 0; g < cntc; ++g) {
    const float* __restrict__ sg = st + g * SF;
    float cb[KA];
#pragma unroll
    for (int q = 0; q < KA / 4; ++q) {
      const float4 v = reinterpret_cast<const float4*>(sg)[q];
      cb[4 * q] = v.x;
      cb[4 * q + 1] = v.y;
      cb[4 * q + 2] = v.z;
      cb[4 * q + 3] = v.w;
    }
    float acc = s.pp + cb[D];
#pragma unroll
    for (int i = 0; i < D; ++i) acc = fmaf(s.m2p[i], cb[i], acc);
    const bool in = act && acc <= cb[D + 1];
    const bool pa = act && !in && acc <= cb[D + 2];
    if constexpr (CNT) {
      wc.part += __popc(__ballot_sync(FULLMASK, pa));
      wc.acc += __popc(__ballot_sync(FULLMASK, in));
    }
    if (__any_sync(FULLMASK, pa)) scan_cell<D, CNT>(a, s, pa, first + g, sg, wc);
    if (__any_sync(FULLMASK, in)) {
      float sb[KB];
#pragma unroll
      for (int q = 0; q < KB / 4; ++q) {
        const float4 v = reinterpret_cast<const float4*>(sg + KA)[q];
        sb[4 * q] = v.x;
        sb[4 * q + 1] = v.y;
        sb[4 * q + 2] = v.z;
        sb[4 * q + 3] = v.w;
      }
      const float f = in ? 1.f : 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        s.S[i] = fmaf(f, sb[i], s.S[i]);
        s.C[i] = fmaf(f, sb[D + i], s.C[i]);
      }
      s.N += in ? __float_as_int(sg[KA + KB]) : 0;
    }
  }
  s.flush();
}

template <int D, bool CNT>
__global__ void __launch_bounds__(kWarpsPerCta * 32) k_update(const UpdArgs<D> a) {
  constexpr int SF = Stage<D>::kFloats;
  constexpr int BS = ceil4(2 * D);
  constexpr int OV = ceil4(D + 1);
  extern __shared__ __align__(16) float smem[];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float* st = smem + wid * 32 * SF;
  float* ov = smem + kWarpsPerCta * 32 * SF + wid * OV;
  int2* stk = reinterpret_cast<int2*>(smem + kWarpsPerCta * (32 * SF + OV)) + wid * a.stack_len;

  const int64_t j = a.lo + ((int64_t)blockIdx.x * kWarpsPerCta + wid) * 32 + lane;
  const bool valid = j < a.hi;
  const unsigned amask = __ballot_sync(FULLMASK, valid);
  if (amask == 0u) return;

  UpdState<D> s;
  // warp MBR centre o (origin for the expanded distance form)
#pragma unroll
  for (int i = 0; i < D; ++i) {
    s.p[i] = valid ? a.xs[(int64_t)i * a.n + j] : 0.f;
    float l = valid ? s.p[i] : 3.0e38f, h = valid ? s.p[i] : -3.0e38f;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      l = fminf(l, __shfl_xor_sync(FULLMASK, l, off));
      h = fmaxf(h, __shfl_xor_sync(FULLMASK, h, off));
    }
    const float o = 0.5f * (l + h);
    if (lane == 0) ov[i] = o;
    const float t = s.p[i] - o;
    s.m2p[i] = -2.f * t;
  }
  s.pp = 0.f;
#pragma unroll
  for (int i = 0; i < D; ++i) s.pp = fmaf(0.5f * s.m2p[i], 0.5f * s.m2p[i], s.pp);
  {
    float b = valid ? s.pp : 0.f;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) b = fmaxf(b, __shfl_xor_sync(FULLMASK, b, off));
    if (lane == 0) ov[D] = b;
  }
#pragma unroll
  for (int i = 0; i < D; ++i) {
    s.S[i] = s.C[i] = 0.f;
    s.Sd[i] = s.Cd[i] = 0.0;
  }
  s.N = 0;

  const float lim_out = a.e2f * (1.f + a.rel), lim_full = a.e2f * (1.f - a.rel);
  WorkCnt wc;
  int sp = 1;
  if (lane == 0) stk[0] = make_int2(a.nc > 1 ? 0 : (int)kLeafBit, (int)amask);
  __syncwarp();
  while (sp > 0) {
    --sp;
    const int2 ent = stk[sp];
    __syncwarp();
    const unsigned m = (unsigned)ent.y;
    const bool act = (m >> lane) & 1u;
    if (ent.x & (int)kLeafBit) {
      process_cells<D, CNT>(a, s, ent.x & 0x7fffffff, 1, m, st, ov, lane, wc);
      continue;
    }
    const int node = ent.x;
    const float* __restrict__ bx = a.t_box + (int64_t)node * BS;
    float mind = 0.f, maxd = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const float dl = bx[i] - s.p[i], dh = s.p[i] - bx[D + i];
      const float mn = fmaxf(fmaxf(dl, dh), 0.f), mx = fmaxf(-dl, -dh);
      mind = fmaf(mn, mn, mind);
      maxd = fmaf(mx, mx, maxd);
    }
    const bool full = act && maxd <= lim_full;
    const bool part = act && !full && mind <= lim_out;
    if constexpr (CNT) {
      wc.node += __popc(m);
      const int nf = __popc(__ballot_sync(FULLMASK, full));
      wc.nfull += nf;
      wc.acc += nf;
    }
    if (__any_sync(FULLMASK, full)) {
      if (full) {
        const float* __restrict__ sm = a.t_sum + (int64_t)node * BS;
#pragma unroll
        for (int i = 0; i < D; ++i) {
          s.Sd[i] += (double)sm[i];
          s.Cd[i] += (double)sm[D + i];
        }
        s.N += a.t_cnt[node];
      }
    }
    const unsigned pm = __ballot_sync(FULLMASK, part);
    if (pm == 0u) continue;
    const int4 meta = a.t_meta[node];
    if (meta.y - meta.x + 1 <= kBucket) {
      process_cells<D, CNT>(a, s, meta.x, meta.y - meta.x + 1, pm, st, ov, lane, wc);
    } else {
      if (sp + 2 > a.stack_len) {  // cannot happen for depth <= key bits; guard anyway
        if (lane == 0) atomicExch(&a.flags[3], 1);
        break;
      }
      if (lane == 0) {
        stk[sp] = make_int2(meta.w, (int)pm);
        stk[sp + 1] = make_int2(meta.z, (int)pm);
      }
      sp += 2;
      __syncwarp();
    }
  }
  s.flush();
  bool f1 = true;
  if (valid) {
    const double inv = 1.0 / (double)s.N;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      double sx, cx;
      const double x = (double)s.p[i];
      sincos(x, &sx, &cx);
      const double xn = x + (cx * s.Sd[i] - sx * s.Cd[i]) * inv;  // Eq.5
      a.xs_next[(int64_t)i * a.n + j] = fminf(fmaxf((float)xn, 0.f), 1.f);
    }
    f1 = s.N == a.c_cnt[a.cell_of[j]];  // Alg 3 l.14-15 (L248)
    if (a.nbr) a.nbr[j] = s.N;
  }
  if (__any_sync(FULLMASK, !f1) && lane == 0) atomicAnd(&a.flags[0], 0);
  if constexpr (CNT) {
    if (lane == 0) {
      atomicAdd(&a.work[0], (unsigned long long)wc.cls);
      atomicAdd(&a.work[1], (unsigned long long)wc.acc);
      atomicAdd(&a.work[2], (unsigned long long)wc.scan);
      atomicAdd(&a.work[3], (unsigned long long)wc.node);
      atomicAdd(&a.work[4], (unsigned long long)wc.exact);
      atomicAdd(&a.work[5], (unsigned long long)wc.part);
      atomicAdd(&a.work[6], (unsigned long long)wc.nfull);
      atomicAdd(&a.work[7], (unsigned long long)wc.staged);
    }
  }
}

template <int D>
int run_update(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr) {
  if (hi <= lo) return EGGSYNC_OK;
  UpdArgs<D> a;
  a.xs = ws.xs[ws.xcur];
  a.xs_next = ws.xs[ws.xcur ^ 1];
  a.sn = ws.sn;
  a.cs = ws.cs;
  a.cell_of = ws.cell_of;
  a.c_cnt = ws.c_cnt;
  a.c_rec = ws.c_rec;
  a.c_lo = ws.c_lo;
  a.c_hi = ws.c_hi;
  a.t_meta = ws.t_meta;
  a.t_box = ws.t_box;
  a.t_sum = ws.t_sum;
  a.t_cnt = ws.t_cnt;
  a.n = ws.n;
  a.cap = ws.cap;
  a.lo = lo;
  a.hi = hi;
  a.nc = ws.n_cells;
  a.stack_len = ws.k.keybits + 4;
  a.e = ws.k.ef;
  a.e2f = ws.k.e2f;
  a.rel = ws.k.rel;
  a.e2d = ws.k.e2;
  a.flags = ws.flags;
  a.nbr = nbr;
  a.work = ws.count_work ? ws.work : nullptr;
  constexpr int SF = Stage<D>::kFloats;
  constexpr int OV = ceil4(D + 1);
  const size_t smem = (size_t)kWarpsPerCta * (32 * SF + OV) * sizeof(float) +
                      (size_t)kWarpsPerCta * a.stack_len * sizeof(int2);
  auto kern = a.work ? k_update<D, true> : k_update<D, false>;
  EGG_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int64_t pts_per_cta = 32 * kWarpsPerCta;
  const unsigned grid = (unsigned)((hi - lo + pts_per_cta - 1) / pts_per_cta);
  kern<<<grid, kWarpsPerCta * 32, smem, ws.stream>>>(a);
  ws.launches += 1;
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

}  // namespace egg
