// update.cuh -- A6 EGG-update (Algorithm 3; §4.3.2) and
// A7a first-term flag (Alg 3 l.14-15, L252), templated on the dimension D.
//
// For every point p:
//   S_i = sum_{q in N_eps(p)} sin(q_i),  C_i = sum_{q in N_eps(p)} cos(q_i)   (Eq.5)
// split into full and partial pieces (Eq.6):
//   * subtree of the cell hierarchy entirely inside the eps-ball of p
//     -> its summary (count, sum sin, sum cos)                [full fast path]
//   * subtree entirely outside -> skipped
//   * otherwise descend; at <= a.bucket cells the cells are staged in shared
//     memory (origin-shifted to the warp's MBR centre) and classified per
//     point: full cell -> cell summary; partial cell -> exact point scan
//                                                              [boundary scan]
// then p_i <- p_i + (cos p_i * S_i - sin p_i * C_i) / |N|      (fp64 epilogue)
// and the first term |N_eps(p)| == |cell(p)| is AND-reduced into flags[0].
//
// Execution: one warp owns 64 consecutive sorted points (2 per lane: two
// independent dependency chains per lane, and every staged cell read from
// shared memory is used twice).  The traversal is a warp "packet": one shared
// stack of (node, 64-bit point mask); a node is visited iff some point still
// needs it, and every point classifies it against itself, so noise points and
// cluster points in one warp do not inflate each other's work.
//
// Arithmetic: the squared distance to a staged cell uses the expanded form
// |q|^2 + |c'|^2 - 2 q.c' in the warp's shifted frame (D FMAs, two chains);
// sums are accumulated in fp32 per bucket and flushed into fp64 masters kept
// in shared memory.  Every "full"/"out" decision carries a proven fp32 error
// margin; point pairs inside the margin are re-decided in fp64 exactly as the
// oracle's sum_i (q_i - p_i)^2 <= eps^2 (dimension order, no FMA).
#pragma once
#include <cstdlib>

#include "common.cuh"

namespace egg {

#define FULLMASK 0xffffffffu
#ifndef EGG_UPD_BUCKET_SPARSE
#define EGG_UPD_BUCKET_SPARSE 256  // cells mostly singletons (early iterations)
#define EGG_UPD_BUCKET_DENSE 64    // dense cells: box pruning pays
#endif
#ifndef EGG_UNCOND_ACC
#define EGG_UNCOND_ACC 1
#endif
#ifndef EGG_UNROLL_G
#define EGG_UNROLL_G 1
#endif
#ifndef EGG_PRED_ACC
#define EGG_PRED_ACC 0
#endif
#ifndef EGG_UPD_MINB
#define EGG_UPD_MINB 1
#endif
// points per lane: 2 while the per-point state fits the register file, else 1
__host__ __device__ constexpr int ppl_for(int d) {
#ifdef EGG_PPL
  return EGG_PPL;
#else
  return d <= 12 ? 2 : 1;
#endif
}
template <int D>
struct PPL {
  static constexpr int v = ppl_for(D);
};
// a subtree of <= a.bucket cells is processed cell by cell (chosen per launch, run_update)

template <int D>
struct UpdArgs {
  const uint32_t* __restrict__ orig;  // sharded runs: original local index (own iff < n_own), else nullptr
  int64_t n_own;
  const float* __restrict__ xs;  // D^t, SoA [D][n], sorted
  float* __restrict__ xs_next;   // D^{t+1}, SoA [D][n], sorted
  const float* __restrict__ sn;  // sin(x), SoA [D][n]
  const float* __restrict__ cs;  // cos(x)
  const int32_t* __restrict__ g_of;   // grid cell of each sorted point (first term, L252)
  const int32_t* __restrict__ g_cnt;  // grid cell counts
  const float* __restrict__ c_rec;  // [nc][CellRec<D>::kFloats]
  const uint32_t* __restrict__ c_lo;  // [D][cap] ordered bits
  const uint32_t* __restrict__ c_hi;
  const int4* __restrict__ t_meta;
  const float* __restrict__ t_box;  // [nc-1][ceil4(2D)]
  const float* __restrict__ t_sum;
  const int32_t* __restrict__ t_cnt;
  int64_t n, cap, lo, hi;
  int32_t nc, stack_len, bucket;
  int32_t stride, offset;  // this launch owns the 32*kP-point blocks b = stride*w + offset
  float e, e2f, rel;
  double e2d;
  int32_t* flags;  // [0] first term AND, [3] error
  int32_t* nbr;    // optional |N(p)| (sorted order)
  unsigned long long* work;  // optional work counters (CNT variant), see WorkCnt
};

// Work counters of the instrumented variant (point-level events, summed per warp).
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

__device__ __forceinline__ int popc64(unsigned long long m) { return __popcll(m); }

// Shared-memory layout of one warp (floats unless noted).
template <int D>
struct WarpSmem {
  static constexpr int kP = PPL<D>::v;
  static constexpr int SF = Stage<D>::kFloats;
  static constexpr int OV = ceil4(D + 4);  // o[D], Bw, pad
  static constexpr int kStageFloats = 32 * SF;
  static constexpr int kRawFloats = 2 * 32 * CellRec<D>::kFloats;  // TMA double buffer of cell records
  static constexpr int kMasterDoubles = kP * 2 * D * 32;
  // [stage | ov | raw[2] floats][2 mbarriers][masters doubles][stack int4]
  __host__ __device__ static constexpr size_t off_bar() { return (size_t)(kStageFloats + OV + kRawFloats) * 4; }
  __host__ __device__ static constexpr size_t off_mst() { return off_bar() + 16; }
  __host__ __device__ static constexpr size_t off_stk() { return off_mst() + (size_t)kMasterDoubles * 8; }
  __host__ __device__ static size_t bytes(int stack_len) { return off_stk() + (size_t)stack_len * 16; }
};

// warps per update CTA: 4, fewer when 4 warps' shared memory at the deepest possible stack
// (512 key bits) would exceed the 227 KB per CTA (d >= ~30)
template <int D>
struct UpdWarps {
  static constexpr size_t kMax = WarpSmem<D>::off_stk() + (size_t)(64 * kMaxKeyWords + 4) * 16;
  static constexpr int v = 4 * kMax <= 232448 ? 4 : 3 * kMax <= 232448 ? 3 : 2;
};

// ---- TMA (cp.async.bulk) staging of cell records: global -> shared, mbarrier completion
__device__ __forceinline__ unsigned smem_u32(const void* p) {
  return static_cast<unsigned>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
  // order earlier generic-proxy accesses of dst before the async-proxy write
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n}" ::"r"(
          smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// Per-warp TMA staging state (warp-uniform): two record buffers, their barriers and phases.
struct TmaStage {
  float* raw;      // raw[2][32 * CellRec<D>::kFloats]
  uint64_t* bar;   // bar[2]
  unsigned phase;  // bit b = parity of the next completion of buffer b
};

template <int D>
struct Lane {
  static constexpr int kP = PPL<D>::v;
  float q[kP][D];  // p - o (shifted point)
  float pp[kP];    // |q|^2
  float S[kP][D], C[kP][D];  // fp32 chunk accumulators
  int N[kP];       // |N_eps(p)|
  bool valid[kP];
  int64_t j[kP];   // sorted position
};

template <int D>
__device__ __forceinline__ void flush(Lane<D>& L, int k, double* __restrict__ mst, int lane) {
#pragma unroll
  for (int i = 0; i < D; ++i) {
    double* ms = mst + ((k * 2 * D + i) * 32 + lane);
    double* mc = mst + ((k * 2 * D + D + i) * 32 + lane);
    *ms += (double)L.S[k][i];
    *mc += (double)L.C[k][i];
    L.S[k][i] = 0.f;
    L.C[k][i] = 0.f;
  }
}

// Exact point scan of one partial cell for point k of the lanes with `pa` (warp-uniform call).
template <int D, bool CNT>
__device__ __forceinline__ void scan_cell(const UpdArgs<D>& a, Lane<D>& L, int k, bool pa, int32_t c,
                                          const float* __restrict__ sg, double* __restrict__ mst, int lane,
                                          WorkCnt& wc) {
  constexpr int KA = Stage<D>::kA, KB = Stage<D>::kB;
  const int32_t cnt = __float_as_int(sg[KA + KB]);
  const int32_t start = __float_as_int(sg[KA + KB + 1]);
  float p[D];  // the exact point (the shifted copy is not exact)
#pragma unroll
  for (int i = 0; i < D; ++i) p[i] = L.valid[k] ? a.xs[(int64_t)i * a.n + L.j[k]] : 0.f;
  // refine with the exact MBR of the cell (fp32 + margin)
  float mind = 0.f, maxd = 0.f;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const float l = ordf(a.c_lo[(int64_t)i * a.cap + c]), h = ordf(a.c_hi[(int64_t)i * a.cap + c]);
    const float dl = l - p[i], dh = p[i] - h;
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
      L.S[k][i] = fmaf(f, sg[KA + i], L.S[k][i]);
      L.C[k][i] = fmaf(f, sg[KA + D + i], L.C[k][i]);
    }
    L.N[k] += full ? cnt : 0;
  }
  if (!__any_sync(FULLMASK, pa)) return;
  flush(L, k, mst, lane);
  const float lim_in = a.e2f * (1.f - a.rel), lim_out = a.e2f * (1.f + a.rel);
  for (int32_t t = 0; t < cnt; ++t) {
    const int64_t q = start + t;
    float qv[D];
    float d2 = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      qv[i] = a.xs[(int64_t)i * a.n + q];
      const float u = qv[i] - p[i];
      d2 = fmaf(u, u, d2);
    }
    bool in = pa && d2 <= lim_in;
    const bool amb = pa && !in && d2 <= lim_out;
    if (__any_sync(FULLMASK, amb)) {
      if (amb) in = exact_d2<D>(qv, p) <= a.e2d;
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
        L.S[k][i] = fmaf(f, a.sn[(int64_t)i * a.n + q], L.S[k][i]);
        L.C[k][i] = fmaf(f, a.cs[(int64_t)i * a.n + q], L.C[k][i]);
      }
      L.N[k] += in ? 1 : 0;
    }
    if ((t & 31) == 31) flush(L, k, mst, lane);
  }
  flush(L, k, mst, lane);
}

// Stage cells [first, first+cntc) (cntc <= 32) into the warp's shared buffer and
// accumulate them for the points in `pm` (bit k*32+lane = point k of lane).
template <int D, bool CNT>
__device__ __forceinline__ void stage_round(const UpdArgs<D>& a, Lane<D>& L, int32_t first, int32_t cntc,
                                            unsigned long long pm, float* __restrict__ st,
                                            const float* __restrict__ ov, double* __restrict__ mst,
                                            int lane, WorkCnt& wc, const float* __restrict__ raw) {
  constexpr int kP = PPL<D>::v;
  constexpr int SF = Stage<D>::kFloats, KA = Stage<D>::kA, KB = Stage<D>::kB;
  constexpr int R = CellRec<D>::kFloats;
  __syncwarp();
  if (lane < cntc) {
    const float* __restrict__ r = raw + lane * R;  // record staged by the TMA bulk copy
    float* dst = st + lane * SF;
    const float Bw = ov[D];
    float cc = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const float t = r[i] - ov[i];
      dst[i] = -2.f * t;
      cc = fmaf(t, t, cc);
    }
    const float rad = r[D];
    const float gerr = (float)(4 * D + 16) * kU * (Bw + cc + a.e2f);
    const float em = a.e - rad;
    const float emr = em * (1.f - 4.f * kU);
    const float ep = (a.e + rad) * (1.f + 4.f * kU);
    dst[D] = cc;
    // limits on |q|^2 - 2 q.c' (= d^2 - |c'|^2): |c'|^2 folded in, saving an add per point
    dst[D + 1] = (em > 0.f ? emr * emr - gerr : -1.f) - cc;
    dst[D + 2] = ep * ep + gerr - cc;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      dst[KA + i] = r[D + 3 + i];
      dst[KA + D + i] = r[2 * D + 3 + i];
    }
    dst[KA + KB] = r[D + 1];      // count bits
    dst[KA + KB + 1] = r[D + 2];  // start bits
  }
  __syncwarp();
  bool act[kP];
#pragma unroll
  for (int k = 0; k < kP; ++k) act[k] = (pm >> (k * 32 + lane)) & 1ull;
  // points not active in this bucket get |q|^2 = 3e38: their distance is never within a limit
  float ppa[kP];
#pragma unroll
  for (int k = 0; k < kP; ++k) ppa[k] = act[k] ? L.pp[k] : 3.0e38f;
  if constexpr (CNT) {
    wc.staged += cntc;
    wc.cls += (long long)cntc * popc64(pm);
  }
  const float* __restrict__ sg = st;
  float cb[KA];  // A part of the current cell; the next cell's is loaded one iteration ahead
#pragma unroll
  for (int q = 0; q < KA / 4; ++q) {
    const float4 v = reinterpret_cast<const float4*>(sg)[q];
    cb[4 * q] = v.x;
    cb[4 * q + 1] = v.y;
    cb[4 * q + 2] = v.z;
    cb[4 * q + 3] = v.w;
  }
  constexpr int kUnrollG = (EGG_UNROLL_G && D <= 12) ? 2 : 1;
  constexpr bool kPrefetch = D <= 16;  // registers: high d reloads the A part in place
#pragma unroll(kUnrollG)
  for (int g = 0; g < cntc; ++g, sg += SF) {
    if constexpr (!kPrefetch) {
      if (g > 0) {
#pragma unroll
        for (int q = 0; q < KA / 4; ++q) {
          const float4 v = reinterpret_cast<const float4*>(sg)[q];
          cb[4 * q] = v.x;
          cb[4 * q + 1] = v.y;
          cb[4 * q + 2] = v.z;
          cb[4 * q + 3] = v.w;
        }
      }
    }
    bool in[kP], pa[kP];
    bool any_pa = false, any_in = false;
#pragma unroll
    for (int k = 0; k < kP; ++k) {
      float a0 = ppa[k], a1 = 0.f;
#pragma unroll
      for (int i = 0; i < D; i += 2) a0 = fmaf(L.q[k][i], cb[i], a0);
#pragma unroll
      for (int i = 1; i < D; i += 2) a1 = fmaf(L.q[k][i], cb[i], a1);
      const float d2 = a0 + a1;
      in[k] = d2 <= cb[D + 1];
      pa[k] = !in[k] && d2 <= cb[D + 2];
      any_pa |= pa[k];
      any_in |= in[k];
    }
    if (kPrefetch && g + 1 < cntc) {  // software pipelining: next cell's A part
#pragma unroll
      for (int q = 0; q < KA / 4; ++q) {
        const float4 v = reinterpret_cast<const float4*>(sg + SF)[q];
        cb[4 * q] = v.x;
        cb[4 * q + 1] = v.y;
        cb[4 * q + 2] = v.z;
        cb[4 * q + 3] = v.w;
      }
    }
    if constexpr (CNT) {
#pragma unroll
      for (int k = 0; k < kP; ++k) {
        wc.part += __popc(__ballot_sync(FULLMASK, pa[k]));
        wc.acc += __popc(__ballot_sync(FULLMASK, in[k]));
      }
    }
    // Low d: masked accumulate without a vote/branch (>90% of staged cells are inside
    // for some point) with the summary loads issued before the (rare) partial-cell
    // branch.  High d: load and accumulate only when some point is inside (registers).
    constexpr bool kEarly = EGG_UNCOND_ACC && D <= 12;
    float sb[KB];
    int cg = 0;
    if constexpr (kEarly) {
#pragma unroll
      for (int q = 0; q < KB / 4; ++q) {
        const float4 v = reinterpret_cast<const float4*>(sg + KA)[q];
        sb[4 * q] = v.x;
        sb[4 * q + 1] = v.y;
        sb[4 * q + 2] = v.z;
        sb[4 * q + 3] = v.w;
      }
      cg = __float_as_int(sg[KA + KB]);
    }
    if (__any_sync(FULLMASK, any_pa)) {
#pragma unroll
      for (int k = 0; k < kP; ++k)
        if (__any_sync(FULLMASK, pa[k])) scan_cell<D, CNT>(a, L, k, pa[k], first + g, sg, mst, lane, wc);
    }
    if (kEarly || __any_sync(FULLMASK, any_in)) {
      if constexpr (!kEarly) {
#pragma unroll
        for (int q = 0; q < KB / 4; ++q) {
          const float4 v = reinterpret_cast<const float4*>(sg + KA)[q];
          sb[4 * q] = v.x;
          sb[4 * q + 1] = v.y;
          sb[4 * q + 2] = v.z;
          sb[4 * q + 3] = v.w;
        }
        cg = __float_as_int(sg[KA + KB]);
      }
#pragma unroll
      for (int k = 0; k < kP; ++k) {
#if EGG_PRED_ACC
        if (in[k]) {  // predicated adds (no mask multiply)
#pragma unroll
          for (int i = 0; i < D; ++i) {
            L.S[k][i] += sb[i];
            L.C[k][i] += sb[D + i];
          }
          L.N[k] += cg;
        }
#else
        const float f = in[k] ? 1.f : 0.f;
#pragma unroll
        for (int i = 0; i < D; ++i) {
          L.S[k][i] = fmaf(f, sb[i], L.S[k][i]);
          L.C[k][i] = fmaf(f, sb[D + i], L.C[k][i]);
        }
        L.N[k] += in[k] ? cg : 0;
#endif
      }
    }
  }
}

// A bucket of <= a.bucket consecutive cells: staged and processed 32 at a time,
// one fp32 -> fp64 flush per bucket (a chunk of at most a.bucket summaries).
template <int D, bool CNT>
__device__ __forceinline__ void process_cells(const UpdArgs<D>& a, Lane<D>& L, int32_t first, int32_t cntc,
                                              unsigned long long pm, float* __restrict__ st,
                                              const float* __restrict__ ov, double* __restrict__ mst,
                                              int lane, WorkCnt& wc, TmaStage& tma) {
  constexpr int kP = PPL<D>::v;
  constexpr int R = CellRec<D>::kFloats;
  const int nr = (cntc + 31) / 32;
  // round r's 32 records are fetched with one bulk copy while round r-1 is processed
  __syncwarp();
  if (lane == 0) tma_load_1d(tma.raw, a.c_rec + (int64_t)first * R, (unsigned)min(32, cntc) * R * 4, tma.bar);
  for (int r = 0; r < nr; ++r) {
    const int b = r & 1;
    if (r + 1 < nr && lane == 0) {
      const int c1 = min(32, cntc - 32 * (r + 1));
      tma_load_1d(tma.raw + (b ^ 1) * 32 * R, a.c_rec + (int64_t)(first + 32 * (r + 1)) * R, (unsigned)c1 * R * 4,
                  tma.bar + (b ^ 1));
    }
    mbar_wait(tma.bar + b, (tma.phase >> b) & 1u);
    tma.phase ^= 1u << b;
    stage_round<D, CNT>(a, L, first + 32 * r, min(32, cntc - 32 * r), pm, st, ov, mst, lane, wc,
                        tma.raw + b * 32 * R);
  }
#pragma unroll
  for (int k = 0; k < kP; ++k) flush(L, k, mst, lane);
}

template <int D, bool CNT>
__global__ void __launch_bounds__(UpdWarps<D>::v * 32, EGG_UPD_MINB) k_update(const UpdArgs<D> a) {
  constexpr int kP = PPL<D>::v;
  using W = WarpSmem<D>;
  constexpr int BS = ceil4(2 * D);
  extern __shared__ __align__(16) float smem[];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // per-warp regions: [stage+ov floats][masters doubles][stack int4]
  char* wbase = reinterpret_cast<char*>(smem) + (size_t)wid * W::bytes(a.stack_len);
  float* st = reinterpret_cast<float*>(wbase);
  float* ov = st + W::kStageFloats;
  TmaStage tma;
  tma.raw = ov + W::OV;
  tma.bar = reinterpret_cast<uint64_t*>(wbase + W::off_bar());
  tma.phase = 0u;
  double* mst = reinterpret_cast<double*>(wbase + W::off_mst());
  int4* stk = reinterpret_cast<int4*>(wbase + W::off_stk());

  // ownership blocks of kOwnBlock points (b % stride == offset), each split into warp blocks
  constexpr int kSub = kOwnBlock / (32 * kP);
  const int64_t g = (int64_t)blockIdx.x * UpdWarps<D>::v + wid;
  const int64_t base = a.lo + ((g / kSub) * a.stride + a.offset) * kOwnBlock + (g % kSub) * (32 * kP);
  Lane<D> L;
  unsigned long long amask = 0ull;
#pragma unroll
  for (int k = 0; k < kP; ++k) {
    L.j[k] = base + k * 32 + lane;
    L.valid[k] = L.j[k] < a.hi;
    amask |= (unsigned long long)__ballot_sync(FULLMASK, L.valid[k]) << (32 * k);
  }
  if (amask == 0ull) return;

  // warp MBR centre o: origin of the shifted frame
  float Rw = 0.f;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    float x[kP];
    float l = 3.0e38f, h = -3.0e38f;
#pragma unroll
    for (int k = 0; k < kP; ++k) {
      x[k] = L.valid[k] ? a.xs[(int64_t)i * a.n + L.j[k]] : 0.f;
      if (L.valid[k]) {
        l = fminf(l, x[k]);
        h = fmaxf(h, x[k]);
      }
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      l = fminf(l, __shfl_xor_sync(FULLMASK, l, off));
      h = fmaxf(h, __shfl_xor_sync(FULLMASK, h, off));
    }
    const float o = 0.5f * (l + h);
    if (lane == 0) ov[i] = o;
#pragma unroll
    for (int k = 0; k < kP; ++k) {
      L.q[k][i] = L.valid[k] ? x[k] - o : 0.f;
      Rw = fmaxf(Rw, fabsf(L.q[k][i]));
    }
  }
  float Bw = 0.f;
#pragma unroll
  for (int k = 0; k < kP; ++k) {
    float pp = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) pp = fmaf(L.q[k][i], L.q[k][i], pp);
    asm volatile("" : "+f"(pp));  // keep it in a register (no rematerialisation in the hot loop)
    L.pp[k] = pp;
    Bw = fmaxf(Bw, pp);
#pragma unroll
    for (int i = 0; i < D; ++i) {
      L.S[k][i] = 0.f;
      L.C[k][i] = 0.f;
    }
    L.N[k] = 0;
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    Bw = fmaxf(Bw, __shfl_xor_sync(FULLMASK, Bw, off));
    Rw = fmaxf(Rw, __shfl_xor_sync(FULLMASK, Rw, off));
  }
  // subtree-box limits in the shifted frame: the rounding of q = fl(p - o) and
  // box' = fl(box - o) moves each per-dimension distance by <= 2u(|t| + Rw)
  const float slack = 2.5f * kU * sqrtf((float)D) * Rw;
  const float nlo = a.e * (1.f + 4.f * kU) + slack;
  const float nfu = fmaxf(a.e * (1.f - 4.f * kU) - slack, 0.f);
  const float lim_out = nlo * nlo * (1.f + (float)(2 * D + 8) * kU);
  const float lim_full = nfu * nfu * (1.f - (float)(2 * D + 8) * kU);
  if (lane == 0) ov[D] = Bw;
  for (int t = lane; t < W::kMasterDoubles; t += 32) mst[t] = 0.0;
  if (lane == 0) {
    mbar_init(tma.bar, 1);
    mbar_init(tma.bar + 1, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();

  WorkCnt wc;
  int sp = 1;
  if (lane == 0)
    stk[0] = make_int4(a.nc > 1 ? 0 : (int)kLeafBit, (int)(uint32_t)amask, (int)(uint32_t)(amask >> 32), 0);
  __syncwarp();
  while (sp > 0) {
    --sp;
    const int4 ent = stk[sp];
    __syncwarp();
    const unsigned long long m = (unsigned long long)(uint32_t)ent.y | ((unsigned long long)(uint32_t)ent.z << 32);
    if (ent.x & (int)kLeafBit) {
      process_cells<D, CNT>(a, L, ent.x & 0x7fffffff, 1, m, st, ov, mst, lane, wc, tma);
      continue;
    }
    const int node = ent.x;
    const float* __restrict__ bx = a.t_box + (int64_t)node * BS;
    bool full[kP], part[kP];
    bool any_full = false;
    float m0[kP], m1[kP], x0[kP], x1[kP];
#pragma unroll
    for (int k = 0; k < kP; ++k) m0[k] = m1[k] = x0[k] = x1[k] = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {  // box in the shifted frame, one dimension at a time
      const float lo = bx[i] - ov[i], hi = bx[D + i] - ov[i];
#pragma unroll
      for (int k = 0; k < kP; ++k) {
        const float dl = lo - L.q[k][i], dh = L.q[k][i] - hi;
        const float mn = fmaxf(fmaxf(dl, dh), 0.f), mx = fmaxf(-dl, -dh);
        if (i & 1) {
          m1[k] = fmaf(mn, mn, m1[k]);
          x1[k] = fmaf(mx, mx, x1[k]);
        } else {
          m0[k] = fmaf(mn, mn, m0[k]);
          x0[k] = fmaf(mx, mx, x0[k]);
        }
      }
    }
#pragma unroll
    for (int k = 0; k < kP; ++k) {
      const bool act = (m >> (k * 32 + lane)) & 1ull;
      full[k] = act && (x0[k] + x1[k]) <= lim_full;
      part[k] = act && !full[k] && (m0[k] + m1[k]) <= lim_out;
      any_full |= full[k];
    }
    if constexpr (CNT) {
      wc.node += popc64(m);
#pragma unroll
      for (int k = 0; k < kP; ++k) {
        const int nf = __popc(__ballot_sync(FULLMASK, full[k]));
        wc.nfull += nf;
        wc.acc += nf;
      }
    }
    if (__any_sync(FULLMASK, any_full)) {
      const float* __restrict__ sm = a.t_sum + (int64_t)node * BS;
      const int cnt = a.t_cnt[node];
#pragma unroll
      for (int k = 0; k < kP; ++k) {
        if (full[k]) {
#pragma unroll
          for (int i = 0; i < D; ++i) {
            mst[(k * 2 * D + i) * 32 + lane] += (double)sm[i];
            mst[(k * 2 * D + D + i) * 32 + lane] += (double)sm[D + i];
          }
          L.N[k] += cnt;
        }
      }
    }
    unsigned long long pm = 0ull;
#pragma unroll
    for (int k = 0; k < kP; ++k) pm |= (unsigned long long)__ballot_sync(FULLMASK, part[k]) << (32 * k);
    if (pm == 0ull) continue;
    const int4 meta = a.t_meta[node];
    if (meta.y - meta.x + 1 <= a.bucket) {
      process_cells<D, CNT>(a, L, meta.x, meta.y - meta.x + 1, pm, st, ov, mst, lane, wc, tma);
    } else {
      if (sp + 2 > a.stack_len) {  // cannot happen for depth <= key bits; guard anyway
        if (lane == 0) atomicExch(&a.flags[3], 1);
        break;
      }
      if (lane == 0) {
        stk[sp] = make_int4(meta.w, (int)(uint32_t)pm, (int)(uint32_t)(pm >> 32), 0);
        stk[sp + 1] = make_int4(meta.z, (int)(uint32_t)pm, (int)(uint32_t)(pm >> 32), 0);
      }
      sp += 2;
      __syncwarp();
    }
  }
  bool f1 = true;
#pragma unroll
  for (int k = 0; k < kP; ++k) {
    flush(L, k, mst, lane);
    if (L.valid[k]) {
      const double inv = 1.0 / (double)L.N[k];
#pragma unroll
      for (int i = 0; i < D; ++i) {
        double sx, cx;
        const double x = (double)a.xs[(int64_t)i * a.n + L.j[k]];
        sincos(x, &sx, &cx);
        const double Sd = mst[(k * 2 * D + i) * 32 + lane], Cd = mst[(k * 2 * D + D + i) * 32 + lane];
        const double xn = x + (cx * Sd - sx * Cd) * inv;  // Eq.5
        // x' lies in the range of N(p) (L104) and so in [0,1]; rounding of the summaries can put
        // it an ulp outside, which the clamp removes (the state stays in the domain, L70)
        a.xs_next[(int64_t)i * a.n + L.j[k]] = fminf(fmaxf((float)xn, 0.f), 1.f);
      }
      const bool own = !a.orig || a.orig[L.j[k]] < (uint32_t)a.n_own;
      f1 = f1 && (!own || L.N[k] == a.g_cnt[a.g_of[L.j[k]]]);  // Alg 3 l.14-15 (L248)
      if (a.nbr) a.nbr[L.j[k]] = L.N[k];
    }
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
int run_update_simt(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr) {
  if (hi <= lo) return EGGSYNC_OK;
  UpdArgs<D> a;
  a.orig = ws.own_orig();
  a.n_own = ws.n_own;
  a.xs = ws.xs[ws.xcur];
  a.xs_next = ws.xs[ws.xcur ^ 1];
  a.sn = ws.sn;
  a.cs = ws.cs;
  a.g_of = ws.g_of;
  a.g_cnt = ws.g_cnt;
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
  // mostly-singleton cells (early iterations): subtree boxes rarely prune or cover, so
  // process bigger buckets; dense cells: descend further and let box tests prune / cover
  a.bucket = (int64_t)ws.n_cells * 2 > ws.n ? EGG_UPD_BUCKET_SPARSE : EGG_UPD_BUCKET_DENSE;
  if (const char* e = getenv("EGGSYNC_BUCKET_SPARSE"); e && (int64_t)ws.n_cells * 2 > ws.n) a.bucket = atoi(e);
  if (const char* e = getenv("EGGSYNC_BUCKET_DENSE"); e && (int64_t)ws.n_cells * 2 <= ws.n) a.bucket = atoi(e);
  a.e = ws.k.ef;
  a.e2f = ws.k.e2f;
  a.rel = ws.k.rel;
  a.e2d = ws.k.e2;
  a.flags = ws.flags;
  a.nbr = nbr;
  a.work = ws.count_work ? ws.work : nullptr;
  const size_t smem = (size_t)UpdWarps<D>::v * WarpSmem<D>::bytes(a.stack_len);
  auto kern = a.work ? k_update<D, true> : k_update<D, false>;
  EGG_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  // all of the 228 KB unified L1/shared to shared memory: occupancy is shared-memory bound
  EGG_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
  // block-interleaved ownership (multi-GPU load balance): blocks b with b % stride == offset
  a.stride = ws.own_stride;
  a.offset = ws.own_offset;
  const int64_t nblocks = (hi - lo + kOwnBlock - 1) / kOwnBlock;
  const int64_t owned = nblocks > a.offset ? (nblocks - a.offset + a.stride - 1) / a.stride : 0;
  if (owned == 0) return EGGSYNC_OK;
  const int64_t warps = owned * (kOwnBlock / (32 * PPL<D>::v));
  const unsigned grid = (unsigned)((warps + UpdWarps<D>::v - 1) / UpdWarps<D>::v);
  kern<<<grid, UpdWarps<D>::v * 32, smem, ws.stream>>>(a);
  ws.launches += 1;
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

}  // namespace egg
