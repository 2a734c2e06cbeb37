// update_tc.cuh -- A6 EGG-update (Algorithm 3; Eq.5-6) on
// the 5th-generation tensor cores, plus the A7a first-term flag (Alg 3 l.14-15, L252).
//
// The per-point sums of Eq.5,
//   S_i(p) = sum_{q in N_eps(p)} sin(q_i),  C_i(p) = sum_{q in N_eps(p)} cos(q_i),  |N_eps(p)|,
// are computed for a tile of 128 consecutive sorted points at a time as two
// dense contractions against "entries" (update units = cells of the hierarchy):
//
//   GEMM1  S[p][e] = -2 q_p . c'_e - L_e        (tf32 x3 split: ~fp32-exact)
//          v = |q_p|^2 + S = |p - c_e|^2 - limF_e   in the tile-shifted frame
//   classify (CUDA cores, one thread per point row of TMEM):
//          v <= 0            -> entry e entirely inside the eps-ball of p (Eq.6 full part)
//          0 < v <= W_e      -> ambiguous band: exact fp64 re-decision (single point) or
//                               exact scan of the unit's points (Eq.6 partial part)
//          v > W_e           -> outside
//          P[p][e] = 1 for "inside", else 0   (written back into TMEM over S)
//   GEMM2  O[p][:] += P[p][:] . V[:][:]        V_e = (sum sin - cnt sin o, sum cos - cnt cos o, cnt)
//                                              split hi/lo into tf32 pairs (N = 2(2D+1))
//
// with fp32 accumulation in TMEM drained every kDrain entry tiles into exact 64-bit
// fixed-point sums (2^-32) per classifier group in shared memory.
// Entries are the cells of the subtrees that the plan pass (k_tc_plan) could not
// decide for the whole tile; subtrees entirely inside for every point that still
// needs them are added per point in the plan pass (full_S / full_N, exact fp64 of
// the fp32 subtree sums, as in k_update).  k_tc_expand turns each tile's ranges into a
// slot list (one unit per entry, padded to whole entry tiles); tiles are launched
// heaviest-first.
//
// Roles (416 threads, one CTA per point tile, one CTA per SM: it owns all 512 TMEM columns):
//   warps 0-3   classifier group 0 (TMEM lanes 0..127), even entry tiles
//   warps 4-7   classifier group 1, odd entry tiles
//   warps 8-11  producers: thread t owns entry slot t; stages the unit record with
//               cp.async one tile ahead and writes the GEMM operands (origin-shifted,
//               tf32-split) into a 3-stage shared-memory ring
//   warp 12     MMA issue (one thread, polling both GEMM conditions) and TMEM owner
// TMEM: Q (K1 columns) | 3 S/P buffers (GEMM1 runs up to 2 tiles ahead) | O per group.
#pragma once
#include <cub/cub.cuh>

#include <vector>

#include "tc.cuh"
#include "update.cuh"

namespace egg {

constexpr int kTcTile = 128;  // points per tile (TMEM lanes, GEMM M)
constexpr int kTcEnt = 128;   // entries per entry tile (GEMM1 N, GEMM2 K)
constexpr int kTcThreads = 13 * 32;  // 8 classifier + 4 producer warps + 1 MMA warp (<= 128 registers)
constexpr int kProd = 128;  // producer threads (warps 8-11): one entry slot each
constexpr int kMmaWarp = 12;  // TMEM owner; its lane 0 issues the MMAs
constexpr int kTcMaxD = 12;
#ifndef EGG_TC_DRAIN
#define EGG_TC_DRAIN 2
#endif
constexpr int kDrain = EGG_TC_DRAIN;  // entry tiles per fp32 chunk of a classifier group

template <int D>
struct TcCfg {
  static constexpr int K1 = ((3 * D + 2) + 7) / 8 * 8;  // GEMM1 K: q_hi, q_lo, q_hi, 1, 1
  static constexpr int NV = 2 * D + 1;                  // sin, cos, count
  static constexpr int N2 = (2 * NV + 15) / 16 * 16;     // GEMM2 N: hi | lo
  // TMEM columns: Q, NS S/P buffers (3 when they fit: GEMM1 runs ahead of both
  // classifier groups), one O accumulator per classifier group
  static constexpr int kColQ = 0;
  static constexpr int kColS = K1;                  // S/P buffers: kColS + 128*b
#ifndef EGG_TC_NS
#define EGG_TC_NS 3
#endif
  static constexpr int kNS0 = (EGG_TC_NS >= 3 && K1 + 3 * kTcEnt + 2 * N2 <= 512) ? 3 : 2;
  static constexpr int kColO0 = K1 + kNS0 * kTcEnt;
  static_assert(K1 + 2 * kTcEnt + 2 * N2 <= 512, "TMEM budget");
  static_assert(N2 % 16 == 0, "drain loads of 16 columns");
  // shared-memory stage: B1 (K-major: entry rows), B2 (K-major: value rows), meta
  static constexpr int SBO1 = (K1 / 4) * 128;
  static constexpr int kB1Bytes = kTcEnt * K1 * 4;
  static constexpr int LBO2 = 144;  // 16-byte gap per 4-entry chunk: conflict-free producer stores
  static constexpr int SBO2 = (kTcEnt / 4) * LBO2;
  static constexpr int kB2Bytes = (N2 / 8) * SBO2;
  static constexpr int kMetaBytes = kTcEnt * 16 + 16;  // W, cnt, start, cell; Wmax[4]
  static constexpr int kStageBytes = kB1Bytes + kB2Bytes + kMetaBytes;
  static constexpr int R = CellRec<D>::kFloats;
  static constexpr int kRawBytes = 2 * kTcEnt * R * 4;      // cell records staged by bulk copies [2][128][R]
  // per classifier group: exact fixed-point sums [NV][row] (rare-path count at 2D) + tensor-core count [row]
  static constexpr int kRareBytes = 2 * (NV + 1) * kTcTile * 8;
  static constexpr int kMiscBytes = 3072;
  static constexpr int kBudget = 227 * 1024 - 1024;
  static constexpr int kStages0 = (kBudget - kRawBytes - kRareBytes - kMiscBytes) / kStageBytes;
  static constexpr int kStages = kStages0 >= 4 ? 4 : (kStages0 >= 3 ? 3 : 2);
  static constexpr int kRingBytes = kStages * kStageBytes;
  static constexpr int kNS = kNS0 < kStages ? kNS0 : kStages;  // the MMA loop needs stages >= S buffers
  static constexpr int kColO = K1 + kNS * kTcEnt;   // O buffers: kColO + N2*g
  static constexpr size_t kSmem = (size_t)kRingBytes + kRawBytes + kRareBytes + kMiscBytes + 1024;  // +1024 align
  static_assert(kSmem <= 227 * 1024, "shared-memory budget");
};

// ----------------------------------------------------------------------------------------
// Plan pass: one warp per 128-point tile (4 points per lane: row t = 32k + lane), warp-packet
// traversal of the cell hierarchy with the per-point box tests of k_update.  A node that some
// active point sees partially is descended (its full points stay active: they will classify
// the cells exactly); a node nobody sees partially is added by its full points here (into
// full_S / full_N, owned exclusively by the point's lane); a subtree of <= bucket cells that
// some point sees partially becomes a range of entries.  One pass: a tile's ranges go into
// chunks of kRangeChunk slots allocated from a global counter (chunk table per tile), so
// no count pass / scan is needed.  Overflow of the range buffer or of the chunk table is
// reported in ctr[0] / ctr[1] (the host grows the buffer and re-plans, or falls back).
// ----------------------------------------------------------------------------------------
template <int D>
struct PlanArgs {
  const float* __restrict__ xs;
  const int4* __restrict__ t_meta;
  const float* __restrict__ t_box;
  const float* __restrict__ t_sum;
  const int32_t* __restrict__ t_cnt;
  const int32_t* __restrict__ c_cnt;  // points per unit (cell)
  int64_t n, lo, hi;
  int32_t nc, stack_len, bucket, ntiles, stride, offset;
  float e;
  int32_t* t_nr;              // [ntiles] ranges per tile
  int32_t* t_ne;              // [ntiles] entries per tile
  int32_t* t_epad;            // [ntiles] entries padded to whole entry tiles
  int32_t* t_pv;              // [ntiles] tile index (values of the launch-order sort)
  int32_t* chunks;            // [ntiles][kChunkMax] first slot of each chunk
  int32_t* ctr;               // [0] slots allocated, [1] chunk-table overflow, [2..3] entries (u64), [4..5] their points (u64)
  int64_t rcap;               // capacity of ranges
  int2* ranges;               // (first cell, count)
  double* full_S;             // [2D][n]
  int32_t* full_N;            // [n]
  int32_t* flags;
};

#ifndef EGG_PLAN_WARPS
#define EGG_PLAN_WARPS 4
#endif
constexpr int kPlanWarps = EGG_PLAN_WARPS;  // point tiles (one warp each) per plan CTA

__device__ __forceinline__ int64_t tc_tile_base(int64_t lo, int64_t tile, int32_t stride, int32_t offset) {
  return lo + (tile * stride + offset) * (int64_t)kTcTile;
}

template <int D>
__global__ void __launch_bounds__(kPlanWarps * 32) k_tc_plan(const PlanArgs<D> a) {
  constexpr int kP = 4;
  constexpr int BS = ceil4(2 * D);
  extern __shared__ __align__(16) unsigned char psm[];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t tile = (int64_t)blockIdx.x * kPlanWarps + wid;
  if (tile >= a.ntiles) return;
  int* stk = reinterpret_cast<int*>(psm) + (size_t)wid * a.stack_len * 8;  // [stack_len][8]: node, m0..m3

  const int64_t base = tc_tile_base(a.lo, tile, a.stride, a.offset);
  float q[kP][D];
  bool valid[kP];
  int64_t j[kP];
  uint32_t am[kP];
#pragma unroll
  for (int k = 0; k < kP; ++k) {
    j[k] = base + 32 * k + lane;
    valid[k] = j[k] < a.hi;
    am[k] = __ballot_sync(FULLMASK, valid[k]);
  }
  float ov[D];
  float Rw = 0.f;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    float x[kP];
    float l = 3.0e38f, h = -3.0e38f;
#pragma unroll
    for (int k = 0; k < kP; ++k) {
      x[k] = valid[k] ? a.xs[(int64_t)i * a.n + j[k]] : 0.f;
      if (valid[k]) {
        l = fminf(l, x[k]);
        h = fmaxf(h, x[k]);
      }
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      l = fminf(l, __shfl_xor_sync(FULLMASK, l, off));
      h = fmaxf(h, __shfl_xor_sync(FULLMASK, h, off));
    }
    ov[i] = 0.5f * (l + h);
#pragma unroll
    for (int k = 0; k < kP; ++k) {
      q[k][i] = valid[k] ? x[k] - ov[i] : 0.f;
      Rw = fmaxf(Rw, fabsf(q[k][i]));
    }
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) Rw = fmaxf(Rw, __shfl_xor_sync(FULLMASK, Rw, off));
  // the box limits of k_update (shifted-frame rounding slack + fp32 margins)
  const float slack = 2.5f * kU * sqrtf((float)D) * Rw;
  const float nlo = a.e * (1.f + 4.f * kU) + slack;
  const float nfu = fmaxf(a.e * (1.f - 4.f * kU) - slack, 0.f);
  const float lim_out = nlo * nlo * (1.f + (float)(2 * D + 8) * kU);
  const float lim_full = nfu * nfu * (1.f - (float)(2 * D + 8) * kU);
  bool touched[kP] = {false, false, false, false};  // full_S of the point initialised
  int N[kP] = {0, 0, 0, 0};
  int32_t nr = 0, ne = 0;
  long long npts = 0;  // points in the tile's entries (= ne while the cells are singletons)
  int32_t cbase = 0;  // first slot of the current chunk (warp-uniform)
  int32_t* __restrict__ tch = a.chunks + tile * kChunkMax;
  // append a range (warp-uniform call)
  auto push = [&](int32_t first, int32_t cnt, int32_t pts) {
    npts += pts;
    const int32_t slot = nr % kRangeChunk;
    if (slot == 0) {
      int32_t b = 0;
      if (lane == 0) {
        b = atomicAdd(&a.ctr[0], kRangeChunk);
        const int32_t ci = nr / kRangeChunk;
        if (ci < kChunkMax) tch[ci] = b;
        else atomicExch(&a.ctr[1], 1);
      }
      cbase = __shfl_sync(FULLMASK, b, 0);
    }
    if (lane == 0 && (int64_t)cbase + slot < a.rcap && nr < kChunkMax * kRangeChunk)
      a.ranges[cbase + slot] = make_int2(first, cnt);
    ++nr;
    ne += cnt;
  };
  __syncwarp();
  if (lane == 0) {
    stk[0] = a.nc > 1 ? 0 : (int)kLeafBit;
#pragma unroll
    for (int k = 0; k < kP; ++k) stk[1 + k] = (int)am[k];
  }
  __syncwarp();
  int sp = 1;
  while (sp > 0) {
    --sp;
    const int node = stk[sp * 8];
    uint32_t m[kP];
#pragma unroll
    for (int k = 0; k < kP; ++k) m[k] = (uint32_t)stk[sp * 8 + 1 + k];
    __syncwarp();
    if (node & (int)kLeafBit) {  // a single cell: always an entry
      push(node & 0x7fffffff, 1, a.c_cnt[node & 0x7fffffff]);
      continue;
    }
    const float* __restrict__ bx = a.t_box + (int64_t)node * BS;
    float m0[kP], x0[kP];
#pragma unroll
    for (int k = 0; k < kP; ++k) m0[k] = x0[k] = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const float blo = bx[i] - ov[i], bhi = bx[D + i] - ov[i];
#pragma unroll
      for (int k = 0; k < kP; ++k) {
        const float dl = blo - q[k][i], dh = q[k][i] - bhi;
        const float mn = fmaxf(fmaxf(dl, dh), 0.f), mx = fmaxf(-dl, -dh);
        m0[k] = fmaf(mn, mn, m0[k]);
        x0[k] = fmaf(mx, mx, x0[k]);
      }
    }
    bool full[kP], part[kP];
    uint32_t pm[kP], fm[kP];
    bool any_part = false;
#pragma unroll
    for (int k = 0; k < kP; ++k) {
      const bool act = (m[k] >> lane) & 1u;
      full[k] = act && x0[k] <= lim_full;
      part[k] = act && !full[k] && m0[k] <= lim_out;
      pm[k] = __ballot_sync(FULLMASK, part[k]);
      fm[k] = __ballot_sync(FULLMASK, full[k]);
      any_part |= pm[k] != 0u;
    }
    if (!any_part) {  // nobody needs to look inside: full points take the subtree summary
      bool anyf = false;
#pragma unroll
      for (int k = 0; k < kP; ++k) anyf |= fm[k] != 0u;
      if (anyf) {
        const int cnt = a.t_cnt[node];
        const float* __restrict__ sm = a.t_sum + (int64_t)node * BS;
#pragma unroll
        for (int k = 0; k < kP; ++k) {
          if (full[k]) {
            N[k] += cnt;
#pragma unroll
            for (int i = 0; i < 2 * D; ++i) {
              double* dst = a.full_S + (int64_t)i * a.n + j[k];
              *dst = (touched[k] ? *dst : 0.0) + (double)sm[i];
            }
            touched[k] = true;
          }
        }
      }
      continue;
    }
    const int4 meta = a.t_meta[node];
    const int ncell = meta.y - meta.x + 1;
    if (ncell <= a.bucket) {
      push(meta.x, ncell, a.t_cnt[node]);
      continue;
    }
    if (sp + 2 > a.stack_len) {
      if (lane == 0) atomicExch(&a.flags[3], 1);
      break;
    }
    if (lane == 0) {
      stk[sp * 8] = meta.w;
      stk[(sp + 1) * 8] = meta.z;
#pragma unroll
      for (int k = 0; k < kP; ++k) {
        stk[sp * 8 + 1 + k] = (int)(pm[k] | fm[k]);
        stk[(sp + 1) * 8 + 1 + k] = (int)(pm[k] | fm[k]);
      }
    }
    sp += 2;
    __syncwarp();
  }
  if (lane == 0) {
    a.t_nr[tile] = nr;
    a.t_ne[tile] = ne;
    atomicAdd(reinterpret_cast<unsigned long long*>(a.ctr + 2), (unsigned long long)ne);  // unpadded entries
    atomicAdd(reinterpret_cast<unsigned long long*>(a.ctr + 4), (unsigned long long)npts);
    a.t_epad[tile] = (ne + kTcEnt - 1) / kTcEnt * kTcEnt;
    a.t_pv[tile] = (int32_t)tile;
  }
#pragma unroll
  for (int k = 0; k < kP; ++k) {
    if (valid[k]) {
      if (!touched[k]) {
#pragma unroll
        for (int i = 0; i < 2 * D; ++i) a.full_S[(int64_t)i * a.n + j[k]] = 0.0;
      }
      a.full_N[j[k]] = N[k];
    }
  }
}

// Expansion of each tile's range list into its entry-slot list (one warp per tile): slot e of
// the tile holds the unit (cell) of entry e; the list is padded with -1 to whole entry tiles.
template <int kUnused>
__global__ void __launch_bounds__(128) k_tc_expand(const int2* __restrict__ ranges, const int32_t* __restrict__ chunks,
                                                   const int32_t* __restrict__ t_nr, const int32_t* __restrict__ t_ne,
                                                   const int32_t* __restrict__ eoff, int32_t* __restrict__ ent,
                                                   int32_t ntiles) {
  const int lane = threadIdx.x & 31;
  const int64_t tile = (int64_t)blockIdx.x * 4 + (threadIdx.x >> 5);
  if (tile >= ntiles) return;
  const int32_t nr = t_nr[tile];
  const int32_t* __restrict__ tch = chunks + tile * kChunkMax;
  int32_t* __restrict__ out = ent + eoff[tile];
  int32_t off = 0;
  for (int32_t r0 = 0; r0 < nr; r0 += 32) {
    const int32_t r = r0 + lane;
    const int2 g = r < nr ? ranges[tch[r / kRangeChunk] + (r % kRangeChunk)] : make_int2(0, 0);
    int32_t incl = g.y;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t u = __shfl_up_sync(FULLMASK, incl, o);
      if (lane >= o) incl += u;
    }
    const int32_t excl = incl - g.y;
    const int32_t tot = __shfl_sync(FULLMASK, incl, 31);
    const int kn = min(32, nr - r0);
    for (int k = 0; k < kn; ++k) {
      const int32_t first = __shfl_sync(FULLMASK, g.x, k), cnt = __shfl_sync(FULLMASK, g.y, k),
                    ex = __shfl_sync(FULLMASK, excl, k);
      for (int32_t t = lane; t < cnt; t += 32) out[off + ex + t] = first + t;
    }
    off += tot;
  }
  const int32_t ne = t_ne[tile];
  const int32_t padded = (ne + kTcEnt - 1) / kTcEnt * kTcEnt;
  for (int32_t t = ne + lane; t < padded; t += 32) out[t] = -1;
}

// ----------------------------------------------------------------------------------------
// Tensor-core update kernel
// ----------------------------------------------------------------------------------------
template <int D>
struct TcArgs {
  const float* __restrict__ xs;
  float* __restrict__ xs_next;
  const float* __restrict__ sn;
  const float* __restrict__ cs;
  const int32_t* __restrict__ g_of;
  const int32_t* __restrict__ g_cnt;
  const float* __restrict__ c_rec;
  const uint32_t* __restrict__ c_lo;
  const uint32_t* __restrict__ c_hi;
  const int32_t* __restrict__ ent;   // unit of every entry slot (-1 = padding)
  const int32_t* __restrict__ eoff;  // [ntiles] first slot of each point tile
  const int32_t* __restrict__ perm;  // [ntiles] launch order
  const int32_t* __restrict__ t_ne;
  const double* __restrict__ full_S;
  const int32_t* __restrict__ full_N;
  int64_t n, cap, lo, hi;
  int32_t ntiles, stride, offset;
  float e, e2f, rel;
  double e2d;
  int32_t* flags;
  int32_t* nbr;
  unsigned long long* prof;  // optional cycle accounting (EGGSYNC_TC_PROF)
};


// shared-memory header of the TC kernel
struct TcMisc {
  uint64_t stage_full[4], stage_empty[4], s_full[3], p_full[3], o_full[2];  // s_full / p_full: per S buffer
  uint32_t tbase;
  float o[kTcMaxD], s0[kTcMaxD], c0[kTcMaxD];
  float lo[4][kTcMaxD], hi[4][kTcMaxD];
  float Rq, Rqi;
};
static_assert(sizeof(TcMisc) <= 3072, "misc header");

// per-thread asynchronous 16-byte global -> shared copies (L2 only), waited per thread
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(tc::smem_addr(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

template <int D>
struct TcStage {
  float* b1;
  float* b2;
  float* W;
  int32_t* cnt;
  int32_t* start;
  int32_t* cell;
  float* wmax;
  __device__ TcStage(unsigned char* ring, int s) {
    using C = TcCfg<D>;
    unsigned char* p = ring + (size_t)s * C::kStageBytes;
    b1 = reinterpret_cast<float*>(p);
    b2 = reinterpret_cast<float*>(p + C::kB1Bytes);
    unsigned char* m = p + C::kB1Bytes + C::kB2Bytes;
    W = reinterpret_cast<float*>(m);
    cnt = reinterpret_cast<int32_t*>(m + 4 * kTcEnt);
    start = reinterpret_cast<int32_t*>(m + 8 * kTcEnt);
    cell = reinterpret_cast<int32_t*>(m + 12 * kTcEnt);
    wmax = reinterpret_cast<float*>(m + 16 * kTcEnt);
  }
};

// Exact path for a multi-point unit e inside the band of point pe (P stays 0 for the pair):
// refine with the unit's exact MBR, then its points one by one (fp32 + fp64 re-decision as
// in k_update).  Sums go into the classifier group's own fixed-point (2^-32) sums [NV][row]:
// exact, and the two groups' arrays are added in the epilogue (order-independent).
__device__ __forceinline__ void rare_add(unsigned long long* rare, int i, int row, double v) {
  rare[i * kTcTile + row] += (unsigned long long)llrint(v * kFix);  // the group's own row: no atomics
}
template <int D>
__device__ __noinline__ void tc_rare(const TcArgs<D>& a, const float* __restrict__ pe, int e,
                                     const TcStage<D>& st, unsigned long long* __restrict__ rare, int row) {
  const int32_t cnt = st.cnt[e];
  const int32_t start = st.start[e];
  const int32_t c = st.cell[e];
  float mind = 0.f, maxd = 0.f;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const float l = ordf(a.c_lo[(int64_t)i * a.cap + c]), h = ordf(a.c_hi[(int64_t)i * a.cap + c]);
    const float dl = l - pe[i], dh = pe[i] - h;
    const float mn = fmaxf(fmaxf(dl, dh), 0.f), mx = fmaxf(-dl, -dh);
    mind = fmaf(mn, mn, mind);
    maxd = fmaf(mx, mx, maxd);
  }
  const float lim_in = a.e2f * (1.f - a.rel), lim_out = a.e2f * (1.f + a.rel);
  if (mind > lim_out) return;
  constexpr int R = CellRec<D>::kFloats;
  if (maxd <= lim_in) {  // the whole unit is inside: its summary
    const float* __restrict__ r = a.c_rec + (int64_t)c * R;
#pragma unroll
    for (int i = 0; i < 2 * D; ++i) rare_add(rare, i, row, (double)r[D + 3 + i]);
    rare[2 * D * kTcTile + row] += (unsigned long long)cnt;
    return;
  }
  unsigned long long nin = 0;
  for (int32_t t = 0; t < cnt; ++t) {
    const int64_t qi = start + t;
    float qv[D];
    float d2 = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      qv[i] = a.xs[(int64_t)i * a.n + qi];
      const float u = qv[i] - pe[i];
      d2 = fmaf(u, u, d2);
    }
    bool in = d2 <= lim_in;
    if (!in && d2 <= lim_out) in = exact_d2<D>(qv, pe) <= a.e2d;
    if (in) {
#pragma unroll
      for (int i = 0; i < D; ++i) {
        rare_add(rare, i, row, (double)a.sn[(int64_t)i * a.n + qi]);
        rare_add(rare, D + i, row, (double)a.cs[(int64_t)i * a.n + qi]);
      }
      ++nin;
    }
  }
  rare[2 * D * kTcTile + row] += nin;
}

// Build entry slot `pt` (unit c, or padding when c < 0) of a stage: B1 row, B2 column, meta.
template <int D>
__device__ __forceinline__ float tc_build_entry(const TcArgs<D>& a, const TcMisc* __restrict__ ms,
                                                const TcStage<D>& st, int pt, int32_t c,
                                                const float* __restrict__ rec, float Rq, float Rqi) {
  using C = TcCfg<D>;
  constexpr int K1 = C::K1, NV = C::NV, N2 = C::N2;
  constexpr int R = CellRec<D>::kFloats;
  float b[K1];
  float vh[NV], vl[NV];
  float W = 0.f;
  int32_t ccnt = 0, cstart = 0;
  if (c >= 0) {
    float r[R];
    const float4* r4 = reinterpret_cast<const float4*>(rec);  // staged by the bulk copy
#pragma unroll
    for (int k = 0; k < R / 4; ++k) {
      const float4 t4 = r4[k];
      r[4 * k] = t4.x;
      r[4 * k + 1] = t4.y;
      r[4 * k + 2] = t4.z;
      r[4 * k + 3] = t4.w;
    }
    float cc = 0.f, cinf = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const float cp = r[i] - ms->o[i];
      const float h = tc::tf32_hi(cp);
      b[i] = -2.f * h;
      b[D + i] = -2.f * h;
      b[2 * D + i] = -2.f * (cp - h);
      cc = fmaf(cp, cp, cc);
      cinf = fmaxf(cinf, fabsf(cp));
    }
    const float rad = r[D];
    ccnt = __float_as_int(r[D + 1]);
    cstart = __float_as_int(r[D + 2]);
    // error budget: eta = rounding of the shifted frame; E = tf32 split
    // (2^-17 |q||c'|) + tensor-core accumulation (4 K-steps x 9 terms x 2^-23 of the sum
    // of |terms| <= 2^-17.8 (2|q||c'| + |L|)) + fp32 |q|^2, |c'|^2, L and v roundings
    const float eta = 2.5f * kU * sqrtf((float)D) * (Rqi + cinf);
    const float ep = (a.e + rad) * (1.f + 8.f * kU) + eta;
    const float em = (a.e - rad) * (1.f - 8.f * kU) - eta;
    const float limF0 = em > 0.f ? em * em * (1.f - 4.f * kU) : -1.f;
    const float E = 1.52587890625e-05f * (2.f * Rq * sqrtf(cc) + fabsf(limF0 - cc) + cc + Rq * Rq + 1e-30f);
    const float limF = em > 0.f ? limF0 - E : -1.f;
    const float limO = ep * ep * (1.f + 4.f * kU) + E;
    W = (limO - limF) * (1.f + 4.f * kU);
    const float L = limF - cc;
    const float Lh = tc::tf32_hi(L);
    b[3 * D] = -Lh;
    b[3 * D + 1] = -(L - Lh);
    const float fc = (float)ccnt;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const float vs = fmaf(-fc, ms->s0[i], r[D + 3 + i]);
      const float vc = fmaf(-fc, ms->c0[i], r[2 * D + 3 + i]);
      vh[i] = tc::tf32_hi(vs);
      vl[i] = vs - vh[i];
      vh[D + i] = tc::tf32_hi(vc);
      vl[D + i] = vc - vh[D + i];
    }
    vh[2 * D] = tc::tf32_hi(fc);
    vl[2 * D] = fc - vh[2 * D];
  } else {
#pragma unroll
    for (int k = 0; k < 3 * D + 2; ++k) b[k] = 0.f;
    b[3 * D] = 1073741824.f;  // v = 2^30: outside, never ambiguous
#pragma unroll
#pragma unroll
    for (int k = 0; k < NV; ++k) vh[k] = vl[k] = 0.f;
    ccnt = 0;
    cstart = 0;
  }
#pragma unroll
  for (int k = 3 * D + 2; k < K1; ++k) b[k] = 0.f;
  // B1: K-major, entry rows
  {
    unsigned char* b1 = reinterpret_cast<unsigned char*>(st.b1) + (pt >> 3) * C::SBO1 + (pt & 7) * 16;
#pragma unroll
    for (int kc = 0; kc < K1 / 4; ++kc)
      *reinterpret_cast<float4*>(b1 + kc * 128) = make_float4(b[4 * kc], b[4 * kc + 1], b[4 * kc + 2], b[4 * kc + 3]);
  }
  // B2: K-major value rows n (hi: n < NV, lo: NV <= n < 2NV), entry columns
  {
    unsigned char* b2 = reinterpret_cast<unsigned char*>(st.b2) + (pt >> 2) * C::LBO2 + (pt & 3) * 4;
#pragma unroll
    for (int n = 0; n < NV; ++n) {
      *reinterpret_cast<float*>(b2 + (n >> 3) * C::SBO2 + (n & 7) * 16) = vh[n];
      const int n2 = NV + n;
      *reinterpret_cast<float*>(b2 + (n2 >> 3) * C::SBO2 + (n2 & 7) * 16) = vl[n];
    }
#pragma unroll
    for (int n = 2 * NV; n < N2; ++n) *reinterpret_cast<float*>(b2 + (n >> 3) * C::SBO2 + (n & 7) * 16) = 0.f;
  }
#pragma unroll
  st.cnt[pt] = ccnt;
  st.start[pt] = cstart;
  st.cell[pt] = c;
  return W;
}

template <int D>
__global__ void __launch_bounds__(kTcThreads, 1) k_update_tc(const TcArgs<D> a) {
  using C = TcCfg<D>;
  constexpr int K1 = C::K1, NV = C::NV, N2 = C::N2, NST = C::kStages;
  extern __shared__ __align__(16) unsigned char tsm_raw[];
  unsigned char* tsm = tsm_raw + ((1024u - (tc::smem_addr(tsm_raw) & 1023u)) & 1023u);
  unsigned char* ring = tsm;
  float* raw = reinterpret_cast<float*>(tsm + C::kRingBytes);  // [2][kTcEnt][R] staged cell records
  unsigned long long* rare = reinterpret_cast<unsigned long long*>(tsm + C::kRingBytes + C::kRawBytes);
  TcMisc* ms = reinterpret_cast<TcMisc*>(tsm + C::kRingBytes + C::kRawBytes + C::kRareBytes);

  const int tid = threadIdx.x, wid = tid >> 5, lane = tid & 31;
  const int64_t tile = a.perm[blockIdx.x];  // heaviest point tiles first (shorter tail)
  const int64_t base = tc_tile_base(a.lo, tile, a.stride, a.offset);
  const int32_t ne = a.t_ne[tile];
  const int T = (ne + kTcEnt - 1) / kTcEnt;  // entry tiles (the slot list is padded to T * kTcEnt)

  // ---- setup -------------------------------------------------------------------------
  if (tid == 0) {
    for (int s = 0; s < NST; ++s) {
      tc::bar_init(&ms->stage_full[s], kProd);
      tc::bar_init(&ms->stage_empty[s], 1);
    }
    for (int b = 0; b < C::kNS; ++b) {
      tc::bar_init(&ms->s_full[b], 1);
      tc::bar_init(&ms->p_full[b], kTcTile);
    }
    for (int b = 0; b < 2; ++b) tc::bar_init(&ms->o_full[b], 1);
    tc::bar_fence_init();
  }
  if (wid == kMmaWarp) tc::tmem_alloc<512>(&ms->tbase);
  for (int t = tid; t < 2 * (NV + 1) * kTcTile; t += kTcThreads) rare[t] = 0ull;

  // classifier rows: every classifier thread holds its point
  const bool is_cls = wid < 8;
  const int grp = wid >> 2;           // classifier group (valid when is_cls)
  const int row = tid & (kTcTile - 1);
  const int64_t j = base + row;
  const bool valid = is_cls && j < a.hi;
  float pe[D];
#pragma unroll
  for (int i = 0; i < D; ++i) pe[i] = valid ? a.xs[(int64_t)i * a.n + j] : 0.f;
  if (is_cls && grp == 0) {  // tile MBR
#pragma unroll
    for (int i = 0; i < D; ++i) {
      float l = valid ? pe[i] : 3.0e38f, h = valid ? pe[i] : -3.0e38f;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        l = fminf(l, __shfl_xor_sync(FULLMASK, l, off));
        h = fmaxf(h, __shfl_xor_sync(FULLMASK, h, off));
      }
      if (lane == 0) {
        ms->lo[wid][i] = l;
        ms->hi[wid][i] = h;
      }
    }
  }
  __syncthreads();
  if (tid < D) {
    float l = fminf(fminf(ms->lo[0][tid], ms->lo[1][tid]), fminf(ms->lo[2][tid], ms->lo[3][tid]));
    float h = fmaxf(fmaxf(ms->hi[0][tid], ms->hi[1][tid]), fmaxf(ms->hi[2][tid], ms->hi[3][tid]));
    const float o = 0.5f * (l + h);
    ms->o[tid] = o;
    ms->s0[tid] = sinf(o);
    ms->c0[tid] = cosf(o);
  }
  if (tid == 0) {
    ms->Rq = 0.f;
    ms->Rqi = 0.f;
  }
  __syncthreads();
  float pp = 3.0e38f;  // |q|^2 (invalid rows never classify inside or ambiguous)
  if (is_cls) {
    float q[D];
    float s = 0.f, rinf = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      q[i] = valid ? pe[i] - ms->o[i] : 0.f;
      s = fmaf(q[i], q[i], s);
      rinf = fmaxf(rinf, fabsf(q[i]));
    }
    if (valid) pp = s;
    if (grp == 0) {
      float r2 = sqrtf(s) * (1.f + 4.f * kU), ri = rinf;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        r2 = fmaxf(r2, __shfl_xor_sync(FULLMASK, r2, off));
        ri = fmaxf(ri, __shfl_xor_sync(FULLMASK, ri, off));
      }
      if (lane == 0) {
        atomicMax(reinterpret_cast<int*>(&ms->Rq), __float_as_int(r2));
        atomicMax(reinterpret_cast<int*>(&ms->Rqi), __float_as_int(ri));
      }
      // Q row -> TMEM columns [0, K1): q_hi, q_lo, q_hi, 1, 1, 0...
      uint32_t v[K1];
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float h = tc::tf32_hi(q[i]);
        v[i] = __float_as_uint(h);
        v[D + i] = __float_as_uint(q[i] - h);
        v[2 * D + i] = __float_as_uint(h);
      }
      v[3 * D] = __float_as_uint(1.f);
      v[3 * D + 1] = __float_as_uint(1.f);
#pragma unroll
      for (int k = 3 * D + 2; k < K1; ++k) v[k] = 0u;
      const uint32_t taddr = ms->tbase + ((uint32_t)(32 * (wid & 3)) << 16) + C::kColQ;
#pragma unroll
      for (int c = 0; c < K1 / 8; ++c) {
        uint32_t w8[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) w8[k] = v[8 * c + k];
        tc::st8(taddr + 8 * c, w8);
      }
      tc::wait_st();
    }
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tb = ms->tbase;

  if (wid >= 8 && wid < kMmaWarp) {
    // ================================ producers ================================
    // Thread pt owns entry slot pt of every entry tile.  While entry tile jt is built from
    // the record staged in raw[jt&1][pt], the record of slot pt of tile jt+1 is fetched by
    // asynchronous copies (cp.async, waited by the same thread: no cross-thread hand-off).
    const int pt = tid - 256;  // 0..kProd-1
    const int pw = wid - 8;
    constexpr int R = C::R;
    const int32_t* __restrict__ ent = a.ent + a.eoff[tile];
    const float Rq = ms->Rq, Rqi = ms->Rqi;
    // records of slot pt of the next entry tile are copied while this one is built; the
    // slot's unit index is loaded one more tile ahead so its latency is hidden as well
    auto fetch = [&](int32_t c, int sb) {
      if (c >= 0) {
        float* dst = raw + ((size_t)sb * kTcEnt + pt) * R;
        const float* src = a.c_rec + (int64_t)c * R;
#pragma unroll
        for (int k = 0; k < R / 4; ++k) cp_async16(dst + 4 * k, src + 4 * k);
      }
      cp_async_commit();
    };
    auto unit_of = [&](int jt) -> int32_t { return jt < T ? ent[(int64_t)jt * kTcEnt + pt] : -1; };
    int32_t c_cur = unit_of(0), c_nxt = unit_of(1);
    if (T > 0) fetch(c_cur, 0);
    unsigned long long pc[4] = {0, 0, 0, 0};
    for (int jt = 0; jt < T; ++jt) {
      const int s = jt % NST, sb = jt & 1;
      const int32_t c = c_cur;
      long long t0 = clock64();
      if (jt + 1 < T) {
        fetch(c_nxt, sb ^ 1);
        c_cur = c_nxt;
        c_nxt = unit_of(jt + 2);
      }
      long long t1 = clock64();
      if (jt >= NST) tc::bar_wait(&ms->stage_empty[s], ((jt / NST) - 1) & 1);  // overlaps the copies
      long long t2 = clock64();
      if (jt + 1 < T) cp_async_wait<1>();
      else cp_async_wait<0>();
      long long t3 = clock64();
      pc[0] += t1 - t0;
      pc[1] += t2 - t1;
      pc[2] += t3 - t2;
      pc[3] -= t3;
      TcStage<D> st(ring, s);
      const float* rb = raw + (size_t)sb * kTcEnt * R;
      const float W = tc_build_entry<D>(a, ms, st, pt, c, rb + pt * R, Rq, Rqi);
      float wm = W;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) wm = fmaxf(wm, __shfl_xor_sync(FULLMASK, wm, off));
      if (lane == 0) st.wmax[pw] = wm;
      tc::fence_proxy_async();
      tc::bar_arrive(&ms->stage_full[s]);
      pc[3] += clock64();
    }
    if (a.prof && tid == 256) {
      for (int k = 0; k < 4; ++k) atomicAdd(&a.prof[k], pc[k]);
      atomicAdd(&a.prof[4], (unsigned long long)T);
    }
  }

  if (wid == kMmaWarp) {
    // ================================ MMA issue ================================
    // One thread issues, in order (the tensor pipe executes them in order):
    //   GEMM1(jt)        S[jt % NS] = Q . B1(jt)^T      once stage jt is built
    //   GEMM2(jt-NS+1)   O[g] (+)= P . B2^T             once its classifier group wrote P
    // so GEMM1 runs NS-1 tiles ahead of the classifiers and GEMM1(jt) follows GEMM2(jt-NS),
    // the last reader of its S buffer.  Blocking waits (the warp is suspended, it does not
    // take issue slots from the classifier / producer warps of its sub-partition).
    if (lane == 0) {
      constexpr uint32_t id1 = tc::idesc_tf32(128, kTcEnt, false);
      constexpr uint32_t id2 = tc::idesc_tf32(128, N2, false);
      constexpr int NS = C::kNS;
      const uint32_t ring_s = tc::smem_addr(ring);
      const int T0 = (T + 1) / 2, T1 = T / 2;  // entry tiles of group 0 / 1
      for (int jt = 0; jt < T + NS - 1; ++jt) {
        if (jt < T) {
          const int s = jt % NST, sb = jt % NS;
          tc::bar_wait(&ms->stage_full[s], (jt / NST) & 1);
          tc::fence_after();
          const uint32_t b1 = ring_s + s * C::kStageBytes;
#pragma unroll
          for (int k = 0; k < K1 / 8; ++k)
            tc::mma_ts(tb + C::kColS + kTcEnt * sb, tb + C::kColQ + 8 * k, tc::sdesc(b1 + k * 256, 128, C::SBO1), id1,
                       k > 0);
          tc::mma_commit(&ms->s_full[sb]);
        }
        const int jj = jt - (NS - 1);
        if (jj >= 0 && jj < T) {
          const int s = jj % NST, sb = jj % NS, g = jj & 1, kk = jj >> 1;
          tc::bar_wait(&ms->p_full[sb], (jj / NS) & 1);  // per S buffer: never two phases ahead
          tc::fence_after();
          const uint32_t b2 = ring_s + s * C::kStageBytes + C::kB1Bytes;
          const uint32_t acc0 = (kk % kDrain) != 0;
#pragma unroll
          for (int k = 0; k < kTcEnt / 8; ++k)
            tc::mma_ts(tb + C::kColO + N2 * g, tb + C::kColS + kTcEnt * sb + 8 * k,
                       tc::sdesc(b2 + k * 2 * C::LBO2, C::LBO2, C::SBO2), id2, (k > 0) || acc0);
          tc::mma_commit(&ms->stage_empty[s]);
          const int Tg = g ? T1 : T0;
          if ((kk % kDrain) == kDrain - 1 || kk == Tg - 1) tc::mma_commit(&ms->o_full[g]);
        }
      }
    }
    __syncwarp();
  }

  if (is_cls) {
    // ================================ classifiers ================================
    const uint32_t lane_off = (uint32_t)(32 * (wid & 3)) << 16;
    const int Tg = grp ? T / 2 : (T + 1) / 2;
    unsigned long long* racc = rare + grp * (NV + 1) * kTcTile;  // this group's sums (rows are exclusive)
    int dc = 0;  // drains done
    unsigned long long cw[3] = {0, 0, 0};
    // O (fp32, <= kDrain entry tiles) -> the row's exact fixed-point sums in shared memory
    // (integer atomics: both groups add to the same rows, order-independent)
    auto drain = [&]() {
      tc::bar_wait(&ms->o_full[grp], dc & 1);
      ++dc;
      tc::fence_after();
      double hi[NV];
#pragma unroll
      for (int c = 0; c < N2 / 16; ++c) {
        uint32_t v[16];
        tc::ld16(tb + lane_off + C::kColO + N2 * grp + 16 * c, v);
        tc::wait_ld();
#pragma unroll
        for (int jx = 0; jx < 16; ++jx) {
          const int col = 16 * c + jx;
          const float f = __uint_as_float(v[jx]);
          if (col < NV) {
            hi[col] = (double)f;
          } else if (col < 2 * NV) {
            const int i = col - NV;
            if (i < 2 * D) {
              const double x = hi[i] + (double)f;
              racc[i * kTcTile + row] += (unsigned long long)llrint(x * kFix);
            } else {  // count: exact integers in both halves
              const long long nc = llrint(hi[i]) + llrint((double)f);
              racc[NV * kTcTile + row] += (unsigned long long)nc;
            }
          }
        }
      }
    };
    for (int kk = 0; kk < Tg; ++kk) {
      const int jt = 2 * kk + grp;
      const int s = jt % NST, sb = jt % C::kNS;
      TcStage<D> st(ring, s);
      long long c0 = clock64();
      tc::bar_wait(&ms->s_full[sb], (jt / C::kNS) & 1);
      tc::fence_after();
      long long c1 = clock64();
      cw[0] += c1 - c0;
#pragma unroll 1
      for (int c = 0; c < kTcEnt / 32; ++c) {
        const uint32_t taddr = tb + lane_off + C::kColS + kTcEnt * sb + 32 * c;
        uint32_t v[32];
        tc::ld32(taddr, v);
        tc::wait_ld();
        const uint32_t wm = __float_as_uint(st.wmax[c]);
        uint32_t mn = 0xFFFFFFFFu;
#pragma unroll
        for (int jx = 0; jx < 32; ++jx) {
          const float f = __uint_as_float(v[jx]) + pp;  // |p - c_e|^2 - limF_e
          v[jx] = __float_as_uint(f);
          mn = __viaddmin_u32(v[jx], 0xFFFFFFFFu, mn);  // min over f > 0 of bits(f) - 1
        }
        if (mn < wm) {  // some pair of this chunk may lie in a band: exact decisions
          // candidates 0 < f <= max band of the chunk (bit trick as for mn); a candidate
          // outside its own entry's band is still decided exactly below (same answer)
          uint32_t bm = 0u;
#pragma unroll
          for (int jx = 0; jx < 32; ++jx) bm |= (v[jx] - 1u < wm) ? (1u << jx) : 0u;
          uint32_t fm = 0u;  // band pairs decided inside (single points)
          while (bm) {
            const int jx = __ffs(bm) - 1;
            bm &= bm - 1u;
            const int e = 32 * c + jx;
            if (st.cnt[e] == 1) {  // Def. of N_eps (L66) exactly as the oracle: fp64, dimension order
              double s2 = 0.0;
#pragma unroll
              for (int i = 0; i < D; ++i) {
                const double t = __dsub_rn((double)a.xs[(int64_t)i * a.n + st.start[e]], (double)pe[i]);
                s2 = __dadd_rn(s2, __dmul_rn(t, t));
              }
              if (s2 <= a.e2d) fm |= 1u << jx;
            } else {
              tc_rare<D>(a, pe, e, st, racc, row);
            }
          }
#pragma unroll
          for (int jx = 0; jx < 32; ++jx)
            v[jx] = (__uint_as_float(v[jx]) <= 0.f || ((fm >> jx) & 1u)) ? 0x3F800000u : 0u;
        } else {
#pragma unroll
          for (int jx = 0; jx < 32; ++jx) v[jx] = __uint_as_float(v[jx]) <= 0.f ? 0x3F800000u : 0u;
        }
        tc::st32(taddr, v);
      }
      tc::wait_st();
      long long c2 = clock64();
      cw[1] += c2 - c1;
      if (kk >= 1 && ((kk - 1) % kDrain) == kDrain - 1) drain();
      cw[2] += clock64() - c2;
      tc::fence_before();
      tc::bar_arrive(&ms->p_full[sb]);
    }
    if (Tg > 0) drain();
    if (a.prof && (tid == 0 || tid == 128)) {
      for (int k = 0; k < 3; ++k) atomicAdd(&a.prof[5 + k], cw[k]);
    }
  }

  // ---- epilogue (group 0 rows): Eq.5 in fp64 from the exact fixed-point sums -------------
  __syncthreads();  // all MMAs drained
  if (is_cls && grp == 0 && valid) {
    const unsigned long long* r0 = rare;
    const unsigned long long* r1 = rare + (NV + 1) * kTcTile;
    auto fx = [&](int k) { return (long long)(r0[k * kTcTile + row] + r1[k * kTcTile + row]); };
    const int64_t Nt = fx(NV);  // tensor-core count
    const int64_t Ni = Nt + fx(2 * D) + (int64_t)a.full_N[j];
    const double inv = 1.0 / (double)Ni;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      const double S = (double)Nt * (double)ms->s0[i] + (double)fx(i) * kInvFix + a.full_S[(int64_t)i * a.n + j];
      const double Cc = (double)Nt * (double)ms->c0[i] + (double)fx(D + i) * kInvFix + a.full_S[(int64_t)(D + i) * a.n + j];
      double sx, cx;
      const double x = (double)pe[i];
      sincos(x, &sx, &cx);
      const double xn = x + (cx * S - sx * Cc) * inv;  // Eq.5
      a.xs_next[(int64_t)i * a.n + j] = fminf(fmaxf((float)xn, 0.f), 1.f);
    }
    const bool f1 = Ni == (int64_t)a.g_cnt[a.g_of[j]];  // Alg 3 l.14-15 (L248)
    if (!f1) atomicAnd(&a.flags[0], 0);
    if (a.nbr) a.nbr[j] = (int32_t)Ni;
  }
  tc::fence_before();
  __syncthreads();
  if (wid == kMmaWarp) {
    tc::fence_after();
    tc::tmem_dealloc<512>(tb);
  }
}

// ----------------------------------------------------------------------------------------
// host side
// ----------------------------------------------------------------------------------------
template <int D>
int run_update_tc(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr) {
  if constexpr (D > kTcMaxD) {
    return EGGSYNC_EINVAL;
  } else {
    using C = TcCfg<D>;
    const int64_t ntot = (hi - lo + kTcTile - 1) / kTcTile;
    const int64_t owned =
        ntot > ws.own_offset ? (ntot - ws.own_offset + ws.own_stride - 1) / ws.own_stride : 0;
    ws.tc_used = 1;
    if (owned == 0) return EGGSYNC_OK;
    PlanArgs<D> p;
    p.xs = ws.xs[ws.xcur];
    p.t_meta = ws.t_meta;
    p.t_box = ws.t_box;
    p.t_sum = ws.t_sum;
    p.t_cnt = ws.t_cnt;
    p.c_cnt = ws.c_cnt;
    p.n = ws.n;
    p.lo = lo;
    p.hi = hi;
    p.nc = ws.n_cells;
    p.stack_len = ws.k.keybits + 4;
    // subtrees of <= bucket cells seen partially by the tile become entry ranges: large
    // while cells are mostly singletons (the tensor cores classify cheaply, the tree walk
    // does not), smaller once they hold many points each (measured sweep, C3 / C4-d10)
    const bool singletons = 2 * (int64_t)ws.n_cells > ws.n;
    p.bucket = singletons ? 512 : 128;
    if (const char* e = getenv(singletons ? "EGGSYNC_TC_BUCKET_S" : "EGGSYNC_TC_BUCKET")) p.bucket = atoi(e);
    p.ntiles = (int32_t)owned;
    p.stride = ws.own_stride;
    p.offset = ws.own_offset;
    p.e = ws.k.ef;
    p.t_nr = ws.tc_nr;
    p.t_ne = ws.tc_ne;
    p.chunks = ws.tc_chunks;
    p.ctr = ws.tc_ctr;
    p.full_S = ws.full_S;
    p.full_N = ws.full_N;
    p.flags = ws.flags;
    const size_t psmem = (size_t)kPlanWarps * p.stack_len * 8 * sizeof(int);
    const unsigned pgrid = (unsigned)((owned + kPlanWarps - 1) / kPlanWarps);
    EGG_CUDA(cudaFuncSetAttribute(k_tc_plan<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)psmem));
    p.t_epad = ws.tc_epad;
    p.t_pv = ws.tc_pv;
    // the range buffer keeps its size across updates (process cache); a first guess of
    // 16 chunks per tile, grown and re-planned when the plan reports more
    EGG_TRY(tc_ranges_reserve(ws, (size_t)owned * 16 * kRangeChunk));
    size_t tmp = 0;
    EGG_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, ws.tc_epad, ws.tc_eoff, (int)owned + 1, ws.stream));
    if (tmp > ws.cub_bytes) {
      set_error("cub scratch too small for the tensor-core plan scan");
      return EGGSYNC_ECUDA;
    }
    int32_t hc[7] = {0, 0, 0, 0, 0, 0, 0};  // ctr[0..5], padded entries
    for (int attempt = 0; attempt < 2; ++attempt) {
      p.ranges = ws.tc_ranges;
      p.rcap = (int64_t)ws.tc_rcap;
      EGG_CUDA(cudaMemsetAsync(ws.tc_ctr, 0, 6 * sizeof(int32_t), ws.stream));
      EGG_CUDA(cudaMemsetAsync(ws.tc_epad + owned, 0, sizeof(int32_t), ws.stream));
      k_tc_plan<D><<<pgrid, kPlanWarps * 32, psmem, ws.stream>>>(p);
      EGG_CUDA(cudaGetLastError());
      EGG_CUDA(cub::DeviceScan::ExclusiveSum(ws.cub_tmp, tmp, ws.tc_epad, ws.tc_eoff, (int)owned + 1, ws.stream));
      EGG_CUDA(cudaMemcpyAsync(hc, ws.tc_ctr, 6 * sizeof(int32_t), cudaMemcpyDeviceToHost, ws.stream));
      EGG_CUDA(cudaMemcpyAsync(hc + 6, ws.tc_eoff + owned, sizeof(int32_t), cudaMemcpyDeviceToHost, ws.stream));
      EGG_CUDA(cudaStreamSynchronize(ws.stream));
      ws.launches += 3;  // plan + scan (2)
      if (hc[1] || (size_t)(uint32_t)hc[0] <= ws.tc_rcap) break;
      EGG_TRY(tc_ranges_reserve(ws, (size_t)(uint32_t)hc[0]));
    }
    if (hc[1] || (size_t)(uint32_t)hc[0] > ws.tc_rcap) {  // a tile with > kChunkMax chunks: SIMT kernel
      ws.tc_used = 0;
      return run_update_simt<D>(ws, lo, hi, nbr);
    }
    unsigned long long ent_u = 0, pts_u = 0;
    memcpy(&ent_u, hc + 2, sizeof(ent_u));
    memcpy(&pts_u, hc + 4, sizeof(pts_u));
    const double occ = ent_u ? (double)pts_u / (double)ent_u : 1.0;
    if (getenv("EGGSYNC_TC_DEBUG"))
      fprintf(stderr, "[tc-plan] entries=%llu points_in_entries=%llu ratio=%.3f slots=%d overflow=%d padded=%d rcap=%zu tiles=%lld\n",
              ent_u, pts_u, occ, hc[0], hc[1], hc[6], ws.tc_rcap, (long long)owned);
    // Entries holding a few points each on average (partly collapsed clusters) put many
    // multi-point cells in the classifiers' exact band, where one lane scans a cell's points
    // alone; the warp-cooperative SIMT kernel is faster there (measured: C4-d10 iterations
    // 5-7, C4-d5 / C2 late iterations).  Singletons (occ ~ 1) and fully collapsed clusters
    // (occ >= 50: whole-cell summaries) stay on the tensor cores.
    // The slot lists are int32-indexed and cost 4 B per (tile, entry): beyond 2^30 slots
    // (e.g. C5 iteration 1: 2.5e10 entries, 3e12 pairs) the SIMT kernel runs instead; so it
    // does when the tiles average less than one entry tile (a CTA per nearly empty tile:
    // C5 iteration 3, 13 entries per tile, 14 ms vs 2 ms).
    if ((occ > 1.1 && occ < 50.0) || ent_u + (unsigned long long)owned * kTcEnt > (1ull << 30) ||
        ent_u < (unsigned long long)owned * kTcEnt) {
      ws.tc_used = 0;
      return run_update_simt<D>(ws, lo, hi, nbr);
    }
    EGG_TRY(tc_ent_reserve(ws, (size_t)(uint32_t)hc[6] + 1));
    k_tc_expand<0><<<(unsigned)((owned + 3) / 4), 128, 0, ws.stream>>>(ws.tc_ranges, ws.tc_chunks, ws.tc_nr, ws.tc_ne,
                                                                    ws.tc_eoff, ws.tc_ent, (int32_t)owned);
    EGG_CUDA(cudaGetLastError());
    ws.launches += 1;
    // launch order: point tiles by descending entry count (longest-processing-time first)
    {
      size_t stmp = 0;
      EGG_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, stmp, ws.tc_ne, ws.tc_pk, ws.tc_pv, ws.tc_perm,
                                                         (int)owned, 0, 32, ws.stream));
      if (stmp > ws.cub_bytes) {
        set_error("cub scratch too small for the tensor-core tile order");
        return EGGSYNC_ECUDA;
      }
      EGG_CUDA(cub::DeviceRadixSort::SortPairsDescending(ws.cub_tmp, stmp, ws.tc_ne, ws.tc_pk, ws.tc_pv, ws.tc_perm,
                                                         (int)owned, 0, 32, ws.stream));
      ws.launches += 4;
    }

    TcArgs<D> a;
    a.xs = ws.xs[ws.xcur];
    a.xs_next = ws.xs[ws.xcur ^ 1];
    a.sn = ws.sn;
    a.cs = ws.cs;
    a.g_of = ws.g_of;
    a.g_cnt = ws.g_cnt;
    a.c_rec = ws.c_rec;
    a.c_lo = ws.c_lo;
    a.c_hi = ws.c_hi;
    a.ent = ws.tc_ent;
    a.eoff = ws.tc_eoff;
    a.perm = ws.tc_perm;
    a.t_ne = ws.tc_ne;
    a.full_S = ws.full_S;
    a.full_N = ws.full_N;
    a.n = ws.n;
    a.cap = ws.cap;
    a.lo = lo;
    a.hi = hi;
    a.ntiles = (int32_t)owned;
    a.stride = ws.own_stride;
    a.offset = ws.own_offset;
    a.e = ws.k.ef;
    a.e2f = ws.k.e2f;
    a.rel = ws.k.rel;
    a.e2d = ws.k.e2;
    a.flags = ws.flags;
    a.nbr = nbr;
    a.prof = nullptr;
    static unsigned long long* prof = nullptr;
    if (getenv("EGGSYNC_TC_PROF")) {
      if (!prof) EGG_CUDA(cudaMalloc((void**)&prof, 16 * sizeof(unsigned long long)));
      EGG_CUDA(cudaMemsetAsync(prof, 0, 16 * sizeof(unsigned long long), ws.stream));
      a.prof = prof;
    }
    EGG_CUDA(cudaFuncSetAttribute(k_update_tc<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::kSmem));
    if (ws.tc_timing) {
      EGG_TRY(ws.tc_flush());
      const long long pairs = (long long)ent_u * kTcTile, padded = (long long)(uint32_t)hc[6] * kTcTile;
      ws.tc_acc[0] += 1;
      ws.tc_acc[1] += pairs;
      ws.tc_acc[2] += padded;
      // algorithmic tensor-core FLOPs: GEMM1 over the 3D+2 operand columns, GEMM2 over the
      // 2(2D+1) value columns (hi/lo split), per (point, entry) pair
      ws.tc_pend_alg = 2LL * pairs * ((3 * D + 2) + 2 * (2 * D + 1));
      ws.tc_acc[3] += ws.tc_pend_alg;
      EGG_CUDA(cudaEventRecord(ws.tc_ev[0], ws.stream));
    }
    k_update_tc<D><<<(unsigned)owned, kTcThreads, C::kSmem, ws.stream>>>(a);
    EGG_CUDA(cudaGetLastError());
    if (ws.tc_timing) {
      EGG_CUDA(cudaEventRecord(ws.tc_ev[1], ws.stream));
      ws.tc_pending = true;
    }
    if (a.prof) {
      unsigned long long h[16];
      EGG_CUDA(cudaMemcpyAsync(h, prof, sizeof(h), cudaMemcpyDeviceToHost, ws.stream));
      EGG_CUDA(cudaStreamSynchronize(ws.stream));
      const double t = (double)(h[4] ? h[4] : 1);
      fprintf(stderr, "[tc-prof] per entry tile (clk): producer fetch %.0f wait_empty %.0f wait_records %.0f build %.0f | "
              "classifier wait_S %.0f classify %.0f drain %.0f\n", h[0] / t, h[1] / t, h[2] / t, h[3] / t,
              2 * h[5] / t, 2 * h[6] / t, 2 * h[7] / t);
    }
    if (getenv("EGGSYNC_TC_DEBUG")) {
      std::vector<int32_t> h((size_t)owned);
      EGG_CUDA(cudaMemcpyAsync(h.data(), ws.tc_ne, owned * sizeof(int32_t), cudaMemcpyDeviceToHost, ws.stream));
      EGG_CUDA(cudaStreamSynchronize(ws.stream));
      long long ent = 0, tiles = 0, mx = 0;
      for (int32_t v : h) {
        ent += v;
        tiles += (v + kTcEnt - 1) / kTcEnt;
        mx = v > mx ? v : mx;
      }
      fprintf(stderr, "[tc] n=%lld cells=%d owned_tiles=%lld ranges=%d entries=%lld entry_tiles=%lld max_entries=%lld pairs=%lld\n",
              (long long)ws.n, ws.n_cells, (long long)owned, hc[0], ent, tiles, mx, tiles * kTcEnt * kTcTile);
    }
    ws.launches += 1;
    return EGGSYNC_OK;
  }
}

// tensor cores when the dimension fits the TMEM / shared-memory budget and the fp32
// tensor-core count sums stay exact (n < 2^24); EGGSYNC_TC=0 forces the SIMT kernel,
// EGGSYNC_TC=2 the tensor cores also for small cell counts
inline bool tc_enabled(const Workspace& ws, int d) {
  static const int env = [] {
    const char* e = getenv("EGGSYNC_TC");
    return e ? atoi(e) : 1;
  }();
  // (a few thousand cells: fully collapsed clusters, the plan / sync overhead of the
  // tensor-core path exceeds the whole SIMT update)
  return env != 0 && d <= kTcMaxD && ws.n < (int64_t(1) << 24) && (ws.n_cells >= 4096 || env == 2);
}

template <int D>
int run_update(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr) {
  ws.tc_used = 0;
  if (hi <= lo) return EGGSYNC_OK;
  if (tc_enabled(ws, D)) return run_update_tc<D>(ws, lo, hi, nbr);
  return run_update_simt<D>(ws, lo, hi, nbr);
}

}  // namespace egg
