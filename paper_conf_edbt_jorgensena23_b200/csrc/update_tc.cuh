// update_tc.cuh -- A6 EGG-update (Algorithm 3; Eq.5-6) on
// the 5th-generation tensor cores, plus the A7a first-term flag (Alg 3 l.14-15, L252).
//
// The per-point sums of Eq.5,
//   S_i(p) = sum_{q in N_eps(p)} sin(q_i),  C_i(p) = sum_{q in N_eps(p)} cos(q_i),  |N_eps(p)|,
// are computed for a tile of 128 consecutive sorted points at a time as two
// dense contractions against "entries" (update units = cells of the hierarchy):
//
//   GEMM1  S[p][e] = -2 q_p . c'_e - L_e        (kind::f16, x3 hi/lo split of 2^8-scaled values)
//          v = |q_p|^2 + S = |p - c_e|^2 - limF_e   in the tile-shifted frame
//   classify (CUDA cores, one thread per point row of TMEM):
//          v < 0 (sign bit)  -> entry e entirely inside the eps-ball of p (Eq.6 full part)
//          0 <= v <= W_e     -> ambiguous band: exact fp64 re-decision (single point) or
//                               exact scan of the unit's points (Eq.6 partial part)
//          v > W_e           -> outside
//          P[p][e] = -1 (int8) for "inside", else 0, written back into TMEM over S
//   GEMM2  O[p][:] += P[p][:] . V[:][:]        (kind::i8, int32 accumulate: EXACT)
//          V_e = the unit's summary as integers v = round(sum sin/cos * 2^21) and its count,
//          each split into balanced base-256 digits (CellDig, built in k_cell_finalize);
//          N = digits x (2D+1) columns, digits from the largest cell count (3 at C3 iteration 1)
//
// Integer accumulation makes the sums exact and order-independent: no fp32 drain of TMEM,
// one accumulator for both classifier groups, read once in the epilogue.  P as int8 is a
// quarter of the TMEM write traffic of an fp32 mask.
// Entries are the cells of the subtrees that the plan pass (k_tc_plan) could not
// decide for the whole tile; subtrees entirely inside for every point that still
// needs them are added per point in the plan pass (full_S / full_N, exact fp64 of
// the fp32 subtree sums, as in k_update).  k_tc_expand turns each tile's ranges into a slot
// list (one unit per entry, padded to whole entry tiles); tiles are launched heaviest-first.
//
// Roles (512 threads, one CTA per point tile, one CTA per SM: it owns all 512 TMEM columns):
//   warps 0-3   classifier group 0 (TMEM lanes 0..127), even entry tiles
//   warps 4-7   classifier group 1, odd entry tiles
//   warps 8-11  builders: thread t owns entry slot t; from the landed record head it writes the
//               origin-shifted, fp16-split GEMM1 operand row and the band width
//   warp 12     MMA issue (one thread issues GEMM1 and GEMM2 in tile order) and TMEM owner
//   warps 13-15 copy warps: fill the ring stages (up to 8) with per-thread cp.async, all three
//               on every entry tile (slots t, t + 96), up to NST tiles ahead (the gathers by unit
//               index are latency-bound per warp)
// Waiting warps poll one per group and park the others in a named barrier.
// TMEM: Q (K1 columns) | 2-3 S/P buffers of 128 columns | O (N columns, int32).
#pragma once
#include <cub/cub.cuh>

#include <vector>

#include "tc.cuh"
#include "update.cuh"

namespace egg {

constexpr int kTcTile = 128;  // points per tile (TMEM lanes, GEMM M)
constexpr int kTcEnt = 128;   // entries per entry tile (GEMM1 N, GEMM2 K)
constexpr int kProdWarps = 4;  // producers: one entry slot per thread
constexpr int kProd = 32 * kProdWarps;
constexpr int kMmaWarp = 8 + kProdWarps;   // GEMM1 + GEMM2 issue (one thread) + TMEM owner
constexpr int kCopyWarp0 = kMmaWarp + 1;   // stage fills by per-lane cp.async (kCopyWarps warps)
constexpr int kCopyWarps = 3;
constexpr int kTcThreads = (kCopyWarp0 + kCopyWarps) * 32;  // 8 classifier + 4 builder + 1 MMA + 3 copy warps
constexpr int kTcMaxStages = 8;

// |q'|^2 folded into GEMM1 (two more K columns; the classifiers read v directly) or added by
// the classifiers (one FADD per value; K = 3D+2 keeps the stages smaller: more of them fit)
#ifndef EGG_TC_PPFOLD
#define EGG_TC_PPFOLD 1
#endif
constexpr bool kTcPP = EGG_TC_PPFOLD != 0;
template <int D>
struct TcCfg {
  static constexpr int KU = 3 * D + 2 + (kTcPP ? 2 : 0);  // used K columns
  static constexpr int K1 = (KU + 15) / 16 * 16;  // GEMM1 K (fp16): q_hi, q_lo, q_hi, s, s[, pp_hi, pp_lo]
  static constexpr int KSTEPS = K1 / 16;                  // MMA K-steps of GEMM1 (error bound of the band)
  static constexpr int QC = (K1 / 2 + 15) / 16 * 16;      // TMEM columns of Q (two fp16 per column), 16-aligned
  static constexpr int NV = 2 * D + 1;                  // sin, cos, count
  static constexpr int DB = CellDig<D>::kBytes;         // digit row of a cell (GEMM2 N <= DB)
  static constexpr int R = CellRec<D>::kFloats;
  static constexpr int R0 = CellDig<D>::kHead;          // record head: centre, radius, count, start
  static constexpr int kRecBytes = kTcEnt * R0 * 4;   // record heads of a stage's entries, [R0/4][kTcEnt][4]
  // shared memory: ring stages (run-time size, TcStage) | rare sums | misc
  static constexpr int SBO1 = (K1 / 8) * 128;
  static constexpr int kB1Bytes = kTcEnt * K1 * 2;
  static constexpr int kRareBytes = NV * kTcTile * 8;   // exact sums [2D][row] (2^-32) + count [row]
  static constexpr int kMiscBytes = 1024;
  static constexpr int kFixedBytes = kRareBytes + kMiscBytes + 1024;  // +1024 alignment
  static constexpr int kBudget = 227 * 1024;
  __host__ __device__ static constexpr int stage_bytes(int n2) {
    return (kB1Bytes + n2 * kTcEnt + kRecBytes + 8 * kTcEnt + 16 + 127) / 128 * 128;
  }
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
  int32_t* t_pv;              // [ntiles] tile index (values of the launch-order sort)
  int32_t* chunks;            // [ntiles][kChunkMax] first slot of each chunk
  int32_t* t_epad;            // [ntiles] entries padded to whole entry tiles (scan -> slot offsets)
  int32_t* ctr;               // [0] slots allocated, [1] chunk-table overflow, [2..3] entries (u64), [4..5] their points (u64), [6..7] entries padded to whole entry tiles (u64)
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
__global__ void __launch_bounds__(kPlanWarps * 32, 3) k_tc_plan(const PlanArgs<D> a) {
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
  // Two stack entries per step: their node data (box, meta, count) are loaded together, so
  // the walk's dependent global-load chain is half as long (the order of the entries within
  // a tile is immaterial: the update's sums are exact integers).
  int sp = 1;
  while (sp > 0) {
    const int nb = sp >= 2 ? 2 : 1;
    int nodes[2];
    uint32_t mk[2][kP];
#pragma unroll
    for (int b = 0; b < 2; ++b) {
      const int e = b < nb ? sp - 1 - b : sp - 1;
      nodes[b] = stk[e * 8];
#pragma unroll
      for (int k = 0; k < kP; ++k) mk[b][k] = (uint32_t)stk[e * 8 + 1 + k];
    }
    sp -= nb;
    __syncwarp();
    float4 bx[2][BS / 4];
    int4 meta[2];
    int tcn[2];
#pragma unroll
    for (int b = 0; b < 2; ++b) {
      const int nd = nodes[b] & 0x7fffffff;
      const bool internal = b < nb && !(nodes[b] & (int)kLeafBit);
      const float4* __restrict__ src = reinterpret_cast<const float4*>(a.t_box + (int64_t)(internal ? nd : 0) * BS);
#pragma unroll
      for (int k = 0; k < BS / 4; ++k) bx[b][k] = src[k];
      meta[b] = a.t_meta[internal ? nd : 0];
      tcn[b] = internal ? a.t_cnt[nd] : (b < nb ? a.c_cnt[nd] : 0);
    }
    bool overflow = false;
#pragma unroll
    for (int b = 0; b < 2; ++b) {
      if (b >= nb) break;
      const int node = nodes[b];
      if (node & (int)kLeafBit) {  // a single cell: always an entry
        push(node & 0x7fffffff, 1, tcn[b]);
        continue;
      }
      const float* bxf = reinterpret_cast<const float*>(bx[b]);
      float m0[kP], x0[kP];
#pragma unroll
      for (int k = 0; k < kP; ++k) m0[k] = x0[k] = 0.f;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const float blo = bxf[i] - ov[i], bhi = bxf[D + i] - ov[i];
#pragma unroll
        for (int k = 0; k < kP; ++k) {
          const float dl = blo - q[k][i], dh = q[k][i] - bhi;
          const float mn = fmaxf(fmaxf(dl, dh), 0.f), mx = fmaxf(-dl, -dh);
          m0[k] = fmaf(mn, mn, m0[k]);
          x0[k] = fmaf(mx, mx, x0[k]);
        }
      }
      bool full[kP];
      uint32_t pm[kP], fm[kP];
      bool any_part = false;
#pragma unroll
      for (int k = 0; k < kP; ++k) {
        const bool act = (mk[b][k] >> lane) & 1u;
        full[k] = act && x0[k] <= lim_full;
        const bool part = act && !full[k] && m0[k] <= lim_out;
        pm[k] = __ballot_sync(FULLMASK, part);
        fm[k] = __ballot_sync(FULLMASK, full[k]);
        any_part |= pm[k] != 0u;
      }
      if (!any_part) {  // nobody needs to look inside: full points take the subtree summary
        bool anyf = false;
#pragma unroll
        for (int k = 0; k < kP; ++k) anyf |= fm[k] != 0u;
        if (anyf) {
          const float4* __restrict__ sm4 = reinterpret_cast<const float4*>(a.t_sum + (int64_t)node * BS);
          float sm[BS];
#pragma unroll
          for (int k = 0; k < BS / 4; ++k) {
            const float4 t4 = sm4[k];
            sm[4 * k] = t4.x;
            sm[4 * k + 1] = t4.y;
            sm[4 * k + 2] = t4.z;
            sm[4 * k + 3] = t4.w;
          }
#pragma unroll
          for (int k = 0; k < kP; ++k) {
            if (full[k]) {
              N[k] += tcn[b];
              // loads before stores, D at a time: the read-modify-writes overlap (two latencies)
#pragma unroll
              for (int h = 0; h < 2; ++h) {
                double cur[D];
#pragma unroll
                for (int i = 0; i < D; ++i) cur[i] = touched[k] ? a.full_S[(int64_t)(h * D + i) * a.n + j[k]] : 0.0;
#pragma unroll
                for (int i = 0; i < D; ++i) a.full_S[(int64_t)(h * D + i) * a.n + j[k]] = cur[i] + (double)sm[h * D + i];
              }
              touched[k] = true;
            }
          }
        }
        continue;
      }
      const int ncell = meta[b].y - meta[b].x + 1;
      if (ncell <= a.bucket) {
        push(meta[b].x, ncell, tcn[b]);
        continue;
      }
      if (sp + 2 > a.stack_len) {
        overflow = true;
        break;
      }
      if (lane == 0) {
        stk[sp * 8] = meta[b].w;
        stk[(sp + 1) * 8] = meta[b].z;
#pragma unroll
        for (int k = 0; k < kP; ++k) {
          stk[sp * 8 + 1 + k] = (int)(pm[k] | fm[k]);
          stk[(sp + 1) * 8 + 1 + k] = (int)(pm[k] | fm[k]);
        }
      }
      sp += 2;
    }
    if (overflow) {
      if (lane == 0) atomicExch(&a.flags[3], 1);
      break;
    }
    __syncwarp();
  }
  if (lane == 0) {
    a.t_nr[tile] = nr;
    a.t_ne[tile] = ne;
    atomicAdd(reinterpret_cast<unsigned long long*>(a.ctr + 2), (unsigned long long)ne);  // unpadded entries
    atomicAdd(reinterpret_cast<unsigned long long*>(a.ctr + 4), (unsigned long long)npts);
    atomicAdd(reinterpret_cast<unsigned long long*>(a.ctr + 6), (unsigned long long)((ne + kTcEnt - 1) / kTcEnt * kTcEnt));
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
  const uint32_t* __restrict__ orig;  // sharded runs: original local index (own iff < n_own), else nullptr
  int64_t n_own;
  const float* __restrict__ xs;
  float* __restrict__ xs_next;
  const float* __restrict__ sn;
  const float* __restrict__ cs;
  const int32_t* __restrict__ g_of;
  const int32_t* __restrict__ g_cnt;
  const float* __restrict__ c_rec;
  const int8_t* __restrict__ c_dig;   // [cap][CellDig::kStride] digit rows
  const float* __restrict__ c_head;   // [cap][CellDig::kHeadS] record heads
  const int32_t* __restrict__ cell_of;  // unit of each sorted point
  const uint32_t* __restrict__ c_lo;
  const uint32_t* __restrict__ c_hi;
  const int32_t* __restrict__ ent;    // unit of every entry slot (-1 = padding), k_tc_expand
  const int32_t* __restrict__ eoff;   // [ntiles] first slot of each point tile
  const int32_t* __restrict__ perm;   // [ntiles] launch order
  const int32_t* __restrict__ t_ne;
  const double* __restrict__ full_S;
  const int32_t* __restrict__ full_N;
  int64_t n, cap, lo, hi;
  int32_t ntiles, stride, offset;
  int32_t ndig, n2, nst, ns;   // digits per value, GEMM2 N, ring stages, S buffers (run-time layout)
  int32_t stage_bytes;
  float e, e2f, rel;
  double e2d;
  int32_t* flags;
  int32_t* nbr;
  unsigned long long* prof;  // EGG_TC_PROF builds: [16] cycle sums
};

// shared-memory header of the TC kernel
struct TcMisc {
  uint64_t stage_landed[kTcMaxStages], stage_full[kTcMaxStages], stage_empty[kTcMaxStages];
  uint64_t s_full[3], p_full[3], o_done;
  uint32_t tbase;
  float o[kTcMaxD];
  float lo[4][kTcMaxD], hi[4][kTcMaxD];
  float Rq, Rqi;
};
static_assert(sizeof(TcMisc) <= 1024, "misc header");

// per-thread asynchronous 16-byte global -> shared copies (L2 only), waited per thread
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(tc::smem_addr(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// One ring stage (run-time size: GEMM2 N = n2 depends on the digits needed):
//   b1   [kTcEnt][K1] fp16, K-major core matrices (GEMM1 B: entry rows)            (producers)
//   b2   [n2/16][kTcEnt][16] int8, MN-major core matrices (GEMM2 B: digits x entries) (cp.async)
//   rec  [R0/4][kTcEnt][4] record heads, block-major like c_head: centre (= the point of a
//        singleton), radius, count, start                                              (TMA)
//   W [kTcEnt] band width of every slot, wmax[4]                                       (builders)
//   cell [kTcEnt] unit of every slot (-1 = padding): the tile's slot list              (TMA)
template <int D>
struct TcStage {
  float* b1;
  int8_t* b2;
  float* rec;
  float* W;
  int32_t* cell;
  float* wmax;
  __device__ TcStage(unsigned char* ring, int s, int stage_bytes, int n2) {
    using C = TcCfg<D>;
    unsigned char* p = ring + (size_t)s * stage_bytes;
    b1 = reinterpret_cast<float*>(p);
    b2 = reinterpret_cast<int8_t*>(p + C::kB1Bytes);
    rec = reinterpret_cast<float*>(p + C::kB1Bytes + n2 * kTcEnt);
    unsigned char* m = p + C::kB1Bytes + n2 * kTcEnt + C::kRecBytes;
    W = reinterpret_cast<float*>(m);
    cell = reinterpret_cast<int32_t*>(m + 4 * kTcEnt);
    wmax = reinterpret_cast<float*>(m + 8 * kTcEnt);
  }
  __device__ float hf(int e, int i) const { return rec[((i >> 2) * kTcEnt + e) * 4 + (i & 3)]; }
  __device__ int32_t cnt(int e) const { return __float_as_int(hf(e, D + 1)); }
  __device__ int32_t start(int e) const { return __float_as_int(hf(e, D + 2)); }
  __device__ float pt(int e, int i) const { return hf(e, i); }
};

// Exact path for a multi-point unit e inside the band of point pe (P stays 0 for the pair):
// refine with the unit's exact MBR, then its points one by one (fp32 + fp64 re-decision as
// in k_update).  Sums go into the row's exact fixed-point (2^-32) sums in shared memory
// (64-bit shared atomics: both classifier groups may add to the same row).
__device__ __forceinline__ void rare_add(unsigned long long* rare, int i, int row, double v) {
  atomicAdd(&rare[i * kTcTile + row], (unsigned long long)llrint(v * kFix));
}
template <int D>
__device__ __forceinline__ void tc_rare(const TcArgs<D>& a, const float* __restrict__ pe, int e,
                                     const TcStage<D>& st, unsigned long long* __restrict__ rare, int row) {
  const int32_t c = st.cell[e];
  const int32_t cnt = st.cnt(e);
  const int32_t start = st.start(e);
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
    bool in = maxd <= lim_in || d2 <= lim_in;
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
  if (nin) atomicAdd(&rare[2 * D * kTcTile + row], nin);
}

// Build entry slot `pt` (unit c, or padding when c < 0) of a stage: B1 row and metadata from
// the unit's record head (prefetched into registers); its digit row (B2) came by cp.async.
// GEMM1 runs in fp16 on values scaled by kTcScale = 2^8 (the products and v by 2^16): shifted
// coordinates |c'|, |q'| <= 1 become <= 256 (fp16 max 65504), their low halves stay normal.
constexpr float kTcScale = 256.f;
constexpr float kTcScale2 = 65536.f;

template <int D>
__device__ __forceinline__ float tc_build_entry(const TcArgs<D>& a, const float (&o)[D],
                                                const TcStage<D>& st, int pt, int32_t c, float Rq, float Rqi) {
  // branchless: a padding slot computes on whatever its record holds and selects the padding
  // row at the end
  using C = TcCfg<D>;
  constexpr int K1 = C::K1;
  const bool real = c >= 0;
  float r[C::R0];
  const float4* r4 = reinterpret_cast<const float4*>(st.rec);  // landed by cp.async, block-major
#pragma unroll
  for (int k = 0; k < C::R0 / 4; ++k) {
    const float4 t4 = r4[k * kTcEnt + pt];
    r[4 * k] = t4.x;
    r[4 * k + 1] = t4.y;
    r[4 * k + 2] = t4.z;
    r[4 * k + 3] = t4.w;
  }
  __half hb[K1];  // B1 row: c'_hi, c'_hi, c'_lo, -L_hi, -L_lo, 2^8, 2^8, 0... (A carries the -2)
  float cc0 = 0.f, cc1 = 0.f, cinf = 0.f;  // two independent chains (latency)
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const float cp = r[i] - o[i];
    const float x = cp * kTcScale;
    const __half h = __float2half_rn(x);
    const __half l = __float2half_rn(x - __half2float(h));
    hb[i] = h;
    hb[D + i] = h;
    hb[2 * D + i] = l;
    if (i & 1) cc1 = fmaf(cp, cp, cc1);
    else cc0 = fmaf(cp, cp, cc0);
    cinf = fmaxf(cinf, fabsf(cp));
  }
  const float cc = cc0 + cc1;
  const float rad = r[D];
  // error budget: eta = rounding of the shifted frame; E bounds |v - v_exact|:
  //   fp16 split of -2 q.c' (round-to-nearest hi, lo rounded again, lo*lo dropped):
  //     <= 2 * 3 * 2^-22 sum|q_i||c'_i| <= 2^-19.4 |q||c'|               (Cauchy-Schwarz)
  //   tensor-core accumulation, KSTEPS K-steps of 16 products + accumulator, each truncating
  //     <= 17 * 2^-23 of the sum of |terms| (2|q||c'| + |L| + |q|^2): acc = KSTEPS * 17 * 2^-23
  //   L = limF - |c'|^2 and |q|^2 split hi/lo (2^-22 each); fp32 |q|^2, |c'|^2 (D FMAs):
  //     (D+2) u (|q|^2 + cc) <= 2^-20 (|q|^2 + cc)
  //   => E <= (2^-19.4 + 2 acc) Rq|c'| + (2^-22 + acc)(|L| + Rq^2) + 2^-20 (Rq^2 + cc)
  //      (Rq >= |q|, D <= 12); coefficients rounded up by 1%; unscaled
  const float eta = 2.5f * kU * sqrtf((float)D) * (Rqi + cinf);
  const float ep = (a.e + rad) * (1.f + 8.f * kU) + eta;
  const float em = (a.e - rad) * (1.f - 8.f * kU) - eta;
  const float limF0 = em > 0.f ? em * em * (1.f - 4.f * kU) : -1.f;
  constexpr float acc = (float)C::KSTEPS * 17.f * 1.1920928955078125e-07f;
  constexpr float e1 = 1.01f * (1.4505753e-06f + 2.f * acc);  // 2^-19.4 = 6 * 2^-22
  constexpr float e2 = 1.01f * (2.384185791015625e-07f + acc);
  const float E = e1 * (Rq * sqrtf(cc)) + e2 * (fabsf(limF0 - cc) + Rq * Rq) +
                  9.5367431640625e-07f * (cc + Rq * Rq) + 1e-30f;
  const float limF = em > 0.f ? limF0 - E : -1.f;
  const float limO = ep * ep * (1.f + 4.f * kU) + E;
  const float W = real ? (limO - limF) * (1.f + 4.f * kU) * kTcScale2 : 0.f;  // in the scaled units of v
  const float xL = -(limF - cc) * kTcScale;  // times A's s = 2^8 column: -L * 2^16
  const __half Lh = __float2half_rn(xL);
  hb[3 * D] = Lh;
  hb[3 * D + 1] = __float2half_rn(xL - __half2float(Lh));
  if constexpr (kTcPP) {
    hb[3 * D + 2] = __float2half_rn(kTcScale);  // times A's 2^8-scaled |q'|^2 halves: + |q'|^2 * 2^16
    hb[3 * D + 3] = __float2half_rn(kTcScale);
  }
#pragma unroll
  for (int k = C::KU; k < K1; ++k) hb[k] = __float2half_rn(0.f);
  if (!real) {  // padding: v = 2^8 * 60000 + |q'|^2 2^16, far outside, never ambiguous (selects)
#pragma unroll
    for (int k = 0; k < 3 * D + 2; ++k) hb[k] = __float2half_rn(k == 3 * D ? 60000.f : 0.f);
  }
  // B1: K-major fp16, entry rows (8 K-values per 16-byte core-matrix row)
  unsigned char* b1 = reinterpret_cast<unsigned char*>(st.b1) + (pt >> 3) * C::SBO1 + (pt & 7) * 16;
#pragma unroll
  for (int kc = 0; kc < K1 / 8; ++kc) {
    uint32_t w[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const __half2 h2 = __halves2half2(hb[8 * kc + 2 * q], hb[8 * kc + 2 * q + 1]);
      w[q] = *reinterpret_cast<const uint32_t*>(&h2);
    }
    *reinterpret_cast<uint4*>(b1 + kc * 128) = make_uint4(w[0], w[1], w[2], w[3]);
  }
  st.W[pt] = W;
  return W;
}

// Development-only cycle accounting (-DEGG_TC_PROF): per-role waits / work summed over CTAs
#ifdef EGG_TC_PROF
#define TCP_T(v) const long long v = clock64()
#define TCP_ADD(k, d) prof_acc[k] += (unsigned long long)(d)
#else
#define TCP_T(v)
#define TCP_ADD(k, d)
#endif

// (t % n, (t / n) & 1) of a ring position t, maintained incrementally (no integer division)
struct RingPos {
  int i = 0;
  uint32_t ph = 0;
  __device__ __forceinline__ void adv(int n) {
    if (++i == n) {
      i = 0;
      ph ^= 1u;
    }
  }
};

// sign bits of four fp32 values -> four int8 mask bytes (0xFF where the value is negative / -0)
// (prmt's default mode: a selector nibble with bit 3 set replicates the selected byte's sign)
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
  uint32_t r;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
  return r;
}
__device__ __forceinline__ uint32_t sign_bytes4(uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  const uint32_t x = prmt(a, b, 0x00FBu);  // [sgn(a.b3), sgn(b.b3), ., .]
  const uint32_t y = prmt(c, d, 0x00FBu);
  return prmt(x, y, 0x5410u);
}

template <int D>
// registers: warps are dealt round-robin to the 4 SM sub-partitions (16K registers each)
__global__ void __launch_bounds__((kTcThreads + 127) / 128 * 128, 1) k_update_tc(const TcArgs<D> a) {
  using C = TcCfg<D>;
  constexpr int K1 = C::K1, NV = C::NV, R0 = C::R0;
  extern __shared__ __align__(16) unsigned char tsm_raw[];
  unsigned char* tsm = tsm_raw + ((1024u - (tc::smem_addr(tsm_raw) & 1023u)) & 1023u);
  const int NST = a.nst, NS = a.ns, SB = a.stage_bytes, N2 = a.n2;
  unsigned char* ring = tsm;
  unsigned long long* rare = reinterpret_cast<unsigned long long*>(tsm + (size_t)NST * SB);
  TcMisc* ms = reinterpret_cast<TcMisc*>(tsm + (size_t)NST * SB + C::kRareBytes);

  const int tid = threadIdx.x, wid = tid >> 5, lane = tid & 31;
  const int64_t tile = a.perm[blockIdx.x];  // heaviest point tiles first (shorter tail)
  const int64_t base = tc_tile_base(a.lo, tile, a.stride, a.offset);
  const int32_t ne = a.t_ne[tile];
  const int T = (ne + kTcEnt - 1) / kTcEnt;  // entry tiles (the slot list is padded to T * kTcEnt)
  const int kColS = C::QC, kColO = C::QC + NS * kTcEnt;
#ifdef EGG_TC_PROF
  unsigned long long prof_acc[6] = {0, 0, 0, 0, 0, 0};
#endif

  // ---- setup -------------------------------------------------------------------------
  if (tid == 0) {
    for (int s = 0; s < NST; ++s) {
      tc::bar_init(&ms->stage_landed[s], 32 * kCopyWarps);  // one cp.async-completion arrival per copy thread
      tc::bar_init(&ms->stage_full[s], kProd);   // one arrival per builder thread (entry slot)
      tc::bar_init(&ms->stage_empty[s], 1);
    }
    for (int b = 0; b < NS; ++b) {
      tc::bar_init(&ms->s_full[b], 1);
      tc::bar_init(&ms->p_full[b], kTcTile);
    }
    tc::bar_init(&ms->o_done, 1);
    tc::bar_fence_init();
  }
  if (wid == kMmaWarp) tc::tmem_alloc<512>(&ms->tbase);
  for (int t = tid; t < NV * kTcTile; t += kTcThreads) rare[t] = 0ull;

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
    ms->o[tid] = 0.5f * (l + h);
  }
  if (tid == 0) {
    ms->Rq = 0.f;
    ms->Rqi = 0.f;
  }
  __syncthreads();
  float pp = 3.0e38f;  // |q'|^2 (invalid rows never classify inside or ambiguous)
  if (is_cls) {
    float q[D];
    float s = 0.f, rinf = 0.f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      q[i] = valid ? pe[i] - ms->o[i] : 0.f;
      s = fmaf(q[i], q[i], s);
      rinf = fmaxf(rinf, fabsf(q[i]));
    }
    if (valid) pp = s * kTcScale2;  // (!kTcPP) v = S + |q'|^2, in the scaled units of GEMM1
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
      // Q row -> TMEM columns [0, K1/2) as fp16 pairs (scaled by 2^8): q_hi, q_lo, q_hi, s, s, 0...
      float v[K1];
#pragma unroll
      for (int i = 0; i < D; ++i) {  // -2 q' halves (exact scaling): B carries c' unscaled
        float h, l;
        tc::split_h(q[i] * kTcScale, h, l);
        v[i] = -2.f * h;
        v[D + i] = -2.f * l;
        v[2 * D + i] = -2.f * h;
      }
      v[3 * D] = kTcScale;
      v[3 * D + 1] = kTcScale;
      // |q'|^2 (scaled by 2^8; B's 2^8 columns make it |q'|^2 * 2^16 in v): the GEMM forms
      // v = |p - c_e|^2 - limF_e directly.  Invalid rows: 60000 * 2^8, never inside or ambiguous.
      if constexpr (kTcPP) {
        if (valid) {
          tc::split_h(s * kTcScale, v[3 * D + 2], v[3 * D + 3]);
        } else {
          v[3 * D + 2] = 60000.f;
          v[3 * D + 3] = 0.f;
        }
      }
#pragma unroll
      for (int k = C::KU; k < K1; ++k) v[k] = 0.f;
      const uint32_t taddr = ms->tbase + ((uint32_t)(32 * (wid & 3)) << 16);
#pragma unroll
      for (int c = 0; c < K1 / 16; ++c) {
        uint32_t w8[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) w8[k] = tc::pack_h2(v[16 * c + 2 * k], v[16 * c + 2 * k + 1]);
        tc::st8(taddr + 8 * c, w8);
      }
      tc::wait_st();
    }
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tb = ms->tbase;

  if (wid >= 8 && wid < 8 + kProdWarps) {
    // ================================ builders ================================
    // Thread pt builds entry slot pt of every entry tile from the record head the copy warp
    // landed: the origin-shifted, fp16-split GEMM1 operand row and the band width W.
    const int pt = tid - 256;  // entry slot 0..127
    const float Rq = ms->Rq, Rqi = ms->Rqi;
    float ov[D];  // tile origin, in registers for the operand builds
#pragma unroll
    for (int i = 0; i < D; ++i) ov[i] = ms->o[i];
    RingPos bp;
    for (int jt = 0; jt < T; ++jt) {
      TCP_T(p0);
      if (wid == 8) tc::bar_poll(&ms->stage_landed[bp.i], bp.ph);
      tc::named_sync(3, kProd);
      TCP_T(p1);
      TcStage<D> st(ring, bp.i, SB, N2);
      const float W = tc_build_entry<D>(a, ov, st, pt, st.cell[pt], Rq, Rqi);
      // chunk maximum of the band widths (W >= 0: its bits order as unsigned integers)
      const uint32_t wm = __reduce_max_sync(FULLMASK, __float_as_uint(W));
      if (lane == 0) st.wmax[pt >> 5] = __uint_as_float(wm);
      tc::fence_proxy_async();
      tc::bar_arrive(&ms->stage_full[bp.i]);
      bp.adv(NST);
      TCP_T(p2);
      TCP_ADD(0, p1 - p0);
      TCP_ADD(1, p2 - p1);
    }
  }

  if (wid >= kCopyWarp0) {
    // ================================ copy warps ================================
    // The copy warps (96 threads) fill the stage of every entry tile together, up to NST tiles
    // ahead: thread t copies slots t and t + 96 -- the slot's unit (slot list), its record head
    // and its digit row, by 16-byte cp.async (block-major global layouts: consecutive threads
    // read consecutive units of a run, so the copies coalesce) -- and the tile's 512 B of slot
    // units come from threads 0..31.  Splitting every tile over all copy threads keeps the time
    // from a stage's release to its refill short (the gathers are latency-bound per warp).
    // Each thread's completion arrives on stage_landed (cp.async.mbarrier.arrive.noinc).
    constexpr int NH = R0 / 4;
    constexpr int kCT = 32 * kCopyWarps;  // copy threads
    const int nchunk = N2 / 16;
    const int ct = tid - 32 * kCopyWarp0;
    const int32_t* __restrict__ ent = a.ent + a.eoff[tile];  // 512-byte aligned (padded tiles)
    const char* __restrict__ hb = reinterpret_cast<const char*>(a.c_head);
    const char* __restrict__ db = reinterpret_cast<const char*>(a.c_dig);
    const int64_t capB = a.cap * 16;  // bytes of one 16-byte block column
    constexpr int kSl = (kTcEnt + kCT - 1) / kCT;  // slots per copy thread
    int cn[kSl];
#pragma unroll
    for (int j = 0; j < kSl; ++j) cn[j] = (T > 0 && ct + kCT * j < kTcEnt) ? ent[ct + kCT * j] : -1;
    RingPos fp;
    for (int t = 0; t < T; ++t) {
      int cu[kSl];
#pragma unroll
      for (int j = 0; j < kSl; ++j) cu[j] = cn[j];
      if (t + 1 < T) {
#pragma unroll
        for (int j = 0; j < kSl; ++j)
          cn[j] = ct + kCT * j < kTcEnt ? ent[(int64_t)(t + 1) * kTcEnt + ct + kCT * j] : -1;
      }
      TCP_T(f0);
      if (t >= NST) {
        if (ct == 0) tc::bar_poll(&ms->stage_empty[fp.i], fp.ph ^ 1u);
        tc::named_sync(4, kCT);
      }
      TCP_T(f1);
      TcStage<D> st(ring, fp.i, SB, N2);
      if (ct < 32) cp_async16(st.cell + 4 * ct, ent + (int64_t)t * kTcEnt + 4 * ct);
#pragma unroll
      for (int j = 0; j < kSl; ++j) {
        const int c = cu[j];
        if (c >= 0) {
          const int e = ct + kCT * j;
          const char* hs = hb + (int64_t)c * 16;
#pragma unroll
          for (int k = 0; k < NH; ++k) cp_async16(st.rec + ((size_t)k * kTcEnt + e) * 4, hs + k * capB);
          const char* ds = db + (int64_t)c * 16;
          int8_t* dd = st.b2 + e * 16;
#pragma unroll
          for (int k = 0; k < C::DB / 16; ++k)
            if (k < nchunk) cp_async16(dd + k * (16 * kTcEnt), ds + k * capB);
        }
      }
      asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(tc::smem_addr(&ms->stage_landed[fp.i]))
                   : "memory");
      fp.adv(NST);
      TCP_T(f2);
      TCP_ADD(0, f2 - f1);
      TCP_ADD(1, f1 - f0);
    }
    cp_async_wait<0>();
  }

  if (wid == kMmaWarp && lane == 0) {
    // ================================ MMA issue ================================
    // One thread issues both GEMMs in tile order: GEMM1(g1) = Q . B1(g1)^T into S[g1 % NS]
    // once stage g1 is built and GEMM2(g1 - NS) has been issued (same-thread tcgen05.mma run
    // in issue order, so that GEMM2 has read P before GEMM1 overwrites the buffer); GEMM2(g2):
    // O += P(g2) . B2(g2)^T (int8 x int8 -> int32, exact) once a classifier group wrote P.
    constexpr uint32_t id1 = tc::idesc_f16(128, kTcEnt);
    const uint32_t id2 = tc::idesc_s8(128, N2, true);
    const uint32_t ring_s = tc::smem_addr(ring);
    RingPos s1, b1q, s2, b2q;
    int g1 = 0, g2 = 0;
    while (g2 < T) {
      bool did = false;
      if (g1 < T && g1 - g2 < NS && tc::bar_test(&ms->stage_full[s1.i], s1.ph)) {
        tc::fence_after();
        const uint32_t b1 = ring_s + s1.i * SB;
#pragma unroll
        for (int k = 0; k < K1 / 16; ++k)  // 16 fp16 K-values per MMA: 8 TMEM columns of A, 2 core matrices of B
          tc::mma_ts_f16(tb + kColS + kTcEnt * b1q.i, tb + 8 * k, tc::sdesc(b1 + k * 256, 128, C::SBO1), id1, k > 0);
        tc::mma_commit(&ms->s_full[b1q.i]);
        s1.adv(NST);
        b1q.adv(NS);
        ++g1;
        did = true;
      }
      if (g2 < g1 && tc::bar_test(&ms->p_full[b2q.i], b2q.ph)) {
        tc::fence_after();
        const uint32_t b2 = ring_s + s2.i * SB + C::kB1Bytes;
#pragma unroll
        for (int k = 0; k < kTcEnt / 32; ++k)
          tc::mma_ts_s8(tb + kColO, tb + kColS + kTcEnt * b2q.i + 8 * k, tc::sdesc(b2 + k * 512, 128, 16 * kTcEnt), id2,
                        (g2 > 0) || (k > 0));
        tc::mma_commit(&ms->stage_empty[s2.i]);
        s2.adv(NST);
        b2q.adv(NS);
        ++g2;
        did = true;
      }
      if (!did) __nanosleep(20);
    }
    tc::mma_commit(&ms->o_done);
  }

  if (is_cls) {
    // ================================ classifiers ================================
    const uint32_t lane_off = (uint32_t)(32 * (wid & 3)) << 16;
    const float lim_in = a.e2f * (1.f - a.rel), lim_out = a.e2f * (1.f + a.rel);
    RingPos sp, bq;  // stage / S buffer of tile jt = 2 kk + grp
    if (grp) {
      sp.adv(NST);
      bq.adv(NS);
    }
    for (int jt = grp; jt < T; jt += 2) {
      const int s = sp.i, b = bq.i;
      TcStage<D> st(ring, s, SB, N2);
      TCP_T(c0);
      // one polling warp per group; the other three sleep in the group's named barrier (the
      // poller's acquire + the barrier order their TMEM reads after the MMA, with fence_after)
      if ((wid & 3) == 0) tc::bar_poll(&ms->s_full[b], bq.ph);
      tc::named_sync(1 + grp, kTcTile);
      TCP_T(c1);
      TCP_ADD(0, c1 - c0);
      tc::fence_after();
      const uint32_t sb = tb + lane_off + kColS + kTcEnt * b;
      // four chunks of 32 entries, software-pipelined: the TMEM load of chunk c+1 is in flight
      // while chunk c is classified
      uint32_t v[2][32];
      tc::ld32(sb, v[0]);
      TCP_T(l0);
      tc::wait_ld_regs(v[0]);
      TCP_T(l1);
      TCP_ADD(1, l1 - l0);
#pragma unroll
      for (int c = 0; c < kTcEnt / 32; ++c) {
        const int h = c & 1;
        if (c + 1 < kTcEnt / 32) tc::ld32(sb + 32 * (c + 1), v[h ^ 1]);
        uint32_t pw[8];
        {
          const uint32_t wm = __float_as_uint(st.wmax[c]);
          uint32_t mn = 0xFFFFFFFFu;
#pragma unroll
          for (int jx = 0; jx < 32; ++jx) {
            if constexpr (!kTcPP) v[h][jx] = __float_as_uint(__uint_as_float(v[h][jx]) + pp);  // |p-c|^2 - limF
            mn = min(mn, v[h][jx]);  // unsigned: negative values (inside) compare large
          }
#pragma unroll
          for (int w = 0; w < 8; ++w)
            pw[w] = sign_bytes4(v[h][4 * w], v[h][4 * w + 1], v[h][4 * w + 2], v[h][4 * w + 3]);
          TCP_T(b0);
          if (mn < wm) {  // some pair of this chunk may lie in a band (0 <= f <= max W): exact decisions
            uint32_t bm = 0u;
#pragma unroll
            for (int jx = 0; jx < 32; ++jx) bm |= (v[h][jx] < wm) ? (1u << jx) : 0u;
            uint32_t fm = 0u;  // band pairs decided inside (single points)
            while (bm) {
              const int jx = __ffs(bm) - 1;
              bm &= bm - 1u;
              const int e = 32 * c + jx;
              if (st.cnt(e) == 1) {
                float qc[D];
#pragma unroll
                for (int i = 0; i < D; ++i) qc[i] = st.pt(e, i);
                // a single point: fp32 distance from the exact coordinates decides unless it lies
                // within the (4D+16)u margin of eps^2 (as k_update); there Def. of N_eps (L66)
                // exactly as the oracle: fp64, dimension order
                float d2 = 0.f;
#pragma unroll
                for (int i = 0; i < D; ++i) {
                  const float u = qc[i] - pe[i];
                  d2 = fmaf(u, u, d2);
                }
                bool in = d2 <= lim_in;
                if (!in && d2 <= lim_out) {
                  double s2 = 0.0;
#pragma unroll
                  for (int i = 0; i < D; ++i) {
                    const double t = __dsub_rn((double)qc[i], (double)pe[i]);
                    s2 = __dadd_rn(s2, __dmul_rn(t, t));
                  }
                  in = s2 <= a.e2d;
                }
                if (in) fm |= 1u << jx;
              } else {
                tc_rare<D>(a, pe, e, st, rare, row);
              }
            }
#pragma unroll
            for (int w = 0; w < 8; ++w) {
              const uint32_t f4 = (fm >> (4 * w)) & 0xFu;
              pw[w] |= (f4 & 1u ? 0xFFu : 0u) | (f4 & 2u ? 0xFF00u : 0u) | (f4 & 4u ? 0xFF0000u : 0u) |
                       (f4 & 8u ? 0xFF000000u : 0u);
            }
          }
          TCP_T(b1);
          TCP_ADD(2, b1 - b0);
        }
        tc::st8(sb + 8 * c, pw);  // P (int8, -1 = inside) over S columns 0..31, already read
        if (c + 1 < kTcEnt / 32) tc::wait_ld_regs(v[h ^ 1]);
      }
      TCP_T(w0);
      tc::wait_st();
      TCP_T(w1);
      TCP_ADD(3, w1 - w0);
      tc::fence_before();
      tc::bar_arrive(&ms->p_full[b]);
      sp.adv(NST);
      sp.adv(NST);
      bq.adv(NS);
      bq.adv(NS);
    }
  }
#ifdef EGG_TC_PROF
  // one reporting thread per role: classifiers 0 / 128, producer 256, GEMM1 / GEMM2 issuers
  {
    int slot = -1;
    if (tid == 0 || tid == 128) slot = 0;
    else if (tid == 256) slot = 4;
    else if (tid == 32 * kCopyWarp0) slot = 10;
    if (slot >= 0 && a.prof) {
      const int nk = slot == 12 ? 1 : slot == 0 ? 4 : 2;
      for (int k = 0; k < nk; ++k) atomicAdd(&a.prof[slot + k], prof_acc[k]);
    }
    if (tid == 0 && a.prof) atomicAdd(&a.prof[15], (unsigned long long)T);
  }
#endif

  // ---- epilogue (group 0 rows): Eq.5 in fp64 from the exact integer sums ----------------
  __syncthreads();  // every role done issuing / classifying
  if (is_cls && grp == 0) {
    tc::bar_sleep(&ms->o_done, 0);
    tc::fence_after();
    if (T > 0) {
      // O[k*NV + jv] = -(sum over inside entries of digit k of value jv): fold into the row's
      // fixed-point sums (mod 2^64 arithmetic: exact since every total fits in int64)
      const uint32_t lane_off = (uint32_t)(32 * (wid & 3)) << 16;
      const int used = a.ndig * NV;
      for (int c16 = 0; c16 < N2 / 16; ++c16) {
        uint32_t v[16];
        tc::ld16(tb + lane_off + kColO + 16 * c16, v);
        tc::wait_ld();
#pragma unroll
        for (int jx = 0; jx < 16; ++jx) {
          const int col = 16 * c16 + jx;
          if (col < used) {
            const int k = col / NV, jv = col - k * NV;
            const unsigned long long t = (unsigned long long)(long long)(int32_t)v[jx];
            const int sh = jv < 2 * D ? 8 * k + (32 - kDigF) : 8 * k;
            rare[jv * kTcTile + row] -= t << sh;
          }
        }
      }
    }
    if (valid) {
      auto fx = [&](int k) { return (long long)rare[k * kTcTile + row]; };
      const int64_t Ni = fx(2 * D) + (int64_t)a.full_N[j];
      const double inv = 1.0 / (double)Ni;
#pragma unroll
      for (int i = 0; i < D; ++i) {
        const double S = (double)fx(i) * kInvFix + a.full_S[(int64_t)i * a.n + j];
        const double Cc = (double)fx(D + i) * kInvFix + a.full_S[(int64_t)(D + i) * a.n + j];
        double sx, cx;
        const double x = (double)pe[i];
        sincos(x, &sx, &cx);
        const double xn = x + (cx * S - sx * Cc) * inv;  // Eq.5
        // x' lies in the range of N(p) (L104) and so in [0,1]; the 2^-21 fixed point of the
        // summaries can put it an ulp or two outside, which the clamp removes (domain, L70)
        a.xs_next[(int64_t)i * a.n + j] = fminf(fmaxf((float)xn, 0.f), 1.f);
      }
      const bool f1 = Ni == (int64_t)a.g_cnt[a.g_of[j]];  // Alg 3 l.14-15 (L248)
      if (!f1 && (!a.orig || a.orig[j] < (uint32_t)a.n_own)) atomicAnd(&a.flags[0], 0);
      if (a.nbr) a.nbr[j] = (int32_t)Ni;
    }
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
int run_planned_tc(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr, int64_t owned);
inline bool tc_choose(const long long* g);

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
    if (ws.tc_mode == 2) return run_planned_tc<D>(ws, lo, hi, nbr, owned);
    if (owned == 0) {
      for (auto& v : ws.tc_local) v = 0;
      ws.tc_local[5] = 1;
      ws.tc_pad = 0;
      return EGGSYNC_OK;
    }
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
    p.t_pv = ws.tc_pv;
    // the range buffer keeps its size across updates (process cache); a first guess of
    // 16 chunks per tile, grown and re-planned when the plan reports more
    EGG_TRY(tc_ranges_reserve(ws, (size_t)owned * 16 * kRangeChunk));
    p.t_epad = ws.tc_epad;
    size_t tmp = 0;
    EGG_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, ws.tc_epad, ws.tc_eoff, (int)owned + 1, ws.stream));
    if (tmp > ws.cub_bytes) {
      set_error("cub scratch too small for the tensor-core plan scan");
      return EGGSYNC_ECUDA;
    }
    int32_t hc[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};  // ctr[0..7] (padded entries at 6..7), largest cell count
    for (int attempt = 0; attempt < 2; ++attempt) {
      p.ranges = ws.tc_ranges;
      p.rcap = (int64_t)ws.tc_rcap;
      EGG_CUDA(cudaMemsetAsync(ws.tc_ctr, 0, 8 * sizeof(int32_t), ws.stream));
      EGG_CUDA(cudaMemsetAsync(ws.tc_epad + owned, 0, sizeof(int32_t), ws.stream));
      k_tc_plan<D><<<pgrid, kPlanWarps * 32, psmem, ws.stream>>>(p);
      EGG_CUDA(cudaGetLastError());
      EGG_CUDA(cub::DeviceScan::ExclusiveSum(ws.cub_tmp, tmp, ws.tc_epad, ws.tc_eoff, (int)owned + 1, ws.stream));
      ws.launches += 2;
      EGG_CUDA(cudaMemcpyAsync(hc, ws.tc_ctr, 8 * sizeof(int32_t), cudaMemcpyDeviceToHost, ws.stream));
      EGG_CUDA(cudaMemcpyAsync(hc + 8, ws.flags + 5, sizeof(int32_t), cudaMemcpyDeviceToHost, ws.stream));
      EGG_CUDA(cudaStreamSynchronize(ws.stream));
      ws.launches += 1;
      if (hc[1] || (size_t)(uint32_t)hc[0] <= ws.tc_rcap) break;
      EGG_TRY(tc_ranges_reserve(ws, (size_t)(uint32_t)hc[0]));
    }
    unsigned long long ent_u = 0, pts_u = 0, pad_u = 0;
    memcpy(&ent_u, hc + 2, sizeof(ent_u));
    memcpy(&pts_u, hc + 4, sizeof(pts_u));
    memcpy(&pad_u, hc + 6, sizeof(pad_u));
    // a tile with > kChunkMax chunks, or a range buffer still too small: the plan is unusable
    const bool overflow = hc[1] || (size_t)(uint32_t)hc[0] > ws.tc_rcap;
    ws.tc_local[0] = (long long)ent_u;
    ws.tc_local[1] = (long long)pts_u;
    ws.tc_local[2] = owned;
    ws.tc_local[3] = overflow ? 1 : 0;
    ws.tc_local[4] = hc[8];
    ws.tc_local[5] = 1;
    ws.tc_pad = (long long)pad_u;
    if (getenv("EGGSYNC_TC_DEBUG"))
      fprintf(stderr, "[tc-plan] entries=%llu points_in_entries=%llu slots=%d overflow=%d padded=%d rcap=%zu tiles=%lld\n",
              ent_u, pts_u, hc[0], hc[1], (int)pad_u, ws.tc_rcap, (long long)owned);
    if (ws.tc_mode == 1) return EGGSYNC_OK;  // plan only: the ranks choose the kernel together
    return run_planned_tc<D>(ws, lo, hi, nbr, owned);
  }
}

// The kernel choice from plan statistics (summed over all ranks in a multi-rank update, so that
// every rank and a single GPU choose alike), then the tensor-core update of the local plan.
inline bool tc_choose(const long long* g) {
  if (!g[5] || g[3]) return false;  // tensor cores not enabled / a rank's plan overflowed
  const unsigned long long ent = (unsigned long long)g[0], pts = (unsigned long long)g[1],
                           tiles = (unsigned long long)g[2];
  const double occ = ent ? (double)pts / (double)ent : 1.0;
    // Entries holding a few points each on average (partly collapsed clusters) put many
    // multi-point cells in the classifiers' exact band, where one lane scans a cell's points
    // alone; the warp-cooperative SIMT kernel is faster there (measured: C4-d10 iterations
    // 5-7, C4-d5 / C2 late iterations).  Singletons (occ ~ 1) and fully collapsed clusters
    // (occ >= 50: whole-cell summaries) stay on the tensor cores.
    // The slot lists are int32-indexed and cost 4 B per (tile, entry): beyond 2^30 slots
    // (e.g. C5 iteration 1: 2.5e10 entries, 3e12 pairs) the SIMT kernel runs instead; so it
    // does when the tiles average less than one entry tile (a CTA per nearly empty tile:
    // C5 iteration 3, 13 entries per tile, 14 ms vs 2 ms).
  return !((occ > 1.1 && occ < 50.0) || ent + tiles * kTcEnt > (1ull << 30) || ent < tiles * kTcEnt);
}

template <int D>
int run_planned_tc(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr, int64_t owned) {
  if constexpr (D > kTcMaxD) {
    return EGGSYNC_EINVAL;
  } else {
    using C = TcCfg<D>;
    if (!tc_choose(ws.tc_mode == 2 ? ws.tc_global : ws.tc_local)) {
      ws.tc_used = 0;
      return run_update_simt<D>(ws, lo, hi, nbr);
    }
    ws.tc_used = 1;
    if (owned == 0) return EGGSYNC_OK;
    const unsigned long long ent_u = (unsigned long long)ws.tc_local[0], pad_u = (unsigned long long)ws.tc_pad;
    int32_t hc[10];
    hc[8] = (int32_t)(ws.tc_mode == 2 ? ws.tc_global[4] : ws.tc_local[4]);
    EGG_TRY(tc_ent_reserve(ws, (size_t)pad_u + 1));
    k_tc_expand<0><<<(unsigned)((owned + 3) / 4), 128, 0, ws.stream>>>(ws.tc_ranges, ws.tc_chunks, ws.tc_nr, ws.tc_ne,
                                                                    ws.tc_eoff, ws.tc_ent, (int32_t)owned);
    EGG_CUDA(cudaGetLastError());
    ws.launches += 1;
    // launch order: point tiles by descending entry count (longest-processing-time first);
    // EGGSYNC_TC_ORDER=0: the sorted (spatial) order, better L2 reuse of neighbouring tiles' cells
    static const int order_env = [] {
      const char* e = getenv("EGGSYNC_TC_ORDER");
      return e ? atoi(e) : 1;
    }();
    const bool heavy_first = order_env != 0;
    if (heavy_first) {
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

    // GEMM2 layout: digits per summary value from the largest cell count (balanced base-256
    // digits of |v| <= count * 2^kDigF hold 0.498 * 2^(8k)), N = digits * (2D+1) -> x16
    const long long maxc = hc[8] > 1 ? hc[8] : 1;
    int ndig = 3;
    while (ndig < kDigMax && (double)maxc * (double)(1 << kDigF) + 1.0 > 0.498 * std::ldexp(1.0, 8 * ndig)) ++ndig;
    const int n2 = (ndig * C::NV + 15) / 16 * 16;
    const int ns = (C::QC + 3 * kTcEnt + n2 <= 512) ? 3 : 2;  // S buffers that fit TMEM next to Q and O
    const int sbytes = C::stage_bytes(n2);
    int nst = (C::kBudget - C::kFixedBytes) / sbytes;
    nst = nst > kTcMaxStages ? kTcMaxStages : nst;
    // >= 3 stages: a worker group builds its next tile (jt + 2) before classifying jt
    if (nst < 3 || C::QC + 2 * kTcEnt + n2 > 512) {  // cannot happen for D <= kTcMaxD
      ws.tc_used = 0;
      return run_update_simt<D>(ws, lo, hi, nbr);
    }
    const size_t smem = (size_t)nst * sbytes + C::kFixedBytes;

    TcArgs<D> a;
    a.orig = ws.own_orig();
    a.n_own = ws.n_own;
    a.xs = ws.xs[ws.xcur];
    a.xs_next = ws.xs[ws.xcur ^ 1];
    a.sn = ws.sn;
    a.cs = ws.cs;
    a.g_of = ws.g_of;
    a.g_cnt = ws.g_cnt;
    a.c_rec = ws.c_rec;
    a.c_dig = ws.c_dig;
    a.c_head = ws.c_head;
    a.cell_of = ws.cell_of;
    a.c_lo = ws.c_lo;
    a.c_hi = ws.c_hi;
    a.ent = ws.tc_ent;
    a.eoff = ws.tc_eoff;
    a.perm = heavy_first ? ws.tc_perm : ws.tc_pv;
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
    a.ndig = ndig;
    a.n2 = n2;
    a.nst = nst;
    a.ns = ns;
    a.stage_bytes = sbytes;
    a.e = ws.k.ef;
    a.e2f = ws.k.e2f;
    a.rel = ws.k.rel;
    a.e2d = ws.k.e2;
    a.flags = ws.flags;
    a.nbr = nbr;
    EGG_CUDA(cudaFuncSetAttribute(k_update_tc<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    if (ws.tc_timing) {
      EGG_TRY(ws.tc_flush());
      const long long pairs = (long long)ent_u * kTcTile, padded = (long long)pad_u * kTcTile;
      ws.tc_acc[0] += 1;
      ws.tc_acc[1] += pairs;
      ws.tc_acc[2] += padded;
      // tensor-core operations per (point, entry) pair as executed: GEMM1 over the 3D+2 fp16
      // operand columns (hi/lo splits), GEMM2 over the digits x (2D+1) int8 value columns
      ws.tc_pend_alg = 2LL * pairs * (C::KU + ndig * C::NV);
      ws.tc_acc[3] += ws.tc_pend_alg;
      EGG_CUDA(cudaEventRecord(ws.tc_ev[0], ws.stream));
    }
    if (getenv("EGGSYNC_TC_DEBUG"))
      fprintf(stderr, "[tc-cfg] ndig=%d n2=%d stages=%d sbuf=%d stage_bytes=%d smem=%zu max_cell=%d\n", ndig, n2, nst,
              ns, sbytes, smem, hc[8]);
    a.prof = nullptr;
#ifdef EGG_TC_PROF
    static unsigned long long* prof = nullptr;
    if (!prof) EGG_CUDA(cudaMalloc((void**)&prof, 16 * sizeof(unsigned long long)));
    EGG_CUDA(cudaMemsetAsync(prof, 0, 16 * sizeof(unsigned long long), ws.stream));
    a.prof = prof;
#endif
    k_update_tc<D><<<(unsigned)owned, kTcThreads, smem, ws.stream>>>(a);
    EGG_CUDA(cudaGetLastError());
#ifdef EGG_TC_PROF
    {
      unsigned long long h[16];
      EGG_CUDA(cudaMemcpyAsync(h, prof, sizeof(h), cudaMemcpyDeviceToHost, ws.stream));
      EGG_CUDA(cudaStreamSynchronize(ws.stream));
      const double t = (double)(h[15] ? h[15] : 1);
      fprintf(stderr, "[tc-prof] clk per entry tile: copy warp issue %.0f (stage wait %.0f) | builders wait_landed %.0f "
              "build %.0f | classifiers (per own tile) wait_S %.0f ld %.0f band %.0f wait_st %.0f | GEMM1 wait_full %.0f "
              "wait_free %.0f | GEMM2 wait_P %.0f\n", h[10] / t, h[11] / t, h[4] / t, h[5] / t, h[0] / t, h[1] / t,
              h[2] / t, h[3] / t, h[8] / t, h[9] / t, h[12] / t);
    }
#endif
    if (ws.tc_timing) {
      EGG_CUDA(cudaEventRecord(ws.tc_ev[1], ws.stream));
      ws.tc_pending = true;
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
  if constexpr (D <= 4) {  // F3 random-access grid when selected (single-process updates)
    if (ws.tc_mode == 0 && dense_choose(ws)) return run_update_dense(ws, lo, hi, nbr);
  }
  if (tc_enabled(ws, D) && hi > lo) return run_update_tc<D>(ws, lo, hi, nbr);
  if (ws.tc_mode == 1) {  // plan only, tensor cores off on every rank (replicated cell count)
    for (auto& v : ws.tc_local) v = 0;
    return EGGSYNC_OK;
  }
  if (hi <= lo) return EGGSYNC_OK;
  return run_update_simt<D>(ws, lo, hi, nbr);
}

}  // namespace egg
