// grid.cu -- structure building of one EGG-SynC iteration (§4.2, §4.3.1).
//
//  A0 ingest        : validate [0,1] (L70, L290), row-major -> SoA
//  A1 cell keys     : c_i = min(floor(x_i * (1/c_w)), w-1) in fp64 (Eq.4, c_w L252),
//                     bit-interleaved (Morton) so that sorting groups cells AND keeps
//                     nearby cells adjacent (replaces the d'-dim outer grid, L183-195)
//  A2 radix sort    : CUB onesweep SortPairs (key, index), LSD over key words;
//                     skipped when the keys are already sorted (late iterations)
//  A3 segment       : head flags + prefix sum -> cell_of, cell_start (list construction
//                     "sizes -> scan -> populate", L157-163)
//  A4 summaries     : fp64 sincos per coordinate; warp-shuffle segmented sums of the
//                     exact 64-bit fixed-point sin/cos, count and MBR per cell
//                     (Eq.5-6; deterministic, unlike the paper's float atomics)
//  A5 hierarchy     : Karras radix tree over the sorted cell keys; bottom-up subtree
//                     summaries (count, sum sin, sum cos, MBR).  It plays the role of
//                     preGrid / mixed grid (L183-218): the neighbour-cell enumeration.
//  A8 labels        : gatherCluster (L256): cells -> canonical cluster ids.
#include <cub/cub.cuh>

#include "common.cuh"

namespace egg {

#define FULLMASK 0xffffffffu

static inline unsigned blocks_for(int64_t n, int t) { return (unsigned)((n + t - 1) / t); }

// ------------------------------------------------------------------- A0 ingest
__global__ void k_ingest(const float* __restrict__ io, int64_t n, int d, float* __restrict__ xs,
                         uint32_t* __restrict__ orig, int32_t* __restrict__ flags) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n * d) return;
  float v = io[t];
  int64_t j = t / d;
  int i = (int)(t - j * d);
  if (!(v >= 0.f && v <= 1.f)) atomicOr(&flags[4], 1);  // NaN/Inf/out of [0,1]
  xs[(int64_t)i * n + j] = v;
  if (i == 0) orig[j] = (uint32_t)j;
}

// --------------------------------------------------------------------- A1 keys
// key of a point: Morton interleave of the fine coordinates f_i = c_i * 2^sub + s_i where
// c_i is the cell coordinate and s_i the sub-cell (F2) inside it; the top D*cbits bits of
// the code are the Morton code of the cell, so sorting groups cells, and sub-cells in them.
template <int D>
__global__ void k_keys(const float* __restrict__ xs, int64_t n, int cbits, int sub, int nw, int64_t w,
                       double inv_cw, uint64_t* __restrict__ keys) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  uint32_t c[D];
#pragma unroll
  for (int i = 0; i < D; ++i) {
    double t = __dmul_rn((double)xs[(int64_t)i * n + j], inv_cw);  // one rounding, as the oracle
    double f = floor(t);
    int64_t ci = (int64_t)f;
    ci = ci > w - 1 ? w - 1 : ci;  // clamp x = 1.0 into the last cell (R2)
    ci = ci < 0 ? 0 : ci;
    int64_t si = 0;
    if (sub) {  // position inside the cell: t - ci is exact in fp64
      si = (int64_t)floor(ldexp(t - (double)ci, sub));
      si = si > (1 << sub) - 1 ? (1 << sub) - 1 : (si < 0 ? 0 : si);
    }
    c[i] = (uint32_t)((ci << sub) | si);
  }
  // Morton interleave, most significant bit-plane first: plane k holds bit (bits-1-k) of every c_i.
  const int bits = cbits + sub;
  int widx = nw - 1;
  int filled = 64 * nw - D * bits;
  uint64_t acc = 0;
  for (int k = 0; k < bits; ++k) {
    const int sh = bits - 1 - k;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      acc = (acc << 1) | (uint64_t)((c[i] >> sh) & 1u);
      if (++filled == 64) {
        keys[(int64_t)widx * n + j] = acc;
        --widx;
        acc = 0;
        filled = 0;
      }
    }
  }
}

__device__ inline int key_cmp(const uint64_t* __restrict__ keys, int64_t n, int nw, int64_t a, int64_t b) {
  for (int w = nw - 1; w >= 0; --w) {
    uint64_t x = keys[(int64_t)w * n + a], y = keys[(int64_t)w * n + b];
    if (x != y) return x < y ? -1 : 1;
  }
  return 0;
}

__global__ void k_check_sorted(const uint64_t* __restrict__ keys, int64_t n, int nw, int32_t* flags) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x + 1;
  bool bad = (j < n) && key_cmp(keys, n, nw, j - 1, j) > 0;
  if (__any_sync(FULLMASK, bad) && (threadIdx.x & 31) == 0) atomicOr(&flags[2], 1);
}

// ------------------------------------------------------------------- A2 sort
__global__ void k_iota(uint32_t* p, int64_t n) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) p[j] = (uint32_t)j;
}

__global__ void k_gather_word(const uint64_t* __restrict__ keys_w, const uint32_t* __restrict__ perm,
                              int64_t n, uint64_t* __restrict__ out) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) out[j] = keys_w[perm[j]];
}

template <int D>
__global__ void k_gather_state(const float* __restrict__ xs_in, const uint32_t* __restrict__ orig_in,
                               const uint64_t* __restrict__ keys_in, const uint32_t* __restrict__ perm,
                               int64_t n, int nw, float* __restrict__ xs_out, uint32_t* __restrict__ orig_out,
                               uint64_t* __restrict__ keys_out) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  const int64_t s = perm[j];
#pragma unroll
  for (int i = 0; i < D; ++i) xs_out[(int64_t)i * n + j] = xs_in[(int64_t)i * n + s];
  orig_out[j] = orig_in[s];
  for (int w = 0; w < nw; ++w) keys_out[(int64_t)w * n + j] = keys_in[(int64_t)w * n + s];
}

// ---------------------------------------------------------------- A3 segment
__global__ void k_heads(const uint64_t* __restrict__ keys, int64_t n, int nw, int32_t* __restrict__ head) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  head[j] = (j == 0) || key_cmp(keys, n, nw, j - 1, j) != 0;
}

__global__ void k_cell_start(const int32_t* __restrict__ head, int32_t* __restrict__ cell_of, int64_t n,
                             int nw, const uint64_t* __restrict__ keys, int64_t cap,
                             int32_t* __restrict__ cell_start, uint64_t* __restrict__ c_key) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  int32_t c = cell_of[j] - 1;  // inclusive scan -> 0-based cell id
  cell_of[j] = c;
  if (head[j]) {
    cell_start[c] = (int32_t)j;
    for (int w = 0; w < nw; ++w) c_key[(int64_t)w * cap + c] = keys[(int64_t)w * n + j];
  }
  if (j == n - 1) cell_start[c + 1] = (int32_t)n;
}

// Grid cells of width eps/(2 sqrt d) when update units are finer (sub > 0): two sorted
// keys are in the same cell iff they agree above their lowest D*sub bits.
__global__ void k_coarse_heads(const uint64_t* __restrict__ keys, int64_t n, int nw, int lowbits,
                               int32_t* __restrict__ head) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  bool h = j == 0;
  if (!h) {
    for (int w = nw - 1; w >= 0; --w) {
      uint64_t x = keys[(int64_t)w * n + j - 1], y = keys[(int64_t)w * n + j];
      const int below = lowbits - 64 * w;  // sub-cell bits inside this word
      if (below >= 64) break;
      if (below > 0) {
        x >>= below;
        y >>= below;
      }
      if (x != y) {
        h = true;
        break;
      }
    }
  }
  head[j] = h;
}

__global__ void k_coarse_start(const int32_t* __restrict__ head, int32_t* __restrict__ co_of, int64_t n,
                               int32_t* __restrict__ co_start) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  const int32_t c = co_of[j] - 1;
  co_of[j] = c;
  if (head[j]) co_start[c] = (int32_t)j;
  if (j == n - 1) co_start[c + 1] = (int32_t)n;
}

template <int D>
__global__ void k_coarse_init(int32_t ncc, int64_t cap, const int32_t* __restrict__ co_start,
                              int32_t* __restrict__ co_cnt, uint32_t* __restrict__ co_lo,
                              uint32_t* __restrict__ co_hi) {
  const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= ncc) return;
  co_cnt[c] = co_start[c + 1] - co_start[c];
#pragma unroll
  for (int i = 0; i < D; ++i) {
    co_lo[(int64_t)i * cap + c] = 0xffffffffu;
    co_hi[(int64_t)i * cap + c] = 0u;
  }
}

// unit -> cell map and cell MBR = union of its units' MBRs (order-independent atomics)
template <int D>
__global__ void k_coarse_mbr(int32_t nc, int64_t cap, const int32_t* __restrict__ cell_start,
                             const int32_t* __restrict__ co_of, const uint32_t* __restrict__ c_lo,
                             const uint32_t* __restrict__ c_hi, int32_t* __restrict__ u2co,
                             uint32_t* __restrict__ co_lo, uint32_t* __restrict__ co_hi) {
  const int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= nc) return;
  const int32_t c = co_of[cell_start[u]];
  u2co[u] = c;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    atomicMin(&co_lo[(int64_t)i * cap + c], c_lo[(int64_t)i * cap + u]);
    atomicMax(&co_hi[(int64_t)i * cap + c], c_hi[(int64_t)i * cap + u]);
  }
}

// -------------------------------------------------------------- A4 summaries
// Cells that span a 32-point warp boundary are combined with integer atomics; initialise them.
template <int D>
__global__ void k_init_span(const int32_t* __restrict__ cell_of, int64_t n, int64_t cap,
                            uint64_t* __restrict__ c_fix, uint32_t* __restrict__ c_lo,
                            uint32_t* __restrict__ c_hi, int32_t* __restrict__ c_cnt) {
  int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x + 1;
  int64_t j2 = 32 * k;
  if (j2 >= n) return;
  int32_t c = cell_of[j2];
  if (cell_of[j2 - 1] != c) return;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    c_fix[(int64_t)i * cap + c] = 0;
    c_fix[(int64_t)(D + i) * cap + c] = 0;
    c_lo[(int64_t)i * cap + c] = 0xffffffffu;
    c_hi[(int64_t)i * cap + c] = 0u;
  }
  c_cnt[c] = 0;
}

template <int D>
__global__ void __launch_bounds__(256) k_cell_sums(const float* __restrict__ xs, int64_t n, int64_t cap,
                                                   const int32_t* __restrict__ cell_of,
                                                   const int32_t* __restrict__ cell_start,
                                                   float* __restrict__ sn, float* __restrict__ cs,
                                                   uint64_t* __restrict__ c_fix, uint32_t* __restrict__ c_lo,
                                                   uint32_t* __restrict__ c_hi, int32_t* __restrict__ c_cnt) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31;
  const bool valid = j < n;
  const int32_t c = valid ? cell_of[j] : -1;
  const int32_t cprev = __shfl_up_sync(FULLMASK, c, 1);
  const int32_t cnext = __shfl_down_sync(FULLMASK, c, 1);
  bool f = (lane == 0) || (c != cprev);  // segment head inside this warp
  uint64_t fs[D], fc[D];
  uint32_t lo[D], hi[D];
  int32_t cnt = valid ? 1 : 0;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    float x = valid ? xs[(int64_t)i * n + j] : 0.f;
    double s, co;
    sincos((double)x, &s, &co);
    if (valid) {
      sn[(int64_t)i * n + j] = (float)s;
      cs[(int64_t)i * n + j] = (float)co;
    }
    fs[i] = valid ? (uint64_t)__double2ll_rn(s * kFix) : 0ull;
    fc[i] = valid ? (uint64_t)__double2ll_rn(co * kFix) : 0ull;
    lo[i] = hi[i] = f2ord(x);
  }
  // segmented inclusive scan (Hillis-Steele with head flags)
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const bool g = __shfl_up_sync(FULLMASK, f, off);
    const int32_t yc = __shfl_up_sync(FULLMASK, cnt, off);
    const bool take = lane >= off && !f;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      uint64_t ys = __shfl_up_sync(FULLMASK, fs[i], off);
      uint64_t yc2 = __shfl_up_sync(FULLMASK, fc[i], off);
      uint32_t yl = __shfl_up_sync(FULLMASK, lo[i], off);
      uint32_t yh = __shfl_up_sync(FULLMASK, hi[i], off);
      if (take) {
        fs[i] += ys;
        fc[i] += yc2;
        lo[i] = min(lo[i], yl);
        hi[i] = max(hi[i], yh);
      }
    }
    if (take) cnt += yc;
    if (lane >= off) f = f || g;
  }
  const bool tail = valid && (lane == 31 || j == n - 1 || cnext != c);
  if (!tail) return;
  const int64_t wfirst = j - lane;
  const bool complete = cell_start[c] >= wfirst && (int64_t)cell_start[c + 1] == j + 1;
  if (complete) {
#pragma unroll
    for (int i = 0; i < D; ++i) {
      c_fix[(int64_t)i * cap + c] = fs[i];
      c_fix[(int64_t)(D + i) * cap + c] = fc[i];
      c_lo[(int64_t)i * cap + c] = lo[i];
      c_hi[(int64_t)i * cap + c] = hi[i];
    }
    c_cnt[c] = cnt;
  } else {
#pragma unroll
    for (int i = 0; i < D; ++i) {
      atomicAdd((unsigned long long*)&c_fix[(int64_t)i * cap + c], (unsigned long long)fs[i]);
      atomicAdd((unsigned long long*)&c_fix[(int64_t)(D + i) * cap + c], (unsigned long long)fc[i]);
      atomicMin(&c_lo[(int64_t)i * cap + c], lo[i]);
      atomicMax(&c_hi[(int64_t)i * cap + c], hi[i]);
    }
    atomicAdd(&c_cnt[c], cnt);
  }
}

// Hot-loop record of each cell (see CellRec in common.cuh), and for the tensor-core update
// (D <= kTcMaxD) the cell's Eq.5 summary as exact integers in balanced base-256 digits
// (CellDig in common.cuh): v_j = round(sum_{q in cell} sin/cos(q_i) * 2^kDigF) from the exact
// 2^32 fixed-point sums, v_2D = count.  The largest count goes to flags[5] (digits needed).
template <int D>
__global__ void k_cell_finalize(int32_t nc, int64_t cap, const int32_t* __restrict__ cell_start,
                                const uint64_t* __restrict__ c_fix, const uint32_t* __restrict__ c_lo,
                                const uint32_t* __restrict__ c_hi, const int32_t* __restrict__ c_cnt,
                                float* __restrict__ c_rec, int8_t* __restrict__ c_dig, float* __restrict__ c_head,
                                int32_t* __restrict__ flags) {
  const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= nc) return;
  if constexpr (D <= kTcMaxD) {
    if (c_dig) {
      constexpr int NV = 2 * D + 1, DB = CellDig<D>::kBytes;
      const int32_t cnt = c_cnt[c];
      atomicMax(&flags[5], cnt);
      uint32_t w[DB / 4];
#pragma unroll
      for (int k = 0; k < DB / 4; ++k) w[k] = 0u;
#pragma unroll
      for (int j = 0; j < NV; ++j) {
        // round half up of fix * 2^(kDigF-32): arithmetic shift of the two's complement sum
        long long v = j < 2 * D ? (((long long)c_fix[(int64_t)j * cap + c] + (1ll << (31 - kDigF))) >> (32 - kDigF))
                                : (long long)cnt;
#pragma unroll
        for (int k = 0; k < kDigMax; ++k) {
          const int dk = (int)(int8_t)(uint8_t)(v & 0xff);  // balanced digit in [-128, 127]
          v = (v - dk) >> 8;
          const int b = k * NV + j;
          w[b >> 2] |= (uint32_t)(uint8_t)dk << (8 * (b & 3));
        }
      }
      uint4* dst = reinterpret_cast<uint4*>(c_dig);
#pragma unroll
      for (int k = 0; k < DB / 16; ++k) dst[k * cap + c] = make_uint4(w[4 * k], w[4 * k + 1], w[4 * k + 2], w[4 * k + 3]);
    }
  }
  constexpr int R = CellRec<D>::kFloats;
  float* r = c_rec + c * R;
  float r2 = 0.f;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    float l = ord2f(c_lo[(int64_t)i * cap + c]), h = ord2f(c_hi[(int64_t)i * cap + c]);
    float m = 0.5f * (l + h);
    float e = fmaxf(h - m, m - l);
    r2 = fmaf(e, e, r2);
    r[i] = m;
  }
  // radius about the stored centre, rounded up to cover the fp32 evaluation (r = 0 for a point)
  r[D] = sqrtf(r2) * (1.0f + (float)(D + 8) * kU);
  r[D + 1] = __int_as_float(c_cnt[c]);
  r[D + 2] = __int_as_float(cell_start[c]);
#pragma unroll
  for (int i = 0; i < D; ++i) {
    r[D + 3 + i] = (float)((double)(long long)c_fix[(int64_t)i * cap + c] * kInvFix);
    r[2 * D + 3 + i] = (float)((double)(long long)c_fix[(int64_t)(D + i) * cap + c] * kInvFix);
  }
  for (int q = 3 * D + 3; q < R; ++q) r[q] = 0.f;
  if constexpr (D <= kTcMaxD) {
    if (c_head) {  // centre, radius, count, start: the tensor-core update's record heads, block-major
      constexpr int H = CellDig<D>::kHead;
      float h[H];
#pragma unroll
      for (int q = 0; q < H; ++q) h[q] = q < D + 3 ? r[q] : 0.f;
      float4* dst = reinterpret_cast<float4*>(c_head);
#pragma unroll
      for (int k = 0; k < H / 4; ++k) dst[k * cap + c] = make_float4(h[4 * k], h[4 * k + 1], h[4 * k + 2], h[4 * k + 3]);
    }
  }
}

// ------------------------------------------------------- A5 radix tree (Karras 2012)
__device__ inline int lcp(const uint64_t* __restrict__ ck, int64_t cap, int nw, int64_t nc, int64_t i,
                          int64_t j) {
  if (j < 0 || j >= nc) return -1;
  for (int w = nw - 1; w >= 0; --w) {
    uint64_t x = ck[(int64_t)w * cap + i] ^ ck[(int64_t)w * cap + j];
    if (x) return (nw - 1 - w) * 64 + __clzll((long long)x);
  }
  return 64 * nw;
}

__global__ void k_tree_build(const uint64_t* __restrict__ ck, int64_t cap, int nw, int32_t nc,
                             int4* __restrict__ meta, int32_t* __restrict__ t_parent,
                             int32_t* __restrict__ l_parent, uint32_t* __restrict__ visit) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= (int64_t)nc - 1) return;
  const int dir = (lcp(ck, cap, nw, nc, i, i + 1) - lcp(ck, cap, nw, nc, i, i - 1)) > 0 ? 1 : -1;
  const int dmin = lcp(ck, cap, nw, nc, i, i - dir);
  int64_t lmax = 2;
  while (lcp(ck, cap, nw, nc, i, i + lmax * dir) > dmin) lmax <<= 1;
  int64_t l = 0;
  for (int64_t t = lmax >> 1; t >= 1; t >>= 1)
    if (lcp(ck, cap, nw, nc, i, i + (l + t) * dir) > dmin) l += t;
  const int64_t j = i + l * dir;
  const int dnode = lcp(ck, cap, nw, nc, i, j);
  int64_t s = 0;
  for (int64_t div = 2;; div <<= 1) {
    int64_t t = (l + div - 1) / div;
    if (lcp(ck, cap, nw, nc, i, i + (s + t) * dir) > dnode) s += t;
    if (t <= 1) break;
  }
  const int64_t gamma = i + s * dir + (dir < 0 ? -1 : 0);
  const int32_t first = (int32_t)min(i, j), last = (int32_t)max(i, j);
  int32_t left, right;
  if (first == gamma) {
    left = (int32_t)(gamma | kLeafBit);
    l_parent[gamma] = (int32_t)i;
  } else {
    left = (int32_t)gamma;
    t_parent[gamma] = (int32_t)i;
  }
  if (last == gamma + 1) {
    right = (int32_t)((gamma + 1) | kLeafBit);
    l_parent[gamma + 1] = (int32_t)i;
  } else {
    right = (int32_t)(gamma + 1);
    t_parent[gamma + 1] = (int32_t)i;
  }
  meta[i] = make_int4(first, last, left, right);
  visit[i] = 0;
  if (i == 0) t_parent[0] = -1;
}

template <int D>
__global__ void k_tree_agg(int32_t nc, int64_t cap, const int4* __restrict__ meta,
                           const int32_t* __restrict__ t_parent, const int32_t* __restrict__ l_parent,
                           uint32_t* __restrict__ visit, const uint64_t* __restrict__ c_fix,
                           const uint32_t* __restrict__ c_lo, const uint32_t* __restrict__ c_hi,
                           const int32_t* __restrict__ c_cnt, uint64_t* t_agg, int32_t* t_cnt,
                           float* __restrict__ t_box, float* __restrict__ t_sum) {
  // t_agg: one row of 3D u64 per internal node (exact sums [2D], then (hi << 32 | lo) [D]):
  // a parent reads an internal child's exact aggregate from one contiguous row (cells keep
  // their SoA c_fix / c_lo / c_hi)
  const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= nc) return;
  constexpr int BS = ceil4(2 * D);
  int32_t node = l_parent[c];
  while (node >= 0) {
    // acq_rel: the first arrival releases its subtree's aggregate (written by this thread the
    // level below), the second acquires the sibling's before reading it (no full fence)
    uint32_t prev;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(prev) : "l"(&visit[node]) : "memory");
    if (prev == 0u) return;  // first arrival: sibling not ready
    const int4 m = meta[node];
    const int32_t ch[2] = {m.z, m.w};
    uint64_t fs[2 * D];
    uint32_t lo[D], hi[D];
    int32_t cnt = 0;
#pragma unroll
    for (int i = 0; i < 2 * D; ++i) fs[i] = 0;
#pragma unroll
    for (int i = 0; i < D; ++i) {
      lo[i] = 0xffffffffu;
      hi[i] = 0u;
    }
#pragma unroll
    for (int k = 0; k < 2; ++k) {
      const int64_t x = ch[k] & 0x7fffffff;
      if (ch[k] & (int32_t)kLeafBit) {
        cnt += __ldcg(&c_cnt[x]);
#pragma unroll
        for (int i = 0; i < 2 * D; ++i) fs[i] += __ldcg((const unsigned long long*)&c_fix[(int64_t)i * cap + x]);
#pragma unroll
        for (int i = 0; i < D; ++i) {
          lo[i] = min(lo[i], __ldcg(&c_lo[(int64_t)i * cap + x]));
          hi[i] = max(hi[i], __ldcg(&c_hi[(int64_t)i * cap + x]));
        }
      } else {
        cnt += __ldcg(&t_cnt[x]);
        const unsigned long long* row = reinterpret_cast<const unsigned long long*>(t_agg + x * (3 * D));
#pragma unroll
        for (int i = 0; i < 2 * D; ++i) fs[i] += __ldcg(row + i);
#pragma unroll
        for (int i = 0; i < D; ++i) {
          const unsigned long long b = __ldcg(row + 2 * D + i);
          lo[i] = min(lo[i], (uint32_t)b);
          hi[i] = max(hi[i], (uint32_t)(b >> 32));
        }
      }
    }
    uint64_t* row = t_agg + (int64_t)node * (3 * D);
#pragma unroll
    for (int i = 0; i < 2 * D; ++i) {
      row[i] = fs[i];
      t_sum[(int64_t)node * BS + i] = (float)((double)(long long)fs[i] * kInvFix);
    }
#pragma unroll
    for (int i = 0; i < D; ++i) {
      row[2 * D + i] = ((uint64_t)hi[i] << 32) | lo[i];
      t_box[(int64_t)node * BS + i] = ord2f(lo[i]);
      t_box[(int64_t)node * BS + D + i] = ord2f(hi[i]);
    }
    t_cnt[node] = cnt;
    node = t_parent[node];
  }
}

// ------------------------------------------------------------------ A8 labels
__global__ void k_lab_min(const int32_t* __restrict__ cell_of, const uint32_t* __restrict__ orig, int64_t n,
                          uint32_t* __restrict__ minorig) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) atomicMin(&minorig[cell_of[j]], orig[j]);
}
__global__ void k_lab_flag(const uint32_t* __restrict__ minorig, int32_t nc, int32_t* __restrict__ isfirst) {
  int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c < nc) isfirst[minorig[c]] = 1;
}
__global__ void k_lab_write(const int32_t* __restrict__ cell_of, const uint32_t* __restrict__ orig,
                            const uint32_t* __restrict__ minorig, const int32_t* __restrict__ rank, int64_t n,
                            int32_t* __restrict__ labels) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) labels[orig[j]] = rank[minorig[cell_of[j]]];
}

__global__ void k_coords_out(const float* __restrict__ xs, const uint32_t* __restrict__ orig, int64_t n, int d,
                             float* __restrict__ out) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n * d) return;
  int64_t j = t % n;
  int i = (int)(t / n);
  out[(int64_t)orig[j] * d + i] = xs[t];
}

__global__ void k_scatter_i32(const int32_t* __restrict__ v, const uint32_t* __restrict__ orig, int64_t n,
                              int32_t* __restrict__ out) {
  int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) out[orig[j]] = v[j];
}

// ===================================================================== hosts
#define EGG_LAUNCH_CHECK() \
  do {                     \
    ws.launches++;         \
    EGG_CUDA(cudaGetLastError()); \
  } while (0)
// CUB launches (onesweep radix sort: histogram + exclusive sum + one pass per 8 bits;
// single-tile sort for small n; scans: init + sweep).
static inline int cub_sort_launches(int64_t n, int bits) { return n <= 4096 ? 1 : 2 + (bits + 7) / 8; }

int stage_ingest(Workspace& ws, const float* points, bool on_device) {
  const int64_t nd = ws.n * ws.d;
  const float* src = points;
  if (!on_device) {
    EGG_CUDA(cudaMemcpyAsync(ws.io, points, (size_t)nd * sizeof(float), cudaMemcpyHostToDevice, ws.stream));
    src = ws.io;
  }
  EGG_CUDA(cudaMemsetAsync(ws.flags, 0, 8 * sizeof(int32_t), ws.stream));
  k_ingest<<<blocks_for(nd, 256), 256, 0, ws.stream>>>(src, ws.n, ws.d, ws.xs[0], ws.orig[0], ws.flags);
  EGG_LAUNCH_CHECK();
  EGG_CUDA(cudaMemcpyAsync(ws.h_flags, ws.flags, 8 * sizeof(int32_t), cudaMemcpyDeviceToHost, ws.stream));
  EGG_CUDA(cudaStreamSynchronize(ws.stream));
  ws.xcur = 0;
  ws.ocur = 0;
  ws.built = false;
  ws.have_final = false;
  if (ws.h_flags[4]) {
    set_error("a coordinate is NaN/Inf or outside [0,1] (PAPER.md L70: data must be normalised)");
    return EGGSYNC_EDOMAIN;
  }
  return EGGSYNC_OK;
}

template <int D>
static int build_d(Workspace& ws) {
  const int64_t n = ws.n, cap = ws.cap;
  const Consts& K = ws.k;
  cudaStream_t st = ws.stream;
  const int T = 256;
  // A1 keys of D^t in its current (previous sorted) order
  k_keys<D><<<blocks_for(n, T), T, 0, st>>>(ws.xs[ws.xcur], n, K.bits, K.sub, K.nw, K.w, K.inv_cw, ws.keys);
  EGG_LAUNCH_CHECK();
  EGG_CUDA(cudaMemsetAsync(ws.flags + 2, 0, sizeof(int32_t), st));
  EGG_CUDA(cudaMemsetAsync(ws.flags + 5, 0, sizeof(int32_t), st));  // largest cell count (k_cell_finalize)
  if (n > 1) {
    k_check_sorted<<<blocks_for(n - 1, T), T, 0, st>>>(ws.keys, n, K.nw, ws.flags);
    EGG_LAUNCH_CHECK();
  }
  EGG_CUDA(cudaMemcpyAsync(ws.h_flags + 2, ws.flags + 2, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
  EGG_CUDA(cudaStreamSynchronize(st));
  if (ws.h_flags[2]) {
    // A2: LSD radix sort over the key words (least significant word first; CUB sorts are stable)
    cub::DoubleBuffer<uint64_t> kbuf(ws.kb[0], ws.kb[1]);
    cub::DoubleBuffer<uint32_t> pbuf(ws.pb[0], ws.pb[1]);
    k_iota<<<blocks_for(n, T), T, 0, st>>>(pbuf.Current(), n);
    EGG_LAUNCH_CHECK();
    for (int w = 0; w < K.nw; ++w) {
      k_gather_word<<<blocks_for(n, T), T, 0, st>>>(ws.keys + (int64_t)w * n, pbuf.Current(), n, kbuf.Current());
      EGG_LAUNCH_CHECK();
      const int wbits = (w < K.nw - 1) ? 64 : (K.keybits - 64 * (K.nw - 1));
      size_t bytes = ws.cub_bytes;
      EGG_CUDA(cub::DeviceRadixSort::SortPairs(ws.cub_tmp, bytes, kbuf, pbuf, (int)n, 0, wbits, st));
      ws.launches += cub_sort_launches(n, wbits);
    }
    k_gather_state<D><<<blocks_for(n, T), T, 0, st>>>(ws.xs[ws.xcur], ws.orig[ws.ocur], ws.keys, pbuf.Current(),
                                                      n, K.nw, ws.xs[ws.xcur ^ 1], ws.orig[ws.ocur ^ 1],
                                                      ws.keys_tmp);
    EGG_LAUNCH_CHECK();
    std::swap(ws.keys, ws.keys_tmp);
    ws.xcur ^= 1;
    ws.ocur ^= 1;
  } else {
    ws.sort_skipped++;
  }
  // A3 segment
  k_heads<<<blocks_for(n, T), T, 0, st>>>(ws.keys, n, K.nw, ws.iscan);
  EGG_LAUNCH_CHECK();
  {
    size_t bytes = ws.cub_bytes;
    EGG_CUDA(cub::DeviceScan::InclusiveSum(ws.cub_tmp, bytes, ws.iscan, ws.cell_of, (int)n, st));
    ws.launches += 2;
  }
  k_cell_start<<<blocks_for(n, T), T, 0, st>>>(ws.iscan, ws.cell_of, n, K.nw, ws.keys, cap, ws.cell_start,
                                               ws.c_key);
  EGG_LAUNCH_CHECK();
  EGG_CUDA(cudaMemcpyAsync(ws.h_flags + 6, ws.cell_of + (n - 1), sizeof(int32_t), cudaMemcpyDeviceToHost, st));
  if (K.sub > 0) {  // grid cells above the update units
    k_coarse_heads<<<blocks_for(n, T), T, 0, st>>>(ws.keys, n, K.nw, D * K.sub, ws.iscan);
    EGG_LAUNCH_CHECK();
    size_t bytes = ws.cub_bytes;
    EGG_CUDA(cub::DeviceScan::InclusiveSum(ws.cub_tmp, bytes, ws.iscan, ws.co_of, (int)n, st));
    ws.launches += 2;
    k_coarse_start<<<blocks_for(n, T), T, 0, st>>>(ws.iscan, ws.co_of, n, ws.co_start);
    EGG_LAUNCH_CHECK();
    EGG_CUDA(cudaMemcpyAsync(ws.h_flags + 7, ws.co_of + (n - 1), sizeof(int32_t), cudaMemcpyDeviceToHost, st));
  }
  // A4 summaries
  if (n > 32) {
    k_init_span<D><<<blocks_for((n - 1) / 32, T), T, 0, st>>>(ws.cell_of, n, cap, ws.c_fix, ws.c_lo, ws.c_hi,
                                                             ws.c_cnt);
    EGG_LAUNCH_CHECK();
  }
  k_cell_sums<D><<<blocks_for(n, 256), 256, 0, st>>>(ws.xs[ws.xcur], n, cap, ws.cell_of, ws.cell_start, ws.sn,
                                                     ws.cs, ws.c_fix, ws.c_lo, ws.c_hi, ws.c_cnt);
  EGG_LAUNCH_CHECK();
  EGG_CUDA(cudaStreamSynchronize(st));
  ws.n_cells = ws.h_flags[6] + 1;
  const int32_t nc = ws.n_cells;
  k_cell_finalize<D><<<blocks_for(nc, T), T, 0, st>>>(nc, cap, ws.cell_start, ws.c_fix, ws.c_lo, ws.c_hi,
                                                      ws.c_cnt, ws.c_rec, ws.c_dig, ws.c_head, ws.flags);
  EGG_LAUNCH_CHECK();
  if (K.sub > 0) {
    ws.n_grid = ws.h_flags[7] + 1;
    k_coarse_init<D><<<blocks_for(ws.n_grid, T), T, 0, st>>>(ws.n_grid, cap, ws.co_start, ws.co_cnt, ws.co_lo,
                                                            ws.co_hi);
    EGG_LAUNCH_CHECK();
    k_coarse_mbr<D><<<blocks_for(nc, T), T, 0, st>>>(nc, cap, ws.cell_start, ws.co_of, ws.c_lo, ws.c_hi, ws.u2co,
                                                     ws.co_lo, ws.co_hi);
    EGG_LAUNCH_CHECK();
    ws.g_of = ws.co_of;
    ws.g_cnt = ws.co_cnt;
    ws.g_lo = ws.co_lo;
    ws.g_hi = ws.co_hi;
    ws.g_u2co = ws.u2co;
  } else {  // units are the grid cells
    ws.n_grid = nc;
    ws.g_of = ws.cell_of;
    ws.g_cnt = ws.c_cnt;
    ws.g_lo = ws.c_lo;
    ws.g_hi = ws.c_hi;
    ws.g_u2co = nullptr;
  }
  // A5 hierarchy
  if (nc > 1) {
    k_tree_build<<<blocks_for(nc - 1, T), T, 0, st>>>(ws.c_key, cap, K.nw, nc, ws.t_meta, ws.t_parent,
                                                      ws.l_parent, ws.t_visit);
    EGG_LAUNCH_CHECK();
    k_tree_agg<D><<<blocks_for(nc, 128), 128, 0, st>>>(nc, cap, ws.t_meta, ws.t_parent, ws.l_parent,
                                                       ws.t_visit, ws.c_fix, ws.c_lo, ws.c_hi, ws.c_cnt,
                                                       ws.t_fix, ws.t_cnt, ws.t_box,
                                                       ws.t_sum);
    EGG_LAUNCH_CHECK();
  }
  ws.built = true;
  return EGGSYNC_OK;
}


int stage_build(Workspace& ws) { EGG_DISPATCH(ws.d, build_d, ws); }

int stage_labels(Workspace& ws, int32_t* labels_dev) {
  const int64_t n = ws.n;
  const int32_t nc = ws.n_grid;  // labels are grid cells (gatherCluster, L256)
  cudaStream_t st = ws.stream;
  const int T = 256;
  EGG_CUDA(cudaMemsetAsync(ws.c_minorig, 0xff, (size_t)nc * sizeof(uint32_t), st));
  k_lab_min<<<blocks_for(n, T), T, 0, st>>>(ws.g_of, ws.orig[ws.ocur], n, ws.c_minorig);
  EGG_LAUNCH_CHECK();
  EGG_CUDA(cudaMemsetAsync(ws.i_lab, 0, (size_t)n * sizeof(int32_t), st));
  k_lab_flag<<<blocks_for(nc, T), T, 0, st>>>(ws.c_minorig, nc, ws.i_lab);
  EGG_LAUNCH_CHECK();
  size_t bytes = ws.cub_bytes;
  EGG_CUDA(cub::DeviceScan::ExclusiveSum(ws.cub_tmp, bytes, ws.i_lab, ws.iscan, (int)n, st));
  ws.launches += 2;
  k_lab_write<<<blocks_for(n, T), T, 0, st>>>(ws.g_of, ws.orig[ws.ocur], ws.c_minorig, ws.iscan, n, labels_dev);
  EGG_LAUNCH_CHECK();
  return EGGSYNC_OK;
}

int stage_coords(Workspace& ws, int which, float* out_dev) {
  const int64_t nd = ws.n * ws.d;
  k_coords_out<<<blocks_for(nd, 256), 256, 0, ws.stream>>>(ws.xs[which], ws.orig[ws.ocur], ws.n, ws.d, out_dev);
  EGG_LAUNCH_CHECK();
  return EGGSYNC_OK;
}

int stage_scatter_i32(Workspace& ws, const int32_t* sorted_vals, int32_t* out_dev) {
  k_scatter_i32<<<blocks_for(ws.n, 256), 256, 0, ws.stream>>>(sorted_vals, ws.orig[ws.ocur], ws.n, out_dev);
  EGG_LAUNCH_CHECK();
  return EGGSYNC_OK;
}

size_t cub_temp_bytes(int64_t n) {
  size_t a = 0, b = 0, c = 0;
  cub::DoubleBuffer<uint64_t> kb(nullptr, nullptr);
  cub::DoubleBuffer<uint32_t> pb(nullptr, nullptr);
  cub::DeviceRadixSort::SortPairs(nullptr, a, kb, pb, (int)n, 0, 64);
  cub::DeviceScan::InclusiveSum(nullptr, b, (int32_t*)nullptr, (int32_t*)nullptr, (int)n);
  cub::DeviceScan::ExclusiveSum(nullptr, c, (int32_t*)nullptr, (int32_t*)nullptr, (int)n);
  return std::max(a, std::max(b, c));
}

}  // namespace egg
