// def42_grid.cu -- F3: Def 4.2 evaluated literally on the grid structure (term_mode =
// EGGSYNC_TERM_DEF42), instead of the all-pairs pass of sync_brute.cu.
//
// Def 4.2, on the state D^t the update read (R7):
//   term (i)  no pair p, q with eps/2 < ||p-q|| <= eps                          (L108, R8)
//   term (ii) no pair p, q with eps < ||p-q|| <= eps + delta and
//             dist(MBR(N_{eps/2}(q)), p) <= eps                                 (L108-110, R9, R10)
// and the labels of the returned state: connected components of the eps-graph (Theorem 4.7,
// L133; canonical numbering R14).  Four passes share one traversal of the radix tree over the
// sorted cells (units) that the update built (A5): a warp owns 32 consecutive sorted points and
// walks the tree as a packet, pruning a node (or a unit) for a point by fp32 MINDIST / MAXDIST
// of its exact MBR with the (4d+16)u margin; the point-level predicates are decided in fp32 when
// clear of the margin and otherwise in fp64 exactly as the oracle (dimension order, no FMA):
//   kFirst  radius eps:      nodes entirely within eps/2 (MAXDIST) or beyond eps are skipped
//   kMbr    radius eps/2:    nodes entirely within eps/2 contribute their box (the exact MBR
//                            of their points), others are scanned: per point lo/hi of N_{eps/2}
//   kSecond radius eps+delta: nodes entirely within eps are skipped (no shell point)
//   kCc     radius eps:      one min-label propagation round over the eps-graph
// Product path only; nothing here is shared with oracle/.
#include <cub/cub.cuh>

#include "update.cuh"

namespace egg {

namespace {

enum DefMode { kFirst = 0, kMbr = 1, kSecond = 2, kCc = 3 };

struct DefArgs {
  const float* __restrict__ xs;        // [d][n] sorted state D^t
  const int4* __restrict__ t_meta;
  const float* __restrict__ t_box;
  const int32_t* __restrict__ cell_start;  // unit point ranges
  const uint32_t* __restrict__ c_lo;   // unit MBR (order-preserving bits)
  const uint32_t* __restrict__ c_hi;
  float* mlo;                          // kMbr out / kSecond in: [d][n] MBR(N_{eps/2}(q))
  float* mhi;
  const int32_t* __restrict__ lab_in;  // kCc: labels (original indices) per sorted point
  int32_t* lab_out;
  int64_t n, cap;
  int32_t nc, stack_len, bucket;
  float e2f, e2hf, ed2f, rel;
  double e2d, e2hd, ed2d;
  int32_t* flags;  // [0] term (i) AND, [1] term (ii) AND, [2] kCc changed, [3] error
};

template <int D>
__device__ __forceinline__ void box_dist(const float* lo, const float* hi, const float (&p)[D], float& mind,
                                         float& maxd) {
  mind = 0.f;
  maxd = 0.f;
#pragma unroll
  for (int i = 0; i < D; ++i) {
    const float dl = lo[i] - p[i], dh = p[i] - hi[i];
    const float mn = fmaxf(fmaxf(dl, dh), 0.f), mx = fmaxf(-dl, -dh);
    mind = fmaf(mn, mn, mind);
    maxd = fmaf(mx, mx, maxd);
  }
}

// does point lane need to look inside a box with these distances?  (kMbr: a box entirely
// within eps/2 is merged here instead)
template <int D, int M>
__device__ __forceinline__ bool box_need(const DefArgs& a, float mind, float maxd, const float* lo, const float* hi,
                                         float (&blo)[D], float (&bhi)[D]) {
  const float up = 1.f + a.rel, dn = 1.f - a.rel;
  if constexpr (M == kFirst) return mind <= a.e2f * up && maxd > a.e2hf * dn;
  if constexpr (M == kSecond) return mind <= a.ed2f * up && maxd > a.e2f * dn;
  if constexpr (M == kCc) return mind <= a.e2f * up;
  if constexpr (M == kMbr) {
    if (mind > a.e2hf * up) return false;
    if (maxd <= a.e2hf * dn) {  // every point of the box is in N_{eps/2}(p): merge the exact box
#pragma unroll
      for (int i = 0; i < D; ++i) {
        blo[i] = fminf(blo[i], lo[i]);
        bhi[i] = fmaxf(bhi[i], hi[i]);
      }
      return false;
    }
    return true;
  }
  return true;
}

template <int D, int M>
__global__ void __launch_bounds__(kWarpsPerCta * 32) k_def42(const DefArgs a) {
  constexpr int BS = ceil4(2 * D);
  extern __shared__ __align__(16) float smem[];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  int2* stk = reinterpret_cast<int2*>(smem) + wid * a.stack_len;
  const int64_t j = ((int64_t)blockIdx.x * kWarpsPerCta + wid) * 32 + lane;
  const bool valid = j < a.n;
  const unsigned amask = __ballot_sync(FULLMASK, valid);
  if (amask == 0u) return;
  float p[D], blo[D], bhi[D];
#pragma unroll
  for (int i = 0; i < D; ++i) p[i] = blo[i] = bhi[i] = valid ? a.xs[(int64_t)i * a.n + j] : 0.f;
  const float up = 1.f + a.rel, dn = 1.f - a.rel;
  int32_t lab = (M == kCc && valid) ? a.lab_in[j] : 0;
  bool viol = false;
  int sp = 1;
  if (lane == 0) stk[0] = make_int2(a.nc > 1 ? 0 : (int)kLeafBit, (int)amask);
  __syncwarp();
  int pops = 0;
  while (sp > 0) {
    if constexpr (M == kFirst || M == kSecond) {  // early exit once some warp found a violation
      if ((++pops & 63) == 0 && *(volatile int32_t*)&a.flags[M == kFirst ? 0 : 1] == 0) break;
    }
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
      float lo[D], hi[D];
#pragma unroll
      for (int i = 0; i < D; ++i) {
        lo[i] = bx[i];
        hi[i] = bx[D + i];
      }
      float mind, maxd;
      box_dist<D>(lo, hi, p, mind, maxd);
      const bool need = act && box_need<D, M>(a, mind, maxd, lo, hi, blo, bhi);
      pm = __ballot_sync(FULLMASK, need);
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
      float lo[D], hi[D];
#pragma unroll
      for (int i = 0; i < D; ++i) {
        lo[i] = ordf(a.c_lo[(int64_t)i * a.cap + c]);
        hi[i] = ordf(a.c_hi[(int64_t)i * a.cap + c]);
      }
      float mind, maxd;
      box_dist<D>(lo, hi, p, mind, maxd);
      const bool cneed = pact && box_need<D, M>(a, mind, maxd, lo, hi, blo, bhi);
      if (!__any_sync(FULLMASK, cneed)) continue;
      const int32_t s0 = a.cell_start[c], s1 = a.cell_start[c + 1];
      for (int32_t q = s0; q < s1; ++q) {
        if constexpr (M == kCc) {  // only a smaller label can change anything
          if (!__any_sync(FULLMASK, cneed && a.lab_in[q] < lab)) continue;
        }
        float qv[D];
        float d2 = 0.f;
#pragma unroll
        for (int i = 0; i < D; ++i) {
          qv[i] = a.xs[(int64_t)i * a.n + q];
          const float t = qv[i] - p[i];
          d2 = fmaf(t, t, d2);
        }
        if constexpr (M == kFirst) {  // eps/2 < ||p-q|| <= eps (L108)
          bool v = cneed && d2 > a.e2hf * up && d2 <= a.e2f * dn;
          const bool amb = cneed && !v && d2 > a.e2hf * dn && d2 <= a.e2f * up;
          if (__any_sync(FULLMASK, amb)) {
            if (amb) {
              const double x = exact_d2<D>(qv, p);
              v = x > a.e2hd && x <= a.e2d;
            }
          }
          viol = viol || v;
        } else if constexpr (M == kMbr) {  // ||p-q|| <= eps/2: q in N_{eps/2}(p)
          bool in = cneed && d2 <= a.e2hf * dn;
          const bool amb = cneed && !in && d2 <= a.e2hf * up;
          if (__any_sync(FULLMASK, amb)) {
            if (amb) in = exact_d2<D>(qv, p) <= a.e2hd;
          }
          if (in) {
#pragma unroll
            for (int i = 0; i < D; ++i) {
              blo[i] = fminf(blo[i], qv[i]);
              bhi[i] = fmaxf(bhi[i], qv[i]);
            }
          }
        } else if constexpr (M == kSecond) {  // eps < ||p-q|| <= eps + delta, then dist(MBR(N(q)), p)
          bool shell = cneed && d2 > a.e2f * up && d2 <= a.ed2f * dn;
          const bool amb = cneed && !shell && d2 > a.e2f * dn && d2 <= a.ed2f * up;
          if (__any_sync(FULLMASK, amb)) {
            if (amb) {
              const double x = exact_d2<D>(qv, p);
              shell = x > a.e2d && x <= a.ed2d;
            }
          }
          if (shell) {  // L110: per-dimension clamp distance, fp64 as the oracle
            double mm = 0.0;
#pragma unroll
            for (int i = 0; i < D; ++i) {
              const double v = (double)p[i], L = (double)a.mlo[(int64_t)i * a.n + q],
                           H = (double)a.mhi[(int64_t)i * a.n + q];
              double t = 0.0;
              if (v < L) t = __dsub_rn(L, v);
              else if (v > H) t = __dsub_rn(v, H);
              mm = __dadd_rn(mm, __dmul_rn(t, t));
            }
            viol = viol || mm <= a.e2d;
          }
        } else {  // kCc: ||p-q|| <= eps
          const int32_t lq = a.lab_in[q];
          bool in = cneed && lq < lab && d2 <= a.e2f * dn;
          const bool amb = cneed && lq < lab && !in && d2 <= a.e2f * up;
          if (__any_sync(FULLMASK, amb)) {
            if (amb) in = exact_d2<D>(qv, p) <= a.e2d;
          }
          if (in) lab = lq;
        }
      }
      if constexpr (M == kFirst || M == kSecond) {
        if (__any_sync(FULLMASK, viol)) break;
      }
    }
    if constexpr (M == kFirst || M == kSecond) {
      if (__any_sync(FULLMASK, viol)) break;
    }
  }
  if constexpr (M == kFirst || M == kSecond) {
    if (__any_sync(FULLMASK, viol) && lane == 0) atomicAnd(&a.flags[M == kFirst ? 0 : 1], 0);
  }
  if constexpr (M == kMbr) {
    if (valid) {
#pragma unroll
      for (int i = 0; i < D; ++i) {
        a.mlo[(int64_t)i * a.n + j] = blo[i];
        a.mhi[(int64_t)i * a.n + j] = bhi[i];
      }
    }
  }
  if constexpr (M == kCc) {
    if (valid) {
      a.lab_out[j] = lab;
      if (lab != a.lab_in[j]) a.flags[2] = 1;
    }
  }
}

// pointer jumping on labels that are original indices: lab[j] <- lab[pos(lab[j])]
__global__ void k_def_jump(const int32_t* __restrict__ in, const int32_t* __restrict__ pos, int64_t n,
                           int32_t* __restrict__ out) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) out[j] = in[pos[in[j]]];
}
__global__ void k_def_init(const uint32_t* __restrict__ orig, int64_t n, int32_t* __restrict__ lab,
                           int32_t* __restrict__ pos, int32_t* __restrict__ iota) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) {
    lab[j] = (int32_t)orig[j];
    pos[orig[j]] = (int32_t)j;
    iota[j] = (int32_t)j;
  }
}

template <int D, int M>
int launch_def(Workspace& ws, DefArgs& a) {
  const size_t smem = (size_t)kWarpsPerCta * a.stack_len * sizeof(int2);
  EGG_CUDA(cudaFuncSetAttribute(k_def42<D, M>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int64_t per = 32 * kWarpsPerCta;
  k_def42<D, M><<<(unsigned)((ws.n + per - 1) / per), kWarpsPerCta * 32, smem, ws.stream>>>(a);
  ws.launches += 1;
  EGG_CUDA(cudaGetLastError());
  return EGGSYNC_OK;
}

DefArgs def_args(Workspace& ws) {
  DefArgs a{};
  a.xs = ws.xs[ws.xcur];
  a.t_meta = ws.t_meta;
  a.t_box = ws.t_box;
  a.cell_start = ws.cell_start;
  a.c_lo = ws.c_lo;
  a.c_hi = ws.c_hi;
  a.n = ws.n;
  a.cap = ws.cap;
  a.nc = ws.n_cells;
  a.stack_len = ws.k.keybits + 4;
  a.bucket = (int64_t)ws.n_cells * 2 > ws.n ? 256 : kBucket;
  a.e2f = ws.k.e2f;
  a.e2hf = ws.k.e2f * 0.25f;  // exact: a power-of-two scaling
  a.ed2f = ws.k.ed2f;
  a.rel = ws.k.rel;
  a.e2d = ws.k.e2;
  a.e2hd = ws.k.e2 / 4.0;  // (eps/2)^2 as the oracle (e2 / 4, exact)
  a.ed2d = ws.k.ed2;
  a.flags = ws.flags;
  return a;
}

// term (i) into flags[0]; when it holds, term (ii) into flags[1] (MBR pass first)
template <int D>
int terms_d(Workspace& ws, float* mlo, float* mhi, const int32_t* f1_host) {
  DefArgs a = def_args(ws);
  a.mlo = mlo;
  a.mhi = mhi;
  if (!f1_host) return launch_def<D, kFirst>(ws, a);
  EGG_TRY((launch_def<D, kMbr>(ws, a)));
  return launch_def<D, kSecond>(ws, a);
}

template <int D>
int cc_round_d(Workspace& ws, const int32_t* in, int32_t* out) {
  DefArgs a = def_args(ws);
  a.lab_in = in;
  a.lab_out = out;
  return launch_def<D, kCc>(ws, a);
}
int cc_round(Workspace& ws, const int32_t* in, int32_t* out) { EGG_DISPATCH(ws.d, cc_round_d, ws, in, out); }

__global__ void k_def_roots(const int32_t* __restrict__ lab, int64_t n, int32_t* __restrict__ isroot) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) isroot[lab[j]] = 1;  // lab = smallest original index of the component
}
__global__ void k_def_write(const uint32_t* __restrict__ orig, const int32_t* __restrict__ lab,
                            const int32_t* __restrict__ rank, int64_t n, int32_t* __restrict__ labels) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) labels[orig[j]] = rank[lab[j]];
}

}  // namespace

int def42_grid_first(Workspace& ws) { EGG_DISPATCH(ws.d, terms_d, ws, nullptr, nullptr, nullptr); }
int def42_grid_second(Workspace& ws, float* mlo, float* mhi) {
  static const int32_t one = 1;
  EGG_DISPATCH(ws.d, terms_d, ws, mlo, mhi, &one);
}

// eps-graph components of the built state (min-label propagation over the tree + pointer
// jumping, rounds until stable), canonical numbering by smallest original index (R14), into
// labels_dev[orig]; scratch: 4 int32 arrays of n.
int def42_grid_labels(Workspace& ws, int32_t* scratch, int32_t* labels_dev) {
  const int64_t n = ws.n;
  int32_t* lab[2] = {scratch, scratch + n};
  int32_t* pos = scratch + 2 * n;
  int32_t* iota = scratch + 3 * n;
  const unsigned nb = (unsigned)((n + 255) / 256);
  k_def_init<<<nb, 256, 0, ws.stream>>>(ws.orig[ws.ocur], n, lab[0], pos, iota);
  EGG_CUDA(cudaGetLastError());
  for (int round = 0;; ++round) {
    EGG_CUDA(cudaMemsetAsync(ws.flags + 2, 0, sizeof(int32_t), ws.stream));
    EGG_TRY(cc_round(ws, lab[0], lab[1]));
    k_def_jump<<<nb, 256, 0, ws.stream>>>(lab[1], pos, n, lab[0]);
    EGG_CUDA(cudaGetLastError());
    ws.launches += 2;
    EGG_CUDA(cudaMemcpyAsync(ws.h_flags, ws.flags, 4 * sizeof(int32_t), cudaMemcpyDeviceToHost, ws.stream));
    EGG_CUDA(cudaStreamSynchronize(ws.stream));
    if (ws.h_flags[3]) {
      set_error("traversal stack overflow (internal error)");
      return EGGSYNC_ECUDA;
    }
    if (!ws.h_flags[2]) break;
    if (round > 64 + 2 * 31) {  // pointer jumping halves the depth each round: cannot happen
      set_error("eps-graph labelling did not converge (internal error)");
      return EGGSYNC_ECUDA;
    }
  }
  // canonical numbering (R14): rank of each component's smallest original index
  int32_t* isroot = pos;  // free now
  int32_t* rank = iota;
  EGG_CUDA(cudaMemsetAsync(isroot, 0, sizeof(int32_t) * n, ws.stream));
  k_def_roots<<<nb, 256, 0, ws.stream>>>(lab[0], n, isroot);
  EGG_CUDA(cudaGetLastError());
  size_t bytes = ws.cub_bytes;
  EGG_CUDA(cub::DeviceScan::ExclusiveSum(ws.cub_tmp, bytes, isroot, rank, (int)n, ws.stream));
  k_def_write<<<nb, 256, 0, ws.stream>>>(ws.orig[ws.ocur], lab[0], rank, n, labels_dev);
  EGG_CUDA(cudaGetLastError());
  ws.launches += 4;
  return EGGSYNC_OK;
}

}  // namespace egg
