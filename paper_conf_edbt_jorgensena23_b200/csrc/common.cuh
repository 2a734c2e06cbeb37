// common.cuh -- internal definitions of libeggsync (product path only).
// Nothing here is shared with oracle/ (test infrastructure).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdio>
#include <string>

#include "../../include/eggsync.h"

namespace egg {

constexpr int kMaxD = EGGSYNC_MAX_D;
constexpr int kMaxKeyWords = 8;  // Morton keys up to 512 bits (d * ceil(log2 w))
constexpr int kWarpsPerCta = 4;  // update / second-term CTAs: 4 independent warps
constexpr int kBucket = 32;      // subtree of <= kBucket cells is processed cell by cell
constexpr int kOwnBlock = 128;  // points per ownership block (multi-GPU interleave) = tensor-core tile
constexpr int kRangeChunk = 64;   // tensor-core plan: ranges are allocated in chunks of 64 ...
constexpr int kChunkMax = 256;    // ... at most 256 chunks (16384 ranges) per point tile
constexpr uint32_t kLeafBit = 0x80000000u;
constexpr float kU = 5.9604644775390625e-08f;  // 2^-24, fp32 unit roundoff

__host__ __device__ constexpr int ceil4(int x) { return (x + 3) & ~3; }

// Hot-loop cell record in global memory (AoS, one per non-empty cell):
//   [0, D)        centre of the cell's MBR (fp32)
//   D             r = radius of the MBR about the centre (rounded up)
//   D+1           count (int32 bits)
//   D+2           start: first sorted position of the cell (int32 bits)
//   [D+3, 2D+3)   sum_{q in cell} sin(q_i)  (fp32, rounded from the exact fixed-point sum)
//   [2D+3, 3D+3)  sum_{q in cell} cos(q_i)
template <int D>
struct CellRec {
  static constexpr int kFloats = ceil4(3 * D + 3);
};

// Tensor-core update (update_tc.cuh): per-cell Eq.5 summary as exact integers for the int8
// GEMM (tcgen05 kind::i8):  v_j = round(sum sin/cos(q_i) * 2^kDigF) (j < 2D), v_2D = count,
// each in kDigMax balanced base-256 digits; digit column k*(2D+1)+j of a cell's kBytes-byte
// row.  Stored block-major, c_dig[kBytes/16][cap][16], so that a run of consecutive cells is
// one contiguous bulk copy per 16-column block (the MN-major GEMM operand layout).  Exact
// integer accumulation makes the masked sums order-independent.
// Record head (c_head[kHead/4][cap][4] floats, block-major as well): centre (D), radius,
// count, start -- a warp reading 32 consecutive cells reads 512 contiguous bytes per block.
constexpr int kTcMaxD = 12;
constexpr int kDigF = 21;    // fixed-point bits of the summaries (error <= 2^-22 per cell)
constexpr int kDigMax = 6;   // |v| <= n * 2^21 < 0.498 * 2^48 for n < 2^24
template <int D>
struct CellDig {
  static constexpr int kBytes = ((kDigMax * (2 * D + 1)) + 15) / 16 * 16;
  static constexpr int kHead = ((D + 3) + 3) / 4 * 4;  // floats of the record head
};

// Per-warp staged cell layout in shared memory (floats):
//   A: c'_0..c'_{D-1}, cc, lim_full, lim_out        (ceil4(D+3))
//   B: ssin_0..ssin_{D-1}, scos_0..scos_{D-1}       (ceil4(2D))
//   M: count, start (int bits), 2 pad               (4)
template <int D>
struct Stage {
  static constexpr int kA = ceil4(D + 3);
  static constexpr int kB = ceil4(2 * D);
  static constexpr int kFloats = kA + kB + 4;
};

// Order-preserving map float -> uint32 (for deterministic atomic min/max of MBRs).
__host__ __device__ inline uint32_t f2ord(float f) {
  uint32_t b;
  memcpy(&b, &f, 4);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}
__host__ __device__ inline float ord2f(uint32_t o) {
  uint32_t b = (o & 0x80000000u) ? (o & 0x7fffffffu) : ~o;
  float f;
  memcpy(&f, &b, 4);
  return f;
}

// Fixed-point scale for exact, order-independent cell / subtree sums of sin and cos
// (values in [-1,1]; |sum| <= n * 2^32 < 2^63 for n < 2^31).
constexpr double kFix = 4294967296.0;       // 2^32
constexpr double kInvFix = 2.3283064365386963e-10;  // 2^-32

// Run-time problem constants, all derived in fp64 from (double)eps.
struct Consts {
  int64_t n;
  int d;
  int bits;    // bits per dimension of a cell coordinate: ceil(log2 w), >= 1
  int sub;     // extra sub-cell bits per dimension (update units finer than the cells, F2)
  int nw;      // 64-bit words per Morton key
  int keybits; // d * (bits + sub)
  int64_t w;   // cells per dimension = ceil(1/c_w)          (Eq.4)
  double e, e2, cw, inv_cw, delta, ed, ed2;  // eps, eps^2, c_w (L252), 1/c_w, delta (L110), eps+delta
  float ef, e2f, edf, ed2f, rel;  // fp32 copies; rel = (4d+16) u relative safety margin
};

bool make_consts(int64_t n, int d, float eps, Consts* c, std::string* why, double cw_factor = 1.0);

// F1 one-launch clustering of small inputs (small.cu)
bool small_eligible(int64_t n, int d, const Consts& k);
int small_cluster(const float* x_dev, int64_t n, int d, const Consts& k, int32_t max_iters, int32_t* labels_dev,
                  float* coords_dev, int32_t* out_dev, cudaStream_t st);

// term_mode = EGGSYNC_TERM_DEF42 clustering on the direct kernels (sync_brute.cu).
int def42_cluster(const float* points, int64_t n, int d, float eps, const eggsync_opts& o, int32_t* labels_out,
                  int32_t* iters_out);

// thread-local error message
void set_error(const char* fmt, ...);

#define EGG_CUDA(call)                                                                   \
  do {                                                                                   \
    cudaError_t _e = (call);                                                             \
    if (_e != cudaSuccess) {                                                             \
      ::egg::set_error("%s failed: %s (%s:%d)", #call, cudaGetErrorString(_e), __FILE__, \
                       __LINE__);                                                        \
      return _e == cudaErrorMemoryAllocation ? EGGSYNC_ENOMEM : EGGSYNC_ECUDA;           \
    }                                                                                    \
  } while (0)

#define EGG_TRY(expr)            \
  do {                           \
    int _rc = (expr);            \
    if (_rc != EGGSYNC_OK) return _rc; \
  } while (0)


// Dimension dispatch (kernels are templated on D = 1..kMaxD).  A development build
// with -DEGG_DEV_D=<d> instantiates a single dimension (fast rebuilds for tuning).
#ifdef EGG_DEV_D
#define EGG_DIM_ENABLED(x) ((x) == EGG_DEV_D)
#else
#define EGG_DIM_ENABLED(x) true
#endif
#define EGG_CASE_D(Dv, FN, ...)                           \
  case Dv:                                                \
    if constexpr (EGG_DIM_ENABLED(Dv)) {                  \
      return FN<Dv>(__VA_ARGS__);                         \
    } else {                                              \
      set_error("d=%d not built (EGG_DEV_D build)", Dv);  \
      return EGGSYNC_EINVAL;                              \
    }
#define EGG_DISPATCH(d, FN, ...)                                                                        \
  switch (d) {                                                                                          \
    EGG_CASE_D(1, FN, __VA_ARGS__) EGG_CASE_D(2, FN, __VA_ARGS__) EGG_CASE_D(3, FN, __VA_ARGS__)        \
    EGG_CASE_D(4, FN, __VA_ARGS__) EGG_CASE_D(5, FN, __VA_ARGS__) EGG_CASE_D(6, FN, __VA_ARGS__)        \
    EGG_CASE_D(7, FN, __VA_ARGS__) EGG_CASE_D(8, FN, __VA_ARGS__) EGG_CASE_D(9, FN, __VA_ARGS__)        \
    EGG_CASE_D(10, FN, __VA_ARGS__) EGG_CASE_D(11, FN, __VA_ARGS__) EGG_CASE_D(12, FN, __VA_ARGS__)     \
    EGG_CASE_D(13, FN, __VA_ARGS__) EGG_CASE_D(14, FN, __VA_ARGS__) EGG_CASE_D(15, FN, __VA_ARGS__)     \
    EGG_CASE_D(16, FN, __VA_ARGS__) EGG_CASE_D(17, FN, __VA_ARGS__) EGG_CASE_D(18, FN, __VA_ARGS__)     \
    EGG_CASE_D(19, FN, __VA_ARGS__) EGG_CASE_D(20, FN, __VA_ARGS__) EGG_CASE_D(21, FN, __VA_ARGS__)     \
    EGG_CASE_D(22, FN, __VA_ARGS__) EGG_CASE_D(23, FN, __VA_ARGS__) EGG_CASE_D(24, FN, __VA_ARGS__)     \
    EGG_CASE_D(25, FN, __VA_ARGS__) EGG_CASE_D(26, FN, __VA_ARGS__) EGG_CASE_D(27, FN, __VA_ARGS__)     \
    EGG_CASE_D(28, FN, __VA_ARGS__) EGG_CASE_D(29, FN, __VA_ARGS__) EGG_CASE_D(30, FN, __VA_ARGS__)     \
    EGG_CASE_D(31, FN, __VA_ARGS__) EGG_CASE_D(32, FN, __VA_ARGS__)                                    \
    default:                                                                                            \
      set_error("unsupported d=%d", d);                                                                 \
      return EGGSYNC_EINVAL;                                                                            \
  }

// ------------------------------------------------------------------ workspace
struct Workspace {
  Consts k;
  int64_t n = 0;
  int d = 0;
  int64_t cap = 0;  // cell capacity (= n)
  // state
  float* xs[2] = {nullptr, nullptr};  // SoA [d][n] (sorted order)
  uint32_t* orig[2] = {nullptr, nullptr};
  int xcur = 0;  // xs[xcur] = D^t (sorted by its cell keys after build); xs[xcur^1] = D^{t+1}
  int ocur = 0;  // orig[ocur] = original index of each sorted position of xs[xcur]
  bool built = false;
  // keys / sort
  uint64_t* keys = nullptr;      // [nw][n] sorted
  uint64_t* keys_tmp = nullptr;  // [nw][n]
  uint64_t* kb[2] = {nullptr, nullptr};
  uint32_t* pb[2] = {nullptr, nullptr};
  void* cub_tmp = nullptr;
  size_t cub_bytes = 0;
  // per point
  float* sn = nullptr;  // [d][n]
  float* cs = nullptr;
  int32_t* cell_of = nullptr;  // [n] update unit ("cell" below) of each sorted point
  int32_t* iscan = nullptr;    // [n] int scratch
  // grid cells of width eps/(2 sqrt d) (L252): first term, second term, labels.
  // Equal to the units when sub == 0; otherwise each cell is a run of units.
  int32_t n_coarse = 0;
  int32_t* co_of = nullptr;     // [n] cell of each sorted point
  int32_t* co_start = nullptr;  // [cap+1]
  int32_t* co_cnt = nullptr;    // [cap]
  uint32_t* co_lo = nullptr;    // [d][cap] MBR (ordered bits)
  uint32_t* co_hi = nullptr;
  int32_t* u2co = nullptr;      // [cap] unit -> cell
  // effective grid-cell arrays of the current build (alias the unit arrays when sub == 0)
  int32_t n_grid = 0;
  const int32_t* g_of = nullptr;
  const int32_t* g_cnt = nullptr;
  const uint32_t* g_lo = nullptr;
  const uint32_t* g_hi = nullptr;
  const int32_t* g_u2co = nullptr;  // nullptr: identity
  // update units (summaries, hierarchy leaves)
  int32_t n_cells = 0;
  int32_t* cell_start = nullptr;  // [cap+1]
  uint64_t* c_fix = nullptr;      // [2d][cap]
  uint32_t* c_lo = nullptr;       // [d][cap] ordered-float bits
  uint32_t* c_hi = nullptr;
  int32_t* c_cnt = nullptr;    // [cap]
  float* c_rec = nullptr;      // [cap][CellRec<D>::kFloats]
  int8_t* c_dig = nullptr;     // [CellDig<D>::kBytes/16][cap][16] (d <= kTcMaxD only)
  float* c_head = nullptr;     // [CellDig<D>::kHead/4][cap][4] (d <= kTcMaxD only)
  uint64_t* c_key = nullptr;   // [nw][cap]
  // tree (Karras radix tree over sorted cell keys; internal nodes 0..nc-2)
  int4* t_meta = nullptr;      // first, last, left, right
  int32_t* t_parent = nullptr; // [cap] parent of internal node
  int32_t* l_parent = nullptr; // [cap] parent of leaf (cell)
  uint32_t* t_visit = nullptr;
  uint64_t* t_fix = nullptr;   // [cap][3d]: exact subtree sums [2d], (hi << 32 | lo) MBR bits [d]
  int32_t* t_cnt = nullptr;
  float* t_box = nullptr;      // [cap][2d] lo then hi
  float* t_sum = nullptr;      // [cap][2d] sin then cos
  // flags: [0]=first term AND, [1]=second term AND, [2]=keys unsorted, [3]=error, [4]=domain error
  int32_t* flags = nullptr;
  int32_t* h_flags = nullptr;  // pinned host mirror
  // io scratch
  float* io = nullptr;         // n*d row-major staging (device)
  int32_t* i_lab = nullptr;    // [n] labels scratch
  uint32_t* c_minorig = nullptr;
  int32_t* nbr = nullptr;      // optional neighbour counts (sorted order)
  int32_t* lab_final = nullptr; // labels recorded when the criterion held (original order)
  uint8_t* second_need = nullptr;  // [cap] grid cells whose points need the second term's point test
  bool have_final = false;
  bool second_checked = false;
  int64_t bytes = 0;
  char* arena = nullptr;  // one device allocation carved into the arrays above
  int cur_device = 0;     // device the arena lives on
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int device = 0;
  cudaEvent_t ev[8];
  bool ev_ok = false;
  int sort_skipped = 0;
  unsigned long long* work = nullptr;  // [8] work counters of the instrumented update
  bool count_work = false;
  int64_t launches = 0;  // kernel launches issued on this workspace (CUB internals counted by pass)
  int32_t own_stride = 1, own_offset = 0;  // block-interleaved ownership of the next update
  // sharded multi-rank runs (E2): the context holds a rank's own points (original local index
  // < n_own) followed by its halo; only own points contribute to the criterion flags
  int64_t n_own = INT64_MAX;
  const uint32_t* own_orig() const { return n_own < n ? orig[ocur] : nullptr; }
  // tensor-core update (update_tc.cuh): plan-pass outputs
  double* full_S = nullptr;     // [2d][n] per-point sums of subtrees added whole (sorted order)
  int32_t* full_N = nullptr;    // [n]
  int32_t* tc_nr = nullptr;     // [tiles+1] ranges per point tile
  int32_t* tc_ne = nullptr;     // [tiles+1] entries per point tile
  int32_t* tc_chunks = nullptr; // [tiles][kChunkMax] first range of each chunk of a tile's range list
  int32_t* tc_epad = nullptr;   // [tiles+1] entries per tile padded to whole entry tiles
  int32_t* tc_eoff = nullptr;   // [tiles+1] first slot of each tile in tc_ent (exclusive scan)
  int32_t* tc_ent = nullptr;    // unit (cell) of every entry slot, -1 = padding (grown on demand)
  size_t tc_ecap = 0;
  int32_t* tc_ctr = nullptr;    // [8] ranges allocated, chunk-table overflow, entries (u64), points in entries (u64), padded entries (u64)
  int32_t* tc_pv = nullptr;     // [tiles] tile index (sort values)
  int32_t* dense = nullptr;     // F3 random-access grid: [w^d] grid cell per cell index (update_dense.cu)
  size_t dense_bytes = 0;
  int32_t* tc_pk = nullptr;     // [tiles] entries, sorted descending (sort keys out)
  int32_t* tc_perm = nullptr;   // [tiles] launch order of the point tiles: most entries first
  int2* tc_ranges = nullptr;    // (first unit, count), grown on demand (process cache)
  size_t tc_rcap = 0;
  int tc_used = 0;              // 1 when the last update ran on the tensor cores
  // multi-rank kernel choice (eggsync_ctx_plan_owned / _update_planned): 0 = plan + choose +
  // run, 1 = plan only (stats into tc_local), 2 = choose from tc_global and run the plan of mode 1
  int tc_mode = 0;
  long long tc_local[6] = {0, 0, 0, 0, 0, 0};   // entries, points in entries, tiles, overflow, max cell, enabled
  long long tc_global[6] = {0, 0, 0, 0, 0, 0};
  long long tc_pad = 0;                          // padded entries of the local plan
  // tensor-core work accounting (eggsync_ctx_tc_work): since the last reset
  bool tc_timing = false;
  long long tc_acc[5] = {0, 0, 0, 0, 0};  // launches, pairs (unpadded), pairs (padded), alg FLOPs, kernel ns
  long long tc_pend_alg = 0;              // FLOPs of the launch whose events are pending
  bool tc_pending = false;
  cudaEvent_t tc_ev[2] = {nullptr, nullptr};
  int tc_flush();                         // fold a pending launch's event time into tc_acc

  int alloc(int64_t n, int d, float eps, int device, cudaStream_t stream, double cw_factor = 1.0);
  void release();
  ~Workspace() { release(); }
};

// ------------------------------------------------------------ pipeline stages
int stage_ingest(Workspace& ws, const float* points, bool on_device);
int stage_build(Workspace& ws);  // keys, sort, segment, summaries, tree
int stage_update(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr_sorted);
int stage_second_term(Workspace& ws, int64_t lo, int64_t hi);
int stage_labels(Workspace& ws, int32_t* labels_dev);  // labels of current cells, original order
int stage_coords(Workspace& ws, int which, float* out_dev);  // row-major, original order
int stage_scatter_i32(Workspace& ws, const int32_t* sorted_vals, int32_t* out_dev);
// F3, Def 4.2 on the grid structure (def42_grid.cu): term (i) into flags[0]; term (ii) into
// flags[1] (mlo/mhi: [d][n] scratch); eps-graph labels of the built state (scratch: 4n int32)
int def42_grid_first(Workspace& ws);
int def42_grid_second(Workspace& ws, float* mlo, float* mhi);
int def42_grid_labels(Workspace& ws, int32_t* scratch, int32_t* labels_dev);
// F3, the random-access grid (§4.2.2) for d <= 4 (update_dense.cu)
int64_t dense_cells(const Workspace& ws);
bool dense_choose(const Workspace& ws);
int dense_reserve(Workspace& ws, size_t cells);
int run_update_dense(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr);

int tc_ranges_reserve(Workspace& ws, size_t need);  // grow ws.tc_ranges to >= need entries
int tc_ent_reserve(Workspace& ws, size_t need);     // grow ws.tc_ent to >= need entries

// dispatch helpers (templated on D in update.cu / term.cu / grid.cu)
int launch_update(Workspace& ws, int64_t lo, int64_t hi, int32_t* nbr_sorted);
int launch_second_term(Workspace& ws, int64_t lo, int64_t hi);

}  // namespace egg
