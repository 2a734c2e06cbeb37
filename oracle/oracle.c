/*
 * oracle.c -- plain, slow, obviously-correct fp64 CPU oracle for EGG-SynC.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (libeggsync.so) never links, calls or reads anything here,
 * and this file includes nothing from the product tree.
 *
 * What it computes is the *definition* the paper's exact method reaches
 * (EGG-SynC is exact): plain SynC iterated with the
 * Kuramoto update (Eq.1) and stopped by the synchronization criterion
 * (Def 4.2).  No grid acceleration, no Eq.5 identity, no pruning:
 * O(T * n^2 * d), fp64, libm sin, compiled with -ffp-contract=off.
 *
 * Readings of the paper it follows (listed in DESIGN.md "Readings"):
 *   R1 cell width c_w = eps / (2 sqrt d)            (L252, equality)
 *   R2 cell coordinate min(floor(x * (1/c_w)), w-1), w = ceil(1/c_w)  (Eq.4)
 *   R3 Jacobi update: every new coordinate reads D^t          (Eq.1, Alg 1 l.5 L53)
 *   R4 N_eps(p) includes p, test is ||p-q|| <= eps evaluated as
 *      sum_i (q_i - p_i)^2 <= eps^2 in fp64, dimension order  (L66)
 *   R6 loop: repeat update; stop after the first update whose *input* state
 *      satisfies the criterion; at least one update is applied  (Alg 4)
 *   R7 both criterion terms are evaluated on D^t, the state the update read
 *   R8 term (i) strict eps/2 < ||p-q||                          (Def 4.2)
 *   R9 term (ii) uses MBR(N_{eps/2}(q)) and the bound <= eps + delta  (L108)
 *   R10 dist(MBR,p) = per-dimension clamp distance (the printed formula, L110)
 *   R11 delta = eps - eps*sqrt(15/16) + eps/2 - sin(eps/2)     (L110)
 *   R14 labels numbered by first occurrence (smallest point index)
 *
 * Pinned by tests/test_oracle_pins.py (closed forms, App.D recurrence,
 * invariants, brute-force re-derivation, Eq.5/6 identity); see DESIGN.md.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_OK 0
#define ORACLE_NOT_CONVERGED 1
#define ORACLE_EINVAL (-1)
#define ORACLE_ENOMEM (-3)
#define ORACLE_EPARTITION (-6) /* CC labels != cell partition (Theorem 4.7 violated) */

/* ---------------------------------------------------------------- constants */

/* out[0]=eps (as fp64 of the fp32 value), out[1]=eps^2, out[2]=c_w,
 * out[3]=1/c_w, out[4]=w, out[5]=delta, out[6]=(eps+delta)^2            */
void oracle_constants_cw(float eps32, int32_t d, double cw_factor, double *out) {
    double e = (double)eps32;
    /* L252: c_w <= sqrt((eps/2)^2/d); cw_factor in (0,1] picks a width below the bound (R1) */
    double cw = cw_factor * (e / (2.0 * sqrt((double)d)));
    double inv_cw = 1.0 / cw;
    double w = ceil(1.0 / cw);                        /* Eq.4: ceil(1/c_w) cells per dim */
    double delta = e - e * sqrt(15.0 / 16.0) + e / 2.0 - sin(e / 2.0); /* L110 */
    out[0] = e;
    out[1] = e * e;
    out[2] = cw;
    out[3] = inv_cw;
    out[4] = w;
    out[5] = delta;
    out[6] = (e + delta) * (e + delta);
}

void oracle_constants(float eps32, int32_t d, double *out) { oracle_constants_cw(eps32, d, 1.0, out); }

/* squared Euclidean distance, dimension order, no contraction (R4) */
static double sqdist(const double *X, int64_t p, int64_t q, int32_t d) {
    double s = 0.0;
    for (int32_t i = 0; i < d; ++i) {
        double t = X[q * d + i] - X[p * d + i];
        s = s + t * t;
    }
    return s;
}

/* cell coordinate of x along one dimension (R2) */
static int64_t cell_coord(double x, double inv_cw, int64_t w) {
    int64_t c = (int64_t)floor(x * inv_cw);
    if (c > w - 1) c = w - 1;
    if (c < 0) c = 0;
    return c;
}

static int same_cell(const double *X, int64_t p, int64_t q, int32_t d, double inv_cw, int64_t w) {
    for (int32_t i = 0; i < d; ++i)
        if (cell_coord(X[p * d + i], inv_cw, w) != cell_coord(X[q * d + i], inv_cw, w)) return 0;
    return 1;
}

/* ------------------------------------------------------------------- step */

/*
 * One synchronous Eq.1 update D^t -> D^{t+1} (L68) plus the criterion on D^t.
 *   X   : n*d row-major fp64, the state D^t (read only)
 *   Xn  : n*d row-major fp64, receives D^{t+1}
 *   nbr : n, receives |N_eps(p)| (may be NULL)
 *   flags[0] = F1 GRID  : for all p, every q in N_eps(p) is in p's cell
 *                         (Alg 3 l.14-15 L248 with the L252 cell width)
 *   flags[1] = F1 DEF42 : no pair with eps/2 < ||p-q|| <= eps  (Def 4.2 term i, L108)
 *   flags[2] = F2       : no pair with eps < ||p-q|| <= eps+delta and
 *                         dist(MBR(N_{eps/2}(q)), p) <= eps   (Def 4.2 term ii, L108-110)
 *                         evaluated iff compute_f2 or flags[0] or flags[1]; else -1
 */
int oracle_step_cw(const double *X, int64_t n, int32_t d, float eps32, double cw_factor, double *Xn,
                   int32_t *nbr, int32_t *flags, int32_t compute_f2) {
    if (!X || !Xn || !flags || n < 1 || d < 1 || !(cw_factor > 0.0 && cw_factor <= 1.0)) return ORACLE_EINVAL;
    double C[7];
    oracle_constants_cw(eps32, d, cw_factor, C);
    const double e2 = C[1], inv_cw = C[3], ed2 = C[6];
    const int64_t w = (int64_t)C[4];
    const double e2h = e2 / 4.0; /* (eps/2)^2 */
    int f1_grid = 1, f1_def = 1;

    /* Eq.1 (L68): p_i^{t+1} = p_i^t + 1/|N(p^t)| * sum_{q in N(p^t)} sin(q_i^t - p_i^t) */
#pragma omp parallel for schedule(dynamic, 16) reduction(&& : f1_grid, f1_def)
    for (int64_t p = 0; p < n; ++p) {
        double *sum = (double *)calloc((size_t)d, sizeof(double));
        int64_t cnt = 0;
        for (int64_t q = 0; q < n; ++q) { /* q ascending */
            double dd = sqdist(X, p, q, d);
            if (dd <= e2) {               /* q in N_eps(p), L66 */
                ++cnt;
                for (int32_t i = 0; i < d; ++i) sum[i] = sum[i] + sin(X[q * d + i] - X[p * d + i]);
                if (!same_cell(X, p, q, d, inv_cw, w)) f1_grid = 0;
                if (dd > e2h) f1_def = 0;
            }
        }
        for (int32_t i = 0; i < d; ++i) Xn[p * d + i] = X[p * d + i] + (1.0 / (double)cnt) * sum[i];
        if (nbr) nbr[p] = (int32_t)cnt;
        free(sum);
    }
    flags[0] = f1_grid;
    flags[1] = f1_def;
    flags[2] = -1;
    if (!(compute_f2 || f1_grid || f1_def)) return ORACLE_OK;

    /* MBR(N_{eps/2}(q)) for every q (Def 4.2 term ii) */
    double *lo = (double *)malloc((size_t)(n * d) * sizeof(double));
    double *hi = (double *)malloc((size_t)(n * d) * sizeof(double));
    if (!lo || !hi) { free(lo); free(hi); return ORACLE_ENOMEM; }
#pragma omp parallel for schedule(dynamic, 16)
    for (int64_t q = 0; q < n; ++q) {
        for (int32_t i = 0; i < d; ++i) { lo[q * d + i] = X[q * d + i]; hi[q * d + i] = X[q * d + i]; }
        for (int64_t r = 0; r < n; ++r) {
            if (sqdist(X, q, r, d) <= e2h) {
                for (int32_t i = 0; i < d; ++i) {
                    double v = X[r * d + i];
                    if (v < lo[q * d + i]) lo[q * d + i] = v;
                    if (v > hi[q * d + i]) hi[q * d + i] = v;
                }
            }
        }
    }
    int f2 = 1;
#pragma omp parallel for schedule(dynamic, 16) reduction(&& : f2)
    for (int64_t p = 0; p < n; ++p) {
        for (int64_t q = 0; q < n; ++q) {
            double dd = sqdist(X, p, q, d);
            if (dd > e2 && dd <= ed2) {
                /* dist(MBR, p)^2 = sum_i (min_{c in MBR} |p_i - c_i|)^2   (L110) */
                double m = 0.0;
                for (int32_t i = 0; i < d; ++i) {
                    double v = X[p * d + i], t = 0.0;
                    if (v < lo[q * d + i]) t = lo[q * d + i] - v;
                    else if (v > hi[q * d + i]) t = v - hi[q * d + i];
                    m = m + t * t;
                }
                if (m <= e2) f2 = 0;
            }
        }
    }
    flags[2] = f2;
    free(lo);
    free(hi);
    return ORACLE_OK;
}

int oracle_step(const double *X, int64_t n, int32_t d, float eps32, double *Xn,
                int32_t *nbr, int32_t *flags, int32_t compute_f2) {
    return oracle_step_cw(X, n, d, eps32, 1.0, Xn, nbr, flags, compute_f2);
}

/* ------------------------------------------------------- order parameter */

/*
 * Cluster order parameter of the state D^t (Eq.2; Alg 1 l.6 L54, SynC's
 * lambda-termination input, L77/L95):
 *   r_c = 1/|D| * sum_{p in D} 1/|N_eps(p^t)| * sum_{q in N_eps(p^t)} exp(-||q^t - p^t||)
 * with N_eps as in R4 (fp64, dimension order, p in N_eps(p)).
 *   rcp : n, receives the inner mean for every p (may be NULL)
 * The outer mean is summed serially in point order.
 */
int oracle_order_parameter(const double *X, int64_t n, int32_t d, float eps32, double *rc_out,
                           double *rcp) {
    if (!X || !rc_out || n < 1 || d < 1) return ORACLE_EINVAL;
    double C[7];
    oracle_constants(eps32, d, C);
    const double e2 = C[1];
    double *inner = (double *)malloc((size_t)n * sizeof(double));
    if (!inner) return ORACLE_ENOMEM;
#pragma omp parallel for schedule(dynamic, 16)
    for (int64_t p = 0; p < n; ++p) {
        double s = 0.0;
        int64_t cnt = 0;
        for (int64_t q = 0; q < n; ++q) {
            double dd = sqdist(X, p, q, d);
            if (dd <= e2) {        /* q in N_eps(p), L66 */
                ++cnt;
                s = s + exp(-sqrt(dd));
            }
        }
        inner[p] = s / (double)cnt;
    }
    double tot = 0.0;
    for (int64_t p = 0; p < n; ++p) tot = tot + inner[p];
    *rc_out = tot / (double)n;
    if (rcp) memcpy(rcp, inner, (size_t)n * sizeof(double));
    free(inner);
    return ORACLE_OK;
}

/* ------------------------------------------------------------- labelling */

/* canonical relabel: ids numbered by first occurrence in point order (R14) */
static void canonicalize(const int64_t *group, int64_t n, int32_t *labels) {
    int64_t *map = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    for (int64_t i = 0; i < n; ++i) map[i] = -1;
    int32_t next = 0;
    for (int64_t p = 0; p < n; ++p) {
        int64_t g = group[p];
        if (map[g] < 0) map[g] = next++;
        labels[p] = (int32_t)map[g];
    }
    free(map);
}

/* connected components of the eps-graph {(p,q): ||p-q|| <= eps} by
 * min-label propagation (each label = smallest index in its component) */
static void eps_components(const double *X, int64_t n, int32_t d, double e2, int32_t *labels) {
    int64_t *lab = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    int64_t *nxt = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    for (int64_t p = 0; p < n; ++p) lab[p] = p;
    int changed = 1;
    while (changed) {
        changed = 0;
#pragma omp parallel for schedule(dynamic, 16) reduction(|| : changed)
        for (int64_t p = 0; p < n; ++p) {
            int64_t m = lab[p];
            for (int64_t q = 0; q < n; ++q)
                if (lab[q] < m && sqdist(X, p, q, d) <= e2) m = lab[q];
            nxt[p] = m;
            if (m != lab[p]) changed = 1;
        }
        for (int64_t p = 0; p < n; ++p) lab[p] = nxt[p];
        for (int64_t p = 0; p < n; ++p) lab[p] = lab[lab[p]]; /* pointer jumping */
    }
    canonicalize(lab, n, labels);
    free(lab);
    free(nxt);
}

/* cell partition of a state (gatherCluster, L256): points sharing all cell coordinates */
static const int64_t *g_cc; /* comparator context */
static int32_t g_d;
static int cmp_cells(const void *a, const void *b) {
    int64_t p = *(const int64_t *)a, q = *(const int64_t *)b;
    for (int32_t i = 0; i < g_d; ++i) {
        int64_t x = g_cc[p * g_d + i], y = g_cc[q * g_d + i];
        if (x != y) return x < y ? -1 : 1;
    }
    return p < q ? -1 : (p > q);
}

static void cell_partition(const double *X, int64_t n, int32_t d, double inv_cw, int64_t w, int32_t *labels) {
    int64_t *cc = (int64_t *)malloc((size_t)(n * d) * sizeof(int64_t));
    int64_t *ord = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    int64_t *grp = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    for (int64_t p = 0; p < n; ++p) {
        ord[p] = p;
        for (int32_t i = 0; i < d; ++i) cc[p * d + i] = cell_coord(X[p * d + i], inv_cw, w);
    }
    g_cc = cc;
    g_d = d;
    qsort(ord, (size_t)n, sizeof(int64_t), cmp_cells);
    int64_t gid = 0;
    for (int64_t k = 0; k < n; ++k) {
        if (k > 0) {
            int diff = 0;
            for (int32_t i = 0; i < d; ++i)
                if (cc[ord[k] * d + i] != cc[ord[k - 1] * d + i]) { diff = 1; break; }
            gid += diff;
        }
        grp[ord[k]] = gid;
    }
    canonicalize(grp, n, labels);
    free(cc);
    free(ord);
    free(grp);
}

/* ------------------------------------------------------------- full loop */

/*
 * EGG-SynC's result by the plain definition (Alg 4 L258-278 semantics, R6/R7):
 *   X32 : n*d row-major float32 input in [0,1]
 *   term_mode : 0 = GRID first term (L252), 1 = DEF42 literal first term (L108)
 *   X_out  : n*d fp64 final coordinates D^{t} at exit (may be NULL)
 *   labels : n, connected components of the eps-graph on the final state,
 *            canonical numbering (Theorem 4.7: at the criterion these are the clusters)
 *   iters  : number of Eq.1 updates applied
 *   cell_labels : n (may be NULL) canonical cell partition of the verified state
 * Returns ORACLE_OK, ORACLE_NOT_CONVERGED (max_iters reached), ORACLE_EPARTITION
 * when GRID termination's cell partition differs from the eps-components.
 */
int oracle_cluster_cw(const float *X32, int64_t n, int32_t d, float eps32, double cw_factor,
                      int32_t term_mode, int32_t max_iters, double *X_out, int32_t *labels,
                      int32_t *iters, int32_t *cell_labels) {
    if (!X32 || !labels || !iters || n < 1 || d < 1 || max_iters < 1) return ORACLE_EINVAL;
    if (!(cw_factor > 0.0 && cw_factor <= 1.0)) return ORACLE_EINVAL;
    double C[7];
    oracle_constants_cw(eps32, d, cw_factor, C);
    const int64_t w = (int64_t)C[4];
    double *X = (double *)malloc((size_t)(n * d) * sizeof(double));
    double *Xn = (double *)malloc((size_t)(n * d) * sizeof(double));
    int32_t *cl = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    if (!X || !Xn || !cl) { free(X); free(Xn); free(cl); return ORACLE_ENOMEM; }
    for (int64_t k = 0; k < n * d; ++k) X[k] = (double)X32[k];
    int32_t t = 0, synced = 0, status = ORACLE_OK;
    for (;;) {
        int32_t f[3];
        int rc = oracle_step_cw(X, n, d, eps32, cw_factor, Xn, NULL, f, 0);
        if (rc != ORACLE_OK) { status = rc; break; }
        int32_t f1 = term_mode == 0 ? f[0] : f[1];
        synced = f1 && f[2] == 1;
        if (synced) cell_partition(X, n, d, C[3], w, cl); /* cells of the verified state D^t */
        double *tmp = X; X = Xn; Xn = tmp;                /* D^{t+1} */
        ++t;
        if (synced) break;
        if (t >= max_iters) { status = ORACLE_NOT_CONVERGED; break; }
    }
    if (status >= 0) {
        eps_components(X, n, d, C[1], labels);
        if (!synced) cell_partition(X, n, d, C[3], w, cl);
        if (cell_labels) memcpy(cell_labels, cl, (size_t)n * sizeof(int32_t));
        if (synced && term_mode == 0 && memcmp(cl, labels, (size_t)n * sizeof(int32_t)) != 0)
            status = ORACLE_EPARTITION;
        if (X_out) memcpy(X_out, X, (size_t)(n * d) * sizeof(double));
        *iters = t;
    }
    free(X);
    free(Xn);
    free(cl);
    return status;
}

int oracle_cluster(const float *X32, int64_t n, int32_t d, float eps32, int32_t term_mode,
                   int32_t max_iters, double *X_out, int32_t *labels, int32_t *iters,
                   int32_t *cell_labels) {
    return oracle_cluster_cw(X32, n, d, eps32, 1.0, term_mode, max_iters, X_out, labels, iters, cell_labels);
}

/* ------------------------------------------------------ sampled variants */

/*
 * Eq.1 update (L68) of the m sampled points idx[] against the FULL float32
 * state X32 (n*d): the per-point definition, for sizes where the full O(n^2)
 * oracle is out of reach.  Xn_m: m*d fp64, nbr_m: m.
 */
int oracle_step_sample(const float *X32, int64_t n, int32_t d, float eps32, const int64_t *idx,
                       int64_t m, double *Xn_m, int32_t *nbr_m) {
    if (!X32 || !idx || !Xn_m || n < 1 || d < 1 || m < 0) return ORACLE_EINVAL;
    const double e = (double)eps32, e2 = e * e;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t k = 0; k < m; ++k) {
        int64_t p = idx[k];
        double *sum = (double *)calloc((size_t)d, sizeof(double));
        int64_t cnt = 0;
        for (int64_t q = 0; q < n; ++q) {
            double s = 0.0;
            for (int32_t i = 0; i < d; ++i) {
                double t = (double)X32[q * d + i] - (double)X32[p * d + i];
                s = s + t * t;
            }
            if (s <= e2) {
                ++cnt;
                for (int32_t i = 0; i < d; ++i)
                    sum[i] = sum[i] + sin((double)X32[q * d + i] - (double)X32[p * d + i]);
            }
        }
        for (int32_t i = 0; i < d; ++i)
            Xn_m[k * d + i] = (double)X32[p * d + i] + (1.0 / (double)cnt) * sum[i];
        if (nbr_m) nbr_m[k] = (int32_t)cnt;
        free(sum);
    }
    return ORACLE_OK;
}

/*
 * Theorem 4.7 (L133) on a final state, for sampled points: with clusters
 * given by labels[], label(p) == label(q)  <=>  ||p - q|| <= eps.
 * Returns the number of violating (p, q) pairs with p in idx[] (>= 0).
 */
int64_t oracle_terminal_sample(const float *X32, int64_t n, int32_t d, float eps32,
                               const int32_t *labels, const int64_t *idx, int64_t m) {
    if (!X32 || !labels || !idx || n < 1 || d < 1 || m < 0) return -1;
    const double e = (double)eps32, e2 = e * e;
    int64_t bad = 0;
#pragma omp parallel for schedule(dynamic, 1) reduction(+ : bad)
    for (int64_t k = 0; k < m; ++k) {
        int64_t p = idx[k];
        for (int64_t q = 0; q < n; ++q) {
            double s = 0.0;
            for (int32_t i = 0; i < d; ++i) {
                double t = (double)X32[q * d + i] - (double)X32[p * d + i];
                s = s + t * t;
            }
            int near = s <= e2;
            int same = labels[p] == labels[q];
            if (near != same) ++bad;
        }
    }
    return bad;
}
