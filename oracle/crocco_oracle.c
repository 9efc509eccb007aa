/*
 * crocco_oracle.c -- CPU fp64 ORACLE for the CRoCCo v2.0 hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no source, header, table or helper with the CUDA product path
 * (paper_conf_ipps_davissngmb23_b200/csrc); the only thing both sides see is
 * the seeded input generators in synth/.
 *
 * What it computes (citations are PAPER.md line numbers, /root/reference;
 * "reading N" = row N of the readings table in DESIGN.md section 3):
 *   - conservation laws, single species (Eq. 1-2; reading 1-2)
 *   - generalised curvilinear strong-conservation form (reading 4)
 *   - grid metrics from coordinates held in memory (Alg.1 l.2, 139, 149;
 *     reading 5-6): Thomas-Lombard metrics with the 6th-order central operator D6
 *   - ghost fill FillPatch + BC_Fill (Alg.2 l.3-4; reading 7,15,16)
 *   - WENO-SYMBO characteristic inviscid fluxes per direction WENOx/y/z
 *     (Alg.2 l.5-7; readings 8-11)
 *   - 4th-order central viscous + heat fluxes "Viscous" (Alg.2 l.8; reading 12)
 *   - low-storage RK3 "Update" (Alg.2 l.1,9; reading 13, Williamson 1980)
 *
 * Style: plain loops, full scratch arrays, one formula per statement, no
 * blocking, no fusion.  Compile with -O2 -ffp-contract=off (no FMA contraction).
 * Parity pins for every function are in tests/test_oracle_*.py.
 *
 * Array layout (all arrays fp64, component-major SoA, C order):
 *   a padded box with ghost width g around n[0] x n[1] x n[2] interior points:
 *   element (c, i, j, k), i in [-g, n0+g) ... , is at
 *     c*P0*P1*P2 + (i+g) + P0*((j+g) + P1*(k+g)),  Pd = n[d] + 2g.
 *   state / metric / rhs arrays use g = 4, coordinates use g = 10.
 *   metric components: 0 = J, 1 + 3*d + a = m^d_a = (d xi_d / d x_a) / J.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define OG 4   /* ghost width of state/metric arrays (reading 7) */
#define OGC 10 /* ghost width of the coordinate array (reading 7) */

enum { O_PERIODIC = 0, O_EXTRAP = 1, O_DIRICHLET = 2, O_WALL = 3 };
enum { O_INVISCID = 1, O_VISCOUS = 2 };
enum { O_FIELD_STATE = 0, O_FIELD_METRIC = 1 };

typedef struct {
    double gamma, R, Pr;
    int32_t mu_law;
    double mu_ref, T_ref, S;
    double weno_eps;
    int32_t terms, dir_mask;
    int32_t weno_linear; /* test flag: 1 forces omega_k = C_k (linear stencil) */
    int32_t weno_weights; /* 0: SYMBO (Martin et al. 2006), 1: SYMOO (reading 22, NEXT-3) */
    int32_t weno_limiter; /* bit 0: relative, bit 1: absolute limiter (reading 23, NEXT-3); 0 = off */
    double weno_alpha_rl, weno_alpha_al; /* thresholds of the two limiters */
    int32_t visc_form; /* 0: conservative point-flux form (reading 12), 1: expanded form with the
                          27-component metrics (readings 27-28, NEXT-3) */
} oracle_phys;

typedef struct {
    int64_t n[3];
    int64_t p[3];
    int64_t g;
    int64_t cs; /* component stride */
} obox;

static obox make_box(const int64_t n[3], int64_t g)
{
    obox b;
    for (int d = 0; d < 3; d++) {
        b.n[d] = n[d];
        b.p[d] = n[d] + 2 * g;
    }
    b.g = g;
    b.cs = b.p[0] * b.p[1] * b.p[2];
    return b;
}

static inline int64_t IX(const obox *b, int64_t i, int64_t j, int64_t k)
{
    return (i + b->g) + b->p[0] * ((j + b->g) + b->p[1] * (k + b->g));
}

static int g_threads = 0;
void oracle_set_threads(int n) { g_threads = n; }
int oracle_get_threads(void)
{
#ifdef _OPENMP
    return g_threads > 0 ? g_threads : omp_get_max_threads();
#else
    return 1;
#endif
}
#ifdef _OPENMP
#define OMP_THREADS num_threads(oracle_get_threads())
#endif

/* ------------------------------------------------------------------ */
/* 1. Ghost fill: FillPatch (periodic / inter-block copies) + BC_Fill  */
/*    (readings 15-16, 19-20).  Three ordered    */
/*    phases xi -> eta -> zeta; phase d spans the ghosts of directions */
/*    < d.  Kinds:                                                     */
/*      PERIODIC  copy from the periodic partner                       */
/*      EXTRAP    copy of the nearest interior layer                   */
/*      DIRICHLET constant conserved state                             */
/*      WALL      no-slip adiabatic: mirror, momentum negated          */
/*      SLIPWALL  inviscid reflecting wall (DMR): mirror,*/
/*                momentum reflected about the plane normal to         */
/*                n = m^d/|m^d| of the mirrored interior point         */
/*      SPLIT     boundary data switching at a moving index along a    */
/*                tangential axis (DMR bottom/top, reading 20): ghost  */
/*                points with g + 1/2 < s(t) = i0 + di_dt t take the   */
/*                left state, the others the right kind (DIRICHLET     */
/*                right state or SLIPWALL).                            */
/* ------------------------------------------------------------------ */
enum { O_SLIPWALL = 4, O_SPLIT = 5 };

typedef struct {
    int32_t axis;       /* tangential axis of the split (0..2) */
    double i0, di_dt;   /* split position s(t) = i0 + di_dt t, in global index units */
    double left[5];     /* conserved state where g + 1/2 < s(t) */
    int32_t right_kind; /* O_DIRICHLET or O_SLIPWALL elsewhere */
    double right[5];
} oracle_split;

/* COARSE_FINE faces (two-level AMR, section 9): the ghosts of a fine-level
   face inside the coarse domain are interpolated from the coarse level (FillPatchTwoLevels,
   PAPER.md:83, 129).  Without a coarse level (amr == NULL) they are left untouched. */
enum { O_COARSE_FINE = 6 };
#define O_MAX_SIB 8
typedef struct {
    int64_t nc[3];    /* coarse-level interior size (one global box, ghost width 4) */
    int64_t c0[3];    /* coarse node index of fine node 0 (refinement ratio 2) */
    const double *Uc; /* coarse state, padded, ghosts filled */
    /* same-level sibling patches (reading 31): sibling s has interior size sn[s], its node 0 at
       fine index so[s] of this patch (so = 2 (c0_s - c0)), state sU[s] (padded); NULL sU: none */
    int32_t nsib;
    int64_t so[O_MAX_SIB][3], sn[O_MAX_SIB][3];
    const double *sU[O_MAX_SIB];
} oracle_amr;
static void cf_interp(const oracle_amr *a, const int64_t f[3], double v[5]);
static void cf_value(const oracle_amr *a, const int64_t f[3], double v[5]);

static void fill_core(const int64_t n[3], const int32_t bc[6], const double dirichlet[30],
                      const oracle_split *split, double t, const double *met, double *f,
                      int32_t ncomp, int32_t kind, const oracle_amr *amr);

void oracle_fill_ex(const int64_t n[3], const int32_t bc[6], const double dirichlet[30],
                    const oracle_split *split, double t, const double *met, double *f,
                    int32_t ncomp, int32_t kind)
{
    fill_core(n, bc, dirichlet, split, t, met, f, ncomp, kind, NULL);
}

static void fill_core(const int64_t n[3], const int32_t bc[6], const double dirichlet[30],
                      const oracle_split *split, double t, const double *met, double *f,
                      int32_t ncomp, int32_t kind, const oracle_amr *amr)
{
    obox b = make_box(n, OG);
    for (int d = 0; d < 3; d++) {
        int64_t lo[3], hi[3];
        for (int e = 0; e < 3; e++) {
            lo[e] = (e < d) ? -OG : 0;
            hi[e] = (e < d) ? n[e] + OG : n[e];
        }
        for (int side = 0; side < 2; side++) {
            int kindbc = bc[2 * d + side];
            if (kind == O_FIELD_METRIC && kindbc != O_PERIODIC)
                continue; /* metrics: only periodic copies; physical faces keep computed ghosts */
            if (kindbc == O_COARSE_FINE && (amr == NULL || kind != O_FIELD_STATE))
                continue; /* no coarse level given: C/F ghosts untouched */
            const oracle_split *sp = (kindbc == O_SPLIT) ? &split[2 * d + side] : NULL;
            const double s_t = sp ? sp->i0 + sp->di_dt * t : 0.0;
            for (int64_t gg = 1; gg <= OG; gg++) {
                int64_t dst = side == 0 ? -gg : n[d] - 1 + gg;
                int64_t src;
                switch (kindbc) {
                case O_PERIODIC: src = side == 0 ? n[d] - gg : gg - 1; break;
                case O_EXTRAP: src = side == 0 ? 0 : n[d] - 1; break;
                case O_WALL:
                case O_SLIPWALL:
                case O_SPLIT: src = side == 0 ? gg - 1 : n[d] - gg; break; /* mirror */
                default: src = 0; break; /* DIRICHLET: constant state */
                }
                for (int64_t c2 = lo[(d + 2) % 3]; c2 < hi[(d + 2) % 3]; c2++)
                    for (int64_t c1 = lo[(d + 1) % 3]; c1 < hi[(d + 1) % 3]; c1++) {
                        int64_t id[3], is[3];
                        id[d] = dst;
                        is[d] = src;
                        id[(d + 1) % 3] = is[(d + 1) % 3] = c1;
                        id[(d + 2) % 3] = is[(d + 2) % 3] = c2;
                        int64_t pd = IX(&b, id[0], id[1], id[2]);
                        int64_t ps = IX(&b, is[0], is[1], is[2]);
                        /* effective kind of this ghost point */
                        int k = kindbc;
                        const double *cst = dirichlet + (2 * d + side) * 5;
                        if (sp) {
                            if ((double)id[sp->axis] + 0.5 < s_t) {
                                k = O_DIRICHLET;
                                cst = sp->left;
                            } else {
                                k = sp->right_kind;
                                cst = sp->right;
                            }
                        }
                        double v[5];
                        if (k == O_COARSE_FINE) {
                            cf_value(amr, id, v);
                            for (int c = 0; c < 5; c++)
                                f[c * b.cs + pd] = v[c];
                            continue;
                        }
                        for (int c = 0; c < ncomp; c++)
                            v[c] = (k == O_DIRICHLET) ? cst[c] : f[c * b.cs + ps];
                        if (k == O_WALL)
                            for (int c = 1; c <= 3; c++)
                                v[c] = -v[c];
                        if (k == O_SLIPWALL) {
                            double m[3], mm = 0.0, mdot = 0.0;
                            for (int a = 0; a < 3; a++) {
                                m[a] = met[(1 + 3 * d + a) * b.cs + ps];
                                mm = mm + m[a] * m[a];
                            }
                            mm = sqrt(mm);
                            for (int a = 0; a < 3; a++) {
                                m[a] = m[a] / mm;
                                mdot = mdot + v[1 + a] * m[a];
                            }
                            for (int a = 0; a < 3; a++)
                                v[1 + a] = v[1 + a] - 2.0 * mdot * m[a];
                        }
                        for (int c = 0; c < ncomp; c++)
                            f[c * b.cs + pd] = v[c];
                    }
            }
        }
    }
}

void oracle_fill(const int64_t n[3], const int32_t bc[6], const double dirichlet[30],
                 double *f, int32_t ncomp, int32_t kind)
{
    oracle_fill_ex(n, bc, dirichlet, NULL, 0.0, NULL, f, ncomp, kind);
}

/* ------------------------------------------------------------------ */
/* 2. Grid metrics (readings 5-6).              */
/*    D6 f_i = [45(f_{i+1}-f_{i-1}) - 9(f_{i+2}-f_{i-2}) + (f_{i+3}-f_{i-3})]/60 */
/*    dx[a][d] = D6_d x_a ;  1/J = det(dx)                             */
/*    m^d_a = D6_{d+2}[(D6_{d+1} x_{a+1}) x_{a+2}]                     */
/*          - D6_{d+1}[(D6_{d+2} x_{a+1}) x_{a+2}]   (indices mod 3)   */
/* ------------------------------------------------------------------ */
static double d6(const double *f, int64_t p, int64_t s)
{
    return (45.0 * (f[p + s] - f[p - s]) - 9.0 * (f[p + 2 * s] - f[p - 2 * s]) +
            (f[p + 3 * s] - f[p - 3 * s])) / 60.0;
}

void oracle_metrics(const int64_t n[3], const int32_t bc[6], const double *xyz, double *met)
{
    obox bc_ = make_box(n, OGC); /* coordinate box */
    obox bm = make_box(n, OG);   /* metric box */
    int64_t sc[3] = {1, bc_.p[0], bc_.p[0] * bc_.p[1]};
    const int64_t W1 = OG + 3; /* derivatives needed on interior +-7 */

    /* dx[a][d] on the coordinate layout */
    double *dx = (double *)calloc((size_t)(9 * bc_.cs), sizeof(double));
    for (int a = 0; a < 3; a++)
        for (int d = 0; d < 3; d++) {
            const double *x = xyz + a * bc_.cs;
            double *out = dx + (3 * a + d) * bc_.cs;
#pragma omp parallel for OMP_THREADS
            for (int64_t k = -W1; k < n[2] + W1; k++)
                for (int64_t j = -W1; j < n[1] + W1; j++)
                    for (int64_t i = -W1; i < n[0] + W1; i++) {
                        int64_t p = IX(&bc_, i, j, k);
                        out[p] = d6(x, p, sc[d]);
                    }
        }

    /* product fields P[a][d][e] = (D6_e x_{a+1}) * x_{a+2}, then outer D6 */
    double *prod = (double *)calloc((size_t)bc_.cs, sizeof(double));
    for (int d = 0; d < 3; d++)
        for (int a = 0; a < 3; a++) {
            int d1 = (d + 1) % 3, d2 = (d + 2) % 3;
            int a1 = (a + 1) % 3, a2 = (a + 2) % 3;
            double *m = met + (1 + 3 * d + a) * bm.cs;
            /* term 1: D6_{d2}[ (D6_{d1} x_{a1}) x_{a2} ] */
            const double *x2 = xyz + a2 * bc_.cs;
            const double *g1 = dx + (3 * a1 + d1) * bc_.cs;
#pragma omp parallel for OMP_THREADS
            for (int64_t k = -W1; k < n[2] + W1; k++)
                for (int64_t j = -W1; j < n[1] + W1; j++)
                    for (int64_t i = -W1; i < n[0] + W1; i++) {
                        int64_t p = IX(&bc_, i, j, k);
                        prod[p] = g1[p] * x2[p];
                    }
#pragma omp parallel for OMP_THREADS
            for (int64_t k = -OG; k < n[2] + OG; k++)
                for (int64_t j = -OG; j < n[1] + OG; j++)
                    for (int64_t i = -OG; i < n[0] + OG; i++)
                        m[IX(&bm, i, j, k)] = d6(prod, IX(&bc_, i, j, k), sc[d2]);
            /* term 2: - D6_{d1}[ (D6_{d2} x_{a1}) x_{a2} ] */
            const double *g2 = dx + (3 * a1 + d2) * bc_.cs;
#pragma omp parallel for OMP_THREADS
            for (int64_t k = -W1; k < n[2] + W1; k++)
                for (int64_t j = -W1; j < n[1] + W1; j++)
                    for (int64_t i = -W1; i < n[0] + W1; i++) {
                        int64_t p = IX(&bc_, i, j, k);
                        prod[p] = g2[p] * x2[p];
                    }
#pragma omp parallel for OMP_THREADS
            for (int64_t k = -OG; k < n[2] + OG; k++)
                for (int64_t j = -OG; j < n[1] + OG; j++)
                    for (int64_t i = -OG; i < n[0] + OG; i++)
                        m[IX(&bm, i, j, k)] = m[IX(&bm, i, j, k)] - d6(prod, IX(&bc_, i, j, k), sc[d1]);
        }

    /* J = 1 / det(dx) */
#pragma omp parallel for OMP_THREADS
    for (int64_t k = -OG; k < n[2] + OG; k++)
        for (int64_t j = -OG; j < n[1] + OG; j++)
            for (int64_t i = -OG; i < n[0] + OG; i++) {
                int64_t p = IX(&bc_, i, j, k);
                double M[3][3];
                for (int a = 0; a < 3; a++)
                    for (int d = 0; d < 3; d++)
                        M[a][d] = dx[(3 * a + d) * bc_.cs + p];
                double det = M[0][0] * (M[1][1] * M[2][2] - M[1][2] * M[2][1]) -
                             M[0][1] * (M[1][0] * M[2][2] - M[1][2] * M[2][0]) +
                             M[0][2] * (M[1][0] * M[2][1] - M[1][1] * M[2][0]);
                met[IX(&bm, i, j, k)] = 1.0 / det;
            }
    free(prod);
    free(dx);
    /* periodic ghost metrics are copies from the owners (reading 6) */
    oracle_fill(n, bc, NULL, met, 10, O_FIELD_METRIC);
}

/* ------------------------------------------------------------------ */
/* 3. WENO-SYMBO reconstruction (PAPER.md:50 -> ref [9]; reading 8)   */
/*    W(v_{-2..3}) reconstructs the value at the +1/2 interface.       */
/* ------------------------------------------------------------------ */
static const double C_SYMBO[4] = {0.094647545896, 0.428074212384, 0.408289331408, 0.068988910311};
static const double C_SYMOO[4] = {1.0 / 20.0, 9.0 / 20.0, 9.0 / 20.0, 1.0 / 20.0};

/* WENO limiters (reading 23; [lit] Taylor, Wu & Martin 2007, not in the
   paper): after the downwind substitution, the reconstruction falls back to the linear
   optimal weights omega_k = C_k when
     (limiter & 1) and max_k beta_k < alpha_rl * min_k beta_k   (relative limiter), or
     (limiter & 2) and max_k beta_k < alpha_al                  (absolute limiter).      */
double oracle_weno_lim(const double v[6], double eps, int linear, int weights, int limiter,
                       double alpha_rl, double alpha_al);

double oracle_weno(const double v[6], double eps, int linear, int weights)
{
    return oracle_weno_lim(v, eps, linear, weights, 0, 0.0, 0.0);
}

double oracle_weno_lim(const double v[6], double eps, int linear, int weights, int limiter,
                       double alpha_rl, double alpha_al)
{
    const double *Cw = weights == 1 ? C_SYMOO : C_SYMBO;
    /* v[0..5] = v_{-2}, v_{-1}, v_0, v_1, v_2, v_3 */
    double q[4], beta[4];
    q[0] = v[0] / 3.0 - 7.0 * v[1] / 6.0 + 11.0 * v[2] / 6.0;
    q[1] = -v[1] / 6.0 + 5.0 * v[2] / 6.0 + v[3] / 3.0;
    q[2] = v[2] / 3.0 + 5.0 * v[3] / 6.0 - v[4] / 6.0;
    q[3] = 11.0 * v[3] / 6.0 - 7.0 * v[4] / 6.0 + v[5] / 3.0;
    double t;
    t = v[0] - 2.0 * v[1] + v[2];
    beta[0] = 13.0 / 12.0 * t * t;
    t = v[0] - 4.0 * v[1] + 3.0 * v[2];
    beta[0] = beta[0] + 0.25 * t * t;
    t = v[1] - 2.0 * v[2] + v[3];
    beta[1] = 13.0 / 12.0 * t * t;
    t = v[1] - v[3];
    beta[1] = beta[1] + 0.25 * t * t;
    t = v[2] - 2.0 * v[3] + v[4];
    beta[2] = 13.0 / 12.0 * t * t;
    t = 3.0 * v[2] - 4.0 * v[3] + v[4];
    beta[2] = beta[2] + 0.25 * t * t;
    t = v[3] - 2.0 * v[4] + v[5];
    beta[3] = 13.0 / 12.0 * t * t;
    t = -5.0 * v[3] + 8.0 * v[4] - 3.0 * v[5];
    beta[3] = beta[3] + 0.25 * t * t;
    /* the downwind stencil is never the smoothest: beta_3 = max(beta_0..beta_3) */
    double bmax = beta[0];
    for (int k = 1; k < 4; k++)
        if (beta[k] > bmax)
            bmax = beta[k];
    beta[3] = bmax;
    if (limiter) {
        double bmin = beta[0];
        for (int k = 1; k < 4; k++)
            if (beta[k] < bmin)
                bmin = beta[k];
        if ((limiter & 1) && bmax < alpha_rl * bmin)
            linear = 1;
        if ((limiter & 2) && bmax < alpha_al)
            linear = 1;
    }
    double alpha[4], asum = 0.0, num = 0.0;
    for (int k = 0; k < 4; k++) {
        if (linear)
            alpha[k] = Cw[k];
        else
            alpha[k] = Cw[k] / ((eps + beta[k]) * (eps + beta[k]));
        asum = asum + alpha[k];
    }
    for (int k = 0; k < 4; k++)
        num = num + alpha[k] * q[k];
    return num / asum;
}

double oracle_weno_symbo(const double v[6], double eps, int linear)
{
    return oracle_weno(v, eps, linear, 0);
}

/* ------------------------------------------------------------------ */
/* 4. Pulliam-Chaussee eigenvectors of A_n = dF_n/dU (reading 9)      */
/*    Columns of T <-> eigenvalues (theta, theta, theta, theta+c, theta-c). */
/* ------------------------------------------------------------------ */
void oracle_eigvecs(const double nrm[3], double rho, double u, double v, double w, double c,
                    double gamma, double T[25], double Ti[25])
{
    double nx = nrm[0], ny = nrm[1], nz = nrm[2];
    double gm1 = gamma - 1.0;
    double phi2 = 0.5 * gm1 * (u * u + v * v + w * w);
    double alpha = rho / (sqrt(2.0) * c);
    double beta = 1.0 / (sqrt(2.0) * rho * c);
    double theta = nx * u + ny * v + nz * w;
    double c2 = c * c;
    /* right eigenvectors, row-major T[r*5+s] */
    T[0] = nx;
    T[1] = ny;
    T[2] = nz;
    T[3] = alpha;
    T[4] = alpha;
    T[5] = nx * u;
    T[6] = ny * u - nz * rho;
    T[7] = nz * u + ny * rho;
    T[8] = alpha * (u + nx * c);
    T[9] = alpha * (u - nx * c);
    T[10] = nx * v + nz * rho;
    T[11] = ny * v;
    T[12] = nz * v - nx * rho;
    T[13] = alpha * (v + ny * c);
    T[14] = alpha * (v - ny * c);
    T[15] = nx * w - ny * rho;
    T[16] = ny * w + nx * rho;
    T[17] = nz * w;
    T[18] = alpha * (w + nz * c);
    T[19] = alpha * (w - nz * c);
    T[20] = nx * phi2 / gm1 + rho * (nz * v - ny * w);
    T[21] = ny * phi2 / gm1 + rho * (nx * w - nz * u);
    T[22] = nz * phi2 / gm1 + rho * (ny * u - nx * v);
    T[23] = alpha * ((phi2 + c2) / gm1 + c * theta);
    T[24] = alpha * ((phi2 + c2) / gm1 - c * theta);
    /* left eigenvectors T^{-1} */
    Ti[0] = nx * (1.0 - phi2 / c2) - (nz * v - ny * w) / rho;
    Ti[1] = nx * gm1 * u / c2;
    Ti[2] = nz / rho + nx * gm1 * v / c2;
    Ti[3] = -ny / rho + nx * gm1 * w / c2;
    Ti[4] = -nx * gm1 / c2;
    Ti[5] = ny * (1.0 - phi2 / c2) - (nx * w - nz * u) / rho;
    Ti[6] = -nz / rho + ny * gm1 * u / c2;
    Ti[7] = ny * gm1 * v / c2;
    Ti[8] = nx / rho + ny * gm1 * w / c2;
    Ti[9] = -ny * gm1 / c2;
    Ti[10] = nz * (1.0 - phi2 / c2) - (ny * u - nx * v) / rho;
    Ti[11] = ny / rho + nz * gm1 * u / c2;
    Ti[12] = -nx / rho + nz * gm1 * v / c2;
    Ti[13] = nz * gm1 * w / c2;
    Ti[14] = -nz * gm1 / c2;
    Ti[15] = beta * (phi2 - c * theta);
    Ti[16] = beta * (nx * c - gm1 * u);
    Ti[17] = beta * (ny * c - gm1 * v);
    Ti[18] = beta * (nz * c - gm1 * w);
    Ti[19] = beta * gm1;
    Ti[20] = beta * (phi2 + c * theta);
    Ti[21] = -beta * (nx * c + gm1 * u);
    Ti[22] = -beta * (ny * c + gm1 * v);
    Ti[23] = -beta * (nz * c + gm1 * w);
    Ti[24] = beta * gm1;
}

/* ------------------------------------------------------------------ */
/* 4b. Roe average of the states at points i (UL) and i+1 (UR)         */
/*     (reading 9; [lit] Roe 1981, J. Comput. Phys. 43:357):            */
/*     r = sqrt(rho_R/rho_L), (u,v,w,H)~ = (q_L + r q_R)/(1+r),          */
/*     rho~ = r rho_L, c~ = sqrt((gamma-1)(H~ - |u~|^2/2)).             */
/*     out = (rho~, u~, v~, w~, c~).                                    */
/* ------------------------------------------------------------------ */
void oracle_roe_state(const double UL[5], const double UR[5], double gamma, double out[5])
{
    const double gm1 = gamma - 1.0;
    const double *U2 = UL, *U3 = UR;
    double uL = U2[1] / U2[0], vL = U2[2] / U2[0], wL = U2[3] / U2[0];
    double uR = U3[1] / U3[0], vR = U3[2] / U3[0], wR = U3[3] / U3[0];
    double pL = gm1 * (U2[4] - 0.5 * U2[0] * (uL * uL + vL * vL + wL * wL));
    double pR = gm1 * (U3[4] - 0.5 * U3[0] * (uR * uR + vR * vR + wR * wR));
    double HL = (U2[4] + pL) / U2[0], HR = (U3[4] + pR) / U3[0];
    double r = sqrt(U3[0] / U2[0]);
    double ut = (uL + r * uR) / (1.0 + r);
    double vt = (vL + r * vR) / (1.0 + r);
    double wt = (wL + r * wR) / (1.0 + r);
    double Ht = (HL + r * HR) / (1.0 + r);
    out[0] = r * U2[0];
    out[1] = ut;
    out[2] = vt;
    out[3] = wt;
    out[4] = sqrt(gm1 * (Ht - 0.5 * (ut * ut + vt * vt + wt * wt)));
}

/* ------------------------------------------------------------------ */
/* 5. Characteristic WENO interface flux (PAPER.md:50, 110-112;        */
/*    readings 8-11).  Inputs: the 6 conserved states U_{i-2..i+3} and */
/*    the metric row m^d at the same 6 points.  Output F^_{i+1/2}.     */
/* ------------------------------------------------------------------ */
void oracle_interface_flux(const oracle_phys *ph, const double Ul[30], const double ml[18],
                           double Fhat[5])
{
    const double gam = ph->gamma, gm1 = ph->gamma - 1.0;
    /* frozen interface metric: R6 reconstruction (reading 6) */
    double mh[3];
    for (int a = 0; a < 3; a++)
        mh[a] = (37.0 * (ml[2 * 3 + a] + ml[3 * 3 + a]) - 8.0 * (ml[1 * 3 + a] + ml[4 * 3 + a]) +
                 (ml[0 * 3 + a] + ml[5 * 3 + a])) / 60.0;
    double mag = sqrt(mh[0] * mh[0] + mh[1] * mh[1] + mh[2] * mh[2]);
    double nrm[3] = {mh[0] / mag, mh[1] / mag, mh[2] / mag};

    /* primitive variables at the 6 points */
    double rho[6], u[6], v[6], w[6], p[6], c[6];
    for (int l = 0; l < 6; l++) {
        const double *U = Ul + 5 * l;
        rho[l] = U[0];
        u[l] = U[1] / U[0];
        v[l] = U[2] / U[0];
        w[l] = U[3] / U[0];
        p[l] = gm1 * (U[4] - 0.5 * rho[l] * (u[l] * u[l] + v[l] * v[l] + w[l] * w[l]));
        c[l] = sqrt(gam * p[l] / rho[l]);
    }
    /* Roe average of points i (l=2) and i+1 (l=3), section 4b */
    double roe[5];
    oracle_roe_state(Ul + 5 * 2, Ul + 5 * 3, gam, roe);
    double T[25], Ti[25];
    oracle_eigvecs(nrm, roe[0], roe[1], roe[2], roe[3], roe[4], gam, T, Ti);

    /* projected fluxes and states, characteristic speeds */
    double g[5][6], wv[5][6], lam[5];
    for (int s = 0; s < 5; s++)
        lam[s] = 0.0;
    for (int l = 0; l < 6; l++) {
        const double *U = Ul + 5 * l;
        double th = nrm[0] * u[l] + nrm[1] * v[l] + nrm[2] * w[l];
        double Fn[5];
        Fn[0] = rho[l] * th;
        Fn[1] = U[1] * th + nrm[0] * p[l];
        Fn[2] = U[2] * th + nrm[1] * p[l];
        Fn[3] = U[3] * th + nrm[2] * p[l];
        Fn[4] = (U[4] + p[l]) * th;
        double eig[5] = {th, th, th, th + c[l], th - c[l]};
        for (int s = 0; s < 5; s++) {
            double gs = 0.0, ws = 0.0;
            for (int q = 0; q < 5; q++) {
                gs = gs + Ti[5 * s + q] * Fn[q];
                ws = ws + Ti[5 * s + q] * U[q];
            }
            g[s][l] = gs;
            wv[s][l] = ws;
            if (fabs(eig[s]) > lam[s])
                lam[s] = fabs(eig[s]);
        }
    }
    /* local Lax-Friedrichs splitting + WENO-SYMBO per characteristic field */
    double gh[5];
    for (int s = 0; s < 5; s++) {
        double vp[6], vm[6];
        for (int l = 0; l < 6; l++) {
            vp[l] = 0.5 * (g[s][l] + lam[s] * wv[s][l]);
            vm[5 - l] = 0.5 * (g[s][l] - lam[s] * wv[s][l]); /* mirrored: i+3 .. i-2 */
        }
        gh[s] = oracle_weno_lim(vp, ph->weno_eps, ph->weno_linear, ph->weno_weights, ph->weno_limiter,
                                ph->weno_alpha_rl, ph->weno_alpha_al) +
                oracle_weno_lim(vm, ph->weno_eps, ph->weno_linear, ph->weno_weights, ph->weno_limiter,
                                ph->weno_alpha_rl, ph->weno_alpha_al);
    }
    for (int q = 0; q < 5; q++) {
        double f = 0.0;
        for (int s = 0; s < 5; s++)
            f = f + T[5 * q + s] * gh[s];
        Fhat[q] = mag * f;
    }
}

/* ------------------------------------------------------------------ */
/* 6. Right-hand side (readings 4, 12)        */
/*    rhs = J ( -sum_d delta_d F^_inv^d + sum_d D4_d F^_v^d )          */
/*    on interior points; U must have its ghosts filled.               */
/* ------------------------------------------------------------------ */
static double mu_of_T(const oracle_phys *ph, double T)
{
    if (ph->mu_law == 1) {
        double t = T / ph->T_ref;
        return ph->mu_ref * t * sqrt(t) * (ph->T_ref + ph->S) / (T + ph->S);
    }
    return ph->mu_ref;
}

static double d4(const double *f, int64_t p, int64_t s)
{
    return (8.0 * (f[p + s] - f[p - s]) - (f[p + 2 * s] - f[p - 2 * s])) / 12.0;
}

static void rhs_core(const int64_t n[3], const oracle_phys *ph, const double *U, const double *met,
                     const double *met2, double *rhs);

void oracle_metrics2(const int64_t n[3], const double *met, double *met2);

void oracle_rhs(const int64_t n[3], const oracle_phys *ph, const double *U, const double *met,
                double *rhs)
{
    if (ph->visc_form == 1 && (ph->terms & O_VISCOUS)) {
        obox b = make_box(n, OG);
        double *met2 = (double *)calloc((size_t)(18 * b.cs), sizeof(double));
        oracle_metrics2(n, met, met2);
        rhs_core(n, ph, U, met, met2, rhs);
        free(met2);
        return;
    }
    rhs_core(n, ph, U, met, NULL, rhs);
}

void oracle_rhs_ex(const int64_t n[3], const oracle_phys *ph, const double *U, const double *met,
                   const double *met2, double *rhs)
{
    rhs_core(n, ph, U, met, met2, rhs);
}

static void visc_expanded(const int64_t n[3], const oracle_phys *ph, const double *U,
                          const double *met, const double *met2, double *V);

static void rhs_core(const int64_t n[3], const oracle_phys *ph, const double *U, const double *met,
                     const double *met2, double *rhs)
{
    obox b = make_box(n, OG);
    const int64_t cs = b.cs;
    int64_t st[3] = {1, b.p[0], b.p[0] * b.p[1]};
    double *R = (double *)calloc((size_t)(5 * cs), sizeof(double));

    /* --- inviscid: WENOx, WENOy, WENOz (Alg. 2 l.5-7) --- */
    if (ph->terms & O_INVISCID) {
        for (int d = 0; d < 3; d++) {
            if (!(ph->dir_mask & (1 << d)))
                continue;
            int e1 = (d + 1) % 3, e2 = (d + 2) % 3;
            /* F[c][ (i+1) + (n_d+1)*line ] for interfaces i+1/2, i = -1 .. n_d-1 */
            int64_t nl = n[e1] * n[e2];
            double *F = (double *)malloc((size_t)(5 * (n[d] + 1) * nl) * sizeof(double));
#pragma omp parallel for OMP_THREADS
            for (int64_t line = 0; line < nl; line++) {
                int64_t idx[3];
                idx[e1] = line % n[e1];
                idx[e2] = line / n[e1];
                for (int64_t i = -1; i < n[d]; i++) {
                    double Ul[30], ml[18], Fh[5];
                    for (int l = 0; l < 6; l++) {
                        idx[d] = i - 2 + l;
                        int64_t p = IX(&b, idx[0], idx[1], idx[2]);
                        for (int c = 0; c < 5; c++)
                            Ul[5 * l + c] = U[c * cs + p];
                        for (int a = 0; a < 3; a++)
                            ml[3 * l + a] = met[(1 + 3 * d + a) * cs + p];
                    }
                    oracle_interface_flux(ph, Ul, ml, Fh);
                    for (int c = 0; c < 5; c++)
                        F[c * (n[d] + 1) * nl + (i + 1) + (n[d] + 1) * line] = Fh[c];
                }
            }
#pragma omp parallel for OMP_THREADS
            for (int64_t line = 0; line < nl; line++) {
                int64_t idx[3];
                idx[e1] = line % n[e1];
                idx[e2] = line / n[e1];
                for (int64_t i = 0; i < n[d]; i++) {
                    idx[d] = i;
                    int64_t p = IX(&b, idx[0], idx[1], idx[2]);
                    for (int c = 0; c < 5; c++) {
                        double fp = F[c * (n[d] + 1) * nl + (i + 1) + (n[d] + 1) * line];
                        double fm = F[c * (n[d] + 1) * nl + i + (n[d] + 1) * line];
                        R[c * cs + p] = R[c * cs + p] - (fp - fm);
                    }
                }
            }
            free(F);
        }
    }

    /* --- viscous and heat fluxes (Alg. 2 l.8) --- */
    double *Vx = NULL; /* expanded form: physical-space viscous divergence at interior points */
    if ((ph->terms & O_VISCOUS) && ph->visc_form == 1) {
        Vx = (double *)calloc((size_t)(5 * cs), sizeof(double));
        visc_expanded(n, ph, U, met, met2, Vx);
    } else if (ph->terms & O_VISCOUS) {
        const double gm1 = ph->gamma - 1.0;
        const double cp = ph->gamma * ph->R / gm1;
        double *pr = (double *)malloc((size_t)(4 * cs) * sizeof(double)); /* u v w T */
#pragma omp parallel for OMP_THREADS
        for (int64_t p = 0; p < cs; p++) {
            double rho = U[p];
            double u = U[cs + p] / rho, v = U[2 * cs + p] / rho, w = U[3 * cs + p] / rho;
            double pres = gm1 * (U[4 * cs + p] - 0.5 * rho * (u * u + v * v + w * w));
            pr[p] = u;
            pr[cs + p] = v;
            pr[2 * cs + p] = w;
            pr[3 * cs + p] = pres / (rho * ph->R);
        }
        /* point viscous fluxes Fv[d][q], q = 0..3 -> momentum x,y,z and energy,
           on the interior +-2 box */
        double *Fv = (double *)calloc((size_t)(12 * cs), sizeof(double));
#pragma omp parallel for OMP_THREADS
        for (int64_t k = -2; k < n[2] + 2; k++)
            for (int64_t j = -2; j < n[1] + 2; j++)
                for (int64_t i = -2; i < n[0] + 2; i++) {
                    int64_t p = IX(&b, i, j, k);
                    double gc[4][3]; /* d phi / d xi_d */
                    for (int f = 0; f < 4; f++)
                        for (int d = 0; d < 3; d++)
                            gc[f][d] = d4(pr + f * cs, p, st[d]);
                    double J = met[p];
                    double m[3][3];
                    for (int d = 0; d < 3; d++)
                        for (int a = 0; a < 3; a++)
                            m[d][a] = met[(1 + 3 * d + a) * cs + p];
                    double gx[4][3]; /* d phi / d x_a = J sum_d m^d_a phi_,d */
                    for (int f = 0; f < 4; f++)
                        for (int a = 0; a < 3; a++) {
                            double s = 0.0;
                            for (int d = 0; d < 3; d++)
                                s = s + m[d][a] * gc[f][d];
                            gx[f][a] = J * s;
                        }
                    double T = pr[3 * cs + p];
                    double mu = mu_of_T(ph, T);
                    double kap = mu * cp / ph->Pr;
                    double div = gx[0][0] + gx[1][1] + gx[2][2];
                    double tau[3][3], q[3], vel[3];
                    for (int a = 0; a < 3; a++)
                        for (int bb = 0; bb < 3; bb++) {
                            tau[a][bb] = mu * (gx[a][bb] + gx[bb][a]);
                            if (a == bb)
                                tau[a][bb] = tau[a][bb] - 2.0 / 3.0 * mu * div;
                        }
                    for (int a = 0; a < 3; a++) {
                        q[a] = -kap * gx[3][a];
                        vel[a] = pr[a * cs + p];
                    }
                    for (int d = 0; d < 3; d++) {
                        for (int a = 0; a < 3; a++) {
                            double s = 0.0;
                            for (int bb = 0; bb < 3; bb++)
                                s = s + m[d][bb] * tau[a][bb];
                            Fv[(4 * d + a) * cs + p] = s;
                        }
                        double s = 0.0;
                        for (int bb = 0; bb < 3; bb++) {
                            double work = 0.0;
                            for (int a = 0; a < 3; a++)
                                work = work + vel[a] * tau[a][bb];
                            s = s + m[d][bb] * (work - q[bb]);
                        }
                        Fv[(4 * d + 3) * cs + p] = s;
                    }
                }
#pragma omp parallel for OMP_THREADS
        for (int64_t k = 0; k < n[2]; k++)
            for (int64_t j = 0; j < n[1]; j++)
                for (int64_t i = 0; i < n[0]; i++) {
                    int64_t p = IX(&b, i, j, k);
                    for (int q = 0; q < 4; q++)
                        for (int d = 0; d < 3; d++)
                            R[(1 + q) * cs + p] = R[(1 + q) * cs + p] + d4(Fv + (4 * d + q) * cs, p, st[d]);
                }
        free(Fv);
        free(pr);
    }

    /* --- rhs = J * R on interior points --- */
#pragma omp parallel for OMP_THREADS
    for (int64_t k = 0; k < n[2]; k++)
        for (int64_t j = 0; j < n[1]; j++)
            for (int64_t i = 0; i < n[0]; i++) {
                int64_t p = IX(&b, i, j, k);
                for (int c = 0; c < 5; c++) {
                    rhs[c * cs + p] = met[p] * R[c * cs + p];
                    if (Vx)
                        rhs[c * cs + p] = rhs[c * cs + p] + Vx[c * cs + p];
                }
            }
    free(R);
    free(Vx);
}

/* ------------------------------------------------------------------ */
/* 6b. The paper's 27-component metric set and the expanded viscous    */
/*     form ("first and second order grid metrics ... a    */
/*     27-component MultiFab"; readings 27-28).          */
/*     First metrics xi_{a,j} = d xi_a / d x_j = J m^a_j (9, from the   */
/*     10-component set); second metrics                                */
/*       xi_{a,jk} = d/dx_k (xi_{a,j}) = sum_b xi_{b,k} D6_b(xi_{a,j})   */
/*     for j <= k (18): component 6a + P(j,k), pairs P = (00, 01, 02,   */
/*     11, 12, 22).  Interior points only.                              */
/* ------------------------------------------------------------------ */
static const int PJ[6] = {0, 0, 0, 1, 1, 2}, PK[6] = {0, 1, 2, 1, 2, 2};
static int pair_of(int j, int k)
{
    int lo = j < k ? j : k, hi = j < k ? k : j;
    return lo == 0 ? hi : (lo == 1 ? 2 + hi : 5);
}

void oracle_metrics2(const int64_t n[3], const double *met, double *met2)
{
    obox b = make_box(n, OG);
    const int64_t cs = b.cs;
    int64_t st[3] = {1, b.p[0], b.p[0] * b.p[1]};
    /* xi_{a,j} on the whole padded box */
    double *xi = (double *)malloc((size_t)(9 * cs) * sizeof(double));
    for (int a = 0; a < 3; a++)
        for (int j = 0; j < 3; j++)
            for (int64_t p = 0; p < cs; p++)
                xi[(3 * a + j) * cs + p] = met[p] * met[(1 + 3 * a + j) * cs + p];
#pragma omp parallel for OMP_THREADS
    for (int64_t k = 0; k < n[2]; k++)
        for (int64_t j = 0; j < n[1]; j++)
            for (int64_t i = 0; i < n[0]; i++) {
                int64_t p = IX(&b, i, j, k);
                for (int a = 0; a < 3; a++)
                    for (int q = 0; q < 6; q++) {
                        int jj = PJ[q], kk = PK[q];
                        double s = 0.0;
                        for (int bb = 0; bb < 3; bb++)
                            s = s + xi[(3 * bb + kk) * cs + p] * d6(xi + (3 * a + jj) * cs, p, st[bb]);
                        met2[(6 * a + q) * cs + p] = s;
                    }
            }
    free(xi);
}

/* d mu / d T of the viscosity law (reading 2) */
static double dmu_dT(const oracle_phys *ph, double T)
{
    if (ph->mu_law == 1)
        return mu_of_T(ph, T) * (1.5 / T - 1.0 / (T + ph->S));
    return 0.0;
}

/* 4th-order central second derivative (5 points) */
static double d2(const double *f, int64_t p, int64_t s)
{
    return (16.0 * (f[p + s] + f[p - s]) - (f[p + 2 * s] + f[p - 2 * s]) - 30.0 * f[p]) / 12.0;
}

/* Expanded viscous form (reading 28): V = div F_v evaluated pointwise with the chain rule,
     G_ij = d u_i/d x_j = sum_a xi_{a,j} D4_a u_i,   g_j = sum_a xi_{a,j} D4_a T,
     d2 phi/dx_j dx_k = sum_{a,b} xi_{a,j} xi_{b,k} phi_ab + sum_a xi_{a,jk} phi_a,
       phi_aa = D2_a phi (5-point 4th order), phi_ab = D4_a(D4_b phi) (a != b),
     d tau_ij/d x_j = mu (lap u_i + (1/3) d_i div u) + sum_j (mu' g_j)(G_ij + G_ji - (2/3) delta_ij div u),
     V_{1+i} = d tau_ij / d x_j,
     V_4 = u_i d tau_ij/d x_j + tau_ij G_ij + kappa lap T + (c_p/Pr) mu' |g|^2,  V_0 = 0. */
static void visc_expanded(const int64_t n[3], const oracle_phys *ph, const double *U,
                          const double *met, const double *met2, double *V)
{
    obox b = make_box(n, OG);
    const int64_t cs = b.cs;
    int64_t st[3] = {1, b.p[0], b.p[0] * b.p[1]};
    const double gm1 = ph->gamma - 1.0;
    const double cp = ph->gamma * ph->R / gm1;
    double *pr = (double *)malloc((size_t)(4 * cs) * sizeof(double)); /* u v w T */
    for (int64_t p = 0; p < cs; p++) {
        double rho = U[p];
        double u = U[cs + p] / rho, v = U[2 * cs + p] / rho, w = U[3 * cs + p] / rho;
        double pres = gm1 * (U[4 * cs + p] - 0.5 * rho * (u * u + v * v + w * w));
        pr[p] = u;
        pr[cs + p] = v;
        pr[2 * cs + p] = w;
        pr[3 * cs + p] = pres / (rho * ph->R);
    }
    /* first computational derivatives D4_b phi on the interior +-2 box (for the mixed ones) */
    double *dphi = (double *)calloc((size_t)(12 * cs), sizeof(double)); /* [4 fields][3 dirs] */
    for (int64_t k = -2; k < n[2] + 2; k++)
        for (int64_t j = -2; j < n[1] + 2; j++)
            for (int64_t i = -2; i < n[0] + 2; i++) {
                int64_t p = IX(&b, i, j, k);
                for (int f = 0; f < 4; f++)
                    for (int d = 0; d < 3; d++)
                        dphi[(3 * f + d) * cs + p] = d4(pr + f * cs, p, st[d]);
            }
#pragma omp parallel for OMP_THREADS
    for (int64_t k = 0; k < n[2]; k++)
        for (int64_t j = 0; j < n[1]; j++)
            for (int64_t i = 0; i < n[0]; i++) {
                int64_t p = IX(&b, i, j, k);
                double xi[3][3], xi2[3][6];
                for (int a = 0; a < 3; a++)
                    for (int c = 0; c < 3; c++)
                        xi[a][c] = met[p] * met[(1 + 3 * a + c) * cs + p];
                for (int a = 0; a < 3; a++)
                    for (int q = 0; q < 6; q++)
                        xi2[a][q] = met2[(6 * a + q) * cs + p];
                double ph1[4][3], ph2[4][3][3]; /* phi_a, phi_ab */
                for (int f = 0; f < 4; f++) {
                    for (int a = 0; a < 3; a++)
                        ph1[f][a] = dphi[(3 * f + a) * cs + p];
                    for (int a = 0; a < 3; a++)
                        for (int c = 0; c < 3; c++) {
                            if (a == c)
                                ph2[f][a][c] = d2(pr + f * cs, p, st[a]);
                            else {
                                int lo = a < c ? a : c, hi = a < c ? c : a;
                                ph2[f][a][c] = d4(dphi + (3 * f + lo) * cs, p, st[hi]);
                            }
                        }
                }
                /* physical first and second derivatives */
                double gx[4][3], hx[4][3][3];
                for (int f = 0; f < 4; f++) {
                    for (int c = 0; c < 3; c++) {
                        double s = 0.0;
                        for (int a = 0; a < 3; a++)
                            s = s + xi[a][c] * ph1[f][a];
                        gx[f][c] = s;
                    }
                    for (int jj = 0; jj < 3; jj++)
                        for (int kk = 0; kk < 3; kk++) {
                            double s = 0.0;
                            for (int a = 0; a < 3; a++)
                                for (int c = 0; c < 3; c++)
                                    s = s + xi[a][jj] * xi[c][kk] * ph2[f][a][c];
                            for (int a = 0; a < 3; a++)
                                s = s + xi2[a][pair_of(jj, kk)] * ph1[f][a];
                            hx[f][jj][kk] = s;
                        }
                }
                double T = pr[3 * cs + p];
                double mu = mu_of_T(ph, T), mup = dmu_dT(ph, T);
                double kap = mu * cp / ph->Pr;
                double div = gx[0][0] + gx[1][1] + gx[2][2];
                double dtau[3];
                for (int a = 0; a < 3; a++) {
                    double lap = hx[a][0][0] + hx[a][1][1] + hx[a][2][2];
                    double gdiv = hx[0][0][a] + hx[1][1][a] + hx[2][2][a];
                    double s = mu * (lap + gdiv / 3.0);
                    for (int c = 0; c < 3; c++) {
                        double sym = gx[a][c] + gx[c][a];
                        if (a == c)
                            sym = sym - 2.0 / 3.0 * div;
                        s = s + mup * gx[3][c] * sym;
                    }
                    dtau[a] = s;
                }
                double work = 0.0;
                for (int a = 0; a < 3; a++)
                    work = work + pr[a * cs + p] * dtau[a];
                double diss = 0.0;
                for (int a = 0; a < 3; a++)
                    for (int c = 0; c < 3; c++) {
                        double tau = mu * (gx[a][c] + gx[c][a]);
                        if (a == c)
                            tau = tau - 2.0 / 3.0 * mu * div;
                        diss = diss + tau * gx[a][c];
                    }
                double lapT = hx[3][0][0] + hx[3][1][1] + hx[3][2][2];
                double gT2 = gx[3][0] * gx[3][0] + gx[3][1] * gx[3][1] + gx[3][2] * gx[3][2];
                V[p] = 0.0;
                for (int a = 0; a < 3; a++)
                    V[(1 + a) * cs + p] = dtau[a];
                V[4 * cs + p] = work + diss + kap * lapT + cp / ph->Pr * mup * gT2;
            }
    free(dphi);
    free(pr);
}

/* ------------------------------------------------------------------ */
/* 7. Williamson low-storage RK3 stage (PAPER.md:50 ref [10], 106,    */
/*    114; reading 13):  dU <- A_s dU + dt rhs ;  U_out = U_in + B_s dU */
/* ------------------------------------------------------------------ */
static const double RK_A[3] = {0.0, -5.0 / 9.0, -153.0 / 128.0};
static const double RK_B[3] = {1.0 / 3.0, 15.0 / 16.0, 8.0 / 15.0};

void oracle_rk_update(const int64_t n[3], int32_t stage, double dt, const double *Uin,
                      double *Uout, double *dU, const double *rhs)
{
    obox b = make_box(n, OG);
    const int64_t cs = b.cs;
#pragma omp parallel for OMP_THREADS
    for (int64_t k = 0; k < n[2]; k++)
        for (int64_t j = 0; j < n[1]; j++)
            for (int64_t i = 0; i < n[0]; i++) {
                int64_t p = IX(&b, i, j, k);
                for (int c = 0; c < 5; c++) {
                    int64_t q = c * cs + p;
                    double du;
                    if (stage == 0)
                        du = dt * rhs[q];
                    else
                        du = RK_A[stage] * dU[q] + dt * rhs[q];
                    dU[q] = du;
                    Uout[q] = Uin[q] + RK_B[stage] * du;
                }
            }
}

/* one RK stage = FillPatch/BC_Fill + RHS + Update (Alg. 2 l.3-9); the boundary
   data of stage s are evaluated at t + c_s dt, c = (0, 1/3, 3/4) (reading 13) */
static const double RK_C[3] = {0.0, 1.0 / 3.0, 3.0 / 4.0};

void oracle_rk_stage_ex(const int64_t n[3], const int32_t bc[6], const double dirichlet[30],
                        const oracle_split *split, double t, const oracle_phys *ph, int32_t stage,
                        double dt, double *Uin, double *Uout, double *dU, const double *met)
{
    obox b = make_box(n, OG);
    double *rhs = (double *)calloc((size_t)(5 * b.cs), sizeof(double));
    oracle_fill_ex(n, bc, dirichlet, split, t + RK_C[stage] * dt, met, Uin, 5, O_FIELD_STATE);
    oracle_rhs(n, ph, Uin, met, rhs);
    oracle_rk_update(n, stage, dt, Uin, Uout, dU, rhs);
    free(rhs);
}

void oracle_rk_stage(const int64_t n[3], const int32_t bc[6], const double dirichlet[30],
                     const oracle_phys *ph, int32_t stage, double dt, double *Uin, double *Uout,
                     double *dU, const double *met)
{
    oracle_rk_stage_ex(n, bc, dirichlet, NULL, 0.0, ph, stage, dt, Uin, Uout, dU, met);
}

/* nsteps full RK3 steps with a fixed dt from time t0 (Alg. 1 l.5-10 without
   Regrid/ComputeDt).  U is the state in/out (padded layout); on return its
   ghosts are filled at t0 + nsteps dt. */
void oracle_advance_ex(const int64_t n[3], const int32_t bc[6], const double dirichlet[30],
                       const oracle_split *split, double t0, const oracle_phys *ph, double dt,
                       int32_t nsteps, double *U, const double *met)
{
    obox b = make_box(n, OG);
    size_t sz = (size_t)(5 * b.cs) * sizeof(double);
    double *V = (double *)malloc(sz);
    double *dU = (double *)calloc((size_t)(5 * b.cs), sizeof(double));
    memcpy(V, U, sz);
    double *a = U, *o = V;
    double t = t0; /* step start time, advanced by repeated addition t <- t + dt */
    for (int32_t s = 0; s < nsteps; s++) {
        for (int st = 0; st < 3; st++) {
            oracle_rk_stage_ex(n, bc, dirichlet, split, t, ph, st, dt, a, o, dU, met);
            double *tmp = a;
            a = o;
            o = tmp;
        }
        t = t + dt;
    }
    if (a != U)
        memcpy(U, a, sz);
    oracle_fill_ex(n, bc, dirichlet, split, t, met, U, 5, O_FIELD_STATE);
    free(V);
    free(dU);
}

void oracle_advance(const int64_t n[3], const int32_t bc[6], const double dirichlet[30],
                    const oracle_phys *ph, double dt, int32_t nsteps, double *U,
                    const double *met)
{
    oracle_advance_ex(n, bc, dirichlet, NULL, 0.0, ph, dt, nsteps, U, met);
}

/* ------------------------------------------------------------------ */
/* 8. ComputeDt (Eq. 3, 95 Alg. 1 l.9, 131, 169;       */
/*    SURVEY 8(f) NEXT-1): the 1-D CFL condition (|u| + a) dt/dx <= CFL */
/*    generalised to the curvilinear grid and summed over directions:   */
/*    dt = CFL / max_i sum_d J_i ( |m^d_i . u_i| + c_i |m^d_i| ).       */
/*    Interior points only; a global minimum of dt (ReduceRealMin).    */
/* ------------------------------------------------------------------ */
double oracle_compute_dt(const int64_t n[3], const oracle_phys *ph, const double *U,
                         const double *met, double cfl)
{
    obox b = make_box(n, OG);
    const int64_t cs = b.cs;
    double lam_max = 0.0;
    for (int64_t k = 0; k < n[2]; k++)
        for (int64_t j = 0; j < n[1]; j++)
            for (int64_t i = 0; i < n[0]; i++) {
                int64_t p = IX(&b, i, j, k);
                double rho = U[p];
                double u = U[cs + p] / rho, v = U[2 * cs + p] / rho, w = U[3 * cs + p] / rho;
                double pres = (ph->gamma - 1.0) * (U[4 * cs + p] - 0.5 * rho * (u * u + v * v + w * w));
                double c = sqrt(ph->gamma * pres / rho);
                double s = 0.0;
                for (int d = 0; d < 3; d++) {
                    double mx = met[(1 + 3 * d) * cs + p];
                    double my = met[(2 + 3 * d) * cs + p];
                    double mz = met[(3 + 3 * d) * cs + p];
                    double mu = mx * u + my * v + mz * w;
                    double mm = sqrt(mx * mx + my * my + mz * mz);
                    s = s + fabs(mu) + c * mm;
                }
                s = met[p] * s;
                if (s > lam_max)
                    lam_max = s;
            }
    return cfl / lam_max;
}

/* ------------------------------------------------------------------ */
/* 9. Two-level block-structured AMR (the paper's  */
/*    v2.1 path with AMReX's trilinear interpolator,  */
/*    115-117, 129, 141, 258; readings 24-26).                         */
/*    Refinement ratio 2, node-centred: fine node f (fine-level index) */
/*    sits at coarse index c0 + f/2, so even fine nodes coincide with  */
/*    coarse nodes and odd ones lie halfway between two (*/
/*    "fine points are always physically located halfway between      */
/*    coarse points ... coefficients always a multiple of 1/2").       */
/*    All levels advance with the same dt, stage by stage (Alg. 2:     */
/*    the level loop sits inside the stage loop).    */
/* ------------------------------------------------------------------ */

/* floor(h / 2) for any sign of h */
static int64_t floor_half(int64_t h)
{
    return h >= 0 ? h / 2 : -((-h + 1) / 2);
}

/* FillPatchTwoLevels value of the fine point f ("the eight neighboring
   coarse vertices"): trilinear interpolation in index space,
   U_f(f) = sum over the 8 corners (I + e), e in {0,1}^3, of prod_d w_d(e_d) U_c(I + e),
   h_d = 2 c0_d + f_d, I_d = floor(h_d / 2), t_d = (h_d - 2 I_d) / 2 in {0, 1/2},
   w_d(0) = 1 - t_d, w_d(1) = t_d.  Corner order e = (e0, e1, e2) with e0 fastest. */
static void cf_interp(const oracle_amr *a, const int64_t f[3], double v[5])
{
    obox cb = make_box(a->nc, OG);
    int64_t I[3];
    double tt[3];
    for (int d = 0; d < 3; d++) {
        int64_t h = 2 * a->c0[d] + f[d];
        I[d] = floor_half(h);
        tt[d] = (double)(h - 2 * I[d]) * 0.5;
    }
    for (int c = 0; c < 5; c++)
        v[c] = 0.0;
    for (int e = 0; e < 8; e++) {
        int e0 = e & 1, e1 = (e >> 1) & 1, e2 = (e >> 2) & 1;
        double w0 = e0 ? tt[0] : 1.0 - tt[0];
        double w1 = e1 ? tt[1] : 1.0 - tt[1];
        double w2 = e2 ? tt[2] : 1.0 - tt[2];
        double w = w0 * w1 * w2;
        int64_t p = IX(&cb, I[0] + e0, I[1] + e1, I[2] + e2);
        for (int c = 0; c < 5; c++)
            v[c] = v[c] + w * a->Uc[c * cb.cs + p];
    }
}

/* sibling s of the patch whose interior holds fine point f (patch-local fine index), or -1 */
static int sibling_of(const oracle_amr *a, const int64_t f[3])
{
    for (int s = 0; s < a->nsib; s++) {
        int in = 1;
        for (int d = 0; d < 3; d++) {
            int64_t q = f[d] - a->so[s][d];
            if (q < 0 || q >= a->sn[s][d])
                in = 0;
        }
        if (in)
            return s;
    }
    return -1;
}

/* value of a ghost point on a COARSE_FINE face (reading 31): a point inside another patch of
   the same level takes that patch's value (FillPatchSingleLevel -> FillBoundary),
   every other point is interpolated from the coarse level (FillPatchTwoLevels) */
static void cf_value(const oracle_amr *a, const int64_t f[3], double v[5])
{
    int s = sibling_of(a, f);
    if (s < 0) {
        cf_interp(a, f, v);
        return;
    }
    int64_t ns[3] = {a->sn[s][0], a->sn[s][1], a->sn[s][2]};
    obox sb = make_box(ns, OG);
    int64_t p = IX(&sb, f[0] - a->so[s][0], f[1] - a->so[s][1], f[2] - a->so[s][2]);
    for (int c = 0; c < 5; c++)
        v[c] = a->sU[s][c * sb.cs + p];
}

static void set_siblings(oracle_amr *a, int32_t nsib, const int64_t *so, const int64_t *sn,
                         const double *const *sU)
{
    a->nsib = nsib < O_MAX_SIB ? nsib : O_MAX_SIB;
    for (int s = 0; s < a->nsib; s++) {
        for (int d = 0; d < 3; d++) {
            a->so[s][d] = so[3 * s + d];
            a->sn[s][d] = sn[3 * s + d];
        }
        a->sU[s] = sU[s];
    }
}

/* FillPatch of a fine level (Alg. 2 l.3-4 at level 1): the three-phase fill of section 1
   with COARSE_FINE faces interpolated from the coarse state Uc (ghosts filled). */
void oracle_fill_two_levels_ex(const int64_t nf[3], const int32_t bcf[6], const double dirichlet[30],
                               const oracle_split *split, double t, const double *metf, double *Uf,
                               const int64_t nc[3], const int64_t c0[3], const double *Uc)
{
    oracle_amr a;
    for (int d = 0; d < 3; d++) {
        a.nc[d] = nc[d];
        a.c0[d] = c0[d];
    }
    a.Uc = Uc;
    a.nsib = 0;
    fill_core(nf, bcf, dirichlet, split, t, metf, Uf, 5, O_FIELD_STATE, &a);
}

/* the same with same-level siblings (reading 31): so/sn: 3 x nsib offsets / sizes, sU their states */
void oracle_fill_two_levels_sib(const int64_t nf[3], const int32_t bcf[6], const double dirichlet[30],
                                const double *metf, double *Uf, const int64_t nc[3], const int64_t c0[3],
                                const double *Uc, int32_t nsib, const int64_t *so, const int64_t *sn,
                                const double *const *sU)
{
    oracle_amr a;
    for (int d = 0; d < 3; d++) {
        a.nc[d] = nc[d];
        a.c0[d] = c0[d];
    }
    a.Uc = Uc;
    set_siblings(&a, nsib, so, sn, sU);
    fill_core(nf, bcf, dirichlet, NULL, 0.0, metf, Uf, 5, O_FIELD_STATE, &a);
}

void oracle_fill_two_levels(const int64_t nf[3], const int32_t bcf[6], const double dirichlet[30],
                            const double *metf, double *Uf, const int64_t nc[3],
                            const int64_t c0[3], const double *Uc)
{
    oracle_fill_two_levels_ex(nf, bcf, dirichlet, NULL, 0.0, metf, Uf, nc, c0, Uc);
}

/* AverageDown (Alg. 2 l.10-12; "sets covered coarse AMR cells to be equal to the
   average of the covering fine cells"; reading 25): a coarse node I is covered when, in every
   direction, the fine level is PERIODIC (spans the whole periodic domain) or the fine nodes
   2(I - c0) - 1 .. 2(I - c0) + 1 are fine interior nodes.  Its new value is the average of
   the fine data over its cell [I - 1/2, I + 1/2]^3 by the trapezoid rule on the fine nodes:
   U_c(I) = sum_{c,b,a in {-1,0,1}} w_a w_b w_c U_f(2(I - c0) + (a, b, c)), w_0 = 1/2,
   w_{+-1} = 1/4 (sum order: c outer, a inner).  The fine ghosts are first refilled in place by
   the same-level periodic copies only (the METRIC kind of fill_core skips every non-periodic
   face): physical and C/F ghosts are never read by a covered node. */
void oracle_average_down(const int64_t nf[3], const int32_t bcf[6], const double dirichlet[30],
                         double *Uf, const int64_t nc[3], const int64_t c0[3], double *Uc)
{
    static const double wt[3] = {0.25, 0.5, 0.25};
    obox fb = make_box(nf, OG), cb = make_box(nc, OG);
    fill_core(nf, bcf, dirichlet, NULL, 0.0, NULL, Uf, 5, O_FIELD_METRIC, NULL);
    for (int64_t k = 0; k < nc[2]; k++)
        for (int64_t j = 0; j < nc[1]; j++)
            for (int64_t i = 0; i < nc[0]; i++) {
                int64_t I[3] = {i, j, k}, fc[3];
                int covered = 1;
                for (int d = 0; d < 3; d++) {
                    fc[d] = 2 * (I[d] - c0[d]);
                    if (bcf[2 * d] != O_PERIODIC && (fc[d] < 1 || fc[d] > nf[d] - 2))
                        covered = 0;
                }
                if (!covered)
                    continue;
                int64_t pc = IX(&cb, i, j, k);
                for (int q = 0; q < 5; q++) {
                    double s = 0.0;
                    for (int c = -1; c <= 1; c++)
                        for (int bb = -1; bb <= 1; bb++)
                            for (int a = -1; a <= 1; a++) {
                                double w = wt[a + 1] * wt[bb + 1] * wt[c + 1];
                                int64_t pf = IX(&fb, fc[0] + a, fc[1] + bb, fc[2] + c);
                                s = s + w * Uf[q * fb.cs + pf];
                            }
                    Uc[q * cb.cs + pc] = s;
                }
            }
}

/* AverageDown with same-level siblings (reading 31): the fine ghosts that lie inside a sibling
   are first set to the sibling's values (with the periodic copies); a coarse node I is averaged
   by the patch whose interior holds its central fine node 2(I - c0) when all 27 fine nodes of its
   cell lie in the interiors of the level's patches (directions the patch spans periodically
   always qualify) -- without siblings exactly oracle_average_down's covered set.  Same formula
   and summation order. */
void oracle_average_down_sib(const int64_t nf[3], const int32_t bcf[6], const double dirichlet[30],
                             double *Uf, const int64_t nc[3], const int64_t c0[3], double *Uc,
                             int32_t nsib, const int64_t *so, const int64_t *sn, const double *const *sU)
{
    static const double wt[3] = {0.25, 0.5, 0.25};
    obox fb = make_box(nf, OG), cb = make_box(nc, OG);
    oracle_amr a;
    for (int d = 0; d < 3; d++) {
        a.nc[d] = nc[d];
        a.c0[d] = c0[d];
    }
    a.Uc = NULL;
    set_siblings(&a, nsib, so, sn, sU);
    fill_core(nf, bcf, dirichlet, NULL, 0.0, NULL, Uf, 5, O_FIELD_METRIC, NULL);
    /* sibling copies into the ghost band */
    for (int64_t k = -OG; k < nf[2] + OG; k++)
        for (int64_t j = -OG; j < nf[1] + OG; j++)
            for (int64_t i = -OG; i < nf[0] + OG; i++) {
                int64_t f[3] = {i, j, k};
                if (i >= 0 && i < nf[0] && j >= 0 && j < nf[1] && k >= 0 && k < nf[2])
                    continue;
                if (sibling_of(&a, f) < 0)
                    continue;
                double v[5];
                cf_value(&a, f, v);
                int64_t p = IX(&fb, i, j, k);
                for (int c = 0; c < 5; c++)
                    Uf[c * fb.cs + p] = v[c];
            }
    for (int64_t k = 0; k < nc[2]; k++)
        for (int64_t j = 0; j < nc[1]; j++)
            for (int64_t i = 0; i < nc[0]; i++) {
                int64_t I[3] = {i, j, k}, fc[3];
                int covered = 1;
                for (int d = 0; d < 3; d++) {
                    fc[d] = 2 * (I[d] - c0[d]);
                    if (bcf[2 * d] != O_PERIODIC && (fc[d] < 0 || fc[d] > nf[d] - 1))
                        covered = 0; /* central node not in this patch */
                }
                for (int c = -1; c <= 1 && covered; c++)
                    for (int bb = -1; bb <= 1 && covered; bb++)
                        for (int aa = -1; aa <= 1 && covered; aa++) {
                            int64_t f[3] = {fc[0] + aa, fc[1] + bb, fc[2] + c};
                            int inside = 1;
                            for (int d = 0; d < 3; d++)
                                if (bcf[2 * d] != O_PERIODIC && (f[d] < 0 || f[d] > nf[d] - 1))
                                    inside = 0;
                            if (!inside && sibling_of(&a, f) < 0)
                                covered = 0;
                        }
                if (!covered)
                    continue;
                int64_t pc = IX(&cb, i, j, k);
                for (int q = 0; q < 5; q++) {
                    double s = 0.0;
                    for (int c = -1; c <= 1; c++)
                        for (int bb = -1; bb <= 1; bb++)
                            for (int aa = -1; aa <= 1; aa++) {
                                double w = wt[aa + 1] * wt[bb + 1] * wt[c + 1];
                                int64_t pf = IX(&fb, fc[0] + aa, fc[1] + bb, fc[2] + c);
                                s = s + w * Uf[q * fb.cs + pf];
                            }
                    Uc[q * cb.cs + pc] = s;
                }
            }
}

/* nsteps two-level RK3 steps with a fixed dt (Alg. 1 l.10 with Alg. 2): per stage, level 0
   (fill, RHS, update), then level 1 (FillPatchTwoLevels from level 0's stage input, whose
   ghosts that fill has just set; RHS; update), then at the third stage AverageDown of the
   new fine state onto the new coarse state.  Uc, Uf in/out (padded). */
void oracle_amr_advance(const int64_t nc[3], const int32_t bcc[6], const double dirc[30],
                        const int64_t nf[3], const int32_t bcf[6], const double dirf[30],
                        const int64_t c0[3], const oracle_phys *ph, double dt, int32_t nsteps,
                        double *Uc, const double *metc, double *Uf, const double *metf)
{
    obox cb = make_box(nc, OG), fb = make_box(nf, OG);
    size_t szc = (size_t)(5 * cb.cs) * sizeof(double), szf = (size_t)(5 * fb.cs) * sizeof(double);
    double *Vc = (double *)malloc(szc), *Vf = (double *)malloc(szf);
    double *dUc = (double *)calloc((size_t)(5 * cb.cs), sizeof(double));
    double *dUf = (double *)calloc((size_t)(5 * fb.cs), sizeof(double));
    double *rf = (double *)calloc((size_t)(5 * fb.cs), sizeof(double));
    memcpy(Vc, Uc, szc);
    memcpy(Vf, Uf, szf);
    double *ac = Uc, *oc = Vc, *af = Uf, *of = Vf;
    for (int32_t s = 0; s < nsteps; s++) {
        for (int st = 0; st < 3; st++) {
            oracle_rk_stage_ex(nc, bcc, dirc, NULL, 0.0, ph, st, dt, ac, oc, dUc, metc);
            oracle_fill_two_levels(nf, bcf, dirf, metf, af, nc, c0, ac);
            oracle_rhs(nf, ph, af, metf, rf);
            oracle_rk_update(nf, st, dt, af, of, dUf, rf);
            if (st == 2)
                oracle_average_down(nf, bcf, dirf, of, nc, c0, oc);
            double *tmp = ac;
            ac = oc;
            oc = tmp;
            tmp = af;
            af = of;
            of = tmp;
        }
    }
    if (ac != Uc)
        memcpy(Uc, ac, szc);
    if (af != Uf)
        memcpy(Uf, af, szf);
    free(Vc);
    free(Vf);
    free(dUc);
    free(dUf);
    free(rf);
}
