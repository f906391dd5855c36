/*
 * mrlbm_oracle.c -- CPU ORACLE for the MR-LBM hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
 * --impl reference) may load this library.  The product path
 * (paper_conf_sc_valero_laravgr23_b200/, libmrlbm.so) never links, imports or
 * calls it, and this file shares no code, header, table or generator with it.
 *
 * What it computes: the plain DISTRIBUTION-FORM regularized lattice Boltzmann
 * method (push: collide every node, then stream every population), fp64,
 * slow and obviously correct.  The moment representation (MR) of the paper is
 * lossless (the state is completely represented by
 * rho, u, Pi), so MR computes exactly this, up to rounding order.
 *
 * Citations are to /root/reference/PAPER.md lines ("P:Lnnn") and to the
 * readings listed in DESIGN.md section "Readings" (R1..R19, = SURVEY 8(c)).
 *
 *   moments           eqs 1-3
 *   equilibrium       eq 4      P:L73 (c_s^2 = 1/3, standard Qian lattices, R1)
 *   Pi^neq            eq 8
 *   projective coll.  eq 9      P:L101 (distribution form)
 *   BGK collision     Alg. 1 lines 21-25 (eq 5; R2): the
 *                     paper's standard-representation (ST) reference, NEXT-2
 *   recursive coll.   eqs 10, 12-14  P:L105; recursion of
 *                     Malaspinas [8] (R8), per-component Hermite
 *                     coefficients 1/(a!b!c! c_s^{2n}) (R9), basis per lattice (R10)
 *   streaming         eq 7      P:L89 (push)
 *   walls             halfway bounce-back, link-wise (R12); moving wall
 *                     (Ladd), rho_w = node pre-collision rho (R13)
 *   open faces        regularized velocity / pressure (Latt et al. [6],
 *                     P:L283, R14); finite-difference variant (the scheme the
 *                     paper's proxy apps used, "finite difference
 *                     boundary conditions at the inlet and outlet [6]"; R20)
 *
 * Parity pins: every function here is pinned by tests/test_oracle_*.py against
 * lattice identities, closed forms (tau = 1, u = 0), the paper's eq 9 == eqs
 * 10-11 equivalence, conservation laws, the analytic Poiseuille and
 * Taylor-Green solutions and an independent moment-form stepper; see DESIGN.md.
 * The numerical values of the open-face rebuild at wall EDGE nodes are
 * "parity unpinned" beyond self-consistency.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define CS2 (1.0 / 3.0) /* lattice speed of sound squared, R1 */

enum { D2Q9 = 0, D3Q19 = 1, D3Q27 = 2 };
enum { PROJECTIVE = 0, RECURSIVE = 1, BGK = 2 };
enum { PERIODIC = 0, WALL = 1, MOVING_WALL = 2, VELOCITY = 3, PRESSURE = 4, VELOCITY_FD = 5, PRESSURE_FD = 6 };
#define IS_OPEN(k) ((k) >= VELOCITY)
#define IS_FD(k) ((k) >= VELOCITY_FD)

typedef struct {
    int D, Q;
    int c[27][3];
    double w[27];
    int opp[27];
    int nh;           /* number of retained Hermite components (= Q) */
    int h[27][3];     /* Hermite component (a,b,c): He_a(c_x) He_b(c_y) He_c(c_z) */
} lattice_t;

/* ---------------------------------------------------------------- lattices */
/* Velocity sets and weights: the standard single-speed lattices of Qian et al.
 * [10] (R1).  Ordering (paper silent): index 0 = rest,
 * then a "positive" half, then its negation, so opp(i) = i +- (Q-1)/2. */
static void set_lattice(int which, lattice_t *L)
{
    memset(L, 0, sizeof(*L));
    int half = 0;
    int pos[13][3];
    double wpos[13];
    double w0 = 0;
    if (which == D2Q9) {
        int p[4][3] = {{1, 0, 0}, {0, 1, 0}, {1, 1, 0}, {1, -1, 0}};
        double wp[4] = {1.0 / 9, 1.0 / 9, 1.0 / 36, 1.0 / 36};
        half = 4; w0 = 4.0 / 9; L->D = 2;
        memcpy(pos, p, sizeof(p)); memcpy(wpos, wp, sizeof(wp));
    } else if (which == D3Q19) {
        int p[9][3] = {{1, 0, 0}, {0, 1, 0}, {0, 0, 1}, {1, 1, 0}, {1, -1, 0},
                       {1, 0, 1}, {1, 0, -1}, {0, 1, 1}, {0, 1, -1}};
        double wp[9] = {1.0 / 18, 1.0 / 18, 1.0 / 18, 1.0 / 36, 1.0 / 36,
                        1.0 / 36, 1.0 / 36, 1.0 / 36, 1.0 / 36};
        half = 9; w0 = 1.0 / 3; L->D = 3;
        memcpy(pos, p, sizeof(p)); memcpy(wpos, wp, sizeof(wp));
    } else {
        int p[13][3] = {{1, 0, 0}, {0, 1, 0}, {0, 0, 1}, {1, 1, 0}, {1, -1, 0},
                        {1, 0, 1}, {1, 0, -1}, {0, 1, 1}, {0, 1, -1},
                        {1, 1, 1}, {1, 1, -1}, {1, -1, 1}, {1, -1, -1}};
        double wp[13] = {2.0 / 27, 2.0 / 27, 2.0 / 27, 1.0 / 54, 1.0 / 54,
                         1.0 / 54, 1.0 / 54, 1.0 / 54, 1.0 / 54,
                         1.0 / 216, 1.0 / 216, 1.0 / 216, 1.0 / 216};
        half = 13; w0 = 8.0 / 27; L->D = 3;
        memcpy(pos, p, sizeof(p)); memcpy(wpos, wp, sizeof(wp));
    }
    L->Q = 2 * half + 1;
    L->w[0] = w0;
    L->opp[0] = 0;
    for (int k = 0; k < half; k++) {
        for (int a = 0; a < 3; a++) {
            L->c[1 + k][a] = pos[k][a];
            L->c[1 + half + k][a] = -pos[k][a];
        }
        L->w[1 + k] = wpos[k];
        L->w[1 + half + k] = wpos[k];
        L->opp[1 + k] = 1 + half + k;
        L->opp[1 + half + k] = 1 + k;
    }
    /* Retained Hermite components (R10): D2Q9 {0,1,2}^2, D3Q27 {0,1,2}^3,
     * D3Q19 all orders <= 2 plus the literal eq-14 terms: (2,1,0)-permutations
     * (third order) and (2,2,0)-permutations (fourth order). */
    L->nh = 0;
    for (int c3 = 0; c3 <= 2; c3++)
        for (int b = 0; b <= 2; b++)
            for (int a = 0; a <= 2; a++) {
                int keep;
                if (which == D2Q9) keep = (c3 == 0);
                else if (which == D3Q27) keep = 1;
                else {
                    int n = a + b + c3;
                    int n2 = (a == 2) + (b == 2) + (c3 == 2);
                    int n1 = (a == 1) + (b == 1) + (c3 == 1);
                    keep = (n <= 2) || (n == 3 && n2 == 1 && n1 == 1) || (n == 4 && n2 == 2);
                }
                if (keep) {
                    L->h[L->nh][0] = a; L->h[L->nh][1] = b; L->h[L->nh][2] = c3;
                    L->nh++;
                }
            }
}

/* 1D Hermite polynomials with c_s^2 = 1/3: He0 = 1, He1 = c, He2 = c^2 - c_s^2
 * (the tensor Hermite polynomials of eqs 1-3 factor per axis on these lattices). */
static double he1d(int order, int c)
{
    if (order == 0) return 1.0;
    if (order == 1) return (double)c;
    return (double)(c * c) - CS2;
}

static double factorial(int n)
{
    double r = 1.0;
    for (int k = 2; k <= n; k++) r *= k;
    return r;
}

/* H^(2)_{i,ab} = c_ia c_ib - c_s^2 delta_ab  (eq 3) */
static double H2(const lattice_t *L, int i, int a, int b)
{
    return (double)(L->c[i][a] * L->c[i][b]) - (a == b ? CS2 : 0.0);
}

/* --------------------------------------------------------------- moments */
/* eqs 1-3: rho = sum f, rho u = sum c f, Pi = sum H2 f */
static void moments_of(const lattice_t *L, const double *f, double *rho, double u[3], double Pi[3][3])
{
    double r = 0, j[3] = {0, 0, 0};
    for (int i = 0; i < L->Q; i++) {
        r += f[i];
        for (int a = 0; a < 3; a++) j[a] += L->c[i][a] * f[i];
    }
    *rho = r;
    for (int a = 0; a < 3; a++) u[a] = j[a] / r;
    if (Pi) {
        memset(Pi, 0, 9 * sizeof(double));
        for (int a = 0; a < L->D; a++)
            for (int b = 0; b < L->D; b++) {
                double s = 0;
                for (int i = 0; i < L->Q; i++) s += H2(L, i, a, b) * f[i];
                Pi[a][b] = s;
            }
    }
}

/* eq 4: f_i^eq = w_i rho (1 + c.u / c_s^2 + H2_i : uu / (2 c_s^4)) */
static double feq_i(const lattice_t *L, int i, double rho, const double u[3])
{
    double cu = 0, Huu = 0;
    for (int a = 0; a < 3; a++) cu += L->c[i][a] * u[a];
    for (int a = 0; a < L->D; a++)
        for (int b = 0; b < L->D; b++) Huu += H2(L, i, a, b) * u[a] * u[b];
    return L->w[i] * rho * (1.0 + cu / CS2 + Huu / (2.0 * CS2 * CS2));
}

/* Recursive non-equilibrium Hermite coefficient (Malaspinas [8], R8):
 *   a^(2)_neq = Pi^neq
 *   a^(n)_{a1..an} = u_{an} a^(n-1)_{a1..a(n-1)}
 *                  + sum_{l<n} ( prod_{m<n, m!=l} u_{am} ) Pi^neq_{al an}
 * idx holds the n axis labels a1..an. */
static double aneq_rec(const int *idx, int n, const double u[3], const double Pneq[3][3])
{
    if (n == 2) return Pneq[idx[0]][idx[1]];
    double r = u[idx[n - 1]] * aneq_rec(idx, n - 1, u, Pneq);
    for (int l = 0; l < n - 1; l++) {
        double p = 1.0;
        for (int m = 0; m < n - 1; m++)
            if (m != l) p *= u[idx[m]];
        r += p * Pneq[idx[l]][idx[n - 1]];
    }
    return r;
}

/* One node's collision: pre-collision f (Q values) -> post-collision f* . */
static void collide_node(const lattice_t *L, int reg, double tau, const double *f, double *fstar)
{
    double rho, u[3], feq[27], fneq[27], Pneq[3][3];
    moments_of(L, f, &rho, u, NULL);                        /* eqs 1-2 */
    for (int i = 0; i < L->Q; i++) {
        feq[i] = feq_i(L, i, rho, u);                       /* eq 4 */
        fneq[i] = f[i] - feq[i];
    }
    memset(Pneq, 0, sizeof(Pneq));
    for (int a = 0; a < L->D; a++)                          /* eq 8 */
        for (int b = 0; b < L->D; b++) {
            double s = 0;
            for (int i = 0; i < L->Q; i++) s += H2(L, i, a, b) * fneq[i];
            Pneq[a][b] = s;
        }
    const double om = 1.0 - 1.0 / tau;
    if (reg == BGK) {
        /* Alg. 1 lines 21-25, the paper's ST reference collision
         * (single-relaxation-time BGK, eq 5), with the f^eq of eq 4
         * (R2: the garbled "cu^2" of line 24 is 4.5 (c.u)^2):
         *   f*_i = f_i (1 - 1/tau) + f^eq_i / tau */
        for (int i = 0; i < L->Q; i++) fstar[i] = f[i] * om + feq[i] / tau;
        return;
    }
    if (reg == PROJECTIVE) {
        /* eq 9: f* = f^eq + (1 - 1/tau) w_i / (2 c_s^4) H2_i : Pi^neq */
        for (int i = 0; i < L->Q; i++) {
            double HP = 0;
            for (int a = 0; a < L->D; a++)
                for (int b = 0; b < L->D; b++) HP += H2(L, i, a, b) * Pneq[a][b];
            fstar[i] = feq[i] + om * L->w[i] / (2.0 * CS2 * CS2) * HP;
        }
        return;
    }
    /* Recursive: collide every retained Hermite coefficient (eqs 10, 12, 13,
     * and their extension to orders 5-6 for D3Q27), then reconstruct (eq 14,
     * per-component coefficient 1/(a!b!c! c_s^{2n}), R9). */
    double A[27];
    for (int k = 0; k < L->nh; k++) {
        const int *h = L->h[k];
        int n = h[0] + h[1] + h[2];
        int idx[6], m = 0;
        for (int a = 0; a < 3; a++)
            for (int t = 0; t < h[a]; t++) idx[m++] = a;
        double aeq = rho;                                   /* a^eq = rho u...u */
        for (int t = 0; t < n; t++) aeq *= u[idx[t]];
        if (n <= 1) A[k] = aeq;                             /* conserved: rho, rho u */
        else A[k] = aeq + om * aneq_rec(idx, n, u, Pneq);   /* eqs 10, 12, 13 */
    }
    for (int i = 0; i < L->Q; i++) {
        double s = 0;
        for (int k = 0; k < L->nh; k++) {
            const int *h = L->h[k];
            int n = h[0] + h[1] + h[2];
            double He = he1d(h[0], L->c[i][0]) * he1d(h[1], L->c[i][1]) * he1d(h[2], L->c[i][2]);
            s += He * A[k] / (factorial(h[0]) * factorial(h[1]) * factorial(h[2]) * pow(CS2, n));
        }
        fstar[i] = L->w[i] * s;                              /* eq 14 */
    }
}

/* ------------------------------------------------------------------ domain */
typedef struct oracle {
    lattice_t L;
    int lattice, reg;
    int64_t n[3], N;
    double tau;
    int kind[6];
    double uw[6][3];
    double rhow[6];
    double *uprof[6];        /* VELOCITY faces: optional per-face-node velocity [D] */
    double *f, *fs, *fn, *rho0;
    int nthreads;
} oracle_t;

static int64_t nid(const oracle_t *o, int64_t x, int64_t y, int64_t z)
{
    return (z * o->n[1] + y) * o->n[0] + x;
}

/* index of node p inside the face-node array of face F (row-major over the
 * two remaining axes, slower axis first) */
static int64_t face_index(const oracle_t *o, int F, const int64_t p[3])
{
    int ax = F / 2;
    int a1 = (ax == 0) ? 1 : 0;
    int a2 = (ax == 2) ? 1 : 2;
    return p[a2] * o->n[a1] + p[a1];
}

int oracle_M(int lattice) { return lattice == D2Q9 ? 6 : 10; }
int oracle_Q(int lattice) { return lattice == D2Q9 ? 9 : (lattice == D3Q19 ? 19 : 27); }

void oracle_destroy(oracle_t *o)
{
    if (!o) return;
    free(o->f); free(o->fs); free(o->fn); free(o->rho0);
    for (int F = 0; F < 6; F++) free(o->uprof[F]);
    free(o);
}

/* kind[6], uw[6*3], rhow[6]; uprof[F] may be NULL (else face_nodes*D values).
 * Returns NULL on invalid input. */
oracle_t *oracle_create(int lattice, int64_t nx, int64_t ny, int64_t nz, double tau, int reg,
                        const int *kind, const double *uw, const double *rhow,
                        const double *const *uprof, int nthreads)
{
    if (lattice < 0 || lattice > 2 || tau <= 0.5) return NULL;
    oracle_t *o = (oracle_t *)calloc(1, sizeof(oracle_t));
    set_lattice(lattice, &o->L);
    o->lattice = lattice; o->reg = reg; o->tau = tau;
    o->n[0] = nx; o->n[1] = ny; o->n[2] = (o->L.D == 2) ? 1 : nz;
    o->N = o->n[0] * o->n[1] * o->n[2];
    for (int F = 0; F < 6; F++) {
        o->kind[F] = kind[F];
        for (int a = 0; a < 3; a++) o->uw[F][a] = uw[3 * F + a];
        o->rhow[F] = rhow[F];
        if (o->L.D == 2 && F >= 4) o->kind[F] = PERIODIC;
        if (uprof && uprof[F] && (o->kind[F] == VELOCITY || o->kind[F] == VELOCITY_FD)) {
            int ax = F / 2;
            int64_t cnt = o->N / o->n[ax] * o->L.D;
            o->uprof[F] = (double *)malloc(sizeof(double) * cnt);
            memcpy(o->uprof[F], uprof[F], sizeof(double) * cnt);
        }
    }
    size_t bytes = sizeof(double) * (size_t)o->L.Q * (size_t)o->N;
    o->f = (double *)malloc(bytes);
    o->fs = (double *)malloc(bytes);
    o->fn = (double *)malloc(bytes);
    o->rho0 = (double *)malloc(sizeof(double) * o->N);
    o->nthreads = nthreads;
    if (!o->f || !o->fs || !o->fn || !o->rho0) { oracle_destroy(o); return NULL; }
    /* rest state */
    for (int i = 0; i < o->L.Q; i++)
        for (int64_t k = 0; k < o->N; k++) o->f[i * o->N + k] = o->L.w[i];
    return o;
}

/* State from moments: f_i = w_i [rho + c_i.(rho u)/c_s^2 + H2_i : Pi / (2 c_s^4)]
 * (the eq 11 map with Pi* -> Pi).  m is [M][N] in the ABI order
 * 2D: rho ux uy Pxx Pyy Pxy; 3D: rho ux uy uz Pxx Pyy Pzz Pxy Pxz Pyz. */
static void unpack_moments(int D, const double *m, int64_t N, int64_t k, double *rho, double u[3], double Pi[3][3])
{
    memset(u, 0, 3 * sizeof(double));
    memset(Pi, 0, 9 * sizeof(double));
    *rho = m[0 * N + k];
    if (D == 2) {
        u[0] = m[1 * N + k]; u[1] = m[2 * N + k];
        Pi[0][0] = m[3 * N + k]; Pi[1][1] = m[4 * N + k];
        Pi[0][1] = Pi[1][0] = m[5 * N + k];
    } else {
        u[0] = m[1 * N + k]; u[1] = m[2 * N + k]; u[2] = m[3 * N + k];
        Pi[0][0] = m[4 * N + k]; Pi[1][1] = m[5 * N + k]; Pi[2][2] = m[6 * N + k];
        Pi[0][1] = Pi[1][0] = m[7 * N + k];
        Pi[0][2] = Pi[2][0] = m[8 * N + k];
        Pi[1][2] = Pi[2][1] = m[9 * N + k];
    }
}

static void pack_moments(int D, double *m, int64_t N, int64_t k, double rho, const double u[3], double Pi[3][3])
{
    m[0 * N + k] = rho;
    if (D == 2) {
        m[1 * N + k] = u[0]; m[2 * N + k] = u[1];
        m[3 * N + k] = Pi[0][0]; m[4 * N + k] = Pi[1][1]; m[5 * N + k] = Pi[0][1];
    } else {
        m[1 * N + k] = u[0]; m[2 * N + k] = u[1]; m[3 * N + k] = u[2];
        m[4 * N + k] = Pi[0][0]; m[5 * N + k] = Pi[1][1]; m[6 * N + k] = Pi[2][2];
        m[7 * N + k] = Pi[0][1]; m[8 * N + k] = Pi[0][2]; m[9 * N + k] = Pi[1][2];
    }
}

void oracle_set_moments(oracle_t *o, const double *m)
{
    const lattice_t *L = &o->L;
    for (int64_t k = 0; k < o->N; k++) {
        double rho, u[3], Pi[3][3];
        unpack_moments(L->D, m, o->N, k, &rho, u, Pi);
        for (int i = 0; i < L->Q; i++) {
            double cj = 0, HP = 0;
            for (int a = 0; a < 3; a++) cj += L->c[i][a] * rho * u[a];
            for (int a = 0; a < L->D; a++)
                for (int b = 0; b < L->D; b++) HP += H2(L, i, a, b) * Pi[a][b];
            o->f[i * o->N + k] = L->w[i] * (rho + cj / CS2 + HP / (2.0 * CS2 * CS2));
        }
    }
}

/* moments (eqs 1-3) of the current (post-stream = pre-collision) state */
void oracle_get_moments(const oracle_t *o, double *m)
{
    const lattice_t *L = &o->L;
    for (int64_t k = 0; k < o->N; k++) {
        double fl[27], rho, u[3], Pi[3][3];
        for (int i = 0; i < L->Q; i++) fl[i] = o->f[i * o->N + k];
        moments_of(L, fl, &rho, u, Pi);
        pack_moments(L->D, m, o->N, k, rho, u, Pi);
    }
}

void oracle_set_f(oracle_t *o, const double *f) { memcpy(o->f, f, sizeof(double) * o->L.Q * o->N); }
void oracle_get_f(const oracle_t *o, double *f) { memcpy(f, o->f, sizeof(double) * o->L.Q * o->N); }

static void collide_all(oracle_t *o)
{
    const lattice_t *L = &o->L;
    const int64_t N = o->N;
#pragma omp parallel for schedule(static) num_threads(o->nthreads > 0 ? o->nthreads : 1)
    for (int64_t k = 0; k < N; k++) {
        double fl[27], fo[27];
        for (int i = 0; i < L->Q; i++) fl[i] = o->f[i * N + k];
        double r = 0;
        for (int i = 0; i < L->Q; i++) r += fl[i];
        o->rho0[k] = r;
        collide_node(L, o->reg, o->tau, fl, fo);
        for (int i = 0; i < L->Q; i++) o->fs[i * N + k] = fo[i];
    }
}

/* post-collision populations f* of the current state, [Q][N] */
void oracle_get_populations(oracle_t *o, double *fstar)
{
    collide_all(o);
    memcpy(fstar, o->fs, sizeof(double) * o->L.Q * o->N);
}

/* Regularized open face (Latt et al. [6], R14) at node p of face F. */
static void open_face_node(oracle_t *o, int F, const int64_t p[3])
{
    const lattice_t *L = &o->L;
    const int64_t N = o->N, k = nid(o, p[0], p[1], p[2]);
    int ax = F / 2;
    int nrm[3] = {0, 0, 0};
    nrm[ax] = (F % 2 == 0) ? 1 : -1; /* inward normal */
    double f[27];
    for (int i = 0; i < L->Q; i++) f[i] = o->fn[i * N + k];
    /* K0: c.n = 0; K-: c.n < 0 (outgoing, known); U+: c.n > 0 (unknown) */
    int cls[27];
    double S = 0;
    for (int i = 0; i < L->Q; i++) {
        int cn = L->c[i][0] * nrm[0] + L->c[i][1] * nrm[1] + L->c[i][2] * nrm[2];
        cls[i] = (cn > 0) ? 1 : (cn < 0 ? -1 : 0);
        if (cls[i] == 0) S += f[i];
        if (cls[i] == -1) S += 2.0 * f[i];
    }
    double rho, u[3] = {0, 0, 0};
    if (o->kind[F] == VELOCITY || o->kind[F] == VELOCITY_FD) {
        if (o->uprof[F]) {
            int64_t fi = face_index(o, F, p);
            for (int a = 0; a < L->D; a++) u[a] = o->uprof[F][fi * L->D + a];
        } else {
            for (int a = 0; a < 3; a++) u[a] = o->uw[F][a];
        }
        double un = u[0] * nrm[0] + u[1] * nrm[1] + u[2] * nrm[2];
        rho = S / (1.0 - un);              /* sum f = rho, sum f c.n = rho u.n */
    } else {
        rho = o->rhow[F];
        double un = 1.0 - S / rho;         /* tangential velocity 0 (R14) */
        for (int a = 0; a < 3; a++) u[a] = un * nrm[a];
    }
    double feq[27], fneq[27];
    for (int i = 0; i < L->Q; i++) feq[i] = feq_i(L, i, rho, u);
    for (int i = 0; i < L->Q; i++) fneq[i] = f[i] - feq[i];
    for (int i = 0; i < L->Q; i++)
        if (cls[i] == 1) fneq[i] = fneq[L->opp[i]];   /* bounce-back of f^neq */
    double Pneq[3][3];
    memset(Pneq, 0, sizeof(Pneq));
    for (int a = 0; a < L->D; a++)
        for (int b = 0; b < L->D; b++) {
            double s = 0;
            for (int i = 0; i < L->Q; i++) s += H2(L, i, a, b) * fneq[i];
            Pneq[a][b] = s;
        }
    for (int i = 0; i < L->Q; i++) {
        double HP = 0;
        for (int a = 0; a < L->D; a++)
            for (int b = 0; b < L->D; b++) HP += H2(L, i, a, b) * Pneq[a][b];
        o->fn[i * N + k] = feq[i] + L->w[i] / (2.0 * CS2 * CS2) * HP;
    }
}

/* Finite-difference open faces (Latt et al. [6], the "FD" scheme; R20).
 * rho and u of a face node come from the same rule as the regularized face
 * (open_face_node above: rho from the known populations on a velocity face,
 * u.n from them on a pressure face).  The non-equilibrium part is the
 * first-order Chapman-Enskog stress of the NEW velocity field,
 *   Pi^neq_ab = -rho tau c_s^2 (d_a u_b + d_b u_a),
 * with second-order finite differences: one-sided along the face normal,
 *   d u = s (-3 u(0) + 4 u(s) - u(2s)) / 2   (s = inward direction),
 * central along the face (wrapped on periodic axes), one-sided at the face's
 * edges.  The node is then set to f = f^eq(rho, u) + w H2 : Pi^neq / (2 c_s^4),
 * i.e. moments (rho, u, rho u u + Pi^neq). */
static double fd_deriv(const oracle_t *o, const double *U, int ax, const int64_t p[3], int comp)
{
    const int64_t n = o->n[ax];
    int64_t q[3] = {p[0], p[1], p[2]};
    const int per = o->kind[2 * ax] == PERIODIC;
    double um, u0, up;
#define UAT(QQ) (U[3 * nid(o, (QQ)[0], (QQ)[1], (QQ)[2]) + comp])
    if (per || (p[ax] > 0 && p[ax] < n - 1)) {
        q[ax] = (p[ax] - 1 + n) % n; um = UAT(q);
        q[ax] = (p[ax] + 1) % n; up = UAT(q);
        return 0.5 * (up - um);
    }
    const int64_t s = (p[ax] == 0) ? 1 : -1;
    u0 = UAT(p);
    q[ax] = p[ax] + s; up = UAT(q);
    q[ax] = p[ax] + 2 * s; um = UAT(q);
#undef UAT
    return (double)s * 0.5 * (-3.0 * u0 + 4.0 * up - um);
}

static void fd_faces(oracle_t *o)
{
    const lattice_t *L = &o->L;
    const int64_t N = o->N;
    double *U = (double *)malloc(sizeof(double) * 3 * N);
    double *R = (double *)malloc(sizeof(double) * N);
    for (int64_t k = 0; k < N; k++) {
        double f[27];
        for (int i = 0; i < L->Q; i++) f[i] = o->fn[i * N + k];
        moments_of(L, f, &R[k], &U[3 * k], NULL);
    }
    for (int F = 0; F < 2 * L->D; F++) {
        if (!IS_FD(o->kind[F])) continue;
        int ax = F / 2;
        int64_t fixed = (F % 2 == 0) ? 0 : o->n[ax] - 1;
        for (int64_t k = 0; k < N; k++) {
            int64_t p[3] = {k % o->n[0], (k / o->n[0]) % o->n[1], k / (o->n[0] * o->n[1])};
            if (p[ax] != fixed) continue;
            double g[3][3]; /* g[a][b] = d_a u_b */
            memset(g, 0, sizeof(g));
            for (int a = 0; a < L->D; a++)
                for (int b = 0; b < L->D; b++) g[a][b] = fd_deriv(o, U, a, p, b);
            const double rho = R[k];
            double Pneq[3][3];
            memset(Pneq, 0, sizeof(Pneq));
            for (int a = 0; a < L->D; a++)
                for (int b = 0; b < L->D; b++) Pneq[a][b] = -rho * o->tau * CS2 * (g[a][b] + g[b][a]);
            for (int i = 0; i < L->Q; i++) {
                double HP = 0;
                for (int a = 0; a < L->D; a++)
                    for (int b = 0; b < L->D; b++) HP += H2(L, i, a, b) * Pneq[a][b];
                o->fn[i * N + k] = feq_i(L, i, rho, &U[3 * k]) + L->w[i] / (2.0 * CS2 * CS2) * HP;
            }
        }
    }
    free(U);
    free(R);
}

static void stream_all(oracle_t *o)
{
    const lattice_t *L = &o->L;
    const int64_t N = o->N;
    for (int64_t t = 0; t < (int64_t)L->Q * N; t++) o->fn[t] = NAN;
#pragma omp parallel for schedule(static) num_threads(o->nthreads > 0 ? o->nthreads : 1)
    for (int64_t k = 0; k < N; k++) {
        int64_t x[3] = {k % o->n[0], (k / o->n[0]) % o->n[1], k / (o->n[0] * o->n[1])};
        for (int i = 0; i < L->Q; i++) {
            int64_t d[3];
            int wall = 0, open = 0;
            double lid = 0;
            for (int a = 0; a < 3; a++) {
                d[a] = x[a] + L->c[i][a];
                int F = -1;
                if (d[a] < 0) F = 2 * a;
                else if (d[a] >= o->n[a]) F = 2 * a + 1;
                if (F < 0) continue;
                int kd = o->kind[F];
                if (kd == PERIODIC) {
                    d[a] = (d[a] + o->n[a]) % o->n[a];
                } else if (kd == WALL || kd == MOVING_WALL) {
                    wall = 1;
                    if (kd == MOVING_WALL) {
                        double cu = 0;
                        for (int b = 0; b < 3; b++) cu += L->c[i][b] * o->uw[F][b];
                        lid += 2.0 * L->w[i] * o->rho0[k] * cu / CS2;
                    }
                } else {
                    open = 1;
                }
            }
            double v = o->fs[i * N + k];
            if (wall) o->fn[L->opp[i] * N + k] = v - lid;   /* halfway bounce-back (R12, R13) */
            else if (open) continue;                         /* rebuilt below */
            else o->fn[i * N + nid(o, d[0], d[1], d[2])] = v; /* eq 7 */
        }
    }
    /* open faces after wall bounce-back (R14) */
    int any_fd = 0;
    for (int F = 0; F < 2 * L->D; F++) {
        if (!IS_OPEN(o->kind[F])) continue;
        any_fd |= IS_FD(o->kind[F]);
        int ax = F / 2;
        int64_t fixed = (F % 2 == 0) ? 0 : o->n[ax] - 1;
        for (int64_t k = 0; k < N; k++) {
            int64_t p[3] = {k % o->n[0], (k / o->n[0]) % o->n[1], k / (o->n[0] * o->n[1])};
            if (p[ax] != fixed) continue;
            open_face_node(o, F, p);
        }
    }
    if (any_fd) fd_faces(o);
    double *t = o->f; o->f = o->fn; o->fn = t;
}

/* n timesteps: collide (eq 6 with regularized f^neq), stream (eq 7), BCs */
void oracle_step(oracle_t *o, int64_t nsteps)
{
    for (int64_t s = 0; s < nsteps; s++) {
        collide_all(o);
        stream_all(o);
    }
}

/* ------------------------------------------------ per-node entry points */
/* Exposed so tests can pin the collision operator node by node. */
void oracle_collide_node(int lattice, int reg, double tau, const double *f, double *fstar)
{
    lattice_t L;
    set_lattice(lattice, &L);
    collide_node(&L, reg, tau, f, fstar);
}

void oracle_feq(int lattice, double rho, const double *u, double *feq)
{
    lattice_t L;
    set_lattice(lattice, &L);
    double uu[3] = {u[0], u[1], L.D == 3 ? u[2] : 0.0};
    for (int i = 0; i < L.Q; i++) feq[i] = feq_i(&L, i, rho, uu);
}

/* lattice tables for tests: c[Q*3], w[Q], opp[Q], h[Q*3] */
int oracle_lattice(int lattice, int *c, double *w, int *opp, int *h)
{
    lattice_t L;
    set_lattice(lattice, &L);
    for (int i = 0; i < L.Q; i++) {
        for (int a = 0; a < 3; a++) { c[3 * i + a] = L.c[i][a]; h[3 * i + a] = L.h[i][a]; }
        w[i] = L.w[i];
        opp[i] = L.opp[i];
    }
    return L.Q;
}

double oracle_aneq(const int *idx, int n, const double *u, const double *Pneq9)
{
    double P[3][3];
    for (int a = 0; a < 3; a++)
        for (int b = 0; b < 3; b++) P[a][b] = Pneq9[3 * a + b];
    return aneq_rec(idx, n, u, P);
}

int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
