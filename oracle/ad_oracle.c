/*
 * ad_oracle.c — plain FP64 CPU oracle for the ADADELTA energy+gradient hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (libad, include/ad.h) never calls it, links it or shares
 * any code, header, table or helper with it.
 *
 * What it computes (citations: P:Ln = /root/reference/PAPER.md line n;
 * O-k / Z-k = the readings in SURVEY.md §8(c), restated in DESIGN.md):
 *
 *   pose()        PoseCalculation: genotype -> atom coordinates.
 *                 Alg 4 lines 1-2, genotype = translation,
 *                 orientation, torsions; reading O-1, Z11, Z13, Z22.
 *   inter()       InterGradient: trilinear interpolation of the type map,
 *                 q * electrostatic map and |q| * desolvation map, and the
 *                 exact derivative of that interpolant ("numerical",
 *                 P:L98-100); out-of-grid restraint.  O-2, Z3, Z4, Z5.
 *   intra()       IntraGradient over the contributor pair list (P:L83
 *                 "analytical"): smoothed 12-6 / 12-10,
 *                 distance-dependent-dielectric electrostatics, desolvation,
 *                 with cutoffs.  O-3, Z6-Z10.
 *   gene gradient Gtrans / Grigidrot / Grotbond: the
 *                 chain rule dE/dg_k = sum_i g_i . dX_i/dg_k written out with
 *                 the explicit per-atom Jacobian.  O-4, Z12.
 *   adadelta()    ADADELTA local search (Alg 3; Zeiler [19] P:L406),
 *                 300 iterations, best tracking.  O-6, Z14-Z16.
 *   best_of_run() argmin per run of Pop_size poses.  O-8, Z21.
 *   exact_sum()   exact sum of FP32 partials (reduction-engine oracle, config
 *                 4, Eq 1-5).  O-7.
 *
 * Everything is FP64, scalar, unblocked, in the paper's order.  The inputs are
 * the same FP32 arrays the GPU receives (converted to double on read).
 *
 * Pins (tests/test_oracle_*.py): closed-form pair energies, affine grid
 * fields, brute-force 8-corner sums, central finite differences on every gene,
 * rigid-motion invariance of E_intra, Newton III, 360-degree periodicity, the
 * closed-form first ADADELTA step, math.fsum.  Docking quality (E50, RMSD) is
 * "parity unpinned" (needs the paper's dataset; out of scope).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ADO_PI 3.14159265358979323846
#define DEG (ADO_PI / 180.0)

/* ---- oracle-private input structs (ctypes mirrors in oracle/oracle.py) ---- */
typedef struct {
    int32_t nx, ny, nz, n_maps;
    double spacing;
    double origin[3];
    const float* maps; /* [n_maps][nz][ny][nx], x fastest */
} ado_grid;

typedef struct {
    double smooth, cut_vdw, cut_el, el_rmin;
    double diel_A, diel_B, diel_k, diel_lambda;
    double coeff_el, coeff_ds, qasp, sigma_ds, w_out;
} ado_ff;

typedef struct {
    int32_t n_atoms, n_tors, n_pairs, n_types;
    const float* ref_xyz;       /* [N][3] */
    const int32_t* atom_map;    /* [N] */
    const int32_t* atom_type;   /* [N] */
    const float* charge;        /* [N] */
    const int32_t* tors_axis;   /* [T][2] (a, c) root->leaf */
    const uint8_t* tors_moving; /* [T][N] */
    const int32_t* pairs;       /* [P][2] */
    const float* tp_coef;       /* [nt][nt][5] cA cB r0 m n */
    const float* type_S;        /* [nt] */
    const float* type_V;        /* [nt] */
} ado_ligand;

/* aux[] layout written by ado_eval */
enum { AUX_EINTER = 0, AUX_EINTRA = 1, AUX_ABS_E = 2, AUX_MARGIN_E = 3, AUX_MARGIN_G = 4, AUX_SENS_E = 5, AUX_N = 6 };

/* ------------------------------------------------------------------------ */
static void cross(const double a[3], const double b[3], double out[3]) {
    out[0] = a[1] * b[2] - a[2] * b[1];
    out[1] = a[2] * b[0] - a[0] * b[2];
    out[2] = a[0] * b[1] - a[1] * b[0];
}
static double dot(const double a[3], const double b[3]) { return a[0] * b[0] + a[1] * b[1] + a[2] * b[2]; }

/* O-1: PoseCalculation (Alg 4).
 * x_i = r_i; for torsions b in root->leaf order rotate the moving set of b by
 * theta_b (degrees) about the CURRENT axis a_b -> c_b (right-handed,
 * Rodrigues); then rotate by the quaternion q = (cos a/2, sin a/2 u(phi,theta))
 * and translate by T = origin + h * (g0, g1, g2).                            */
int ado_pose(const ado_ligand* L, const ado_grid* G, const double* g, double* X /*[N][3]*/, double T[3]) {
    const int N = L->n_atoms;
    for (int i = 0; i < N; i++)
        for (int k = 0; k < 3; k++) X[3 * i + k] = (double)L->ref_xyz[3 * i + k];
    for (int b = 0; b < L->n_tors; b++) {
        const int a = L->tors_axis[2 * b], c = L->tors_axis[2 * b + 1];
        double P[3], u[3];
        for (int k = 0; k < 3; k++) { P[k] = X[3 * a + k]; u[k] = X[3 * c + k] - X[3 * a + k]; }
        const double nu = sqrt(dot(u, u));
        for (int k = 0; k < 3; k++) u[k] /= nu;
        const double t = g[6 + b] * DEG, ct = cos(t), st = sin(t);
        for (int i = 0; i < N; i++) {
            if (!L->tors_moving[(size_t)b * N + i]) continue;
            double v[3], uxv[3];
            for (int k = 0; k < 3; k++) v[k] = X[3 * i + k] - P[k];
            cross(u, v, uxv);
            const double ud = dot(u, v);
            for (int k = 0; k < 3; k++) X[3 * i + k] = P[k] + v[k] * ct + uxv[k] * st + u[k] * ud * (1.0 - ct);
        }
    }
    const double phi = g[3] * DEG, th = g[4] * DEG, al = g[5] * DEG;
    const double ax[3] = {sin(th) * cos(phi), sin(th) * sin(phi), cos(th)};
    const double w = cos(0.5 * al), s = sin(0.5 * al);
    const double qv[3] = {s * ax[0], s * ax[1], s * ax[2]};
    for (int k = 0; k < 3; k++) T[k] = G->origin[k] + G->spacing * g[k];
    for (int i = 0; i < N; i++) {
        double p[3] = {X[3 * i], X[3 * i + 1], X[3 * i + 2]}, c1[3], c2[3];
        cross(qv, p, c1);
        cross(qv, c1, c2);
        for (int k = 0; k < 3; k++) X[3 * i + k] = p[k] + 2.0 * w * c1[k] + 2.0 * c2[k] + T[k];
    }
    return 0;
}

/* grid sample V[m][z][y][x] */
static double gv(const ado_grid* G, int m, int x, int y, int z) {
    return (double)G->maps[(((size_t)m * G->nz + z) * G->ny + y) * G->nx + x];
}

/* O-2: InterGradient for one atom.
 * u = (X - o)/h; outside if any u_k < 0 or u_k >= n_k - 1 (Z5).
 * inside : E = sum_c prod_k w_k(c) * (T_m + q E + |q| D)[corner c]  (trilinear)
 *          dE/dX = (1/h) d/du of the same interpolant (Z3)
 * outside: E = w_out * sum_k (u_k - c_k)^2, c = (n-1)/2, dE/dX = 2 w_out (u-c)/h (Z4).
 * abs_e: magnitude sum for the Z18 tolerance (sum over the weighted corner
 * terms of |term|).  margin_e / margin_g: distance
 * (A) to the nearest energy discontinuity (grid boundary) / gradient kink
 * (cell face).                                                               */
static double inter_atom(const ado_grid* G, const ado_ff* F, int map, double q, const double X[3], double grad[3],
                         double* abs_e, double* margin_e, double* margin_g) {
    const int n[3] = {G->nx, G->ny, G->nz};
    const double h = G->spacing;
    double u[3];
    int out = 0;
    for (int k = 0; k < 3; k++) {
        u[k] = (X[k] - G->origin[k]) / h;
        if (u[k] < 0.0 || u[k] >= (double)(n[k] - 1)) out = 1;
    }
    double me = 1e30, mg = 1e30;
    for (int k = 0; k < 3; k++) {
        double d0 = fabs(u[k]) * h, d1 = fabs(u[k] - (double)(n[k] - 1)) * h;
        if (d0 < me) me = d0;
        if (d1 < me) me = d1;
        double fr = u[k] - floor(u[k]);
        double df = (fr < 0.5 ? fr : 1.0 - fr) * h;
        if (df < mg) mg = df;
    }
    *margin_e = me;
    *margin_g = mg;
    if (out) {
        double E = 0.0;
        for (int k = 0; k < 3; k++) {
            const double c = 0.5 * (double)(n[k] - 1);
            E += F->w_out * (u[k] - c) * (u[k] - c);
            grad[k] = 2.0 * F->w_out * (u[k] - c) / h;
        }
        *abs_e = fabs(E);
        return E;
    }
    int i0[3];
    double f[3];
    for (int k = 0; k < 3; k++) {
        i0[k] = (int)floor(u[k]);
        f[k] = u[k] - (double)i0[k];
    }
    const int m_e = G->n_maps - 2, m_d = G->n_maps - 1;
    const double coef[3] = {1.0, q, fabs(q)};
    const int mm[3] = {map, m_e, m_d};
    double E = 0.0, dEdu[3] = {0.0, 0.0, 0.0}, aE = 0.0;
    for (int cz = 0; cz < 2; cz++)
        for (int cy = 0; cy < 2; cy++)
            for (int cx = 0; cx < 2; cx++) {
                const int c[3] = {cx, cy, cz};
                double wk[3], dk[3];
                for (int k = 0; k < 3; k++) {
                    wk[k] = c[k] ? f[k] : 1.0 - f[k];
                    dk[k] = c[k] ? 1.0 : -1.0;
                }
                const double wgt = wk[0] * wk[1] * wk[2];
                const double dw[3] = {dk[0] * wk[1] * wk[2], wk[0] * dk[1] * wk[2], wk[0] * wk[1] * dk[2]};
                for (int t = 0; t < 3; t++) {
                    const double v = coef[t] * gv(G, mm[t], i0[0] + cx, i0[1] + cy, i0[2] + cz);
                    E += wgt * v;
                    aE += fabs(wgt * v);
                    for (int k = 0; k < 3; k++) dEdu[k] += dw[k] * v;
                }
            }
    for (int k = 0; k < 3; k++) grad[k] = dEdu[k] / h;
    *abs_e = aE;
    return E;
}

/* O-3: IntraGradient for one pair at distance r.
 * Returns E; *dEdr = dE/dr.  *abs_e = |cA s^-m| + |cB s^-n| + |E_el| + |E_ds|
 * (the Z18 magnitude sum).  Smoothing (Z6): delta = smooth/2,
 *   s = r + delta if r <= r0 - delta; s = r0 if r < r0 + delta; else r - delta.
 * vdW / H-bond if r < cut_vdw (Z7):  E = cA s^-m - cB s^-n  (Z10).
 * electrostatics if r < cut_el:      E = c_el qi qj / (r_e eps(r_e)),
 *   r_e = max(r, el_rmin) (Z8), eps(r) = A + B / (1 + k exp(-lambda B r)).
 * desolvation if r < cut_el:
 *   E = c_ds [(S_i + Q|q_i|) V_j + (S_j + Q|q_j|) V_i] exp(-r^2 / (2 sigma^2)). */
static double intra_pair(const ado_ligand* L, const ado_ff* F, int i, int j, double r, double* dEdr, double* abs_e,
                         double* margin_e, double* margin_g) {
    const int ti = L->atom_type[i], tj = L->atom_type[j];
    const float* tp = L->tp_coef + ((size_t)ti * L->n_types + tj) * 5;
    const double cA = tp[0], cB = tp[1], r0 = tp[2], m = tp[3], nn = tp[4];
    const double qi = L->charge[i], qj = L->charge[j];
    double E = 0.0, D = 0.0, aE = 0.0;
    const double delta = 0.5 * F->smooth;
    double me = fmin(fabs(r - F->cut_vdw), fabs(r - F->cut_el));
    double mg = fmin(fmin(fabs(r - (r0 - delta)), fabs(r - (r0 + delta))), fabs(r - F->el_rmin));
    if (r < F->cut_vdw) {
        double s, dsdr;
        if (r <= r0 - delta) { s = r + delta; dsdr = 1.0; }
        else if (r < r0 + delta) { s = r0; dsdr = 0.0; }
        else { s = r - delta; dsdr = 1.0; }
        const double ea = cA * pow(s, -m), eb = cB * pow(s, -nn);
        E += ea - eb;
        const double da = -m * cA * pow(s, -m - 1.0) * dsdr, db = -nn * cB * pow(s, -nn - 1.0) * dsdr;
        D += da - db;
        aE += fabs(ea) + fabs(eb);
    }
    if (r < F->cut_el) {
        const double lB = F->diel_lambda * F->diel_B;
        const int clamped = r < F->el_rmin;
        const double re = clamped ? F->el_rmin : r;
        const double ex = exp(-lB * re);
        const double eps = F->diel_A + F->diel_B / (1.0 + F->diel_k * ex);
        const double deps = F->diel_B * F->diel_k * lB * ex / ((1.0 + F->diel_k * ex) * (1.0 + F->diel_k * ex));
        const double eel = F->coeff_el * qi * qj / (re * eps);
        const double del = clamped ? 0.0 : -F->coeff_el * qi * qj * (eps + re * deps) / ((re * eps) * (re * eps));
        E += eel;
        D += del;
        aE += fabs(eel);
        const double Si = L->type_S[ti], Sj = L->type_S[tj], Vi = L->type_V[ti], Vj = L->type_V[tj];
        const double pref = F->coeff_ds * ((Si + F->qasp * fabs(qi)) * Vj + (Sj + F->qasp * fabs(qj)) * Vi);
        const double s2 = F->sigma_ds * F->sigma_ds;
        const double eds = pref * exp(-r * r / (2.0 * s2));
        const double dds = -eds * r / s2;
        E += eds;
        D += dds;
        aE += fabs(eds);
    }
    *dEdr = D;
    *abs_e = aE;
    *margin_e = me;
    *margin_g = mg;
    return E;
}

/* Per-atom Jacobian dX_i/dg_k (O-4, Z12): J[(i*G + k)*3 + c]. */
static void jacobian(const ado_ligand* L, const ado_grid* G, const double* g, const double* X, const double T[3],
                     double* J) {
    const int N = L->n_atoms, Gn = 6 + L->n_tors;
    memset(J, 0, sizeof(double) * (size_t)N * Gn * 3);
    const double phi = g[3] * DEG, th = g[4] * DEG, al = g[5] * DEG;
    const double u[3] = {sin(th) * cos(phi), sin(th) * sin(phi), cos(th)};
    const double uphi[3] = {-sin(th) * sin(phi), sin(th) * cos(phi), 0.0};
    const double uth[3] = {cos(th) * cos(phi), cos(th) * sin(phi), -sin(th)};
    /* angular velocity of R(u(phi,theta), alpha) per unit change of each angle */
    double om[3][3], t1[3], t2[3];
    cross(uphi, u, t1);
    cross(uth, u, t2);
    for (int k = 0; k < 3; k++) {
        om[0][k] = sin(al) * uphi[k] - (1.0 - cos(al)) * t1[k];
        om[1][k] = sin(al) * uth[k] - (1.0 - cos(al)) * t2[k];
        om[2][k] = u[k];
    }
    for (int i = 0; i < N; i++) {
        double* Ji = J + (size_t)i * Gn * 3;
        for (int k = 0; k < 3; k++) Ji[k * 3 + k] = G->spacing; /* translation, grid units */
        double r[3] = {X[3 * i] - T[0], X[3 * i + 1] - T[1], X[3 * i + 2] - T[2]}, c[3];
        for (int p = 0; p < 3; p++) {
            cross(om[p], r, c);
            for (int k = 0; k < 3; k++) Ji[(3 + p) * 3 + k] = DEG * c[k];
        }
    }
    for (int b = 0; b < L->n_tors; b++) {
        const int a = L->tors_axis[2 * b], cc = L->tors_axis[2 * b + 1];
        double ub[3];
        for (int k = 0; k < 3; k++) ub[k] = X[3 * cc + k] - X[3 * a + k];
        const double nb = sqrt(dot(ub, ub));
        for (int k = 0; k < 3; k++) ub[k] /= nb;
        for (int i = 0; i < N; i++) {
            if (!L->tors_moving[(size_t)b * N + i]) continue;
            double r[3] = {X[3 * i] - X[3 * a], X[3 * i + 1] - X[3 * a + 1], X[3 * i + 2] - X[3 * a + 2]}, c[3];
            cross(ub, r, c);
            for (int k = 0; k < 3; k++) J[((size_t)i * Gn + 6 + b) * 3 + k] = DEG * c[k];
        }
    }
}

/* One pose: E (O-5: inter + intra), gene gradient grad[G] (may be NULL),
 * aux[AUX_N] (may be NULL), agrad[G] (may be NULL), X_out [N][3] (may be NULL).
 * Scales of the Z18 tolerance:
 *   aux[AUX_ABS_E] = A_E = sum over every energy term of |term|
 *   agrad[k]       = A_grad[k] = sum of |summand| over the summands of the O-4
 *                    chain rule dE/dg_k = sum_i dX_i/dg_k . g_i, with g_i split
 *                    into its terms: |dX_i/dg_k . g_inter,i| per atom and
 *                    |dX_i/dg_k . F_p| + |dX_j/dg_k . F_p| per intra pair p
 *                    (F_p = dE_p/dr d_hat, the pair's force on i and on j).
 * aux[AUX_MARGIN_E] / aux[AUX_MARGIN_G]: distance (A) to the nearest energy
 * discontinuity (grid boundary, cutoff) / gradient kink (cell face, smoothing
 * band edge, electrostatic floor).
 * aux[AUX_SENS_E] = S_E, used ONLY by the separately labelled clash gate
 * (A_E >= 500): the first-order change of E when every
 * atom coordinate moves by its own length, sum_i |grad E_inter,i|_2 |X_i|_2 +
 * sum_p |dE_p/dr| (|X_i|_2 + |X_j|_2) -- times 2^-20 it bounds what rounding
 * the coordinates to 16 FP32 ulps can do to E.                              */
int ado_eval(const ado_ligand* L, const ado_grid* G, const ado_ff* F, const double* g, double* E_out, double* grad,
             double* aux, double* agrad, double* X_out) {
    const int N = L->n_atoms, Gn = 6 + L->n_tors;
    double* X = (double*)malloc(sizeof(double) * 3 * N);
    double* gi = (double*)calloc((size_t)3 * N, sizeof(double)); /* atom gradients */
    double* J = (double*)malloc(sizeof(double) * 3 * (size_t)N * Gn);
    double* acc = agrad ? (double*)calloc((size_t)Gn, sizeof(double)) : NULL;
    if (!X || !gi || !J || (agrad && !acc)) return -4;
    double T[3];
    ado_pose(L, G, g, X, T);
    jacobian(L, G, g, X, T, J);
    double Einter = 0.0, Eintra = 0.0, AE = 0.0, ME = 1e30, MG = 1e30, SE = 0.0;
    for (int i = 0; i < N; i++) {
        double gr[3], ae, me, mg;
        Einter += inter_atom(G, F, L->atom_map[i], (double)L->charge[i], X + 3 * i, gr, &ae, &me, &mg);
        AE += ae;
        SE += sqrt(dot(gr, gr)) * sqrt(dot(X + 3 * i, X + 3 * i));
        ME = fmin(ME, me);
        MG = fmin(MG, mg);
        for (int k = 0; k < 3; k++) gi[3 * i + k] += gr[k];
        if (acc)
            for (int q = 0; q < Gn; q++) acc[q] += fabs(dot(J + ((size_t)i * Gn + q) * 3, gr));
    }
    for (int p = 0; p < L->n_pairs; p++) {
        const int i = L->pairs[2 * p], j = L->pairs[2 * p + 1];
        double d[3];
        for (int k = 0; k < 3; k++) d[k] = X[3 * i + k] - X[3 * j + k];
        const double r = sqrt(dot(d, d));
        double dEdr, ae, me, mg;
        Eintra += intra_pair(L, F, i, j, r, &dEdr, &ae, &me, &mg);
        AE += ae;
        SE += fabs(dEdr) * (sqrt(dot(X + 3 * i, X + 3 * i)) + sqrt(dot(X + 3 * j, X + 3 * j)));
        ME = fmin(ME, me);
        MG = fmin(MG, mg);
        if (r > 0.0) {
            double fp[3];
            for (int k = 0; k < 3; k++) {
                fp[k] = dEdr * d[k] / r;
                gi[3 * i + k] += fp[k];
                gi[3 * j + k] -= fp[k];
            }
            if (acc)
                for (int q = 0; q < Gn; q++)
                    acc[q] += fabs(dot(J + ((size_t)i * Gn + q) * 3, fp)) + fabs(dot(J + ((size_t)j * Gn + q) * 3, fp));
        }
    }
    if (grad)
        for (int q = 0; q < Gn; q++) {
            double s = 0.0;
            for (int i = 0; i < N; i++) {
                const double* Jq = J + ((size_t)i * Gn + q) * 3;
                s += Jq[0] * gi[3 * i] + Jq[1] * gi[3 * i + 1] + Jq[2] * gi[3 * i + 2];
            }
            grad[q] = s;
        }
    *E_out = Einter + Eintra;
    if (aux) {
        aux[AUX_EINTER] = Einter;
        aux[AUX_EINTRA] = Eintra;
        aux[AUX_ABS_E] = AE;
        aux[AUX_MARGIN_E] = ME;
        aux[AUX_MARGIN_G] = MG;
        aux[AUX_SENS_E] = SE;
    }
    if (agrad)
        for (int q = 0; q < Gn; q++) agrad[q] = acc[q];
    if (X_out) memcpy(X_out, X, sizeof(double) * 3 * N);
    free(X);
    free(gi);
    free(J);
    free(acc);
    return 0;
}

/* Batch of poses (genes are FP32 rows of length `stride`), OpenMP over poses. */
int ado_score(const ado_ligand* L, const ado_grid* G, const ado_ff* F, int32_t n_poses, const float* genes,
              int32_t stride, double* E, double* grad /*[n][stride] or NULL*/, double* aux /*[n][AUX_N] or NULL*/,
              double* agrad /*[n][stride] or NULL*/, int32_t n_threads) {
    const int Gn = 6 + L->n_tors;
    if (stride < Gn) return -1;
    int err = 0;
#ifdef _OPENMP
#pragma omp parallel for schedule(dynamic, 1) num_threads(n_threads > 0 ? n_threads : 1)
#endif
    for (int p = 0; p < n_poses; p++) {
        double g[64 + 6];
        for (int q = 0; q < Gn; q++) g[q] = (double)genes[(size_t)p * stride + q];
        int rc = ado_eval(L, G, F, g, E + p, grad ? grad + (size_t)p * stride : NULL,
                          aux ? aux + (size_t)p * AUX_N : NULL, agrad ? agrad + (size_t)p * stride : NULL, NULL);
        if (rc) err = rc;
    }
    return err;
}

/* O-6: one ADADELTA update (Zeiler [19]) of every gene:
 *   E[g^2] <- rho E[g^2] + (1-rho) g^2
 *   dx     <- -g * sqrt(E[dx^2] + eps) / sqrt(E[g^2] + eps)
 *   E[dx^2]<- rho E[dx^2] + (1-rho) dx^2 ;  x <- x + dx                    */
int ado_adadelta_step(int32_t n_genes, const double* grad, double* eg2, double* ed2, double* genes, double rho,
                      double eps) {
    for (int k = 0; k < n_genes; k++) {
        eg2[k] = rho * eg2[k] + (1.0 - rho) * grad[k] * grad[k];
        const double dx = -grad[k] * sqrt(ed2[k] + eps) / sqrt(eg2[k] + eps);
        ed2[k] = rho * ed2[k] + (1.0 - rho) * dx * dx;
        genes[k] += dx;
    }
    return 0;
}

/* O-6: ADADELTA local search (Alg 3), per pose, max_iters evals
 * (300 by default).  Each iteration: (E, grad) = eval(genes); keep the
 * genotype if E < best_E (strict, earliest wins, Z15); update all genes.  The
 * update after the last eval is not evaluated (Z15).  No angle wrapping (Z16).
 * Outputs: best_genes [n][stride] (double), best_E [n], and (trace != NULL)
 * for every step (E, A_E, S_E, margin_e, margin_g) of the evaluated genotype,
 * trace [n][max_iters][5] (Z19 ii free-running trajectories: the gate scales
 * of the step and its distances to the nearest energy discontinuity / gradient
 * kink). */
int ado_local_search(const ado_ligand* L, const ado_grid* G, const ado_ff* F, int32_t n_poses, const float* genes,
                     int32_t stride, int32_t max_iters, double rho, double eps, double* best_genes, double* best_E,
                     double* trace, int32_t n_threads) {
    const int Gn = 6 + L->n_tors;
    if (stride < Gn) return -1;
    int err = 0;
#ifdef _OPENMP
#pragma omp parallel for schedule(dynamic, 1) num_threads(n_threads > 0 ? n_threads : 1)
#endif
    for (int p = 0; p < n_poses; p++) {
        double x[70], gr[70], eg2[70], ed2[70], best[70];
        for (int q = 0; q < Gn; q++) {
            x[q] = (double)genes[(size_t)p * stride + q];
            eg2[q] = 0.0;
            ed2[q] = 0.0;
            best[q] = x[q];
        }
        double bE = INFINITY;
        for (int it = 0; it < max_iters; it++) {
            double E, aux[AUX_N];
            int rc = ado_eval(L, G, F, x, &E, gr, trace ? aux : NULL, NULL, NULL);
            if (rc) err = rc;
            if (trace) {
                double* t = trace + ((size_t)p * max_iters + it) * 5;
                t[0] = E;
                t[1] = aux[AUX_ABS_E];
                t[2] = aux[AUX_SENS_E];
                t[3] = aux[AUX_MARGIN_E];
                t[4] = aux[AUX_MARGIN_G];
            }
            if (E < bE) {
                bE = E;
                for (int q = 0; q < Gn; q++) best[q] = x[q];
            }
            ado_adadelta_step(Gn, gr, eg2, ed2, x, rho, eps);
        }
        best_E[p] = bE;
        for (int q = 0; q < stride; q++) best_genes[(size_t)p * stride + q] = q < Gn ? best[q] : 0.0;
    }
    return err;
}

/* O-8: best of run: argmin of best_E over each run of `pop`
 * consecutive poses, ties -> lowest index. */
int ado_best_of_run(int32_t n_poses, int32_t pop, const double* best_E, int32_t* run_best) {
    if (pop <= 0 || n_poses % pop) return -1;
    for (int r = 0; r < n_poses / pop; r++) {
        int bi = r * pop;
        for (int p = r * pop + 1; p < (r + 1) * pop; p++)
            if (best_E[p] < best_E[bi]) bi = p;
        run_best[r] = bi;
    }
    return 0;
}

/* O-7: exact sum of n FP32 values (stride `stride`), rounded once to double.
 * Shewchuk's non-overlapping expansion (the algorithm behind math.fsum). */
double ado_exact_sum(const float* x, int64_t n, int64_t stride) {
    double part[64];
    int np = 0;
    for (int64_t t = 0; t < n; t++) {
        double v = (double)x[t * stride];
        int k = 0;
        for (int q = 0; q < np; q++) {
            double y = part[q];
            if (fabs(v) < fabs(y)) { double tmp = v; v = y; y = tmp; }
            double hi = v + y;
            double lo = y - (hi - v);
            if (lo != 0.0) part[k++] = lo;
            v = hi;
        }
        part[k++] = v;
        np = k;
    }
    double s = 0.0;
    for (int q = np - 1; q >= 0; q--) {
        /* sum from the largest magnitude partial downward (partials are
         * non-overlapping and increasing), then correct the final rounding
         * like math.fsum does */
        double hi = s + part[q];
        double lo = part[q] - (hi - s);
        s = hi;
        if (lo != 0.0) {
            if (q > 0 && ((lo < 0.0 && part[q - 1] < 0.0) || (lo > 0.0 && part[q - 1] > 0.0))) {
                double yv = lo * 2.0, xv = s + yv;
                if (yv == xv - s) s = xv;
            }
            break;
        }
    }
    return s;
}

/* ---- NEXT-3: one generation of the Lamarckian GA (Alg 1) ----
 * The paper names the operators (selection, crossover, mutation) and the
 * driver loop, not their parameters; the readings (AutoDock-GPU
 * defaults [ext]) are: elitism, binary tournaments (the better of two random
 * individuals wins with probability tour_rate), two-point crossover with
 * probability cross_rate, per-gene uniform mutation with probability mut_rate
 * (+-dmov grid units on translation genes, +-dang degrees on angle genes), LS on
 * each new individual with probability ls_rate.
 *
 * Random numbers: a counter-based generator (each side implements it; nothing
 * is shared): x = mix(mix(mix(seed ^ (gen << 32 | run)) ^ (ind << 32 | d)))
 * with mix = the SplitMix64 step (add the golden gamma, then the finaliser);
 * a uniform u = (x >> 40) * 2^-24 (exact in FP32); an index = (x >> 32) % m.
 * Draw ids d per new individual: 0/1/2 tournament 1 (a, b, coin), 3/4/5
 * tournament 2, 6 crossover coin, 7/8 cut points, 16+i mutation coin of gene i,
 * 80+i its delta, 150 LS coin.
 * The mutation arithmetic is done in FP32 exactly as written (t = 2u - 1 is
 * exact, delta = t * max one rounding, gene + delta one rounding): the genotype
 * is FP32, so this reproduces the GPU bit for bit (compiled without
 * contraction); selection compares the FP32 energies it is given. */
static uint64_t ado_mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t ado_rng_mix(uint64_t z) { return ado_mix(z); }

uint64_t ado_rng(uint64_t seed, uint32_t gen, uint32_t run, uint32_t ind, uint32_t d) {
    return ado_mix(ado_mix(ado_mix(seed ^ (((uint64_t)gen << 32) | run)) ^ (((uint64_t)ind << 32) | d)));
}

static float ado_u24(uint64_t x) { return (float)(x >> 40) * (1.0f / 16777216.0f); }

typedef struct {
    int32_t pop, n_genes, stride, elitism;
    float cross_rate, mut_rate, tour_rate, ls_rate;
    float dmov, dang; /* mutation half-widths: grid units, degrees */
} ado_ga;

/* index of the better of a, b: lower energy, ties -> lower index */
static int ado_better(const float* E, int a, int b) { return (E[a] < E[b] || (E[a] == E[b] && a < b)) ? a : b; }

static int ado_tournament(const ado_ga* P, const float* E, uint64_t seed, uint32_t gen, uint32_t run, uint32_t ind,
                          uint32_t d0) {
    const int a = (int)((ado_rng(seed, gen, run, ind, d0) >> 32) % (uint64_t)P->pop);
    const int b = (int)((ado_rng(seed, gen, run, ind, d0 + 1) >> 32) % (uint64_t)P->pop);
    const int best = ado_better(E, a, b), worst = best == a ? b : a;
    return ado_u24(ado_rng(seed, gen, run, ind, d0 + 2)) < P->tour_rate ? best : worst;
}

/* genes_in/out [pop][stride] of ONE run, E_in [pop] its energies. */
int ado_ga_generation(const ado_ga* P, const float* genes_in, const float* E_in, float* genes_out, uint64_t seed,
                      uint32_t gen, uint32_t run) {
    const int pop = P->pop, G = P->n_genes, S = P->stride;
    if (pop < 2 || G < 1 || G > 64 || S < G || P->elitism < 0 || P->elitism > pop) return -1;
    /* elitism: the `elitism` best individuals, in order of increasing energy */
    char* used = (char*)calloc((size_t)pop, 1);
    for (int k = 0; k < P->elitism; k++) {
        int bi = -1;
        for (int q = 0; q < pop; q++)
            if (!used[q] && (bi < 0 || ado_better(E_in, q, bi) == q)) bi = q;
        used[bi] = 1;
        memcpy(genes_out + (size_t)k * S, genes_in + (size_t)bi * S, sizeof(float) * (size_t)S);
    }
    free(used);
    for (int k = P->elitism; k < pop; k++) {
        const int p1 = ado_tournament(P, E_in, seed, gen, run, (uint32_t)k, 0);
        const int p2 = ado_tournament(P, E_in, seed, gen, run, (uint32_t)k, 3);
        float* c = genes_out + (size_t)k * S;
        memcpy(c, genes_in + (size_t)p1 * S, sizeof(float) * (size_t)S);
        if (ado_u24(ado_rng(seed, gen, run, (uint32_t)k, 6)) < P->cross_rate) {
            int c1 = (int)((ado_rng(seed, gen, run, (uint32_t)k, 7) >> 32) % (uint64_t)(G + 1));
            int c2 = (int)((ado_rng(seed, gen, run, (uint32_t)k, 8) >> 32) % (uint64_t)(G + 1));
            if (c1 > c2) { int t = c1; c1 = c2; c2 = t; }
            for (int i = c1; i < c2; i++) c[i] = genes_in[(size_t)p2 * S + i];
        }
        for (int i = 0; i < G; i++) {
            if (!(ado_u24(ado_rng(seed, gen, run, (uint32_t)k, 16 + (uint32_t)i)) < P->mut_rate)) continue;
            const float u = ado_u24(ado_rng(seed, gen, run, (uint32_t)k, 80 + (uint32_t)i));
            const float t = 2.0f * u - 1.0f;
            const float delta = t * (i < 3 ? P->dmov : P->dang);
            c[i] = c[i] + delta;
        }
    }
    return 0;
}

/* LS coin of every individual of one run: sel[k] = u < ls_rate (draw id 150). */
int ado_ls_select(const ado_ga* P, uint64_t seed, uint32_t gen, uint32_t run, uint8_t* sel) {
    for (int k = 0; k < P->pop; k++) sel[k] = ado_u24(ado_rng(seed, gen, run, (uint32_t)k, 150)) < P->ls_rate;
    return 0;
}

int ado_version(void) { return 1; }
