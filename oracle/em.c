/*
 * em.c -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.
 *
 * Plain, slow, single-threaded CPU oracle of the CabanaPIC-style
 * electromagnetic Move_Deposit routine:
 * for every particle, interpolate E and B from its cell's interpolator,
 * Boris-push the momentum, then move the particle along its straight
 * displacement through the faces it crosses (next cell from the c2c map) and
 * deposit the Eq. 11 current of every segment into the accumulator of the cell
 * the segment lies in.  Only tests/ and bench.py's cpu_baseline /
 * --impl reference legs may load it; it shares no code with csrc/.
 *
 * Passages followed (PAPER.md line ranges):
 *   Lorentz force / equations of motion ...... 533-583  (Eqs. 7-9; with B: Boris)
 *   Eq. 11 current along the straight path ... 617-680  (i_i = Q_p/dt int W^1_i dL,
 *                                                        "fields assessed on each
 *                                                        cell along the path")
 *   CabanaPIC structure ...................... 1514-1542, 1656-1682 (Interpolate ->
 *                                                        Move_Deposit -> accumulator;
 *                                                        periodic; next cell from the
 *                                                        direction of motion + int map,
 *                                                        1861-1873)
 * Everything else is a reading, listed in DESIGN.md §10 (E1-E9): the
 * interpolator form, the relativistic Boris rotation, offset coordinates in
 * [-1, 1]^3, the face order of c2c, the tie rules, the crossing cap.
 *
 * The Eq. 11 integral is evaluated here by 2-point Gauss-Legendre quadrature
 * (exact: the integrand is quadratic in the path parameter); the CUDA kernel
 * uses the closed form.  Compiled with -O2 -ffp-contract=off (no FMA).
 *
 * Pins (tests/test_oracle_em.py): ballistic motion with periodic wrap in zero
 * field (closed form), B = 0 momentum update (closed form), E = 0 rotation
 * angle 2 atan(|t|) and |u| conservation, the discrete charge-continuity
 * identity of the Whitney pair W0/W1 (node weights at the end minus at the
 * start equal the divergence of the deposited edge currents), axis-aligned
 * segments against the one-dimensional closed form, and the interpolator
 * reproducing its edge values.
 */
#include <math.h>
#include <stdint.h>

#define EM_NI 18   /* interpolator doubles per cell  */
#define EM_NA 12   /* accumulator doubles per cell   */

typedef struct {
    double qdt_2mc;     /* q dt / (2 m c): E and B enter the push scaled by it   */
    double cdt_2h[3];   /* 2 c dt / h_a: offset units per unit velocity/c        */
    double qsp;         /* charge per unit weight                                */
    int32_t kcap;       /* face crossings allowed per particle and step          */
    int32_t pad;
} em_params;

typedef struct {
    int64_t n_crossings;
    int64_t n_capped;
    int32_t max_crossings;
    int32_t pad;
} em_stats;

/* E and B at offset (x, y, z) of a cell: the interpolator of VPIC/CabanaPIC
 * ("Interpolate ... computes derivatives of field values, storing them as
 * interpolator values within cell data"):
 *   ex ey ez bilinear in the two transverse offsets, b_a linear along a. */
static void em_fields(const double *f, double x, double y, double z, double E[3], double B[3]) {
    E[0] = (f[0] + y * f[1]) + z * (f[2] + y * f[3]);
    E[1] = (f[4] + z * f[5]) + x * (f[6] + z * f[7]);
    E[2] = (f[8] + x * f[9]) + y * (f[10] + x * f[11]);
    B[0] = f[12] + x * f[13];
    B[1] = f[14] + y * f[15];
    B[2] = f[16] + z * f[17];
}

/* Relativistic Boris push (Eqs. 7-9 with the Lorentz force; reading E2):
 * half electric kick, magnetic rotation with t = qdt_2mc B / gamma,
 * s = 2 t / (1 + |t|^2), second half kick.  u = gamma v / c. */
void em_boris(const double f_at[6], double qdt_2mc, double u[3]) {
    const double hE[3] = {qdt_2mc * f_at[0], qdt_2mc * f_at[1], qdt_2mc * f_at[2]};
    double um[3] = {u[0] + hE[0], u[1] + hE[1], u[2] + hE[2]};
    const double gamma = sqrt(1.0 + (um[0] * um[0] + um[1] * um[1] + um[2] * um[2]));
    const double r = qdt_2mc / gamma;
    const double t[3] = {r * f_at[3], r * f_at[4], r * f_at[5]};
    const double tt = t[0] * t[0] + t[1] * t[1] + t[2] * t[2];
    const double up[3] = {um[0] + (um[1] * t[2] - um[2] * t[1]),
                          um[1] + (um[2] * t[0] - um[0] * t[2]),
                          um[2] + (um[0] * t[1] - um[1] * t[0])};
    const double sc = 2.0 / (1.0 + tt);
    const double s[3] = {sc * t[0], sc * t[1], sc * t[2]};
    um[0] = um[0] + (up[1] * s[2] - up[2] * s[1]);
    um[1] = um[1] + (up[2] * s[0] - up[0] * s[2]);
    um[2] = um[2] + (up[0] * s[1] - up[1] * s[0]);
    u[0] = um[0] + hE[0];
    u[1] = um[1] + hE[1];
    u[2] = um[2] + hE[2];
}

/* Eq. 11 for one straight segment p -> q inside a cell, charge Q:
 * acc[4a + k] += Q * int_0^1 N_{a,k}(p + t (q - p)) (q_a - p_a) dt, where for
 * the edges along axis a the transverse offsets are (b, c) = ((a+1)%3, (a+2)%3),
 * edge k = (sb, sc) in the order (-,-), (+,-), (-,+), (+,+) and
 * N_{a,k} = (1 + sb * b)(1 + sc * c) / 4 -- the Whitney edge function of that
 * edge dotted with the path (W^1 = N grad(offset_a)).
 * Two-point Gauss-Legendre, exact for the quadratic integrand. */
void em_segment_current(const double p[3], const double q[3], double Q, double acc[EM_NA]) {
    const double g = 0.5 / sqrt(3.0);
    const double tq[2] = {0.5 - g, 0.5 + g};
    for (int a = 0; a < 3; a++) {
        const int b = (a + 1) % 3, c = (a + 2) % 3;
        const double da = q[a] - p[a];
        for (int k = 0; k < 4; k++) {
            const double sb = (k & 1) ? 1.0 : -1.0, sc = (k & 2) ? 1.0 : -1.0;
            double sum = 0.0;
            for (int m = 0; m < 2; m++) {
                const double xb = p[b] + tq[m] * (q[b] - p[b]);
                const double xc = p[c] + tq[m] * (q[c] - p[c]);
                sum += (1.0 + sb * xb) * (1.0 + sc * xc) / 4.0;
            }
            acc[4 * a + k] += Q * (da * (sum / 2.0));
        }
    }
}

/* One Move_Deposit step for particles [0, n).  SoA columns:
 * off[3][n] offsets in [-1, 1], u[3][n] momenta, w[n] weights, cell[n].
 * interp[nc][18], c2c[nc][6] (faces -x,+x,-y,+y,-z,+z), acc[nc][12] (added to). */
void em_move_deposit(int64_t n, double *off, double *u, const double *w, int32_t *cell,
                     const double *interp, const int32_t *c2c, double *acc,
                     const em_params *P, em_stats *st) {
    for (int64_t i = 0; i < n; i++) {
        int c = cell[i];
        double p[3] = {off[i], off[n + i], off[2 * n + i]};
        double uu[3] = {u[i], u[n + i], u[2 * n + i]};
        /* Interpolate + push */
        double E[3], B[3];
        em_fields(interp + (int64_t)EM_NI * c, p[0], p[1], p[2], E, B);
        const double fa[6] = {E[0], E[1], E[2], B[0], B[1], B[2]};
        em_boris(fa, P->qdt_2mc, uu);
        /* streak in offset units (reading E4) */
        const double rg = 1.0 / sqrt(1.0 + (uu[0] * uu[0] + uu[1] * uu[1] + uu[2] * uu[2]));
        double d[3] = {P->cdt_2h[0] * (uu[0] * rg), P->cdt_2h[1] * (uu[1] * rg),
                       P->cdt_2h[2] * (uu[2] * rg)};
        const double Q = P->qsp * w[i];
        /* move through the faces crossed, in order (reading E5) */
        int k = 0;
        for (;;) {
            double t = 1.0;
            int face = -1;
            for (int a = 0; a < 3; a++) {
                if (d[a] > 0.0) {
                    const double ta = (1.0 - p[a]) / d[a];
                    if (ta < t) { t = ta; face = 2 * a + 1; }
                } else if (d[a] < 0.0) {
                    const double ta = (-1.0 - p[a]) / d[a];
                    if (ta < t) { t = ta; face = 2 * a; }
                }
            }
            double q[3];
            for (int a = 0; a < 3; a++) q[a] = p[a] + t * d[a];
            if (face >= 0) q[face >> 1] = (face & 1) ? 1.0 : -1.0;   /* exactly on the face */
            em_segment_current(p, q, Q, acc + (int64_t)EM_NA * c);
            if (face < 0) {
                for (int a = 0; a < 3; a++) p[a] = q[a];
                break;
            }
            if (k >= P->kcap) {   /* cap: stop on the face, inside this cell */
                for (int a = 0; a < 3; a++) p[a] = q[a];
                st->n_capped++;
                break;
            }
            for (int a = 0; a < 3; a++) {
                d[a] = d[a] - (q[a] - p[a]);
                p[a] = q[a];
            }
            p[face >> 1] = -p[face >> 1];   /* +1 in this cell is -1 in the next */
            c = c2c[6 * (int64_t)c + face];
            k++;
        }
        st->n_crossings += k;
        if (k > st->max_crossings) st->max_crossings = k;
        off[i] = p[0]; off[n + i] = p[1]; off[2 * n + i] = p[2];
        u[i] = uu[0]; u[n + i] = uu[1]; u[2 * n + i] = uu[2];
        cell[i] = c;
    }
}

/* Interpolate from edge-centred E and face-centred B on a
 * periodic nx*ny*nz grid: cell (i,j,k), E_a on the 4 edges of the cell along a,
 * B_a on the 2 faces normal to a.  Field layout: e[3][nc] holds, for every cell,
 * the value on its edge at the (-,-) corner of the transverse offsets; the other
 * three edges of a cell are those of its transverse neighbours (periodic);
 * b[3][nc] the value on its face at offset -1.  The coefficients make E_a the
 * bilinear interpolant of its 4 edge values and B_a the linear interpolant of its
 * 2 face values. */
void em_interpolate(int nx, int ny, int nz, const double *e, const double *b, double *interp) {
    const int64_t nc = (int64_t)nx * ny * nz;
    for (int k = 0; k < nz; k++)
        for (int j = 0; j < ny; j++)
            for (int i = 0; i < nx; i++) {
                const int64_t c = i + (int64_t)nx * (j + (int64_t)ny * k);
                const int ip = (i + 1) % nx, jp = (j + 1) % ny, kp = (k + 1) % nz;
#define ID(I, J, K) ((I) + (int64_t)nx * ((J) + (int64_t)ny * (K)))
                double v[3][4];
                /* x edges: transverse (y, z); order (-,-), (+,-), (-,+), (+,+) */
                v[0][0] = e[ID(i, j, k)];        v[0][1] = e[ID(i, jp, k)];
                v[0][2] = e[ID(i, j, kp)];       v[0][3] = e[ID(i, jp, kp)];
                /* y edges: transverse (z, x) */
                v[1][0] = e[nc + ID(i, j, k)];   v[1][1] = e[nc + ID(i, j, kp)];
                v[1][2] = e[nc + ID(ip, j, k)];  v[1][3] = e[nc + ID(ip, j, kp)];
                /* z edges: transverse (x, y) */
                v[2][0] = e[2 * nc + ID(i, j, k)];  v[2][1] = e[2 * nc + ID(ip, j, k)];
                v[2][2] = e[2 * nc + ID(i, jp, k)]; v[2][3] = e[2 * nc + ID(ip, jp, k)];
                double *f = interp + EM_NI * c;
                for (int a = 0; a < 3; a++) {
                    const double *q = v[a];
                    /* f0 + s*f1 + t*(f2 + s*f3) with (s, t) the transverse offsets */
                    f[4 * a + 0] = ((q[0] + q[1]) + (q[2] + q[3])) / 4.0;
                    f[4 * a + 1] = ((q[1] - q[0]) + (q[3] - q[2])) / 4.0;
                    f[4 * a + 2] = ((q[2] - q[0]) + (q[3] - q[1])) / 4.0;
                    f[4 * a + 3] = ((q[3] - q[2]) - (q[1] - q[0])) / 4.0;
                }
                const double b0x = b[ID(i, j, k)], b1x = b[ID(ip, j, k)];
                const double b0y = b[nc + ID(i, j, k)], b1y = b[nc + ID(i, jp, k)];
                const double b0z = b[2 * nc + ID(i, j, k)], b1z = b[2 * nc + ID(i, j, kp)];
                f[12] = (b0x + b1x) / 2.0; f[13] = (b1x - b0x) / 2.0;
                f[14] = (b0y + b1y) / 2.0; f[15] = (b1y - b0y) / 2.0;
                f[16] = (b0z + b1z) / 2.0; f[17] = (b1z - b0z) / 2.0;
#undef ID
            }
}
