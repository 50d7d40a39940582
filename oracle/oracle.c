/*
 * oracle.c -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.
 *
 * A plain, slow, single-threaded CPU implementation of the OP-PIC
 * Mini-FEM-PIC particle loop (one time step = inject -> zero node charge ->
 * push -> locate -> deposit -> compact), written from the paper and SURVEY.md
 * §8(c).  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  It shares no code, header, table or
 * helper with the CUDA path (paper_conf_icpp_lantra0m24_b200/csrc); the only
 * thing both sides see is the seeded input generator in gen/.
 *
 * Compiled with -O2 -ffp-contract=off (no FMA contraction, S11); every
 * floating-point expression is evaluated left to right as written.
 *
 * Passages followed (PAPER.md line ranges; the section/figure/equation in
 * parentheses):
 *   loop order ........................ 398-410   (§2, Fig. 1)
 *   cell-constant E (no weighting) .... 1576-1585 (§4.1.1)
 *   leap-frog push .................... 569-583   (§2 step 3, Eqs. 7-9, B = 0)
 *   multi-hop walk, statuses .......... 595-603, 1098-1146, 1324-1334 (Fig. 6, 7a)
 *   direct-hop seeding ................ 603-615, 1356-1370 (Fig. 7b)
 *   charge deposit, Eq. 10 ............ 617-660   (q_i = Q_p W^0_i(r_p))
 *   removal at the boundary ........... 1508-1510
 *   injection ......................... 1014-1018, 1502-1508
 *   hole fill ......................... 1346-1352 (the oracle compacts stably;
 *                                       any permutation is correct, S10)
 * Readings where the paper is silent are SURVEY.md §8(c) S1-S22 and are listed
 * in DESIGN.md §3.  Every function below is pinned by a -m "not gpu" test
 * (tests/test_oracle_pins.py); see the per-function notes.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_DONE 0
#define ORC_REMOVE 2

/* ------------------------------------------------------------------------ */
/* Mesh                                                                      */
/* ------------------------------------------------------------------------ */
typedef struct {
    int64_t nn, nc;
    double *xyz;     /* nn*3 node coordinates                               */
    int32_t *c2n;    /* nc*4, positive orientation                          */
    int32_t *c2c;    /* nc*4, c2c[c][i] = neighbour across face opposite i   */
    double *g;       /* nc*9, rows = grad lambda_1..3 (S: node-relative form)*/
    double *p0;      /* nc*3, coordinates of local node 0                   */
    double *vol6;    /* nc, 6 * signed volume                               */
    double *ef;      /* nc*3 cell electric field (cell-constant, 1576-1585) */
    /* direct-hop overlay (S19) */
    double ov_x0[3], ov_dx;
    int ov_n[3];
    int32_t *ov_map;
} orc_mesh;

/*
 * Cell geometry.  With a = p1-p0, b = p2-p0, c = p3-p0 the map
 * lambda_{1..3} -> x - p0 is the matrix M = [a b c]; its inverse has rows
 * (b x c)/det, (c x a)/det, (a x b)/det with det = a . (b x c) (Cramer's
 * rule).  So lambda_i = g_i . (x - p0), lambda_0 = 1 - (l1 + l2 + l3): the
 * barycentric coordinates of Eq. 10's W^0.
 * Pinned by P1 (sum to 1, reconstruct x, Kronecker delta at the nodes).
 */
static void cross3(const double *u, const double *v, double *w) {
    w[0] = u[1] * v[2] - u[2] * v[1];
    w[1] = u[2] * v[0] - u[0] * v[2];
    w[2] = u[0] * v[1] - u[1] * v[0];
}

static void cell_geometry(orc_mesh *m, int64_t c) {
    const double *P[4];
    for (int i = 0; i < 4; i++) P[i] = m->xyz + 3 * (int64_t)m->c2n[4 * c + i];
    double a[3], b[3], cc[3], bxc[3], cxa[3], axb[3];
    for (int k = 0; k < 3; k++) {
        a[k] = P[1][k] - P[0][k];
        b[k] = P[2][k] - P[0][k];
        cc[k] = P[3][k] - P[0][k];
    }
    cross3(b, cc, bxc);
    cross3(cc, a, cxa);
    cross3(a, b, axb);
    double det = a[0] * bxc[0] + a[1] * bxc[1] + a[2] * bxc[2];
    double *g = m->g + 9 * c;
    for (int k = 0; k < 3; k++) {
        g[0 + k] = bxc[k] / det;
        g[3 + k] = cxa[k] / det;
        g[6 + k] = axb[k] / det;
        m->p0[3 * c + k] = P[0][k];
    }
    m->vol6[c] = det;
}

orc_mesh *orc_mesh_new(int64_t nn, const double *xyz, int64_t nc, const int32_t *c2n,
                       const int32_t *c2c) {
    orc_mesh *m = (orc_mesh *)calloc(1, sizeof(orc_mesh));
    if (!m) return NULL;
    m->nn = nn;
    m->nc = nc;
    m->xyz = (double *)malloc(sizeof(double) * 3 * (nn > 0 ? nn : 1));
    m->c2n = (int32_t *)malloc(sizeof(int32_t) * 4 * (nc > 0 ? nc : 1));
    m->c2c = (int32_t *)malloc(sizeof(int32_t) * 4 * (nc > 0 ? nc : 1));
    m->g = (double *)malloc(sizeof(double) * 9 * (nc > 0 ? nc : 1));
    m->p0 = (double *)malloc(sizeof(double) * 3 * (nc > 0 ? nc : 1));
    m->vol6 = (double *)malloc(sizeof(double) * (nc > 0 ? nc : 1));
    m->ef = (double *)calloc(3 * (nc > 0 ? nc : 1), sizeof(double));
    memcpy(m->xyz, xyz, sizeof(double) * 3 * nn);
    memcpy(m->c2n, c2n, sizeof(int32_t) * 4 * nc);
    memcpy(m->c2c, c2c, sizeof(int32_t) * 4 * nc);
    for (int64_t c = 0; c < nc; c++) cell_geometry(m, c);
    return m;
}

void orc_mesh_free(orc_mesh *m) {
    if (!m) return;
    free(m->xyz); free(m->c2n); free(m->c2c); free(m->g); free(m->p0);
    free(m->vol6); free(m->ef); free(m->ov_map);
    free(m);
}

void orc_mesh_geometry(const orc_mesh *m, double *g, double *p0, double *vol6) {
    if (g) memcpy(g, m->g, sizeof(double) * 9 * m->nc);
    if (p0) memcpy(p0, m->p0, sizeof(double) * 3 * m->nc);
    if (vol6) memcpy(vol6, m->vol6, sizeof(double) * m->nc);
}

void orc_mesh_set_field(orc_mesh *m, const double *ef) {
    memcpy(m->ef, ef, sizeof(double) * 3 * m->nc);
}

/* Barycentric coordinates of x in cell c (node-relative form). */
void orc_bary(const orc_mesh *m, int32_t c, const double *x, double *lam) {
    const double *g = m->g + 9 * (int64_t)c;
    const double *p0 = m->p0 + 3 * (int64_t)c;
    double d0 = x[0] - p0[0], d1 = x[1] - p0[1], d2 = x[2] - p0[2];
    double l1 = g[0] * d0 + g[1] * d1 + g[2] * d2;
    double l2 = g[3] * d0 + g[4] * d1 + g[5] * d2;
    double l3 = g[6] * d0 + g[7] * d1 + g[8] * d2;
    lam[1] = l1;
    lam[2] = l2;
    lam[3] = l3;
    lam[0] = 1.0 - (l1 + l2 + l3);
}

/* Inside test, inclusive (S1): 0 <= lambda_i <= 1 for every i. */
static int inside(const double *lam) {
    for (int i = 0; i < 4; i++)
        if (!(lam[i] >= 0.0 && lam[i] <= 1.0)) return 0;
    return 1;
}

/*
 * Plain definition of point location, for pins: the lowest-index cell whose
 * barycentric coordinates are all >= -tol.  -1 if none.  O(nc) per query.
 */
int32_t orc_locate_brute(const orc_mesh *m, const double *x, double tol) {
    double lam[4];
    for (int64_t c = 0; c < m->nc; c++) {
        orc_bary(m, (int32_t)c, x, lam);
        if (lam[0] >= -tol && lam[1] >= -tol && lam[2] >= -tol && lam[3] >= -tol)
            return (int32_t)c;
    }
    return -1;
}

/*
 * Multi-hop walk ("jumping to the most probable neighbor
 * ... iterative process starting from the initial location"; the Fig. 6
 * template 1098-1124; statuses MOVE_DONE / NEED_MOVE / NEED_REMOVE).
 * Most probable neighbour = across the face opposite the most negative
 * lambda, lowest index on ties (S2).  Hop cap (S4): once `hops` reaches
 * hcap the current cell is accepted as DONE and *capped is set.
 * On return lam holds the coordinates in the final (or exit) cell.
 * Pinned by P2 (brute force, Kuhn closed form, REMOVE <=> outside the box).
 */
int orc_walk(const orc_mesh *m, int32_t cell, const double *x, int32_t hops0, int32_t hcap,
             int32_t *out_cell, int32_t *out_hops, double *lam, int32_t *capped) {
    int32_t hops = hops0;
    *capped = 0;
    for (;;) {
        orc_bary(m, cell, x, lam);
        if (inside(lam)) break;
        if (hops >= hcap) {
            *capped = 1;
            break;
        }
        int imin = 0;
        for (int i = 1; i < 4; i++)
            if (lam[i] < lam[imin]) imin = i;
        int32_t nb = m->c2c[4 * (int64_t)cell + imin];
        if (nb < 0) {
            *out_cell = cell;
            *out_hops = hops;
            return ORC_REMOVE;
        }
        cell = nb;
        hops++;
    }
    *out_cell = cell;
    *out_hops = hops;
    return ORC_DONE;
}

/*
 * Direct-hop overlay cell-map ("mapping from
 * structured-mesh cell to unstructured-mesh cells"; S19): cell g of a
 * regular grid (origin x0, spacing dx, n[3] cells) maps to the lowest-index
 * tet containing its centre (inclusive test), -1 if none.  Brute force over
 * all tets -- the plain definition; O(grid * nc), small meshes only.
 * Pinned by P7 (DH == MH final cells) and by the closed-form Kuhn location.
 */
int orc_overlay_build(orc_mesh *m, const double *x0, double dx, const int32_t *n) {
    int64_t tot = (int64_t)n[0] * n[1] * n[2];
    free(m->ov_map);
    m->ov_map = (int32_t *)malloc(sizeof(int32_t) * (tot > 0 ? tot : 1));
    if (!m->ov_map) return -1;
    for (int k = 0; k < 3; k++) {
        m->ov_x0[k] = x0[k];
        m->ov_n[k] = n[k];
    }
    m->ov_dx = dx;
    for (int64_t gz = 0; gz < n[2]; gz++)
        for (int64_t gy = 0; gy < n[1]; gy++)
            for (int64_t gx = 0; gx < n[0]; gx++) {
                double ctr[3] = {x0[0] + ((double)gx + 0.5) * dx, x0[1] + ((double)gy + 0.5) * dx,
                                 x0[2] + ((double)gz + 0.5) * dx};
                m->ov_map[gx + n[0] * (gy + n[1] * gz)] = orc_locate_brute(m, ctr, 0.0);
            }
    return 0;
}

void orc_overlay_get(const orc_mesh *m, int32_t *out) {
    int64_t tot = (int64_t)m->ov_n[0] * m->ov_n[1] * m->ov_n[2];
    memcpy(out, m->ov_map, sizeof(int32_t) * tot);
}

/* DH seed: the overlay cell of x if x is inside the overlay box and the map
 * entry is a tet, otherwise the start cell (S19).  The overlay index is
 * floor((x - x0) * (1/dx)) with 1/dx rounded once (reading S19'):
 * the paper gives no formula; a multiply keeps the GPU seed free of a
 * division per particle and both sides evaluate it identically. */
static int32_t dh_seed(const orc_mesh *m, const double *x, int32_t cell) {
    int64_t g[3];
    for (int k = 0; k < 3; k++) {
        double t = (x[k] - m->ov_x0[k]) * (1.0 / m->ov_dx);   /* reading S19': index by x * (1/dx) */
        if (!(t >= 0.0)) return cell;
        g[k] = (int64_t)floor(t);
        if (g[k] >= m->ov_n[k]) return cell;
    }
    int32_t s = m->ov_map[g[0] + m->ov_n[0] * (g[1] + m->ov_n[1] * g[2])];
    return s >= 0 ? s : cell;
}

/* ------------------------------------------------------------------------ */
/* Particles (AoS, plain arrays; ids int64 never reused, S21)               */
/* ------------------------------------------------------------------------ */
typedef struct {
    int64_t n, cap;
    double *pos, *vel, *margin;
    int32_t *cell;
    int64_t *id;
    /* particles removed by the last orc_step: id and exit margin */
    int64_t n_rem, rem_cap;
    int64_t *rem_id;
    double *rem_margin;
} orc_parts;

static int parts_reserve(orc_parts *p, int64_t need) {
    if (need <= p->cap) return 0;
    int64_t cap = p->cap ? p->cap : 1024;
    while (cap < need) cap *= 2;
    double *pos = (double *)realloc(p->pos, sizeof(double) * 3 * cap);
    if (!pos) return -1;
    p->pos = pos;
    double *vel = (double *)realloc(p->vel, sizeof(double) * 3 * cap);
    if (!vel) return -1;
    p->vel = vel;
    double *mg = (double *)realloc(p->margin, sizeof(double) * cap);
    if (!mg) return -1;
    p->margin = mg;
    int32_t *cell = (int32_t *)realloc(p->cell, sizeof(int32_t) * cap);
    if (!cell) return -1;
    p->cell = cell;
    int64_t *id = (int64_t *)realloc(p->id, sizeof(int64_t) * cap);
    if (!id) return -1;
    p->id = id;
    p->cap = cap;
    return 0;
}

orc_parts *orc_parts_new(void) { return (orc_parts *)calloc(1, sizeof(orc_parts)); }

void orc_parts_free(orc_parts *p) {
    if (!p) return;
    free(p->pos); free(p->vel); free(p->margin); free(p->cell); free(p->id);
    free(p->rem_id); free(p->rem_margin);
    free(p);
}

int64_t orc_parts_count(const orc_parts *p) { return p->n; }

int64_t orc_parts_removed(const orc_parts *p, int64_t *ids, double *margin) {
    if (ids) memcpy(ids, p->rem_id, sizeof(int64_t) * p->n_rem);
    if (margin) memcpy(margin, p->rem_margin, sizeof(double) * p->n_rem);
    return p->n_rem;
}

/* Append n particles (the OPP_ITERATE_INJECTED range [N, N+n), 1014-1018). */
int orc_parts_append(orc_parts *p, int64_t n, const double *pos, const double *vel,
                     const int32_t *cell, const int64_t *id) {
    if (parts_reserve(p, p->n + n)) return -1;
    memcpy(p->pos + 3 * p->n, pos, sizeof(double) * 3 * n);
    memcpy(p->vel + 3 * p->n, vel, sizeof(double) * 3 * n);
    memcpy(p->cell + p->n, cell, sizeof(int32_t) * n);
    memcpy(p->id + p->n, id, sizeof(int64_t) * n);
    for (int64_t i = 0; i < n; i++) p->margin[p->n + i] = INFINITY;
    p->n += n;
    return 0;
}

void orc_parts_get(const orc_parts *p, double *pos, double *vel, int32_t *cell, int64_t *id,
                   double *margin) {
    if (pos) memcpy(pos, p->pos, sizeof(double) * 3 * p->n);
    if (vel) memcpy(vel, p->vel, sizeof(double) * 3 * p->n);
    if (cell) memcpy(cell, p->cell, sizeof(int32_t) * p->n);
    if (id) memcpy(id, p->id, sizeof(int64_t) * p->n);
    if (margin) memcpy(margin, p->margin, sizeof(double) * p->n);
}

/* ------------------------------------------------------------------------ */
/* One time step                                                             */
/* ------------------------------------------------------------------------ */
typedef struct {
    double c1;      /* (q/m)*dt, computed once on the host (S: push)        */
    double dt;
    double w;       /* macro-particle weight Q_p (Eq. 10, 682-696)          */
    int32_t hcap;   /* H_cap, S4                                             */
    int32_t use_dh; /* 1: overlay seed for every particle; 2: only for those
                       that left their cell (reading S19'')                  */
    int32_t zero_charge;
    int32_t pad;
} orc_params;

typedef struct {
    int64_t n_before, n_injected, n_removed, n_after, total_hops, n_capped;
    int32_t max_hops, pad;
} orc_stats;

/*
 * One Mini-FEM-PIC particle step on an already-injected population:
 *   zero node charge; for each particle in storage order
 *     E = E[cell]                          (start-of-step cell, S6)
 *     v <- v + c1*E ; x <- x + v*dt        (leap-frog, v at half steps, S5)
 *     [DH=1] cell <- overlay seed(x)
 *     [DH=2] if x is not inside cell: cell <- overlay seed(x)
 *     walk -> DONE | REMOVE                (MH)
 *     DONE: Q[c2n[cell][i]] += w*lambda_i  (Eq. 10)
 *   compact: drop REMOVE particles, keep the survivors' order.
 * margin[p] records min_i |lambda_i| of the final evaluation (S15): the
 * barycentric distance to the nearest face, used by parity tests to exclude
 * particles whose cell is decided by rounding.
 */
int orc_step(const orc_mesh *m, orc_parts *p, const orc_params *prm, double *Q, orc_stats *st) {
    if (prm->zero_charge)
        for (int64_t i = 0; i < m->nn; i++) Q[i] = 0.0;
    st->n_before = p->n;
    st->n_injected = 0;
    st->n_removed = 0;
    st->total_hops = 0;
    st->n_capped = 0;
    st->max_hops = 0;
    if (p->rem_cap < p->n) {
        int64_t cap = p->n > 0 ? p->n : 1;
        int64_t *ri = (int64_t *)realloc(p->rem_id, sizeof(int64_t) * cap);
        if (!ri) return -1;
        p->rem_id = ri;
        double *rm = (double *)realloc(p->rem_margin, sizeof(double) * cap);
        if (!rm) return -1;
        p->rem_margin = rm;
        p->rem_cap = cap;
    }
    p->n_rem = 0;
    int64_t out = 0;
    for (int64_t i = 0; i < p->n; i++) {
        double *x = p->pos + 3 * i, *v = p->vel + 3 * i;
        int32_t cell = p->cell[i];
        const double *E = m->ef + 3 * (int64_t)cell;
        for (int k = 0; k < 3; k++) {
            v[k] = v[k] + prm->c1 * E[k];
            x[k] = x[k] + v[k] * prm->dt;
        }
        if (prm->use_dh == 1) {
            cell = dh_seed(m, x, cell);
        } else if (prm->use_dh == 2) {
            /* DESIGN.md reading S19'': only a particle that is no longer in
             * its cell takes the overlay seed ("particles are moved directly
             * to a cell closer to the final destination") */
            double l0[4];
            orc_bary(m, cell, x, l0);
            if (!inside(l0)) cell = dh_seed(m, x, cell);
        }
        double lam[4];
        int32_t fc, hops, capped;
        int status = orc_walk(m, cell, x, 0, prm->hcap, &fc, &hops, lam, &capped);
        double mg = fabs(lam[0]);
        for (int k = 1; k < 4; k++)
            if (fabs(lam[k]) < mg) mg = fabs(lam[k]);
        if (status == ORC_REMOVE) {
            /* exit margin: |lambda| of the face it leaves through */
            int imin = 0;
            for (int k = 1; k < 4; k++)
                if (lam[k] < lam[imin]) imin = k;
            mg = fabs(lam[imin]);
        }
        st->total_hops += hops;
        if (hops > st->max_hops) st->max_hops = hops;
        st->n_capped += capped;
        if (status == ORC_REMOVE) {
            st->n_removed++;
            p->rem_id[p->n_rem] = p->id[i];
            p->rem_margin[p->n_rem] = (p->margin[i] < mg) ? p->margin[i] : mg;
            p->n_rem++;
            continue;
        }
        for (int k = 0; k < 4; k++) Q[m->c2n[4 * (int64_t)fc + k]] += prm->w * lam[k];
        /* stable compaction (survivor keeps its relative order) */
        if (out != i) {
            memcpy(p->pos + 3 * out, x, sizeof(double) * 3);
            memcpy(p->vel + 3 * out, v, sizeof(double) * 3);
            p->id[out] = p->id[i];
        }
        p->cell[out] = fc;
        p->margin[out] = (p->margin[i] < mg) ? p->margin[i] : mg;
        out++;
    }
    p->n = out;
    st->n_after = out;
    return 0;
}
