/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, fp64 CPU oracle for the accessibility map (AM).  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this library.  It shares no code with the CUDA path
 * (paper_conf_icpp_chenktkv19_b200/csrc) and never reads its results.
 *
 * What it computes is the plain DEFINITION of the AM, not the AICA algorithm:
 *
 *   AM[i][j] = 1  <=>  some voxel box B intersects the tool T(d_ij)
 *
 * (problem statement PAPER.md L86-88, Fig. 2 L60 "a black point indicates a
 * collision", L173 "any collision could damage the target part").  The tool is
 * the union of N_c coaxial closed solid cylinders fixed at the pivot (L56,
 * L73, L88, L311); cylinder k spans axial [z_k, z_k + H_k] with z_0 = 0 and has
 * radius R_k (readings G3/G4).  Orientation (phi_i, gamma_j) are cell centres
 * phi_i = (i + 1/2) pi / m, gamma_j = (j + 1/2) 2 pi / n (reading G1, L56, L60),
 * d = (sin phi cos gamma, sin phi sin gamma, cos phi).
 *
 * Per (voxel, cylinder) the exact test mirrors the paper's CHECKBOX steps
 * (L97, Fig. 4 L82): DECOMPOSITION of the box into its 12 edges, ROTATION of
 * the box into the cylinder frame (e1, e2, d), PROJECTION onto the plane
 * normal to the axis after clipping each edge to the cylinder's axial slab.
 * The clipped endpoints are exactly the vertices of B cap slab (the two slab
 * planes are parallel), so
 *
 *     hit  <=>  slab cap B != empty  and  dist(0, conv(projected points)) <= R.
 *
 * 3-state margin (reading G10, north_star "1e-5 rad band"): with
 * eps = delta (|c - p| + sqrt(3) h), a pair is ROBUST-HIT if the exact test
 * hits the deflated tool (R - eps, [z + eps, z + H - eps]) and ROBUST-MISS if
 * it misses the inflated tool (R + eps, [z - eps, z + H + eps]).  Rotating the
 * tool by <= delta about the pivot moves every point within |c-p| + sqrt(3)h of
 * the pivot by <= eps, so robust decisions survive any such rotation.  Cell
 * state: 2 if any voxel is robust-hit, else 0 if every voxel is robust-miss,
 * else 1 (band; either GPU value is accepted there).
 *
 * Optional exact-safe shortcuts (bit-identical to the plain path, checked by
 * tests): the inscribed ball (radius h) of B meeting the deflated cylinder
 * implies robust-hit; the circumscribed ball (sqrt(3) h) missing the inflated
 * cylinder implies robust-miss.  Both are 2-D meridian distances
 * (Fig. 6-7: a sphere is rotation-invariant).
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC oracle.c -o liboracle.so -lm
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define MAXC 16

typedef struct { double x, y; } P2;

/* Orthonormal frame (e1, e2, d): e1 = normalize(d x a) where a is the world
 * axis least aligned with d, e2 = d x e1. */
static void make_frame(const double d[3], double e1[3], double e2[3]) {
    double ax = fabs(d[0]), ay = fabs(d[1]), az = fabs(d[2]);
    double a[3] = {0, 0, 0};
    if (ax <= ay && ax <= az) a[0] = 1; else if (ay <= az) a[1] = 1; else a[2] = 1;
    double c[3] = {d[1] * a[2] - d[2] * a[1], d[2] * a[0] - d[0] * a[2], d[0] * a[1] - d[1] * a[0]};
    double nc = sqrt(c[0] * c[0] + c[1] * c[1] + c[2] * c[2]);
    e1[0] = c[0] / nc; e1[1] = c[1] / nc; e1[2] = c[2] / nc;
    e2[0] = d[1] * e1[2] - d[2] * e1[1];
    e2[1] = d[2] * e1[0] - d[0] * e1[2];
    e2[2] = d[0] * e1[1] - d[1] * e1[0];
}

static double cross2(P2 o, P2 a, P2 b) { return (a.x - o.x) * (b.y - o.y) - (a.y - o.y) * (b.x - o.x); }

static int cmp_p2(const void* A, const void* B) {
    const P2* a = (const P2*)A;
    const P2* b = (const P2*)B;
    if (a->x < b->x) return -1;
    if (a->x > b->x) return 1;
    if (a->y < b->y) return -1;
    if (a->y > b->y) return 1;
    return 0;
}

/* Andrew's monotone chain; returns hull size, hull counter-clockwise in H. */
static int convex_hull(P2* pts, int n, P2* H) {
    qsort(pts, (size_t)n, sizeof(P2), cmp_p2);
    int k = 0;
    for (int i = 0; i < n; ++i) {
        while (k >= 2 && cross2(H[k - 2], H[k - 1], pts[i]) <= 0) k--;
        H[k++] = pts[i];
    }
    for (int i = n - 2, t = k + 1; i >= 0; --i) {
        while (k >= t && cross2(H[k - 2], H[k - 1], pts[i]) <= 0) k--;
        H[k++] = pts[i];
    }
    if (k > 1) k--; /* last point repeats the first */
    return k;
}

static double seg_dist2_origin(P2 a, P2 b) {
    double ux = b.x - a.x, uy = b.y - a.y;
    double uu = ux * ux + uy * uy;
    double t = 0.0;
    if (uu > 0.0) {
        t = -(a.x * ux + a.y * uy) / uu;
        if (t < 0.0) t = 0.0;
        if (t > 1.0) t = 1.0;
    }
    double x = a.x + t * ux, y = a.y + t * uy;
    return x * x + y * y;
}

/*
 * Distance, in the plane normal to d, from the axis line through the pivot to
 * the polytope B cap {z0 <= w.d <= z1}, where B is the cube of half size h
 * centred at v (v = voxel centre - pivot).  Returns -1 when the slab misses
 * the cube.  (CHECKBOX decomposition/rotation/projection.)
 */
double oracle_axis_dist(const double v[3], double h, const double d[3], double z0, double z1) {
    double e1[3], e2[3];
    make_frame(d, e1, e2);
    double X[8], Y[8], Z[8];
    for (int k = 0; k < 8; ++k) {
        double w[3] = {v[0] + ((k & 1) ? h : -h), v[1] + ((k & 2) ? h : -h), v[2] + ((k & 4) ? h : -h)};
        X[k] = w[0] * e1[0] + w[1] * e1[1] + w[2] * e1[2];
        Y[k] = w[0] * e2[0] + w[1] * e2[1] + w[2] * e2[2];
        Z[k] = w[0] * d[0] + w[1] * d[1] + w[2] * d[2];
    }
    P2 pts[24];
    int np = 0;
    /* the 12 edges: vertex pairs differing in exactly one coordinate bit */
    for (int a = 0; a < 8; ++a) {
        for (int bit = 1; bit < 8; bit <<= 1) {
            if (a & bit) continue;
            int b = a | bit;
            double za = Z[a], zb = Z[b];
            double t0, t1;
            if (za == zb) {
                if (za < z0 || za > z1) continue;
                t0 = 0.0; t1 = 1.0;
            } else {
                double ta = (z0 - za) / (zb - za), tb = (z1 - za) / (zb - za);
                t0 = ta < tb ? ta : tb;
                t1 = ta < tb ? tb : ta;
                if (t0 < 0.0) t0 = 0.0;
                if (t1 > 1.0) t1 = 1.0;
                if (t0 > t1) continue;
            }
            P2 p0 = {X[a] + t0 * (X[b] - X[a]), Y[a] + t0 * (Y[b] - Y[a])};
            P2 p1 = {X[a] + t1 * (X[b] - X[a]), Y[a] + t1 * (Y[b] - Y[a])};
            pts[np++] = p0;
            pts[np++] = p1;
        }
    }
    if (np == 0) return -1.0;
    P2 H[26];
    int nh = convex_hull(pts, np, H);
    if (nh == 1) return sqrt(H[0].x * H[0].x + H[0].y * H[0].y);
    if (nh == 2) return sqrt(seg_dist2_origin(H[0], H[1]));
    int inside = 1;
    double best = INFINITY;
    P2 o = {0.0, 0.0};
    for (int i = 0; i < nh; ++i) {
        P2 a = H[i], b = H[(i + 1) % nh];
        if (cross2(a, b, o) < 0.0) inside = 0;
        double d2 = seg_dist2_origin(a, b);
        if (d2 < best) best = d2;
    }
    if (inside) return 0.0;
    return sqrt(best);
}

/* Exact closed-cylinder vs closed-box test (one cylinder). */
int oracle_box_cyl_hit(const double v[3], double h, const double d[3], double z0, double z1, double R) {
    if (z0 > z1 || R < 0.0) return 0;
    double dist = oracle_axis_dist(v, h, d, z0, z1);
    return dist >= 0.0 && dist <= R;
}

/* 2-D meridian distance from (a, rho) to the rectangle [z0, z1] x [0, R]. */
static double meridian_dist(double a, double rho, double z0, double z1, double R) {
    double da = a < z0 ? z0 - a : (a > z1 ? a - z1 : 0.0);
    double dr = rho > R ? rho - R : 0.0;
    return sqrt(da * da + dr * dr);
}

/*
 * 3-state classification of one (voxel, orientation) pair against the whole
 * tool: 2 robust-hit, 1 band, 0 robust-miss (see header).
 */
int oracle_pair_state(const double v[3], double h, const double d[3], const double* R,
                      const double* H, int ncyl, double delta, int shortcuts) {
    double D = sqrt(v[0] * v[0] + v[1] * v[1] + v[2] * v[2]);
    double eps = delta * (D + 1.7320508075688772 * h);
    double a = v[0] * d[0] + v[1] * d[1] + v[2] * d[2];
    double px = v[0] - a * d[0], py = v[1] - a * d[1], pz = v[2] - a * d[2];
    double rho = sqrt(px * px + py * py + pz * pz);
    int band = 0;
    double z = 0.0;
    for (int k = 0; k < ncyl; ++k) {
        double z0 = z, z1 = z + H[k];
        z = z1;
        if (shortcuts) {
            /* circumscribed ball misses the inflated cylinder -> robust-miss for k */
            if (meridian_dist(a, rho, z0 - eps, z1 + eps, R[k] + eps) > 1.7320508075688772 * h) continue;
            /* inscribed ball meets the deflated cylinder -> robust-hit */
            if (z0 + eps <= z1 - eps && R[k] - eps >= 0.0 &&
                meridian_dist(a, rho, z0 + eps, z1 - eps, R[k] - eps) <= h)
                return 2;
        }
        if (oracle_box_cyl_hit(v, h, d, z0 + eps, z1 - eps, R[k] - eps)) return 2;
        if (oracle_box_cyl_hit(v, h, d, z0 - eps, z1 + eps, R[k] + eps)) band = 1;
    }
    return band;
}

static void cell_dir(int i, int j, int m, int n, double d[3]) {
    const double PI = 3.14159265358979323846;
    double phi = (i + 0.5) * PI / m;
    double gam = (j + 0.5) * 2.0 * PI / n;
    d[0] = sin(phi) * cos(gam);
    d[1] = sin(phi) * sin(gam);
    d[2] = cos(phi);
}

/* Direction of AM cell (i, j) (reading G1). */
void oracle_cell_dir(int i, int j, int m, int n, double* d) { cell_dir(i, j, m, n, d); }

static int cell_state(const float* centers, const float* halfs, int64_t N, const double* R,
                      const double* H, int ncyl, const double p[3], const double d[3],
                      double delta, int shortcuts) {
    int band = 0;
    for (int64_t q = 0; q < N; ++q) {
        double v[3] = {(double)centers[3 * q] - p[0], (double)centers[3 * q + 1] - p[1],
                       (double)centers[3 * q + 2] - p[2]};
        int s = oracle_pair_state(v, (double)halfs[q], d, R, H, ncyl, delta, shortcuts);
        if (s == 2) return 2;
        if (s == 1) band = 1;
    }
    return band;
}

/*
 * 3-state AM for `ncells` listed cells (cells[k] = i * n + j), or for every
 * cell when cells == NULL (then ncells must be m * n).  states[k] in {0,1,2}.
 * Inputs are the float32 values the GPU sees, widened to double.
 * nthreads <= 0 uses all OpenMP threads.  Returns the thread count used.
 */
int oracle_am_cells(const float* centers, const float* halfs, int64_t N, const float* radii,
                    const float* heights, int ncyl, const float* pivot, int m, int n,
                    const int64_t* cells, int64_t ncells, double delta, int shortcuts,
                    int nthreads, uint8_t* states) {
    double R[MAXC], H[MAXC];
    if (ncyl > MAXC) return -1;
    for (int k = 0; k < ncyl; ++k) { R[k] = radii[k]; H[k] = heights[k]; }
    double p[3] = {pivot[0], pivot[1], pivot[2]};
    int used = 1;
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#endif
#pragma omp parallel
    {
#ifdef _OPENMP
#pragma omp single
        used = omp_get_num_threads();
#endif
#pragma omp for schedule(dynamic, 1)
        for (int64_t k = 0; k < ncells; ++k) {
            int64_t c = cells ? cells[k] : k;
            int i = (int)(c / n), j = (int)(c % n);
            double d[3];
            cell_dir(i, j, m, n, d);
            states[k] = (uint8_t)cell_state(centers, halfs, N, R, H, ncyl, p, d, delta, shortcuts);
        }
    }
    return used;
}
