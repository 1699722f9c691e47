/*
 * scenes/octree.c -- seeded synthetic INPUT generator shared by the CUDA path's
 * tests/bench and the oracle's tests.  It holds none of the method's arithmetic
 * (no cones, no cylinder tests): only analytic signed-distance models and the
 * adaptive-octree leaf rule that turns them into the voxel lists the paper's
 * benchmarks are made of ("adaptive octree", Table 1;
 * recipe in DESIGN.md "Input recipe").
 *
 * Octree rule:  a cell with centre c and half-size h
 *   f(c) >  sqrt(3) h  -> dropped (entirely outside; f is a Lipschitz-1 lower
 *                          bound on the signed distance)
 *   f(c) < -sqrt(3) h  -> full interior leaf (any depth)
 *   otherwise          -> split, or a boundary leaf at max depth.
 * Children are visited in Morton order (bit0 = x, bit1 = y, bit2 = z), so the
 * output list is Morton-sorted.
 *
 * Models (all lengths in mm):
 *   0 SPHERE    radius p[0] at the origin (exact distance)
 *   1 HEAD      union of 4 ellipsoids and 3 capsules fitted to 48.6 x 46.0 x 64.4 (Table 1 "Head")
 *   2 BLADE     hub block 48.9 x 48.9 x 31.1 plus a twisted, tapered thin airfoil
 *               wall (chord 40, span 60, thickness 2.0 -> 0.3)  ("Turbine"-like)
 *   3 IMPELLER  hub disc + 7 main + 7 splitter swept blades, diameter 120, height 60
 *   4 SHELL     hollow sphere: outer radius p[0], inner radius p[1] (enclosing-pivot tests)
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC octree.c -o libscenes.so -lm
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

enum { M_SPHERE = 0, M_HEAD = 1, M_BLADE = 2, M_IMPELLER = 3, M_SHELL = 4 };

/* ---------- signed-distance lower bounds (Lipschitz <= 1) ---------- */

static double ellipsoid(double x, double y, double z, double cx, double cy, double cz,
                        double rx, double ry, double rz) {
    /* (|q| - 1) * r_min with q = (p - c) / r: Lipschitz <= 1, same zero set. */
    double qx = (x - cx) / rx, qy = (y - cy) / ry, qz = (z - cz) / rz;
    double rmin = rx < ry ? (rx < rz ? rx : rz) : (ry < rz ? ry : rz);
    return (sqrt(qx * qx + qy * qy + qz * qz) - 1.0) * rmin;
}

static double sd_box(double x, double y, double z, double cx, double cy, double cz,
                     double hx, double hy, double hz) {
    double qx = fabs(x - cx) - hx, qy = fabs(y - cy) - hy, qz = fabs(z - cz) - hz;
    double ox = qx > 0 ? qx : 0, oy = qy > 0 ? qy : 0, oz = qz > 0 ? qz : 0;
    double outside = sqrt(ox * ox + oy * oy + oz * oz);
    double m = qx > qy ? (qx > qz ? qx : qz) : (qy > qz ? qy : qz);
    double inside = m < 0 ? m : 0;
    return outside + inside;
}

static double capsule(double x, double y, double z, double ax, double ay, double az,
                      double bx, double by, double bz, double r) {
    double px = x - ax, py = y - ay, pz = z - az;
    double ux = bx - ax, uy = by - ay, uz = bz - az;
    double t = (px * ux + py * uy + pz * uz) / (ux * ux + uy * uy + uz * uz);
    t = t < 0 ? 0 : (t > 1 ? 1 : t);
    double dx = px - t * ux, dy = py - t * uy, dz = pz - t * uz;
    return sqrt(dx * dx + dy * dy + dz * dz) - r;
}

static double head_sdf(double x, double y, double z) {
    double f = ellipsoid(x, y, z, 0.0, 0.0, 8.2, 21.0, 21.0, 24.0);           /* cranium */
    double g;
    g = ellipsoid(x, y, z, 0.0, -4.0, -10.0, 17.0, 17.0, 18.0); f = g < f ? g : f; /* face */
    g = capsule(x, y, z, 0.0, -18.0, 0.0, 0.0, -21.5, -7.0, 3.5); f = g < f ? g : f; /* nose */
    g = ellipsoid(x, y, z, 0.0, -9.0, -26.2, 8.0, 8.0, 6.0);    f = g < f ? g : f; /* chin */
    g = capsule(x, y, z, 21.3, 0.0, -5.0, 21.3, 0.0, 5.0, 3.0);   f = g < f ? g : f; /* ears */
    g = capsule(x, y, z, -21.3, 0.0, -5.0, -21.3, 0.0, 5.0, 3.0); f = g < f ? g : f;
    return f;
}

static double blade_sdf(double x, double y, double z) {
    /* hub: 48.9 x 48.9 x 31.1 block, top face at z = 0 */
    double f = sd_box(x, y, z, 0.0, 0.0, -15.55, 24.45, 24.45, 15.55);
    /* airfoil wall: span along z in [0, 60], twisted by 35 degrees over the span,
     * stadium section with semi-chord 20 and half-thickness 1.0 -> 0.15 */
    double zc = z < 0.0 ? 0.0 : (z > 60.0 ? 60.0 : z);
    double s = zc / 60.0;
    double tw = 0.6108652381980153 * s; /* 35 deg */
    double c = cos(tw), sn = sin(tw);
    double u = c * x + sn * y, v = -sn * x + c * y;
    double b = 1.0 - 0.85 * s;          /* half-thickness */
    /* stadium section: distance to the chord segment |u| <= 20 - b, minus b */
    double cu = fabs(u) - (20.0 - b);
    cu = cu > 0 ? cu : 0;
    double sec = sqrt(cu * cu + v * v) - b;
    double cap = fabs(z - 30.0) - 30.0;
    double wall = sec > cap ? sec : cap;
    /* the twist (0.0102 rad/mm at radius <= 20) and taper raise the gradient
     * norm to at most ~1.03: rescale */
    wall /= 1.1;
    return wall < f ? wall : f;
}

static double impeller_sdf(double x, double y, double z) {
    /* hub disc: radius 30, height 12 (z in [0, 12]) plus a central boss */
    double r = sqrt(x * x + y * y);
    double hub = fabs(z - 6.0) - 6.0;
    double hr = r - 30.0;
    double f = hub > hr ? hub : hr;
    double boss = (r - 12.0) > (fabs(z - 30.0) - 30.0) ? (r - 12.0) : (fabs(z - 30.0) - 30.0);
    f = boss < f ? boss : f;
    double th = atan2(y, x);
    /* blades: mid-surface theta = theta_k + 0.9 * (r - 12) / 48 (sweep), thickness 1.2,
     * spanning r in [12, 60]; main blades height 60 -> 30 (tapers with r),
     * splitters start at r = 30 */
    const double TWO_PI = 6.283185307179586;
    for (int k = 0; k < 14; ++k) {
        int splitter = k & 1;
        double thk = TWO_PI * (double)k / 14.0;
        double rin = splitter ? 30.0 : 12.0;
        double sweep = 0.9 * (r - 12.0) / 48.0;
        double d = th - thk - sweep;
        d = d - TWO_PI * floor(d / TWO_PI + 0.5);
        /* distance-like bound to the swept mid-surface; the sweep raises the
         * gradient norm to <= sqrt(1 + (0.9 r / 48)^2) <= 1.45, so rescale */
        double ad = fabs(d);
        double lat = ad < 1.5707963267948966 ? r * sin(ad) : r;
        double wall = (lat - 0.6) / 1.5;
        double hgt = 60.0 - 30.0 * (r - 12.0) / 48.0;
        double zc = fabs(z - 0.5 * hgt) - 0.5 * hgt;
        double rc = fabs(r - 0.5 * (rin + 60.0)) - 0.5 * (60.0 - rin);
        double b = wall;
        if (zc > b) b = zc;
        if (rc > b) b = rc;
        if (b < f) f = b;
    }
    return f;
}

double scene_sdf1(int model, const double* p, double x, double y, double z) {
    switch (model) {
    case M_SPHERE: return sqrt(x * x + y * y + z * z) - p[0];
    case M_HEAD: return head_sdf(x, y, z);
    case M_BLADE: return blade_sdf(x, y, z);
    case M_IMPELLER: return impeller_sdf(x, y, z);
    case M_SHELL: {
        double d = sqrt(x * x + y * y + z * z);
        double a = d - p[0], b = p[1] - d;
        return a > b ? a : b;
    }
    default: return 1e30;
    }
}

/* Evaluate the model's distance bound at n points (xyz interleaved). */
void scene_sdf(int model, const double* params, const double* pts, int64_t n, double* out) {
    for (int64_t i = 0; i < n; ++i)
        out[i] = scene_sdf1(model, params, pts[3 * i], pts[3 * i + 1], pts[3 * i + 2]);
}

/* ---------- adaptive octree ---------- */

typedef struct {
    float* c;    /* 3 per leaf */
    float* h;
    int64_t n, cap;
} leafbuf;

static int push_leaf(leafbuf* b, double cx, double cy, double cz, double h) {
    if (b->n == b->cap) {
        int64_t nc = b->cap ? b->cap * 2 : 4096;
        float* c2 = (float*)realloc(b->c, (size_t)nc * 3 * sizeof(float));
        if (!c2) return -1;
        b->c = c2;
        float* h2 = (float*)realloc(b->h, (size_t)nc * sizeof(float));
        if (!h2) return -1;
        b->h = h2;
        b->cap = nc;
    }
    b->c[3 * b->n] = (float)cx;
    b->c[3 * b->n + 1] = (float)cy;
    b->c[3 * b->n + 2] = (float)cz;
    b->h[b->n] = (float)h;
    b->n++;
    return 0;
}

static const double SQRT3 = 1.7320508075688772;

static int recurse(int model, const double* p, double cx, double cy, double cz, double h,
                   int depth, int max_depth, leafbuf* b) {
    double f = scene_sdf1(model, p, cx, cy, cz);
    if (f > SQRT3 * h) return 0;
    if (f < -SQRT3 * h || depth == max_depth) return push_leaf(b, cx, cy, cz, h);
    double q = 0.5 * h;
    for (int k = 0; k < 8; ++k) {
        double x = cx + ((k & 1) ? q : -q);
        double y = cy + ((k & 2) ? q : -q);
        double z = cz + ((k & 4) ? q : -q);
        if (recurse(model, p, x, y, z, q, depth + 1, max_depth, b)) return -1;
    }
    return 0;
}

/* task = a cell at depth `split` (or a shallower leaf) in Morton order */
typedef struct { double cx, cy, cz, h; int depth; int is_leaf; } task;

static int collect(int model, const double* p, double cx, double cy, double cz, double h, int depth,
                   int split, int max_depth, task** ts, int64_t* nt, int64_t* capt) {
    double f = scene_sdf1(model, p, cx, cy, cz);
    if (f > SQRT3 * h) return 0;
    int leaf = (f < -SQRT3 * h || depth == max_depth);
    if (leaf || depth == split) {
        if (*nt == *capt) {
            int64_t nc = *capt ? *capt * 2 : 1024;
            task* t2 = (task*)realloc(*ts, (size_t)nc * sizeof(task));
            if (!t2) return -1;
            *ts = t2;
            *capt = nc;
        }
        task t = {cx, cy, cz, h, depth, leaf};
        (*ts)[(*nt)++] = t;
        return 0;
    }
    double q = 0.5 * h;
    for (int k = 0; k < 8; ++k) {
        double x = cx + ((k & 1) ? q : -q);
        double y = cy + ((k & 2) ? q : -q);
        double z = cz + ((k & 4) ? q : -q);
        if (collect(model, p, x, y, z, q, depth + 1, split, max_depth, ts, nt, capt)) return -1;
    }
    return 0;
}

/*
 * Generate the leaves of the adaptive octree of `model` in the root cube
 * [lo, lo+size]^3 down to `max_depth`.  Leaves are written Morton-ordered into
 * freshly malloc'ed arrays returned through *out_c (N*3 floats) and *out_h (N
 * floats); release them with scene_free().  Returns 0, or -1 on allocation
 * failure.
 */
int scene_octree(int model, const double* params, const double lo[3], double size, int max_depth,
                 float** out_c, float** out_h, int64_t* out_n) {
    double h0 = 0.5 * size;
    double cx = lo[0] + h0, cy = lo[1] + h0, cz = lo[2] + h0;
    int split = max_depth < 4 ? max_depth : 4;
    task* ts = NULL;
    int64_t nt = 0, capt = 0;
    if (collect(model, params, cx, cy, cz, h0, 0, split, max_depth, &ts, &nt, &capt)) {
        free(ts);
        return -1;
    }
    leafbuf* bufs = (leafbuf*)calloc((size_t)(nt > 0 ? nt : 1), sizeof(leafbuf));
    int err = 0;
#pragma omp parallel for schedule(dynamic, 1) reduction(| : err)
    for (int64_t i = 0; i < nt; ++i) {
        task t = ts[i];
        if (t.is_leaf)
            err |= push_leaf(&bufs[i], t.cx, t.cy, t.cz, t.h) != 0;
        else
            err |= recurse(model, params, t.cx, t.cy, t.cz, t.h, t.depth, max_depth, &bufs[i]) != 0;
    }
    int64_t total = 0;
    for (int64_t i = 0; i < nt; ++i) total += bufs[i].n;
    float* C = NULL;
    float* H = NULL;
    if (!err) {
        C = (float*)malloc((size_t)(total > 0 ? total : 1) * 3 * sizeof(float));
        H = (float*)malloc((size_t)(total > 0 ? total : 1) * sizeof(float));
        if (!C || !H) err = 1;
    }
    int64_t off = 0;
    for (int64_t i = 0; i < nt; ++i) {
        if (!err && bufs[i].n) {
            memcpy(C + 3 * off, bufs[i].c, (size_t)bufs[i].n * 3 * sizeof(float));
            memcpy(H + off, bufs[i].h, (size_t)bufs[i].n * sizeof(float));
            off += bufs[i].n;
        }
        free(bufs[i].c);
        free(bufs[i].h);
    }
    free(bufs);
    free(ts);
    if (err) {
        free(C);
        free(H);
        return -1;
    }
    *out_c = C;
    *out_h = H;
    *out_n = total;
    return 0;
}

void scene_free(void* p) { free(p); }
