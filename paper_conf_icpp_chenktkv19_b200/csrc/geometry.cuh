// geometry.cuh -- device geometry of the AICA hot path (fp32, sm_100a).
//
// Three pieces, each citing the passage it implements:
//   * tool_cones():  the two inaccessible cone angles of a voxel (GETTOOLICA for
//     the inscribed radius h and the circumscribed radius sqrt(3) h, PAPER.md
//     Alg. 1; crossed points on the 5 components of every expanded
//     cylinder rectangle, L163-169, L175, Fig. 7), in the cosine domain,
//     with reading G8 (inner cone on the monotone-shrunk tool; ring voxels).
//   * gamma_interval(): one phi-row of a cone as a gamma interval -- Alg. 1
//     L149-155 ("angle <= ica") evaluated for all cells of a row at once.
//   * exact_hit(): the exact cylinder-box test (CHECKBOX, L97, Fig. 4 L82).
//
// Nothing here is shared with oracle/ (independent implementation; the oracle
// uses a clip -> convex-hull formulation in fp64, this file a min-over-edges
// formulation in fp32).
#pragma once
#include <cstdint>

#define AM_MAX_CYL 8

namespace am {

constexpr float kSqrt3 = 1.7320508075688772f;
constexpr float kPi = 3.14159265358979323846f;

struct ToolDev {
    int ncyl;
    float z0[AM_MAX_CYL];   // axial start of cylinder k (z0[0] = 0 at the pivot)
    float z1[AM_MAX_CYL];   // axial end
    float R[AM_MAX_CYL];    // radius
    float Rin[AM_MAX_CYL];  // monotone-shrunk radius min_{j >= k} R_j (reading G8)
    float Rpm[AM_MAX_CYL];  // prefix max max_{j <= k} R_j (cheap outer bound)
    float L;                // total length z1[ncyl-1]
    float rho_max;          // max_k |(z1_k, R_k)|: reach of the tool from the pivot
    // cheap-cone radius as a step function of the reach D + sqrt3 h: R_first up
    // to bp_z[0], then bp_R[k] from bp_z[k] on (only where the prefix max grows;
    // unused entries are +inf)
    int nbp;
    float R_first;
    float bp_z[AM_MAX_CYL];
    float bp_R[AM_MAX_CYL];
    // rounded corners of the expanded rectangles (L175): distance from the pivot of
    // (z0_k | z1_k, R_k | Rin_k) and its reciprocal, [radius set][end][k] (host, fp64)
    float cD[2][2][AM_MAX_CYL];
    float ciD[2][2][AM_MAX_CYL];
};

// An upper bound on the radius of every cylinder that starts within `reach`
// of the pivot: the leading radius up to the first growth point, the tool's
// largest radius beyond it (exact for tools whose radius grows once, like the
// 3-cylinder tip/shank/holder tool).
__device__ __forceinline__ float reach_radius(const ToolDev& T, float reach) {
    float R = T.R_first;
    if (T.bp_z[0] <= reach) R = T.Rpm[AM_MAX_CYL - 1];
    return R;
}

struct GridDev {
    int m, n, W;            // rows (phi), columns (gamma), words per row
    float dphi, inv_dphi;   // pi / m
    float dgam, inv_dgam;   // 2 pi / n
    int rowscan;            // clear map: above this many clear cells, the row-ordered search (AM_OPT_CMAP_ROWSCAN)
    int brute;              // clear map: up to this many, every texel tries every clear cell (AM_OPT_CMAP_BRUTE)
    int cblock;             // clear map: texel block side of the candidate-bounded path (AM_OPT_CMAP_BLOCK)
    float far_cos;          // clear map: blocks whose centre is farther than this (cosine) from every clear
                            // cell store the block-level bound (AM_OPT_CMAP_FAR; -2 = never)
};

// Guards: the inner cone is shrunk and the outer cone
// grown so that every fp32 rounding error lands in the band, which is resolved
// by the exact test.  None of them can change a robust cell; they only add a
// few band cells.
constexpr float kCosGuard = 2e-6f;     // cosine-domain cone guard
constexpr float kRadRel = 4e-6f;       // relative sphere-radius guard (x (D + r))
constexpr float kGamGuard = 4e-6f;     // gamma-domain interval guard (rad)
constexpr float kCellSlack = 1e-4f;    // interval ends, in cells
constexpr float kRowSlack = 1e-4f;     // phi-row range slack (rad); loop bound only
constexpr float kClearSlack = 1e-4f;   // cosine slack of the live voxels' clear-cell check (stream.cuh)

// Blocked-angle candidates of a sphere of radius r whose centre is at distance D
// from the pivot, against ONE cylinder's meridian rectangle [z0, z1] x [0, R]
// expanded by r ("crossed points" of the arc of radius D with
// the expanded rectangle; five components, L175: bottom edge, top edge, side,
// and the two rounded corners).  Every candidate is a point of the expanded
// rectangle, and every boundary crossing is a candidate, so
//   cmin = cos(largest blocked angle)   (2 if nothing is blocked)
//   cmax = cos(smallest blocked angle)  (-2 if nothing is blocked).
__device__ __forceinline__ void ica_cylinder(float D, float D2, float invD, float r, float z0,
                                             float z1, float R, const ToolDev& T, int set, int k,
                                             float& cmin, float& cmax) {
    cmin = 2.f;
    cmax = -2.f;
    if (D + z0 <= r) cmin = -1.f;               // theta = pi lies inside
    if (D >= z0 - r && D <= z1 + r) cmax = 1.f; // theta = 0 lies inside
    const float R2 = R * R;
    {   // bottom edge: a = z0 - r, 0 <= rho <= R
        const float a = z0 - r;
        const float t = D2 - a * a;
        if (t >= 0.f && t <= R2) {
            const float c = a * invD;
            cmin = fminf(cmin, c);
            cmax = fmaxf(cmax, c);
        }
    }
    {   // top edge: a = z1 + r, 0 <= rho <= R
        const float a = z1 + r;
        const float t = D2 - a * a;
        if (t >= 0.f && t <= R2) {
            const float c = a * invD;
            cmin = fminf(cmin, c);
            cmax = fmaxf(cmax, c);
        }
    }
    {   // side: rho = R + r, z0 <= a <= z1 (a >= 0 because z0 >= 0)
        const float s = R + r;
        const float t = D2 - s * s;
        if (t >= 0.f) {
            const float a = sqrtf(t);
            if (a >= z0 && a <= z1) {
                const float c = a * invD;
                cmin = fminf(cmin, c);
                cmax = fmaxf(cmax, c);
            }
        }
    }
#pragma unroll
    for (int e = 0; e < 2; ++e) {  // rounded corners centred (zc, R), radius r
        const float zc = e ? z1 : z0;
        const float Dc = T.cD[set][e][k], iDc = T.ciD[set][e][k];  // |(zc, R)|, 1 / |(zc, R)|
        const float dd = D - Dc;
        if (fabsf(dd) <= r) {
            // arc of radius D meets the corner circle at theta_c +- beta with
            // cos(beta) = (D^2 + Dc^2 - r^2) / (2 D Dc); 1 -+ cos(beta) factored
            // so sin(beta) keeps its relative accuracy near tangency
            const float inv2 = 0.5f * invD * iDc;
            const float omc = (r - dd) * (r + dd) * inv2;               // 1 - cos(beta)
            const float sp = D + Dc;
            const float opc = (sp - r) * (sp + r) * inv2;               // 1 + cos(beta)
            const float cb = 0.5f * (opc - omc);
            const float sb = sqrtf(fmaxf(omc * opc, 0.f));
            const float ct = zc * iDc, st = R * iDc;
            const float s_hi = st * cb + ct * sb;                       // sin(theta_c + beta)
            const float c_hi = (s_hi < 0.f) ? -1.f : (ct * cb - st * sb);
            const float s_lo = st * cb - ct * sb;                       // sin(theta_c - beta)
            const float c_lo = (s_lo < 0.f) ? 1.f : (ct * cb + st * sb);
            cmin = fminf(cmin, c_hi);
            cmax = fmaxf(cmax, c_lo);
        }
    }
}

struct Cones {
    float cin;   // inner cone: cells with cos(theta) >= cin are certainly blocked (> 1: none)
    float cout;  // outer cone: cells with cos(theta) <  cout are certainly clear  (> 1: none)
    float clo;   // ring voxels: cells with cos(theta) >  clo are certainly clear (> 1: no ring)
};

// GETTOOLICA(r = h) on the monotone-shrunk tool and GETTOOLICA(r = sqrt(3) h) on
// the true tool (Alg. 1), guarded.  Reading G8: for the shrunk tool
// (radii non-decreasing away from the pivot) the blocked set is exactly
// [0, ica1] whenever D <= L + r; beyond the tool end (D > L + r) the blocked set
// is a ring [lo, hi], so the inner cone is empty and the outer set is the ring.
__device__ __forceinline__ Cones tool_cones(float D, float h, const ToolDev& T) {
    const float r1 = fmaxf(h - kRadRel * (D + h), 0.f);
    const float r2 = kSqrt3 * h + kRadRel * (D + kSqrt3 * h);
    const float D2 = D * D;
    const float invD = 1.f / D;
    Cones c;
    c.cin = 2.f;
    if (D * (1.f + kRadRel) <= T.L + r1 && r1 > 0.f) {
        float cm = 2.f;
        for (int k = 0; k < T.ncyl; ++k) {
            float a, b;
            ica_cylinder(D, D2, invD, r1, T.z0[k], T.z1[k], T.Rin[k], T, 1, k, a, b);
            cm = fminf(cm, a);
        }
        c.cin = (cm <= 1.f) ? cm + kCosGuard : 2.f;
    }
    float co = 2.f, cx = -2.f;
    for (int k = 0; k < T.ncyl; ++k) {
        float a, b;
        ica_cylinder(D, D2, invD, r2, T.z0[k], T.z1[k], T.R[k], T, 0, k, a, b);
        co = fminf(co, a);
        cx = fmaxf(cx, b);
    }
    c.cout = (co <= 1.f) ? co - kCosGuard : 2.f;
    c.clo = 2.f;
    if (D * (1.f - kRadRel) > T.L + r2 && cx >= -1.f) c.clo = cx + kCosGuard;
    return c;
}

// Inner cone only (GETTOOLICA(r = h) on the monotone-shrunk tool), guarded;
// > 1 when empty.  Used by the coarse levels, which only need certainly-blocked
// cells.
__device__ __forceinline__ float inner_cone(float D, float h, const ToolDev& T) {
    const float r1 = fmaxf(h - kRadRel * (D + h), 0.f);
    if (!(D * (1.f + kRadRel) <= T.L + r1 && r1 > 0.f)) return 2.f;
    const float D2 = D * D;
    const float invD = 1.f / D;
    float cm = 2.f;
    for (int k = 0; k < T.ncyl; ++k) {
        float a, b;
        ica_cylinder(D, D2, invD, r1, T.z0[k], T.z1[k], T.Rin[k], T, 1, k, a, b);
        cm = fminf(cm, a);
    }
    return (cm <= 1.f) ? cm + kCosGuard : 2.f;
}

// acos on [-1, 1] with |error| <= 2e-8 (Abramowitz & Stegun 4.4.46) plus fp32
// rounding (~1e-7): far inside the kGamGuard the interval ends carry.
__device__ __forceinline__ float fast_acos(float x) {
    const float a = fabsf(x);
    float p = -0.0012624911f;
    p = fmaf(p, a, 0.0066700901f);
    p = fmaf(p, a, -0.0170881256f);
    p = fmaf(p, a, 0.0308918810f);
    p = fmaf(p, a, -0.0501743046f);
    p = fmaf(p, a, 0.0889789874f);
    p = fmaf(p, a, -0.2145988016f);
    p = fmaf(p, a, 1.5707963050f);
    const float r = sqrtf(1.f - a) * p;
    return x < 0.f ? kPi - r : r;
}

// Cells j of one phi-row with base + den * cos(gamma_j - gv) >= cthr, as the
// cyclic range [lo, lo + len) (mod n).  grow = +1 widens the interval by the
// guards (outer cone), grow = -1 narrows it (inner cone / ring exclusion).
struct Interval {
    int lo, len;  // len == 0: empty; len == n: full row
};

__device__ __forceinline__ Interval gamma_interval(float cthr, float base, float den, float gv,
                                                   int grow, const GridDev& g) {
    Interval I{0, 0};
    if (cthr > 1.5f) return I;
    float dl;
    if (den <= 1e-20f) {
        if (base < cthr) return I;
        I.len = g.n;
        return I;
    }
    const float x = (cthr - base) / den;
    if (x <= -1.f) { I.len = g.n; return I; }
    if (x > 1.f) return I;
    dl = fast_acos(x) + (grow > 0 ? kGamGuard : -kGamGuard);
    if (dl < 0.f) return I;
    if (dl >= kPi) { I.len = g.n; return I; }
    const float slack = grow > 0 ? kCellSlack : -kCellSlack;
    const float a = (gv - dl) * g.inv_dgam - 0.5f - slack;
    const float b = (gv + dl) * g.inv_dgam - 0.5f + slack;
    int lo = (int)ceilf(a);
    const int hi = (int)floorf(b);
    if (hi < lo) return I;
    int len = hi - lo + 1;
    if (len >= g.n) { I.len = g.n; return I; }
    // gv in (-pi, pi] and dl in [0, pi) keep lo within [-n, n): one wrap suffices
    if (lo < 0) lo += g.n;
    if (lo >= g.n) lo -= g.n;
    I.lo = lo;
    I.len = len;
    return I;
}

// Bits of word w (cells 32w .. 32w+31) covered by the cyclic range I.
__device__ __forceinline__ uint32_t interval_bits(const Interval& I, int w, int n) {
    if (I.len == 0) return 0u;
    const int c0 = w << 5;
    const int c1 = min(c0 + 31, n - 1);
    uint32_t valid = (c1 - c0 == 31) ? 0xffffffffu : ((1u << (c1 - c0 + 1)) - 1u);
    if (I.len >= n) return valid;
    uint32_t bits = 0u;
    // first segment [lo, min(lo+len-1, n-1)], second [0, lo+len-1-n]
    int a = I.lo, b = min(I.lo + I.len - 1, n - 1);
    {
        const int x = max(a, c0), y = min(b, c1);
        if (x <= y) bits |= ((y - x == 31) ? 0xffffffffu : (((1u << (y - x + 1)) - 1u))) << (x - c0);
    }
    const int e = I.lo + I.len - 1 - n;
    if (e >= 0) {
        const int x = c0, y = min(e, c1);
        if (x <= y) bits |= ((y - x == 31) ? 0xffffffffu : (((1u << (y - x + 1)) - 1u))) << (x - c0);
    }
    return bits;
}

// ---------------------------------------------------------------------------
// Exact closed cylinder vs closed box (CHECKBOX, Fig. 4 L82).
//
// Q = box cap slab{z0 <= w.d <= z1}.  The tool cylinder meets the box iff the
// distance rho from the axis line to Q is <= R.  rho^2 is convex on Q; it is 0
// iff the axis segment [z0, z1] d crosses the box; otherwise its minimum is on
// an edge of Q (it is a positive-definite quadratic on every facet that is not
// parallel to d, and constant along d on the others).  The edges of Q are the
// box edges clipped to the slab (decomposition: 12 segments) and, on each cap
// plane, the segments between the crossing points of one box face's edges.
// All geometry is expressed in the cylinder frame (rotation) and the distance
// is taken in the plane normal to d (projection).
// ---------------------------------------------------------------------------

__device__ __forceinline__ float seg_dist2(float ax, float ay, float bx, float by) {
    const float ux = bx - ax, uy = by - ay;
    const float uu = ux * ux + uy * uy;
    float t = 0.f;
    if (uu > 0.f) t = fminf(fmaxf(-(ax * ux + ay * uy) / uu, 0.f), 1.f);
    const float x = fmaf(t, ux, ax), y = fmaf(t, uy, ay);
    return x * x + y * y;
}

// Edge e in 0..11: axis = e >> 2, the other two vertex bits from e & 3.
// Vertex index bits: bit0 = x side, bit1 = y side, bit2 = z side.
__device__ __forceinline__ void edge_vertices(int e, int& a, int& b) {
    const int ax = e >> 2, q = e & 3;
    int v = 0;
    if (ax == 0) v = (q & 1) << 1 | (q >> 1) << 2;  // y, z bits
    if (ax == 1) v = (q & 1) | (q >> 1) << 2;       // x, z bits
    if (ax == 2) v = (q & 1) | (q >> 1) << 1;       // x, y bits
    a = v;
    b = v | (1 << ax);
}

// The test is an OR of 15 sub-tests per cylinder c -- (0) the axis crossing the box, (1..12) box
// edge e clipped to the slab, (13, 14) the cap planes -- so it can be split over the lanes of a
// group: sub-test s = 15 c + k is done by the lane with s % nparts == part (default: all of them,
// one lane).  The OR of the parts is the whole test, value for value.
__device__ __noinline__ bool exact_hit(float vx, float vy, float vz, float h, float dx, float dy,
                                       float dz, const ToolDev& T, int part = 0, int nparts = 1) {
    // frame: e1 = normalize(d x a), a = the world axis least aligned with d; e2 = d x e1
    const float adx = fabsf(dx), ady = fabsf(dy), adz = fabsf(dz);
    float e1x, e1y, e1z;
    if (adx <= ady && adx <= adz) { e1x = 0.f; e1y = dz; e1z = -dy; }      // d x (1,0,0)
    else if (ady <= adz)          { e1x = -dz; e1y = 0.f; e1z = dx; }      // d x (0,1,0)
    else                          { e1x = dy; e1y = -dx; e1z = 0.f; }      // d x (0,0,1)
    const float in1 = rsqrtf(e1x * e1x + e1y * e1y + e1z * e1z);
    e1x *= in1; e1y *= in1; e1z *= in1;
    const float e2x = dy * e1z - dz * e1y, e2y = dz * e1x - dx * e1z, e2z = dx * e1y - dy * e1x;

    // rotated vertices (x, y) in the plane normal to d, z along d
    float X[8], Y[8], Z[8];
    const float cX = vx * e1x + vy * e1y + vz * e1z;
    const float cY = vx * e2x + vy * e2y + vz * e2z;
    const float cZ = vx * dx + vy * dy + vz * dz;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const float sx = (k & 1) ? h : -h, sy = (k & 2) ? h : -h, sz = (k & 4) ? h : -h;
        X[k] = cX + sx * e1x + sy * e1y + sz * e1z;
        Y[k] = cY + sx * e2x + sy * e2y + sz * e2z;
        Z[k] = cZ + sx * dx + sy * dy + sz * dz;
    }
    for (int c = 0; c < T.ncyl; ++c) {
        const int s0 = 15 * c;  // this cylinder's sub-tests s0 .. s0 + 14
        const float z0 = T.z0[c], z1 = T.z1[c], R = T.R[c], R2 = R * R;
        // (0) the axis segment crosses the box: slab test in world coordinates
        if (s0 % nparts == part) {
            float tlo = z0, thi = z1;
            const float dv[3] = {dx, dy, dz}, vv[3] = {vx, vy, vz};
#pragma unroll
            for (int a = 0; a < 3; ++a) {
                if (dv[a] != 0.f) {
                    const float inv = 1.f / dv[a];
                    float t0 = (vv[a] - h) * inv, t1 = (vv[a] + h) * inv;
                    if (t0 > t1) { const float t = t0; t0 = t1; t1 = t; }
                    tlo = fmaxf(tlo, t0);
                    thi = fminf(thi, t1);
                } else if (fabsf(vv[a]) > h) {
                    thi = -1e30f;
                }
            }
            if (tlo <= thi) return true;
        }
        // (1) box edges clipped to the slab
#pragma unroll
        for (int e = 0; e < 12; ++e) {
            if ((s0 + 1 + e) % nparts != part) continue;
            int a, b;
            edge_vertices(e, a, b);
            const float za = Z[a], zb = Z[b];
            float t0, t1;
            if (za == zb) {
                if (za < z0 || za > z1) continue;
                t0 = 0.f; t1 = 1.f;
            } else {
                const float inv = 1.f / (zb - za);
                float ta = (z0 - za) * inv, tb = (z1 - za) * inv;
                t0 = fmaxf(fminf(ta, tb), 0.f);
                t1 = fminf(fmaxf(ta, tb), 1.f);
                if (t0 > t1) continue;
            }
            const float ux = X[b] - X[a], uy = Y[b] - Y[a];
            if (seg_dist2(fmaf(t0, ux, X[a]), fmaf(t0, uy, Y[a]), fmaf(t1, ux, X[a]), fmaf(t1, uy, Y[a])) <= R2)
                return true;
        }
        // (2) on each cap plane, segments between crossing points of one face's edges
        for (int cap = 0; cap < 2; ++cap) {
            if ((s0 + 13 + cap) % nparts != part) continue;
            const float zc = cap ? z1 : z0;
            float PX[12], PY[12];
            bool ok[12];
#pragma unroll
            for (int e = 0; e < 12; ++e) {
                int a, b;
                edge_vertices(e, a, b);
                const float za = Z[a], zb = Z[b];
                ok[e] = (za != zb) && ((za - zc) * (zb - zc) <= 0.f);
                const float t = ok[e] ? (zc - za) / (zb - za) : 0.f;
                PX[e] = fmaf(t, X[b] - X[a], X[a]);
                PY[e] = fmaf(t, Y[b] - Y[a], Y[a]);
            }
#pragma unroll
            for (int f = 0; f < 6; ++f) {
                const int fa = f >> 1, fs = f & 1;
                // the 4 edges of face (fa, fs): edges along the other two axes whose fa-bit == fs
                int ids[4];
                int k = 0;
#pragma unroll
                for (int e = 0; e < 12; ++e) {
                    if ((e >> 2) == fa) continue;
                    int a, b;
                    edge_vertices(e, a, b);
                    if (((a >> fa) & 1) == fs) ids[k++] = e;
                }
#pragma unroll
                for (int p = 0; p < 4; ++p) {
                    if (!ok[ids[p]]) continue;
                    if (PX[ids[p]] * PX[ids[p]] + PY[ids[p]] * PY[ids[p]] <= R2) return true;
#pragma unroll
                    for (int q = p + 1; q < 4; ++q) {
                        if (!ok[ids[q]]) continue;
                        if (seg_dist2(PX[ids[p]], PY[ids[p]], PX[ids[q]], PY[ids[q]]) <= R2) return true;
                    }
                }
            }
        }
    }
    return false;
}

// The same test by a whole warp (warp-uniform call, every lane gets the result): the sub-tests run
// side by side instead of one after the other -- lane k & 7 holds box vertex k, lane e < 12 clips
// edge e to the slab, lanes 16 cap + e put edge e's crossing of cap plane `cap`, and the 2 x 36
// polygon sides between crossings on one face are spread over the lanes -- with the very same
// arithmetic per sub-test as exact_hit, so the OR is the same value for value.  A latency path:
// one test costs a few hundred cycles instead of ~10^4 (exact_hit is ~8K dependent instructions for
// 3 cylinders, and lanes that branch on different sub-tests of one warp run serially).
__device__ __forceinline__ int face_side(int u) {  // (edge p) | (edge q) << 4 of polygon side u < 36
    const unsigned long long w = u < 8    ? 0x9575a8a686a48464ull
                                 : u < 16 ? 0x82908020b9b797b5ull
                                 : u < 24 ? 0xbab3a3b1a1319892ull
                                 : u < 32 ? 0x6232545141504010ull
                                          : 0x76736372ull;
    return (int)((w >> ((u & 7) * 8)) & 0xffull);
}

__device__ __noinline__ bool exact_hit_warp(float vx, float vy, float vz, float h, float dx, float dy, float dz,
                                            const ToolDev& T) {
    const int lane = threadIdx.x & 31;
    const float adx = fabsf(dx), ady = fabsf(dy), adz = fabsf(dz);
    float e1x, e1y, e1z;
    if (adx <= ady && adx <= adz) { e1x = 0.f; e1y = dz; e1z = -dy; }      // d x (1,0,0)
    else if (ady <= adz)          { e1x = -dz; e1y = 0.f; e1z = dx; }      // d x (0,1,0)
    else                          { e1x = dy; e1y = -dx; e1z = 0.f; }      // d x (0,0,1)
    const float in1 = rsqrtf(e1x * e1x + e1y * e1y + e1z * e1z);
    e1x *= in1; e1y *= in1; e1z *= in1;
    const float e2x = dy * e1z - dz * e1y, e2y = dz * e1x - dx * e1z, e2z = dx * e1y - dy * e1x;
    const float cX = vx * e1x + vy * e1y + vz * e1z;
    const float cY = vx * e2x + vy * e2y + vz * e2z;
    const float cZ = vx * dx + vy * dy + vz * dz;
    // vertex k = lane & 7
    const int k = lane & 7;
    const float sx = (k & 1) ? h : -h, sy = (k & 2) ? h : -h, sz = (k & 4) ? h : -h;
    const float Xk = cX + sx * e1x + sy * e1y + sz * e1z;
    const float Yk = cY + sx * e2x + sy * e2y + sz * e2z;
    const float Zk = cZ + sx * dx + sy * dy + sz * dz;
    // edge lanes (e = lane < 12) and cap-crossing lanes (cap = lane >> 4, e = lane & 15 < 12)
    int a, b;
    edge_vertices(lane < 12 ? lane : 0, a, b);
    const float Xa = __shfl_sync(0xffffffffu, Xk, a), Xb = __shfl_sync(0xffffffffu, Xk, b);
    const float Ya = __shfl_sync(0xffffffffu, Yk, a), Yb = __shfl_sync(0xffffffffu, Yk, b);
    const float za = __shfl_sync(0xffffffffu, Zk, a), zb = __shfl_sync(0xffffffffu, Zk, b);
    const int ec = lane & 15;
    int ca, cb;
    edge_vertices(ec < 12 ? ec : 0, ca, cb);
    const float cXa = __shfl_sync(0xffffffffu, Xk, ca), cXb = __shfl_sync(0xffffffffu, Xk, cb);
    const float cYa = __shfl_sync(0xffffffffu, Yk, ca), cYb = __shfl_sync(0xffffffffu, Yk, cb);
    const float cza = __shfl_sync(0xffffffffu, Zk, ca), czb = __shfl_sync(0xffffffffu, Zk, cb);
    for (int c = 0; c < T.ncyl; ++c) {
        const float z0 = T.z0[c], z1 = T.z1[c], R = T.R[c], R2 = R * R;
        bool hit;
        {   // (0) the axis segment crosses the box (every lane, the same values)
            float tlo = z0, thi = z1;
            const float dv[3] = {dx, dy, dz}, vv[3] = {vx, vy, vz};
#pragma unroll
            for (int ax = 0; ax < 3; ++ax) {
                if (dv[ax] != 0.f) {
                    const float inv = 1.f / dv[ax];
                    float t0 = (vv[ax] - h) * inv, t1 = (vv[ax] + h) * inv;
                    if (t0 > t1) { const float t = t0; t0 = t1; t1 = t; }
                    tlo = fmaxf(tlo, t0);
                    thi = fminf(thi, t1);
                } else if (fabsf(vv[ax]) > h) {
                    thi = -1e30f;
                }
            }
            hit = tlo <= thi;
        }
        if (lane < 12) {  // (1) box edge `lane` clipped to the slab
            float t0, t1;
            bool valid;
            if (za == zb) {
                valid = !(za < z0 || za > z1);
                t0 = 0.f; t1 = 1.f;
            } else {
                const float inv = 1.f / (zb - za);
                float ta = (z0 - za) * inv, tb = (z1 - za) * inv;
                t0 = fmaxf(fminf(ta, tb), 0.f);
                t1 = fminf(fmaxf(ta, tb), 1.f);
                valid = !(t0 > t1);
            }
            const float ux = Xb - Xa, uy = Yb - Ya;
            if (valid && seg_dist2(fmaf(t0, ux, Xa), fmaf(t0, uy, Ya), fmaf(t1, ux, Xa), fmaf(t1, uy, Ya)) <= R2)
                hit = true;
        }
        // (2) cap planes: crossing of edge ec with plane zc, then the cross-section's vertices and
        //     the sides between crossings on one face
        const float zc = (lane >> 4) ? z1 : z0;
        const bool ok = ec < 12 && (cza != czb) && ((cza - zc) * (czb - zc) <= 0.f);
        const float t = ok ? (zc - cza) / (czb - cza) : 0.f;
        const float PX = fmaf(t, cXb - cXa, cXa), PY = fmaf(t, cYb - cYa, cYa);
        if (ok && PX * PX + PY * PY <= R2) hit = true;
        const int okm = (int)ok;
#pragma unroll
        for (int u0 = 0; u0 < 72; u0 += 32) {
            const int u = u0 + lane;
            const int cap = u >= 36 ? 1 : 0;
            const int sd = face_side(u < 72 ? u - 36 * cap : 0);
            const int lp = 16 * cap + (sd & 15), lq = 16 * cap + (sd >> 4);
            const float px = __shfl_sync(0xffffffffu, PX, lp), py = __shfl_sync(0xffffffffu, PY, lp);
            const float qx = __shfl_sync(0xffffffffu, PX, lq), qy = __shfl_sync(0xffffffffu, PY, lq);
            const int op = __shfl_sync(0xffffffffu, okm, lp), oq = __shfl_sync(0xffffffffu, okm, lq);
            if (u < 72 && op && oq && seg_dist2(px, py, qx, qy) <= R2) hit = true;
        }
        if (__any_sync(0xffffffffu, hit)) return true;
    }
    return false;
}

// ---------------------------------------------------------------------------
// CHECKICA on whole cubes and the corner-case expansion (Alg. 1, §4.3)
// ---------------------------------------------------------------------------

// Cones of a cube whose centre is v (relative to the pivot) at distance D;
// (cin, cout, clo, 1/D) with 1/D = 0 and cin = -2 ("always meets") when the
// pivot lies in the closed cube (the tool contains the pivot).
__device__ __forceinline__ float4 node_cones(float vx, float vy, float vz, float h, const ToolDev& T) {
    if (fabsf(vx) <= h && fabsf(vy) <= h && fabsf(vz) <= h) return make_float4(-2.f, -2.f, 2.f, 0.f);
    const float D = sqrtf(vx * vx + vy * vy + vz * vz);
    const Cones c = tool_cones(D, h, T);
    return make_float4(c.cin, c.cout, c.clo, 1.f / D);
}

// CHECKICA decision from the cones: 1 = certainly meets (angle <= ica1),
// 0 = certainly misses (angle >= ica2, or inside the ring's hole), 2 = corner case.
__device__ __forceinline__ int ica_decide(float4 c, float vx, float vy, float vz, float dx, float dy, float dz) {
    const float ct = (vx * dx + vy * dy + vz * dz) * c.w;
    if (ct >= c.x) return 1;
    if (c.y > 1.f || ct < c.y || ct > c.z) return 0;
    return 2;
}

// The corner-case optimisation of PAPER.md §4.3 (L248-256) on a leaf: the leaf (solid cube) meets the tool iff one
// of its virtual 2x2x2 sub-cubes does; each is decided by CHECKICA, recursing
// `depth` levels, CHECKBOX at the bottom.
__device__ bool leaf_expand(float vx, float vy, float vz, float h, float dx, float dy, float dz, int depth,
                            const ToolDev& T, unsigned int& nbox, unsigned int& nica) {
    float4 st[8 * 4];
    int lv[8 * 4];
    int sp = 0;
    st[sp] = make_float4(vx, vy, vz, h);
    lv[sp++] = 0;
    while (sp > 0) {
        --sp;
        const float4 c = st[sp];
        const int l = lv[sp];
        if (l > 0) {  // the root of this expansion is already known to be in the band
            ++nica;
            const int dcs = ica_decide(node_cones(c.x, c.y, c.z, c.w, T), c.x, c.y, c.z, dx, dy, dz);
            if (dcs == 1) return true;
            if (dcs == 0) continue;
        }
        if (l >= depth) {
            ++nbox;
            if (exact_hit(c.x, c.y, c.z, c.w, dx, dy, dz, T)) return true;
            continue;
        }
        const float q = 0.5f * c.w;
        for (int k = 0; k < 8; ++k) {
            st[sp] = make_float4(c.x + ((k & 1) ? q : -q), c.y + ((k & 2) ? q : -q), c.z + ((k & 4) ? q : -q), q);
            lv[sp++] = l + 1;
        }
    }
    return false;
}

}  // namespace am
