// octree.cuh -- the paper's own orientation-per-thread schemes on B200
// (SURVEY.md 8(f) NEXT 3): one thread per orientation traverses the octree
// (root + interior nodes + leaves) with Alg. 2 CHECKOCTREE
// (L198-221): pop a node, test it against the tool at this orientation; a
// node that misses is pruned with all its descendants, a leaf that meets the
// tool ends the thread with "collision" (L220-221), an interior node that
// (maybe) meets it pushes its children.  The elementary test is the scheme's
// (L266-273):
//   PBOX       CHECKBOX (exact cylinder-box test, L97) on every popped node;
//   PBOX_AABB  the "optimized PBox": the node's axis-aligned bounding box in
//              the tool frame (after the rotation) against each cylinder's box
//              first, CHECKBOX only when they overlap (L268);
//   PICA       CHECKICA (Alg. 1): the two inaccessible cone angles computed on
//              the fly per node and orientation; certainly blocked / clear
//              decided by the cones, the corner case (between the cones) by
//              CHECKBOX (L156-157);
//   MICA       PICA with the cones of the top S levels memoised by a parallel
//              precomputation (one thread per node, §4.2);
//   AICA       MICA + the corner-case optimisation of §4.3 (L248-256): a node in
//              the band is expanded into its children, which are tested with
//              CHECKICA again; a leaf in the band is expanded into virtual
//              2x2x2 sub-cubes (the leaf is solid, so it meets the tool iff
//              one of them does) down to `vdepth` extra levels, and only then
//              CHECKBOX is the fallback.
// Every scheme is exact (up to the fp32 guards of geometry.cuh, which only
// move decisions into the band that CHECKBOX resolves), so all five give the
// same map as am_compute; they differ only in work -- which is what the
// paper's Table 3 / Fig. 13-18 comparisons measure.
//
// The cone tests (node_cones, ica_decide, leaf_expand) live in geometry.cuh
// beside tool_cones (reading G8: inner cone on the
// monotone-shrunk tool, outer on the true tool, ring voxels beyond the tool
// end) -- the same device functions as the streaming path.
#pragma once
#include "geometry.cuh"

namespace am {

enum { SCHEME_PBOX = 0, SCHEME_PBOX_AABB = 1, SCHEME_PICA = 2, SCHEME_MICA = 3, SCHEME_AICA = 4 };

struct OctParams {
    const float4* __restrict__ box;   // node cube (cx, cy, cz, h); leaves = the uploaded voxels
    const int2* __restrict__ link;    // (first child, child count); count 0 = leaf (solid)
    const float4* __restrict__ memo;  // MICA / AICA: (cin, cout, clo, 1/D) of nodes [0, nmemo)
    long long nmemo;
    float px, py, pz;
    ToolDev tool;
    GridDev grid;
    const float* __restrict__ tab;    // cos phi_i, sin phi_i, cos gamma_j, sin gamma_j
    uint32_t* gam;
    int vdepth;                       // AICA: virtual expansion depth of band leaves
    unsigned long long* stats;        // [nodes popped, CHECKBOX calls, ICA evaluations, max popped per thread]
};

constexpr int kOctStack = 8 * 24;     // 8 children x (max depth 21 + slack)

// The optimized PBox's reject: the rotated cube's axis-aligned box in the
// tool frame (e1, e2, d) against every cylinder's box [-R, R]^2 x [z0, z1].
__device__ __forceinline__ bool aabb_overlaps(float vx, float vy, float vz, float h, float dx, float dy, float dz,
                                              const ToolDev& T) {
    const float adx = fabsf(dx), ady = fabsf(dy), adz = fabsf(dz);
    float e1x, e1y, e1z;
    if (adx <= ady && adx <= adz) { e1x = 0.f; e1y = dz; e1z = -dy; }
    else if (ady <= adz)          { e1x = -dz; e1y = 0.f; e1z = dx; }
    else                          { e1x = dy; e1y = -dx; e1z = 0.f; }
    const float in1 = rsqrtf(e1x * e1x + e1y * e1y + e1z * e1z);
    e1x *= in1; e1y *= in1; e1z *= in1;
    const float e2x = dy * e1z - dz * e1y, e2y = dz * e1x - dx * e1z, e2z = dx * e1y - dy * e1x;
    const float cX = vx * e1x + vy * e1y + vz * e1z, cY = vx * e2x + vy * e2y + vz * e2z;
    const float cZ = vx * dx + vy * dy + vz * dz;
    // half extents of the rotated cube, grown by a relative guard (rounding)
    const float g = 1e-5f * (fabsf(cX) + fabsf(cY) + fabsf(cZ) + 3.f * h);
    const float hX = h * (fabsf(e1x) + fabsf(e1y) + fabsf(e1z)) + g;
    const float hY = h * (fabsf(e2x) + fabsf(e2y) + fabsf(e2z)) + g;
    const float hZ = h * (adx + ady + adz) + g;
    for (int k = 0; k < T.ncyl; ++k) {
        const float R = T.R[k];
        if (fabsf(cX) <= R + hX && fabsf(cY) <= R + hY && cZ + hZ >= T.z0[k] && cZ - hZ <= T.z1[k]) return true;
    }
    return false;
}

// Alg. 2 CHECKOCTREE for orientation (i, j) = one thread.
template <int SCHEME>
__global__ void __launch_bounds__(32) octree_kernel(const __grid_constant__ OctParams P) {
    const int cell = blockIdx.x * blockDim.x + threadIdx.x;
    const GridDev& g = P.grid;
    if (cell >= g.m * g.n) return;
    const int i = cell / g.n, j = cell - i * g.n;
    const float cph = __ldg(P.tab + i), sph = __ldg(P.tab + g.m + i);
    const float dx = sph * __ldg(P.tab + 2 * g.m + j), dy = sph * __ldg(P.tab + 2 * g.m + g.n + j), dz = cph;
    int stack[kOctStack];
    int sp = 0;
    stack[sp++] = 0;  // the root (line 2: the top level)
    unsigned int popped = 0, nbox = 0, nica = 0;
    bool hit = false;
    while (sp > 0 && !hit) {
        const int k = stack[--sp];  // line 4
        ++popped;
        const float4 b = P.box[k];
        const int2 ln = P.link[k];
        const float vx = b.x - P.px, vy = b.y - P.py, vz = b.z - P.pz;
        bool meets;  // line 5: intersected?
        if (SCHEME == SCHEME_PBOX || SCHEME == SCHEME_PBOX_AABB) {
            if (SCHEME == SCHEME_PBOX_AABB && !aabb_overlaps(vx, vy, vz, b.w, dx, dy, dz, P.tool)) {
                meets = false;
            } else {
                ++nbox;
                meets = exact_hit(vx, vy, vz, b.w, dx, dy, dz, P.tool);
            }
        } else {
            float4 c;
            if (SCHEME != SCHEME_PICA && k < P.nmemo) {
                c = P.memo[k];  // memoised (the parallel ICA calculation, §4.2)
            } else {
                ++nica;
                c = node_cones(vx, vy, vz, b.w, P.tool);
            }
            const int dcs = ica_decide(c, vx, vy, vz, dx, dy, dz);
            if (dcs == 2) {  // corner case
                if (SCHEME == SCHEME_AICA) {
                    // §4.3: interior node -> its children are tested with CHECKICA (push);
                    // leaf -> virtual sub-cubes, CHECKBOX only at the bottom
                    meets = ln.y > 0 ? true : leaf_expand(vx, vy, vz, b.w, dx, dy, dz, P.vdepth, P.tool, nbox, nica);
                } else {
                    ++nbox;
                    meets = exact_hit(vx, vy, vz, b.w, dx, dy, dz, P.tool);  // L156-157
                }
            } else {
                meets = dcs == 1;
            }
        }
        if (!meets) continue;        // lines 6-7
        if (ln.y == 0) {             // lines 8-9: a solid leaf meets the tool
            hit = true;
        } else {                     // line 11: push the children
            for (int c = ln.y - 1; c >= 0; --c) stack[sp++] = ln.x + c;
        }
    }
    if (hit) atomicOr(P.gam + i * g.W + (j >> 5), 1u << (j & 31));
    if (P.stats) {
        atomicAdd(P.stats + 0, (unsigned long long)popped);
        atomicAdd(P.stats + 1, (unsigned long long)nbox);
        atomicAdd(P.stats + 2, (unsigned long long)nica);
        atomicMax(P.stats + 3, (unsigned long long)popped);
    }
}

// The parallel ICA calculation (§4.1-4.2): cones of the nodes of the top S
// levels (BFS order: a prefix of the node array), one thread per node.
__global__ void __launch_bounds__(256) ica_memo_kernel(const float4* __restrict__ box, long long n, float px, float py,
                                                       float pz, const ToolDev T, float4* __restrict__ memo) {
    for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < n; k += (long long)gridDim.x * blockDim.x) {
        const float4 b = box[k];
        memo[k] = node_cones(b.x - px, b.y - py, b.z - pz, b.w, T);
    }
}

}  // namespace am
