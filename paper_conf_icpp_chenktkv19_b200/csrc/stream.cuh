// stream.cuh -- the voxel-streaming AICA kernels.
//
// The full stream is split in two launches so the part that touches every
// voxel stays lean:
//
// filter_kernel (a1, a2, cheap cones; every voxel): coalesced 16-byte float4
//   loads (4 independent LDG.128 per thread in flight, streaming cache hint),
//   then an exact-safe FILTER per voxel: reach cull, then a cheap outer cone --
//   a sphere of radius sqrt(3) h at distance D only touches cylinders starting
//   within D + sqrt(3) h, of radius at most Reff, so its blocked directions
//   satisfy sin(theta) <= (Reff + sqrt3 h) / D, and none lies more than r2 behind
//   the tool's end face at the pivot -- against the clear-direction map
//   (kernels.cuh clear_map_kernel).  A voxel whose cheap cone holds no
//   still-clear cell cannot change the AM and is dropped after ~60
//   instructions; the survivors ("live") are appended to a global list with one
//   warp-aggregated atomic.
//
// live_kernel (a3-a6; the live voxels only, ~0.1-1 %): one voxel per thread,
//   the paper's two ICA cones (Alg. 1) checked against the map once
//   more, then rasterised row by row into the CTA's shared AM; band cells are
//   deferred to the global band queue; the shared AM is OR-ed into the global
//   AM at the end (a7).
//
// coarse_kernel (levels 0/1, the largest voxels): one warp per voxel, phi-rows
//   across lanes, inner cones only -- these few voxels have cones spanning most
//   rows, so row parallelism is what they need.
#pragma once
#include "kernels.cuh"

namespace am {

constexpr int kWarps = kThreads / 32;
constexpr int kLiveBlocksPerSM = 4;
static_assert(sizeof(StreamParams) % 4 == 0 && sizeof(StreamParams) / 4 <= kThreads,
              "StreamParams is copied to shared memory one word per thread");

__device__ __forceinline__ float rcp_approx(float x) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}

enum { F_DROP = 0, F_LIVE = 1, F_CULLED = 2 };

__device__ __forceinline__ int texel_of(float vx, float vy, float vz, int T);

// a2 + cheap cone vs clear-direction map (p.cmap is never null: before any map
// is built it is the all-clear map).  The map stores V = U |U|, where U bounds
// from above the cosine of the angle from any direction of the texel to the
// nearest still-clear cell; V is monotone in U, so U < x <=> V < x |x|.
// F_LIVE when the voxel may still change the AM, F_CULLED beyond reach,
// F_DROP otherwise.  A voxel holding the pivot blocks every orientation: it
// fills `am` (shared or global) directly.
__device__ __forceinline__ int fast_filter(const StreamParams& p, float4 q, uint32_t* am) {
    const float vx = q.x - p.px, vy = q.y - p.py, vz = q.z - p.pz, h = q.w;
    const float D2 = fmaf(vx, vx, fmaf(vy, vy, vz * vz));
    const float r2 = kSqrt3 * h;
    if (D2 <= 3.0001f * h * h) {
        if (fabsf(vx) <= h && fabsf(vy) <= h && fabsf(vz) <= h) {
            fill_all(p, am);
            return F_DROP;
        }
        return F_LIVE;
    }
    const float invD = rsqrtf(D2);
    const float D = D2 * invD;
    if (p.may_cull && D - r2 > p.cull_dist) return F_CULLED;
    const float Reff = reach_radius(p.tool, (D + r2) * (1.f + kRadRel));
    // drop when cos(cheap cone) > U.  Far voxels (s < 1): sin(theta) <= s, so
    // cos(cone) = sqrt(1 - s^2).  Near voxels: the tool has nothing behind the
    // plane of its end face at the pivot, so a blocked direction keeps the
    // sphere centre within r2 of that plane: cos(cone) = -c with c = r2 / D.
    const float s = fmaf((Reff + r2) * invD, 1.f + 1.6e-5f, 1e-6f);
    const float c = fmaf(r2 * invD, 1.f + 1.6e-5f, 1e-6f);
    const float thr = (s < 1.f) ? fmaf(-s, s, 1.f) : -c * c;
    return __ldg(p.cmap + texel_of(vx, vy, vz, p.cmapT)) < thr ? F_DROP : F_LIVE;
}

// Cube-map texel of v (cube_texel of kernels.cuh with an approximate
// reciprocal; ties between axes may pick either face, and the texel radii
// carry 2e-5 rad of slack for rounding at texel edges).
__device__ __forceinline__ int texel_of(float vx, float vy, float vz, int T) {
    const float ax = fabsf(vx), ay = fabsf(vy), az = fabsf(vz);
    const float a = fmaxf(ax, fmaxf(ay, az));
    const bool xm = ax == a;
    const bool ym = !xm && ay == a;
    const float u = xm ? vy : vx;
    const float w = (xm || ym) ? vz : vy;
    const float maj = xm ? vx : (ym ? vy : vz);
    const int face = (xm ? 0 : (ym ? 2 : 4)) + (maj < 0.f);
    const float hs = 0.5f * (float)T;
    const float sc = hs * rcp_approx(a);
    const int iu = min(T - 1, max(0, __float2int_rz(fmaf(u, sc, hs))));
    const int iw = min(T - 1, max(0, __float2int_rz(fmaf(w, sc, hs))));
    return (face * T + iw) * T + iu;
}

// a3-a6 for one live voxel: both cones, rasterised row by row, band deferred.
// COARSE (level 1 of the clear-direction map) rasterises the inner cone only:
// the map needs certainly-blocked cells, and every coarse voxel is streamed
// again, with its band, by the full stream.
template <bool COARSE>
__device__ __noinline__ void process_live(const StreamParams& p, unsigned int vidx, float4 q, uint32_t* sAM,
                                          const uint32_t* sRowFull, const float* sCos, const float* sSin,
                                          Counters cnt) {
    const ToolDev& T = p.tool;
    const GridDev& g = p.grid;
    const float vx = q.x - p.px, vy = q.y - p.py, vz = q.z - p.pz, h = q.w;
    const float D2 = vx * vx + vy * vy + vz * vz;
    const float D = sqrtf(D2);
    if (D <= kSqrt3 * h && fabsf(vx) <= h && fabsf(vy) <= h && fabsf(vz) <= h) return;  // filled already
    const float rxy = sqrtf(vx * vx + vy * vy);
    const float phv = atan2f(rxy, vz);
    // a4: the two cones (GETTOOLICA twice, Alg. 1)
    atomicAdd(cnt.c + CT_LIVE, 1u);
    Cones c;
    if (COARSE) {
        c.cin = c.cout = inner_cone(D, h, T);
        c.clo = 2.f;
    } else {
        c = tool_cones(D, h, T);
    }
    if (c.cout > 1.f) return;
    // the exact outer cone against the clear-direction map: no clear cell
    // within it means this voxel cannot change the map
    if (__ldg(p.cmap + texel_of(vx, vy, vz, p.cmapT)) < c.cout * fabsf(c.cout)) return;
    const float ao = acosf(fmaxf(c.cout, -1.f));
    const int i0 = max(0, (int)ceilf((phv - ao - kRowSlack) * g.inv_dphi - 0.5f));
    const int i1 = min(g.m - 1, (int)floorf((phv + ao + kRowSlack) * g.inv_dphi - 0.5f));
    if (i0 > i1 || rows_all_full(sRowFull, i0, i1)) return;
    const float invD = 1.f / D;
    const float cphv = vz * invD, sphv = rxy * invD;
    const float gv = atan2f(vy, vx);
    const int W = g.W;
    unsigned int rows = 0;
    // a5: rasterise row by row (Alg. 1 L149-155 for all cells of a row at once)
    for (int i = i0; i <= i1; ++i) {
        if ((ld_vol_shared(sRowFull + (i >> 5)) >> (i & 31)) & 1u) continue;
        const float base = sCos[i] * cphv, den = sSin[i] * sphv;
        if (COARSE) {
            const Interval In = gamma_interval(c.cin, base, den, gv, -1, g);
            if (In.len == 0) continue;
            ++rows;
            for (int w = 0; w < W; ++w) {
                const uint32_t ib = interval_bits(In, w, g.n);
                uint32_t* wp = sAM + i * W + w;
                if (ib & ~ld_vol_shared(wp)) atomicOr(wp, ib);
            }
            continue;
        }
        const Interval O = gamma_interval(c.cout, base, den, gv, +1, g);
        if (O.len == 0) continue;
        ++rows;
        const Interval In = gamma_interval(c.cin, base, den, gv, -1, g);
        const Interval X = gamma_interval(c.clo, base, den, gv, -1, g);
        for (int w = 0; w < W; ++w) {
            uint32_t ob = interval_bits(O, w, g.n);
            if (!ob) continue;
            const uint32_t xb = interval_bits(X, w, g.n);
            const uint32_t ib = interval_bits(In, w, g.n) & ~xb;
            ob &= ~xb;
            uint32_t* wp = sAM + i * W + w;
            uint32_t cur = ld_vol_shared(wp);
            if (ib & ~cur) {
                atomicOr(wp, ib);
                cur |= ib;
            }
            uint32_t band = ob & ~ib & ~cur;
            while (band) {
                const int b = __ffs(band) - 1;
                band &= band - 1u;
                push_band(p, sAM, vidx, q, i * g.n + (w << 5) + b, wp, 1u << b, cnt);
            }
        }
    }
    if (rows) atomicAdd(cnt.c + CT_ROWS, rows);
}


// Dynamic shared memory of live_kernel for an m x n grid.
__host__ __device__ inline size_t live_smem_bytes(int m, int W) {
    return (size_t)(m * W + ((m + 31) >> 5)) * sizeof(uint32_t) + (size_t)2 * m * sizeof(float);
}

// Append the live voxels among one warp-row of 32 to the global live list.
__device__ __forceinline__ void append_live(const StreamParams& p, bool live, unsigned int idx,
                                            unsigned int& npassed) {
    const unsigned int mlive = __ballot_sync(0xffffffffu, live);
    if (mlive) {
        const int lane = threadIdx.x & 31;
        npassed += __popc(mlive);
        unsigned int pos = 0;
        const int leader = __ffs(mlive) - 1;
        if (lane == leader) pos = atomicAdd(p.live_count, (unsigned int)__popc(mlive));
        pos = __shfl_sync(0xffffffffu, pos, leader) + __popc(mlive & ((1u << lane) - 1u));
        if (live) p.live_idx[pos] = idx;
    }
}

// a1-a2 + cheap cones over vox[0, N): live indices go to p.live_idx.  Full
// tiles of kTile voxels take the unguarded path (kVPT independent LDG.128 per
// thread, streaming cache hint); the ragged last tile is guarded.
__global__ void __launch_bounds__(kThreads) filter_kernel(const __grid_constant__ StreamParams p) {
    __shared__ unsigned int sCulled, sPassed;
    if (threadIdx.x == 0) sCulled = sPassed = 0u;
    __syncthreads();
    unsigned int nculled = 0, npassed = 0;
    const unsigned int nfull = (unsigned int)(p.N / kTile);
    for (unsigned int t = blockIdx.x; t < nfull; t += gridDim.x) {
        const unsigned int base = t * kTile + threadIdx.x;
        const float4* src = p.vox + base;
        float4 q[kVPT];
#pragma unroll
        for (int k = 0; k < kVPT; ++k) q[k] = __ldcs(src + k * kThreads);
        int f[kVPT];
#pragma unroll
        for (int k = 0; k < kVPT; ++k) f[k] = fast_filter(p, q[k], p.gam);
#pragma unroll
        for (int k = 0; k < kVPT; ++k) {
            nculled += f[k] >> 1;
            append_live(p, f[k] == F_LIVE, base + k * kThreads, npassed);
        }
    }
    if (blockIdx.x == nfull % gridDim.x && (long long)nfull * kTile < p.N) {  // ragged tail
        const unsigned int base = nfull * kTile + threadIdx.x;
#pragma unroll
        for (int k = 0; k < kVPT; ++k) {
            const unsigned int idx = base + k * kThreads;
            const int f = idx < p.N ? fast_filter(p, p.vox[idx], p.gam) : F_DROP;
            nculled += f >> 1;
            append_live(p, f == F_LIVE, idx, npassed);
        }
    }
    if ((threadIdx.x & 31) == 0) atomicAdd(&sPassed, npassed);
    if (nculled) atomicAdd(&sCulled, nculled);
    __syncthreads();
    if (threadIdx.x == 0) {
        atomicAdd(p.stats + ST_CULLED, (unsigned long long)sCulled);
        atomicAdd(p.stats + ST_PASSED, (unsigned long long)sPassed);
    }
}

// a3-a6 over the live list, one voxel per thread, into a shared AM seeded from
// the global AM; a7 at the end.
template <bool COARSE>
__global__ void __launch_bounds__(kThreads) live_kernel(const __grid_constant__ StreamParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ unsigned int sCnt[CT_COUNT];
    // shared copy of the parameters for the out-of-line process_live (a
    // reference to the kernel parameter would make every call copy it)
    __shared__ StreamParams sP;
    if (threadIdx.x < (int)(sizeof(StreamParams) / 4))
        reinterpret_cast<unsigned int*>(&sP)[threadIdx.x] = reinterpret_cast<const unsigned int*>(&p)[threadIdx.x];
    const int m = p.grid.m, W = p.grid.W, MW = m * W;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_raw);
    uint32_t* sRowFull = sAM + MW;
    float* sCos = reinterpret_cast<float*>(sRowFull + ((m + 31) >> 5));
    float* sSin = sCos + m;
    const unsigned int nlive = *p.live_count;
    if ((unsigned long long)blockIdx.x * kThreads >= nlive) return;
    for (int i = threadIdx.x; i < m; i += blockDim.x) {
        sCos[i] = p.tab[i];
        sSin[i] = p.tab[m + i];
    }
    for (int w = threadIdx.x; w < MW; w += blockDim.x) sAM[w] = ld_cg(p.gam + w);
    if (threadIdx.x < CT_COUNT) sCnt[threadIdx.x] = 0u;
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int base = 0; base < m; base += blockDim.x) {
        const int i = base + threadIdx.x;
        bool full = false;
        if (i < m) {
            full = true;
            for (int w = 0; w < W; ++w)
                if (sAM[i * W + w] != row_word_mask(w, p.grid.n)) full = false;
        }
        const uint32_t bal = __ballot_sync(0xffffffffu, full);
        if (lane == 0 && base + warp * 32 < m) sRowFull[(base + warp * 32) >> 5] = bal;
    }
    __syncthreads();
    const Counters cnt{sCnt};
    for (unsigned long long e = blockIdx.x * (unsigned long long)kThreads + threadIdx.x; e < nlive;
         e += (unsigned long long)gridDim.x * kThreads) {
        const unsigned int vidx = p.live_idx[e];
        process_live<COARSE>(sP, vidx, p.vox[vidx], sAM, sRowFull, sCos, sSin, cnt);
    }
    __syncthreads();
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t sv = sAM[w];
        if (sv & ~ld_cg(p.gam + w)) atomicOr(p.gam + w, sv);
    }
    if (threadIdx.x == 0) {
        atomicAdd(p.stats + ST_LIVE, (unsigned long long)sCnt[CT_LIVE]);
        atomicAdd(p.stats + ST_ROWS, (unsigned long long)sCnt[CT_ROWS]);
        atomicAdd(p.stats + ST_BAND, (unsigned long long)sCnt[CT_BAND]);
        atomicAdd(p.stats + ST_OVERFLOW, (unsigned long long)sCnt[CT_OVERFLOW]);
    }
}

// Coarse levels: inner cones of the largest voxels, one warp per voxel with
// phi-rows across lanes, into a shared AM flushed to the global AM at the end.
// Voxels whose cheap cone holds no clear cell of p.cmap are skipped.
__global__ void __launch_bounds__(kThreads) coarse_kernel(const __grid_constant__ StreamParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    const GridDev& g = p.grid;
    const int m = g.m, W = g.W, MW = m * W;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_raw);
    float* sCos = reinterpret_cast<float*>(sAM + MW);
    float* sSin = sCos + m;
    for (int i = threadIdx.x; i < m; i += blockDim.x) {
        sCos[i] = p.tab[i];
        sSin[i] = p.tab[m + i];
    }
    for (int w = threadIdx.x; w < MW; w += blockDim.x) sAM[w] = 0u;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    const int B = p.tile;  // voxels per warp iteration: 1 (level 0, all live) or 32 (level 1, filtered)
    for (long long base = gw * B; base < p.N; base += nw * B) {
        const long long idx = base + lane;
        float4 q = make_float4(0.f, 0.f, 0.f, 1.f);
        int f = F_DROP;
        if (lane < B && idx < p.N) {
            q = p.vox[idx];
            f = fast_filter(p, q, sAM);
        }
        unsigned int live = __ballot_sync(0xffffffffu, f == F_LIVE);
        while (live) {
            const int src = __ffs(live) - 1;
            live &= live - 1u;
            const float4 v = make_float4(__shfl_sync(0xffffffffu, q.x, src), __shfl_sync(0xffffffffu, q.y, src),
                                         __shfl_sync(0xffffffffu, q.z, src), __shfl_sync(0xffffffffu, q.w, src));
            const float vx = v.x - p.px, vy = v.y - p.py, vz = v.z - p.pz, h = v.w;
            const float D = sqrtf(vx * vx + vy * vy + vz * vz);
            const float cin = inner_cone(D, h, p.tool);
            if (cin > 1.f) continue;
            const float rxy = sqrtf(vx * vx + vy * vy);
            const float phv = atan2f(rxy, vz);
            const float ai = acosf(fmaxf(cin, -1.f));
            const int i0 = max(0, (int)ceilf((phv - ai - kRowSlack) * g.inv_dphi - 0.5f));
            const int i1 = min(m - 1, (int)floorf((phv + ai + kRowSlack) * g.inv_dphi - 0.5f));
            const float invD = 1.f / D;
            const float cphv = vz * invD, sphv = rxy * invD;
            const float gv = atan2f(vy, vx);
            for (int i = i0 + lane; i <= i1; i += 32) {
                const Interval In = gamma_interval(cin, sCos[i] * cphv, sSin[i] * sphv, gv, -1, g);
                if (In.len == 0) continue;
                for (int w = 0; w < W; ++w) {
                    const uint32_t ib = interval_bits(In, w, g.n);
                    if (ib & ~ld_vol_shared(sAM + i * W + w)) atomicOr(sAM + i * W + w, ib);
                }
            }
        }
    }
    __syncthreads();
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t sv = sAM[w];
        if (sv) atomicOr(p.gam + w, sv);
    }
}


}  // namespace am
