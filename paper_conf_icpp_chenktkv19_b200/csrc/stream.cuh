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
// live_kernel (a3-a6; the live voxels only, ~0.01-1 %): 32 voxels per warp,
//   one per lane for the paper's two ICA cones (Alg. 1), checked
//   against the map once more; the (voxel, phi-row) pairs of the warp are then
//   dealt evenly over the lanes and rasterised into the CTA's shared AM; band
//   cells are deferred to the global band queue; the shared AM is OR-ed into
//   the global AM at the end (a7).  The clear-map levels use the same kernel
//   with inner cones only (level 0: every voxel of the level is live).
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

// a3-a6 for the live voxels of one warp (one per lane, `valid` lanes only).
// Each lane first computes its own voxel's two cones (GETTOOLICA twice, Alg. 1
// L147-148), checks the exact outer cone against the clear-direction map and
// finds its phi-row range; the warp then shares out the (voxel, row) pairs of
// all 32 voxels evenly over its lanes (a warp scan of the row counts), so a
// voxel with a 64-row cone and one with a 2-row cone cost the same latency.
// Per row (Alg. 1 L149-155 for all cells of a row at once): the inner-cone
// interval is OR-ed into the shared AM, outer-minus-inner cells still clear go
// to the band queue.  COARSE (clear-map levels) rasterises inner cones only.
template <bool COARSE>
__device__ __noinline__ void process_live_warp(const StreamParams& p, bool valid, unsigned int vidx, float4 q,
                                               uint32_t* sAM, const uint32_t* sRowFull, const float* sCos,
                                               const float* sSin, Counters cnt) {
    const ToolDev& T = p.tool;
    const GridDev& g = p.grid;
    const int lane = threadIdx.x & 31;
    float cin = 2.f, cout = 2.f, clo = 2.f, cphv = 0.f, sphv = 0.f, gv = 0.f;
    int i0 = 0, nrows = 0;
    if (valid) {
        const float vx = q.x - p.px, vy = q.y - p.py, vz = q.z - p.pz, h = q.w;
        const float D = sqrtf(vx * vx + vy * vy + vz * vz);
        const bool inside = D <= kSqrt3 * h && fabsf(vx) <= h && fabsf(vy) <= h && fabsf(vz) <= h;
        if (!inside) {  // (a voxel holding the pivot was filled by the filter)
            Cones c;
            if (COARSE) {
                c.cin = c.cout = inner_cone(D, h, T);
                c.clo = 2.f;
            } else {
                c = tool_cones(D, h, T);
            }
            // the exact outer cone against the clear-direction map: no clear
            // cell within it means this voxel cannot change the map
            if (c.cout <= 1.f &&
                __ldg(p.cmap + texel_of(vx, vy, vz, p.cmapT)) >= c.cout * fabsf(c.cout)) {
                const float rxy = sqrtf(vx * vx + vy * vy);
                const float phv = atan2f(rxy, vz);
                const float ao = acosf(fmaxf(c.cout, -1.f));
                const int a0 = max(0, (int)ceilf((phv - ao - kRowSlack) * g.inv_dphi - 0.5f));
                const int a1 = min(g.m - 1, (int)floorf((phv + ao + kRowSlack) * g.inv_dphi - 0.5f));
                if (a0 <= a1 && !rows_all_full(sRowFull, a0, a1)) {
                    const float invD = 1.f / D;
                    cin = c.cin;
                    cout = c.cout;
                    clo = c.clo;
                    cphv = vz * invD;
                    sphv = rxy * invD;
                    gv = atan2f(vy, vx);
                    i0 = a0;
                    nrows = a1 - a0 + 1;
                }
            }
        }
    }
    if (valid) atomicAdd(cnt.c + CT_LIVE, 1u);
    // warp scan of the row counts; (voxel, row) pairs are dealt round-robin
    int incl = nrows;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    const int total = __shfl_sync(0xffffffffu, incl, 31);
    const int W = g.W;
    unsigned int rows = 0;
    for (int base = 0; base < total; base += 32) {
        const int k = base + lane;
        // owner = number of lanes whose inclusive count is <= k
        int owner = 0;
#pragma unroll
        for (int step = 16; step > 0; step >>= 1) {
            const int cand = owner + step;
            if (__shfl_sync(0xffffffffu, incl, cand - 1) <= k) owner = cand;
        }
        owner = min(owner, 31);
        const int o_incl = __shfl_sync(0xffffffffu, incl, owner);
        const int o_n = __shfl_sync(0xffffffffu, nrows, owner);
        const int o_i0 = __shfl_sync(0xffffffffu, i0, owner);
        const float o_cin = __shfl_sync(0xffffffffu, cin, owner);
        const float o_cout = __shfl_sync(0xffffffffu, cout, owner);
        const float o_clo = __shfl_sync(0xffffffffu, clo, owner);
        const float o_c = __shfl_sync(0xffffffffu, cphv, owner);
        const float o_s = __shfl_sync(0xffffffffu, sphv, owner);
        const float o_gv = __shfl_sync(0xffffffffu, gv, owner);
        const unsigned int o_vidx = __shfl_sync(0xffffffffu, vidx, owner);
        if (k >= total) continue;
        const int i = o_i0 + (k - (o_incl - o_n));
        if ((ld_vol_shared(sRowFull + (i >> 5)) >> (i & 31)) & 1u) continue;
        const float rb = sCos[i] * o_c, rd = sSin[i] * o_s;
        if (COARSE) {
            const Interval In = gamma_interval(o_cin, rb, rd, o_gv, -1, g);
            if (In.len == 0) continue;
            ++rows;
            for (int w = 0; w < W; ++w) {
                const uint32_t ib = interval_bits(In, w, g.n);
                uint32_t* wp = sAM + i * W + w;
                if (ib & ~ld_vol_shared(wp)) atomicOr(wp, ib);
            }
            continue;
        }
        const Interval O = gamma_interval(o_cout, rb, rd, o_gv, +1, g);
        if (O.len == 0) continue;
        ++rows;
        const Interval In = gamma_interval(o_cin, rb, rd, o_gv, -1, g);
        const Interval X = gamma_interval(o_clo, rb, rd, o_gv, -1, g);
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
                push_band(p, sAM, o_vidx, p.vox_main[o_vidx], i * g.n + (w << 5) + b, wp, 1u << b, cnt);
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

// a3-a6 over the live list, 32 voxels per warp, into a shared AM seeded from
// the global AM; a7 (OR into the global AM) at the end.  With p.live_idx ==
// nullptr every voxel of vox[0, N) is live (clear-map level 0).
template <bool COARSE>
__global__ void __launch_bounds__(kThreads) live_kernel(const __grid_constant__ StreamParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ unsigned int sCnt[CT_COUNT];
    // shared copy of the parameters for the out-of-line process_live_warp (a
    // reference to the kernel parameter would make every call copy it)
    __shared__ StreamParams sP;
    if (threadIdx.x < (int)(sizeof(StreamParams) / 4))
        reinterpret_cast<unsigned int*>(&sP)[threadIdx.x] = reinterpret_cast<const unsigned int*>(&p)[threadIdx.x];
    const int m = p.grid.m, W = p.grid.W, MW = m * W;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_raw);
    uint32_t* sRowFull = sAM + MW;
    float* sCos = reinterpret_cast<float*>(sRowFull + ((m + 31) >> 5));
    float* sSin = sCos + m;
    const unsigned long long nlive = p.live_idx ? (unsigned long long)*p.live_count : (unsigned long long)p.N;
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
    // warps stride over groups of 32 entries (the loop bound is warp-uniform)
    for (unsigned long long e0 = (blockIdx.x * (unsigned long long)kThreads) + warp * 32ull; e0 < nlive;
         e0 += (unsigned long long)gridDim.x * kThreads) {
        const unsigned long long e = e0 + lane;
        const bool valid = e < nlive;
        unsigned int vidx = 0;
        float4 q = make_float4(0.f, 0.f, 0.f, 1.f);
        if (valid) {
            vidx = p.live_idx ? p.live_idx[e] : (unsigned int)e;
            q = p.vox[vidx];
        }
        process_live_warp<COARSE>(sP, valid, vidx, q, sAM, sRowFull, sCos, sSin, cnt);
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

}  // namespace am
