// stream.cuh -- the voxel-streaming AICA kernels.
//
// The full stream is split in three launches so the part that touches every
// voxel stays lean and the rest stays balanced:
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
// cone_kernel (a3-a4; the live voxels only, ~0.01-1 %): one voxel per thread,
//   the paper's two ICA cones (Alg. 1), checked against the map once
//   more; each survivor writes a cone record and one task per phi-row of its
//   outer cone.
//
// row_kernel (a5-a7): one (voxel, row) task per thread -- perfectly balanced
//   whatever the cone sizes -- rasterised into the CTA's shared AM (seeded from
//   the global AM); band cells go to the global band queue; the shared AM is
//   OR-ed into the global AM at the end.
//
// The clear-map levels use the same two kernels with inner cones only (level
// 0 without the filter: every voxel of the level is live).
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

// Can a sphere / voxel whose blocked directions all satisfy U |U| >= thr (thr = the squared-sign
// cosine of its cheap or exact outer cone) be dropped, from the clear-direction map (m, texel
// centres tex, T per side)?  First the texel-wide bound U_t (as every direction of the texel);
// when that keeps it, the bound for v itself: with theta' = the stored (rounded-down) nearest-clear
// angle of the texel centre c and a = angle(v, c), every cell still clear is at least theta' - a
// from v (triangle inequality, for ANY texel), so U = cos(max(0, theta' - a)) = cos theta' cos a +
// sin theta' sin a (a < theta'), guarded.  sin a from |v x c| (accurate for small a).
#ifndef AM_SPHERE_REFINE
#define AM_SPHERE_REFINE true  // brick / sub-brick spheres too (false: the texel-wide bound only)
#endif
template <bool REFINE = true>
__device__ __forceinline__ bool cmap_drop(const float4* __restrict__ m, const float4* __restrict__ tex, int T,
                                          float vx, float vy, float vz, float thr) {
    const int t = texel_of(vx, vy, vz, T);
    const float4 cs = __ldg(m + t);
    if (cs.z < thr) return true;
    if (!REFINE) return false;
    if (cs.y == 0.f) return false;  // theta' = 0 (a clear cell at the texel centre): U = 1
    const float4 c = __ldg(tex + t);
    const float inv = rsqrtf(fmaf(vx, vx, fmaf(vy, vy, vz * vz)));
    const float ca = fmaf(vx, c.x, fmaf(vy, c.y, vz * c.z)) * inv;
    if (ca <= cs.x) return false;  // a >= theta': U = 1
    const float x = fmaf(vy, c.z, -vz * c.y), y = fmaf(vz, c.x, -vx * c.z), z = fmaf(vx, c.y, -vy * c.x);
    const float sa = sqrtf(fmaf(x, x, fmaf(y, y, z * z))) * inv;
    const float u = fminf(fmaf(cs.x, ca, cs.y * sa) + 4e-6f, 1.f);
    return u * fabsf(u) < thr;
}

// a2 + cheap cone vs clear-direction map (p.cmap is never null: before any map
// is built it is the all-clear map).  The map stores V = U |U|, where U bounds
// from above the cosine of the angle from any direction of the texel to the
// nearest still-clear cell; V is monotone in U, so U < x <=> V < x |x|.
// F_LIVE when the voxel may still change the AM, F_CULLED beyond reach,
// F_DROP otherwise.  A voxel holding the pivot blocks every orientation: it
// fills `am` (shared or global) directly.
// T: texels per face of the clear-direction map in p.cmap (0 = p.cmapT).
__device__ __forceinline__ int fast_filter(const StreamParams& p, float4 q, uint32_t* am, int T = 0,
                                           const float4* tex = nullptr) {
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
    return cmap_drop(p.cmap, T ? tex : p.cmap_tex, T ? T : p.cmapT, vx, vy, vz, thr) ? F_DROP : F_LIVE;
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

// Append the live voxels among one warp-row of 32 to the global live list (the single-pivot paths'
// lists hold every voxel of the stream, so live_cap is never reached there).
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
        if (live && pos < p.live_cap) p.live_idx[pos] = idx;
    }
}

// a1-a2 + cheap cones over vox[0, N): live indices go to p.live_idx.  Full
// tiles of kTile voxels take the unguarded path (kVPT independent LDG.128 per
// thread, streaming cache hint); the ragged last tile is guarded.
__global__ void __launch_bounds__(kThreads) filter_kernel(const __grid_constant__ StreamParams p) {
    __shared__ unsigned int sCulled, sPassed;
    if (map_full(p.early)) return;
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
        if (blockIdx.x == 0) atomicAdd(p.stats + ST_STREAMED, (unsigned long long)p.N);  // every voxel is read
    }
}

// ---------------------------------------------------------------------------
// filter_tma_kernel: the same full-stream filter with the voxel tiles staged
// in shared memory by the Tensor Memory Accelerator (1-D bulk copies,
// cp.async.bulk, completing on an mbarrier; north_star: "coalesced 16-byte
// float4 voxel loads staged via TMA").  Persistent CTAs (SMs x occupancy)
// each own the tiles blockIdx.x + k gridDim.x; a ring of kTmaStages 16 KB
// tiles keeps kTmaStages - 1 tiles in flight per CTA while the threads filter
// the current one, so the HBM stream no longer waits on the filter's
// registers (the LDG version holds its 4 loads per thread only until the
// filter starts).  Thread 0 is the producer: it arms the tile's mbarrier with
// the byte count and issues the copy with an L2 evict-first hint (each voxel
// is read once per map); every thread waits on the mbarrier's phase, copies
// its 4 voxels to registers, and after a CTA barrier thread 0 refills the
// stage with the tile kTmaStages ahead.  Same decisions per voxel as
// filter_kernel (same fast_filter), so the same live list up to order.
// ---------------------------------------------------------------------------
// Ring shapes (AM_OPT_STREAM_TMA value): voxels per thread per tile x stages.
template <int VPT, int STAGES>
struct TmaRing {
    static constexpr int kTileVox = kThreads * VPT;
    static constexpr unsigned int kBytes = kTileVox * (unsigned int)sizeof(float4);
    static constexpr size_t kSmem = (size_t)STAGES * kBytes;
};

__device__ __forceinline__ unsigned int smem_u32(const void* p) {
    return (unsigned int)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned int count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned int parity) {
    unsigned int done = 0;
    do {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
    } while (!done);
}

// One tile into stage buffer dst: arm bar with the byte count, then one 1-D bulk copy that completes on it.
__device__ __forceinline__ void tma_tile(void* dst, const void* src, unsigned int bytes, unsigned long long* bar,
                                         unsigned long long policy) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::
            "r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}

template <int VPT, int STAGES>
__global__ void __launch_bounds__(kThreads) filter_tma_kernel(const __grid_constant__ StreamParams p) {
    using R = TmaRing<VPT, STAGES>;
    constexpr int kT = R::kTileVox;
    extern __shared__ __align__(128) unsigned char smem_tma[];
    __shared__ __align__(8) unsigned long long sBar[STAGES];
    __shared__ unsigned int sCulled, sPassed;
    if (map_full(p.early)) return;
    float4* ring = reinterpret_cast<float4*>(smem_tma);
    const unsigned int nfull = (unsigned int)(p.N / kT);
    const unsigned int mine = nfull > blockIdx.x ? (nfull - blockIdx.x + gridDim.x - 1) / gridDim.x : 0u;
    unsigned long long policy = 0;
    if (threadIdx.x == 0) {
        sCulled = sPassed = 0u;
        asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(policy));
        for (int s = 0; s < STAGES; ++s) mbar_init(sBar + s, 1u);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (unsigned int k = 0; k < mine && k < (unsigned int)STAGES; ++k)
            tma_tile(ring + k * kT, p.vox + (size_t)(blockIdx.x + k * gridDim.x) * kT, R::kBytes, sBar + k, policy);
    }
    __syncthreads();
    unsigned int nculled = 0, npassed = 0;
    for (unsigned int k = 0; k < mine; ++k) {
        const int s = (int)(k % STAGES);
        mbar_wait(sBar + s, (k / STAGES) & 1u);
        const float4* tile = ring + s * kT;
        float4 q[VPT];
#pragma unroll
        for (int j = 0; j < VPT; ++j) q[j] = tile[j * kThreads + threadIdx.x];
        __syncthreads();  // every thread holds its voxels: the stage may be refilled
        if (threadIdx.x == 0 && k + STAGES < mine) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // (generic reads before async writes)
            tma_tile(ring + s * kT, p.vox + (size_t)(blockIdx.x + (k + STAGES) * gridDim.x) * kT, R::kBytes, sBar + s,
                     policy);
        }
        const unsigned int base = (blockIdx.x + k * gridDim.x) * kT + threadIdx.x;
        int f[VPT];
#pragma unroll
        for (int j = 0; j < VPT; ++j) f[j] = fast_filter(p, q[j], p.gam);
#pragma unroll
        for (int j = 0; j < VPT; ++j) {
            nculled += f[j] >> 1;
            append_live(p, f[j] == F_LIVE, base + j * kThreads, npassed);
        }
    }
    if (blockIdx.x == nfull % gridDim.x && (long long)nfull * kT < p.N) {  // ragged tail: plain loads
        const unsigned int base = nfull * kT + threadIdx.x;
#pragma unroll
        for (int j = 0; j < VPT; ++j) {
            const unsigned int idx = base + j * kThreads;
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
        if (blockIdx.x == 0) atomicAdd(p.stats + ST_STREAMED, (unsigned long long)p.N);  // every voxel is read
    }
}

// Warp-specialised variant: a 9th warp is the producer (lane 0 refills a stage as soon as the 8
// consumer warps have released it on the stage's "empty" mbarrier), so no CTA-wide barrier per tile:
// each consumer warp runs ahead as far as the ring allows.
template <int VPT, int STAGES>
__global__ void __launch_bounds__(kThreads + 32) filter_tma_ws_kernel(const __grid_constant__ StreamParams p) {
    using R = TmaRing<VPT, STAGES>;
    constexpr int kT = R::kTileVox;
    extern __shared__ __align__(128) unsigned char smem_tma[];
    __shared__ __align__(8) unsigned long long sFull[STAGES], sEmpty[STAGES];
    __shared__ unsigned int sCulled, sPassed;
    if (map_full(p.early)) return;
    float4* ring = reinterpret_cast<float4*>(smem_tma);
    const unsigned int nfull = (unsigned int)(p.N / kT);
    const unsigned int mine = nfull > blockIdx.x ? (nfull - blockIdx.x + gridDim.x - 1) / gridDim.x : 0u;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        sCulled = sPassed = 0u;
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(sFull + s, 1u);
            mbar_init(sEmpty + s, (unsigned int)kWarps);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    unsigned int nculled = 0, npassed = 0;
    if (warp == kWarps) {  // producer
        if (lane == 0) {
            unsigned long long policy;
            asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(policy));
            for (unsigned int k = 0; k < mine; ++k) {
                const int s = (int)(k % STAGES);
                if (k >= (unsigned int)STAGES) mbar_wait(sEmpty + s, ((k / STAGES) - 1u) & 1u);
                tma_tile(ring + s * kT, p.vox + (size_t)(blockIdx.x + k * gridDim.x) * kT, R::kBytes, sFull + s,
                         policy);
            }
        }
    } else {
        for (unsigned int k = 0; k < mine; ++k) {
            const int s = (int)(k % STAGES);
            mbar_wait(sFull + s, (k / STAGES) & 1u);
            const float4* tile = ring + s * kT;
            float4 q[VPT];
#pragma unroll
            for (int j = 0; j < VPT; ++j) q[j] = tile[j * kThreads + threadIdx.x];
            __syncwarp();
            if (lane == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(sEmpty + s)) : "memory");
            const unsigned int base = (blockIdx.x + k * gridDim.x) * kT + threadIdx.x;
            int f[VPT];
#pragma unroll
            for (int j = 0; j < VPT; ++j) f[j] = fast_filter(p, q[j], p.gam);
#pragma unroll
            for (int j = 0; j < VPT; ++j) {
                nculled += f[j] >> 1;
                append_live(p, f[j] == F_LIVE, base + j * kThreads, npassed);
            }
        }
        if (blockIdx.x == nfull % gridDim.x && (long long)nfull * kT < p.N) {  // ragged tail: plain loads
            const unsigned int base = nfull * kT + threadIdx.x;
#pragma unroll
            for (int j = 0; j < VPT; ++j) {
                const unsigned int idx = base + j * kThreads;
                const int f = idx < p.N ? fast_filter(p, p.vox[idx], p.gam) : F_DROP;
                nculled += f >> 1;
                append_live(p, f == F_LIVE, idx, npassed);
            }
        }
        if (lane == 0) atomicAdd(&sPassed, npassed);
        if (nculled) atomicAdd(&sCulled, nculled);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        atomicAdd(p.stats + ST_CULLED, (unsigned long long)sCulled);
        atomicAdd(p.stats + ST_PASSED, (unsigned long long)sPassed);
        if (blockIdx.x == 0) atomicAdd(p.stats + ST_STREAMED, (unsigned long long)p.N);  // every voxel is read
    }
}

// The cheap outer cone of a sphere (centre p + v, radius r) against the
// clear-direction map: true when the sphere -- hence every voxel inside it --
// can no longer change the AM (all its possibly blocked directions are
// blocked already) or lies beyond the tool's reach.
__device__ __forceinline__ bool sphere_dropped(const StreamParams& p, float vx, float vy, float vz, float r,
                                               int T = 0, const float4* tex = nullptr) {
    const float D2 = fmaf(vx, vx, fmaf(vy, vy, vz * vz));
    if (D2 <= r * r * 1.0001f) return false;  // the pivot is (almost) inside: keep
    const float invD = rsqrtf(D2);
    const float D = D2 * invD;
    if (p.may_cull && D - r > p.cull_dist) return true;
    const float Reff = reach_radius(p.tool, (D + r) * (1.f + kRadRel));
    const float s = fmaf((Reff + r) * invD, 1.f + 1.6e-5f, 1e-6f);
    const float c = fmaf(r * invD, 1.f + 1.6e-5f, 1e-6f);
    const float thr = (s < 1.f) ? fmaf(-s, s, 1.f) : -c * c;
    return cmap_drop<AM_SPHERE_REFINE>(p.cmap, T ? tex : p.cmap_tex, T ? T : p.cmapT, vx, vy, vz, thr);
}

// Full stream with brick culling (the paper's octree
// pruning of Alg. 2 L218-219 turned into a bulk test): the voxels are grouped
// into bricks of kThreads Morton-consecutive voxels, each with a bounding
// sphere (upload).  brick_test_kernel tests every brick (one per thread) and
// lists the bricks whose sphere still reaches a clear cell; brick_voxels_kernel
// streams only those, kVPT bricks per CTA step (one voxel per thread per
// brick), through fast_filter.  Exact-safe: a voxel's cone lies inside its
// brick's.
__global__ void __launch_bounds__(kThreads) brick_test_kernel(const __grid_constant__ StreamParams p) {
    if (map_full(p.early)) return;
    const int lane = threadIdx.x & 31;
    const unsigned int nb = p.nbricks;
    for (unsigned int b0 = blockIdx.x * kThreads; b0 < nb; b0 += gridDim.x * kThreads) {
        const unsigned int b = b0 + threadIdx.x;
        bool keep = false;
        if (b < nb) {
            const float4 s = __ldg(p.bricks + b);
            keep = !sphere_dropped(p, s.x - p.px, s.y - p.py, s.z - p.pz, s.w);
        }
        const unsigned int mk = __ballot_sync(0xffffffffu, keep);
        if (mk) {
            unsigned int base = 0;
            const int leader = __ffs(mk) - 1;
            if (lane == leader) base = atomicAdd(p.brick_count, (unsigned int)__popc(mk));
            base = __shfl_sync(0xffffffffu, base, leader);
            if (keep) p.brick_list[base + __popc(mk & ((1u << lane) - 1u))] = b;
        }
    }
}

__global__ void __launch_bounds__(kThreads) brick_voxels_kernel(const __grid_constant__ StreamParams p) {
    __shared__ unsigned int sCulled, sPassed;
    __shared__ unsigned long long sStreamed;
    if (map_full(p.early)) return;
    if (threadIdx.x == 0) {
        sCulled = sPassed = 0u;
        sStreamed = 0ull;
    }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    unsigned int nculled = 0, npassed = 0;
    unsigned long long streamed = 0;
    const unsigned int nk = *p.brick_count;
    for (unsigned int k0 = blockIdx.x * kVPT; k0 < nk; k0 += gridDim.x * kVPT) {
        float4 q[kVPT];
        unsigned int idx[kVPT];
        bool ok[kVPT];
#pragma unroll
        for (int k = 0; k < kVPT; ++k) {
            ok[k] = k0 + k < nk;
            idx[k] = ok[k] ? p.brick_list[k0 + k] * (unsigned int)kThreads + threadIdx.x : 0u;
            ok[k] = ok[k] && idx[k] < (unsigned long long)p.N;
            q[k] = ok[k] ? __ldcs(p.vox + idx[k]) : make_float4(0.f, 0.f, 0.f, 1.f);
        }
#pragma unroll
        for (int k = 0; k < kVPT; ++k) {
            const int f = ok[k] ? fast_filter(p, q[k], p.gam) : F_DROP;
            nculled += f >> 1;
            append_live(p, f == F_LIVE, idx[k], npassed);
            streamed += ok[k];
        }
    }
    if (lane == 0) atomicAdd(&sPassed, npassed);
    if (nculled) atomicAdd(&sCulled, nculled);
    if (streamed) atomicAdd(&sStreamed, streamed);
    __syncthreads();
    if (threadIdx.x == 0) {
        atomicAdd(p.stats + ST_CULLED, (unsigned long long)sCulled);
        atomicAdd(p.stats + ST_PASSED, (unsigned long long)sPassed);
        atomicAdd(p.stats + ST_STREAMED, sStreamed);
    }
}

// Bounding spheres of the bricks of bs consecutive voxels (one warp per
// brick): centre of the box enclosing the voxel cubes, radius its half
// diagonal, grown for rounding.
__global__ void brick_bounds_kernel(const float4* __restrict__ vox, long long N, float4* __restrict__ bricks,
                                    unsigned int nb, int bs) {
    const int lane = threadIdx.x & 31;
    const unsigned int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (w >= nb) return;
    float lo[3] = {3e38f, 3e38f, 3e38f}, hi[3] = {-3e38f, -3e38f, -3e38f};
    for (int k = lane; k < bs; k += 32) {
        const long long i = (long long)w * bs + k;
        if (i >= N) break;
        const float4 q = vox[i];
        lo[0] = fminf(lo[0], q.x - q.w); hi[0] = fmaxf(hi[0], q.x + q.w);
        lo[1] = fminf(lo[1], q.y - q.w); hi[1] = fmaxf(hi[1], q.y + q.w);
        lo[2] = fminf(lo[2], q.z - q.w); hi[2] = fmaxf(hi[2], q.z + q.w);
    }
#pragma unroll
    for (int a = 0; a < 3; ++a) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            lo[a] = fminf(lo[a], __shfl_xor_sync(0xffffffffu, lo[a], o));
            hi[a] = fmaxf(hi[a], __shfl_xor_sync(0xffffffffu, hi[a], o));
        }
    }
    if (lane == 0) {
        const float cx = 0.5f * (lo[0] + hi[0]), cy = 0.5f * (lo[1] + hi[1]), cz = 0.5f * (lo[2] + hi[2]);
        const float ex = hi[0] - lo[0], ey = hi[1] - lo[1], ez = hi[2] - lo[2];
        const float r = 0.5f * sqrtf(ex * ex + ey * ey + ez * ez);
        bricks[w] = make_float4(cx, cy, cz, r * (1.f + 1e-5f) + 1e-6f * (fabsf(cx) + fabsf(cy) + fabsf(cz)));
    }
}

// Dynamic shared memory of row_kernel for an m x n grid: AM + row-full bits.
__host__ __device__ inline size_t live_smem_bytes(int m, int W) {
    return (size_t)(m * W + ((m + 31) >> 5)) * sizeof(uint32_t);
}

// A task entry that names no cone (its cone was rasterised inline when the buffers were full).
constexpr unsigned long long kInertTask = ~0ull;

// A live voxel's cones and phi-row range, as the row kernel needs them.
struct ConeRec {
    float cin, cout, clo;  // guarded cone cosines (geometry.cuh Cones)
    float cphv, sphv, gv;  // cone axis: cos/sin of phi_v, gamma_v
    unsigned int vidx;     // voxel index (band queue entries)
    int i0;                // first phi-row of the outer cone
};

// AM_OPT_REUSE: voxel `id` set the cells `fresh` of word w of row i (in this CTA's view): it becomes
// their witness (any voxel whose inner cone holds a cell is a valid one; the last writer wins).
__device__ __forceinline__ void note_witness(const StreamParams& p, unsigned int id, int i, int w, uint32_t fresh) {
    if (!p.wit) return;
    unsigned int* row = p.wit + i * p.grid.n + (w << 5);
    while (fresh) {
        const int b = __ffs(fresh) - 1;
        fresh &= fresh - 1u;
        row[b] = id;
    }
}

// Rows of a voxel processed inline when the record/task buffers are full
// (correct, only slower).
template <bool COARSE>
__device__ void raster_row(const StreamParams& p, const ConeRec& r, int i, uint32_t* am, Counters cnt);

// a3-a4 for one live voxel q (index vidx): the paper's two cones (GETTOOLICA
// twice, Alg. 1; COARSE: the inner one only), the exact outer cone
// checked against the clear-direction map, the phi-row range.  Returns the
// number of phi-rows to rasterise (0: nothing to do) and fills r.  `counted`
// tells whether the voxel reached the cone computation (am_stats voxels_live).
//
// With a list of the cells still clear (clear[0, nclear), nclear >= 0) the
// exact cones are also checked against it: a voxel none of whose relevant
// cells (outer cone, minus the inside of a ring) is still clear cannot change
// the map -- its inner cone lies in blocked cells and its band cells are
// blocked -- so it is dropped before any row is emitted.  The slack covers the
// raster's own interval slack, so the check never drops a voxel the raster
// would use.
template <bool COARSE>
__device__ __forceinline__ int cone_of_voxel(const StreamParams& p, float4 q, unsigned int vidx, ConeRec& r,
                                             bool& counted, const float4* clear = nullptr, int nclear = -1,
                                             int cmT = 0, const int* rowStart = nullptr,
                                             const float4* cmTex = nullptr) {
    const ToolDev& T = p.tool;
    const GridDev& g = p.grid;
    counted = false;
    const float vx = q.x - p.px, vy = q.y - p.py, vz = q.z - p.pz, h = q.w;
    const float D = sqrtf(vx * vx + vy * vy + vz * vz);
    if (D <= kSqrt3 * h && fabsf(vx) <= h && fabsf(vy) <= h && fabsf(vz) <= h) {
        fill_all(p, p.gam);  // the pivot lies in the closed box: every orientation collides
        return 0;
    }
    counted = true;
    Cones c;
    if (COARSE) {
        c.cin = c.cout = inner_cone(D, h, T);
        c.clo = 2.f;
    } else {
        c = tool_cones(D, h, T);
    }
    // the exact outer cone against the clear-direction map: no clear cell
    // within it means this voxel cannot change the map
    if (c.cout > 1.f || cmap_drop(p.cmap, cmT ? cmTex : p.cmap_tex, cmT ? cmT : p.cmapT, vx, vy, vz,
                                  c.cout * fabsf(c.cout)))
        return 0;
    const float rxy = sqrtf(vx * vx + vy * vy);
    const float phv = atan2f(rxy, vz);
    const float ao = acosf(fmaxf(c.cout, -1.f));
    const int a0 = max(0, (int)ceilf((phv - ao - kRowSlack) * g.inv_dphi - 0.5f));
    const int a1 = min(g.m - 1, (int)floorf((phv + ao + kRowSlack) * g.inv_dphi - 0.5f));
    if (a0 > a1) return 0;
    if (nclear >= 0) {
        // only cells of the rows a0..a1 the raster would visit can be changed by this voxel
        const float inv = 1.f / D;
        const float ux = vx * inv, uy = vy * inv, uz = vz * inv;
        const float lo = c.cout - kClearSlack, hi = c.clo + kClearSlack;
        bool any = false;
        const int e0 = rowStart ? rowStart[a0] : 0, e1 = rowStart ? rowStart[a1 + 1] : nclear;
        auto dotc = [&](int e) {
            const float4 d = clear[e];
            return fmaf(ux, d.x, fmaf(uy, d.y, uz * d.z));
        };
        int e = e0;
        if (hi > 1.5f) {  // no ring (the common case): only the outer cone, 4 cells per test
            for (; e + 4 <= e1; e += 4)
                if (fmaxf(fmaxf(dotc(e), dotc(e + 1)), fmaxf(dotc(e + 2), dotc(e + 3))) >= lo) {
                    any = true;
                    break;
                }
        }
        for (; e < e1 && !any; ++e) {
            const float cd = dotc(e);
            any = cd >= lo && cd <= hi;
        }
        if (!any) return 0;
    }
    const float invD = 1.f / D;
    r.cin = c.cin;
    r.cout = c.cout;
    r.clo = c.clo;
    r.cphv = vz * invD;
    r.sphv = rxy * invD;
    r.gv = atan2f(vy, vx);
    r.vidx = vidx;
    r.i0 = a0;
    return a1 - a0 + 1;
}

// Warp-uniform: store the records of the lanes with nrows > 0 and one task per
// (voxel, row), with one pair of atomics per warp.  When the buffers are full
// the lane rasterises its rows itself, straight into the global AM.
template <bool COARSE>
__device__ __forceinline__ void emit_cones(const StreamParams& p, int nrows, const ConeRec& r, bool counted) {
    const int lane = threadIdx.x & 31;
    const unsigned int mcount = __ballot_sync(0xffffffffu, counted);
    if (lane == 0 && mcount) atomicAdd(p.stats + ST_LIVE, (unsigned long long)__popc(mcount));
    const unsigned int mrec = __ballot_sync(0xffffffffu, nrows > 0);
    if (!mrec) return;
    int incl = nrows;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    unsigned int sbase = 0;
    unsigned long long tbase = 0;
    const int total = __shfl_sync(0xffffffffu, incl, 31);
    if (lane == 0) {
        sbase = atomicAdd(p.rec_count, (unsigned int)__popc(mrec));
        tbase = atomicAdd(p.task_count, (unsigned long long)total);
    }
    sbase = __shfl_sync(0xffffffffu, sbase, 0);
    tbase = __shfl_sync(0xffffffffu, tbase, 0);
    if (nrows > 0) {
        const unsigned int slot = sbase + __popc(mrec & ((1u << lane) - 1u));
        const unsigned long long t0 = tbase + (unsigned long long)(incl - nrows);
        if (slot < p.rec_cap && t0 + nrows <= p.task_cap) {
            p.recs[slot] = r;
            for (int k = 0; k < nrows; ++k) p.tasks[t0 + k] = ((unsigned long long)slot << 16) | (unsigned int)k;
        } else {
            // buffers full: rasterise inline; the record slot and the reserved task entries inside the
            // buffers are made inert (the row pass reads every entry below the capacities)
            for (int k = 0; k < nrows; ++k) raster_row<COARSE>(p, r, r.i0 + k, p.gam, Counters{nullptr});
            if (slot < p.rec_cap) p.recs[slot].i0 = -1;
            for (unsigned long long t = t0; t < t0 + nrows && t < p.task_cap; ++t) p.tasks[t] = kInertTask;
        }
    }
}

// a3-a4 over the live list (one voxel per thread): records and row tasks.
// With p.live_idx == nullptr every voxel of vox[0, N) is live (clear-map level 0).
template <bool COARSE>
__global__ void __launch_bounds__(kThreads) cone_kernel(const __grid_constant__ StreamParams p) {
    if (map_full(p.early)) return;
    const int lane = threadIdx.x & 31;
    const unsigned long long nlive =
        p.live_idx ? (unsigned long long)min(*p.live_count, p.live_cap) : (unsigned long long)p.N;
    const unsigned long long wstride = (unsigned long long)gridDim.x * blockDim.x;
    // warp-uniform loop: the slot reservations are warp-aggregated
    for (unsigned long long e0 = blockIdx.x * (unsigned long long)blockDim.x + (threadIdx.x & ~31u); e0 < nlive;
         e0 += wstride) {
        const unsigned long long e = e0 + lane;
        int nrows = 0;
        bool counted = false;
        ConeRec r;
        if (e < nlive) {
            const unsigned int vidx = p.live_idx ? p.live_idx[e] : (unsigned int)e;
            nrows = cone_of_voxel<COARSE>(p, p.vox[vidx], vidx, r, counted);
        }
        emit_cones<COARSE>(p, nrows, r, counted);
    }
}

// One phi-row of one cone (Alg. 1 L149-155 for all cells of a row at once):
// the inner-cone interval is OR-ed into `am`; outer-minus-inner cells still
// clear go to the band queue (COARSE: inner cone only).
template <bool COARSE>
__device__ void raster_row(const StreamParams& p, const ConeRec& r, int i, uint32_t* am, Counters cnt) {
    const GridDev& g = p.grid;
    const int W = g.W;
    const float rb = __ldg(p.tab + i) * r.cphv, rd = __ldg(p.tab + g.m + i) * r.sphv;
    if (COARSE) {
        const Interval In = gamma_interval(r.cin, rb, rd, r.gv, -1, g);
        if (In.len == 0) return;
        for (int w = 0; w < W; ++w) {
            const uint32_t ib = interval_bits(In, w, g.n);
            uint32_t* wp = am + i * W + w;
            const uint32_t fresh = ib & ~*reinterpret_cast<volatile uint32_t*>(wp);
            if (fresh) {
                atomicOr(wp, ib);
                note_witness(p, r.vidx, i, w, fresh);
            }
        }
        return;
    }
    const Interval O = gamma_interval(r.cout, rb, rd, r.gv, +1, g);
    if (O.len == 0) return;
    {  // nothing to do when every cell of the outer interval is already blocked
        uint32_t fresh = 0u;
        for (int w = 0; w < W; ++w)
            fresh |= interval_bits(O, w, g.n) & ~*reinterpret_cast<volatile uint32_t*>(am + i * W + w);
        if (!fresh) return;
    }
    const Interval In = gamma_interval(r.cin, rb, rd, r.gv, -1, g);
    const Interval X = gamma_interval(r.clo, rb, rd, r.gv, -1, g);
    for (int w = 0; w < W; ++w) {
        uint32_t ob = interval_bits(O, w, g.n);
        if (!ob) continue;
        const uint32_t xb = interval_bits(X, w, g.n);
        const uint32_t ib = interval_bits(In, w, g.n) & ~xb;
        ob &= ~xb;
        uint32_t* wp = am + i * W + w;
        uint32_t cur = *reinterpret_cast<volatile uint32_t*>(wp);
        if (ib & ~cur) {
            atomicOr(wp, ib);
            note_witness(p, r.vidx, i, w, ib & ~cur);
            cur |= ib;
        }
        uint32_t band = ob & ~ib & ~cur;
        while (band) {
            const int b = __ffs(band) - 1;
            band &= band - 1u;
            push_band(p, am, r.vidx, p.vox_main[r.vidx], i * g.n + (w << 5) + b, wp, 1u << b, cnt);
        }
    }
}

// a5-a7: one (voxel, phi-row) task per thread into a shared AM seeded from the
// global AM (rows already full are skipped), then OR-ed into the global AM.
template <bool COARSE>
__global__ void __launch_bounds__(kThreads) row_kernel(const __grid_constant__ StreamParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ unsigned int sCnt[CT_COUNT];
    const int m = p.grid.m, W = p.grid.W, MW = m * W;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_raw);
    uint32_t* sRowFull = sAM + MW;
    const unsigned long long ntask = min(*p.task_count, p.task_cap);
    if ((unsigned long long)blockIdx.x * kThreads >= ntask) return;  // CTA-uniform
    if (map_full(p.early)) return;
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
    unsigned int rows = 0, rfull = 0;
    for (unsigned long long k = blockIdx.x * (unsigned long long)kThreads + threadIdx.x; k < ntask;
         k += (unsigned long long)gridDim.x * kThreads) {
        const unsigned long long t = p.tasks[k];
        if (t == kInertTask) continue;  // (a cone rasterised inline: see emit_cones)
        const ConeRec r = p.recs[t >> 16];
        if (r.i0 < 0) continue;
        const int i = r.i0 + (int)(t & 0xffffu);
        if ((sRowFull[i >> 5] >> (i & 31)) & 1u) {
            ++rfull;
            continue;
        }
        ++rows;
        raster_row<COARSE>(p, r, i, sAM, cnt);
    }
    if (rows) atomicAdd(sCnt + CT_ROWS, rows);
    if (rfull) atomicAdd(sCnt + CT_ROWFULL, rfull);
    __syncthreads();
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t sv = sAM[w];
        if (sv & ~ld_cg(p.gam + w)) atomicOr(p.gam + w, sv);
    }
    if (threadIdx.x == 0) {
        atomicAdd(p.stats + ST_ROWS, (unsigned long long)sCnt[CT_ROWS]);
        atomicAdd(p.stats + ST_BAND, (unsigned long long)sCnt[CT_BAND]);
        atomicAdd(p.stats + ST_OVERFLOW, (unsigned long long)sCnt[CT_OVERFLOW]);
        if (!COARSE) atomicAdd(p.stats + ST_ROWFULL, (unsigned long long)sCnt[CT_ROWFULL]);
    }
}

}  // namespace am
