// stream.cuh -- the voxel-streaming AICA kernel.
//
// One persistent CTA per SM slot.  Tiles of voxels are claimed dynamically from
// an atomic counter and copied global -> shared with the 1-D TMA engine
// (cp.async.bulk + mbarrier complete_tx, SASS UBLKCP) into a 2-stage ring, so
// the HBM stream runs ahead of the arithmetic without holding registers.
//
// Per voxel the CTA first runs a cheap, exact-safe FILTER (fast_filter): reach
// cull, then the cheap outer cone -- a sphere of radius sqrt(3) h at distance D
// only touches cylinders starting within D + sqrt(3) h, whose radii are at most
// Reff, so its blocked directions satisfy sin(theta) <= (Reff + sqrt3 h) / D --
// against the clear-direction map (kernels.cuh clear_map_kernel).  A voxel whose
// cheap cone contains no still-clear cell cannot change the AM and is dropped
// after ~50 instructions.  Survivors ("live" voxels, ~1-2 % at the paper's 1 mm
// offset) are appended to a shared-memory queue with a warp ballot and, once
// enough have accumulated, processed one per thread with full warps
// (process_live): the paper's two ICA cones (Alg. 1) rasterised row by
// row into the per-CTA shared AM, band cells deferred to the global queue.
#pragma once
#include "kernels.cuh"

namespace am {

constexpr int kStages = 2;
static_assert(sizeof(StreamParams) % 4 == 0 && sizeof(StreamParams) / 4 <= kThreads,
              "StreamParams is copied to shared memory one word per thread");
constexpr int kLiveCap = kTile + kThreads;  // a whole tile may go live on top of a part-full queue

__device__ __forceinline__ unsigned int smem_u32(const void* p) {
    return static_cast<unsigned int>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned int count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, unsigned int bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned int parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

// 1-D bulk copy global -> shared, completion signalled on `bar` (bytes % 16 == 0).
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, unsigned int bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

enum { F_DROP = 0, F_LIVE = 1, F_CULLED = 2 };

// a2 + cheap cone vs clear-direction map.  F_LIVE when the voxel may still
// change the AM, F_CULLED beyond reach, F_DROP otherwise.
__device__ __forceinline__ int fast_filter(const StreamParams& p, float4 q, uint32_t* sAM) {
    const ToolDev& T = p.tool;
    const float vx = q.x - p.px, vy = q.y - p.py, vz = q.z - p.pz, h = q.w;
    const float D2 = fmaf(vx, vx, fmaf(vy, vy, vz * vz));
    const float r2 = kSqrt3 * h;
    if (D2 <= 3.0001f * h * h) {
        // the pivot may lie in the closed box: then every orientation collides
        if (fabsf(vx) <= h && fabsf(vy) <= h && fabsf(vz) <= h) {
            fill_all(p, sAM);
            return F_DROP;
        }
        return F_LIVE;
    }
    const float invD = rsqrtf(D2);
    const float D = D2 * invD;
    if (D - r2 > p.cull_dist) return F_CULLED;
    if (!p.cmap) return F_LIVE;
    // cheap outer cone; z0 is padded with +inf beyond the last cylinder
    const float reach = (D + r2) * (1.f + kRadRel);
    float Reff = T.Rpm[0];
#pragma unroll
    for (int k = 1; k < AM_MAX_CYL; ++k)
        if (T.z0[k] <= reach) Reff = T.Rpm[k];
    const float s = fmaf((Reff + r2) * invD, 1.f + 1.6e-5f, 1e-6f);
    const float U = __ldg(p.cmap + cube_texel(vx, vy, vz, p.cmapT));
    // U bounds cos(angle to the nearest clear cell) from above for every
    // direction of the texel: drop when cos(cheap cone) > U.
    const bool drop = (s < 1.f) ? (U < 0.f || U * U < 1.f - s * s) : (U < -1.5f);
    return drop ? F_DROP : F_LIVE;
}

// a3-a6 for one live voxel.  COARSE launches only rasterise the inner cones
// (the clear-direction map needs certainly-blocked cells only; every coarse
// voxel is streamed again, with its band, by the full launch).
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
    const Cones c = tool_cones(D, h, T);
    const float cthr = COARSE ? c.cin : c.cout;
    if (cthr > 1.f) return;
    const float ao = acosf(fmaxf(cthr, -1.f));
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
        ++rows;
        const Interval In = gamma_interval(c.cin, base, den, gv, -1, g);
        if (COARSE) {
            if (In.len == 0) continue;
            for (int w = 0; w < W; ++w) {
                const uint32_t ib = interval_bits(In, w, g.n);
                uint32_t* wp = sAM + i * W + w;
                if (ib & ~ld_vol_shared(wp)) atomicOr(wp, ib);
            }
            continue;
        }
        const Interval O = gamma_interval(c.cout, base, den, gv, +1, g);
        if (O.len == 0) continue;
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

// a7: merge the CTA's shared AM with the global AM (one atomicOr per word that
// gained bits), read the union back, recompute the row-full bits.  Returns
// true when the whole AM is blocked (early exit).
__device__ __noinline__ bool cta_merge(const StreamParams& p, uint32_t* sAM, uint32_t* sShadow,
                                       uint32_t* sRowFull, int* sCount) {
    const int MW = p.grid.m * p.grid.W;
    const int W = p.grid.W;
    __syncthreads();
    if (threadIdx.x == 0) *sCount = 0;
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t s = sAM[w];
        uint32_t gv;
        if (s & ~sShadow[w])
            gv = atomicOr(p.gam + w, s) | s;
        else
            gv = ld_cg(p.gam + w) | s;
        sAM[w] = gv;
        sShadow[w] = gv;
    }
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int base = 0; base < p.grid.m; base += blockDim.x) {
        const int i = base + threadIdx.x;
        bool full = false;
        if (i < p.grid.m) {
            full = true;
            for (int w = 0; w < W; ++w)
                if (sAM[i * W + w] != row_word_mask(w, p.grid.n)) full = false;
        }
        const uint32_t bal = __ballot_sync(0xffffffffu, full);
        if (lane == 0 && base + warp * 32 < p.grid.m) {
            sRowFull[(base + warp * 32) >> 5] = bal;
            atomicAdd(sCount, __popc(bal));
        }
    }
    __syncthreads();
    return *sCount == p.grid.m;
}

// Dynamic shared memory of aica_stream_kernel for an m x n grid.
__host__ __device__ inline size_t stream_smem_bytes(int m, int W) {
    size_t b = (size_t)kStages * kTile * sizeof(float4);            // TMA ring
    b += (size_t)kLiveCap * sizeof(float4);                           // live queue voxels
    b += (size_t)kLiveCap * sizeof(unsigned int);                     // live queue indices
    b += (size_t)(2 * m * W + ((m + 31) >> 5)) * sizeof(uint32_t);  // AM, shadow, row-full bits
    b += (size_t)2 * m * sizeof(float);                               // cos / sin phi rows
    return b;
}

// Process the live queue with one voxel per thread.
template <bool COARSE>
__device__ __forceinline__ void drain_live(const StreamParams& p, int nlive, const unsigned int* sQi,
                                           const float4* sQv, uint32_t* sAM, const uint32_t* sRowFull,
                                           const float* sCos, const float* sSin, Counters cnt) {
    for (int e = threadIdx.x; e < nlive; e += kThreads)
        process_live<COARSE>(p, sQi[e], sQv[e], sAM, sRowFull, sCos, sSin, cnt);
}

template <bool COARSE>
__global__ void __launch_bounds__(kThreads, 3) aica_stream_kernel(const __grid_constant__ StreamParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ uint64_t bar[kStages];
    __shared__ long long sTileIdx[kStages];
    __shared__ int sCount, sLiveN;
    __shared__ unsigned int sCnt[CT_COUNT];
    __shared__ unsigned long long sStreamed, sCulled, sPassed;
    // shared copy of the parameters for the out-of-line cold path (a reference
    // to the kernel parameter would make every call copy it to local memory)
    __shared__ StreamParams sP;
    if (threadIdx.x < (int)(sizeof(StreamParams) / 4))
        reinterpret_cast<unsigned int*>(&sP)[threadIdx.x] = reinterpret_cast<const unsigned int*>(&p)[threadIdx.x];
    const int m = p.grid.m;
    const int MW = m * p.grid.W;
    float4* sVox = reinterpret_cast<float4*>(smem_raw);
    float4* sQv = sVox + kStages * kTile;
    unsigned int* sQi = reinterpret_cast<unsigned int*>(sQv + kLiveCap);
    uint32_t* sAM = sQi + kLiveCap;
    uint32_t* sShadow = sAM + MW;
    uint32_t* sRowFull = sShadow + MW;
    float* sCos = reinterpret_cast<float*>(sRowFull + ((m + 31) >> 5));
    float* sSin = sCos + m;
    const Counters cnt{sCnt};

    const int tile = p.tile;
    const long long ntiles = (p.N + tile - 1) / tile;
    for (int i = threadIdx.x; i < m; i += blockDim.x) {
        sCos[i] = p.tab[i];
        sSin[i] = p.tab[m + i];
    }
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        sAM[w] = 0u;
        sShadow[w] = 0u;
    }
    if (threadIdx.x < CT_COUNT) sCnt[threadIdx.x] = 0u;
    if (threadIdx.x == 0) {
        sLiveN = 0;
        sStreamed = sCulled = sPassed = 0ull;
        for (int s = 0; s < kStages; ++s) mbar_init(&bar[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int s = 0; s < kStages; ++s) {  // claim and load the first tiles
            const long long t = atomicAdd(p.tile_ctr, 1u);
            sTileIdx[s] = t;
            if (t < ntiles) {
                const long long first = t * tile;
                const unsigned int bytes = (unsigned int)(min((long long)tile, p.N - first) * sizeof(float4));
                mbar_expect_tx(&bar[s], bytes);
                tma_load_1d(sVox + s * kTile, p.vox + first, bytes, &bar[s]);
            }
        }
    }
    bool early = cta_merge(p, sAM, sShadow, sRowFull, &sCount);  // also publishes the setup above
    const int lane = threadIdx.x & 31;
    unsigned int phase = 0;  // bit s = parity of stage s
    unsigned int nculled = 0, npassed = 0;  // per-warp tallies (lane 0)
    int since = 0;
    for (int s = 0; !early; s ^= 1) {
        const long long t = sTileIdx[s];
        if (t >= ntiles) break;
        mbar_wait(&bar[s], (phase >> s) & 1u);
        phase ^= 1u << s;
        const long long first = t * tile;
        const int cntv = (int)min((long long)tile, p.N - first);
        const float4* tv = sVox + s * kTile;
#pragma unroll
        for (int k = 0; k < kVPT; ++k) {
            const int local = k * kThreads + threadIdx.x;
            int f = F_DROP;
            float4 q = make_float4(0.f, 0.f, 0.f, 0.f);
            if (local < cntv) {
                q = tv[local];
                f = fast_filter(p, q, sAM);
            }
            const unsigned int mlive = __ballot_sync(0xffffffffu, f == F_LIVE);
            const unsigned int mcull = __ballot_sync(0xffffffffu, f == F_CULLED);
            nculled += __popc(mcull);
            npassed += __popc(mlive);
            if (mlive) {
                int basepos = 0;
                const int leader = __ffs(mlive) - 1;
                if (lane == leader) basepos = atomicAdd(&sLiveN, __popc(mlive));
                basepos = __shfl_sync(0xffffffffu, basepos, leader);
                if (f == F_LIVE) {
                    const int pos = basepos + __popc(mlive & ((1u << lane) - 1u));
                    sQv[pos] = q;
                    sQi[pos] = (p.vbase + (unsigned int)(first + local)) | p.vtag;
                }
            }
        }
        __syncthreads();  // stage s consumed; live queue complete for this tile
        if (threadIdx.x == 0) {
            sStreamed += (unsigned long long)cntv;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            const long long tn = atomicAdd(p.tile_ctr, 1u);
            sTileIdx[s] = tn;
            if (tn < ntiles) {
                const long long f2 = tn * tile;
                const unsigned int bytes = (unsigned int)(min((long long)tile, p.N - f2) * sizeof(float4));
                mbar_expect_tx(&bar[s], bytes);
                tma_load_1d(sVox + s * kTile, p.vox + f2, bytes, &bar[s]);
            }
        }
        const int nlive = sLiveN;
        if (nlive >= kLiveCap - kTile) {
            drain_live<COARSE>(sP, nlive, sQi, sQv, sAM, sRowFull, sCos, sSin, cnt);
            __syncthreads();
            if (threadIdx.x == 0) sLiveN = 0;
        }
        if (++since >= p.refresh_tiles) {
            since = 0;
            early = cta_merge(p, sAM, sShadow, sRowFull, &sCount);
        } else {
            __syncthreads();  // publishes sTileIdx[s] and sLiveN
        }
    }
    drain_live<COARSE>(sP, sLiveN, sQi, sQv, sAM, sRowFull, sCos, sSin, cnt);
    // an early exit may leave bulk copies in flight: wait for them before the
    // CTA retires (its shared memory must not be written after it exits)
    if (early) {
        for (int s = 0; s < kStages; ++s)
            if (sTileIdx[s] < ntiles) mbar_wait(&bar[s], (phase >> s) & 1u);
    }
    if (lane == 0) {
        atomicAdd(&sCulled, (unsigned long long)nculled);
        atomicAdd(&sPassed, (unsigned long long)npassed);
    }
    // final flush of words that gained bits
    __syncthreads();
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t sv = sAM[w];
        if (sv & ~sShadow[w]) atomicOr(p.gam + w, sv);
    }
    if (threadIdx.x == 0) {
        atomicAdd(p.stats + ST_STREAMED, sStreamed);
        atomicAdd(p.stats + ST_CULLED, sCulled);
        atomicAdd(p.stats + ST_SKIPPED, sStreamed - sCulled - sPassed);
        atomicAdd(p.stats + ST_LIVE, (unsigned long long)sCnt[CT_LIVE]);
        atomicAdd(p.stats + ST_ROWS, (unsigned long long)sCnt[CT_ROWS]);
        atomicAdd(p.stats + ST_BAND, (unsigned long long)sCnt[CT_BAND]);
        atomicAdd(p.stats + ST_OVERFLOW, (unsigned long long)sCnt[CT_OVERFLOW]);
        if (early) atomicMax(p.stats + ST_EARLY, 1ULL);
    }
}

}  // namespace am
