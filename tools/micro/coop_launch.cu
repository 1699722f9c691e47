// Microbenchmark: launch cost of a kernel shaped like am_latency_kernel (296 CTAs x 256 threads,
// ~44 KB dynamic shared memory, a ~2.7 KB __grid_constant__ parameter): cooperative vs plain
// launch, big vs small parameter, graph-captured, and the cost of cooperative grid barriers.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
struct Big { float v[680]; };
__global__ void __launch_bounds__(256, 2) k_big(const __grid_constant__ Big b, int* out, int phases) {
    extern __shared__ int sm[];
    sm[threadIdx.x] = threadIdx.x;
    for (int p = 0; p < phases; ++p) cooperative_groups::this_grid().sync();
    if (threadIdx.x == 0 && blockIdx.x == 0) out[0] = sm[5] + (int)b.v[7];
}
__global__ void __launch_bounds__(256, 2) k_small(int* out, int phases) {
    extern __shared__ int sm[];
    sm[threadIdx.x] = threadIdx.x;
    for (int p = 0; p < phases; ++p) cooperative_groups::this_grid().sync();
    if (threadIdx.x == 0 && blockIdx.x == 0) out[0] = sm[5];
}
int main() {
    int* out; cudaMalloc(&out, 1 << 20);
    Big b{};
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    size_t smem = 44 * 1024;
    cudaFuncSetAttribute(k_big, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_small, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_big, 256, smem);
    int grid = occ * sms;
    cudaStream_t s; cudaStreamCreate(&s);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto timeit = [&](const char* name, auto fn) {
        float sum = 0, best = 1e9; int n = 100;
        for (int it = 0; it < n + 10; ++it) {
            cudaEventRecord(e0, s); fn(); cudaEventRecord(e1, s); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            if (it >= 10) { sum += ms; best = ms < best ? ms : best; }
        }
        printf("%-48s mean %6.1f us  min %6.1f us  (%s)\n", name, 1e3 * sum / n, 1e3 * best, cudaGetErrorString(cudaGetLastError()));
    };
    for (int ph : {0, 1, 6}) {
        char nm[128];
        snprintf(nm, sizeof nm, "coop big param, %d grid syncs", ph);
        timeit(nm, [&] { void* a[] = {&b, &out, &ph}; cudaLaunchCooperativeKernel((void*)k_big, grid, 256, a, smem, s); });
        snprintf(nm, sizeof nm, "coop small param, %d grid syncs", ph);
        timeit(nm, [&] { void* a[] = {&out, &ph}; cudaLaunchCooperativeKernel((void*)k_small, grid, 256, a, smem, s); });
    }
    int z = 0;
    timeit("plain big param, no sync", [&] { k_big<<<grid, 256, smem, s>>>(b, out, z); });
    timeit("plain small param, no sync", [&] { k_small<<<grid, 256, smem, s>>>(out, z); });
    timeit("plain small param, 1 CTA", [&] { k_small<<<1, 256, smem, s>>>(out, z); });
    // graph of (memset, memset, coop kernel with 6 syncs)
    int six = 6;
    cudaGraph_t g; cudaGraphExec_t ge;
    cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
    cudaMemsetAsync(out + 1024, 0, 512, s); cudaMemsetAsync(out + 4096, 0, 512, s);
    { void* a[] = {&b, &out, &six}; cudaLaunchCooperativeKernel((void*)k_big, grid, 256, a, smem, s); }
    cudaStreamEndCapture(s, &g); cudaGraphInstantiate(&ge, g, 0);
    timeit("graph: 2 memsets + coop big, 6 syncs", [&] { cudaGraphLaunch(ge, s); });
    timeit("stream: 2 memsets + coop big, 6 syncs", [&] {
        cudaMemsetAsync(out + 1024, 0, 512, s); cudaMemsetAsync(out + 4096, 0, 512, s);
        void* a[] = {&b, &out, &six}; cudaLaunchCooperativeKernel((void*)k_big, grid, 256, a, smem, s); });
    return 0;
}
