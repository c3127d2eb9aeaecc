// probe: green contexts + runtime-API launches into green streams, SM confinement, clusters of 2
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <set>
#include <cstdlib>
#define DR(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { const char* s; cuGetErrorString(r, &s); printf("%s -> %s\n", #x, s); return 1; } } while (0)
#define RT(x) do { cudaError_t r = (x); if (r != cudaSuccess) { printf("%s -> %s\n", #x, cudaGetErrorString(r)); return 1; } } while (0)
__global__ void smid_k(int* out) {
    unsigned s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
    volatile int x = 0; for (int i = 0; i < 100000; ++i) x += i;
    if (threadIdx.x == 0) out[blockIdx.x] = s;
}
__global__ void __cluster_dims__(2, 1, 1) cl_k(int* out) {
    unsigned s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
    if (threadIdx.x == 0) out[blockIdx.x] = s;
}
int main() {
    RT(cudaFree(0));
    CUdevice dev; DR(cuDeviceGet(&dev, 0));
    CUdevResource all; DR(cuDeviceGetDevResource(dev, &all, CU_DEV_RESOURCE_TYPE_SM));
    printf("total SMs %u\n", all.sm.smCount);
    for (unsigned flags : {0u, 1u}) for (unsigned mc : {2u, 4u, 8u}) {
        unsigned n = 0; CUresult r = cuDevSmResourceSplitByCount(nullptr, &n, &all, nullptr, flags, mc);
        printf("flags %u minCount %u -> groups %u (r=%d)\n", flags, mc, n, (int)r);
    }
    const unsigned FL = getenv("FL") ? atoi(getenv("FL")) : 0, MC = getenv("MC") ? atoi(getenv("MC")) : 8;
    const unsigned KA = getenv("KA") ? atoi(getenv("KA")) : 1, KB = getenv("KB") ? atoi(getenv("KB")) : 3;
    unsigned n = 148; std::vector<CUdevResource> g(148); CUdevResource rem;
    DR(cuDevSmResourceSplitByCount(g.data(), &n, &all, &rem, FL, MC));
    printf("groups %u, each %u SMs, remainder %u\n", n, g[0].sm.smCount, rem.sm.smCount);
    // device A: 1 group (8 SMs), device B: 3 groups (24 SMs)
    CUdevResourceDesc dA, dB;
    DR(cuDevResourceGenerateDesc(&dA, &g[0], KA));
    DR(cuDevResourceGenerateDesc(&dB, &g[KA], KB));
    CUgreenCtx gA, gB; DR(cuGreenCtxCreate(&gA, dA, dev, CU_GREEN_CTX_DEFAULT_STREAM)); DR(cuGreenCtxCreate(&gB, dB, dev, CU_GREEN_CTX_DEFAULT_STREAM));
    CUdevResource rA, rB; DR(cuGreenCtxGetDevResource(gA, &rA, CU_DEV_RESOURCE_TYPE_SM)); DR(cuGreenCtxGetDevResource(gB, &rB, CU_DEV_RESOURCE_TYPE_SM));
    printf("green A %u SMs, B %u SMs\n", rA.sm.smCount, rB.sm.smCount);
    CUstream sA, sB; DR(cuGreenCtxStreamCreate(&sA, gA, CU_STREAM_NON_BLOCKING, 0)); DR(cuGreenCtxStreamCreate(&sB, gB, CU_STREAM_NON_BLOCKING, 0));
    int* d; RT(cudaMalloc(&d, 4096 * sizeof(int)));  // primary-context allocation
    int* d2; RT(cudaMalloc(&d2, 4096 * sizeof(int)));
    smid_k<<<512, 64, 0, (cudaStream_t)sA>>>(d);
    RT(cudaGetLastError());
    smid_k<<<512, 64, 0, (cudaStream_t)sB>>>(d2);
    RT(cudaGetLastError());
    RT(cudaDeviceSynchronize());
    std::vector<int> h(512), h2(512);
    RT(cudaMemcpy(h.data(), d, 512 * 4, cudaMemcpyDeviceToHost)); RT(cudaMemcpy(h2.data(), d2, 512 * 4, cudaMemcpyDeviceToHost));
    std::set<int> sa(h.begin(), h.end()), sb(h2.begin(), h2.end());
    printf("A ran on %zu SMs:", sa.size()); for (int x : sa) printf(" %d", x); printf("\n");
    printf("B ran on %zu SMs:", sb.size()); for (int x : sb) printf(" %d", x); printf("\n");
    cl_k<<<512, 64, 0, (cudaStream_t)sB>>>(d);
    RT(cudaGetLastError()); RT(cudaDeviceSynchronize());
    RT(cudaMemcpy(h.data(), d, 512 * 4, cudaMemcpyDeviceToHost));
    std::set<int> sc(h.begin(), h.begin() + 512);
    int bad = 0; for (int i = 0; i < 512; i += 2) bad += (h[i] / 2 != h[i + 1] / 2);
    printf("cluster pairs not on one TPC: %d\n", bad);
    printf("cluster kernel in B on %zu SMs, pairs:", sc.size()); for (int i = 0; i < 8; i += 2) printf(" (%d,%d)", h[i], h[i + 1]); printf("\n");
    // event across green streams and a normal stream
    cudaEvent_t e; RT(cudaEventCreate(&e)); RT(cudaEventRecord(e, (cudaStream_t)sA));
    cudaStream_t s0; RT(cudaStreamCreate(&s0)); RT(cudaStreamWaitEvent(s0, e, 0)); RT(cudaStreamSynchronize(s0));
    printf("event ok\n");
    return 0;
}
