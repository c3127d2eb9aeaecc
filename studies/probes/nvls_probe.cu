// Probe: is NVLS multicast (cuMulticastCreate + multimem.st) usable on this box
// with a single GPU?  Creates a 1-device multicast object, binds a physical
// allocation, writes through the multicast VA with multimem.st and reads the
// unicast VA back; times multimem.st against plain stores.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o nvls_probe nvls_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { CUresult r_ = (x); if (r_ != CUDA_SUCCESS) { const char* s_ = nullptr; cuGetErrorString(r_, &s_); \
    printf("{\"ok\": false, \"step\": \"%s\", \"err\": \"%s\"}\n", #x, s_ ? s_ : "?"); return 0; } } while (0)

__global__ void mc_store(float* mc, size_t n4, float v) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
        float* p = mc + 4 * i;
        float a = v + (float)(i & 1023);
        asm volatile("multimem.st.global.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(a), "f"(a), "f"(a), "f"(a) : "memory");
    }
}
__global__ void uc_store(float4* uc, size_t n4, float v) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
        float a = v + (float)(i & 1023);
        uc[i] = make_float4(a, a, a, a);
    }
}

int main() {
    CK(cuInit(0));
    CUdevice dev; CK(cuDeviceGet(&dev, 0));
    int mc = 0; CK(cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
    int ndev = 0; cudaGetDeviceCount(&ndev);
    printf("{\"multicast_supported\": %d, \"devices\": %d}\n", mc, ndev);
    if (!mc) return 0;
    cudaSetDevice(0); cudaFree(0);
    const size_t bytes = 1ull << 30;
    CUmulticastObjectProp mp = {};
    mp.numDevices = 1; mp.size = bytes; mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    size_t gran = 0; CK(cuMulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED));
    printf("{\"gran_recommended\": %zu}\n", gran);
    {   // which property combinations does cuMulticastCreate accept here?
        size_t gmin = 0; cuMulticastGetGranularity(&gmin, &mp, CU_MULTICAST_GRANULARITY_MINIMUM);
        const CUmemAllocationHandleType hts[3] = {CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, CU_MEM_HANDLE_TYPE_NONE, CU_MEM_HANDLE_TYPE_FABRIC};
        const size_t szs[3] = {gmin, gran, bytes};
        for (int h = 0; h < 3; ++h) for (int z = 0; z < 3; ++z) {
            CUmulticastObjectProp q = mp; q.handleTypes = hts[h]; q.size = szs[z];
            CUmemGenericAllocationHandle t; CUresult r = cuMulticastCreate(&t, &q);
            const char* es = nullptr; cuGetErrorString(r, &es);
            printf("{\"try_handle\": %d, \"size\": %zu, \"rc\": %d, \"err\": \"%s\"}\n", (int)hts[h], szs[z], (int)r, es ? es : "");
            if (r == CUDA_SUCCESS) cuMemRelease(t);
        }
    }
    for (unsigned nd = 2; nd <= 8; nd *= 2) {   // teams larger than the GPUs present
        CUmulticastObjectProp q = mp; q.numDevices = nd; q.size = gran;
        CUmemGenericAllocationHandle t; CUresult r = cuMulticastCreate(&t, &q);
        const char* es = nullptr; cuGetErrorString(r, &es);
        printf("{\"try_num_devices\": %u, \"rc\": %d, \"err\": \"%s\"}\n", nd, (int)r, es ? es : "");
        if (r == CUDA_SUCCESS) {
            CUresult ra = cuMulticastAddDevice(t, dev);
            CUmemAllocationProp pq = {};
            pq.type = CU_MEM_ALLOCATION_TYPE_PINNED; pq.location.type = CU_MEM_LOCATION_TYPE_DEVICE; pq.location.id = 0;
            pq.requestedHandleTypes = (CUmemAllocationHandleType)q.handleTypes;
            CUmemGenericAllocationHandle ph2; CUresult rc = cuMemCreate(&ph2, gran, &pq, 0);
            CUresult rb = rc == CUDA_SUCCESS ? cuMulticastBindMem(t, 0, ph2, 0, gran, 0) : rc;
            printf("{\"add_rc\": %d, \"create_rc\": %d, \"bind_rc\": %d}\n", (int)ra, (int)rc, (int)rb);
            if (rc == CUDA_SUCCESS) cuMemRelease(ph2);
            cuMemRelease(t);
        }
    }
    mp.handleTypes = CU_MEM_HANDLE_TYPE_NONE;
    CUmemGenericAllocationHandle mch; CK(cuMulticastCreate(&mch, &mp));
    CK(cuMulticastAddDevice(mch, dev));
    CUmemAllocationProp pp = {};
    pp.type = CU_MEM_ALLOCATION_TYPE_PINNED; pp.location.type = CU_MEM_LOCATION_TYPE_DEVICE; pp.location.id = 0;
    pp.requestedHandleTypes = CU_MEM_HANDLE_TYPE_NONE;
    CUmemGenericAllocationHandle ph; CK(cuMemCreate(&ph, bytes, &pp, 0));
    CK(cuMulticastBindMem(mch, 0, ph, 0, bytes, 0));
    CUdeviceptr uc, mcp;
    CK(cuMemAddressReserve(&uc, bytes, gran, 0, 0)); CK(cuMemMap(uc, bytes, 0, ph, 0));
    CK(cuMemAddressReserve(&mcp, bytes, gran, 0, 0)); CK(cuMemMap(mcp, bytes, 0, mch, 0));
    CUmemAccessDesc ad = {}; ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ad.location.id = 0; ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CK(cuMemSetAccess(uc, bytes, &ad, 1)); CK(cuMemSetAccess(mcp, bytes, &ad, 1));
    size_t n4 = bytes / 16;
    mc_store<<<148 * 8, 256>>>((float*)mcp, n4, 1.0f);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("{\"ok\": false, \"step\": \"mc_store\", \"err\": \"%s\"}\n", cudaGetErrorString(e)); return 0; }
    std::vector<float> h(4096);
    cudaMemcpy(h.data(), (void*)uc, h.size() * 4, cudaMemcpyDeviceToHost);
    int bad = 0; for (size_t i = 0; i < h.size(); ++i) bad += h[i] != 1.0f + (float)((i / 4) & 1023);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float tm = 0, tu = 0;
    for (int r = 0; r < 3; ++r) {
        cudaEventRecord(a); mc_store<<<148 * 8, 256>>>((float*)mcp, n4, 2.0f); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&tm, a, b);
        cudaEventRecord(a); uc_store<<<148 * 8, 256>>>((float4*)uc, n4, 3.0f); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&tu, a, b);
    }
    printf("{\"ok\": %s, \"mismatch\": %d, \"gran\": %zu, \"mc_store_GBps\": %.1f, \"uc_store_GBps\": %.1f}\n", bad ? "false" : "true", bad, gran,
           bytes / (tm * 1e6), bytes / (tu * 1e6));
    return 0;
}
