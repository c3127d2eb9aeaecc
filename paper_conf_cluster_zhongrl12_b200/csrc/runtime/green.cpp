// Green-context SM partitions (see green.hpp).
#include "runtime/green.hpp"

#include <mutex>

#include "common.hpp"

namespace fpm {
namespace {

struct DriverApi {
    CUresult (*DeviceGet)(CUdevice*, int) = nullptr;
    CUresult (*DeviceGetDevResource)(CUdevice, CUdevResource*, CUdevResourceType) = nullptr;
    CUresult (*DevSmResourceSplitByCount)(CUdevResource*, unsigned*, const CUdevResource*, CUdevResource*, unsigned,
                                          unsigned) = nullptr;
    CUresult (*DevResourceGenerateDesc)(CUdevResourceDesc*, CUdevResource*, unsigned) = nullptr;
    CUresult (*GreenCtxCreate)(CUgreenCtx*, CUdevResourceDesc, CUdevice, unsigned) = nullptr;
    CUresult (*GreenCtxDestroy)(CUgreenCtx) = nullptr;
    CUresult (*GreenCtxGetDevResource)(CUgreenCtx, CUdevResource*, CUdevResourceType) = nullptr;
    CUresult (*GreenCtxStreamCreate)(CUstream*, CUgreenCtx, unsigned, int) = nullptr;
    CUresult (*GetErrorString)(CUresult, const char**) = nullptr;
};

template <class F>
void load(F& fn, const char* name) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaError_t e = cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !p)
        fail(FPM_EUNSUPPORTED, "driver entry point %s unavailable (green contexts need CUDA 12.5+)", name);
    fn = reinterpret_cast<F>(p);
}

const DriverApi& api() {
    static DriverApi a;
    static std::once_flag once;
    static bool ok = false;
    std::call_once(once, [] {
        load(a.DeviceGet, "cuDeviceGet");
        load(a.DeviceGetDevResource, "cuDeviceGetDevResource");
        load(a.DevSmResourceSplitByCount, "cuDevSmResourceSplitByCount");
        load(a.DevResourceGenerateDesc, "cuDevResourceGenerateDesc");
        load(a.GreenCtxCreate, "cuGreenCtxCreate");
        load(a.GreenCtxDestroy, "cuGreenCtxDestroy");
        load(a.GreenCtxGetDevResource, "cuGreenCtxGetDevResource");
        load(a.GreenCtxStreamCreate, "cuGreenCtxStreamCreate");
        load(a.GetErrorString, "cuGetErrorString");
        ok = true;
    });
    if (!ok) fail(FPM_EUNSUPPORTED, "green-context driver API unavailable");
    return a;
}

void check(CUresult r, const char* what) {
    if (r == CUDA_SUCCESS) return;
    const char* s = "?";
    if (api().GetErrorString) api().GetErrorString(r, &s);
    fail(FPM_ECUDA, "%s: %s", what, s);
}

}  // namespace

std::vector<GreenPartition> green_partitions(int cuda_dev, const std::vector<int>& caps) {
    const DriverApi& a = api();
    cudaError_t ce = cudaSetDevice(cuda_dev);
    if (ce != cudaSuccess) fail(FPM_ECUDA, "cudaSetDevice(%d): %s", cuda_dev, cudaGetErrorString(ce));
    cudaFree(nullptr);  // primary context active first (cuGreenCtxCreate retains it)
    CUdevice dev;
    check(a.DeviceGet(&dev, cuda_dev), "cuDeviceGet");
    CUdevResource all;
    check(a.DeviceGetDevResource(dev, &all, CU_DEV_RESOURCE_TYPE_SM), "cuDeviceGetDevResource");
    // one split of the whole GPU into SM pairs (TPCs); co-scheduling hierarchy
    // ignored so partitions can be any even size -- CTA-pair clusters still land
    // on one TPC (measured)
    unsigned n = all.sm.smCount;
    std::vector<CUdevResource> groups(n);
    check(a.DevSmResourceSplitByCount(groups.data(), &n, &all, nullptr, CU_DEV_SM_RESOURCE_SPLIT_IGNORE_SM_COSCHEDULING,
                                      2),
          "cuDevSmResourceSplitByCount");
    unsigned need = 0;
    for (int c : caps) {
        if (c < 2 || c % 2 != 0)
            fail(FPM_EUNSUPPORTED, "green partition of %d SMs: must be even and >= 2 (SM pairs)", c);
        need += (unsigned)c / 2;
    }
    if (need > n)
        fail(FPM_EUNSUPPORTED, "green partitions of %u SMs in total do not fit the %u SM pairs of GPU %d", 2 * need, n,
             cuda_dev);
    std::vector<GreenPartition> out(caps.size());
    unsigned next = 0;
    try {
        for (size_t i = 0; i < caps.size(); ++i) {
            CUdevResourceDesc desc;
            check(a.DevResourceGenerateDesc(&desc, &groups[next], (unsigned)caps[i] / 2), "cuDevResourceGenerateDesc");
            next += (unsigned)caps[i] / 2;
            check(a.GreenCtxCreate(&out[i].ctx, desc, dev, CU_GREEN_CTX_DEFAULT_STREAM), "cuGreenCtxCreate");
            CUdevResource got;
            check(a.GreenCtxGetDevResource(out[i].ctx, &got, CU_DEV_RESOURCE_TYPE_SM), "cuGreenCtxGetDevResource");
            out[i].sms = (int)got.sm.smCount;
            if (out[i].sms != caps[i])
                fail(FPM_EUNSUPPORTED, "green partition got %d SMs, asked %d", out[i].sms, caps[i]);
        }
    } catch (...) {
        for (auto& g : out) green_destroy(g);
        throw;
    }
    return out;
}

cudaStream_t green_stream(const GreenPartition& g) {
    CUstream s = nullptr;
    check(api().GreenCtxStreamCreate(&s, g.ctx, CU_STREAM_NON_BLOCKING, 0), "cuGreenCtxStreamCreate");
    return reinterpret_cast<cudaStream_t>(s);
}

void green_destroy(GreenPartition& g) {
    if (g.ctx) api().GreenCtxDestroy(g.ctx);
    g.ctx = nullptr;
    g.sms = 0;
}

}  // namespace fpm
