// Green contexts: disjoint SM partitions of one GPU (CUDA driver API, reached
// through cudaGetDriverEntryPoint so the library needs no -lcuda).  Used to
// emulate heterogeneous devices (BASELINE.json north_star: "Heterogeneity is
// emulated by capping SMs per GPU (green contexts)"): every kernel a device
// launches -- update, staging, NCCL -- runs inside its own SMs.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <vector>

namespace fpm {

struct GreenPartition {
    CUgreenCtx ctx = nullptr;
    int sms = 0;  // SMs provisioned (as reported by the driver)
};

// Carve disjoint partitions of caps[i] SMs (even, >= 2) out of CUDA device
// `cuda_dev`, all from one split (TPC granularity: pairs of SMs, so CTA-pair
// clusters stay schedulable).  FPM_EUNSUPPORTED if they do not fit.
std::vector<GreenPartition> green_partitions(int cuda_dev, const std::vector<int>& caps);

// A non-blocking stream whose kernels run on the partition's SMs only.
cudaStream_t green_stream(const GreenPartition& g);

void green_destroy(GreenPartition& g);

}  // namespace fpm
