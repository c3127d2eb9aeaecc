// NCCL entry points resolved at run time (dlopen "libnccl.so.2"), so the
// library loads on machines without NCCL and shares the process's NCCL copy
// (PyTorch's, when torch was imported first).  Types come from nccl.h.
#pragma once

#include <nccl.h>

namespace fpm {

struct NcclApi {
    ncclResult_t (*GetUniqueId)(ncclUniqueId*);
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int);
    ncclResult_t (*CommInitRankConfig)(ncclComm_t*, int, ncclUniqueId, int, ncclConfig_t*);
    ncclResult_t (*CommCount)(const ncclComm_t, int*);
    ncclResult_t (*CommAbort)(ncclComm_t);
    ncclResult_t (*CommSplit)(ncclComm_t, int, int, ncclComm_t*, ncclConfig_t*);
    ncclResult_t (*CommDestroy)(ncclComm_t);
    ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*);
    ncclResult_t (*GroupStart)();
    ncclResult_t (*GroupEnd)();
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    const char* (*GetErrorString)(ncclResult_t);
};

// Loads once; throws fpm::Error(FPM_ENCCL) if NCCL is unavailable.
const NcclApi& nccl();

}  // namespace fpm
