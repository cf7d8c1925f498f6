// nccl_dl.h -- NCCL loaded at run time (dlopen libnccl.so.2), so libtqr.so loads and runs
// single-process plans on machines without NCCL and never pins a second NCCL next to the
// one PyTorch already loaded (same soname -> the already-mapped library is reused).
#pragma once
#include <nccl.h>

namespace tqr {

struct NcclApi {
    bool ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
    ncclResult_t (*CommAbort)(ncclComm_t) = nullptr;
    ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

// Returns nullptr (with *why set) when libnccl.so.2 or a symbol is missing.
const NcclApi* nccl_api(const char** why);

}  // namespace tqr
