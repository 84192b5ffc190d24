// nccl_dl.h -- NCCL loaded at run time (dlopen "libnccl.so.2").
//
// The process already holds torch's NCCL (2.28.9, bundled in the venv); a
// dlopen by soname returns that same copy, so there is one NCCL per process
// and the library does not need NCCL at all for world_size == 1.
#pragma once

#include <dlfcn.h>
#include <nccl.h>

namespace ratel {

struct NcclApi {
  void* handle = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;

  // Returns nullptr on success, else a message.
  const char* load() {
    if (handle != nullptr) return nullptr;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (h == nullptr) return dlerror();
#define RATEL_NCCL_SYM(field, name)                                  \
  field = reinterpret_cast<decltype(field)>(dlsym(h, name));         \
  if (field == nullptr) return "libnccl.so.2 lacks symbol " name;
    RATEL_NCCL_SYM(GetUniqueId, "ncclGetUniqueId")
    RATEL_NCCL_SYM(CommInitRank, "ncclCommInitRank")
    RATEL_NCCL_SYM(AllReduce, "ncclAllReduce")
    RATEL_NCCL_SYM(AllGather, "ncclAllGather")
    RATEL_NCCL_SYM(CommDestroy, "ncclCommDestroy")
    RATEL_NCCL_SYM(CommGetAsyncError, "ncclCommGetAsyncError")
    RATEL_NCCL_SYM(GetErrorString, "ncclGetErrorString")
    RATEL_NCCL_SYM(GroupStart, "ncclGroupStart")
    RATEL_NCCL_SYM(GroupEnd, "ncclGroupEnd")
#undef RATEL_NCCL_SYM
    handle = h;
    return nullptr;
  }
};

}  // namespace ratel
