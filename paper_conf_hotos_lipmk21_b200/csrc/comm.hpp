// comm.hpp — NCCL, loaded with dlopen at harmony_init (world_size > 1) or harmony_get_unique_id.
// The library therefore loads (and its CPU tests run) on hosts without NCCL or a GPU.
// Path: $HARMONY_NCCL_PATH (set by the Python binding to the venv's nvidia/nccl/lib/libnccl.so.2),
// else the soname "libnccl.so.2".
#pragma once
#include <dlfcn.h>
#include <stdlib.h>

#include <mutex>
#include <string>

#include "nccl.h"

namespace hm {

struct NcclApi {
  void* lib = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*ReduceScatter)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                                cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  std::string err;

  bool load() {
    if (lib) return true;
    const char* env = getenv("HARMONY_NCCL_PATH");
    if (env && *env) lib = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
    if (!lib) lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!lib) {
      const char* e = dlerror();
      err = std::string("cannot dlopen libnccl.so.2: ") + (e ? e : "?");
      return false;
    }
#define HM_SYM(name, sym)                                                   \
  name = reinterpret_cast<decltype(name)>(dlsym(lib, sym));                 \
  if (!name) { err = std::string("missing NCCL symbol ") + sym; return false; }
    HM_SYM(GetUniqueId, "ncclGetUniqueId");
    HM_SYM(CommInitRank, "ncclCommInitRank");
    HM_SYM(CommDestroy, "ncclCommDestroy");
    HM_SYM(AllGather, "ncclAllGather");
    HM_SYM(ReduceScatter, "ncclReduceScatter");
    HM_SYM(AllReduce, "ncclAllReduce");
    HM_SYM(GetErrorString, "ncclGetErrorString");
#undef HM_SYM
    return true;
  }
};

inline NcclApi& nccl() {
  static NcclApi api;
  return api;
}

}  // namespace hm
