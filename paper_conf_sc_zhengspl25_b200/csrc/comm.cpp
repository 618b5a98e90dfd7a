// comm.cpp -- the optional native NCCL path of the C-ABI (SURVEY 8(b)
// magus_comm_init): one communicator per context, and the sweep's single
// collective -- an in-place uint64 SUM all-reduce of the per-config totals
// over NVLink / NVSwitch (north_star (3)).
//
// NCCL is opened lazily with dlopen("libnccl.so.2") on the first call, so
// the library has no link-time NCCL dependency and, inside a process that
// already loaded PyTorch, shares the NCCL that torch loaded (one libnccl per
// process).  Only <nccl.h>'s types are used at compile time.
#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
#include <mutex>

#include "magus_internal.h"

namespace magus {
namespace {

struct NcclApi {
  bool tried = false, ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi& api() {
  static NcclApi a;
  static std::mutex m;
  std::lock_guard<std::mutex> lk(m);
  if (!a.tried) {
    a.tried = true;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (h) {
      a.GetUniqueId = (decltype(a.GetUniqueId))dlsym(h, "ncclGetUniqueId");
      a.CommInitRank = (decltype(a.CommInitRank))dlsym(h, "ncclCommInitRank");
      a.CommDestroy = (decltype(a.CommDestroy))dlsym(h, "ncclCommDestroy");
      a.AllReduce = (decltype(a.AllReduce))dlsym(h, "ncclAllReduce");
      a.GetErrorString = (decltype(a.GetErrorString))dlsym(h, "ncclGetErrorString");
      a.ok = a.GetUniqueId && a.CommInitRank && a.CommDestroy && a.AllReduce && a.GetErrorString;
    }
  }
  return a;
}

}  // namespace

static_assert(sizeof(ncclUniqueId) == MAGUS_COMM_ID_BYTES, "ncclUniqueId size");

bool nccl_available() { return api().ok; }

const char* nccl_error(int r) { return api().ok ? api().GetErrorString((ncclResult_t)r) : "libnccl.so.2 not found"; }

int nccl_unique_id(void* out) {
  if (!api().ok) return -1;
  ncclUniqueId id;
  const ncclResult_t r = api().GetUniqueId(&id);
  if (r != ncclSuccess) return (int)r;
  std::memcpy(out, &id, sizeof(id));
  return 0;
}

int nccl_comm_init(void** comm, const void* id_bytes, int nranks, int rank) {
  if (!api().ok) return -1;
  ncclUniqueId id;
  std::memcpy(&id, id_bytes, sizeof(id));
  ncclComm_t c = nullptr;
  const ncclResult_t r = api().CommInitRank(&c, nranks, id, rank);
  if (r != ncclSuccess) return (int)r;
  *comm = c;
  return 0;
}

int nccl_comm_destroy(void* comm) {
  if (!comm || !api().ok) return 0;
  return (int)api().CommDestroy((ncclComm_t)comm);
}

int nccl_allreduce_u64_sum(void* comm, uint64_t* buf, size_t count, cudaStream_t s) {
  if (!api().ok) return -1;
  return (int)api().AllReduce(buf, buf, count, ncclUint64, ncclSum, (ncclComm_t)comm, s);
}

}  // namespace magus
