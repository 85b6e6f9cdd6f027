// comm.cu — NCCL for the one exchange of the multi-GPU group-by (SURVEY §8(b) mr_group with
// R > 1, §8(e)): libnccl.so.2 is loaded at run time (the copy torch has already loaded when it is
// in the process, else BMR_NCCL_LIB, else the loader's libnccl.so.2), so libbmr.so has no link-time
// NCCL dependency and a single-GPU job never touches NCCL.  The communicator is created by the
// library (mr_comm_unique_id on rank 0, the 128-byte id broadcast by the caller, mr_comm_init on
// every rank) and handed to jobs through mr_config.nccl_comm.
#include <dlfcn.h>
#include <nccl.h>

#include <cstdlib>
#include <mutex>
#include <string>

#include "bmr.h"
#include "comm.h"

namespace bmr {

namespace {
NcclApi g_api;
std::once_flag g_once;

template <typename F>
bool sym(void* h, const char* name, F& f) {
  f = reinterpret_cast<F>(dlsym(h, name));
  return f != nullptr;
}

void load() {
  void* h = nullptr;
  const char* env = getenv("BMR_NCCL_LIB");
  if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_LOCAL);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);   // torch's copy, if loaded
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
  if (!h) {
    const char* e = dlerror();
    g_api.err = std::string("cannot load libnccl.so.2: ") + (e ? e : "?");
    return;
  }
  bool ok = sym(h, "ncclGetUniqueId", g_api.GetUniqueId) && sym(h, "ncclCommInitRank", g_api.CommInitRank) &&
            sym(h, "ncclCommDestroy", g_api.CommDestroy) && sym(h, "ncclSend", g_api.Send) &&
            sym(h, "ncclRecv", g_api.Recv) && sym(h, "ncclGroupStart", g_api.GroupStart) &&
            sym(h, "ncclGroupEnd", g_api.GroupEnd) && sym(h, "ncclGetErrorString", g_api.GetErrorString) &&
            sym(h, "ncclGetVersion", g_api.GetVersion);
  if (!ok) {
    g_api.err = "libnccl.so.2 lacks a required symbol";
    return;
  }
  sym(h, "ncclAlltoAll", g_api.AlltoAll);   // NCCL >= 2.28; else grouped send/recv
  g_api.GetVersion(&g_api.version);
  g_api.ok = true;
}
}  // namespace

const NcclApi* nccl_api() {
  std::call_once(g_once, load);
  return &g_api;
}

std::string nccl_error(const NcclApi* a, int r) {
  return a && a->GetErrorString ? a->GetErrorString(static_cast<ncclResult_t>(r)) : "nccl error " + std::to_string(r);
}

// counts[r] (2 u64 per rank: entries, heap bytes) -> recv[r] of every rank: the count exchange
cudaError_t nccl_alltoall_u64x2(const NcclApi* a, const uint64_t* send, uint64_t* recv, int nranks, void* comm,
                                cudaStream_t s, int* nres) {
  ncclComm_t c = static_cast<ncclComm_t>(comm);
  ncclResult_t r;
  if (a->AlltoAll) {
    r = a->AlltoAll(send, recv, 2, ncclUint64, c, s);
  } else {
    r = a->GroupStart();
    for (int p = 0; p < nranks && r == ncclSuccess; ++p) {
      r = a->Send(send + 2 * p, 2, ncclUint64, p, c, s);
      if (r == ncclSuccess) r = a->Recv(recv + 2 * p, 2, ncclUint64, p, c, s);
    }
    const ncclResult_t r2 = a->GroupEnd();
    if (r == ncclSuccess) r = r2;
  }
  *nres = static_cast<int>(r);
  return cudaSuccess;
}

// Variable all-to-all of two byte streams (entries, heap): slice p of each send buffer goes to
// rank p, slice p of each receive buffer comes from rank p.  One NCCL group.
int nccl_alltoallv2(const NcclApi* a, const uint8_t* se, const uint64_t* se_off, uint8_t* re, const uint64_t* re_off,
                    const uint8_t* sh, const uint64_t* sh_off, uint8_t* rh, const uint64_t* rh_off, int nranks,
                    void* comm, cudaStream_t s) {
  ncclComm_t c = static_cast<ncclComm_t>(comm);
  ncclResult_t r = a->GroupStart();
  for (int p = 0; p < nranks && r == ncclSuccess; ++p) {
    const uint64_t ne = se_off[p + 1] - se_off[p], me = re_off[p + 1] - re_off[p];
    const uint64_t nh = sh_off[p + 1] - sh_off[p], mh = rh_off[p + 1] - rh_off[p];
    if (ne && r == ncclSuccess) r = a->Send(se + se_off[p], ne, ncclUint8, p, c, s);
    if (me && r == ncclSuccess) r = a->Recv(re + re_off[p], me, ncclUint8, p, c, s);
    if (nh && r == ncclSuccess) r = a->Send(sh + sh_off[p], nh, ncclUint8, p, c, s);
    if (mh && r == ncclSuccess) r = a->Recv(rh + rh_off[p], mh, ncclUint8, p, c, s);
  }
  const ncclResult_t r2 = a->GroupEnd();
  return static_cast<int>(r == ncclSuccess ? r2 : r);
}

}  // namespace bmr

using namespace bmr;

extern "C" {

mr_status mr_comm_unique_id(void* id) {
  if (!id) return MR_ERR_INVALID;
  const NcclApi* a = nccl_api();
  if (!a->ok) return MR_ERR_NCCL;
  ncclUniqueId u;
  if (a->GetUniqueId(&u) != ncclSuccess) return MR_ERR_NCCL;
  static_assert(sizeof(u) == MR_NCCL_ID_BYTES, "NCCL unique id size");
  memcpy(id, &u, sizeof(u));
  return MR_OK;
}

mr_status mr_comm_init(const void* id, int nranks, int rank, int device, void** comm) {
  if (!id || !comm || nranks < 1 || rank < 0 || rank >= nranks) return MR_ERR_INVALID;
  *comm = nullptr;
  const NcclApi* a = nccl_api();
  if (!a->ok) return MR_ERR_NCCL;
  if (cudaSetDevice(device) != cudaSuccess) {
    cudaGetLastError();
    return MR_ERR_CUDA;
  }
  ncclUniqueId u;
  memcpy(&u, id, sizeof(u));
  ncclComm_t c = nullptr;
  if (a->CommInitRank(&c, nranks, u, rank) != ncclSuccess) return MR_ERR_NCCL;
  *comm = c;
  return MR_OK;
}

mr_status mr_comm_destroy(void* comm) {
  if (!comm) return MR_OK;
  const NcclApi* a = nccl_api();
  if (!a->ok) return MR_ERR_NCCL;
  return a->CommDestroy(static_cast<ncclComm_t>(comm)) == ncclSuccess ? MR_OK : MR_ERR_NCCL;
}

const char* mr_comm_backend(void) {
  static std::string s;
  const NcclApi* a = nccl_api();
  s = a->ok ? "nccl " + std::to_string(a->version) + (a->AlltoAll ? " (ncclAlltoAll)" : " (send/recv)") : a->err;
  return s.c_str();
}

}  // extern "C"
