// comm.h — run-time loaded NCCL entry points used by the exchange in mr_group (comm.cu).
#pragma once
#include <cstdint>
#include <string>

#include <cuda_runtime.h>
#include <nccl.h>

namespace bmr {

struct NcclApi {
  bool ok = false;
  std::string err;
  int version = 0;
  decltype(&ncclGetUniqueId) GetUniqueId = nullptr;
  decltype(&ncclCommInitRank) CommInitRank = nullptr;
  decltype(&ncclCommDestroy) CommDestroy = nullptr;
  decltype(&ncclSend) Send = nullptr;
  decltype(&ncclRecv) Recv = nullptr;
  decltype(&ncclGroupStart) GroupStart = nullptr;
  decltype(&ncclGroupEnd) GroupEnd = nullptr;
  decltype(&ncclGetErrorString) GetErrorString = nullptr;
  decltype(&ncclGetVersion) GetVersion = nullptr;
  decltype(&ncclAlltoAll) AlltoAll = nullptr;   // optional (NCCL >= 2.28)
};

const NcclApi* nccl_api();
std::string nccl_error(const NcclApi* a, int r);
cudaError_t nccl_alltoall_u64x2(const NcclApi* a, const uint64_t* send, uint64_t* recv, int nranks, void* comm,
                                cudaStream_t s, int* nres);
int nccl_alltoallv2(const NcclApi* a, const uint8_t* se, const uint64_t* se_off, uint8_t* re, const uint64_t* re_off,
                    const uint8_t* sh, const uint64_t* sh_off, uint8_t* rh, const uint64_t* rh_off, int nranks,
                    void* comm, cudaStream_t s);

}  // namespace bmr
