// dynload.h -- NCCL and cuBLAS loaded with dlopen on demand (element split, tensor cache)
#pragma once
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <mutex>

namespace landau {

// ------------------------------------------------------------------------------------------------
// NCCL, loaded on demand (only LANDAU_DIST_ELEMENTS needs it)
// ------------------------------------------------------------------------------------------------
typedef struct {
  char internal[128];
} ncclUniqueId_;
typedef void *ncclComm_;
struct NcclApi {
  void *so = nullptr;
  int (*GetUniqueId)(ncclUniqueId_ *) = nullptr;
  int (*CommInitRank)(ncclComm_ *, int, ncclUniqueId_, int) = nullptr;
  int (*AllGather)(const void *, void *, size_t, int, ncclComm_, cudaStream_t) = nullptr;
  int (*AllReduce)(const void *, void *, size_t, int, int, ncclComm_, cudaStream_t) = nullptr;
  int (*CommDestroy)(ncclComm_) = nullptr;
  const char *(*GetErrorString)(int) = nullptr;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;
bool load_nccl() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (g_nccl.so) return true;
  const char *names[] = {"libnccl.so.2", "libnccl.so"};
  void *so = nullptr;
  for (const char *n : names)
    if ((so = dlopen(n, RTLD_NOW | RTLD_GLOBAL))) break;
  if (!so) return false;
  g_nccl.GetUniqueId = (int (*)(ncclUniqueId_ *))dlsym(so, "ncclGetUniqueId");
  g_nccl.CommInitRank = (int (*)(ncclComm_ *, int, ncclUniqueId_, int))dlsym(so, "ncclCommInitRank");
  g_nccl.AllGather = (int (*)(const void *, void *, size_t, int, ncclComm_, cudaStream_t))dlsym(so, "ncclAllGather");
  g_nccl.AllReduce = (int (*)(const void *, void *, size_t, int, int, ncclComm_, cudaStream_t))dlsym(so, "ncclAllReduce");
  g_nccl.CommDestroy = (int (*)(ncclComm_))dlsym(so, "ncclCommDestroy");
  g_nccl.GetErrorString = (const char *(*)(int))dlsym(so, "ncclGetErrorString");
  if (!g_nccl.GetUniqueId || !g_nccl.CommInitRank || !g_nccl.AllGather || !g_nccl.AllReduce || !g_nccl.CommDestroy)
    return false;
  g_nccl.so = so;
  return true;
}
constexpr int kNcclFloat64 = 8;
constexpr int kNcclSum = 0;

// cuBLAS, loaded on demand (only the tensor-cache path uses it: a plain library DGEMM)
typedef void *cublasHandle_;
struct CublasApi {
  void *so = nullptr;
  int (*Create)(cublasHandle_ *) = nullptr;
  int (*Destroy)(cublasHandle_) = nullptr;
  int (*SetStream)(cublasHandle_, cudaStream_t) = nullptr;
  int (*Dgemm)(cublasHandle_, int, int, int, int, int, const double *, const double *, int, const double *, int,
               const double *, double *, int) = nullptr;
};
CublasApi g_cublas;
std::mutex g_cublas_mu;
bool load_cublas() {
  std::lock_guard<std::mutex> lk(g_cublas_mu);
  if (g_cublas.so) return true;
  void *so = nullptr;
  for (const char *n : {"libcublas.so.12", "libcublas.so"})
    if ((so = dlopen(n, RTLD_NOW | RTLD_GLOBAL))) break;
  if (!so) return false;
  g_cublas.Create = (int (*)(cublasHandle_ *))dlsym(so, "cublasCreate_v2");
  g_cublas.Destroy = (int (*)(cublasHandle_))dlsym(so, "cublasDestroy_v2");
  g_cublas.SetStream = (int (*)(cublasHandle_, cudaStream_t))dlsym(so, "cublasSetStream_v2");
  g_cublas.Dgemm = (int (*)(cublasHandle_, int, int, int, int, int, const double *, const double *, int, const double *,
                            int, const double *, double *, int))dlsym(so, "cublasDgemm_v2");
  if (!g_cublas.Create || !g_cublas.Destroy || !g_cublas.SetStream || !g_cublas.Dgemm) return false;
  g_cublas.so = so;
  return true;
}

thread_local std::string g_create_error;


}  // namespace landau
