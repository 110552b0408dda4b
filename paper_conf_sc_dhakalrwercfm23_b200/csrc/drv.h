// CUDA driver entry points resolved at run time (cudaGetDriverEntryPointByVersion),
// so libmx.so loads on machines without a driver (host-only placement API) and
// fails loudly at mx_init instead of falling back.
#pragma once

#include <cuda.h>

namespace mx {

#define MX_DRV_FUNCS(X)            \
  X(cuInit)                        \
  X(cuDeviceGet)                   \
  X(cuDeviceGetCount)              \
  X(cuDeviceGetAttribute)          \
  X(cuDeviceTotalMem)              \
  X(cuDevicePrimaryCtxRetain)      \
  X(cuDevicePrimaryCtxRelease)     \
  X(cuCtxSetCurrent)               \
  X(cuCtxPushCurrent)              \
  X(cuCtxPopCurrent)               \
  X(cuDeviceGetDevResource)        \
  X(cuDevSmResourceSplitByCount)   \
  X(cuDevResourceGenerateDesc)     \
  X(cuGreenCtxCreate)              \
  X(cuGreenCtxDestroy)             \
  X(cuGreenCtxGetDevResource)      \
  X(cuCtxFromGreenCtx)             \
  X(cuGreenCtxStreamCreate)        \
  X(cuStreamCreate)                \
  X(cuStreamDestroy)               \
  X(cuStreamSynchronize)           \
  X(cuStreamWaitEvent)             \
  X(cuEventCreate)                 \
  X(cuEventDestroy)                \
  X(cuEventRecord)                 \
  X(cuEventQuery)                  \
  X(cuEventSynchronize)            \
  X(cuEventElapsedTime)            \
  X(cuMemcpyHtoDAsync)             \
  X(cuMemcpyDtoHAsync)             \
  X(cuMemcpyDtoH)                  \
  X(cuMemsetD8Async)               \
  X(cuMemAddressReserve)           \
  X(cuMemAddressFree)              \
  X(cuMemCreate)                   \
  X(cuMemRelease)                  \
  X(cuMemMap)                      \
  X(cuMemUnmap)                    \
  X(cuMemSetAccess)                \
  X(cuMemGetAllocationGranularity) \
  X(cuMemGetInfo)                  \
  X(cuMemHostAlloc)                \
  X(cuMemFreeHost)                 \
  X(cuMemHostGetDevicePointer)     \
  X(cuStreamQuery)                 \
  X(cuLaunchKernel)                \
  X(cuLaunchCooperativeKernel)     \
  X(cuKernelSetAttribute)          \
  X(cuTensorMapEncodeTiled)        \
  X(cuGetErrorString)

struct Drv {
#define MX_DECL(name) decltype(&::name) name = nullptr;
  MX_DRV_FUNCS(MX_DECL)
#undef MX_DECL
  bool loaded = false;
  // Resolve every entry point; returns false (with `why`) if any is missing.
  bool load(const char** why);
};

Drv& drv();

}  // namespace mx
