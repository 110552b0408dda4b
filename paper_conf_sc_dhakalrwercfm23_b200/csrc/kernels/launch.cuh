// Kernel launches go through the driver entry point cuLaunchKernel with
// context-less CUkernel handles (cudaGetKernel): the launch context is taken
// from the stream, i.e. the partition's green context (cuda.h: cuLaunchKernel,
// "the context to launch the kernel on will ... be taken from the specified
// stream"). Driver entry points are resolved at mx_init through
// cudaGetDriverEntryPointByVersion, so libmx.so never links libcuda directly.
#pragma once

#include <atomic>
#include <cuda.h>
#include <cuda_runtime.h>

namespace mxk {

struct DriverLaunch {
  CUresult (*launch)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                     unsigned, CUstream, void**, void**) = nullptr;
  CUresult (*launch_coop)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                          unsigned, CUstream, void**) = nullptr;
  CUresult (*kernel_set_attr)(CUfunction_attribute, int, CUkernel, CUdevice) = nullptr;
};

DriverLaunch& driver_launch();
std::atomic<uint64_t>& launch_count_ref();

template <typename K>
inline int launch_kernel(K* kern, dim3 grid, dim3 block, unsigned smem, void* stream, void** args,
                         bool cooperative = false) {
  cudaKernel_t k = nullptr;
  if (cudaGetKernel(&k, reinterpret_cast<const void*>(kern)) != cudaSuccess || !k) return -1;
  DriverLaunch& d = driver_launch();
  if (!d.launch || (cooperative && !d.launch_coop)) return -2;
  CUresult r = cooperative
                   ? d.launch_coop(reinterpret_cast<CUfunction>(k), grid.x, grid.y, grid.z, block.x,
                                   block.y, block.z, smem, reinterpret_cast<CUstream>(stream), args)
                   : d.launch(reinterpret_cast<CUfunction>(k), grid.x, grid.y, grid.z, block.x,
                              block.y, block.z, smem, reinterpret_cast<CUstream>(stream), args,
                              nullptr);
  if (r != CUDA_SUCCESS) return (int)r;
  launch_count_ref().fetch_add(1, std::memory_order_relaxed);
  return 0;
}

template <typename K>
inline int set_max_smem(K* kern, int bytes, int device) {
  cudaKernel_t k = nullptr;
  if (cudaGetKernel(&k, reinterpret_cast<const void*>(kern)) != cudaSuccess || !k) return -1;
  DriverLaunch& d = driver_launch();
  if (!d.kernel_set_attr) return -2;
  return (int)d.kernel_set_attr(CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, bytes,
                                reinterpret_cast<CUkernel>(k), (CUdevice)device);
}

}  // namespace mxk
