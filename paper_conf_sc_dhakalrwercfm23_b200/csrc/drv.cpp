#include "drv.h"

#include <cuda_runtime.h>

namespace mx {

Drv& drv() {
  static Drv d;
  return d;
}

bool Drv::load(const char** why) {
  if (loaded) return true;
  cudaDriverEntryPointQueryResult q;
#define MX_LOAD(name)                                                                          \
  {                                                                                            \
    void* fp = nullptr;                                                                        \
    if (cudaGetDriverEntryPointByVersion(#name, &fp, CUDA_VERSION, cudaEnableDefault, &q) !=   \
            cudaSuccess ||                                                                     \
        q != cudaDriverEntryPointSuccess || !fp) {                                             \
      if (why) *why = "driver entry point missing: " #name;                                    \
      return false;                                                                            \
    }                                                                                          \
    name = reinterpret_cast<decltype(name)>(fp);                                               \
  }
  MX_DRV_FUNCS(MX_LOAD)
#undef MX_LOAD
  loaded = true;
  return true;
}

}  // namespace mx
