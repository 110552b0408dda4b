#include "arena.h"

#include "../../include/mx.h"
#include "drv.h"

namespace mx {

static CUmemAllocationProp device_prop(int ordinal) {
  CUmemAllocationProp p = {};
  p.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  p.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  p.location.id = ordinal;
  return p;
}

int Arena::init(int ordinal, uint64_t quota, uint64_t va_bytes) {
  ordinal_ = ordinal;
  quota_ = quota;
  CUmemAllocationProp prop = device_prop(ordinal);
  size_t g = 0;
  if (drv().cuMemGetAllocationGranularity(&g, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) !=
      CUDA_SUCCESS)
    return MX_EDEVICE;
  gran_ = g;
  va_ = (va_bytes + gran_ - 1) / gran_ * gran_;
  if (drv().cuMemAddressReserve(&base_, va_, gran_, 0, 0) != CUDA_SUCCESS) return MX_ENOMEM;
  return MX_OK;
}

int Arena::map_to(uint64_t end) {
  if (mapped_ >= end) return MX_OK;
  // one physical allocation per extension (rounded to the granularity)
  const uint64_t size = (end - mapped_ + gran_ - 1) / gran_ * gran_;
  CUmemAllocationProp prop = device_prop(ordinal_);
  CUmemGenericAllocationHandle h;
  if (drv().cuMemCreate(&h, size, &prop, 0) != CUDA_SUCCESS) return MX_ENOMEM;
  if (drv().cuMemMap(base_ + mapped_, size, 0, h, 0) != CUDA_SUCCESS) {
    drv().cuMemRelease(h);
    return MX_EDEVICE;
  }
  CUmemAccessDesc acc = {};
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = ordinal_;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  if (drv().cuMemSetAccess(base_ + mapped_, size, &acc, 1) != CUDA_SUCCESS) {
    drv().cuMemUnmap(base_ + mapped_, size);
    drv().cuMemRelease(h);
    return MX_EDEVICE;
  }
  chunks_.push_back({h, mapped_, size});
  mapped_ += size;
  return MX_OK;
}

int Arena::alloc(uint64_t bytes, uint64_t align, CUdeviceptr* out) {
  if (align == 0) align = 256;
  uint64_t off = (used_ + align - 1) / align * align;
  uint64_t end = off + bytes;
  if (end > quota_ || end > va_) return MX_ENOMEM;
  int rc = map_to(end);
  if (rc) return rc;
  used_ = end;
  if (used_ > peak_) peak_ = used_;
  *out = base_ + off;
  return MX_OK;
}

int Arena::set_quota(uint64_t q) {
  if (used_ > q) return MX_EBUSY;
  if (q > va_) return MX_ENOMEM;
  quota_ = q;
  return MX_OK;
}

void Arena::release() {
  if (!base_) return;
  for (const Chunk& c : chunks_) {
    drv().cuMemUnmap(base_ + c.off, c.size);
    drv().cuMemRelease(c.h);
  }
  chunks_.clear();
  drv().cuMemAddressFree(base_, va_);
  base_ = 0;
  mapped_ = used_ = 0;
}

}  // namespace mx
