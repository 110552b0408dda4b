// Per-partition HBM arena with a quota (the MIG memory-slice analog: PAPER.md
// Table 1 P:136 "Compute and memory isolation"; §4.2 P:181 "1g.10gb ... 10 GB
// of GPU memory"; reading A23 — a capacity limit enforced by this allocator,
// not bandwidth or fault isolation).
//
// CUDA VMM: one virtual range is reserved per partition (device-memory sized,
// so the quota can grow in place), physical chunks of the allocation
// granularity are created and mapped on demand as the bump pointer advances.
// used = bytes handed out, peak = max used; an allocation that would take used
// above the quota fails with MX_ENOMEM and changes nothing.
#pragma once

#include <cstdint>
#include <vector>

#include <cuda.h>

namespace mx {

class Arena {
 public:
  int init(int ordinal, uint64_t quota, uint64_t va_bytes);   // mx_status
  void release();
  // Allocate `bytes` aligned to `align` (<= granularity). MX_ENOMEM over quota.
  int alloc(uint64_t bytes, uint64_t align, CUdeviceptr* out);
  int set_quota(uint64_t q);   // MX_EBUSY if used > q
  uint64_t quota() const { return quota_; }
  uint64_t used() const { return used_; }
  uint64_t peak() const { return peak_; }
  uint64_t mapped() const { return mapped_; }

 private:
  int map_to(uint64_t end);
  int ordinal_ = 0;
  CUdeviceptr base_ = 0;
  uint64_t va_ = 0, gran_ = 0, quota_ = 0, used_ = 0, peak_ = 0, mapped_ = 0;
  struct Chunk { CUmemGenericAllocationHandle h; uint64_t off, size; };
  std::vector<Chunk> chunks_;
};

}  // namespace mx
