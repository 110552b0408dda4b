// Placement engine: SM-group allocation, HBM quota sums, deterministic task
// placement and the canonical trace (§4.1
// GPU% per listed accelerator, §4.2 P:181 MIG slices, Fig. 4 P:195 equal division).
// Pure C++ with no CUDA dependency: the runtime owns one instance and every
// part_create / part_resize / part_destroy / fn_submit goes through it.
#pragma once

#include <cstdint>
#include <string>
#include <vector>

namespace mx {

enum RecType : uint64_t { REC_HEADER = 0, REC_CREATE = 1, REC_RESIZE = 2, REC_DESTROY = 3, REC_PLACE = 4 };
constexpr uint64_t kTraceVersion = 1;

struct SchedPart {
  int32_t gpu = 0;
  std::vector<int> groups;   // ascending group indices
  int32_t sm_count = 0;
  bool whole = false;
  bool shared = false;       // N1: no SM groups; runs anywhere on the device (sm_count = grid)
  uint64_t quota = 0;
  uint32_t epoch = 0;
  bool live = false;
  uint64_t assigned = 0;     // A_p: never decremented (timing-independent placement)
  uint64_t seq = 0;          // next seq_in_part
  uint64_t mask() const {
    uint64_t m = 0;
    for (int g : groups) m |= (1ull << g);
    return m;
  }
};

struct Placement {
  uint64_t task;
  int32_t gpu, part;
  uint64_t seq;
  uint32_t epoch;
};

class Sched {
 public:
  Sched(int n_gpus, int n_groups, int group_size, int total_sms, uint64_t mem_bytes);
  // All return an mx_status code (0 ok).
  int create(int gpu, int sm, uint64_t hbm, int* out_part);
  // Unpartitioned ("shared") partition: a stream on the whole device that owns
  // no SM groups (not counted in I2); n_ctas is its grid size and its WLAW weight.
  int create_shared(int gpu, int n_ctas, uint64_t hbm, int* out_part);
  int plan_create_shared(int gpu, int n_ctas, uint64_t hbm) const;
  int resize(int part, int sm, uint64_t hbm);
  int destroy(int part);
  int submit(int fn, int part, uint64_t cost, Placement* out);
  // Validation without mutation (the runtime checks before touching the device).
  int plan_create(int gpu, int sm, uint64_t hbm, std::vector<int>* groups, int* smc, bool* whole) const;
  int plan_resize(int part, int sm, uint64_t hbm, std::vector<int>* groups, int* smc, bool* whole,
                  uint64_t* quota) const;
  const SchedPart& part(int p) const { return parts_[p]; }
  bool is_live(int p) const { return p >= 0 && p < (int)parts_.size() && parts_[p].live; }
  int n_parts() const { return (int)parts_.size(); }
  std::vector<uint8_t> trace_bytes() const;

 private:
  int alloc(int gpu, int sm, int exclude, std::vector<int>* groups, int* smc, bool* whole) const;
  bool quota_ok(int gpu, uint64_t quota, int exclude) const;
  uint64_t flags(const SchedPart& p) const { return (p.whole ? 1u : 0u) | (p.shared ? 2u : 0u); }
  void record(uint64_t a, uint64_t b, uint64_t c, uint64_t d, uint64_t e, uint64_t f, uint64_t g, uint64_t h);

  int n_gpus_, n_groups_, group_size_, total_sms_;
  uint64_t mem_bytes_;
  std::vector<SchedPart> parts_;
  std::vector<uint64_t> records_;   // 8 words per record
  uint64_t next_task_ = 1;
};

}  // namespace mx
