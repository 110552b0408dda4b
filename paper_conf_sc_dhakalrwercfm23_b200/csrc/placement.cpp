// Placement engine implementation — see placement.h. Rules:
//  * k = ceil(sm / group_size) lowest-index free groups; sm >= total_sms (or k >
//    n_groups) = the whole device, which needs every group free (A20).
//  * resize releases the partition's own groups first, then reallocates.
//  * I5: sum of live quotas per GPU <= device memory.
//  * ANY: weighted least-assigned-work, argmin (A_p + c)/s_p compared exactly
//    in 128-bit integers, ties -> lowest part id; A_p += c for every placement.
//  * STATIC equal division (A6) is done by the caller with explicit parts.
//  * shared partitions (N1, unpartitioned comparison modes) own no groups; their
//    sm_count is the grid size (<= total_sms); record flag word: bit0 whole, bit1 shared.
#include "placement.h"

#include "../../include/mx.h"

namespace mx {

Sched::Sched(int n_gpus, int n_groups, int group_size, int total_sms, uint64_t mem_bytes)
    : n_gpus_(n_gpus), n_groups_(n_groups), group_size_(group_size), total_sms_(total_sms),
      mem_bytes_(mem_bytes) {
  record(REC_HEADER, kTraceVersion, (uint64_t)n_gpus, (uint64_t)n_groups, (uint64_t)group_size,
         (uint64_t)total_sms, 0, 0);
}

void Sched::record(uint64_t a, uint64_t b, uint64_t c, uint64_t d, uint64_t e, uint64_t f,
                   uint64_t g, uint64_t h) {
  uint64_t r[8] = {a, b, c, d, e, f, g, h};
  records_.insert(records_.end(), r, r + 8);
}

int Sched::alloc(int gpu, int sm, int exclude, std::vector<int>* groups, int* smc,
                 bool* whole) const {
  std::vector<bool> used(n_groups_, false);
  for (int p = 0; p < (int)parts_.size(); ++p) {
    const SchedPart& q = parts_[p];
    if (!q.live || q.gpu != gpu || p == exclude) continue;
    for (int g : q.groups) used[g] = true;
  }
  std::vector<int> free;
  for (int g = 0; g < n_groups_; ++g)
    if (!used[g]) free.push_back(g);
  int k = (sm + group_size_ - 1) / group_size_;
  if (sm >= total_sms_ || k > n_groups_) {
    if ((int)free.size() != n_groups_) return MX_ENOSM;
    *groups = free;
    *smc = total_sms_;
    *whole = true;
    return MX_OK;
  }
  if ((int)free.size() < k) return MX_ENOSM;
  groups->assign(free.begin(), free.begin() + k);
  *smc = k * group_size_;
  *whole = false;
  return MX_OK;
}

bool Sched::quota_ok(int gpu, uint64_t quota, int exclude) const {
  unsigned __int128 s = quota;
  for (int p = 0; p < (int)parts_.size(); ++p)
    if (parts_[p].live && parts_[p].gpu == gpu && p != exclude) s += parts_[p].quota;
  return s <= mem_bytes_;
}

int Sched::plan_create(int gpu, int sm, uint64_t hbm, std::vector<int>* groups, int* smc,
                       bool* whole) const {
  if (gpu < 0 || gpu >= n_gpus_) return MX_ENODEV;
  if (sm <= 0 || hbm == 0) return MX_EINVAL;
  if (!quota_ok(gpu, hbm, -1)) return MX_ENOMEM;
  return alloc(gpu, sm, -1, groups, smc, whole);
}

int Sched::create(int gpu, int sm, uint64_t hbm, int* out_part) {
  std::vector<int> groups;
  int smc = 0;
  bool whole = false;
  int rc = plan_create(gpu, sm, hbm, &groups, &smc, &whole);
  if (rc) return rc;
  SchedPart p;
  p.gpu = gpu;
  p.groups = groups;
  p.sm_count = smc;
  p.whole = whole;
  p.quota = hbm;
  p.live = true;
  parts_.push_back(p);
  int id = (int)parts_.size() - 1;
  record(REC_CREATE, (uint64_t)id, (uint64_t)gpu, (uint64_t)smc, p.mask(), hbm, 0, flags(p));
  *out_part = id;
  return MX_OK;
}

int Sched::plan_create_shared(int gpu, int n_ctas, uint64_t hbm) const {
  if (gpu < 0 || gpu >= n_gpus_) return MX_ENODEV;
  if (n_ctas <= 0 || hbm == 0) return MX_EINVAL;
  if (!quota_ok(gpu, hbm, -1)) return MX_ENOMEM;
  return MX_OK;
}

int Sched::create_shared(int gpu, int n_ctas, uint64_t hbm, int* out_part) {
  int rc = plan_create_shared(gpu, n_ctas, hbm);
  if (rc) return rc;
  SchedPart p;
  p.gpu = gpu;
  p.sm_count = n_ctas < total_sms_ ? n_ctas : total_sms_;
  p.shared = true;
  p.quota = hbm;
  p.live = true;
  parts_.push_back(p);
  int id = (int)parts_.size() - 1;
  record(REC_CREATE, (uint64_t)id, (uint64_t)gpu, (uint64_t)p.sm_count, 0, hbm, 0, flags(p));
  *out_part = id;
  return MX_OK;
}

int Sched::plan_resize(int part, int sm, uint64_t hbm, std::vector<int>* groups, int* smc,
                       bool* whole, uint64_t* quota) const {
  if (!is_live(part)) return MX_EINVAL;
  const SchedPart& p = parts_[part];
  if (sm <= 0) sm = p.sm_count;
  if (hbm == 0) hbm = p.quota;
  if (!quota_ok(p.gpu, hbm, part)) return MX_ENOMEM;
  *quota = hbm;
  if (p.shared) {   // stays unpartitioned: only the grid size changes
    groups->clear();
    *smc = sm < total_sms_ ? sm : total_sms_;
    *whole = false;
    return MX_OK;
  }
  return alloc(p.gpu, sm, part, groups, smc, whole);
}

int Sched::resize(int part, int sm, uint64_t hbm) {
  std::vector<int> groups;
  int smc = 0;
  bool whole = false;
  uint64_t quota = 0;
  int rc = plan_resize(part, sm, hbm, &groups, &smc, &whole, &quota);
  if (rc) return rc;
  SchedPart& p = parts_[part];
  p.groups = groups;
  p.sm_count = smc;
  p.whole = whole;
  p.quota = quota;
  p.epoch += 1;
  record(REC_RESIZE, (uint64_t)part, (uint64_t)p.gpu, (uint64_t)smc, p.mask(), quota, p.epoch,
         flags(p));
  return MX_OK;
}

int Sched::destroy(int part) {
  if (!is_live(part)) return MX_EINVAL;
  SchedPart& p = parts_[part];
  p.live = false;
  record(REC_DESTROY, (uint64_t)part, (uint64_t)p.gpu, 0, 0, 0, p.epoch, 0);
  return MX_OK;
}

int Sched::submit(int fn, int part, uint64_t cost, Placement* out) {
  int chosen = -1;
  if (part == MX_PART_ANY) {
    for (int q = 0; q < (int)parts_.size(); ++q) {
      if (!parts_[q].live) continue;
      if (chosen < 0) {
        chosen = q;
        continue;
      }
      const SchedPart& b = parts_[chosen];
      const SchedPart& c = parts_[q];
      unsigned __int128 lhs = (unsigned __int128)(c.assigned + cost) * (uint64_t)b.sm_count;
      unsigned __int128 rhs = (unsigned __int128)(b.assigned + cost) * (uint64_t)c.sm_count;
      if (lhs < rhs) chosen = q;
    }
    if (chosen < 0) return MX_EINVAL;
  } else {
    if (!is_live(part)) return MX_EINVAL;
    chosen = part;
  }
  SchedPart& p = parts_[chosen];
  out->task = next_task_++;
  out->gpu = p.gpu;
  out->part = chosen;
  out->seq = p.seq++;
  out->epoch = p.epoch;
  p.assigned += cost;
  record(REC_PLACE, out->task, (uint64_t)(int64_t)fn, (uint64_t)p.gpu, (uint64_t)chosen, out->seq,
         p.epoch, cost);
  return MX_OK;
}

std::vector<uint8_t> Sched::trace_bytes() const {
  std::vector<uint8_t> out(records_.size() * 8);
  for (size_t i = 0; i < records_.size(); ++i)
    for (int b = 0; b < 8; ++b) out[i * 8 + b] = (uint8_t)(records_[i] >> (8 * b));
  return out;
}

}  // namespace mx
