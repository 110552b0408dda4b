// Decode megakernel: host-side helpers and the batch-size dispatch. The
// kernel template lives in decode_impl.cuh and is instantiated once per batch
// size in decode_b*.cu (separate translation units, compiled in parallel).
#include <algorithm>

#include "kernels.h"

namespace mxk {


template <int B>
int launch_b(const DecodeParams& p, void* stream, int cooperative);
template <int B>
int set_attrs_b(int device);

int decode_smem_bytes(int B, int kmax, int* n_stages, int fuse_att) {
  // 1024-byte alignment slack + activation operand + attention scratch +
  // mbarriers (TMEM slots, operand copy) + small scratch; the rest is the weight ring
  const int att = decode_att_in_act(B, kmax, fuse_att) ? 0 : kConsumerWarps * 3 * kAttHd * 4;
  const int fixed = 1024 + decode_act_bytes(B, kmax) + att +
                    4 * 2 * 8 + 32 + 8 * 8 + 8 * 4 + kConsumerWarps * 8 * 4 + 8 * 4 + 6 * 4 * 4 + 16;
  const int per_stage = kStageBytes + 16;
  const int cap = 227 * 1024;
  int ns = (cap - fixed) / per_stage;
  if (ns > MX_MAX_STAGES) ns = MX_MAX_STAGES;
  if (n_stages) *n_stages = ns;
  if (ns < 2) return -1;
  return ns * per_stage + fixed;
}

int decode_prof_buckets() {
#ifdef MX_PROF_BUCKETS
  return 1;
#else
  return 0;
#endif
}

#ifndef MX_FUSE_MAX_CTAS
#define MX_FUSE_MAX_CTAS 100000
#endif
// Fused attention (every CTA computes all heads inside the O phase) saves a
// grid barrier per layer but replicates the K/V reads over the grid: used for
// small attention on grids of at most MX_FUSE_MAX_CTAS CTAs.
uint64_t decode_kpart_floats(int B, int d, int q_dim, int qkv_rows, int ff, int V, int fuse_att) {
  // (rows, input width, gate/up pair, splittable) of QKV, O, GU, DOWN, LM
  const long long sh[5][4] = {{qkv_rows, d, 1, 1}, {d, q_dim, 1, !fuse_att}, {ff, d, 2, 1},
                              {d, ff, 1, 1}, {V, d, 1, 1}};
  uint64_t m = 0;
  for (const auto& t : sh) {
    const int ns = decode_nseg(B, t[0], (int)t[1], (int)t[3]);
    if (ns > 1) m = std::max(m, (uint64_t)ns * (uint64_t)t[0] * (uint64_t)t[2] * (uint64_t)B);
  }
  return m;
}

int decode_fuse_attention(int B, int H, int hd, int n_ctas) {
  return (B * H * hd <= 1024 && n_ctas <= MX_FUSE_MAX_CTAS) ? 1 : 0;
}

uint64_t decode_barriers(int L, int P, int G, int fuse_att) {
  const uint64_t S = (uint64_t)(P + G - 1);
  return S * (uint64_t)(fuse_att ? 4 : 5) * (uint64_t)L + (uint64_t)G;   // phases_per_layer() x L + G LM phases
}

int launch_decode(const DecodeParams& p, void* stream, int cooperative) {
  switch (p.B) {
    case 1: return launch_b<1>(p, stream, cooperative);
    case 2: return launch_b<2>(p, stream, cooperative);
    case 3: return launch_b<3>(p, stream, cooperative);
    case 4: return launch_b<4>(p, stream, cooperative);
    case 5: return launch_b<5>(p, stream, cooperative);
    case 6: return launch_b<6>(p, stream, cooperative);
    case 7: return launch_b<7>(p, stream, cooperative);
    case 8: return launch_b<8>(p, stream, cooperative);
    default: return -4;
  }
}

int decode_set_attrs(int device) {
  int rc = 0;
  rc |= set_attrs_b<1>(device);
  rc |= set_attrs_b<2>(device);
  rc |= set_attrs_b<3>(device);
  rc |= set_attrs_b<4>(device);
  rc |= set_attrs_b<5>(device);
  rc |= set_attrs_b<6>(device);
  rc |= set_attrs_b<7>(device);
  rc |= set_attrs_b<8>(device);
  return rc;
}

}  // namespace mxk
