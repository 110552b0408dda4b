// Persistent greedy-decode megakernel (sm_100a) — one launch runs a whole
// decode task (all P+G-1 steps, all layers) on one partition.
//
// Method: Llama-style block, §3.2
// P:113-115 (LLaMa2), §3.4 P:159 (20-word completions), §5.2 P:195 (100
// paragraph completions). Per step s (position t = s), per layer l:
//   QKV : h = RMSNorm(x, g_attn[l]);  qkv = [Wq;Wk;Wv] h
//   ATT : q,k <- RoPE(t) (rotate-half, A11); Kc[l][t] = bf16(k), Vc[l][t] = bf16(v)
//         (the only activation rounding point, A16); o_h = softmax(q.K/sqrt(hd)) V
//   O   : x += Wo o
//   GU  : h = RMSNorm(x, g_mlp[l]);  a = silu(Wgate h) * (Wup h)
//   DOWN: x += Wdown a
// then (steps s >= P-1 only) LM: logits = Wlm RMSNorm(x, g_final); token = argmax.
//
// B200 design:
//  * grid = the partition's SMs (one CTA per SM); phases are separated by a
//    device-wide barrier on a monotone counter (no atomics in the math).
//  * weights (98.5% of the bytes) are streamed by a producer warp with 1-D TMA
//    bulk copies (cp.async.bulk) into a 6 x 32 KB shared-memory ring guarded by
//    mbarriers. The weight stream is static, so the producer runs ahead ACROSS
//    phase barriers: the HBM stream never waits for the barrier latency.
//  * 8 consumer warps: each (row, 256-column chunk) unit is one 16-byte load
//    per lane from shared memory, an FMA chain, and a fixed shuffle tree; row
//    sums add the chunk partials in chunk order. Every output row is owned by
//    exactly one CTA, so the results do not depend on the partition size
//    (bit-identical for any sm_count), and nothing uses floating-point atomics.
//  * rows are split across CTAs with a per-phase rotation so the per-CTA byte
//    totals of a step stay balanced.
#include <cfloat>

#include "common.cuh"
#include "kernels.h"
#include "launch.cuh"

namespace mxk {

enum PhaseKind { PH_QKV = 0, PH_ATT = 1, PH_O = 2, PH_GU = 3, PH_DOWN = 4, PH_LM = 5 };

constexpr int kNCT = 32 * kConsumerWarps;   // consumer threads
constexpr int kAttHd = 128;                 // max head_dim
constexpr int kCPG = 4;                     // 256-column chunks per GEMV work unit

struct Phase {
  int kind, layer, R, K, NC, NG, TR;
  const uint16_t* w0;
  const uint16_t* w1;
};

__device__ __forceinline__ Phase make_phase(const DecodeParams& p, int kind, int layer) {
  Phase ph;
  ph.kind = kind;
  ph.layer = layer;
  ph.w1 = nullptr;
  ph.w0 = nullptr;
  ph.R = 0;
  ph.K = 0;
  const uint16_t* lw = p.w_layers + (uint64_t)layer * p.layer_stride;
  switch (kind) {
    case PH_QKV: ph.R = p.qkv_rows; ph.K = p.d; ph.w0 = lw + p.off_wqkv; break;
    case PH_O: ph.R = p.d; ph.K = p.q_dim; ph.w0 = lw + p.off_wo; break;
    case PH_GU: ph.R = p.ff; ph.K = p.d; ph.w0 = lw + p.off_wgate; ph.w1 = lw + p.off_wup; break;
    case PH_DOWN: ph.R = p.d; ph.K = p.ff; ph.w0 = lw + p.off_wdown; break;
    case PH_LM: ph.R = p.V; ph.K = p.d; ph.w0 = p.lm_head; break;
    default: break;
  }
  ph.NC = (ph.K + 255) / 256;
  ph.NG = (ph.NC + kCPG - 1) / kCPG;
  const int mult = (kind == PH_GU) ? 2 : 1;
  int tr = 1;
  if (ph.K > 0) {
    tr = kStageBytes / (mult * ph.K * 2);
    int tr2 = kMaxUnits / (mult * ph.NG);
    tr = max(1, min(tr, tr2));
  }
  ph.TR = tr;
  return ph;
}

// Rows [r0, r1) of a phase owned by this CTA; `rot` rotates the assignment so
// remainders land on different CTAs in different phases.
__device__ __forceinline__ void my_rows(int R, int C, int cta, int rot, int* r0, int* r1) {
  int c = (cta + rot) % C;
  *r0 = (int)(((long long)R * c) / C);
  *r1 = (int)(((long long)R * (c + 1)) / C);
}

__device__ __forceinline__ int phase_kind(int k, int L) { return (k == 5 * L) ? PH_LM : (k % 5); }

struct Smem {
  uint8_t* ring;
  float* xin;     // [B][K]
  float* red;     // [2][kMaxUnits][B]
  float* att;     // [kConsumerWarps][3][kAttHd]
  uint64_t* full;
  uint64_t* empty;
  unsigned long long* best;  // [8]
  int* tok;                  // [8]
  float* wsum;               // [kConsumerWarps][8]
};

__device__ __forceinline__ Smem carve(uint8_t* base, int n_stages, int B, int kmax) {
  Smem s;
  uint8_t* p = base;
  s.ring = p;
  p += (size_t)n_stages * kStageBytes;
  s.xin = reinterpret_cast<float*>(p);
  p += (size_t)B * kmax * 4;
  s.red = reinterpret_cast<float*>(p);
  p += (size_t)2 * kMaxUnits * B * 4;
  s.att = reinterpret_cast<float*>(p);
  p += (size_t)kConsumerWarps * 3 * kAttHd * 4;
  s.full = reinterpret_cast<uint64_t*>(p);
  p += (size_t)n_stages * 8;
  s.empty = reinterpret_cast<uint64_t*>(p);
  p += (size_t)n_stages * 8;
  s.best = reinterpret_cast<unsigned long long*>(p);
  p += 8 * 8;
  s.tok = reinterpret_cast<int*>(p);
  p += 8 * 4;
  s.wsum = reinterpret_cast<float*>(p);
  return s;
}

int decode_smem_bytes(int B, int kmax, int* n_stages) {
  int fixed = B * kmax * 4 + 2 * kMaxUnits * B * 4 + kConsumerWarps * 3 * kAttHd * 4 + 8 * 8 +
              8 * 4 + kConsumerWarps * 8 * 4 + 128;
  const int cap = 227 * 1024;
  int ns = (cap - fixed - 16 * 8) / kStageBytes;
  if (ns > 6) ns = 6;
  if (n_stages) *n_stages = ns;
  if (ns < 2) return -1;
  return ns * kStageBytes + fixed + 2 * ns * 8;
}

// Device-wide barrier among all CTAs of the launch (consumer warps only; the
// producer warp never waits on it). A 4 s timeout sets *err; afterwards every
// barrier passes without waiting, so a failed launch still terminates.
__device__ __forceinline__ void grid_barrier(const DecodeParams& p, unsigned long long target,
                                             int tid_c) {
  named_bar_sync(1, kNCT);
  if (tid_c == 0) {
    __threadfence();
    atomicAdd(p.bar, 1ull);
    if (!ld_volatile_i32(p.err)) {
      uint64_t t0 = globaltimer();
      uint32_t spins = 0;
      while (ld_acquire_u64(p.bar) < target) {
        if ((++spins & 255u) == 0) {
          if (ld_volatile_i32(p.err)) break;
          if (globaltimer() - t0 > 4000000000ull) {
            atomicExch(p.err, 1);
            break;
          }
        }
      }
    }
    __threadfence();
  }
  named_bar_sync(1, kNCT);
}

// ---------------------------------------------------------------------------
// Producer: stream this CTA's weight rows of every phase of every step.
// ---------------------------------------------------------------------------
__device__ void producer_loop(const DecodeParams& p, const Smem& sm, int n_stages) {
  const int C = p.n_ctas, cta = blockIdx.x, L = p.L;
  const int S = p.P + p.G - 1;
  uint32_t stage = 0, phase_bit = 0;
  const uint64_t pol = policy_evict_first();
  for (int s = 0; s < S; ++s) {
    const int nph = 5 * L + (s >= p.P - 1 ? 1 : 0);
    for (int k = 0; k < nph; ++k) {
      const int kind = phase_kind(k, L);
      if (kind == PH_ATT) continue;
      const Phase ph = make_phase(p, kind, k / 5);
      int r0, r1;
      my_rows(ph.R, C, cta, k, &r0, &r1);
      for (int r = r0; r < r1; r += ph.TR) {
        const int n = min(ph.TR, r1 - r);
        // never abandons the stream: after a barrier timeout the consumers run
        // through the remaining phases without waiting, so every slot is freed.
        while (!mbar_try_wait(&sm.empty[stage], phase_bit ^ 1u)) {
        }
        const uint32_t one = (uint32_t)n * (uint32_t)ph.K * 2u;
        const uint32_t total = (kind == PH_GU) ? 2u * one : one;
        uint8_t* dst = sm.ring + (size_t)stage * kStageBytes;
        mbar_arrive_expect_tx(&sm.full[stage], total);
        bulk_g2s_evict_first(dst, ph.w0 + (size_t)r * ph.K, one, &sm.full[stage], pol);
        if (kind == PH_GU)
          bulk_g2s_evict_first(dst + one, ph.w1 + (size_t)r * ph.K, one, &sm.full[stage], pol);
        if (++stage == (uint32_t)n_stages) {
          stage = 0;
          phase_bit ^= 1u;
        }
      }
    }
  }
}

// ---------------------------------------------------------------------------
// Consumers.
// ---------------------------------------------------------------------------

// Stage the phase input into shared memory (RMSNorm'd where the block says so).
template <int B>
__device__ void stage_input(const DecodeParams& p, const Smem& sm, int kind, int layer, int s,
                            int K, int tid_c) {
  const int cta = blockIdx.x, C = p.n_ctas;
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const uint16_t* gain = nullptr;
  if (kind == PH_QKV && layer == 0) {
    // input token: prompt for s < P, else the argmax of step s-1 (reduced from
    // the per-CTA candidates, identically in every CTA).
    if (tid_c < B) {
      int tok;
      if (s < p.P) {
        tok = p.prompt[tid_c * p.P + s];
      } else {
        unsigned long long best = 0;
        for (int c = 0; c < C; ++c) {
          unsigned long long v = p.cand[c * B + tid_c];
          best = v > best ? v : best;
        }
        tok = (int)argmax_key_index(best);
        if (cta == 0) p.tokens[tid_c * p.G + (s - p.P)] = tok;
      }
      sm.tok[tid_c] = tok;
    }
    named_bar_sync(1, kNCT);
    for (int i = tid_c; i < B * K; i += kNCT) {
      const int b = i / K, kk = i - b * K;
      const float v = bf16_bits_to_f32(p.embed[(size_t)sm.tok[b] * K + kk]);
      sm.xin[i] = v;
      if (cta == 0) p.x[b * p.d + kk] = v;
    }
    gain = p.w_layers + p.off_gattn;
  } else {
    const float* src = (kind == PH_O) ? p.o : (kind == PH_DOWN) ? p.a : p.x;
    for (int i = tid_c; i < B * K; i += kNCT) sm.xin[i] = src[i];
    if (kind == PH_QKV) gain = p.w_layers + (uint64_t)layer * p.layer_stride + p.off_gattn;
    if (kind == PH_GU) gain = p.w_layers + (uint64_t)layer * p.layer_stride + p.off_gmlp;
    if (kind == PH_LM) gain = p.g_final;
  }
  if (gain) {
    // RMSNorm (normalise, then scale; eps inside the sqrt): fixed-order block sum.
    float part[B];
#pragma unroll
    for (int b = 0; b < B; ++b) part[b] = 0.f;
    named_bar_sync(1, kNCT);
#pragma unroll
    for (int b = 0; b < B; ++b) {
      for (int kk = tid_c; kk < K; kk += kNCT) {
        const float v = sm.xin[b * K + kk];
        part[b] = fmaf(v, v, part[b]);
      }
      part[b] = warp_sum(part[b]);
      if (lane == 0) sm.wsum[warp * 8 + b] = part[b];
    }
    named_bar_sync(1, kNCT);
    float inv[B];
#pragma unroll
    for (int b = 0; b < B; ++b) {
      float t = 0.f;
      for (int w = 0; w < kConsumerWarps; ++w) t += sm.wsum[w * 8 + b];
      inv[b] = 1.0f / sqrtf(t / (float)K + p.eps);
    }
    for (int i = tid_c; i < B * K; i += kNCT) {
      const int b = i / K, kk = i - b * K;
      float ib = inv[0];
#pragma unroll
      for (int q = 1; q < B; ++q)
        if (b == q) ib = inv[q];
      sm.xin[i] = sm.xin[i] * ib * bf16_bits_to_f32(gain[kk]);
    }
  }
  named_bar_sync(1, kNCT);
}

// GEMV phase over this CTA's rows, consuming the TMA ring.
template <int B>
__device__ void gemv_phase(const DecodeParams& p, const Smem& sm, const Phase& ph, int k, int s,
                           int tid_c, uint32_t& stage, uint32_t& phase_bit, int& buf,
                           int n_stages) {
  const int C = p.n_ctas, cta = blockIdx.x;
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const int K = ph.K, NC = ph.NC, NG = ph.NG;
  const int mult = (ph.kind == PH_GU) ? 2 : 1;
  int r0, r1;
  my_rows(ph.R, C, cta, k, &r0, &r1);
  if (ph.kind == PH_LM && tid_c < B) sm.best[tid_c] = 0ull;
  for (int r = r0; r < r1; r += ph.TR) {
    const int n = min(ph.TR, r1 - r);
    const int units = n * mult * NG;
    while (!mbar_try_wait(&sm.full[stage], phase_bit)) {
    }
    const uint16_t* wt = reinterpret_cast<const uint16_t*>(sm.ring + (size_t)stage * kStageBytes);
    float* red = sm.red + (size_t)buf * kMaxUnits * B;
    for (int u = warp; u < units; u += kConsumerWarps) {
      // unit = (row, group of up to kCPG 256-column chunks): all weight loads of
      // the group are issued first, then two independent FMA chains per
      // sequence, then ONE fixed shuffle tree per unit.
      const int row = u / NG;
      const int g = u - row * NG;
      const int c0 = g * kCPG;
      const int nch = min(kCPG, NC - c0);
      const uint16_t* wr = wt + (size_t)row * K;
      uint4 wv[kCPG];
#pragma unroll
      for (int c = 0; c < kCPG; ++c) {
        const int col = (c0 + c) * 256 + lane * 8;
        wv[c] = (c < nch && col < K) ? *reinterpret_cast<const uint4*>(wr + col) : make_uint4(0, 0, 0, 0);
      }
      float acc0[B], acc1[B];
#pragma unroll
      for (int b = 0; b < B; ++b) acc0[b] = acc1[b] = 0.f;
#pragma unroll
      for (int c = 0; c < kCPG; ++c) {
        const int col = (c0 + c) * 256 + lane * 8;
        if (c < nch && col < K) {
          float wf[8];
          unpack8(wv[c], wf);
#pragma unroll
          for (int b = 0; b < B; ++b) {
            const float4 x0 = *reinterpret_cast<const float4*>(sm.xin + b * K + col);
            const float4 x1 = *reinterpret_cast<const float4*>(sm.xin + b * K + col + 4);
            acc0[b] = fmaf(wf[0], x0.x, acc0[b]);
            acc1[b] = fmaf(wf[1], x0.y, acc1[b]);
            acc0[b] = fmaf(wf[2], x0.z, acc0[b]);
            acc1[b] = fmaf(wf[3], x0.w, acc1[b]);
            acc0[b] = fmaf(wf[4], x1.x, acc0[b]);
            acc1[b] = fmaf(wf[5], x1.y, acc1[b]);
            acc0[b] = fmaf(wf[6], x1.z, acc0[b]);
            acc1[b] = fmaf(wf[7], x1.w, acc1[b]);
          }
        }
      }
#pragma unroll
      for (int b = 0; b < B; ++b) acc0[b] = warp_sum(acc0[b] + acc1[b]);
      if (lane == 0) {
#pragma unroll
        for (int b = 0; b < B; ++b) red[u * B + b] = acc0[b];
      }
    }
    named_bar_sync(1, kNCT);
    if (tid_c == 0) mbar_arrive(&sm.empty[stage]);
    if (++stage == (uint32_t)n_stages) {
      stage = 0;
      phase_bit ^= 1u;
    }
    // epilogue: unit partials summed in column order (deterministic).
    if (ph.kind == PH_GU) {
      for (int i = tid_c; i < n * B; i += kNCT) {
        const int j = i / B, b = i - j * B;
        float g = 0.f, up = 0.f;
        for (int c = 0; c < NG; ++c) g += red[(j * NG + c) * B + b];
        for (int c = 0; c < NG; ++c) up += red[((n + j) * NG + c) * B + b];
        p.a[b * p.ff + r + j] = g / (1.0f + expf(-g)) * up;
      }
    } else {
      for (int i = tid_c; i < n * B; i += kNCT) {
        const int j = i / B, b = i - j * B;
        float v = 0.f;
        for (int c = 0; c < NG; ++c) v += red[(j * NG + c) * B + b];
        const int row = r + j;
        switch (ph.kind) {
          case PH_QKV: p.qkv[b * p.qkv_rows + row] = v; break;
          case PH_O:
          case PH_DOWN: p.x[b * p.d + row] += v; break;
          case PH_LM: {
            if (p.logits) p.logits[((size_t)(s - (p.P - 1)) * B + b) * p.V + row] = v;
            atomicMax(&sm.best[b], argmax_key(v, (uint32_t)row));
          } break;
          default: break;
        }
      }
    }
    buf ^= 1;
  }
  if (ph.kind == PH_LM) {
    named_bar_sync(1, kNCT);
    if (tid_c < B) p.cand[cta * B + tid_c] = sm.best[tid_c];
  }
}

// Attention over the KV cache for (sequence, head) items, one warp per item.
template <int B>
__device__ void attention_phase(const DecodeParams& p, const Smem& sm, int layer, int t,
                                int tid_c) {
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const int H = p.H, Hkv = p.Hkv, hd = p.hd, half = hd / 2;
  const int group = H / Hkv;
  const int items = B * H;
  const int stride = p.n_ctas * kConsumerWarps;
  float* qs = sm.att + warp * 3 * kAttHd;
  float* ks = qs + kAttHd;
  float* vs = ks + kAttHd;
  const float scale_div = sqrtf((float)hd);
  for (int it = blockIdx.x * kConsumerWarps + warp; it < items; it += stride) {
    const int b = it / H, h = it - b * H, kvh = h / group;
    const float* base = p.qkv + (size_t)b * p.qkv_rows;
    const size_t cache_row0 = ((((size_t)layer * B + b) * Hkv + kvh) * p.max_seq) * hd;
    uint16_t* kcache = p.kc + cache_row0;
    uint16_t* vcache = p.vc + cache_row0;
    const bool writer = (h % group) == 0;
    for (int i = lane; i < half; i += 32) {
      const float c = p.rope_cs[((size_t)t * half + i) * 2 + 0];
      const float sn = p.rope_cs[((size_t)t * half + i) * 2 + 1];
      const float q1 = base[h * hd + i], q2 = base[h * hd + i + half];
      qs[i] = q1 * c - q2 * sn;
      qs[i + half] = q2 * c + q1 * sn;
      const float* kb = base + p.q_dim + kvh * hd;
      const float k1 = kb[i], k2 = kb[i + half];
      const uint16_t kb1 = f32_to_bf16_rne(k1 * c - k2 * sn);
      const uint16_t kb2 = f32_to_bf16_rne(k2 * c + k1 * sn);
      const float* vb = base + p.q_dim + p.kv_dim + kvh * hd;
      const uint16_t vb1 = f32_to_bf16_rne(vb[i]);
      const uint16_t vb2 = f32_to_bf16_rne(vb[i + half]);
      ks[i] = bf16_bits_to_f32(kb1);
      ks[i + half] = bf16_bits_to_f32(kb2);
      vs[i] = bf16_bits_to_f32(vb1);
      vs[i + half] = bf16_bits_to_f32(vb2);
      if (writer) {
        kcache[(size_t)t * hd + i] = kb1;
        kcache[(size_t)t * hd + i + half] = kb2;
        vcache[(size_t)t * hd + i] = vb1;
        vcache[(size_t)t * hd + i + half] = vb2;
      }
    }
    __syncwarp();
    // scores: lane owns keys j = lane + 32 m
    float sc[kMaxSeqCap / 32];
    float mx = -FLT_MAX;
#pragma unroll
    for (int m = 0; m < kMaxSeqCap / 32; ++m) {
      sc[m] = -FLT_MAX;
      if (32 * m <= t) {
        const int j = lane + 32 * m;
        if (j <= t) {
          float dot = 0.f;
          if (j < t) {
            const uint16_t* kr = kcache + (size_t)j * hd;
            for (int e = 0; e < hd; e += 8) {
              const uint4 kv = *reinterpret_cast<const uint4*>(kr + e);
              float kf[8];
              unpack8(kv, kf);
#pragma unroll
              for (int q = 0; q < 8; ++q) dot = fmaf(qs[e + q], kf[q], dot);
            }
          } else {
            for (int e = 0; e < hd; ++e) dot = fmaf(qs[e], ks[e], dot);
          }
          sc[m] = dot / scale_div;
          mx = fmaxf(mx, sc[m]);
        }
      }
    }
    mx = warp_max(mx);
    float e[kMaxSeqCap / 32];
    float lsum = 0.f;
#pragma unroll
    for (int m = 0; m < kMaxSeqCap / 32; ++m) {
      const int j = lane + 32 * m;
      e[m] = (32 * m <= t && j <= t) ? expf(sc[m] - mx) : 0.f;
      lsum += e[m];
    }
    const float sum = warp_sum(lsum);
    // output: lane owns dims lane + 32 q
    float acc[kAttHd / 32];
#pragma unroll
    for (int q = 0; q < kAttHd / 32; ++q) acc[q] = 0.f;
#pragma unroll
    for (int m = 0; m < kMaxSeqCap / 32; ++m) {
      if (32 * m <= t) {
        const int jmax = min(31, t - 32 * m);
        for (int jj = 0; jj <= jmax; ++jj) {
          const float ej = __shfl_sync(0xffffffffu, e[m], jj);
          const int j = 32 * m + jj;
#pragma unroll
          for (int q = 0; q < kAttHd / 32; ++q) {
            const int dd = lane + 32 * q;
            if (dd < hd) {
              const float vv = (j == t) ? vs[dd] : bf16_bits_to_f32(vcache[(size_t)j * hd + dd]);
              acc[q] = fmaf(ej, vv, acc[q]);
            }
          }
        }
      }
    }
#pragma unroll
    for (int q = 0; q < kAttHd / 32; ++q) {
      const int dd = lane + 32 * q;
      if (dd < hd) p.o[(size_t)b * p.q_dim + h * hd + dd] = acc[q] / sum;
    }
    __syncwarp();
  }
}

template <int B>
__global__ void __launch_bounds__(kDecodeThreads, 1) decode_kernel(DecodeParams p, int n_stages,
                                                                   int kmax) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const Smem sm = carve(smem_raw, n_stages, B, kmax);
  const int warp_id = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    for (int i = 0; i < n_stages; ++i) {
      mbar_init(&sm.full[i], 1);
      mbar_init(&sm.empty[i], 1);
    }
    fence_mbar_init();
    if (blockIdx.x == 0) p.stamps[0] = globaltimer();
  }
  __syncthreads();

  if (warp_id == 0) {
    if ((threadIdx.x & 31) == 0) producer_loop(p, sm, n_stages);
    return;
  }

  const int tid_c = threadIdx.x - 32;
  const int L = p.L, S = p.P + p.G - 1;
  uint32_t stage = 0, phase_bit = 0;
  int buf = 0;
  unsigned long long target = p.bar_base;
  for (int s = 0; s < S; ++s) {
    const int nph = 5 * L + (s >= p.P - 1 ? 1 : 0);
    for (int k = 0; k < nph; ++k) {
      const int kind = phase_kind(k, L);
      const int layer = k / 5;
      if (kind == PH_ATT) {
        attention_phase<B>(p, sm, layer, s, tid_c);
      } else {
        const Phase ph = make_phase(p, kind, layer);
        stage_input<B>(p, sm, kind, layer, s, ph.K, tid_c);
        gemv_phase<B>(p, sm, ph, k, s, tid_c, stage, phase_bit, buf, n_stages);
      }
      target += (unsigned long long)p.n_ctas;
      grid_barrier(p, target, tid_c);
    }
  }
  // final token (argmax of the last step)
  if (blockIdx.x == 0) {
    if (tid_c < B) {
      unsigned long long best = 0;
      for (int c = 0; c < p.n_ctas; ++c) {
        unsigned long long v = p.cand[c * B + tid_c];
        best = v > best ? v : best;
      }
      p.tokens[tid_c * p.G + (p.G - 1)] = (int)argmax_key_index(best);
    }
    named_bar_sync(1, kNCT);
    if (tid_c == 0) p.stamps[1] = globaltimer();
  }
}

template <int B>
static int launch_b(const DecodeParams& p, void* stream) {
  const int kmax = max(max(p.d, p.q_dim), p.ff);
  int ns = 0;
  const int smem = decode_smem_bytes(B, kmax, &ns);
  if (smem < 0) return -3;
  DecodeParams pc = p;
  int ns_arg = ns, kmax_arg = kmax;
  void* args[] = {&pc, &ns_arg, &kmax_arg};
  return launch_kernel(decode_kernel<B>, dim3(p.n_ctas), dim3(kDecodeThreads), (unsigned)smem,
                       stream, args);
}

int launch_decode(const DecodeParams& p, void* stream) {
  switch (p.B) {
    case 1: return launch_b<1>(p, stream);
    case 2: return launch_b<2>(p, stream);
    case 3: return launch_b<3>(p, stream);
    case 4: return launch_b<4>(p, stream);
    case 5: return launch_b<5>(p, stream);
    case 6: return launch_b<6>(p, stream);
    case 7: return launch_b<7>(p, stream);
    case 8: return launch_b<8>(p, stream);
    default: return -4;
  }
}

int decode_set_attrs(int device) {
  const int cap = 227 * 1024;
  int rc = 0;
  rc |= set_max_smem(decode_kernel<1>, cap, device);
  rc |= set_max_smem(decode_kernel<2>, cap, device);
  rc |= set_max_smem(decode_kernel<3>, cap, device);
  rc |= set_max_smem(decode_kernel<4>, cap, device);
  rc |= set_max_smem(decode_kernel<5>, cap, device);
  rc |= set_max_smem(decode_kernel<6>, cap, device);
  rc |= set_max_smem(decode_kernel<7>, cap, device);
  rc |= set_max_smem(decode_kernel<8>, cap, device);
  return rc;
}

}  // namespace mxk
