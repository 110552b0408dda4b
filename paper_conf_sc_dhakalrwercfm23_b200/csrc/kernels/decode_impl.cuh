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
//    device-wide barrier on a monotone counter (no floating-point atomics).
//    When the attention is small (B*H*hd <= 1024) every CTA computes all heads
//    itself as the O phase's input, removing one barrier per layer.
//  * weights (>98% of the bytes) are streamed by a producer warp with 1-D TMA
//    bulk copies (cp.async.bulk) into a shared-memory ring of 32 KB stages
//    guarded by mbarriers. The weight stream is static, so the producer runs
//    ahead ACROSS phase barriers.
//  * 11 decoupled consumer warps (12 warps per CTA = 3 per SM sub-partition, so
//    the 168-register budget holds the GEMV without spills): a work unit is (output row, <= 1024-column
//    group); each lane owns 8 consecutive columns of each 256-column chunk
//    (one 16-byte smem load), the activations are staged in a lane-permuted
//    layout so both 16-byte activation loads are bank-conflict free, and each
//    unit ends in one fixed shuffle tree. A row split over several units sums
//    its partials in a fixed order. Every output row is owned by exactly one
//    CTA, so results do not depend on the partition size.
//  * rows are split across CTAs with a per-phase rotation so the per-CTA byte
//    totals of a step stay balanced.
#include <cfloat>

#include "common.cuh"
#include "kernels.h"
#include "launch.cuh"

namespace mxk {

enum PhaseKind { PH_QKV = 0, PH_ATT = 1, PH_O = 2, PH_GU = 3, PH_DOWN = 4, PH_LM = 5 };

constexpr int kNCT = 32 * kConsumerWarps;   // consumer threads

#ifdef MX_NO_SLEEP
#define MX_FULL_WAIT(b, ph) mbar_try_wait(b, ph)
#define MX_EMPTY_WAIT(b, ph) mbar_try_wait(b, ph)
#else
#define MX_FULL_WAIT(b, ph) mbar_try_wait_sleep(b, ph, 20000u)
#define MX_EMPTY_WAIT(b, ph) mbar_try_wait_sleep(b, ph, 20000u)
#endif
// Bounded mbarrier wait: a launch that would otherwise hang (a protocol error
// or a failed copy) raises *err after 4 s and stops waiting, so the task
// completes with MX_EDEVICE instead of wedging its partition.
__device__ __forceinline__ void mbar_wait_bounded(uint64_t* bar, uint32_t parity, int* err) {
  if (MX_FULL_WAIT(bar, parity)) return;
  const uint64_t t0 = globaltimer();
  while (!MX_FULL_WAIT(bar, parity)) {
    if (ld_volatile_i32(err)) return;
    if (globaltimer() - t0 > 4000000000ull) {
      atomicExch(err, 1);
      return;
    }
  }
}

// Per-CTA cycle buckets (MX_DECODE_PROF=1) exist only in profiling builds
// (MX_DEFS=-DMX_PROF_BUCKETS): in the product build the counters fold to
// constants and cost no registers in the GEMV loop.
#ifdef MX_PROF_BUCKETS
#define MX_CLK() clock64()
#else
#define MX_CLK() 0ll
#endif

#ifndef MX_CPG
#define MX_CPG 8
#endif
constexpr int kCPG = MX_CPG;                // 256-column chunks per GEMV work unit

// One GEMV phase, or one K segment of it. Phases whose staged activations
// (B * K * 4 bytes) exceed kXinSegBytes run as `nseg` column segments
// [k0, k0 + K) inside the owning CTA (split-K): each segment streams the same
// rows restricted to its columns, partial sums of all but the last segment go
// to the slot's kacc buffer, and the last segment applies the epilogue to
// (kacc + partial). Segment widths depend only on the shape, so results stay
// independent of the partition size.
constexpr int kTcRows = 8;   // weight rows per tensor-core tile (the n of mma.m16n8k16)
// kTcGroups tensor-core tiles are in progress at once (consumer warps beyond
// kTcGroups * kTcSplit only observe and release the stages).
constexpr int kTcGroups = kConsumerWarps / kTcSplit;
static_assert(kTcGroups >= 1, "tensor-core split wider than the consumer warps");

struct Phase {
  int kind, layer, R, K, KP, NC, NG, TR;
  int ldw;         // row stride of the weight matrix in HBM (= the full K)
  int k0, seg, nseg;
  const uint16_t* w0;
  const uint16_t* w1;
};

__host__ __device__ __forceinline__ int round256(int k) { return (k + 255) & ~255; }

template <int B>
__device__ __forceinline__ Phase make_phase(const DecodeParams& p, int kind, int layer, int seg) {
  Phase ph;
  ph.kind = kind;
  ph.layer = layer;
  ph.w1 = nullptr;
  ph.w0 = nullptr;
  ph.R = 0;
  int K = 0;
  const uint16_t* lw = p.w_layers + (uint64_t)layer * p.layer_stride;
  switch (kind) {
    case PH_QKV: ph.R = p.qkv_rows; K = p.d; ph.w0 = lw + p.off_wqkv; break;
    case PH_O: ph.R = p.d; K = p.q_dim; ph.w0 = lw + p.off_wo; break;
    case PH_GU: ph.R = p.ff; K = p.d; ph.w0 = lw + p.off_wgate; ph.w1 = lw + p.off_wup; break;
    case PH_DOWN: ph.R = p.d; K = p.ff; ph.w0 = lw + p.off_wdown; break;
    case PH_LM: ph.R = p.V; K = p.d; ph.w0 = p.lm_head; break;
    default: break;
  }
  ph.ldw = K;
  ph.seg = seg;
  if constexpr (B >= kTcMinBatch) {
    // tensor-core path: K segments of <= kTcCols columns (multiples of 32), one
    // tile = 8 weight rows (GU: 4 gate + 4 up) x the segment = one stage
    ph.nseg = max(1, (K + kTcCols - 1) / kTcCols);
    const int w = (((K + ph.nseg - 1) / ph.nseg) + 31) & ~31;
    ph.k0 = seg * w;
    ph.K = min(w, K - ph.k0);
    ph.KP = (ph.K + 31) & ~31;
    ph.NC = 1;
    ph.NG = 1;
    ph.TR = (kind == PH_GU) ? kTcRows / 2 : kTcRows;
    return ph;
  }
  constexpr int KS = decode_seg_cols(B);
  ph.nseg = (K + KS - 1) / KS;
  if (ph.nseg < 1) ph.nseg = 1;
  if (ph.nseg > 1) {
    const int w = round256((K + ph.nseg - 1) / ph.nseg);
    ph.k0 = seg * w;
    ph.K = min(w, K - ph.k0);
  } else {
    ph.k0 = 0;
    ph.K = K;
  }
  ph.KP = round256(ph.K);
  ph.NC = ph.KP / 256;
  ph.NG = (ph.NC + kCPG - 1) / kCPG;
  const int mult = (kind == PH_GU) ? 2 : 1;
  int tr = 1;
  if (ph.K > 0) {
    tr = kStageBytes / (mult * ph.K * 2);
    const int tr2 = kMaxUnits / (mult * ph.NG);
    tr = max(1, min(tr, tr2));
  }
  ph.TR = tr;
  return ph;
}

template <int B>
__device__ __forceinline__ int phase_segments(const DecodeParams& p, int kind) {
  const int K = (kind == PH_O) ? p.q_dim : (kind == PH_DOWN) ? p.ff : p.d;
  constexpr int KS = (B >= kTcMinBatch) ? kTcCols : decode_seg_cols(B);
  return kind == PH_ATT ? 1 : max(1, (K + KS - 1) / KS);
}

// Rows [r0, r1) of a phase owned by this CTA; `rot` rotates the assignment so
// remainders land on different CTAs in different phases.
__device__ __forceinline__ void my_rows(int R, int C, int cta, int rot, int* r0, int* r1) {
  const int c = (cta + rot) % C;
  *r0 = (int)(((long long)R * c) / C);
  *r1 = (int)(((long long)R * (c + 1)) / C);
}

__host__ __device__ __forceinline__ int phases_per_layer(int fuse_att) { return fuse_att ? 4 : 5; }

__device__ __forceinline__ int phase_kind(int k, int L, int fuse_att) {
  const int pl = phases_per_layer(fuse_att);
  if (k == pl * L) return PH_LM;
  const int r = k % pl;
  if (fuse_att) return r == 0 ? PH_QKV : r == 1 ? PH_O : r == 2 ? PH_GU : PH_DOWN;
  return r;   // QKV, ATT, O, GU, DOWN
}

// Lane-permuted activation layout: within each 256-column chunk, lane l's
// columns 8l..8l+3 live at [4l, 4l+4) and 8l+4..8l+7 at [128+4l, 128+4l+4).
__device__ __forceinline__ int xidx(int b, int kk, int KP) {
  const int c = kk >> 8, w = kk & 255, l = w >> 3, e = w & 7;
  return b * KP + (c << 8) + ((e >> 2) << 7) + (l << 2) + (e & 3);
}

struct Smem {
  uint8_t* ring;
  float* xin;     // [B][KP] lane-permuted phase input
  float* red;     // [n_stages][kMaxUnits][B] partial sums of multi-unit outputs
  int* cnt;       // [n_stages][kMaxUnits] per-output completion counters
  float* att;     // [kConsumerWarps][3][kAttHd]
  uint64_t* full;
  uint64_t* empty;
  unsigned long long* best;  // [8]
  int* tok;                  // [8]
  float* wsum;               // [kConsumerWarps][8]
  float* inv;                // [8] RMSNorm scale of the phase input (kept across K segments)
  uint8_t* zero;             // [64] zeros (tensor-core path)
};

template <int B>
__device__ __forceinline__ Smem carve(uint8_t* base, int n_stages, int kmax) {
  Smem s;
  uint8_t* p = base;
  s.ring = p;
  p += (size_t)n_stages * kStageBytes;
  s.xin = reinterpret_cast<float*>(p);
  p += (size_t)decode_xin_bytes(B, kmax);
  s.zero = p - 64;   // tensor-core path: 64 zero bytes (ldmatrix rows of absent sequences)
  s.red = reinterpret_cast<float*>(p);
  p += (size_t)n_stages * decode_red_floats(B) * 4;
  s.cnt = reinterpret_cast<int*>(p);
  p += (size_t)n_stages * kMaxUnits * 4;
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
  p += (size_t)kConsumerWarps * 8 * 4;
  s.inv = reinterpret_cast<float*>(p);
  return s;
}

// Device-wide barrier among all CTAs of the launch (consumer warps only; the
// producer warp never waits on it). A 4 s timeout sets *err; afterwards every
// barrier passes without waiting, so a failed launch still terminates.
__device__ __forceinline__ void grid_barrier(const DecodeParams& p, unsigned long long target,
                                             int tid_c) {
  named_bar_sync(1, kNCT);
  if (tid_c == 0) {
    // release: this CTA's phase outputs (ordered before by bar.sync) become visible
    asm volatile("red.release.gpu.global.add.u64 [%0], 1;" ::"l"(p.bar) : "memory");
    if (!ld_volatile_i32(p.err)) {
      const uint64_t t0 = globaltimer();
      uint32_t spins = 0;
      while (ld_relaxed_u64(p.bar) < target) {
        if ((++spins & 255u) == 0) {
          if (ld_volatile_i32(p.err)) break;
          if (globaltimer() - t0 > 4000000000ull) {
            atomicExch(p.err, 1);
            break;
          }
        }
      }
    }
    // acquire: one acquire load of the final count synchronizes with every CTA's
    // release RMW (and invalidates this SM's L1 once for the whole CTA)
    (void)ld_acquire_u64(p.bar);
  }
  named_bar_sync(1, kNCT);
}

// ---------------------------------------------------------------------------
// Producer: stream this CTA's weight rows of every phase of every step.
// ---------------------------------------------------------------------------
template <int B>
__device__ void producer_loop(const DecodeParams& p, const Smem& sm, int n_stages) {
  const int C = p.n_ctas, cta = blockIdx.x, L = p.L;
  const int S = p.P + p.G - 1;
  const int pl = phases_per_layer(p.fuse_att);
  uint32_t stage = 0, phase_bit = 0;
  long long wait_cyc = 0;
  const uint64_t pol = policy_evict_first();
  for (int s = 0; s < S; ++s) {
    const int nph = pl * L + (s >= p.P - 1 ? 1 : 0);
    for (int k = 0; k < nph; ++k) {
      const int kind = phase_kind(k, L, p.fuse_att);
      if (kind == PH_ATT) continue;
      // L2 prefetch of the small operands the consumers will need a few us from
      // now (they are evicted by the weight stream between steps): the norm
      // gain of this phase, and for QKV(l) the cached keys/values of layer l
      // (this CTA's share) plus the RoPE row of step s.
      {
        const int layer = k / pl;
        const uint16_t* lw = p.w_layers + (uint64_t)layer * p.layer_stride;
        if (kind == PH_QKV) prefetch_l2(lw + p.off_gattn, (uint32_t)p.d * 2u);
        if (kind == PH_GU) prefetch_l2(lw + p.off_gmlp, (uint32_t)p.d * 2u);
        if (kind == PH_LM) prefetch_l2(p.g_final, (uint32_t)p.d * 2u);
        if (kind == PH_QKV) {
          if (layer == 0) prefetch_l2(p.rope_cs + (size_t)s * p.hd, (uint32_t)p.hd * 4u);
          if (s > 0) {
            const uint32_t bytes = (uint32_t)s * (uint32_t)p.hd * 2u;
            for (int it = cta; it < p.B * p.Hkv; it += C) {
              const size_t row0 = ((size_t)layer * p.B * p.Hkv + it) * p.max_seq * p.hd;
              prefetch_l2(p.kc + row0, bytes);
              prefetch_l2(p.vc + row0, bytes);
            }
          }
        }
      }
      const int nseg = phase_segments<B>(p, kind);
      for (int seg = 0; seg < nseg; ++seg) {
        const Phase ph = make_phase<B>(p, kind, k / pl, seg);
        int r0, r1;
        my_rows(ph.R, C, cta, k, &r0, &r1);
        for (int r = r0; r < r1; r += ph.TR) {
          const int n = min(ph.TR, r1 - r);
          // never abandons the stream: after a barrier timeout the consumers run
          // through the remaining phases without waiting, so every slot is freed.
          const long long tw = MX_CLK();
          mbar_wait_bounded(&sm.empty[stage], phase_bit ^ 1u, p.err);
          wait_cyc += MX_CLK() - tw;
          const uint32_t one = (uint32_t)n * (uint32_t)ph.K * 2u;
          const uint32_t total = (kind == PH_GU) ? 2u * one : one;
          uint8_t* dst = sm.ring + (size_t)stage * kStageBytes;
          mbar_arrive_expect_tx(&sm.full[stage], total);
          if constexpr (B >= kTcMinBatch) {
            // tensor-core tile: rows at a padded stride (conflict-free ldmatrix);
            // GU: gate rows 0..3, up rows 4..7
            const uint32_t rb = (uint32_t)ph.K * 2u, ws = (uint32_t)ph.KP * 2u + 16u;
            for (int i = 0; i < n; ++i) {
              const size_t src = (size_t)(r + i) * ph.ldw + ph.k0;
              bulk_g2s_evict_first(dst + i * ws, ph.w0 + src, rb, &sm.full[stage], pol);
              if (kind == PH_GU)
                bulk_g2s_evict_first(dst + (kTcRows / 2 + i) * ws, ph.w1 + src, rb,
                                     &sm.full[stage], pol);
            }
          } else if (ph.nseg == 1) {
            // whole rows: one contiguous copy per matrix
            bulk_g2s_evict_first(dst, ph.w0 + (size_t)r * ph.K, one, &sm.full[stage], pol);
            if (kind == PH_GU)
              bulk_g2s_evict_first(dst + one, ph.w1 + (size_t)r * ph.K, one, &sm.full[stage], pol);
          } else {
            // K segment: one copy per row of columns [k0, k0 + K), packed
            const uint32_t rb = (uint32_t)ph.K * 2u;
            for (int i = 0; i < n; ++i) {
              const size_t src = (size_t)(r + i) * ph.ldw + ph.k0;
              bulk_g2s_evict_first(dst + i * rb, ph.w0 + src, rb, &sm.full[stage], pol);
              if (kind == PH_GU)
                bulk_g2s_evict_first(dst + one + i * rb, ph.w1 + src, rb, &sm.full[stage], pol);
            }
          }
          if (++stage == (uint32_t)n_stages) {
            stage = 0;
            phase_bit ^= 1u;
          }
        }
      }
    }
  }
  if (p.prof) p.prof[cta * 16 + 6] = (unsigned long long)wait_cyc;
}

// ---------------------------------------------------------------------------
// Attention for one (sequence b, head h) item by one warp. Writes o_h either to
// global o (separate ATT phase) or into the lane-permuted O-phase input in
// shared memory (fused). `writer` selects the single writer of Kc/Vc[t].
//
// Latency-oriented: the cached keys/values of a block of KB positions are
// loaded together with the current token's q/k/v (one round trip for t < KB),
// then consumed with an online (running-max) softmax block by block. Lanes own
// keys for the scores (LPK lanes per key) and dims for the output.
// ---------------------------------------------------------------------------
template <int B, int HD>
__device__ __forceinline__ void attend_hd(const DecodeParams& p, const Smem& sm, int layer, int t,
                                          int b, int h, bool writer, bool to_smem, int warp,
                                          int lane) {
  constexpr int HALF = HD / 2;
  constexpr int PPL = (HALF + 31) / 32;       // rope pairs per lane
  constexpr int KB = (HD <= 64) ? 32 : 16;    // keys per block
  constexpr int LPK = 32 / KB;                // lanes per key
  constexpr int KSEG = HD / LPK;              // key elements per lane
  constexpr int KV4 = KSEG / 8;               // 16-byte loads per lane per key
  constexpr int DPL = HD / 32;                // output dims per lane
  const int Hkv = p.Hkv;
  const int kvh = h / (p.H / Hkv);
  float* qs = sm.att + warp * 3 * kAttHd;
  float* ks = qs + kAttHd;
  float* vs = ks + kAttHd;
  const float scale_div = sqrtf((float)HD);
  const float* base = p.qkv + (size_t)b * p.qkv_rows;
  const size_t cache_row0 = ((((size_t)layer * B + b) * Hkv + kvh) * p.max_seq) * HD;
  uint16_t* kcache = p.kc + cache_row0;
  uint16_t* vcache = p.vc + cache_row0;
  const int kslot = lane / LPK, kseg = (lane % LPK) * KSEG;

  // --- block loads (independent of the current token) ---------------------
  uint4 kr[KV4];
  uint32_t vv[KB][(DPL + 1) / 2];
  auto load_block = [&](int m) {
    const int j = m * KB + kslot;
#pragma unroll
    for (int i = 0; i < KV4; ++i)
      kr[i] = (j < t) ? *reinterpret_cast<const uint4*>(kcache + (size_t)j * HD + kseg + 8 * i)
                      : make_uint4(0, 0, 0, 0);
#pragma unroll
    for (int jj = 0; jj < KB; ++jj) {
      const int jk = m * KB + jj;
      const uint16_t* src = vcache + (size_t)jk * HD + lane * DPL;
      if (DPL == 4) {
        uint2 v2 = make_uint2(0u, 0u);
        if (jk < t) v2 = *reinterpret_cast<const uint2*>(src);
        vv[jj][0] = v2.x;
        vv[jj][(DPL + 1) / 2 - 1] = v2.y;
      } else if (DPL == 2) {
        vv[jj][0] = (jk < t) ? *reinterpret_cast<const uint32_t*>(src) : 0u;
      } else {
        vv[jj][0] = (jk < t) ? (uint32_t)*src : 0u;
      }
    }
  };
  load_block(0);

  // --- current token: RoPE(q), RoPE(k) -> bf16, v -> bf16 --------------------
#pragma unroll
  for (int pi = 0; pi < PPL; ++pi) {
    const int i = lane + 32 * pi;
    if (i < HALF) {
      const float c = p.rope_cs[((size_t)t * HALF + i) * 2 + 0];
      const float sn = p.rope_cs[((size_t)t * HALF + i) * 2 + 1];
      const float q1 = base[h * HD + i], q2 = base[h * HD + i + HALF];
      const float* kb = base + p.q_dim + kvh * HD;
      const float k1 = kb[i], k2 = kb[i + HALF];
      const float* vb = base + p.q_dim + p.kv_dim + kvh * HD;
      const float v1 = vb[i], v2 = vb[i + HALF];
      qs[i] = q1 * c - q2 * sn;
      qs[i + HALF] = q2 * c + q1 * sn;
      const uint16_t kb1 = f32_to_bf16_rne(k1 * c - k2 * sn);
      const uint16_t kb2 = f32_to_bf16_rne(k2 * c + k1 * sn);
      const uint16_t vb1 = f32_to_bf16_rne(v1);
      const uint16_t vb2 = f32_to_bf16_rne(v2);
      ks[i] = bf16_bits_to_f32(kb1);
      ks[i + HALF] = bf16_bits_to_f32(kb2);
      vs[i] = bf16_bits_to_f32(vb1);
      vs[i + HALF] = bf16_bits_to_f32(vb2);
      if (writer) {
        kcache[(size_t)t * HD + i] = kb1;
        kcache[(size_t)t * HD + i + HALF] = kb2;
        vcache[(size_t)t * HD + i] = vb1;
        vcache[(size_t)t * HD + i + HALF] = vb2;
      }
    }
  }
  __syncwarp();

  // --- blocks with online softmax -------------------------------------------
  float m_run = -FLT_MAX, l_run = 0.f;
  float acc[DPL];
#pragma unroll
  for (int d = 0; d < DPL; ++d) acc[d] = 0.f;
  for (int m = 0; m * KB <= t; ++m) {
    if (m > 0) load_block(m);
    const int j = m * KB + kslot;
    float dot = 0.f;
    // q / k rows in smem are 16-byte aligned (kAttHd floats per row, kseg a
    // multiple of 8): read them as float4 (a quarter of the LDS instructions)
    if (j < t) {
#pragma unroll
      for (int i = 0; i < KV4; ++i) {
        float kf[8];
        unpack8(kr[i], kf);
        const float4 qa = *reinterpret_cast<const float4*>(qs + kseg + 8 * i);
        const float4 qb = *reinterpret_cast<const float4*>(qs + kseg + 8 * i + 4);
        dot = fmaf(qa.x, kf[0], dot);
        dot = fmaf(qa.y, kf[1], dot);
        dot = fmaf(qa.z, kf[2], dot);
        dot = fmaf(qa.w, kf[3], dot);
        dot = fmaf(qb.x, kf[4], dot);
        dot = fmaf(qb.y, kf[5], dot);
        dot = fmaf(qb.z, kf[6], dot);
        dot = fmaf(qb.w, kf[7], dot);
      }
    } else if (j == t) {
#pragma unroll 4
      for (int e = 0; e < KSEG; e += 4) {
        const float4 qa = *reinterpret_cast<const float4*>(qs + kseg + e);
        const float4 ka = *reinterpret_cast<const float4*>(ks + kseg + e);
        dot = fmaf(qa.x, ka.x, dot);
        dot = fmaf(qa.y, ka.y, dot);
        dot = fmaf(qa.z, ka.z, dot);
        dot = fmaf(qa.w, ka.w, dot);
      }
    }
    if (LPK == 2) dot += __shfl_xor_sync(0xffffffffu, dot, 1);
    const float sc = (j <= t) ? dot / scale_div : -FLT_MAX;
    const float bm = warp_max(sc);
    const float new_m = fmaxf(m_run, bm);
    const float ej = (j <= t) ? expf(sc - new_m) : 0.f;
    const float scale = expf(m_run - new_m);
    const float bsum = warp_sum((lane % LPK) == 0 ? ej : 0.f);
    l_run = l_run * scale + bsum;
#pragma unroll
    for (int d = 0; d < DPL; ++d) acc[d] *= scale;
#pragma unroll
    for (int jj = 0; jj < KB; ++jj) {
      const int jk = m * KB + jj;
      const float e = __shfl_sync(0xffffffffu, ej, jj * LPK);
      float v[4];
      if (jk == t) {
#pragma unroll
        for (int d = 0; d < 4; ++d) v[d] = (d < DPL) ? vs[lane * DPL + d] : 0.f;
      } else {
        v[0] = __uint_as_float(vv[jj][0] << 16);
        v[1] = __uint_as_float(vv[jj][0] & 0xffff0000u);
        v[2] = __uint_as_float(vv[jj][(DPL + 1) / 2 - 1] << 16);
        v[3] = __uint_as_float(vv[jj][(DPL + 1) / 2 - 1] & 0xffff0000u);
      }
#pragma unroll
      for (int d = 0; d < DPL; ++d) acc[d] = fmaf(e, v[d], acc[d]);
    }
    m_run = new_m;
  }
  const int KP = round256(p.q_dim);
#pragma unroll
  for (int d = 0; d < DPL; ++d) {
    const int dd = lane * DPL + d;
    const float o = acc[d] / l_run;
    if (to_smem)
      sm.xin[xidx(b, h * HD + dd, KP)] = o;
    else
      p.o[(size_t)b * p.q_dim + h * HD + dd] = o;
  }
  __syncwarp();
}

template <int B>
__device__ __forceinline__ void attend(const DecodeParams& p, const Smem& sm, int layer, int t,
                                       int b, int h, bool writer, bool to_smem, int warp, int lane) {
  switch (p.hd) {
    case 32: attend_hd<B, 32>(p, sm, layer, t, b, h, writer, to_smem, warp, lane); break;
    case 64: attend_hd<B, 64>(p, sm, layer, t, b, h, writer, to_smem, warp, lane); break;
    default: attend_hd<B, 128>(p, sm, layer, t, b, h, writer, to_smem, warp, lane); break;
  }
}

// Separate attention phase (large attention): items spread over all warps of all CTAs.
template <int B>
__device__ void attention_phase(const DecodeParams& p, const Smem& sm, int layer, int t,
                                int tid_c) {
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const int items = B * p.H;
  const int stride = p.n_ctas * kConsumerWarps;
  const int group = p.H / p.Hkv;
  for (int it = blockIdx.x * kConsumerWarps + warp; it < items; it += stride) {
    const int b = it / p.H, h = it - b * p.H;
    attend<B>(p, sm, layer, t, b, h, (h % group) == 0, false, warp, lane);
  }
}

// ---------------------------------------------------------------------------
// Phase input staging (RMSNorm'd where the block says so), lane-permuted.
// ---------------------------------------------------------------------------
// Strided loop over [0, n) with U independent loads in flight per thread (the
// inputs come from L2, ~1 us away: a plain loop would serialise them).
template <int U, typename Load, typename Use>
__device__ __forceinline__ void batched_loop(int n, int tid, int stride, Load load, Use use) {
  using V = decltype(load(0));
  for (int base = tid; base < n; base += U * stride) {
    V v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int i = base + u * stride;
      if (i < n) v[u] = load(i);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int i = base + u * stride;
      if (i < n) use(i, v[u]);
    }
  }
}

// Tensor-core path (B >= kTcMinBatch) phase input from global fp32 activations
// (x, o or a; RMSNorm'd where the phase has a gain): float4 loads (row widths
// are multiples of 8) with kV4 loads in flight per thread, stored as the bf16
// hi/lo operand. At batch 8 a K segment is 8 x ~1400 floats, so the scalar
// 4-deep loop took ~8 L2 round trips per segment; this takes 2.
constexpr int kV4 = 4;

template <int B>
__device__ __forceinline__ void stage_vec_tc(const DecodeParams& p, const Smem& sm,
                                             const Phase& ph, const float* src,
                                             const uint16_t* gain, int tid_c) {
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const int K = ph.K, KP = ph.KP, k0 = ph.k0, KF = ph.ldw;
  const int KP4 = KP >> 2, n4 = B * KP4;
  if (gain && ph.seg == 0) {
    // RMSNorm over the FULL input (normalise, then scale; eps inside the sqrt):
    // per-thread partials, warp shuffle trees, fixed-order sum over warps; the
    // scale is kept in smem for later K segments.
    float acc[B];
#pragma unroll
    for (int b = 0; b < B; ++b) acc[b] = 0.f;
    const int KF4 = KF >> 2, nf4 = B * KF4;
    for (int base = tid_c; base < nf4; base += kV4 * kNCT) {
      float4 v[kV4];
#pragma unroll
      for (int u = 0; u < kV4; ++u) {
        const int i4 = base + u * kNCT;
        if (i4 < nf4) {
          const int b = i4 / KF4;
          v[u] = *reinterpret_cast<const float4*>(src + (size_t)b * KF + ((i4 - b * KF4) << 2));
        }
      }
#pragma unroll
      for (int u = 0; u < kV4; ++u) {
        const int i4 = base + u * kNCT;
        if (i4 < nf4) {
          const int bi = i4 / KF4;
          const float q = fmaf(v[u].x, v[u].x, fmaf(v[u].y, v[u].y, fmaf(v[u].z, v[u].z, v[u].w * v[u].w)));
#pragma unroll
          for (int b = 0; b < B; ++b)
            if (b == bi) acc[b] += q;
        }
      }
    }
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const float t = warp_sum(acc[b]);
      if (lane == 0) sm.wsum[warp * 8 + b] = t;
    }
    named_bar_sync(1, kNCT);
    if (tid_c < B) {
      float t = 0.f;
      for (int w = 0; w < kConsumerWarps; ++w) t += sm.wsum[w * 8 + tid_c];
      sm.inv[tid_c] = 1.0f / sqrtf(t / (float)KF + p.eps);
    }
    named_bar_sync(1, kNCT);
  }
  uint16_t* xh = reinterpret_cast<uint16_t*>(sm.xin);
  uint16_t* xl = xh + B * (KP + 8);
  for (int base = tid_c; base < n4; base += kV4 * kNCT) {
    float4 v[kV4];
#pragma unroll
    for (int u = 0; u < kV4; ++u) {
      const int i4 = base + u * kNCT;
      if (i4 < n4) {
        const int b = i4 / KP4, kk = (i4 - b * KP4) << 2;
        v[u] = (kk < K) ? *reinterpret_cast<const float4*>(src + (size_t)b * KF + k0 + kk)
                        : make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
#pragma unroll
    for (int u = 0; u < kV4; ++u) {
      const int i4 = base + u * kNCT;
      if (i4 >= n4) continue;
      const int b = i4 / KP4, kk = (i4 - b * KP4) << 2;
      float f[4] = {v[u].x, v[u].y, v[u].z, v[u].w};
      if (gain && kk < K) {
        const uint2 g = *reinterpret_cast<const uint2*>(gain + k0 + kk);
        const float ib = sm.inv[b];
        f[0] = f[0] * ib * bf16_bits_to_f32(g.x & 0xffffu);
        f[1] = f[1] * ib * bf16_bits_to_f32(g.x >> 16);
        f[2] = f[2] * ib * bf16_bits_to_f32(g.y & 0xffffu);
        f[3] = f[3] * ib * bf16_bits_to_f32(g.y >> 16);
      }
      uint16_t h[4], l[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        h[j] = f32_to_bf16_rne(f[j]);
        l[j] = f32_to_bf16_rne(f[j] - bf16_bits_to_f32(h[j]));
      }
      *reinterpret_cast<uint2*>(xh + b * (KP + 8) + kk) =
          make_uint2(h[0] | ((uint32_t)h[1] << 16), h[2] | ((uint32_t)h[3] << 16));
      *reinterpret_cast<uint2*>(xl + b * (KP + 8) + kk) =
          make_uint2(l[0] | ((uint32_t)l[1] << 16), l[2] | ((uint32_t)l[3] << 16));
    }
  }
  named_bar_sync(1, kNCT);
}

template <int B>
__device__ __forceinline__ void stage_input(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                            int s, int tid_c) {
  const int kind = ph.kind, layer = ph.layer;
  const int cta = blockIdx.x, C = p.n_ctas;
  const int warp = tid_c >> 5, lane = tid_c & 31;
  // K: this segment's columns [k0, k0 + K) of the full input width KF
  const int K = ph.K, KP = ph.KP, k0 = ph.k0, KF = ph.ldw;
  if (ph.seg > 0) named_bar_sync(1, kNCT);   // every warp is done with the previous segment
  if (kind == PH_O && p.fuse_att) {
    // every CTA computes all heads (small attention): o lands directly in xin
    for (int b = 0; b < B; ++b)
      for (int kk = K + tid_c; kk < KP; kk += kNCT) sm.xin[xidx(b, kk, KP)] = 0.f;
    const int group = p.H / p.Hkv;
    for (int it = warp; it < B * p.H; it += kConsumerWarps) {
      const int b = it / p.H, h = it - b * p.H;
      attend<B>(p, sm, layer, s, b, h, cta == 0 && (h % group) == 0, true, warp, lane);
    }
    named_bar_sync(1, kNCT);
    return;
  }
  const uint16_t* gain = nullptr;
  const uint16_t* emb = nullptr;   // layer-0 input: the embedding rows of the tokens
  const float* src = nullptr;
  if (kind == PH_QKV && layer == 0) {
    if (ph.seg == 0) {
      // input token: prompt for s < P, else the argmax of step s-1 (reduced from
      // the per-CTA candidates, identically in every CTA).
      if (tid_c < B) {
        int tok;
        if (s < p.P) {
          tok = p.prompt[tid_c * p.P + s];
        } else {
          unsigned long long best = 0;
          for (int c = 0; c < C; ++c) {
            const unsigned long long v = p.cand[c * B + tid_c];
            best = v > best ? v : best;
          }
          tok = (int)argmax_key_index(best);
          if (cta == 0) {
            p.tokens[tid_c * p.G + (s - p.P)] = tok;
            __threadfence_system();   // ordered before the completion flag
          }
        }
        sm.tok[tid_c] = tok;
      }
      named_bar_sync(1, kNCT);
    }
    emb = p.embed;
    gain = p.w_layers + p.off_gattn;
  } else {
    src = (kind == PH_O) ? p.o : (kind == PH_DOWN) ? p.a : p.x;
    if (kind == PH_QKV) gain = p.w_layers + (uint64_t)layer * p.layer_stride + p.off_gattn;
    if (kind == PH_GU) gain = p.w_layers + (uint64_t)layer * p.layer_stride + p.off_gmlp;
    if (kind == PH_LM) gain = p.g_final;
  }
  if constexpr (B >= kTcMinBatch) {
    if (!emb) {
      stage_vec_tc<B>(p, sm, ph, src, gain, tid_c);
      return;
    }
  }
  // Inputs are read once into registers (up to kRegVals per thread), then the
  // RMSNorm scale is applied on the way into the lane-permuted smem layout.
#ifndef MX_REG_VALS
#define MX_REG_VALS 8
#endif
  constexpr int kRegVals = MX_REG_VALS;
  const bool in_regs = (B == 1) && (ph.nseg == 1) && (KP <= kRegVals * kNCT);
  float rv[kRegVals];
  auto load_in = [&](int b, int col) -> float {
    return emb ? bf16_bits_to_f32(emb[(size_t)sm.tok[b] * KF + col]) : src[b * KF + col];
  };
  // staged column kk of the segment: (input, gain) loaded together
  auto load_staged = [&](int b, int kk) -> float2 {
    if (kk >= K) return make_float2(0.f, 0.f);
    const int col = k0 + kk;
    return make_float2(load_in(b, col), gain ? bf16_bits_to_f32(gain[col]) : 1.f);
  };
  if (in_regs) {
#pragma unroll
    for (int i = 0; i < kRegVals; ++i) {
      const int kk = tid_c + i * kNCT;
      rv[i] = (kk < K) ? load_in(0, kk) : 0.f;
    }
  }
  if (gain && ph.seg == 0) {
    // RMSNorm over the FULL input (normalise, then scale; eps inside the sqrt):
    // fixed-order block sum; the scale is kept in smem for later K segments.
    if (in_regs) {
      float acc = 0.f;
#pragma unroll
      for (int i = 0; i < kRegVals; ++i) acc = fmaf(rv[i], rv[i], acc);
      acc = warp_sum(acc);
      if (lane == 0) sm.wsum[warp * 8] = acc;
    } else {
      for (int b = 0; b < B; ++b) {
        float acc = 0.f;
        batched_loop<4>(KF, tid_c, kNCT, [&](int kk) { return load_in(b, kk); },
                        [&](int, float v) { acc = fmaf(v, v, acc); });
        acc = warp_sum(acc);
        if (lane == 0) sm.wsum[warp * 8 + b] = acc;
      }
    }
    named_bar_sync(1, kNCT);
    if (tid_c < B) {
      float t = 0.f;
      for (int w = 0; w < kConsumerWarps; ++w) t += sm.wsum[w * 8 + tid_c];
      sm.inv[tid_c] = 1.0f / sqrtf(t / (float)KF + p.eps);
    }
    named_bar_sync(1, kNCT);
  }
  if constexpr (B >= kTcMinBatch) {
    // tensor-core operand: x = hi + lo (bf16 pair), rows [b][KP + 8] (padded)
    uint16_t* xh = reinterpret_cast<uint16_t*>(sm.xin);
    uint16_t* xl = xh + B * (KP + 8);
    for (int b = 0; b < B; ++b) {
      const float ib = gain ? sm.inv[b] : 1.f;
      batched_loop<4>(KP, tid_c, kNCT, [&](int kk) { return load_staged(b, kk); },
                      [&](int kk, float2 xg) {
                        float v = 0.f;
                        if (kk < K) {
                          v = xg.x;
                          if (emb && cta == 0) p.x[b * p.d + k0 + kk] = v;
                          if (gain) v = v * ib * xg.y;
                        }
                        const uint16_t h = f32_to_bf16_rne(v);
                        xh[b * (KP + 8) + kk] = h;
                        xl[b * (KP + 8) + kk] = f32_to_bf16_rne(v - bf16_bits_to_f32(h));
                      });
    }
  } else if (in_regs) {
#pragma unroll
    for (int i = 0; i < kRegVals; ++i) {
      const int kk = tid_c + i * kNCT;
      if (kk < KP) {
        float v = rv[i];
        if (kk < K) {
          if (emb && cta == 0) p.x[kk] = v;
          if (gain) v = v * sm.inv[0] * bf16_bits_to_f32(gain[kk]);
        }
        sm.xin[xidx(0, kk, KP)] = v;
      }
    }
  } else {
    for (int b = 0; b < B; ++b) {
      const float ib = gain ? sm.inv[b] : 1.f;
      batched_loop<4>(KP, tid_c, kNCT, [&](int kk) { return load_staged(b, kk); },
                      [&](int kk, float2 xg) {
                        float v = 0.f;
                        if (kk < K) {
                          v = xg.x;
                          if (emb && cta == 0) p.x[b * p.d + k0 + kk] = v;
                          if (gain) v = v * ib * xg.y;
                        }
                        sm.xin[xidx(b, kk, KP)] = v;
                      });
    }
  }
  named_bar_sync(1, kNCT);
}

// ---------------------------------------------------------------------------
// GEMV phase over this CTA's rows, consuming the TMA ring. Warps are decoupled:
// each warp waits for a stage, processes its work units of that stage, and
// releases the stage on its own (the empty barrier counts kConsumerWarps
// arrivals); there is no CTA-wide barrier per tile.
//
// A work unit is NR rows (B<=2: 4, B<=4: 2, else 1; GU: NR/2 gate/up output
// pairs) over one group of <= kCPG 256-column chunks. Each lane owns 8
// consecutive columns per chunk (one 16-byte smem load per row), the
// activation loads are shared by the unit's rows, and the unit ends in NR
// interleaved shuffle trees. When a row spans several groups (K > kCPG*256),
// the group partials go through shared memory and the warp completing the last
// one sums them in group order — every output is computed in one fixed order.
// ---------------------------------------------------------------------------
template <int B>
struct RowsPerUnit {
  static constexpr int value = (B == 1) ? MX_ROWS_B1 : (B <= 2) ? 4 : (B <= 4 ? 2 : 1);
};

template <int B, int NR, int NCH>
__device__ __forceinline__ void multi_dot(const uint16_t* const (&w)[NR], const bool (&has)[NR],
                                          const float* __restrict__ xc, int KP, int col0, int K,
                                          int lane, float (&out)[NR][B]) {
  // acc.x sums the even columns of the lane's 8, acc.y the odd ones (FFMA2)
  unsigned long long acc[NR][B];
#pragma unroll
  for (int r = 0; r < NR; ++r)
#pragma unroll
    for (int b = 0; b < B; ++b) acc[r][b] = 0ull;
  constexpr int CB = (NR >= 4) ? 1 : (NR == 2 ? 2 : 4);   // chunks per load batch (bounds registers)
#pragma unroll
  for (int cb = 0; cb < NCH; cb += CB) {
    uint4 wv[CB][NR];
#pragma unroll
    for (int i = 0; i < CB; ++i) {
      const int c = cb + i;
      if (c < NCH) {
        const int col = col0 + c * 256 + lane * 8;
        const bool ok = (c < NCH - 1) || col < K;   // only the last chunk can be ragged
#pragma unroll
        for (int r = 0; r < NR; ++r)
          wv[i][r] = (ok && has[r]) ? *reinterpret_cast<const uint4*>(w[r] + col)
                                    : make_uint4(0, 0, 0, 0);
      }
    }
#pragma unroll
    for (int i = 0; i < CB; ++i) {
      const int c = cb + i;
      if (c < NCH) {
#pragma unroll
        for (int b = 0; b < B; ++b) {
          const float4 x0 = *reinterpret_cast<const float4*>(xc + c * 256 + b * KP);
          const float4 x1 = *reinterpret_cast<const float4*>(xc + c * 256 + b * KP + 128);
#pragma unroll
          for (int r = 0; r < NR; ++r) {
            float f[8];
            unpack8(wv[i][r], f);
            ffma2(acc[r][b], f[0], f[1], x0.x, x0.y);
            ffma2(acc[r][b], f[2], f[3], x0.z, x0.w);
            ffma2(acc[r][b], f[4], f[5], x1.x, x1.y);
            ffma2(acc[r][b], f[6], f[7], x1.z, x1.w);
          }
        }
      }
    }
  }
#pragma unroll
  for (int r = 0; r < NR; ++r)
#pragma unroll
    for (int b = 0; b < B; ++b) out[r][b] = f32x2_sum(acc[r][b]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1)
#pragma unroll
    for (int r = 0; r < NR; ++r)
#pragma unroll
      for (int b = 0; b < B; ++b) out[r][b] += __shfl_xor_sync(0xffffffffu, out[r][b], o);
}

template <int B, int NR>
__device__ __forceinline__ void multi_dot_n(int nch, const uint16_t* const (&w)[NR],
                                            const bool (&has)[NR], const float* xc, int KP,
                                            int col0, int K, int lane, float (&out)[NR][B]) {
  switch (nch) {
    case 1: multi_dot<B, NR, 1>(w, has, xc, KP, col0, K, lane, out); break;
    case 2: multi_dot<B, NR, 2>(w, has, xc, KP, col0, K, lane, out); break;
    case 3: multi_dot<B, NR, 3>(w, has, xc, KP, col0, K, lane, out); break;
    case 4: multi_dot<B, NR, 4>(w, has, xc, KP, col0, K, lane, out); break;
    case 5: multi_dot<B, NR, 5>(w, has, xc, KP, col0, K, lane, out); break;
    case 6: multi_dot<B, NR, 6>(w, has, xc, KP, col0, K, lane, out); break;
    case 7: multi_dot<B, NR, 7>(w, has, xc, KP, col0, K, lane, out); break;
    default: multi_dot<B, NR, 8>(w, has, xc, KP, col0, K, lane, out); break;
  }
}

template <int B, int NR, int KIND>
__device__ __forceinline__ void gemv_phase_nr(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                              int k, int s,
                              int tid_c, uint32_t& stage, uint32_t& phase_bit, int n_stages,
                              long long& wait_cyc, long long& unit_cyc, long long& unit_cnt) {
  const int C = p.n_ctas, cta = blockIdx.x;
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const int K = ph.K, KP = ph.KP, NC = ph.NC, NG = ph.NG;
  constexpr bool gu = (KIND == PH_GU);
  constexpr bool resid = (KIND == PH_O || KIND == PH_DOWN);
  constexpr int OPU_GU = NR / 2;            // GU outputs per unit (gate + up rows)
  int r0, r1;
  my_rows(ph.R, C, cta, k, &r0, &r1);
  if (KIND == PH_LM) {
    if (tid_c < B) sm.best[tid_c] = 0ull;
    named_bar_sync(1, kNCT);
  }
  int start = 0;   // first warp of the current tile (rotates the assignment across tiles)
  for (int r = r0; r < r1; r += ph.TR) {
    const int n = min(ph.TR, r1 - r);
    const int per = gu ? OPU_GU : NR;        // outputs per unit
    const int groups = (n + per - 1) / per;
    const int units = groups * NG;
    int u = warp - start;
    if (u < 0) u += kConsumerWarps;
    start = (start + units) % kConsumerWarps;
    // every warp observes the stage fill before releasing it (keeps the empty
    // barrier's arrival count per round exact)
    const long long tw = MX_CLK();
    mbar_wait_bounded(&sm.full[stage], phase_bit, p.err);
    wait_cyc += MX_CLK() - tw;
    const uint16_t* wt = reinterpret_cast<const uint16_t*>(sm.ring + (size_t)stage * kStageBytes);
    float* red = sm.red + (size_t)stage * decode_red_floats(B);
    int* cnt = sm.cnt + stage * kMaxUnits;
    for (; u < units; u += kConsumerWarps) {
      const long long tu = MX_CLK();
      const int gi = (NG == 1) ? u : u / NG;   // output group within the tile
      const int g = u - gi * NG;
      const int j0 = gi * per;                 // first tile-local output of the unit
      const uint16_t* w[NR];
      bool has[NR];
#pragma unroll
      for (int q = 0; q < NR; ++q) {
        if (gu) {
          const int j = j0 + (q >> 1);
          has[q] = j < n;
          w[q] = wt + (size_t)((q & 1) ? n + j : j) * K;
        } else {
          const int j = j0 + q;
          has[q] = j < n;
          w[q] = wt + (size_t)j * K;
        }
      }
      // residual rows prefetched before the dot product (latency hidden)
      float res[NR];
#pragma unroll
      for (int q = 0; q < NR; ++q) res[q] = 0.f;
      if (resid && NG == 1 && lane < B) {
#pragma unroll
        for (int q = 0; q < NR; ++q)
          if (has[q]) res[q] = p.x[lane * p.d + r + j0 + q];
      }
      const int c0 = g * kCPG;
      float out[NR][B];
      multi_dot_n<B, NR>(min(kCPG, NC - c0), w, has, sm.xin + c0 * 256 + 4 * lane, KP, c0 * 256, K,
                         lane, out);
      if (NG > 1) {
        // group partials -> smem; the last arriving warp finishes the unit's outputs
        if (lane == 0) {
#pragma unroll
          for (int q = 0; q < NR; ++q)
#pragma unroll
            for (int b = 0; b < B; ++b) red[(u * NR + q) * B + b] = out[q][b];
        }
        __threadfence_block();
        int old = 0;
        if (lane == 0) old = atomicAdd(&cnt[gi], 1);
        old = __shfl_sync(0xffffffffu, old, 0);
        if (old != NG - 1) continue;
        __threadfence_block();
#pragma unroll
        for (int q = 0; q < NR; ++q)
#pragma unroll
          for (int b = 0; b < B; ++b) {
            float v = 0.f;
            for (int gg = 0; gg < NG; ++gg) v += red[((gi * NG + gg) * NR + q) * B + b];
            out[q][b] = v;
          }
        if (lane == 0) cnt[gi] = 0;   // reset for the stage's next round
        if (resid && lane < B) {
#pragma unroll
          for (int q = 0; q < NR; ++q)
            if (has[q]) res[q] = p.x[lane * p.d + r + j0 + q];
        }
      }
      if (lane < B) {
        const int b = lane;
        float v[NR];
#pragma unroll
        for (int q = 0; q < NR; ++q) {
          v[q] = out[q][0];
#pragma unroll
          for (int bb = 1; bb < B; ++bb)
            if (bb == b) v[q] = out[q][bb];
        }
        bool final_seg = true;
        if (ph.nseg > 1) {
          // split-K: kacc[b][row] holds the sum of the earlier segments (GU: gate
          // and up interleaved); the last segment adds its part and goes on to
          // the epilogue. Rows are owned by this CTA, so no atomics are needed.
          float* acc = p.kacc + (size_t)b * ph.R * (gu ? 2 : 1);
          final_seg = (ph.seg == ph.nseg - 1);
#pragma unroll
          for (int q = 0; q < NR; ++q)
            if (has[q]) {
              const int idx = gu ? 2 * (r + j0 + (q >> 1)) + (q & 1) : r + j0 + q;
              const float t = (ph.seg == 0) ? v[q] : acc[idx] + v[q];
              if (final_seg)
                v[q] = t;
              else
                acc[idx] = t;
            }
        }
        if (final_seg) switch (KIND) {
          case PH_QKV:
#pragma unroll
            for (int q = 0; q < NR; ++q)
              if (has[q]) p.qkv[b * p.qkv_rows + r + j0 + q] = v[q];
            break;
          case PH_O:
          case PH_DOWN:
#pragma unroll
            for (int q = 0; q < NR; ++q)
              if (has[q]) p.x[b * p.d + r + j0 + q] = res[q] + v[q];
            break;
          case PH_GU:
#pragma unroll
            for (int q = 0; q < NR; q += 2)
              if (has[q]) {
                const float gt = v[q], up = v[q + 1];
                p.a[b * p.ff + r + j0 + q / 2] = gt / (1.0f + expf(-gt)) * up;
              }
            break;
          case PH_LM: {
            unsigned long long kb = 0ull;
#pragma unroll
            for (int q = 0; q < NR; ++q)
              if (has[q]) {
                const int row = r + j0 + q;
                const unsigned long long kq = argmax_key(v[q], (uint32_t)row);
                kb = kq > kb ? kq : kb;
                if (p.logits) p.logits[((size_t)(s - (p.P - 1)) * B + b) * p.V + row] = v[q];
              }
            atomicMax(&sm.best[b], kb);
          } break;
          default: break;
        }
      }
      unit_cyc += MX_CLK() - tu;
      ++unit_cnt;
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.empty[stage]);
    if (++stage == (uint32_t)n_stages) {
      stage = 0;
      phase_bit ^= 1u;
    }
  }
  if (KIND == PH_LM && ph.seg == ph.nseg - 1) {
    named_bar_sync(1, kNCT);
    if (tid_c < B) p.cand[cta * B + tid_c] = sm.best[tid_c];
  }
}

// ---------------------------------------------------------------------------
// Tensor-core GEMV (K7, batch >= kTcMinBatch): at batch 4-8 the CUDA-core unit
// is shared-memory bound (each weight needs B fp32 activations), so the GEMV
// runs as mma.sync.m16n8k16: A = activations (rows = sequences, only the first
// B of 16 real; the rest point at a zero block), B = 8 weight rows of the tile
// ("col" operand = the row-major weight rows), fp32 accumulate. Activations are
// fed as a bf16 hi/lo pair (two MMAs, ~16-bit mantissa, reading A17); weights
// are exact in bf16. One tile (8 rows x one K segment) is one stage and is
// consumed entirely by its owner warp (row group g -> warp g % 12), with four
// independent accumulator chains summed in a fixed order at the end.
// D fragment: lane (g, t) holds sequence g, tile rows 2t and 2t+1.
// ---------------------------------------------------------------------------
template <int B, int KIND>
__device__ __forceinline__ void gemv_phase_tc(const DecodeParams& p, const Smem& sm,
                                              const Phase& ph, int k, int s, int tid_c,
                                              uint32_t& stage, uint32_t& phase_bit, int n_stages,
                                              long long& wait_cyc, long long& unit_cyc,
                                              long long& unit_cnt) {
  const int C = p.n_ctas, cta = blockIdx.x;
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const int g8 = lane >> 2, t4 = lane & 3;
  const int lr = lane & 7, lm = lane >> 3;
  constexpr bool gu = (KIND == PH_GU);
  const int K = ph.K, KP = ph.KP;
  const uint32_t ws = (uint32_t)KP * 2u + 16u;   // weight / activation row stride (bytes)
  const uint32_t xh = smem_u32(sm.xin);
  const uint32_t xl = xh + (uint32_t)B * ws;
  const uint32_t zero = smem_u32(sm.zero);
  // per-lane ldmatrix row addresses (row lr of matrix lm = columns 8*lm..8*lm+7)
  const bool arow = lr < B;
  const uint32_t a_hi = arow ? xh + (uint32_t)lr * ws + (uint32_t)lm * 16u : zero;
  const uint32_t a_lo = arow ? xl + (uint32_t)lr * ws + (uint32_t)lm * 16u : zero;
  const uint32_t a_step = arow ? 64u : 0u;   // 32 columns per iteration
  const bool last_seg = (ph.seg == ph.nseg - 1);
  int r0, r1;
  my_rows(ph.R, C, cta, k, &r0, &r1);
  if (KIND == PH_LM) {
    if (tid_c < B) sm.best[tid_c] = 0ull;
    named_bar_sync(1, kNCT);
  }
  int gidx = 0;
  for (int r = r0; r < r1; r += ph.TR, ++gidx) {
    // Every warp observes every stage fill and arrives on its empty barrier
    // (count kConsumerWarps): a parity wait only tells two consecutive phases
    // apart, so no warp may skip stages and run a full ring ahead. Only the
    // owner group computes the tile.
    const long long tw = MX_CLK();
    mbar_wait_bounded(&sm.full[stage], phase_bit, p.err);
    const long long tu = MX_CLK();
    wait_cyc += tu - tw;
    // tile gidx belongs to warp group gidx % kTcGroups; its kTcSplit warps split
    // the K iterations and combine their partials in a fixed order
    const int grp = gidx % kTcGroups;
    if (warp / kTcSplit != grp) {
      __syncwarp();
      if (lane == 0) mbar_arrive(&sm.empty[stage]);
    } else {
      const int q = warp - grp * kTcSplit;
      const int n = min(ph.TR, r1 - r);
      const int IT = (K + 31) >> 5;
      const int it0 = (q * IT) / kTcSplit, it1 = ((q + 1) * IT) / kTcSplit;
      const uint32_t wt = smem_u32(sm.ring + (size_t)stage * kStageBytes) + (uint32_t)lr * ws +
                          (uint32_t)lm * 16u;
      float acc[4][4];
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[c][j] = 0.f;
      uint32_t ah = a_hi + (uint32_t)it0 * a_step, al = a_lo + (uint32_t)it0 * a_step;
      uint32_t wp = wt + (uint32_t)it0 * 64u;
      for (int kk = it0 * 32; kk < it1 * 32; kk += 32) {
        uint32_t w0, w1, w2, w3, h0, h1, h2, h3, l0, l1, l2, l3;
        ldsm_x4(wp, w0, w1, w2, w3);
        ldsm_x4(ah, h0, h1, h2, h3);
        ldsm_x4(al, l0, l1, l2, l3);
        if (kk + 32 > K) {
          // ragged end: weight columns >= K hold stale data -> zero their fragments
          // (b0: k = 2t, 2t+1; b1: k = 8 + 2t, 8 + 2t + 1 of each 16-column step)
          const int kb = kk + 2 * t4;
          if (kb >= K) w0 = 0u;
          if (kb + 8 >= K) w1 = 0u;
          if (kb + 16 >= K) w2 = 0u;
          if (kb + 24 >= K) w3 = 0u;
        }
        mma_bf16(acc[0], h0, 0u, h1, 0u, w0, w1);
        mma_bf16(acc[1], l0, 0u, l1, 0u, w0, w1);
        mma_bf16(acc[2], h2, 0u, h3, 0u, w2, w3);
        mma_bf16(acc[3], l2, 0u, l3, 0u, w2, w3);
        wp += 64u;
        ah += a_step;
        al += a_step;
      }
      float v0 = (acc[0][0] + acc[1][0]) + (acc[2][0] + acc[3][0]);
      float v1 = (acc[0][1] + acc[1][1]) + (acc[2][1] + acc[3][1]);
      bool last = true;
      if (kTcSplit > 1) {
        // partials -> smem; the warp arriving last sums them in warp order. It
        // reads them before releasing the stage, so the slot (and its partial
        // buffer) cannot be reused underneath it.
        float* red = sm.red + (size_t)stage * decode_red_floats(B);
        int* cnt = sm.cnt + stage * kMaxUnits;
        red[(q * 32 + lane) * 2] = v0;
        red[(q * 32 + lane) * 2 + 1] = v1;
        __threadfence_block();
        __syncwarp();
        int old = 0;
        if (lane == 0) old = atomicAdd(cnt, 1);
        old = __shfl_sync(0xffffffffu, old, 0);
        last = (old == kTcSplit - 1);
        if (last) {
          __threadfence_block();
          v0 = 0.f;
          v1 = 0.f;
#pragma unroll
          for (int qq = 0; qq < kTcSplit; ++qq) {
            v0 += red[(qq * 32 + lane) * 2];
            v1 += red[(qq * 32 + lane) * 2 + 1];
          }
          if (lane == 0) *cnt = 0;   // reset for the slot's next round
        }
      }
      // all smem reads of the tile are done: release the stage to the producer
      __syncwarp();
      if (lane == 0) mbar_arrive(&sm.empty[stage]);
      if (last && gu) {
        // tile rows 0..3 = gate rows, 4..7 = up rows: lanes t4 < 2 (gate) fetch
        // the matching up values from lane ^ 2
        const float u0 = __shfl_xor_sync(0xffffffffu, v0, 2);
        const float u1 = __shfl_xor_sync(0xffffffffu, v1, 2);
        if (g8 < B && t4 < 2) {
          const int b = g8;
          float gv[2] = {v0, v1}, uv[2] = {u0, u1};
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const int j = 2 * t4 + e;
            if (j >= n) continue;
            const int row = r + j;
            float gt = gv[e], up = uv[e];
            if (ph.nseg > 1) {
              float* acc_g = p.kacc + (size_t)b * ph.R * 2 + 2 * row;
              if (ph.seg > 0) {
                gt += acc_g[0];
                up += acc_g[1];
              }
              if (!last_seg) {
                acc_g[0] = gt;
                acc_g[1] = up;
                continue;
              }
            }
            p.a[b * p.ff + row] = gt / (1.0f + expf(-gt)) * up;
          }
        }
      } else if (last && g8 < B) {
        const int b = g8;
        float vv[2] = {v0, v1};
        unsigned long long kb = 0ull;
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          const int j = 2 * t4 + e;
          if (j >= n) continue;
          const int row = r + j;
          float v = vv[e];
          if (ph.nseg > 1) {
            float* acc_r = p.kacc + (size_t)b * ph.R + row;
            if (ph.seg > 0) v += *acc_r;
            if (!last_seg) {
              *acc_r = v;
              continue;
            }
          }
          switch (KIND) {
            case PH_QKV: p.qkv[b * p.qkv_rows + row] = v; break;
            case PH_O:
            case PH_DOWN: p.x[b * p.d + row] += v; break;
            case PH_LM: {
              const unsigned long long kq = argmax_key(v, (uint32_t)row);
              kb = kq > kb ? kq : kb;
              if (p.logits) p.logits[((size_t)(s - (p.P - 1)) * B + b) * p.V + row] = v;
            } break;
            default: break;
          }
        }
        if (KIND == PH_LM && last_seg && kb) atomicMax(&sm.best[b], kb);
      }
      unit_cyc += MX_CLK() - tu;
      ++unit_cnt;
    }
    if (++stage == (uint32_t)n_stages) {
      stage = 0;
      phase_bit ^= 1u;
    }
  }
  if (KIND == PH_LM && last_seg) {
    named_bar_sync(1, kNCT);
    if (tid_c < B) p.cand[cta * B + tid_c] = sm.best[tid_c];
  }
}

template <int B>
__device__ __forceinline__ void gemv_phase(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                           int k, int s, int tid_c, uint32_t& stage,
                                           uint32_t& phase_bit, int n_stages, long long& wait_cyc,
                                           long long& unit_cyc, long long& unit_cnt) {
  constexpr int NR = RowsPerUnit<B>::value;
  constexpr int NRG = NR < 2 ? 2 : NR;   // GU units always hold gate/up pairs
  if constexpr (B >= kTcMinBatch) {
    switch (ph.kind) {
      case PH_QKV:
        gemv_phase_tc<B, PH_QKV>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
        break;
      case PH_O:
        gemv_phase_tc<B, PH_O>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
        break;
      case PH_GU:
        gemv_phase_tc<B, PH_GU>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
        break;
      case PH_DOWN:
        gemv_phase_tc<B, PH_DOWN>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
        break;
      default:
        gemv_phase_tc<B, PH_LM>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
        break;
    }
  } else {
  switch (ph.kind) {
    case PH_QKV:
      gemv_phase_nr<B, NR, PH_QKV>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
      break;
    case PH_O:
      gemv_phase_nr<B, NR, PH_O>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
      break;
    case PH_GU:
      gemv_phase_nr<B, NRG, PH_GU>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
      break;
    case PH_DOWN:
      gemv_phase_nr<B, NR, PH_DOWN>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
      break;
    default:
      gemv_phase_nr<B, NR, PH_LM>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, wait_cyc, unit_cyc, unit_cnt);
      break;
  }
  }
}

template <int B>
__global__ void __launch_bounds__(kDecodeThreads, 1) decode_kernel(DecodeParams p, int n_stages,
                                                                   int kmax) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const Smem sm = carve<B>(smem_raw, n_stages, kmax);
  const int warp_id = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    for (int i = 0; i < n_stages; ++i) {
      mbar_init(&sm.full[i], 1);
      mbar_init(&sm.empty[i], kConsumerWarps);
    }
    fence_mbar_init();
    if (blockIdx.x == 0) p.stamps[0] = globaltimer();
  }
  for (int i = threadIdx.x; i < n_stages * kMaxUnits; i += blockDim.x) sm.cnt[i] = 0;
  if (B >= kTcMinBatch && threadIdx.x < 16) reinterpret_cast<uint32_t*>(sm.zero)[threadIdx.x] = 0u;
  __syncthreads();

  if (warp_id == 0) {
    if ((threadIdx.x & 31) == 0) producer_loop<B>(p, sm, n_stages);
    return;
  }

  const int tid_c = threadIdx.x - 32;
  const int L = p.L, S = p.P + p.G - 1;
  const int pl = phases_per_layer(p.fuse_att);
  uint32_t stage = 0, phase_bit = 0;
  unsigned long long target = p.bar_base;
  long long c_bar = 0, c_stage = 0, c_wait = 0, c_gemv = 0, c_att = 0, c_unit = 0, c_units = 0;
  const long long t_begin = MX_CLK();
  for (int s = 0; s < S; ++s) {
    const int nph = pl * L + (s >= p.P - 1 ? 1 : 0);
    for (int k = 0; k < nph; ++k) {
      const int kind = phase_kind(k, L, p.fuse_att);
      const int layer = k / pl;
      long long t0 = MX_CLK();
      if (kind == PH_ATT) {
        attention_phase<B>(p, sm, layer, s, tid_c);
        const long long t1 = MX_CLK();
        c_att += t1 - t0;
        t0 = t1;
      } else {
        const int nseg = phase_segments<B>(p, kind);
        for (int seg = 0; seg < nseg; ++seg) {
          const Phase ph = make_phase<B>(p, kind, layer, seg);
          stage_input<B>(p, sm, ph, s, tid_c);
          const long long t1 = MX_CLK();
          if (kind == PH_O && p.fuse_att)
            c_att += t1 - t0;
          else
            c_stage += t1 - t0;
          gemv_phase<B>(p, sm, ph, k, s, tid_c, stage, phase_bit, n_stages, c_wait, c_unit, c_units);
          const long long t2 = MX_CLK();
          c_gemv += t2 - t1;
          t0 = t2;
        }
      }
      target += (unsigned long long)p.n_ctas;
      grid_barrier(p, target, tid_c);
      c_bar += MX_CLK() - t0;
    }
  }
  if (p.prof && tid_c == 0) {
    unsigned long long* pr = p.prof + blockIdx.x * 16;
    pr[0] = (unsigned long long)(MX_CLK() - t_begin);
    pr[1] = (unsigned long long)c_bar;
    pr[2] = (unsigned long long)c_stage;
    pr[3] = (unsigned long long)c_wait;
    pr[4] = (unsigned long long)c_gemv;
    pr[5] = (unsigned long long)c_att;
    pr[7] = (unsigned long long)c_unit;
    pr[8] = (unsigned long long)c_units;
  }
  // final token (argmax of the last step)
  if (blockIdx.x == 0) {
    if (tid_c < B) {
      unsigned long long best = 0;
      for (int c = 0; c < p.n_ctas; ++c) {
        const unsigned long long v = p.cand[c * B + tid_c];
        best = v > best ? v : best;
      }
      p.tokens[tid_c * p.G + (p.G - 1)] = (int)argmax_key_index(best);
      __threadfence_system();
    }
    named_bar_sync(1, kNCT);
    if (tid_c == 0) {
      const unsigned long long t_end = globaltimer();
      p.stamps[1] = t_end;
      if (p.inject_err && !p.h_stamps) atomicExch(p.err, p.inject_err);
      if (p.h_stamps) {
        // every CTA passed the last grid barrier, so all outputs are final
        volatile unsigned long long* h = p.h_stamps;
        h[0] = p.stamps[0];
        h[1] = t_end;
        if (p.inject_err) atomicExch(p.err, p.inject_err);   // fault-path test hook
        h[2] = (unsigned long long)(unsigned)ld_volatile_i32(p.err);
        __threadfence_system();
        h[3] = p.done_tag;
      }
    }
  }
}

template <int B>
int launch_b(const DecodeParams& p, void* stream, int cooperative) {
  const int kmax = max(max(p.d, p.q_dim), p.ff);
  int ns = 0;
  const int smem = decode_smem_bytes(B, kmax, &ns);
  if (smem < 0) return -3;
  DecodeParams pc = p;
  int ns_arg = ns, kmax_arg = kmax;
  void* args[] = {&pc, &ns_arg, &kmax_arg};
  return launch_kernel(decode_kernel<B>, dim3(p.n_ctas), dim3(kDecodeThreads), (unsigned)smem,
                       stream, args, cooperative != 0);
}

template <int B>
int set_attrs_b(int device) {
  return set_max_smem(decode_kernel<B>, 227 * 1024, device);
}

}  // namespace mxk

// One translation unit per batch size (parallel compilation).
#define MX_DECODE_INSTANTIATE(B)                                      \
  namespace mxk {                                                     \
  template int launch_b<B>(const DecodeParams& p, void* stream, int); \
  template int set_attrs_b<B>(int device);                            \
  }
