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
//  * every GEMV is a tcgen05 MMA: D[rows][16] = W[rows][K] . X[16][K]^T with
//    the weights as the A operand (M = 128 rows) and the activations as the B
//    operand (N = 16: a bf16 hi/lo pair per sequence, reading A17), fp32
//    accumulators in tensor memory. One elected thread issues the MMAs; four
//    epilogue warps drain the accumulators (tcgen05.ld) and apply the phase's
//    epilogue (residual add, SiLU-gate, argmax). The CUDA cores no longer touch
//    the weights, so the kernel is HBM-bound at any clock.
//  * weights (>98% of the bytes) are streamed by a producer thread with 4-D
//    tiled TMA (one CUtensorMap per matrix kind and box height, covering all
//    layers) into a ring of 32 KiB stages (a tile's exact rows x up to 8
//    64-column blocks, K-major SWIZZLE_128B: the UMMA A-operand layout)
//    guarded by mbarriers; MMA completion (tcgen05.commit) frees a stage. The
//    weight stream is static, so the producer runs ahead ACROSS phase barriers.
//  * rows are split across CTAs in multiples of 8 with a per-phase rotation
//    (rows of other CTAs are never read); inputs wider than the operand
//    region run as K segments whose partials the row owner chains in segment
//    order. When that split would leave < 64 rows per CTA (O/DOWN of a 7B on
//    148 SMs) the (segment, 8-row group) pieces are spread over the CTAs and
//    statically assigned CTAs finish each 128-row block from the partials,
//    summed in the same segment order. Segment boundaries depend only on the
//    shape, so results do not depend on the partition size.
//  * the phase inputs are operand images written by the producing epilogue
//    (one bulk copy per K segment); the RMSNorm scale is an output-column
//    factor the epilogue warps reduce while the MMAs run.
//  * a separate attention phase splits each (sequence, head) over warps by
//    key block (block partials folded in block order, flash-decoding style).
#include <cfloat>

#include "common.cuh"
#include "kernels.h"
#include "launch.cuh"
#include "tc05.cuh"

namespace mxk {

enum PhaseKind { PH_QKV = 0, PH_ATT = 1, PH_O = 2, PH_GU = 3, PH_DOWN = 4, PH_LM = 5 };
// tensor-map matrix index (kernels.h kDecodeMats)
enum DecodeMat { MAT_QKV = 0, MAT_O = 1, MAT_GATE = 2, MAT_UP = 3, MAT_DOWN = 4, MAT_LM = 5 };

constexpr int kNCT = 32 * kConsumerWarps;   // consumer threads
constexpr int kMmaWarp = 1;                 // warp whose lane 0 issues the MMAs
constexpr int kEpiWarp0 = 2;                // warps 2..5 drain TMEM (lane quarter = warp % 4)
constexpr int kStageWarp = 6;               // lane 0 copies the operand images (bulk copies)
constexpr int kAccSlots = 4;                // TMEM accumulator slots of 32 columns
#ifndef MX_MMA_WARP
#define MX_MMA_WARP 2                       // 1: warp-wide issue, one elect per MMA; 2: one elect per K block (tc05.cuh)
#endif
constexpr uint32_t kTmemCols = 32 * kAccSlots;
static_assert(kConsumerWarps >= 5, "MMA warp + 4 epilogue warps");

#ifdef MX_NO_SLEEP
#define MX_FULL_WAIT(b, ph) mbar_try_wait(b, ph)
#else
#define MX_FULL_WAIT(b, ph) mbar_try_wait_sleep(b, ph, 20000u)
#endif
// Bounded mbarrier wait: a launch that would otherwise hang (a protocol error
// or a failed copy) raises *err after 4 s and stops waiting, so the task
// completes with MX_EDEVICE instead of wedging its partition. SPIN = 1 polls
// without the suspend hint (lower wake-up latency for the pipeline roles).
template <int SPIN = 0>
__device__ __forceinline__ void mbar_wait_bounded(uint64_t* bar, uint32_t parity, int* err) {
  auto done = [&]() { return SPIN ? mbar_try_wait(bar, parity) : MX_FULL_WAIT(bar, parity); };
  if (done()) return;
  const uint64_t t0 = globaltimer();
  while (!done()) {
    if (ld_volatile_i32(err)) return;
    if (globaltimer() - t0 > 4000000000ull) {
      atomicExch(err, 1);
      return;
    }
  }
}
#ifndef MX_WAIT_PROD
#define MX_WAIT_PROD 1
#endif
#ifndef MX_WAIT_MMA
#define MX_WAIT_MMA 1
#endif
#ifndef MX_WAIT_EPI
#define MX_WAIT_EPI 0
#endif

// Per-CTA cycle buckets (MX_DECODE_PROF=1) exist only in profiling builds
// (MX_DEFS=-DMX_PROF_BUCKETS).
#ifdef MX_PROF_BUCKETS
#define MX_CLK() clock64()
#else
#define MX_CLK() 0ll
#endif

// One GEMV phase, or one K segment [k0, k0 + K) of it (split-K inside the
// owning CTA when the input is wider than one activation segment; segment
// widths are multiples of 64 and depend only on the shape).
struct Phase {
  int kind, layer, R, KF, K, k0, seg, nseg, nkb, mat, lz;
  int w;     // full segment width (the last segment may be narrower: K)
  int dist;  // multi-segment phase whose (segment, rows) pieces are spread over the CTAs
};

__host__ __device__ __forceinline__ int round64(int k) { return (k + 63) & ~63; }

// K segments of a phase: one when the input fits the operand region (64 KiB),
// else segments of at most half of it, so that the operand of segment s + 1 is
// copied into one half while the MMAs of segment s read the other.
template <int B>
__device__ __forceinline__ int phase_segments(const DecodeParams& p, int kind) {
  if (kind == PH_ATT) return 1;
  const int KF = (kind == PH_O) ? p.q_dim : (kind == PH_DOWN) ? p.ff : p.d;
  const int R = (kind == PH_QKV) ? p.qkv_rows : (kind == PH_GU) ? p.ff : (kind == PH_LM) ? p.V : p.d;
  return decode_nseg(B, R, KF, !(kind == PH_O && p.fuse_att));
}

template <int B>
__device__ __forceinline__ Phase make_phase(const DecodeParams& p, int kind, int layer, int seg) {
  Phase ph;
  ph.kind = kind;
  ph.layer = layer;
  ph.lz = layer;
  switch (kind) {
    case PH_QKV: ph.R = p.qkv_rows; ph.KF = p.d; ph.mat = MAT_QKV; break;
    case PH_O: ph.R = p.d; ph.KF = p.q_dim; ph.mat = MAT_O; break;
    case PH_GU: ph.R = p.ff; ph.KF = p.d; ph.mat = MAT_GATE; break;
    case PH_DOWN: ph.R = p.d; ph.KF = p.ff; ph.mat = MAT_DOWN; break;
    default: ph.R = p.V; ph.KF = p.d; ph.mat = MAT_LM; ph.lz = 0; break;
  }
  ph.nseg = phase_segments<B>(p, kind);
  const int w = (ph.nseg == 1) ? round64(ph.KF)
                               : ((ph.KF + ph.nseg - 1) / ph.nseg + kSegGrain - 1) / kSegGrain * kSegGrain;
  ph.seg = seg;
  ph.w = w;
  // a plain row split would leave a CTA < 64 rows per MMA (issue-bound: a
  // skinny MMA costs the same for 8 or 128 rows), so spread the pieces; else
  // each CTA runs every segment of its rows and chains the partials itself.
  // Either way the row's sum is ((p0 + p1) + p2) + ...: the same bits.
  ph.dist = ((kind == PH_O || kind == PH_DOWN) && ph.nseg > 1 && ph.R < 64 * p.n_ctas) ? 1 : 0;
  ph.k0 = seg * w;
  ph.K = min(w, ph.KF - ph.k0);
  ph.nkb = (ph.K + kBlkK - 1) / kBlkK;
  return ph;
}


// Rows [r0, r1) of a phase owned by this CTA: boundaries at multiples of 8
// (the last is R); `rot` rotates the assignment so remainders land on
// different CTAs in different phases.
__device__ __forceinline__ void my_rows(int R, int C, int cta, int rot, int* r0, int* r1) {
  // 32-bit arithmetic: R * C < 2^32 for every admitted shape (R <= 2^24, C <= kMaxCtas)
  const uint32_t c = (uint32_t)(cta + rot) % (uint32_t)C;
  *r0 = (int)(((uint32_t)R * c) / (uint32_t)C) & ~7;
  *r1 = (c + 1 == (uint32_t)C) ? R : ((int)(((uint32_t)R * (c + 1)) / (uint32_t)C) & ~7);
}

// Multi-segment phases: the work (segment g, 8-row group i), ordered segment-
// major and weighted by the segment's width, is cut into n_ctas equal
// contiguous ranges; CTA c's piece of segment g is the rows [r0, r1) of its
// range inside g (empty for most g). Which CTA computes a partial does not
// change its value, so results do not depend on the partition size.
__device__ __forceinline__ void seg_pos(long long T, int G8, int w, int KF, int nseg, int* g,
                                        int* i) {
  const long long segW = (long long)G8 * w;
  const int gg = (int)min(T / segW, (long long)(nseg - 1));
  const int wg = min(w, KF - gg * w);
  *g = gg;
  *i = (int)min((T - gg * segW) / wg, (long long)G8);
}

// This CTA's pieces of a multi-segment phase kind (computed once per launch,
// kept in shared memory): segments [ga, gb], rows [r0a, R) of ga ... rows
// [0, r1b) of gb (ga > gb: none).
__device__ __forceinline__ void cta_span(const Phase& ph, int C, int cta, int* sp) {
  const int G8 = (ph.R + 7) >> 3;
  const long long W = (long long)G8 * ph.KF;
  int gs, is, ge, ie;
  seg_pos(W * cta / C, G8, ph.w, ph.KF, ph.nseg, &gs, &is);
  seg_pos(W * (cta + 1) / C, G8, ph.w, ph.KF, ph.nseg, &ge, &ie);
  int ga = gs, r0a = is * 8, gb = ge, r1b = min(ie * 8, ph.R);
  if (r0a >= ph.R) {
    ++ga;
    r0a = 0;
  }
  if (r1b <= 0) {
    --gb;
    r1b = ph.R;
  }
  if (ga > gb || (ga == gb && r0a >= r1b)) {
    ga = 1;
    gb = 0;
  }
  sp[0] = ga;
  sp[1] = r0a;
  sp[2] = gb;
  sp[3] = r1b;
}

__device__ __forceinline__ void piece_rows(const Phase& ph, const int* span, int C, int cta, int k,
                                           int* r0, int* r1) {
  if (!ph.dist) {
    my_rows(ph.R, C, cta, k, r0, r1);
    return;
  }
  const int* sp = span + 4 * ph.kind;
  const int g = ph.seg;
  if (g < sp[0] || g > sp[2]) {
    *r0 = *r1 = 0;
    return;
  }
  *r0 = (g == sp[0]) ? sp[1] : 0;
  *r1 = (g == sp[2]) ? sp[3] : ph.R;
}

__host__ __device__ __forceinline__ int phases_per_layer(int fuse_att) { return fuse_att ? 4 : 5; }

__device__ __forceinline__ int phase_kind(int k, int L, int fuse_att) {
  const int pl = phases_per_layer(fuse_att);
  if (k == pl * L) return PH_LM;
  const int r = k % pl;
  if (fuse_att) return r == 0 ? PH_QKV : r == 1 ? PH_O : r == 2 ? PH_GU : PH_DOWN;
  return r;   // QKV, ATT, O, GU, DOWN
}

struct Smem {
  uint8_t* ring;             // [n_stages][kStageBytes] weight boxes (1024-aligned)
  uint8_t* act;              // activation operand (B rows hi + B rows lo, SWIZZLE_128B)
  float* att;                // [kConsumerWarps][3][kAttHd]
  uint64_t* full;            // [n_stages] TMA -> MMA
  uint64_t* empty;           // [n_stages] MMA -> TMA
  uint64_t* tfull;           // [kAccSlots] MMA -> epilogue
  uint64_t* tempty;          // [kAccSlots] epilogue -> MMA
  uint64_t* actfull;         // [2] operand half: bulk copy -> MMA
  uint64_t* actfree;         // [2] operand half: MMAs done -> next bulk copy
  unsigned long long* best;  // [8]
  int* tok;                  // [8]
  float* wsum;               // [kConsumerWarps][8]
  float* inv;                // [8] RMSNorm scale of the phase input (kept across K segments)
  int* span;                 // [6][4] this CTA's pieces per multi-segment phase kind (cta_span)
  uint32_t* tmem;            // TMEM base address
};

template <int B>
__device__ __forceinline__ Smem carve(uint8_t* raw, int n_stages, int kmax, int fuse_att) {
  Smem s;
  uint8_t* p = raw + ((1024 - (smem_u32(raw) & 1023)) & 1023);
  s.ring = p;
  p += (size_t)n_stages * kStageBytes;
  s.act = p;
  p += (size_t)decode_act_bytes(B, kmax);
  if (decode_att_in_act(B, kmax, fuse_att)) {
    // separate attention phase: the operand is idle while attention runs
    s.att = reinterpret_cast<float*>(s.act);
  } else {
    s.att = reinterpret_cast<float*>(p);
    p += (size_t)kConsumerWarps * 3 * kAttHd * 4;
  }
  s.full = reinterpret_cast<uint64_t*>(p);
  p += (size_t)n_stages * 8;
  s.empty = reinterpret_cast<uint64_t*>(p);
  p += (size_t)n_stages * 8;
  s.tfull = reinterpret_cast<uint64_t*>(p);
  p += kAccSlots * 8;
  s.tempty = reinterpret_cast<uint64_t*>(p);
  p += kAccSlots * 8;
  s.actfull = reinterpret_cast<uint64_t*>(p);
  p += 16;
  s.actfree = reinterpret_cast<uint64_t*>(p);
  p += 16;
  s.best = reinterpret_cast<unsigned long long*>(p);
  p += 8 * 8;
  s.tok = reinterpret_cast<int*>(p);
  p += 8 * 4;
  s.wsum = reinterpret_cast<float*>(p);
  p += (size_t)kConsumerWarps * 8 * 4;
  s.inv = reinterpret_cast<float*>(p);
  p += 8 * 4;
  s.span = reinterpret_cast<int*>(p);
  p += 6 * 4 * 4;
  s.tmem = reinterpret_cast<uint32_t*>(p);
  return s;
}

// Byte offset of 16-byte chunk q (columns 8q..8q+7 of the segment) of operand
// row `row` in the activation operand: 64-column blocks, 8-row atoms of 1 KiB,
// chunk index XOR (row & 7) inside an atom (the SWIZZLE_128B pattern).
template <int B>
__device__ __forceinline__ uint32_t act_off(int row, int q) {
  const int ch = q & 7, r = row & 7;
  return (uint32_t)((q >> 3) * decode_act_blk_bytes(B) + (row >> 3) * 1024 + r * 128 +
                    ((ch ^ r) << 4));
}

// fp32 -> bf16 hi/lo pair (x = hi + lo to ~16 mantissa bits, reading A17).
__device__ __forceinline__ void split8(const float (&f)[8], uint4& hi, uint4& lo) {
  uint16_t h[8], l[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    h[j] = f32_to_bf16_rne(f[j]);
    l[j] = f32_to_bf16_rne(f[j] - bf16_bits_to_f32(h[j]));
  }
  hi = make_uint4(h[0] | ((uint32_t)h[1] << 16), h[2] | ((uint32_t)h[3] << 16),
                  h[4] | ((uint32_t)h[5] << 16), h[6] | ((uint32_t)h[7] << 16));
  lo = make_uint4(l[0] | ((uint32_t)l[1] << 16), l[2] | ((uint32_t)l[3] << 16),
                  l[4] | ((uint32_t)l[5] << 16), l[6] | ((uint32_t)l[7] << 16));
}

// One activation element (sequence b, column col) into an operand laid out as
// above: the shared-memory operand (segment column) or a global operand image
// (input column).
template <int B>
__device__ __forceinline__ void act_store1(uint8_t* base, int b, int col, float v) {
  const uint16_t h = f32_to_bf16_rne(v);
  const uint16_t l = f32_to_bf16_rne(v - bf16_bits_to_f32(h));
  const uint32_t e = (uint32_t)(col & 7) * 2u;
  *reinterpret_cast<uint16_t*>(base + act_off<B>(b, col >> 3) + e) = h;
  *reinterpret_cast<uint16_t*>(base + act_off<B>(decode_act_lo(B) + b, col >> 3) + e) = l;
}

// Columns [n, round64(n)) of every sequence of an operand image: the last
// block's padding, multiplied by weight columns past the input width (the
// tensor maps read them from the next row). Written by the writer of column
// n - 1: a slot's image is shared by tasks of different batch layouts.
template <int B>
__device__ __forceinline__ void img_zero_tail(uint8_t* img, int n) {
  for (int c = n; c < round64(n); ++c)
#pragma unroll
    for (int b = 0; b < B; ++b) act_store1<B>(img, b, c, 0.f);
}

// Generic-proxy global writes (operand images) -> later async-proxy reads
// (bulk copies issued by other CTAs after the grid barrier).
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

// Device-wide barrier among all CTAs of the launch (consumer warps only; the
// producer warp never waits on it). A 4 s timeout sets *err; afterwards every
// barrier passes without waiting, so a failed launch still terminates.
__device__ __forceinline__ void grid_barrier(const DecodeParams& p, unsigned long long target,
                                             int tid_c, unsigned long long* tl = nullptr) {
  named_bar_sync(1, kNCT);
  if (tid_c == 0) {
    if (tl) tl[4] = globaltimer();
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
    if (tl) tl[5] = globaltimer();
  }
  named_bar_sync(1, kNCT);
}

// tensor map of matrix `mat` with box height h8 (a multiple of 8, <= 128)
__device__ __forceinline__ const void* tmap(const DecodeParams& p, int mat, int h8) {
  return reinterpret_cast<const uint8_t*>(p.tmaps) + (size_t)(mat * kDecodeBoxH + (h8 >> 3) - 1) * 128;
}

// ---------------------------------------------------------------------------
// Producer: stream this CTA's weight boxes of every phase of every step, in
// the order the MMA thread consumes them: per segment, per 128-row tile, per
// 64-column block, (gate, up) for GU.
// ---------------------------------------------------------------------------
template <int B>
__device__ void producer_loop(const DecodeParams& p, const Smem& sm, int n_stages) {
  const int C = p.n_ctas, cta = blockIdx.x, L = p.L;
  const int S = p.P + p.G - 1;
  const int pl = phases_per_layer(p.fuse_att);
  uint32_t stage = 0, phase_bit = 0;
  long long wait_cyc = 0;
  const uint64_t pol = policy_evict_first();
  for (int i = 0; i < kDecodeMaps; ++i)
    prefetch_tensormap(reinterpret_cast<const uint8_t*>(p.tmaps) + (size_t)i * 128);
  const uint32_t ring0 = smem_u32(sm.ring);
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
        const int nm = (kind == PH_GU) ? 2 : 1;
        int r0, r1;
        piece_rows(ph, sm.span, C, cta, k, &r0, &r1);
        for (int rt = r0; rt < r1; rt += kTileM) {
          const int h8 = (min(kTileM, r1 - rt) + 7) & ~7;
          const int nk = decode_box_blocks(h8);
          const uint32_t bytes = (uint32_t)(h8 * nk * 128);
          for (int kb = 0; kb < ph.nkb; kb += nk) {
            for (int m = 0; m < nm; ++m) {
              const long long tw = MX_CLK();
              mbar_wait_bounded<MX_WAIT_PROD>(&sm.empty[stage], phase_bit ^ 1u, p.err);
              wait_cyc += MX_CLK() - tw;
              // the full box (blocks past K are out of bounds: zero-filled, counted)
              mbar_arrive_expect_tx(&sm.full[stage], bytes);
              tma_load_4d(ring0 + stage * (uint32_t)kStageBytes, tmap(p, ph.mat + m, h8), 0, rt,
                          ph.k0 / kBlkK + kb, ph.lz, &sm.full[stage], pol);
              if (++stage == (uint32_t)n_stages) {
                stage = 0;
                phase_bit ^= 1u;
              }
            }
          }
        }
      }
    }
  }
  if (p.prof) p.prof[cta * 16 + 6] = (unsigned long long)wait_cyc;
}

// ---------------------------------------------------------------------------
// MMA issuer (warp kMmaWarp, every lane runs the loop, one elected lane
// issues): per 128-row tile an accumulator slot in TMEM (32 columns: gate at
// +0, up at +16 for GU), 4 MMAs of K = 16 per 64-column box. tcgen05.commit
// frees each ring stage and, per tile, signals the epilogue.
// ---------------------------------------------------------------------------
template <int B>
__device__ __forceinline__ void mma_phase(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                          int k, uint32_t& stage, uint32_t& phase_bit,
                                          int n_stages, uint32_t& tc, uint32_t tmem_base,
                                          long long& w_full, long long& w_acc,
                                          uint32_t act_byte_off = 0) {
  constexpr uint32_t idesc = umma_idesc_bf16(kTileM, 16);
  constexpr uint32_t sbo = (B <= 4) ? 0u : 1024u;   // B <= 4: the 8-row atom is read twice
  const uint32_t act0 = smem_u32(sm.act) + act_byte_off, ring0 = smem_u32(sm.ring);
  const int nm = (ph.kind == PH_GU) ? 2 : 1;
  const bool lane0 = (threadIdx.x & 31) == 0;
  (void)lane0;
  int r0, r1;
  piece_rows(ph, sm.span, p.n_ctas, blockIdx.x, k, &r0, &r1);
  for (int rt = r0; rt < r1; rt += kTileM) {
    const uint32_t slot = tc % kAccSlots, use = tc / kAccSlots;
    const long long ta = MX_CLK();
    mbar_wait_bounded<MX_WAIT_MMA>(&sm.tempty[slot], (use & 1u) ^ 1u, p.err);
    __syncwarp();
    w_acc += MX_CLK() - ta;
    tc_fence_after();
    const uint32_t dcol = tmem_base + slot * 32u;
    const int h8 = (min(kTileM, r1 - rt) + 7) & ~7;
    const int nk = decode_box_blocks(h8);
    for (int kb = 0; kb < ph.nkb; kb += nk) {
      const int nkc = min(nk, ph.nkb - kb);
      for (int m = 0; m < nm; ++m) {
        const long long tf = MX_CLK();
        mbar_wait_bounded<MX_WAIT_MMA>(&sm.full[stage], phase_bit, p.err);
        __syncwarp();
        w_full += MX_CLK() - tf;
        tc_fence_after();
        const uint32_t d = dcol + 16u * (uint32_t)m;
        const uint32_t sa = ring0 + stage * (uint32_t)kStageBytes;
        for (int j = 0; j < nkc; ++j) {
          // block j of the box: [h8 rows][128 B]; an M = 128 MMA on a tail tile
          // also reads the rows after it (garbage rows -> discarded outputs)
          const uint64_t ad = umma_desc_sw128(sa + (uint32_t)(j * h8 * 128));
          const uint64_t bd =
              umma_desc_sw128(act0 + (uint32_t)((kb + j) * decode_act_blk_bytes(B)), sbo);
#if MX_MMA_WARP == 2
          umma_f16_warp_k64(d, ad, bd, idesc, (kb + j > 0) ? 1u : 0u);
#elif MX_MMA_WARP
#pragma unroll
          for (int jj = 0; jj < kBlkK / 16; ++jj)
            umma_f16_warp(d, ad + 2u * (uint32_t)jj, bd + 2u * (uint32_t)jj, idesc,
                          (kb + j > 0 || jj > 0) ? 1u : 0u);
#else
          if (lane0) {
#pragma unroll
            for (int jj = 0; jj < kBlkK / 16; ++jj)
              umma_f16(d, ad + 2u * (uint32_t)jj, bd + 2u * (uint32_t)jj, idesc,
                       (kb + j > 0 || jj > 0) ? 1u : 0u);
          }
          __syncwarp();
#endif
        }
#if MX_MMA_WARP
        umma_commit_warp(smem_u32(&sm.empty[stage]));   // stage free once these MMAs completed
#else
        if (lane0) umma_commit(smem_u32(&sm.empty[stage]));
        __syncwarp();
#endif
        if (++stage == (uint32_t)n_stages) {
          stage = 0;
          phase_bit ^= 1u;
        }
      }
    }
#if MX_MMA_WARP
    umma_commit_warp(smem_u32(&sm.tfull[slot]));         // accumulator ready for the epilogue
#else
    if (lane0) umma_commit(smem_u32(&sm.tfull[slot]));
    __syncwarp();
#endif
    ++tc;
  }
}

// ---------------------------------------------------------------------------
// Epilogue warps: warp w reads TMEM lanes 32(w%4).. (tile rows) of each tile's
// slot; column n of the accumulator is operand row n: sequence b's value is
// D[b] + D[lo + b] (hi + lo parts). Single-segment phases finish each row
// straight from TMEM; multi-segment phases store the segment's partial
// (kpart) and the CTA completing a row block finishes it (epi_finalize).
// ---------------------------------------------------------------------------

// The phase's output for one row (all 32 lanes of the warp call it, `ok`
// masks rows past the tile): v (and u, the up projection of GU) is the full
// K reduction of sequence b.
template <int B, int KIND>
__device__ __forceinline__ void epi_final(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                          int s, int row, bool ok, int lane, const float (&v)[B],
                                          const float (&u)[B]) {
  float xn[B];
  unsigned long long key[B];
#pragma unroll
  for (int b = 0; b < B; ++b) {
    key[b] = 0ull;
    xn[b] = 0.f;
    if (!ok) continue;
    // normed phases: the operand held x * gain, so the RMSNorm scale of
    // sequence b multiplies the output column here
    switch (KIND) {
      case PH_QKV: p.qkv[b * p.qkv_rows + row] = v[b] * sm.inv[b]; break;
      case PH_O:
      case PH_DOWN: {
        const float t = p.x[b * p.d + row] + v[b];
        p.x[b * p.d + row] = t;
        xn[b] = t;
        break;
      }
      case PH_GU: {
        const float g = v[b] * sm.inv[b], up = u[b] * sm.inv[b];
        act_store1<B>(p.img_a, b, row, g / (1.0f + expf(-g)) * up);
        if (b == 0 && row == ph.R - 1) img_zero_tail<B>(p.img_a, ph.R);
        break;
      }
      case PH_LM: {
        const float y = v[b] * sm.inv[b];
        key[b] = argmax_key(y, (uint32_t)row);
        if (p.logits) p.logits[((size_t)(s - (p.P - 1)) * B + b) * p.V + row] = y;
        break;
      }
      default: break;
    }
  }
  if (KIND == PH_O || KIND == PH_DOWN) {
    // the next normed phase's input: x * gain as an operand image, and the
    // sums of squares of x over 8-row groups (fixed xor tree: independent of
    // the grid); 8-row groups never straddle CTAs or row blocks
    const uint16_t* gn =
        (KIND == PH_O) ? p.w_layers + (uint64_t)ph.layer * p.layer_stride + p.off_gmlp
        : (ph.layer + 1 < p.L) ? p.w_layers + (uint64_t)(ph.layer + 1) * p.layer_stride + p.off_gattn
                               : p.g_final;
    const float gr = ok ? bf16_bits_to_f32(gn[row]) : 0.f;
#pragma unroll
    for (int b = 0; b < B; ++b) {
      float t = xn[b] * xn[b];
      t += __shfl_xor_sync(0xffffffffu, t, 1);
      t += __shfl_xor_sync(0xffffffffu, t, 2);
      t += __shfl_xor_sync(0xffffffffu, t, 4);
      if (ok) {
        if ((lane & 7) == 0) p.ssq[b * (p.d >> 3) + (row >> 3)] = t;
        act_store1<B>(p.img_x, b, row, xn[b] * gr);
        if (b == 0 && row == ph.R - 1) img_zero_tail<B>(p.img_x, ph.R);
      }
    }
  }
  if (KIND == PH_LM) {
#pragma unroll
    for (int b = 0; b < B; ++b) {
      unsigned long long kk = key[b];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long y = __shfl_xor_sync(0xffffffffu, kk, o);
        kk = y > kk ? y : kk;
      }
      if (lane == 0 && kk) atomicMax(&sm.best[b], kk);
    }
  }
}

// partial of segment g, sequence b, at index idx (row, or 2 row + {0, 1} for GU)
__device__ __forceinline__ float* kpart_at(const DecodeParams& p, const Phase& ph, int g, int b, int idx) {
  const size_t rr = (size_t)ph.R * (ph.kind == PH_GU ? 2 : 1);
  return p.kpart + ((size_t)g * p.B + b) * rr + idx;
}

template <int B, int KIND>
__device__ __forceinline__ void epi_phase(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                          int k, int s, int warp, int lane, uint32_t& tc,
                                          uint32_t tmem_base, long long& w_tf) {
  constexpr int LO = decode_act_lo(B);
  constexpr bool gu = (KIND == PH_GU);
  const int q = warp & 3;
  int r0, r1;
  piece_rows(ph, sm.span, p.n_ctas, blockIdx.x, k, &r0, &r1);
  for (int rt = r0; rt < r1; rt += kTileM) {
    const uint32_t slot = tc % kAccSlots, use = tc / kAccSlots;
    ++tc;
    const long long tw = MX_CLK();
    mbar_wait_bounded<MX_WAIT_EPI>(&sm.tfull[slot], use & 1u, p.err);
    __syncwarp();   // tcgen05.ld is .sync.aligned: the warp must be converged
    w_tf += MX_CLK() - tw;
    tc_fence_after();
    const uint32_t taddr = tmem_base + ((uint32_t)(32 * q) << 16) + slot * 32u;
    uint32_t d0[16], d1[16];
    tmem_ld16_nowait(taddr, d0);
    if (gu) tmem_ld16_nowait(taddr + 16u, d1);
    tmem_ld_wait();
    tc_fence_before();
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.tempty[slot]);
    const int row = rt + 32 * q + lane;
    const bool ok = row < r1;
    float v[B], u[B];
#pragma unroll
    for (int b = 0; b < B; ++b) {
      v[b] = __uint_as_float(d0[b]) + __uint_as_float(d0[LO + b]);
      u[b] = gu ? __uint_as_float(d1[b]) + __uint_as_float(d1[LO + b]) : 0.f;
    }
    if (ph.nseg > 1) {   // (warp-uniform branches: the final epilogue uses shuffles)
      if (ph.dist) {
        // distributed: this piece's raw partial (summed by epi_finalize)
        if (ok) {
#pragma unroll
          for (int b = 0; b < B; ++b) {
            if (gu) {
              *reinterpret_cast<float2*>(kpart_at(p, ph, ph.seg, b, 2 * row)) = make_float2(v[b], u[b]);
            } else {
              *kpart_at(p, ph, ph.seg, b, row) = v[b];
            }
          }
        }
        continue;
      }
      // chained: the running sum ((p0 + p1) + ...) of this row's segments so
      // far lives in slot 0 (written by this thread for the earlier segments)
      if (ok) {
        const int idx = gu ? 2 * row : row;
#pragma unroll
        for (int b = 0; b < B; ++b) {
          float* acc = kpart_at(p, ph, 0, b, idx);
          if (ph.seg > 0) {
            v[b] += acc[0];
            if (gu) u[b] += acc[1];
          }
          if (ph.seg < ph.nseg - 1) {
            acc[0] = v[b];
            if (gu) acc[1] = u[b];
          }
        }
      }
      if (ph.seg < ph.nseg - 1) continue;
    }
    epi_final<B, KIND>(p, sm, ph, s, row, ok, lane, v, u);
  }
}

// Distributed multi-segment phases, the 4 epilogue warps after all of this
// CTA's pieces: publish "my partials are stored" (a monotone per-CTA flag =
// the phase's barrier target, release), then finish the row blocks this CTA
// is assigned statically — block j goes to CTA floor(j C / nblk), so the
// epilogue work is spread evenly — once the CTAs that computed the block's
// pieces have published (acquire). A row's sum is ((p0 + p1) + p2) + ...,
// the order of the chained mode, so the bits do not depend on the mode or on
// which CTA computed a piece.
__device__ __forceinline__ void st_release_u64(unsigned long long* a, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(a), "l"(v) : "memory");
}

// CTA owning group i of segment g (the c with T_c < end(g, i) <= T_{c+1},
// T_c = floor(W c / C); see cta_span)
__device__ __forceinline__ int group_owner(const Phase& ph, int C, int g, int i) {
  const long long G8 = (ph.R + 7) >> 3;
  const long long W = G8 * ph.KF;
  const int wg = min(ph.w, ph.KF - g * ph.w);
  const long long E = (long long)g * G8 * ph.w + (long long)(i + 1) * wg;
  return (int)((E * C + W - 1) / W) - 1;
}


template <int B, int KIND>
__device__ __forceinline__ void epi_finalize(const DecodeParams& p, const Smem& sm, const Phase& ph0,
                                             int s, int warp, int lane, unsigned long long seq) {
  constexpr bool gu = (KIND == PH_GU);
  const int et = 32 * (warp & 3) + lane;
  const int R = ph0.R, nseg = ph0.nseg, C = p.n_ctas, cta = blockIdx.x;
  const int G8 = (R + 7) >> 3, nblk = (R + kFinRows - 1) / kFinRows;
  named_bar_sync(2, 128);   // this CTA's partial stores are done (the release is cumulative)
  if (et == 0) st_release_u64(p.pflag + cta, seq);
  const int j0 = (int)(((long long)cta * nblk + C - 1) / C);
  const int j1 = (int)(((long long)(cta + 1) * nblk + C - 1) / C);
  for (int j = j0; j < j1; ++j) {
    // thread g waits for the CTAs holding segment g's groups of block j
    for (int g = et; g < nseg; g += 128) {
      const int i0 = j * (kFinRows / 8), i1 = min(G8, (j + 1) * (kFinRows / 8)) - 1;
      const int c0 = group_owner(ph0, C, g, i0), c1 = group_owner(ph0, C, g, i1);
      for (int c = c0; c <= c1; ++c) {
        if (c == cta) continue;
        const uint64_t t0 = globaltimer();
        while (ld_acquire_u64(p.pflag + c) < seq) {
          if (ld_volatile_i32(p.err)) break;
          if (globaltimer() - t0 > 4000000000ull) {
            atomicExch(p.err, 1);
            break;
          }
        }
      }
    }
    named_bar_sync(2, 128);
    const int row = j * kFinRows + et;   // warp q takes rows 32q.. of the block
    const bool ok = row < R;
    float v[B], u[B];
#pragma unroll
    for (int b = 0; b < B; ++b) {
      v[b] = 0.f;
      u[b] = 0.f;
    }
    if (ok) {
      // partials in segment order, four segments' loads (x B) in flight at a time
      // (only O and DOWN are distributed: one value per row and sequence)
      static_assert(!gu, "gate/up phases are never distributed");
      constexpr int GR = 4;
      for (int g0 = 0; g0 < nseg; g0 += GR) {
        float tv[GR][B];
#pragma unroll
        for (int t = 0; t < GR; ++t) {
#pragma unroll
          for (int b = 0; b < B; ++b)
            tv[t][b] = (g0 + t < nseg) ? __ldcg(kpart_at(p, ph0, g0 + t, b, row)) : 0.f;
        }
#pragma unroll
        for (int t = 0; t < GR; ++t) {
          if (g0 + t < nseg) {
#pragma unroll
            for (int b = 0; b < B; ++b) v[b] = (g0 + t == 0) ? tv[t][b] : tv[t][b] + v[b];
          }
        }
      }
    }
    epi_final<B, KIND>(p, sm, ph0, s, row, ok, lane, v, u);
  }
}

template <int B>
__device__ __forceinline__ void epi_dispatch(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                             int k, int s, int warp, int lane, uint32_t& tc,
                                             uint32_t tmem_base, long long& w_tf) {
  switch (ph.kind) {
    case PH_QKV: epi_phase<B, PH_QKV>(p, sm, ph, k, s, warp, lane, tc, tmem_base, w_tf); break;
    case PH_O: epi_phase<B, PH_O>(p, sm, ph, k, s, warp, lane, tc, tmem_base, w_tf); break;
    case PH_GU: epi_phase<B, PH_GU>(p, sm, ph, k, s, warp, lane, tc, tmem_base, w_tf); break;
    case PH_DOWN: epi_phase<B, PH_DOWN>(p, sm, ph, k, s, warp, lane, tc, tmem_base, w_tf); break;
    default: epi_phase<B, PH_LM>(p, sm, ph, k, s, warp, lane, tc, tmem_base, w_tf); break;
  }
}

// All segments of a phase done: finish multi-segment rows, then make the
// operand images written here visible to the next phase's bulk copies.
template <int B>
__device__ __forceinline__ void epi_close(const DecodeParams& p, const Smem& sm, const Phase& ph0,
                                          int s, int warp, int lane, unsigned long long seq) {
  if (ph0.dist) {   // only O and DOWN phases are distributed (make_phase)
    if (ph0.kind == PH_O)
      epi_finalize<B, PH_O>(p, sm, ph0, s, warp, lane, seq);
    else
      epi_finalize<B, PH_DOWN>(p, sm, ph0, s, warp, lane, seq);
  }
  if (ph0.kind == PH_O || ph0.kind == PH_DOWN || ph0.kind == PH_GU) fence_proxy_async_global();
}

// ---------------------------------------------------------------------------
// Attention for one (sequence b, head h) item by one warp. Writes o_h either to
// global o (separate ATT phase) or into the O phase's activation operand in
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
#pragma unroll
  for (int d = 0; d < DPL; ++d) {
    const int dd = lane * DPL + d;
    const float o = acc[d] / l_run;
    act_store1<B>(to_smem ? sm.act : p.img_o, b, h * HD + dd, o);
    if (!to_smem && b == 0 && h * HD + dd == p.q_dim - 1) img_zero_tail<B>(p.img_o, p.q_dim);
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

// ---------------------------------------------------------------------------
// Separate attention phase, key-block split (flash-decoding inside a CTA):
// item (b, h) goes to CTA (b H + h) mod C; its keys are cut into blocks of KB
// positions, one warp computes one block's softmax partial (block max m_i,
// sum l_i of exp(s - m_i), exp-weighted values a_i) into shared memory, and
// one warp folds the partials in block order (M' = max(M, m_i), rescale by
// exp(M - M') / exp(m_i - M')). The blocks and the fold order depend only on
// t and the shape, so the result does not depend on the partition size.
// ---------------------------------------------------------------------------
template <int B, int HD>
__device__ __forceinline__ void att_block(const DecodeParams& p, const Smem& sm, int layer, int t,
                                          int b, int h, int m, bool writer, int warp, int lane,
                                          float* part) {
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
  const float* base = p.qkv + (size_t)b * p.qkv_rows;
  const size_t cache_row0 = ((((size_t)layer * B + b) * Hkv + kvh) * p.max_seq) * HD;
  uint16_t* kcache = p.kc + cache_row0;
  uint16_t* vcache = p.vc + cache_row0;
  const int kslot = lane / LPK, kseg = (lane % LPK) * KSEG;
  const int j = m * KB + kslot;
  const bool cur = (t / KB == m);   // this block holds the current token
  // the block's cached keys / values (independent of the current token)
  uint4 kr[KV4];
#pragma unroll
  for (int i = 0; i < KV4; ++i)
    kr[i] = (j < t) ? *reinterpret_cast<const uint4*>(kcache + (size_t)j * HD + kseg + 8 * i)
                    : make_uint4(0, 0, 0, 0);
  uint32_t vv[KB][(DPL + 1) / 2];
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
  // RoPE(q) at position t (every block), RoPE(k) / v of the current token
  // (its block only; the cache row is written once per kv head)
#pragma unroll
  for (int pi = 0; pi < PPL; ++pi) {
    const int i = lane + 32 * pi;
    if (i < HALF) {
      const float c = p.rope_cs[((size_t)t * HALF + i) * 2 + 0];
      const float sn = p.rope_cs[((size_t)t * HALF + i) * 2 + 1];
      const float q1 = base[h * HD + i], q2 = base[h * HD + i + HALF];
      qs[i] = q1 * c - q2 * sn;
      qs[i + HALF] = q2 * c + q1 * sn;
      if (cur) {
        const float* kb = base + p.q_dim + kvh * HD;
        const float k1 = kb[i], k2 = kb[i + HALF];
        const float* vb = base + p.q_dim + p.kv_dim + kvh * HD;
        const uint16_t kb1 = f32_to_bf16_rne(k1 * c - k2 * sn);
        const uint16_t kb2 = f32_to_bf16_rne(k2 * c + k1 * sn);
        const uint16_t vb1 = f32_to_bf16_rne(vb[i]);
        const uint16_t vb2 = f32_to_bf16_rne(vb[i + HALF]);
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
  }
  __syncwarp();
  float dot = 0.f;
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
  const float sc = (j <= t) ? dot / sqrtf((float)HD) : -FLT_MAX;
  const float bm = warp_max(sc);
  const float ej = (j <= t) ? expf(sc - bm) : 0.f;
  const float l = warp_sum((lane % LPK) == 0 ? ej : 0.f);
  float acc[DPL];
#pragma unroll
  for (int d = 0; d < DPL; ++d) acc[d] = 0.f;
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
#pragma unroll
  for (int d = 0; d < DPL; ++d) part[lane * DPL + d] = acc[d];
  if (lane == 0) {
    part[HD] = bm;
    part[HD + 1] = l;
  }
  __syncwarp();
}

// Fold of one item's block partials (block order) -> o_h in the O phase's image.
template <int B, int HD>
__device__ __forceinline__ void att_fold(const DecodeParams& p, int b, int h, int nb,
                                         const float* part, int lane) {
  constexpr int DPL = HD / 32;
  float M = -FLT_MAX, L = 0.f, acc[DPL];
#pragma unroll
  for (int d = 0; d < DPL; ++d) acc[d] = 0.f;
  for (int m = 0; m < nb; ++m) {
    const float* pm = part + m * (HD + 2);
    const float mi = pm[HD], li = pm[HD + 1];
    const float Mn = fmaxf(M, mi);
    const float sa = expf(M - Mn), sb = expf(mi - Mn);
    L = L * sa + li * sb;
#pragma unroll
    for (int d = 0; d < DPL; ++d) acc[d] = acc[d] * sa + pm[lane * DPL + d] * sb;
    M = Mn;
  }
#pragma unroll
  for (int d = 0; d < DPL; ++d) {
    const int dd = lane * DPL + d;
    act_store1<B>(p.img_o, b, h * HD + dd, acc[d] / L);
    if (b == 0 && h * HD + dd == p.q_dim - 1) img_zero_tail<B>(p.img_o, p.q_dim);
  }
}

template <int B, int HD>
__device__ __forceinline__ void attention_split(const DecodeParams& p, const Smem& sm, int layer,
                                                int t, int tid_c, float* part_base, int avail) {
  constexpr int KB = (HD <= 64) ? 32 : 16;
  constexpr int PW = HD + 2;
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const int C = p.n_ctas, cta = blockIdx.x, items = B * p.H, group = p.H / p.Hkv;
  const int nb = t / KB + 1;
  const int slots = avail / (nb * PW);
  const int n_my = (cta < items) ? (items - cta + C - 1) / C : 0;
  for (int i0 = 0; i0 < n_my; i0 += slots) {
    const int ni = min(slots, n_my - i0);
    for (int task = warp; task < ni * nb; task += kConsumerWarps) {
      const int sl = task / nb, m = task - sl * nb;
      const int it = cta + (i0 + sl) * C;
      const int b = it / p.H, h = it - b * p.H;
      att_block<B, HD>(p, sm, layer, t, b, h, m, (h % group) == 0, warp, lane,
                       part_base + (size_t)(sl * nb + m) * PW);
    }
    named_bar_sync(1, kNCT);
    for (int sl = warp; sl < ni; sl += kConsumerWarps) {
      const int it = cta + (i0 + sl) * C;
      const int b = it / p.H, h = it - b * p.H;
      att_fold<B, HD>(p, b, h, nb, part_base + (size_t)sl * nb * PW, lane);
    }
    named_bar_sync(1, kNCT);   // the partial region is reused by the next round
  }
}

// Shared-memory floats the key-block split may use for its partials (0: not
// available, every item runs whole in one warp): the operand region past the
// attention scratch (the operand is idle during the attention phase).
template <int B>
__device__ __forceinline__ int att_part_floats(const DecodeParams& p, int kmax) {
  const int act = decode_act_bytes(B, kmax);
  const int used = decode_att_in_act(B, kmax, p.fuse_att) ? kConsumerWarps * 3 * kAttHd * 4 : 0;
  const int kb = (p.hd <= 64) ? 32 : 16;
  const int need = ((p.max_seq - 1) / kb + 1) * (p.hd + 2);
  const int avail = (act - used) / 4;
  return avail >= need ? avail : 0;
}

// Separate attention phase (large attention).
template <int B>
__device__ void attention_phase(const DecodeParams& p, const Smem& sm, int layer, int t,
                                int tid_c, int kmax) {
  const int warp = tid_c >> 5, lane = tid_c & 31;
  const int avail = att_part_floats<B>(p, kmax);
  if (avail > 0) {
    float* part = reinterpret_cast<float*>(
        sm.act + (decode_att_in_act(B, kmax, p.fuse_att) ? kConsumerWarps * 3 * kAttHd * 4 : 0));
    switch (p.hd) {
      case 32: attention_split<B, 32>(p, sm, layer, t, tid_c, part, avail); break;
      case 64: attention_split<B, 64>(p, sm, layer, t, tid_c, part, avail); break;
      default: attention_split<B, 128>(p, sm, layer, t, tid_c, part, avail); break;
    }
  } else {
    // items spread over all warps of all CTAs, one warp per (b, h)
    const int items = B * p.H;
    const int stride = p.n_ctas * kConsumerWarps;
    const int group = p.H / p.Hkv;
    for (int it = blockIdx.x * kConsumerWarps + warp; it < items; it += stride) {
      const int b = it / p.H, h = it - b * p.H;
      attend<B>(p, sm, layer, t, b, h, (h % group) == 0, false, warp, lane);
    }
  }
  // o image -> the O phase's bulk copies; the scratch (inside the operand
  // region) -> the next bulk copy into it
  fence_proxy_async_global();
  fence_proxy_async();
}

// ---------------------------------------------------------------------------
// Phase input -> activation operand. The phase that produces an input writes
// it as a global operand image (act_store1 layout, x already multiplied by the
// next norm's gain), so staging a K segment is ONE bulk copy of its blocks;
// the RMSNorm scale 1/rms(x) of sequence b is a per-column factor of the
// GEMV's output, applied by the epilogue (sm.inv), and rms(x) is reduced here
// from the producer's 8-row sums of squares while the copy is in flight.
// Exceptions: the layer-0 QKV input (embedding rows of the tokens, staged
// item by item) and the fused-attention O input (computed into the operand).
// ---------------------------------------------------------------------------
constexpr int kCache = 2;
constexpr int kDecodeTl = 2560;   // timeline words in the profile buffer (after [n_ctas][16])

// Fixed-order RMSNorm reduction of the per-thread partials acc[b]: warp
// shuffle trees, then warps in order; sm.inv[b] = 1 / sqrt(mean + eps).
template <int B>
__device__ __forceinline__ void norm_finish(const DecodeParams& p, const Smem& sm, float (&acc)[B],
                                            int KF, int tid_c) {
  const int warp = tid_c >> 5, lane = tid_c & 31;
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
}

// Operand-image phases, the 4 epilogue warps only (the MMAs start as soon as
// the operand copy lands; only the epilogue needs the RMSNorm scale): reset the
// LM argmax, reduce rms(x) from the producer's sums of squares over 8-row
// groups (the group -> thread assignment and the warp order are fixed: the
// result does not depend on the grid).
template <int B>
__device__ __forceinline__ void epi_prep(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                         int warp, int lane) {
  const int q = warp & 3, et = 32 * q + lane;
  if (ph.kind == PH_LM && et < B) sm.best[et] = 0ull;
  if (ph.kind == PH_QKV || ph.kind == PH_GU || ph.kind == PH_LM) {
    const int G8 = ph.KF >> 3;
    float acc[B];
#pragma unroll
    for (int b = 0; b < B; ++b) acc[b] = 0.f;
    for (int g = et; g < G8; g += 128) {
#pragma unroll
      for (int b = 0; b < B; ++b) acc[b] += p.ssq[b * G8 + g];
    }
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const float t = warp_sum(acc[b]);
      if (lane == 0) sm.wsum[q * 8 + b] = t;
    }
    named_bar_sync(2, 128);
    if (et < B) {
      float t = 0.f;
      for (int w = 0; w < 4; ++w) t += sm.wsum[w * 8 + et];
      sm.inv[et] = 1.0f / sqrtf(t / (float)ph.KF + p.eps);
    }
  }
  named_bar_sync(2, 128);
}

__device__ __forceinline__ bool img_phase(const DecodeParams& p, int kind, int layer) {
  return !(kind == PH_QKV && layer == 0) && !(kind == PH_O && p.fuse_att);
}

// Operand-image phases, one thread: copy segment ph's blocks of the image into
// operand half `buf` (the whole region when the phase has one segment) once the
// MMAs of that half's previous use (`use` - 1) have completed.
template <int B>
__device__ __forceinline__ void issue_img_copy(const DecodeParams& p, const Smem& sm,
                                               const Phase& ph, uint32_t buf, uint32_t use) {
  if (use > 0) {
    while (!mbar_try_wait(&sm.actfree[buf], (use - 1) & 1u)) {
    }
  }
  const uint8_t* img = (ph.kind == PH_O) ? p.img_o : (ph.kind == PH_DOWN) ? p.img_a : p.img_x;
  const uint32_t blk = (uint32_t)decode_act_blk_bytes(B);
  const uint32_t bytes = (uint32_t)ph.nkb * blk;
  const uint8_t* src = img + (size_t)(ph.k0 / kBlkK) * blk;
  uint8_t* dst = sm.act + buf * (uint32_t)(decode_act_bytes(B, decode_seg_cols(B)) / 2);
  fence_proxy_async_global();
  mbar_arrive_expect_tx(&sm.actfull[buf], bytes);
  for (uint32_t o = 0; o < bytes; o += 16384u)
    bulk_g2s(dst + o, src + o, min(16384u, bytes - o), &sm.actfull[buf]);
}

template <int B>
__device__ __forceinline__ void stage_act(const DecodeParams& p, const Smem& sm, const Phase& ph,
                                          int s, int tid_c, bool prologue, bool fill) {
  const int kind = ph.kind, layer = ph.layer;
  const int cta = blockIdx.x, C = p.n_ctas;
  const int warp = tid_c >> 5, lane = tid_c & 31;
  constexpr int LO = decode_act_lo(B);
  const int K = ph.K, k0 = ph.k0, KF = ph.KF;
  const int nq = ph.nkb * 8;            // 16-byte chunks per operand row
  if (!prologue) named_bar_sync(1, kNCT);   // the previous segment's MMAs have completed
  if (kind == PH_LM && prologue && tid_c < B) sm.best[tid_c] = 0ull;
  if (kind == PH_O && p.fuse_att) {
    // every CTA computes all heads (small attention): o lands in the operand
    for (int i = tid_c; i < B * nq; i += kNCT) {
      const int b = i / nq, q = i - b * nq;
      if (q * 8 >= K) {
        *reinterpret_cast<uint4*>(sm.act + act_off<B>(b, q)) = make_uint4(0, 0, 0, 0);
        *reinterpret_cast<uint4*>(sm.act + act_off<B>(LO + b, q)) = make_uint4(0, 0, 0, 0);
      }
    }
    const int group = p.H / p.Hkv;
    for (int it = warp; it < B * p.H; it += kConsumerWarps) {
      const int b = it / p.H, h = it - b * p.H;
      attend<B>(p, sm, layer, s, b, h, cta == 0 && (h % group) == 0, true, warp, lane);
    }
    fence_proxy_async();
    named_bar_sync(1, kNCT);
    return;
  }
  // --- layer-0 QKV: embedding rows of the step's tokens ---------------------
  if (prologue) {
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
  const uint16_t* emb = p.embed;
  const uint16_t* gain = p.w_layers + p.off_gattn;
  // 8 input values of sequence b at input column col (col < KF)
  auto load8 = [&](int b, int col, float (&f)[8]) {
    unpack8(*reinterpret_cast<const uint4*>(emb + (size_t)sm.tok[b] * KF + col), f);
  };
  const int n_items = B * nq;
  // single pass: the whole input is this segment and fits the register cache
  const bool cached = fill && (ph.nseg == 1) && (n_items <= kCache * kNCT);
  float cv[kCache][8];
  if (cached) {
#pragma unroll
    for (int u = 0; u < kCache; ++u) {
      const int i = tid_c + u * kNCT;
      const int b = i / nq, q = i - b * nq;
      if (i < n_items && q * 8 < K) {
        load8(b, k0 + q * 8, cv[u]);
      } else {
#pragma unroll
        for (int j = 0; j < 8; ++j) cv[u][j] = 0.f;
      }
    }
  }
  if (prologue) {
    // RMSNorm over the FULL input (normalise, then scale; eps inside the sqrt)
    float acc[B];
#pragma unroll
    for (int b = 0; b < B; ++b) acc[b] = 0.f;
    if (cached) {
#pragma unroll
      for (int u = 0; u < kCache; ++u) {
        const int i = tid_c + u * kNCT;
        const int bi = i / nq;
        float t = 0.f;
#pragma unroll
        for (int j = 0; j < 8; ++j) t = fmaf(cv[u][j], cv[u][j], t);
#pragma unroll
        for (int b = 0; b < B; ++b)
          if (b == bi) acc[b] += t;
      }
    } else {
      const int nf = B * (KF / 8);
      for (int base = tid_c; base < nf; base += kCache * kNCT) {
        float f[kCache][8];
#pragma unroll
        for (int u = 0; u < kCache; ++u) {
          const int i = base + u * kNCT;
          if (i < nf) load8(i / (KF / 8), (i % (KF / 8)) * 8, f[u]);
        }
#pragma unroll
        for (int u = 0; u < kCache; ++u) {
          const int i = base + u * kNCT;
          if (i >= nf) continue;
          const int bi = i / (KF / 8);
          float t = 0.f;
#pragma unroll
          for (int j = 0; j < 8; ++j) t = fmaf(f[u][j], f[u][j], t);
#pragma unroll
          for (int b = 0; b < B; ++b)
            if (b == bi) acc[b] += t;
        }
      }
    }
    norm_finish<B>(p, sm, acc, KF, tid_c);
    // the residual stream x = the embedding rows (CTA 0, every column; a
    // single-segment phase writes it while staging)
    if (cta == 0 && ph.nseg > 1) {
      for (int i = tid_c; i < B * (KF / 8); i += kNCT) {
        const int b = i / (KF / 8), col = (i % (KF / 8)) * 8;
        float f[8];
        load8(b, col, f);
        *reinterpret_cast<float4*>(p.x + (size_t)b * p.d + col) = make_float4(f[0], f[1], f[2], f[3]);
        *reinterpret_cast<float4*>(p.x + (size_t)b * p.d + col + 4) = make_float4(f[4], f[5], f[6], f[7]);
      }
    }
    if (!fill) {
      named_bar_sync(1, kNCT);
      return;
    }
  }
  // gain-scaled operand split hi/lo; columns >= K are zero
  auto put = [&](int i, float (&f)[8]) {
    const int b = i / nq, q = i - b * nq;
    const int col = k0 + q * 8;
    if (q * 8 < K) {
      if (cta == 0 && ph.nseg == 1) {
        *reinterpret_cast<float4*>(p.x + (size_t)b * p.d + col) = make_float4(f[0], f[1], f[2], f[3]);
        *reinterpret_cast<float4*>(p.x + (size_t)b * p.d + col + 4) = make_float4(f[4], f[5], f[6], f[7]);
      }
      float g[8];
      unpack8(*reinterpret_cast<const uint4*>(gain + col), g);
#pragma unroll
      for (int j = 0; j < 8; ++j) f[j] = f[j] * g[j];
    } else {
#pragma unroll
      for (int j = 0; j < 8; ++j) f[j] = 0.f;
    }
    uint4 hi, lo;
    split8(f, hi, lo);
    *reinterpret_cast<uint4*>(sm.act + act_off<B>(b, q)) = hi;
    *reinterpret_cast<uint4*>(sm.act + act_off<B>(LO + b, q)) = lo;
  };
  if (cached) {
#pragma unroll
    for (int u = 0; u < kCache; ++u) {
      const int i = tid_c + u * kNCT;
      if (i < n_items) put(i, cv[u]);
    }
  } else {
    for (int base = tid_c; base < n_items; base += kCache * kNCT) {
      float f[kCache][8];
#pragma unroll
      for (int u = 0; u < kCache; ++u) {
        const int i = base + u * kNCT;
        const int b = i / nq, q = i - b * nq;
        if (i < n_items && q * 8 < K) load8(b, k0 + q * 8, f[u]);
      }
#pragma unroll
      for (int u = 0; u < kCache; ++u) {
        const int i = base + u * kNCT;
        if (i < n_items) put(i, f[u]);
      }
    }
  }
  fence_proxy_async();   // generic-proxy operand writes -> tensor-core reads
  named_bar_sync(1, kNCT);
}

template <int B>
__global__ void __launch_bounds__(kDecodeThreads, 1) decode_kernel(DecodeParams p, int n_stages,
                                                                   int kmax) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  const Smem sm = carve<B>(smem_raw, n_stages, kmax, p.fuse_att);
  // warp index through a shuffle: provably warp-uniform, so role branches are
  // uniform and the MMA descriptors stay in uniform registers
  const int warp_id = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < n_stages; ++i) {
      mbar_init(&sm.full[i], 1);
      mbar_init(&sm.empty[i], 1);
    }
    for (int i = 0; i < kAccSlots; ++i) {
      mbar_init(&sm.tfull[i], 1);
      mbar_init(&sm.tempty[i], 4);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&sm.actfull[i], 1);
      mbar_init(&sm.actfree[i], 1);
    }
    fence_mbar_init();
    if (blockIdx.x == 0) p.stamps[0] = globaltimer();
  }
  if (threadIdx.x >= 32 && threadIdx.x < 32 + 6 && threadIdx.x - 32 != PH_ATT) {
    const Phase ph = make_phase<B>(p, (int)threadIdx.x - 32, 0, 0);
    if (ph.dist) cta_span(ph, p.n_ctas, blockIdx.x, sm.span + 4 * ph.kind);
  }
  // operand rows of absent sequences stay zero for the whole launch
  const int act_chunks = decode_act_bytes(B, kmax) / 16;
  for (int i = threadIdx.x; i < act_chunks; i += blockDim.x)
    reinterpret_cast<uint4*>(sm.act)[i] = make_uint4(0, 0, 0, 0);
  if (warp_id == kMmaWarp) tmem_alloc(sm.tmem, kTmemCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = __shfl_sync(0xffffffffu, *sm.tmem, 0);   // warp-uniform

  if (warp_id == 0) {
    if (lane == 0) producer_loop<B>(p, sm, n_stages);
    return;
  }

  const int tid_c = threadIdx.x - 32;
  const int L = p.L, S = p.P + p.G - 1;
  const int pl = phases_per_layer(p.fuse_att);
  uint32_t stage = 0, phase_bit = 0, tc = 0;
  uint32_t img_seq = 0, act_use[2] = {0u, 0u}, mma_use[2] = {0u, 0u};
  unsigned long long target = p.bar_base;
  long long c_bar = 0, c_stage = 0, c_gemv = 0, c_att = 0, w_full = 0, w_acc = 0, w_tf = 0, w_act = 0;
  const long long t_begin = MX_CLK();
  for (int s = 0; s < S; ++s) {
    const int nph = pl * L + (s >= p.P - 1 ? 1 : 0);
    for (int k = 0; k < nph; ++k) {
      const int kind = phase_kind(k, L, p.fuse_att);
      const int layer = k / pl;
#ifdef MX_PROF_BUCKETS
      // timeline (globaltimer) of the phases of layer L/2 at step S/2, per CTA:
      // [0] start [1] operand ready [2] last MMA issued / attention done
      // [3] epilogue done (warp 2) [4] barrier arrive [5] barrier exit
      unsigned long long* tl =
          (p.prof && s == S / 2 && layer == L / 2 && kind != PH_LM)
              ? p.prof + kDecodeTl + ((size_t)blockIdx.x * 5 + (k % pl)) * 6 : nullptr;
#else
      unsigned long long* tl = nullptr;
#endif
      if (tl && tid_c == 0) tl[0] = globaltimer();
      long long t0 = MX_CLK();
      if (kind == PH_ATT) {
        attention_phase<B>(p, sm, layer, s, tid_c, kmax);
        if (tl && tid_c == 0) tl[1] = tl[2] = globaltimer();
        const long long t1 = MX_CLK();
        c_att += t1 - t0;
        t0 = t1;
      } else {
        const int nseg = phase_segments<B>(p, kind);
        const Phase ph0 = make_phase<B>(p, kind, layer, 0);
        // this CTA's segments [ga, gb] (contiguous; empty when ga > gb); a
        // single-segment phase is staged even by a CTA without rows
        const int ga = ph0.dist ? sm.span[4 * kind] : 0;
        const int gb = ph0.dist ? sm.span[4 * kind + 2] : nseg - 1;
        const int n_act = gb - ga + 1 > 0 ? gb - ga + 1 : 0;
        if (img_phase(p, kind, layer)) {
          // the operand of this CTA's next segment is copied into one half while
          // the MMAs of its current segment read the other (kStageWarp lane 0
          // runs the copies)
          const uint32_t img0 = img_seq;
          img_seq += (uint32_t)n_act;
          const bool stager = (warp_id == kStageWarp);   // lane 0 issues, the warp stays converged
          auto half = [&](int seg) { return nseg == 1 ? 0u : (img0 + (uint32_t)(seg - ga)) & 1u; };
          auto copy_seg = [&](int seg) {
            const uint32_t hb = half(seg);
            if (lane == 0) issue_img_copy<B>(p, sm, make_phase<B>(p, kind, layer, seg), hb, act_use[hb]);
            ++act_use[hb];
            __syncwarp();
          };
          if (stager && n_act > 0) copy_seg(ga);
          if (tl && tid_c == 0) tl[1] = globaltimer();
          const long long t1 = MX_CLK();
          c_stage += t1 - t0;
          if (stager) {
            for (int seg = ga + 1; seg <= gb; ++seg) copy_seg(seg);
          } else if (warp_id == kMmaWarp) {
            for (int seg = ga; seg <= gb; ++seg) {
              const Phase ph = make_phase<B>(p, kind, layer, seg);
              const uint32_t hb = half(seg);
              const long long tw = MX_CLK();
              while (!mbar_try_wait(&sm.actfull[hb], mma_use[hb] & 1u)) {
              }
              __syncwarp();
              w_act += MX_CLK() - tw;
              ++mma_use[hb];
              mma_phase<B>(p, sm, ph, k, stage, phase_bit, n_stages, tc, tmem_base, w_full, w_acc,
                           hb * (uint32_t)(decode_act_bytes(B, decode_seg_cols(B)) / 2));
              umma_commit_warp(smem_u32(&sm.actfree[hb]));   // half free once these MMAs completed
            }
            if (tl && lane == 0) tl[2] = globaltimer();
          } else if (warp_id >= kEpiWarp0 && warp_id < kEpiWarp0 + 4) {
            epi_prep<B>(p, sm, ph0, warp_id, lane);
            for (int seg = ga; seg <= gb; ++seg)
              epi_dispatch<B>(p, sm, make_phase<B>(p, kind, layer, seg), k, s, warp_id, lane, tc,
                              tmem_base, w_tf);
            epi_close<B>(p, sm, ph0, s, warp_id, lane, target + (unsigned long long)p.n_ctas);
            if (tl && tid_c == 32) tl[3] = globaltimer();
          }
          const long long t2 = MX_CLK();
          c_gemv += t2 - t1;
          t0 = t2;
        } else {
          // layer-0 QKV (embedding rows) or the fused-attention O phase (never
          // distributed: every CTA runs all segments, so the prologue — input
          // tokens, RMSNorm / attention — runs everywhere)
          for (int seg = ga; seg <= gb; ++seg) {
            const Phase ph = make_phase<B>(p, kind, layer, seg);
            stage_act<B>(p, sm, ph, s, tid_c, seg == ga, true);
            if (tl && tid_c == 0 && seg == ga) tl[1] = globaltimer();
            const long long t1 = MX_CLK();
            if (kind == PH_O && p.fuse_att)
              c_att += t1 - t0;
            else
              c_stage += t1 - t0;
            if (warp_id == kMmaWarp) {
              mma_phase<B>(p, sm, ph, k, stage, phase_bit, n_stages, tc, tmem_base, w_full, w_acc);
              if (tl && lane == 0) tl[2] = globaltimer();
            } else if (warp_id >= kEpiWarp0 && warp_id < kEpiWarp0 + 4) {
              epi_dispatch<B>(p, sm, ph, k, s, warp_id, lane, tc, tmem_base, w_tf);
            }
            const long long t2 = MX_CLK();
            c_gemv += t2 - t1;
            t0 = t2;
          }
          if (warp_id >= kEpiWarp0 && warp_id < kEpiWarp0 + 4) {
            epi_close<B>(p, sm, ph0, s, warp_id, lane, target + (unsigned long long)p.n_ctas);
            if (tl && tid_c == 32) tl[3] = globaltimer();
          }
        }
        if (kind == PH_LM) {
          named_bar_sync(1, kNCT);
          if (tid_c < B) p.cand[blockIdx.x * B + tid_c] = sm.best[tid_c];
        }
      }
      target += (unsigned long long)p.n_ctas;
      grid_barrier(p, target, tid_c, tl);
      c_bar += MX_CLK() - t0;
    }
  }
  if (p.prof && tid_c == 0) {
    unsigned long long* pr = p.prof + blockIdx.x * 16;
    pr[0] = (unsigned long long)(MX_CLK() - t_begin);
    pr[1] = (unsigned long long)c_bar;
    pr[2] = (unsigned long long)c_stage;
    pr[3] = (unsigned long long)w_full;
    pr[4] = (unsigned long long)c_gemv;
    pr[5] = (unsigned long long)c_att;
    pr[7] = (unsigned long long)w_acc;
  }
  if (p.prof && tid_c == 32) p.prof[blockIdx.x * 16 + 8] = (unsigned long long)w_tf;
  if (p.prof && tid_c == 0) p.prof[blockIdx.x * 16 + 9] = (unsigned long long)w_act;
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
  // every MMA was waited on by the epilogue warps before the last grid barrier
  tc_fence_before();
  named_bar_sync(1, kNCT);
  if (warp_id == kMmaWarp) {
    tc_fence_after();
    tmem_dealloc(tmem_base, kTmemCols);
  }
}

template <int B>
int launch_b(const DecodeParams& p, void* stream, int cooperative) {
  const int kmax = max(max(p.d, p.q_dim), p.ff);
  int ns = 0;
  const int smem = decode_smem_bytes(B, kmax, &ns, p.fuse_att);
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
