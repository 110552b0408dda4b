// IP-emulator TRAINING step: PAPER.md §3.1 P:109 steps (3)
// and (7) "train an ML model that acts as an emulator of the simulations",
// §3.4 P:163 (training is one of the workflow's two GPU phases). Loss, optimiser
// and state are reading R10: L = (1/M) sum_m (y_m - t_m)^2 over the
// task's molecules, one SGD step theta -= lr * dL/dtheta on fp32 parameters.
//
// Two launches per task on the partition's stream:
//  1. mpnn_train_tile_kernel — one CTA per 128-atom tile (the inference
//     kernel's packing). Every [128 x 128] x [128 x 128] contraction runs on the
//     5th-generation tensor cores (tcgen05.mma, fp32 accumulators in TMEM, one
//     elected lane of warp 0 issues): the forward U h + sum_b W_b s_b with
//     activations AND the fp32 parameters split into bf16 hi/lo terms (three
//     products per K step, reading A17), then per step in reverse order
//     dU^T = h^T-rows . dq-rows, dW_b^T = s_b^T-rows . dq-rows and
//     dh = dq U + sum_b gather_b(dq) W_b with single bf16 terms (gradients are
//     held to 2e-2, R10). Operands are staged in the K-major SWIZZLE_128B layout
//     in whichever orientation makes the reduction index K (transposes happen
//     while staging), h^0..h^T are kept in HBM scratch, the neighbour gathers
//     and the readout / head run on the CUDA cores, and each weight gradient is
//     drained from TMEM into this tile's partial (no atomics).
//  2. mpnn_train_apply_kernel — every parameter element sums the tile
//     partials in tile order (deterministic, independent of the partition
//     size), applies the SGD update in place, and the loss is reduced in
//     molecule order; the last CTA publishes the completion record.
#include "common.cuh"
#include "kernels.h"
#include "launch.cuh"
#include "tc05.cuh"

namespace mxk {

namespace {
constexpr int kF = 128;
constexpr int kA = 128;            // atoms per tile (MMA M / K over atoms)
constexpr int kTE = 512;           // bonds per tile
constexpr int kThreads = 256;      // 8 warps: warp w drains TMEM lanes 32 (w % 4).., columns 64 (w / 4)..
constexpr int kOp = kF * kA * 2;   // one [128][128] bf16 operand (two K-major SWIZZLE_128B halves)
constexpr int kHalf = kOp / 2;

// smem map (bytes from a 1024-aligned base). Forward: H hi/lo, S hi/lo, W hi/lo.
// Backward (single bf16 terms): dqT [f][v], dq [v][f], hT [k][v], X (sT_b [k][v]
// or gq_b [v][f]), Wt [k][f] (U^T or W_b^T), h [v][k].
constexpr int kOffOp0 = 0;                  // H hi | H lo      ; dqT | dq
constexpr int kOffOp1 = kOffOp0 + 2 * kOp;  // S hi | S lo      ; hT  | X
constexpr int kOffOp2 = kOffOp1 + 2 * kOp;  // W hi | W lo      ; Wt  | h
constexpr int kOffNbrOff = kOffOp2 + 2 * kOp;       // int [kA + 4]
constexpr int kOffNbr = kOffNbrOff + (kA + 4) * 4;  // int [2 * kTE]: (u << 2) | b
constexpr int kOffOff4 = kOffNbr + 2 * kTE * 4;     // int [kA][5]: per-bond-type neighbour ranges
constexpr int kOffRed = kOffOff4 + kA * 5 * 4;      // float [4][kF] column partials (dc) / head vectors
constexpr int kOffVec = kOffRed + 4 * kF * 4;       // float [4][kF]: r, a, da, dr
constexpr int kOffC = kOffVec + 4 * kF * 4;         // float [kF] bias c
constexpr int kOffMisc = kOffC + kF * 4;            // float [16]
constexpr int kOffBar = kOffMisc + 64;              // uint64 MMA-done mbarrier, uint64 copy-done mbarrier
constexpr int kOffTmem = kOffBar + 16;              // uint32 TMEM base
constexpr int kMaskT = 8;                            // steps whose ReLU masks fit shared memory
constexpr int kMaskW = 5;                            // words per row (4 + 1 pad: conflict-free)
constexpr int kOffMask = kOffTmem + 16;              // uint32 [kMaskT][kA][kMaskW]: bit f of row v = h^{t+1}[v][f] > 0
constexpr int kTrainSmem = kOffMask + kMaskT * kA * kMaskW * 4 + 1024;   // + alignment slack
static_assert(kTrainSmem <= 227 * 1024, "shared memory plan");
// setup-only aliases inside Op1 (before the first gather)
constexpr int kOffEdges = kOffOp1;                  // int4 [kTE]
constexpr int kOffMolE = kOffOp1 + 16 * kTE;        // int2 [kA]
constexpr uint32_t kTmemCols = 256;                 // acc0: cols 0..127, acc1: cols 128..255
constexpr uint32_t kIdesc = umma_idesc_bf16(128, 128);

// 16-byte chunk ch (columns 8ch..8ch+7) of row `row` of a [128][128] operand
__device__ __forceinline__ uint32_t chunk_off(int row, int ch) {
  return (uint32_t)((ch >> 3) * kHalf + row * 128 + (((ch & 7) ^ (row & 7)) << 4));
}
__device__ __forceinline__ uint32_t elem_off(int row, int col) {
  return chunk_off(row, col >> 3) + (col & 7) * 2;
}

__device__ __forceinline__ uint4 pack8(const uint16_t (&v)[8]) {
  return make_uint4(v[0] | ((uint32_t)v[1] << 16), v[2] | ((uint32_t)v[3] << 16),
                    v[4] | ((uint32_t)v[5] << 16), v[6] | ((uint32_t)v[7] << 16));
}
// two fp32 -> packed bf16 pair (RNE; a in the low half), one conversion instruction
__device__ __forceinline__ uint32_t bf16x2(float a, float b) {
  const __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<const uint32_t*>(&v);
}
// 8 fp32 -> bf16 hi (and lo = bf16(x - hi) if lo != nullptr) at operand chunk (row, ch)
__device__ __forceinline__ void put8(uint8_t* hi, uint8_t* lo, int row, int ch, const float (&f)[8]) {
  uint32_t h[4], l[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    h[j] = bf16x2(f[2 * j], f[2 * j + 1]);
    l[j] = bf16x2(f[2 * j] - __uint_as_float(h[j] << 16), f[2 * j + 1] - __uint_as_float(h[j] & 0xffff0000u));
  }
  const uint32_t o = chunk_off(row, ch);
  *reinterpret_cast<uint4*>(hi + o) = make_uint4(h[0], h[1], h[2], h[3]);
  if (lo) *reinterpret_cast<uint4*>(lo + o) = make_uint4(l[0], l[1], l[2], l[3]);
}
__device__ __forceinline__ void get8(const uint8_t* op, int row, int ch, float (&f)[8]) {
  unpack8(*reinterpret_cast<const uint4*>(op + chunk_off(row, ch)), f);
}

// Weight operand from fp32 parameters W[128][128] (row-major): rows r of the
// operand = W rows (trans = 0) or W columns (trans = 1); hi (+ lo) bf16 terms.
__device__ void stage_w(uint8_t* hi, uint8_t* lo, const float* __restrict__ W, bool trans, int tid) {
  for (int i = tid; i < kF * 16; i += kThreads) {
    const int r = i >> 4, ch = i & 15;
    float f[8];
    if (!trans) {
      const float4 a = *reinterpret_cast<const float4*>(W + r * kF + 8 * ch);
      const float4 b = *reinterpret_cast<const float4*>(W + r * kF + 8 * ch + 4);
      f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w; f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
    } else {
#pragma unroll
      for (int j = 0; j < 8; ++j) f[j] = W[(8 * ch + j) * kF + r];
    }
    put8(hi, lo, r, ch, f);
  }
}

// out[v] = sum over the type-b neighbours u of v of src[u] (edge order), rows
// of [128][128] operands (src hi (+ lo) summed); written as rows (trans = 0,
// hi (+ lo)) or transposed as columns (trans = 1, hi only).
__device__ void gather(uint8_t* out_hi, uint8_t* out_lo, const uint8_t* src_hi, const uint8_t* src_lo,
                       const int* off4, const int* nbr, int na, int b, bool trans, int tid) {
  for (int i = tid; i < kA * 16; i += kThreads) {
    const int v = i >> 4, ch = i & 15;
    const int q0 = (v < na) ? off4[v * 5 + b] : 0, q1 = (v < na) ? off4[v * 5 + b + 1] : 0;
    float acc[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[j] = 0.f;
    for (int q = q0; q < q1; ++q) {
      const int u = nbr[q] >> 2;
      float fh[8];
      get8(src_hi, u, ch, fh);
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[j] += fh[j];
      if (src_lo) {
        float fl[8];
        get8(src_lo, u, ch, fl);
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[j] += fl[j];
      }
    }
    if (!trans) {
      put8(out_hi, out_lo, v, ch, acc);
    } else {
      // column v of the transposed operand: lanes l and l + 16 hold rows v and
      // v + 1 (v even: i = 16 v + ch, 32 consecutive i per warp), one 32-bit
      // word per (f, v pair)
      const int lane = tid & 31;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t b0 = f32_to_bf16_rne(acc[j]);
        const uint32_t b1 = __shfl_down_sync(0xffffffffu, b0, 16);
        if (lane < 16) *reinterpret_cast<uint32_t*>(out_hi + elem_off(8 * ch + j, v)) = b0 | (b1 << 16);
      }
    }
  }
}

// Copy a precomputed operand image (global, L2-resident) into shared memory:
// one bulk (async-proxy) copy issued by ONE thread, completing on
// `cbar`; the other threads go on (neighbour gathers) while it lands. The
// destination's previous readers (MMAs) have completed (waited + barrier).
__device__ __forceinline__ void copy_img_async(uint8_t* dst, const uint8_t* src, int bytes,
                                               uint64_t* cbar) {
  fence_proxy_async();   // earlier generic writes of this shared memory -> async-proxy writes
  mbar_arrive_expect_tx(cbar, (uint32_t)bytes);
  for (int o = 0; o < bytes; o += 16384) bulk_g2s(dst + o, src + o, (uint32_t)min(16384, bytes - o), cbar);
}
__device__ __forceinline__ void copy_wait(uint64_t* cbar, uint32_t& cph) {
  while (!mbar_try_wait(cbar, cph)) {
  }
  cph ^= 1u;
}
// per matrix (U, W_0..W_3): forward image hi | lo ([f][k]) and backward image ([k][f], hi)
constexpr int kImgBytes = 3 * kOp;

// D (+)= A . B^T over K = 128 (8 MMAs of K = 16 per term pair), issued by warp 0
// (warp-uniform descriptors, one elected lane), then committed to `bar`.
__device__ __forceinline__ void mma_128(uint32_t d, uint32_t a, uint32_t b, bool accumulate) {
#pragma unroll
  for (int kk = 0; kk < kF / 16; ++kk) {
    const uint32_t ko = (uint32_t)((kk >> 2) * kHalf + (kk & 3) * 32);
    umma_f16_warp(d, umma_desc_sw128(a + ko), umma_desc_sw128(b + ko), kIdesc,
                  (accumulate || kk > 0) ? 1u : 0u);
  }
}

// every thread: wait for the committed MMAs (phase parity `ph`, flipped after)
__device__ __forceinline__ void mma_wait(uint64_t* bar, uint32_t& ph) {
  while (!mbar_try_wait(bar, ph)) {
  }
  __syncwarp();   // converged for the .sync.aligned tcgen05 loads that follow
  ph ^= 1u;
  tc_fence_after();
}

// This warp's 64 accumulator columns [c0, c0 + 64) of TMEM lane row (32 (w % 4) + lane).
__device__ __forceinline__ void tmem_row64(uint32_t taddr, float (&v)[64]) {
  uint32_t r[4][16];
#pragma unroll
  for (int q = 0; q < 4; ++q) tmem_ld16_nowait(taddr + 16u * q, r[q]);
  tmem_ld_wait();
#pragma unroll
  for (int q = 0; q < 4; ++q)
#pragma unroll
    for (int j = 0; j < 16; ++j) v[16 * q + j] = __uint_as_float(r[q][j]);
}
}  // namespace

int mpnn_train_smem_bytes() { return kTrainSmem; }
// per tile: h^0..h^T ([T+1][k][v]), dh^0 ([k][v]), per molecule (<= 128) dr, r, da ([m][k])
uint64_t mpnn_train_tile_scratch_floats(int T) { return (uint64_t)(T + 5) * kF * kA; }
uint64_t mpnn_train_img_bytes() { return 5ull * kImgBytes; }

// Operand images of the task's fp32 parameters (the same for every tile):
// U and W_b as forward B operands ([f][k], bf16 hi | lo) and backward B
// operands ([k][f], bf16 hi), in the shared-memory layout, one CTA per matrix.
__global__ void __launch_bounds__(kThreads) mpnn_train_prep_kernel(MpnnTrainParams p) {
  const int m = blockIdx.x;   // 0 = U, 1 + b = W_b
  if (m > p.n_bonds) return;
  const float* W = p.params + (m == 0 ? p.off[5] : p.off[1] + (size_t)(m - 1) * kF * kF);
  uint8_t* img = p.wimg + (size_t)m * kImgBytes;
  stage_w(img, img + kOp, W, false, threadIdx.x);
  stage_w(img + 2 * kOp, nullptr, W, true, threadIdx.x);
}

__global__ void __launch_bounds__(kThreads, 1) mpnn_train_tile_kernel(MpnnTrainParams p) {
  extern __shared__ __align__(1024) uint8_t smem_dyn[];
  uint8_t* sm = smem_dyn + ((1024 - (smem_u32(smem_dyn) & 1023)) & 1023);
  uint8_t* op0 = sm + kOffOp0;
  uint8_t* op1 = sm + kOffOp1;
  uint8_t* op2 = sm + kOffOp2;
  int* nbr_off = reinterpret_cast<int*>(sm + kOffNbrOff);
  int* nbr = reinterpret_cast<int*>(sm + kOffNbr);
  int* off4 = reinterpret_cast<int*>(sm + kOffOff4);
  float* red = reinterpret_cast<float*>(sm + kOffRed);
  float* cvec = reinterpret_cast<float*>(sm + kOffC);
  float* misc = reinterpret_cast<float*>(sm + kOffMisc);
  uint64_t* bar = reinterpret_cast<uint64_t*>(sm + kOffBar);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(sm + kOffTmem);
  uint32_t* rmask = reinterpret_cast<uint32_t*>(sm + kOffMask);
  const bool masks_smem = p.T <= kMaskT;   // else the backward reads h^{t+1} from the saved rows
  int4* ed = reinterpret_cast<int4*>(sm + kOffEdges);
  int2* mol_e = reinterpret_cast<int2*>(sm + kOffMolE);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int F = kF;
  if (blockIdx.x == 0 && tid == 0) p.stamps[0] = globaltimer();
  const uint8_t* eb = reinterpret_cast<const uint8_t*>(p.edges);
  const float* E = p.params + p.off[0];
  const float* W1 = p.params + p.off[7];
  const float* c1 = p.params + p.off[8];
  const float* w2 = p.params + p.off[9];
  const float c2 = p.params[p.off[10]];
  uint64_t* cbar = bar + 1;
  if (tid == 0) {
    mbar_init(bar, 1);
    mbar_init(cbar, 1);
    fence_mbar_init();
  }
  if (warp == 0) tmem_alloc(tmem_slot, kTmemCols);
  for (int i = tid; i < F; i += kThreads) cvec[i] = p.params[p.off[6] + i];
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = __shfl_sync(0xffffffffu, *tmem_slot, 0);
  const uint32_t bar_s = smem_u32(bar);
  uint32_t ph = 0, cph = 0;   // MMA-done / copy-done mbarrier parities (every thread tracks both)
  const uint32_t s0 = smem_u32(op0), s1 = smem_u32(op1), s2 = smem_u32(op2);
  const uint32_t acc0 = tmem, acc1 = tmem + 128u;
  // this thread's TMEM row (lane) and column half
  const int trow = 32 * (warp & 3) + lane, tc0 = 64 * (warp >> 2);
  const uint32_t lane_off = (uint32_t)(32 * (warp & 3)) << 16;

  for (int tile = blockIdx.x; tile < p.n_tiles; tile += p.n_ctas) {
    float* G = p.partials + (uint64_t)tile * p.n_params;
    float* hs = p.hsave + (uint64_t)tile * (p.T + 5) * kF * kA;   // [T+1][k][v]
    float* drm = hs + (uint64_t)(p.T + 2) * kF * kA;               // [molecule][k]
    const int m0 = p.tile_off[tile], m1 = p.tile_off[tile + 1];
    const int a0 = p.atom_off[m0], na = p.atom_off[m1] - a0;
    const int e0 = p.edge_off[m0], ne = p.edge_off[m1] - e0;
    {
      // zero this tile's partial except U and the W_b the backward writes whole
      // (W_b of bond types absent from the tile stay zero)
      // (layout: E, W_0..W_3, U, c, W1, c1, w2, c2 in offset order; the zeroed
      // ranges [0, off[1]) and [off[6], n_params) are everything but W_b and U)
      for (int i = tid; i < (int)p.off[1]; i += kThreads) G[i] = 0.f;
      for (int i = (int)p.off[6] + tid; i < p.n_params; i += kThreads) G[i] = 0.f;
    }
    // --- tile CSR (as the inference kernel): edges in tile-local atom ids --------
    for (int i = tid; i < kA; i += kThreads) mol_e[i] = make_int2(0, 0);
    __syncthreads();
    for (int m = m0 + tid; m < m1; m += kThreads) {
      const int ab = p.atom_off[m] - a0, ae = p.atom_off[m + 1] - a0;
      const int eb0 = p.edge_off[m] - e0, ee = p.edge_off[m + 1] - e0;
      for (int v = ab; v < ae; ++v) mol_e[v] = make_int2(eb0, ee);
    }
    for (int i = tid; i < ne; i += kThreads) {
      const uint8_t* e = eb + (size_t)(e0 + i) * 6;
      int lo = m0, hi = m1 - 1;
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (p.edge_off[mid] - e0 <= i) lo = mid; else hi = mid - 1;
      }
      const int base = p.atom_off[lo] - a0;
      ed[i] = make_int4(base + (int)(int16_t)(e[0] | (e[1] << 8)),
                        base + (int)(int16_t)(e[2] | (e[3] << 8)), (int)e[4], 0);
    }
    __syncthreads();
    {
      int deg = 0;
      const int v = tid;
      if (v < kA && v < na) {
        const int2 er = mol_e[v];
        for (int e = er.x; e < er.y; ++e) deg += (ed[e].x == v) + (ed[e].y == v);
      }
      int incl = deg;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += y;
      }
      if (lane == 31 && warp < 4) red[warp] = __int_as_float(incl);
      __syncthreads();
      int base = 0;
      for (int w = 0; w < warp && w < 4; ++w) base += __float_as_int(red[w]);
      if (v < kA) {
        int pos = base + incl - deg;
        nbr_off[v] = pos;
        if (v == kA - 1) nbr_off[kA] = base + incl;
        if (v < na) {
          // bucket v's neighbours by bond type, edge order inside a bucket
          const int2 er = mol_e[v];
          int cnt = 0;   // 8-bit count per bond type
          for (int e = er.x; e < er.y; ++e) {
            const int4 Ev = ed[e];
            cnt += ((Ev.x == v) + (Ev.y == v)) << (8 * Ev.z);
          }
          int o0 = pos, o1 = o0 + (cnt & 255), o2 = o1 + ((cnt >> 8) & 255),
              o3 = o2 + ((cnt >> 16) & 255);
          off4[v * 5 + 0] = o0;
          off4[v * 5 + 1] = o1;
          off4[v * 5 + 2] = o2;
          off4[v * 5 + 3] = o3;
          off4[v * 5 + 4] = pos + deg;
          for (int e = er.x; e < er.y; ++e) {
            const int4 Ev = ed[e];
            for (int side = 0; side < 2; ++side) {
              const int me = side ? Ev.y : Ev.x, other = side ? Ev.x : Ev.y;
              if (me != v) continue;
              const int val = (other << 2) | Ev.z;
              if (Ev.z == 0) nbr[o0++] = val;
              else if (Ev.z == 1) nbr[o1++] = val;
              else if (Ev.z == 2) nbr[o2++] = val;
              else nbr[o3++] = val;
            }
          }
        }
      }
    }
    __syncthreads();
    int present = 0;
    for (int q = 0; q < nbr_off[kA]; ++q) present |= 1 << (nbr[q] & 3);
    for (int b = 0; b < 4; ++b)   // absent bond types: zero gradient partial
      if (!(present & (1 << b)))
        for (int i = tid; i < F * F; i += kThreads) G[p.off[1] + (size_t)b * F * F + i] = 0.f;
    // ===================== forward (C4), h^{t+1} = ReLU(U h + sum_b W_b s_b + c) ===
    for (int i = tid; i < kA * 16; i += kThreads) {
      const int v = i >> 4, ch = i & 15;
      float f[8];
#pragma unroll
      for (int j = 0; j < 8; ++j)
        f[j] = (v < na) ? E[(int)p.atom_type[a0 + v] * F + 8 * ch + j] : 0.f;
      put8(op0, op0 + kOp, v, ch, f);
#pragma unroll
      for (int j = 0; j < 8; ++j) hs[(8 * ch + j) * kA + v] = f[j];
    }
    for (int t = 0; t < p.T; ++t) {
      bool first = true;
      for (int b = -1; b < p.n_bonds; ++b) {
        if (b >= 0 && !(present & (1 << b))) continue;
        // operands: A = H (b = -1) or S_b, B = U or W_b, both hi/lo (3 products)
        __syncthreads();   // previous MMAs done (waited) -> S / W buffers free
        if (tid == 0) copy_img_async(op2, p.wimg + (size_t)(b + 1) * kImgBytes, 2 * kOp, cbar);   // W (hi | lo)
        if (b >= 0) gather(op1, op1 + kOp, op0, op0 + kOp, off4, nbr, na, b, false, tid);
        fence_proxy_async();
        tc_fence_before();
        __syncthreads();
        if (warp == 0) copy_wait(cbar, cph); else cph ^= 1u;
        if (warp == 0) {
          tc_fence_after();
          const uint32_t a = b < 0 ? s0 : s1;
          mma_128(acc0, a, s2, !first);                  // A_hi . W_hi
          mma_128(acc0, a + kOp, s2, true);              // A_lo . W_hi
          mma_128(acc0, a, s2 + kOp, true);              // A_hi . W_lo
          umma_commit_warp(bar_s);
        }
        mma_wait(bar, ph);
        first = false;
      }
      // epilogue: h = ReLU(acc + c) -> H (hi/lo) and hs[t+1] ([k][v], fp32)
      {
        float v64[64];
        tmem_row64(acc0 + lane_off + (uint32_t)tc0, v64);
        tc_fence_before();
        __syncthreads();   // every warp read its accumulator rows before H is overwritten
        const int v = trow;
        float* hn = hs + (size_t)(t + 1) * F * kA;
        uint32_t bits[2] = {0u, 0u};
#pragma unroll
        for (int c8 = 0; c8 < 8; ++c8) {
          float o[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const int f = tc0 + 8 * c8 + j;
            o[j] = (v < na) ? fmaxf(v64[8 * c8 + j] + cvec[f], 0.f) : 0.f;
            hn[f * kA + v] = o[j];
            bits[c8 >> 2] |= (o[j] > 0.f ? 1u : 0u) << ((8 * c8 + j) & 31);
          }
          put8(op0, op0 + kOp, v, (tc0 >> 3) + c8, o);
        }
        if (masks_smem) {
          uint32_t* mrow = rmask + ((size_t)t * kA + v) * kMaskW + (tc0 >> 5);
          mrow[0] = bits[0];
          mrow[1] = bits[1];
        }
      }
    }
    __syncthreads();
    // ===================== readout, loss, head gradients (all molecules of the tile) ==
    // Batched over the tile's molecules (the per-molecule version left half the
    // threads idle and paid a global round trip per molecule and step); every
    // sum keeps the per-molecule version's order, so the results are unchanged.
    // Scratch: the three operand buffers (64 KiB each) are free until the
    // backward stages its first operands (h^T comes from the saved fp32 rows).
    {
      const float* hT = hs + (size_t)p.T * F * kA;
      const int nm = m1 - m0;                             // <= kA (every molecule has an atom)
      float* Rs = reinterpret_cast<float*>(op0);          // [nm][F] r_m (readout sums)
      float* As = reinterpret_cast<float*>(op1);          // [nm][F] a_m (pre-activation)
      float* Ds = reinterpret_cast<float*>(op2);          // [nm][F] da_m
      float* Ys = red;                                    // [nm] dy_m (red: [4][kF] floats)
      const int f = tid & (kF - 1), half = tid >> 7;     // two molecule halves in parallel
      // r_m[k] = sum over m's atoms (atom order) of h^T[k][v]
      for (int m = half; m < nm; m += 2) {
        const int ab = p.atom_off[m0 + m] - a0, ae = p.atom_off[m0 + m + 1] - a0;
        float r = 0.f;
        for (int v = ab; v < ae; ++v) r += hT[f * kA + v];
        Rs[m * F + f] = r;
      }
      __syncthreads();
      // a_m[f] = c1[f] + sum_k W1[f][k] r_m[k] (k order), 8 molecules per pass
      for (int mb = 8 * half; mb < nm; mb += 16) {
        float acc[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] = c1[f];
        for (int k = 0; k < F; ++k) {
          const float w = W1[f * F + k];
#pragma unroll
          for (int i = 0; i < 8; ++i)
            if (mb + i < nm) acc[i] = fmaf(w, Rs[(mb + i) * F + k], acc[i]);
        }
#pragma unroll
        for (int i = 0; i < 8; ++i)
          if (mb + i < nm) As[(mb + i) * F + f] = acc[i];
      }
      __syncthreads();
      // y_m = c2 + w2 . relu(a_m) (lane-strided partials + the fixed shuffle tree), dy_m
      for (int m = warp; m < nm; m += kThreads / 32) {
        float part = 0.f;
        for (int ff = lane; ff < F; ff += 32) part = fmaf(w2[ff], fmaxf(As[m * F + ff], 0.f), part);
        part = warp_sum(part);
        if (lane == 0) {
          const float y = part + c2;
          p.y[m0 + m] = y;
          p.out[m0 + m] = y;
          Ys[m] = 2.0f * (y - p.targets[m0 + m]) / (float)p.n_mol;   // dy
        }
      }
      __syncthreads();
      // da_m[f]; head gradients summed in molecule order (as the per-molecule RMWs)
      if (tid < F) {
        float gw2 = G[p.off[9] + f], gc1 = G[p.off[8] + f], gc2 = (f == 0) ? G[p.off[10]] : 0.f;
        for (int m = 0; m < nm; ++m) {
          const float dy = Ys[m], a = As[m * F + f];
          gw2 += dy * fmaxf(a, 0.f);
          const float d = (a > 0.f) ? dy * w2[f] : 0.f;
          Ds[m * F + f] = d;
          gc1 += d;
          if (f == 0) gc2 += dy;
        }
        G[p.off[9] + f] = gw2;
        G[p.off[8] + f] = gc1;
        if (f == 0) G[p.off[10]] = gc2;
      }
      __syncthreads();
      // dW1 += sum_m da_m r_m^T (molecule order, one pass over the partial)
      for (int i = tid; i < F * F; i += kThreads) {
        const int fi = i / F, k = i - fi * F;
        float g = 0.f;
        for (int m = 0; m < nm; ++m) g = fmaf(Ds[m * F + fi], Rs[m * F + k], g);
        G[p.off[7] + i] = g;   // zeroed at the tile start: 0 + g
      }
      // dr_m[k] = sum_f W1[f][k] da_m[f] (f order): dh^T of every atom of m
      for (int mb = 8 * half; mb < nm; mb += 16) {
        float acc[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] = 0.f;
        for (int ff = 0; ff < F; ++ff) {
          const float w = W1[ff * F + f];
#pragma unroll
          for (int i = 0; i < 8; ++i)
            if (mb + i < nm) acc[i] = fmaf(w, Ds[(mb + i) * F + ff], acc[i]);
        }
#pragma unroll
        for (int i = 0; i < 8; ++i)
          if (mb + i < nm) drm[(mb + i) * F + f] = acc[i];
      }
      fence_proxy_async();   // generic scratch writes before the backward's async-proxy copies / MMAs
      __syncthreads();
    }
    // ===================== backward through the T message-passing steps ==========
    // per step (reverse): dq = dh * [h^{t+1} > 0]; dc += sum_v dq; dU += dq^T h;
    // dW_b += dq^T s_b; dh^t = dq U + sum_b gather_b(dq) W_b
    uint8_t* dqT = op0;            // [f][v]  (B of the weight gradients)
    uint8_t* dq = op0 + kOp;       // [v][f]  (A of dh)
    uint8_t* hTo = op1;            // [k][v]  (A of dU)
    uint8_t* X = op1 + kOp;        // sT_b [k][v] (A of dW_b) / gq_b [v][f] (A of dh)
    uint8_t* Wt = op2;             // [k][f]  (B of dh)
    uint8_t* hv = op2 + kOp;       // [v][k]  (gather source for s_b)
    const uint32_t sdqT = s0, sdq = s0 + kOp, shT = s1, sX = s1 + kOp, sWt = s2;
    for (int t = p.T - 1; t >= 0; --t) {
      // U^T into Wt while (a) and (b) run (Wt's last readers, the previous
      // step's MMAs, were waited; (b) writes only the other half, hv)
      if (tid == 0) copy_img_async(Wt, p.wimg + 2 * kOp, kOp, cbar);
      // (a) dq from dh (acc1, or the readout's dr at the last step) and the mask
      {
        float dh64[64];
        const int v = trow;
        if (t == p.T - 1) {
          int ml = 0;   // v's molecule (tile-local)
          while (ml + 1 < m1 - m0 && p.atom_off[m0 + ml + 1] - a0 <= v) ++ml;
#pragma unroll
          for (int j = 0; j < 64; ++j) dh64[j] = (v < na) ? drm[ml * F + tc0 + j] : 0.f;
        } else {
          tmem_row64(acc1 + lane_off + (uint32_t)tc0, dh64);
        }
        tc_fence_before();
        __syncthreads();   // acc1 read everywhere; operands of step t+1 free
        const float* hn = hs + (size_t)(t + 1) * F * kA;
        uint32_t mb[2] = {0u, 0u};   // ReLU mask bits of h^{t+1}, this thread's row and 64 columns
        if (masks_smem) {
          const uint32_t* mrow = rmask + ((size_t)t * kA + v) * kMaskW + (tc0 >> 5);
          mb[0] = mrow[0];
          mb[1] = mrow[1];
        }
#pragma unroll
        for (int c8 = 0; c8 < 8; ++c8) {
          float o[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const int f = tc0 + 8 * c8 + j;
            const bool pos = masks_smem ? ((mb[c8 >> 2] >> ((8 * c8 + j) & 31)) & 1u) != 0u
                                        : (v < na && hn[f * kA + v] > 0.f);
            o[j] = pos ? dh64[8 * c8 + j] : 0.f;
            // dqT[f][v]: lanes v, v + 1 (v even) share one 32-bit word
            const uint32_t bq = f32_to_bf16_rne(o[j]);
            const uint32_t bn = __shfl_down_sync(0xffffffffu, bq, 1);
            if ((lane & 1) == 0) *reinterpret_cast<uint32_t*>(dqT + elem_off(f, v)) = bq | (bn << 16);
            // dc: column sums over this warp's 32 rows (fixed shuffle tree)
            const float cs = warp_sum(o[j]);
            if (lane == 0) red[(warp & 3) * F + f] = cs;
          }
          put8(dq, nullptr, v, (tc0 >> 3) + c8, o);
        }
      }
      // (b) h^t as hT [k][v] and h [v][k] (bf16) from the saved fp32 rows
      {
        const float* ht = hs + (size_t)t * F * kA;
        for (int i = tid; i < kF * 16; i += kThreads) {
          const int k = i >> 4, ch = i & 15;
          float f[8];
          const float4 a4 = *reinterpret_cast<const float4*>(ht + k * kA + 8 * ch);
          const float4 b4 = *reinterpret_cast<const float4*>(ht + k * kA + 8 * ch + 4);
          f[0] = a4.x; f[1] = a4.y; f[2] = a4.z; f[3] = a4.w; f[4] = b4.x; f[5] = b4.y; f[6] = b4.z; f[7] = b4.w;
          put8(hTo, nullptr, k, ch, f);
#pragma unroll
          for (int j = 0; j < 8; ++j)
            *reinterpret_cast<uint16_t*>(hv + elem_off(8 * ch + j, k)) = f32_to_bf16_rne(f[j]);
        }
      }
      fence_proxy_async();
      tc_fence_before();
      __syncthreads();
      if (tid < F) G[p.off[6] + tid] += (red[tid] + red[F + tid]) + (red[2 * F + tid] + red[3 * F + tid]);   // dc
      if (warp == 0) copy_wait(cbar, cph); else cph ^= 1u;   // U^T (issued at the step start)
      if (warp == 0) {
        tc_fence_after();
        mma_128(acc0, shT, sdqT, false);     // dU^T[k][f] = sum_v h[v][k] dq[v][f]
        mma_128(acc1, sdq, sWt, false);      // dh[v][k]   = sum_f dq[v][f] U[f][k]
        umma_commit_warp(bar_s);
      }
      mma_wait(bar, ph);
      // flush a weight gradient (acc0 = [k][f]) into this tile's partial G[f][k]
      // (the partial of U / W_b is written by the first backward step, t = T-1)
      auto flush = [&](float* Gm, bool set) {
        float g64[64];
        tmem_row64(acc0 + lane_off + (uint32_t)tc0, g64);
        const int k = trow;
        if (set) {
#pragma unroll
          for (int j = 0; j < 64; ++j) Gm[(tc0 + j) * F + k] = g64[j];
        } else {
#pragma unroll
          // fire-and-forget reductions (red.global.add.f32): this thread is the only
          // writer of these elements, so they apply in program order, the same
          // sequence of fp32 adds as a load-add-store, without the round trip
          for (int j = 0; j < 64; ++j) atomicAdd(&Gm[(tc0 + j) * F + k], g64[j]);
        }
      };
      flush(G + p.off[5], t == p.T - 1);                            // dU
      for (int b = 0; b < p.n_bonds; ++b) {
        if (!(present & (1 << b))) continue;
        tc_fence_before();
        __syncthreads();   // acc0 flushed, X free
        gather(X, nullptr, hv, nullptr, off4, nbr, na, b, true, tid);   // sT_b [k][v]
        fence_proxy_async();
        tc_fence_before();
        __syncthreads();
        if (warp == 0) {
          tc_fence_after();
          mma_128(acc0, sX, sdqT, false);    // dW_b^T[k][f] = sum_v s_b[v][k] dq[v][f]
          umma_commit_warp(bar_s);
        }
        mma_wait(bar, ph);
        flush(G + p.off[1] + (size_t)b * F * F, t == p.T - 1);      // dW_b
        tc_fence_before();
        __syncthreads();   // X and Wt free
        if (tid == 0) copy_img_async(Wt, p.wimg + (size_t)(b + 1) * kImgBytes + 2 * kOp, kOp, cbar);   // W_b^T
        gather(X, nullptr, dq, nullptr, off4, nbr, na, b, false, tid);  // gq_b [v][f]
        fence_proxy_async();
        tc_fence_before();
        __syncthreads();
        if (warp == 0) copy_wait(cbar, cph); else cph ^= 1u;
        if (warp == 0) {
          tc_fence_after();
          mma_128(acc1, sX, sWt, true);      // dh[v][k] += sum_f gq_b[v][f] W_b[f][k]
          umma_commit_warp(bar_s);
        }
        mma_wait(bar, ph);
      }
      tc_fence_before();
      __syncthreads();
    }
    // dE[type_v] += dh^0_v (atom order): dh^0 through shared memory ([v][k], row
    // stride F + 1: conflict-free both ways), per-type sums in shared memory
    // (zero-initialised like the partial, so the sums are the same bits)
    {
      float* Hs = reinterpret_cast<float*>(op0);   // [kA][F + 1] (op0 + op1)
      float* Es = reinterpret_cast<float*>(op2);   // [n_types][F]
      const int n_types = (int)(p.off[1] - p.off[0]) / F;   // E is [n_types][F], W_0 follows
      float dh64[64];
      tmem_row64(acc1 + lane_off + (uint32_t)tc0, dh64);
      const int v = trow;
#pragma unroll
      for (int j = 0; j < 64; ++j) Hs[v * (F + 1) + tc0 + j] = (v < na) ? dh64[j] : 0.f;
      if (n_types * F * 4 <= 2 * kOp) {
        for (int i = tid; i < n_types * F; i += kThreads) Es[i] = 0.f;
        __syncthreads();
        if (tid < F)
          for (int vv = 0; vv < na; ++vv) Es[(int)p.atom_type[a0 + vv] * F + tid] += Hs[vv * (F + 1) + tid];
        __syncthreads();
        for (int i = tid; i < n_types * F; i += kThreads) G[p.off[0] + i] = Es[i];   // zeroed: 0 + sum
      } else {
        // more than 128 atom types: the per-type sums do not fit op2; accumulate
        // in the (zeroed) partial directly, same order
        __syncthreads();
        if (tid < F)
          for (int vv = 0; vv < na; ++vv)
            G[p.off[0] + (int)p.atom_type[a0 + vv] * F + tid] += Hs[vv * (F + 1) + tid];
      }
    }
    fence_proxy_async();   // generic scratch writes before the next tile's async-proxy copies
    tc_fence_before();
    __syncthreads();
  }
  if (warp == 0) {
    tc_fence_after();
    tmem_dealloc(tmem, kTmemCols);
  }
}

__global__ void __launch_bounds__(kThreads) mpnn_train_apply_kernel(MpnnTrainParams p) {
  const int tid = threadIdx.x;
  // SGD: theta_j -= lr * sum_tiles partial[tile][j] (tile order)
  for (int j = blockIdx.x * kThreads + tid; j < p.n_params; j += gridDim.x * kThreads) {
    float g = 0.f;
    for (int t = 0; t < p.n_tiles; ++t) g += p.partials[(uint64_t)t * p.n_params + j];
    p.params[j] -= p.lr * g;
  }
  __syncthreads();
  if (tid == 0) {
    if (blockIdx.x == 0) {
      // loss = mean squared error in molecule order
      float s = 0.f;
      for (int m = 0; m < p.n_mol; ++m) {
        const float e = p.y[m] - p.targets[m];
        s = fmaf(e, e, s);
      }
      p.out[p.n_mol] = s / (float)p.n_mol;
    }
    __threadfence_system();
    atomicMax(&p.stamps[1], (unsigned long long)globaltimer());
    if (atomicAdd(&p.stamps[4], 1ull) == (unsigned long long)(gridDim.x - 1)) {
      __threadfence();
      volatile unsigned long long* st = p.stamps;
      volatile unsigned long long* h = p.h_stamps;
      h[0] = st[0];
      h[1] = globaltimer();
      h[2] = (unsigned long long)(unsigned)p.inject_err;   // 0 unless the fault-path test hook is set
      p.stamps[4] = 0;
      __threadfence_system();
      h[3] = p.done_tag;
    }
  }
}

// fp32 training parameters from the bf16 seeded block (exact widening).
__global__ void widen_bf16_kernel(float* dst, const uint16_t* src, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    dst[i] = bf16_bits_to_f32(src[i]);
}

int launch_mpnn_train(const MpnnTrainParams& p, void* stream) {
  MpnnTrainParams pc = p;
  void* args[] = {&pc};
  int rc = launch_kernel(mpnn_train_prep_kernel, dim3(1 + p.n_bonds), dim3(kThreads), 0u, stream, args);
  if (rc) return rc;
  rc = launch_kernel(mpnn_train_tile_kernel, dim3(p.n_ctas), dim3(kThreads),
                     (unsigned)kTrainSmem, stream, args);
  if (rc) return rc;
  return launch_kernel(mpnn_train_apply_kernel, dim3(p.n_ctas), dim3(kThreads), 0u, stream, args);
}

int launch_widen_bf16(float* dst, const uint16_t* src, uint64_t n, int n_ctas, void* stream) {
  void* args[] = {&dst, &src, &n};
  return launch_kernel(widen_bf16_kernel, dim3(n_ctas), dim3(256), 0u, stream, args);
}

int mpnn_train_set_attrs(int device) {
  return set_max_smem(mpnn_train_tile_kernel, kTrainSmem, device);
}

}  // namespace mxk
