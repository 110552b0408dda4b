// IP-emulator TRAINING step: PAPER.md §3.1 P:109 steps (3)
// and (7) "train an ML model that acts as an emulator of the simulations",
// §3.4 P:163 (training is one of the workflow's two GPU phases). Loss, optimiser
// and state are reading R10: L = (1/M) sum_m (y_m - t_m)^2 over the
// task's molecules, one SGD step theta -= lr * dL/dtheta on fp32 parameters.
//
// Two launches per task on the partition's stream:
//  1. mpnn_train_tile_kernel — one CTA per 128-atom tile (the inference
//     kernel's packing): forward C4 keeping h^0..h^T (tile scratch in HBM),
//     readout + loss terms, then the reverse-mode chain rule step by step
//     (same order as oracle/mpnn_train.py), accumulating this tile's gradient
//     of every parameter into its own partial buffer (no atomics).
//  2. mpnn_train_apply_kernel — every parameter element sums the tile
//     partials in tile order (deterministic, independent of the partition
//     size), applies the SGD update in place, and the loss is reduced in
//     molecule order; the last CTA publishes the completion record.
// Round-1 arithmetic is fp32 on CUDA cores (8x8 register blocks over
// [128 x 128] shared-memory tiles); the tensor-core (tcgen05) version of the
// backward contractions is the next step.
#include "common.cuh"
#include "kernels.h"
#include "launch.cuh"

namespace mxk {

namespace {
constexpr int kF = 128;
constexpr int kA = 128;            // atoms per tile
constexpr int kTE = 512;           // bonds per tile
constexpr int kThreads = 256;
constexpr int kS = 132;            // row stride (floats) of the [feature][atom] buffers
constexpr int kBuf = kF * kS;      // floats per buffer
constexpr int kWc = 16;            // weight rows per staged chunk

// smem map (floats / ints)
constexpr int kOffH = 0;
constexpr int kOffS = kOffH + kBuf;
constexpr int kOffD = kOffS + kBuf;
constexpr int kOffW = kOffD + kBuf;                 // [kWc][kS] weight chunk
constexpr int kOffNbrOff = kOffW + kWc * kS;        // int [kA + 4]
constexpr int kOffNbr = kOffNbrOff + kA + 4;        // int [2 * kTE]: (u << 2) | b
constexpr int kOffR = kOffNbr + 2 * kTE;            // float [kF] readout r
constexpr int kOffZ = kOffR + kF;                   // float [kF] a (pre-activation)
constexpr int kOffDA = kOffZ + kF;                  // float [kF] da
constexpr int kOffDR = kOffDA + kF;                 // float [kF] dr
constexpr int kOffRed = kOffDR + kF;                // float [16]
constexpr int kOffOff4 = kOffRed + 16;              // int [kA][5]: per-bond-type neighbour ranges
constexpr int kTrainSmem = (kOffOff4 + kA * 5) * 4;
// setup-only aliases inside the S buffer (before the first neighbour gather)
constexpr int kOffEdges = kOffS;                    // int4 [kTE]
constexpr int kOffMolE = kOffS + 4 * kTE;           // int2 [kA]

__device__ __forceinline__ float* fbuf(float* sm, int off) { return sm + off; }

// acc[i][j] (rows r = ta + 16 i of the OUTPUT's first index, cols c = tb + 16 j)
struct Acc {
  float v[8][8];
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j) v[i][j] = 0.f;
  }
};

// G1: acc[v][f] += sum_k X[k][v] * W[f][k]   (X: smem [k][v]; W: global row-major [f][k])
__device__ void gemm_xw_t(Acc& acc, const float* X, const float* __restrict__ W, float* Wt, int ta,
                          int tb, int tid) {
  for (int k0 = 0; k0 < kF; k0 += kWc) {
    __syncthreads();
    // Wt[kk][f] = W[f][k0 + kk]
    for (int i = tid; i < kF * kWc; i += kThreads) {
      const int f = i / kWc, kk = i - f * kWc;
      Wt[kk * kS + f] = W[f * kF + k0 + kk];
    }
    __syncthreads();
#pragma unroll 4
    for (int kk = 0; kk < kWc; ++kk) {
      float x[8], w[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) x[i] = X[(k0 + kk) * kS + ta + 16 * i];
#pragma unroll
      for (int j = 0; j < 8; ++j) w[j] = Wt[kk * kS + tb + 16 * j];
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc.v[i][j] = fmaf(x[i], w[j], acc.v[i][j]);
    }
  }
}

// G2: acc[v][k] += sum_f X[f][v] * W[f][k]   (X: smem [f][v]; W: global row-major [f][k])
__device__ void gemm_xw(Acc& acc, const float* X, const float* __restrict__ W, float* Wc, int ta,
                        int tb, int tid) {
  for (int f0 = 0; f0 < kF; f0 += kWc) {
    __syncthreads();
    for (int i = tid; i < kWc * kF; i += kThreads) {
      const int ff = i / kF, k = i - ff * kF;
      Wc[ff * kS + k] = W[(f0 + ff) * kF + k];
    }
    __syncthreads();
#pragma unroll 4
    for (int ff = 0; ff < kWc; ++ff) {
      float x[8], w[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) x[i] = X[(f0 + ff) * kS + ta + 16 * i];
#pragma unroll
      for (int j = 0; j < 8; ++j) w[j] = Wc[ff * kS + tb + 16 * j];
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc.v[i][j] = fmaf(x[i], w[j], acc.v[i][j]);
    }
  }
}

// G3: G[f][k] += sum_v Z[f][v] * Y[k][v]  (both smem [.][v]); thread owns f = ta + 16 i,
// k = tb + 16 j; accumulated into the tile's global gradient partial (owned, no atomics).
__device__ void gemm_grad(float* __restrict__ G, const float* Z, const float* Y, int ta, int tb) {
  Acc acc;
  acc.zero();
#pragma unroll 2
  for (int v = 0; v < kA; v += 4) {
    float4 z[8], y[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) z[i] = *reinterpret_cast<const float4*>(Z + (ta + 16 * i) * kS + v);
#pragma unroll
    for (int j = 0; j < 8; ++j) y[j] = *reinterpret_cast<const float4*>(Y + (tb + 16 * j) * kS + v);
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        float a = acc.v[i][j];
        a = fmaf(z[i].x, y[j].x, a);
        a = fmaf(z[i].y, y[j].y, a);
        a = fmaf(z[i].z, y[j].z, a);
        a = fmaf(z[i].w, y[j].w, a);
        acc.v[i][j] = a;
      }
  }
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) G[(ta + 16 * i) * kF + tb + 16 * j] += acc.v[i][j];
}

// S[k][v] = sum over the type-b neighbours u of v of X[k][u] (edge order). A
// thread owns one atom v and half the features: its neighbour list is read
// once (bucketed by bond type, off4[v][b] .. off4[v][b+1]) and reused for
// every feature.
constexpr int kGatherRegs = 8;
__device__ void gather(float* S, const float* X, const int* off4, const int* nbr, int na, int b,
                       int tid) {
  const int v = tid % kA, k0 = tid / kA;
  int u[kGatherRegs];
  int q0 = 0, q1 = 0;
  if (v < na) {
    q0 = off4[v * 5 + b];
    q1 = off4[v * 5 + b + 1];
  }
  const int c = q1 - q0;
#pragma unroll
  for (int q = 0; q < kGatherRegs; ++q) u[q] = (q < c) ? (nbr[q0 + q] >> 2) : 0;
  for (int k = k0; k < kF; k += kThreads / kA) {
    float t = 0.f;
#pragma unroll
    for (int q = 0; q < kGatherRegs; ++q)
      if (q < c) t += X[k * kS + u[q]];
    for (int q = q0 + kGatherRegs; q < q1; ++q) t += X[k * kS + (nbr[q] >> 2)];   // rare: deg > 8
    S[k * kS + v] = t;
  }
}

__device__ void save_buf(float* __restrict__ dst, const float* X, int tid) {
  for (int i = tid; i < kF * kA / 4; i += kThreads) {
    const int k = i / (kA / 4), v4 = (i - k * (kA / 4)) * 4;
    *reinterpret_cast<float4*>(dst + k * kA + v4) = *reinterpret_cast<const float4*>(X + k * kS + v4);
  }
}
__device__ void load_buf(float* X, const float* __restrict__ src, int tid) {
  for (int i = tid; i < kF * kA / 4; i += kThreads) {
    const int k = i / (kA / 4), v4 = (i - k * (kA / 4)) * 4;
    *reinterpret_cast<float4*>(X + k * kS + v4) = *reinterpret_cast<const float4*>(src + k * kA + v4);
  }
}
}  // namespace

int mpnn_train_smem_bytes() { return kTrainSmem; }
uint64_t mpnn_train_tile_scratch_floats(int T) { return (uint64_t)(T + 1) * kF * kA; }

__global__ void __launch_bounds__(kThreads, 1) mpnn_train_tile_kernel(MpnnTrainParams p) {
  extern __shared__ __align__(16) float sm[];
  float* H = sm + kOffH;
  float* S = sm + kOffS;
  float* D = sm + kOffD;
  float* Wst = sm + kOffW;
  int* nbr_off = reinterpret_cast<int*>(sm + kOffNbrOff);
  int* nbr = reinterpret_cast<int*>(sm + kOffNbr);
  int* off4 = reinterpret_cast<int*>(sm + kOffOff4);
  float* rr = sm + kOffR;
  float* aa = sm + kOffZ;
  float* da = sm + kOffDA;
  float* dr = sm + kOffDR;
  float* red = sm + kOffRed;
  int4* ed = reinterpret_cast<int4*>(sm + kOffEdges);
  int2* mol_e = reinterpret_cast<int2*>(sm + kOffMolE);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int ta = tid >> 4, tb = tid & 15;
  const int F = kF;
  if (blockIdx.x == 0 && tid == 0) p.stamps[0] = globaltimer();
  const uint8_t* eb = reinterpret_cast<const uint8_t*>(p.edges);
  const float* E = p.params + p.off[0];
  const float* Wb = p.params + p.off[1];
  const float* U = p.params + p.off[5];
  const float* cvec = p.params + p.off[6];
  const float* W1 = p.params + p.off[7];
  const float* c1 = p.params + p.off[8];
  const float* w2 = p.params + p.off[9];
  const float c2 = p.params[p.off[10]];

  for (int tile = blockIdx.x; tile < p.n_tiles; tile += p.n_ctas) {
    float* G = p.partials + (uint64_t)tile * p.n_params;
    float* hs = p.hsave + (uint64_t)tile * (p.T + 1) * kF * kA;
    const int m0 = p.tile_off[tile], m1 = p.tile_off[tile + 1];
    const int a0 = p.atom_off[m0], na = p.atom_off[m1] - a0;
    const int e0 = p.edge_off[m0], ne = p.edge_off[m1] - e0;
    // zero this tile's gradient partial
    for (int i = tid; i < p.n_params; i += kThreads) G[i] = 0.f;
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
    // --- forward: h^0 = E[type], h^{t+1} = ReLU(U h + sum_b W_b s_b + c) ------
    for (int i = tid; i < F * kA; i += kThreads) {
      const int k = i / kA, v = i - k * kA;
      H[k * kS + v] = (v < na) ? E[(int)p.atom_type[a0 + v] * F + k] : 0.f;
    }
    __syncthreads();
    save_buf(hs, H, tid);
    for (int t = 0; t < p.T; ++t) {
      Acc acc;
      acc.zero();
      gemm_xw_t(acc, H, U, Wst, ta, tb, tid);
      for (int b = 0; b < p.n_bonds; ++b) {
        if (!(present & (1 << b))) continue;
        __syncthreads();
        gather(S, H, off4, nbr, na, b, tid);
        gemm_xw_t(acc, S, Wb + (size_t)b * F * F, Wst, ta, tb, tid);   // syncs before reading S
      }
      __syncthreads();
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int v = ta + 16 * i, f = tb + 16 * j;
          H[f * kS + v] = (v < na) ? fmaxf(acc.v[i][j] + cvec[f], 0.f) : 0.f;
        }
      __syncthreads();
      save_buf(hs + (size_t)(t + 1) * F * kA, H, tid);
    }
    // --- readout, loss term, head gradients, dh^T (per molecule, atom order) --
    for (int i = tid; i < F * kA; i += kThreads) D[(i / kA) * kS + (i % kA)] = 0.f;
    for (int m = m0; m < m1; ++m) {
      const int ab = p.atom_off[m] - a0, ae = p.atom_off[m + 1] - a0;
      __syncthreads();
      if (tid < F) {
        float r = 0.f;
        for (int v = ab; v < ae; ++v) r += H[tid * kS + v];
        rr[tid] = r;
      }
      __syncthreads();
      if (tid < F) {
        float a = c1[tid];
        for (int k = 0; k < F; ++k) a = fmaf(W1[tid * F + k], rr[k], a);
        aa[tid] = a;
      }
      __syncthreads();
      // y = w2 . ReLU(a) + c2 (warp 0, fixed shuffle tree)
      if (warp == 0) {
        float part = 0.f;
        for (int f = lane; f < F; f += 32) part = fmaf(w2[f], fmaxf(aa[f], 0.f), part);
        part = warp_sum(part);
        if (lane == 0) {
          const float y = part + c2;
          p.y[m] = y;
          p.out[m] = y;
          red[8] = 2.0f * (y - p.targets[m]) / (float)p.n_mol;   // dy
        }
      }
      __syncthreads();
      const float dy = red[8];
      if (tid < F) {
        const float z = fmaxf(aa[tid], 0.f);
        G[p.off[9] + tid] += dy * z;                               // dw2
        const float d = (aa[tid] > 0.f) ? dy * w2[tid] : 0.f;      // da
        da[tid] = d;
        G[p.off[8] + tid] += d;                                    // dc1
      }
      if (tid == 0) G[p.off[10]] += dy;                            // dc2
      __syncthreads();
      // dW1 += da r^T ; dr = W1^T da
      for (int i = tid; i < F * F; i += kThreads) {
        const int f = i / F, k = i - f * F;
        G[p.off[7] + i] += da[f] * rr[k];
      }
      if (tid < F) {
        float s = 0.f;
        for (int f = 0; f < F; ++f) s = fmaf(W1[f * F + tid], da[f], s);
        dr[tid] = s;
      }
      __syncthreads();
      for (int i = tid; i < F * (ae - ab); i += kThreads) {
        const int k = i / (ae - ab), v = ab + (i - k * (ae - ab));
        D[k * kS + v] = dr[k];
      }
    }
    __syncthreads();
    // --- backward through the T message-passing steps --------------------------
    for (int t = p.T - 1; t >= 0; --t) {
      const float* hn = hs + (size_t)(t + 1) * F * kA;
      // dq = dh^{t+1} * [h^{t+1} > 0]   (in place in D)
      for (int i = tid; i < F * kA; i += kThreads) {
        const int k = i / kA, v = i - k * kA;
        if (!(hn[k * kA + v] > 0.f)) D[k * kS + v] = 0.f;
      }
      load_buf(H, hs + (size_t)t * F * kA, tid);
      __syncthreads();
      if (tid < F) {
        float s = 0.f;
        for (int v = 0; v < na; ++v) s += D[tid * kS + v];
        G[p.off[6] + tid] += s;                                    // dc
      }
      gemm_grad(G + p.off[5], D, H, ta, tb);                       // dU += dq^T h
      Acc acc;
      acc.zero();
      gemm_xw(acc, D, U, Wst, ta, tb, tid);                        // dh = dq U
      for (int b = 0; b < p.n_bonds; ++b) {
        if (!(present & (1 << b))) continue;
        __syncthreads();
        gather(S, H, off4, nbr, na, b, tid);                    // s_b(h^t)
        __syncthreads();
        gemm_grad(G + p.off[1] + (size_t)b * F * F, D, S, ta, tb); // dW_b += dq^T s_b
        __syncthreads();
        gather(S, D, off4, nbr, na, b, tid);                    // sum of neighbours' dq
        gemm_xw(acc, S, Wb + (size_t)b * F * F, Wst, ta, tb, tid); // dh += (.) W_b
      }
      __syncthreads();
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int v = ta + 16 * i, k = tb + 16 * j;
          D[k * kS + v] = (v < na) ? acc.v[i][j] : 0.f;
        }
      __syncthreads();
    }
    // dE[type_v] += dh^0_v (atom order)
    if (tid < F)
      for (int v = 0; v < na; ++v) G[p.off[0] + (int)p.atom_type[a0 + v] * F + tid] += D[tid * kS + v];
    __syncthreads();
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
  int rc = launch_kernel(mpnn_train_tile_kernel, dim3(p.n_ctas), dim3(kThreads),
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
