// IP-emulator inference (the paper's scientific function, §3.1
// step (4): "use the trained emulator to estimate the IPs of a larger pool of
// newly generated molecules"; architecture = reading A22 / SURVEY.md §8(c) C4):
//   h_v = E_atom[a_v]
//   T times: m_v = sum_{bonds (u,v,b) or (v,u,b)} W_b h_u ; h_v = ReLU(U h_v + m_v + c)
//   y = w2 . ReLU(W1 sum_v h_v + c1) + c2
// Computed per molecule as h' = ReLU(c + U h + sum_b W_b s_b) with the
// per-bond-type neighbour sums s_b[v] = sum_{u ~_b v} h_u (linearity: the same
// function, one transform per (atom, bond type) present instead of per bond).
//
// Round-1 B200 design: persistent grid = partition SMs; every CTA stages all
// transforms (U, W_0..W_3: 160 KB bf16, transposed so lanes read consecutive
// features) in shared memory once, then walks molecules m = cta, cta + C, ...
// Each molecule (<= 32 atoms) is a [n x 128] x [128 x 128] contraction per
// transform on CUDA cores with 4x4 register blocking (fp32 accumulate).
#include "common.cuh"
#include "kernels.h"
#include "launch.cuh"

namespace mxk {

constexpr int kF = 128;
constexpr int kMaxAtoms = 32;
constexpr int kMaxMolEdges = 64;
constexpr int kMpnnThreads = 256;

int mpnn_smem_bytes() {
  return 5 * kF * kF * 2            // Wt: U, W_0..W_3 transposed [k][f] bf16
         + 3 * kMaxAtoms * kF * 4   // h, s, acc
         + kMaxMolEdges * 4 * 4     // edges (u, v, b)
         + kF * 4 * 2               // r, z
         + 64;
}

__global__ void __launch_bounds__(kMpnnThreads, 1) mpnn_kernel(MpnnParams p) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  uint16_t* wt = reinterpret_cast<uint16_t*>(smem_raw);       // [5][k][f]
  float* h = reinterpret_cast<float*>(smem_raw + 5 * kF * kF * 2);
  float* s = h + kMaxAtoms * kF;
  float* acc = s + kMaxAtoms * kF;
  int* ed = reinterpret_cast<int*>(acc + kMaxAtoms * kF);       // [kMaxMolEdges][4]
  float* rv = reinterpret_cast<float*>(ed + kMaxMolEdges * 4);  // [F]
  float* zv = rv + kF;
  float* red = zv + kF;                                          // [8]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (blockIdx.x == 0 && tid == 0) p.stamps[0] = globaltimer();

  // stage transposed transforms: slot 0 = U, slots 1..4 = W_b
  for (int i = tid; i < 5 * kF * kF; i += kMpnnThreads) {
    const int slot = i / (kF * kF), rem = i - slot * kF * kF;
    const int f = rem / kF, k = rem - f * kF;   // source row-major [f][k]
    const uint16_t* src = (slot == 0) ? p.u : (p.w_b + (size_t)(slot - 1) * kF * kF);
    wt[slot * kF * kF + k * kF + f] = src[rem];
  }
  __syncthreads();

  const int fg = tid & 31;        // features 4fg .. 4fg+3
  const int ag = tid >> 5;        // atoms 4ag .. 4ag+3
  for (int m = blockIdx.x; m < p.n_mol; m += p.n_ctas) {
    const int a0 = p.atom_off[m], n = p.atom_off[m + 1] - a0;
    const int e0 = p.edge_off[m], ne = p.edge_off[m + 1] - e0;
    const uint8_t* eb = reinterpret_cast<const uint8_t*>(p.edges);
    for (int i = tid; i < ne; i += kMpnnThreads) {
      const uint8_t* e = eb + (size_t)(e0 + i) * 6;
      ed[i * 4 + 0] = (int)(int16_t)(e[0] | (e[1] << 8));
      ed[i * 4 + 1] = (int)(int16_t)(e[2] | (e[3] << 8));
      ed[i * 4 + 2] = (int)e[4];
    }
    for (int i = tid; i < kMaxAtoms * kF; i += kMpnnThreads) {
      const int v = i / kF, f = i - v * kF;
      h[i] = (v < n) ? bf16_bits_to_f32(p.e_atom[(size_t)p.atom_type[a0 + v] * kF + f]) : 0.f;
    }
    __syncthreads();
    for (int step = 0; step < p.T; ++step) {
      float c4[4][4];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) c4[i][j] = bf16_bits_to_f32(p.c[4 * fg + j]);
      for (int slot = 0; slot < 5; ++slot) {
        const float* in = h;
        if (slot > 0) {
          const int b = slot - 1;
          bool any = false;
          for (int i = 0; i < ne; ++i) any |= (ed[i * 4 + 2] == b);
          if (!any) continue;
          // s_b[v] = sum over bonds of type b touching v of the other atom's h (edge order)
          for (int i = tid; i < kMaxAtoms * kF; i += kMpnnThreads) {
            const int v = i / kF, f = i - v * kF;
            float t = 0.f;
            for (int q = 0; q < ne; ++q) {
              if (ed[q * 4 + 2] != b) continue;
              const int u = ed[q * 4 + 0], w = ed[q * 4 + 1];
              if (w == v) t += h[u * kF + f];
              if (u == v) t += h[w * kF + f];
            }
            s[i] = t;
          }
          __syncthreads();
          in = s;
        }
        if (4 * ag < n) {
          const uint16_t* W = wt + slot * kF * kF;
#pragma unroll 4
          for (int k = 0; k < kF; ++k) {
            const uint2 wv = *reinterpret_cast<const uint2*>(W + k * kF + 4 * fg);
            float wf[4];
            wf[0] = __uint_as_float(wv.x << 16);
            wf[1] = __uint_as_float(wv.x & 0xffff0000u);
            wf[2] = __uint_as_float(wv.y << 16);
            wf[3] = __uint_as_float(wv.y & 0xffff0000u);
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const float xv = in[(4 * ag + i) * kF + k];
#pragma unroll
              for (int j = 0; j < 4; ++j) c4[i][j] = fmaf(wf[j], xv, c4[i][j]);
            }
          }
        }
        __syncthreads();   // s is rewritten by the next bond type
      }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[(4 * ag + i) * kF + 4 * fg + j] = fmaxf(c4[i][j], 0.f);
      __syncthreads();
      for (int i = tid; i < kMaxAtoms * kF; i += kMpnnThreads) h[i] = (i / kF < n) ? acc[i] : 0.f;
      __syncthreads();
    }
    // readout: r = sum_v h_v (atom order); z = ReLU(W1 r + c1); y = w2 . z + c2
    if (tid < kF) {
      float t = 0.f;
      for (int v = 0; v < n; ++v) t += h[v * kF + tid];
      rv[tid] = t;
    }
    __syncthreads();
    if (tid < kF) {
      float t = bf16_bits_to_f32(p.c1[tid]);
      const uint16_t* w1r = p.w1 + (size_t)tid * kF;
      for (int k = 0; k < kF; ++k) t = fmaf(bf16_bits_to_f32(w1r[k]), rv[k], t);
      zv[tid] = fmaxf(t, 0.f);
    }
    __syncthreads();
    float part = (tid < kF) ? bf16_bits_to_f32(p.w2[tid]) * zv[tid] : 0.f;
    part = warp_sum(part);
    if (lane == 0) red[warp] = part;
    __syncthreads();
    if (tid == 0) {
      float y = 0.f;
      for (int w = 0; w < kMpnnThreads / 32; ++w) y += red[w];
      p.out[m] = y + bf16_bits_to_f32(p.c2[0]);
    }
    __syncthreads();
  }
  if (tid == 0) atomicMax(&p.stamps[1], (unsigned long long)globaltimer());
}

int launch_mpnn(const MpnnParams& p, void* stream) {
  MpnnParams pc = p;
  void* args[] = {&pc};
  return launch_kernel(mpnn_kernel, dim3(p.n_ctas), dim3(kMpnnThreads), (unsigned)mpnn_smem_bytes(),
                       stream, args);
}

int mpnn_set_attrs(int device) { return set_max_smem(mpnn_kernel, mpnn_smem_bytes(), device); }

}  // namespace mxk
