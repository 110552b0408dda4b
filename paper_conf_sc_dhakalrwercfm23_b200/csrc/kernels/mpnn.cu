// IP-emulator inference (the paper's scientific function, §3.1
// step (4): "use the trained emulator to estimate the IPs of a larger pool of
// newly generated molecules"; architecture = reading A22 / SURVEY.md §8(c) C4):
//   h_v = E_atom[a_v]
//   T times: m_v = sum_{bonds (u,v,b) or (v,u,b)} W_b h_u ; h_v = ReLU(U h_v + m_v + c)
//   y = w2 . ReLU(W1 sum_v h_v + c1) + c2
// Computed as h' = ReLU(c + U h + sum_b W_b s_b) with s_b[v] = sum over
// type-b bonds of v of the neighbour's h (linearity; reading R7).
//
// B200 design: the per-step transforms are dense [atoms x 128] x [128 x 128]
// contractions, so they run on the tensor cores. Molecules are packed (host,
// deterministic greedy) into tiles of <= 128 atoms; a CTA (8 warps) owns a
// tile, warp w owns atom rows 16w..16w+15 and all 128 output features
// (64 fp32 accumulators per thread). Activations are fed as a bf16 hi/lo pair
// (x = hi + lo, two MMAs: ~16-bit mantissa, reading A17), weights are exact in
// bf16. Operands sit in shared memory with a 16-byte XOR swizzle and are
// fetched with ldmatrix; the next weight matrix is prefetched with cp.async
// while the current one is consumed. mma.sync m16n8k16 (legacy tensor path)
// in round 1; tcgen05/TMEM is NEXT.
#include "common.cuh"
#include "kernels.h"
#include "launch.cuh"

namespace mxk {

constexpr int kF = 128;
constexpr int kTileAtoms = 128;
constexpr int kTileEdges = 512;
constexpr int kMpnnThreads = 256;
constexpr int kMatBytes = kF * kF * 2;        // one 128x128 bf16 operand

// smem map
constexpr int kOffHhi = 0;
constexpr int kOffHlo = kOffHhi + kMatBytes;
constexpr int kOffShi = kOffHlo + kMatBytes;
constexpr int kOffSlo = kOffShi + kMatBytes;
constexpr int kOffW0 = kOffSlo + kMatBytes;
constexpr int kOffW1 = kOffW0 + kMatBytes;
constexpr int kOffEdges = kOffW1 + kMatBytes;                  // int4 [kTileEdges]
constexpr int kOffMolE = kOffEdges + kTileEdges * 16;          // int2 [kTileAtoms]: edge range
constexpr int kOffNbrOff = kOffMolE + kTileAtoms * 8;          // int [kTileAtoms+1] CSR offsets
constexpr int kOffNbr = kOffNbrOff + (kTileAtoms + 4) * 4;     // int [2*kTileEdges]: (u<<2)|b
constexpr int kReadoutMols = 4;                                // molecules per readout batch
constexpr int kOffR = kOffNbr + 2 * kTileEdges * 4;            // float [kReadoutMols][2][kF]: r, z
constexpr int kOffRed = kOffR + kReadoutMols * 2 * kF * 4;     // float [16]
constexpr int kMpnnSmem = kOffRed + 64;

int mpnn_smem_bytes() { return kMpnnSmem; }

// byte offset of element (row, col) of a swizzled [128][128] bf16 operand
__device__ __forceinline__ uint32_t sw_off(int row, int col) {
  return (uint32_t)(row * 256 + ((((col >> 3) ^ (row & 7))) << 4) + (col & 7) * 2);
}

__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// Async load of a row-major [128][128] bf16 matrix (global) into a swizzled smem operand.
__device__ __forceinline__ void load_matrix_async(uint32_t dst_base, const uint16_t* src, int tid) {
  for (int i = tid; i < kF * kF / 8; i += kMpnnThreads) {
    const int row = i >> 4, ch = i & 15;
    cp_async16(dst_base + (uint32_t)(row * 256 + ((ch ^ (row & 7)) << 4)), src + (size_t)i * 8);
  }
  cp_async_commit();
}

// fp32 -> (hi, lo) bf16 split; hi = RN(x), lo = RN(x - hi).
__device__ __forceinline__ void split_bf16(float x, uint16_t& hi, uint16_t& lo) {
  hi = f32_to_bf16_rne(x);
  lo = f32_to_bf16_rne(x - bf16_bits_to_f32(hi));
}

// acc[16 n-tiles][4] += A(16 rows of this warp, 128 k) . W^T  for A given as hi+lo.
__device__ __forceinline__ void mma_segment(float (&acc)[16][4], uint32_t a_hi, uint32_t a_lo,
                                            uint32_t w, int warp, int lane) {
  const int q = lane >> 3, r = lane & 7;
  const int arow = warp * 16 + (q & 1) * 8 + r;
#pragma unroll 2
  for (int k0 = 0; k0 < kF; k0 += 16) {
    const int acol = k0 + (q >> 1) * 8;
    uint32_t h0, h1, h2, h3, l0, l1, l2, l3;
    ldsm_x4(a_hi + sw_off(arow, acol), h0, h1, h2, h3);
    ldsm_x4(a_lo + sw_off(arow, acol), l0, l1, l2, l3);
#pragma unroll
    for (int nt = 0; nt < 16; nt += 2) {
      const int brow = nt * 8 + r + (q >> 1) * 8;
      const int bcol = k0 + (q & 1) * 8;
      uint32_t b0, b1, b2, b3;
      ldsm_x4(w + sw_off(brow, bcol), b0, b1, b2, b3);
      mma_bf16(acc[nt], h0, h1, h2, h3, b0, b1);
      mma_bf16(acc[nt], l0, l1, l2, l3, b0, b1);
      mma_bf16(acc[nt + 1], h0, h1, h2, h3, b2, b3);
      mma_bf16(acc[nt + 1], l0, l1, l2, l3, b2, b3);
    }
  }
}

__global__ void __launch_bounds__(kMpnnThreads, 1) mpnn_kernel(MpnnParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  const uint32_t sbase = smem_u32(smem_raw);
  const uint32_t Hhi = sbase + kOffHhi, Hlo = sbase + kOffHlo;
  const uint32_t Shi = sbase + kOffShi, Slo = sbase + kOffSlo;
  const uint32_t Wbuf[2] = {sbase + kOffW0, sbase + kOffW1};
  int4* ed = reinterpret_cast<int4*>(smem_raw + kOffEdges);
  int2* mol_e = reinterpret_cast<int2*>(smem_raw + kOffMolE);
  int* nbr_off = reinterpret_cast<int*>(smem_raw + kOffNbrOff);
  int* nbr = reinterpret_cast<int*>(smem_raw + kOffNbr);
  float* rz = reinterpret_cast<float*>(smem_raw + kOffR);
  float* red = reinterpret_cast<float*>(smem_raw + kOffRed);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int g = lane >> 2, t4 = lane & 3;
  if (blockIdx.x == 0 && tid == 0) p.stamps[0] = globaltimer();
  const uint8_t* eb = reinterpret_cast<const uint8_t*>(p.edges);

  for (int tile = blockIdx.x; tile < p.n_tiles; tile += p.n_ctas) {
    const int m0 = p.tile_off[tile], m1 = p.tile_off[tile + 1];
    const int a0 = p.atom_off[m0], na = p.atom_off[m1] - a0;
    const int e0 = p.edge_off[m0], ne = p.edge_off[m1] - e0;
    // atom -> its molecule's edge range (tile-local); edges in tile-local atom ids
    for (int i = tid; i < kTileAtoms; i += kMpnnThreads) mol_e[i] = make_int2(0, 0);
    __syncthreads();
    for (int m = m0 + tid; m < m1; m += kMpnnThreads) {
      const int ab = p.atom_off[m] - a0, ae = p.atom_off[m + 1] - a0;
      const int eb0 = p.edge_off[m] - e0, ee = p.edge_off[m + 1] - e0;
      for (int v = ab; v < ae; ++v) mol_e[v] = make_int2(eb0, ee);
    }
    for (int i = tid; i < ne; i += kMpnnThreads) {
      const uint8_t* e = eb + (size_t)(e0 + i) * 6;
      // local atom ids -> tile ids: add the molecule's first atom (found below)
      ed[i] = make_int4((int)(int16_t)(e[0] | (e[1] << 8)), (int)(int16_t)(e[2] | (e[3] << 8)),
                        (int)e[4], 0);
    }
    __syncthreads();
    for (int i = tid; i < ne; i += kMpnnThreads) {
      // molecule of edge i: binary search over the tile's edge offsets
      int lo = m0, hi = m1 - 1;
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (p.edge_off[mid] - e0 <= i) lo = mid; else hi = mid - 1;
      }
      const int base = p.atom_off[lo] - a0;
      ed[i].x += base;
      ed[i].y += base;
    }
    // h0 = E_atom[type] (bf16-exact: hi = value, lo = 0); padded rows = 0
    for (int i = tid; i < kTileAtoms * kF / 8; i += kMpnnThreads) {
      const int row = i >> 4, ch = i & 15;
      uint4 hv = make_uint4(0, 0, 0, 0);
      if (row < na) hv = *reinterpret_cast<const uint4*>(p.e_atom + (size_t)p.atom_type[a0 + row] * kF + ch * 8);
      const uint32_t off = (uint32_t)(row * 256 + ((ch ^ (row & 7)) << 4));
      *reinterpret_cast<uint4*>(smem_raw + kOffHhi + off) = hv;
      *reinterpret_cast<uint4*>(smem_raw + kOffHlo + off) = make_uint4(0, 0, 0, 0);
    }
    __syncthreads();
    // per-atom neighbour lists (CSR) in edge order: deterministic, built once per tile
    {
      int deg = 0;
      const int v = tid;
      if (v < kTileAtoms && v < na) {
        const int2 er = mol_e[v];
        for (int e = er.x; e < er.y; ++e) deg += (ed[e].x == v) + (ed[e].y == v);
      }
      // exclusive scan of degrees over the first 128 threads (4 warps)
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
      if (v < kTileAtoms) {
        int pos = base + incl - deg;
        nbr_off[v] = pos;
        if (v == kTileAtoms - 1) nbr_off[kTileAtoms] = base + incl;
        if (v < na) {
          const int2 er = mol_e[v];
          for (int e = er.x; e < er.y; ++e) {
            const int4 E = ed[e];
            if (E.x == v) nbr[pos++] = (E.y << 2) | E.z;
            if (E.y == v) nbr[pos++] = (E.x << 2) | E.z;
          }
        }
      }
    }
    __syncthreads();
    // which bond types occur in the tile (uniform loop, smem broadcast)
    int present = 0;
    for (int i = 0; i < ne; ++i) present |= 1 << ed[i].z;

    int wi = 0;   // weight buffer in use
    load_matrix_async(Wbuf[wi], p.u, tid);
    for (int step = 0; step < p.T; ++step) {
      float acc[16][4];
#pragma unroll
      for (int nt = 0; nt < 16; ++nt)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[nt][j] = 0.f;
      // segments: 0 = U . h, 1..4 = W_b . s_b for bond types present
      int seg_next[5];
      int nseg = 0;
      seg_next[nseg++] = 0;
      for (int b = 0; b < p.n_bonds; ++b)
        if (present & (1 << b)) seg_next[nseg++] = 1 + b;
      for (int si = 0; si < nseg; ++si) {
        const int seg = seg_next[si];
        // prefetch the next segment's weights (or U of the next step)
        const uint16_t* nxt = nullptr;
        if (si + 1 < nseg) nxt = p.w_b + (size_t)(seg_next[si + 1] - 1) * kF * kF;
        else if (step + 1 < p.T) nxt = p.u;
        uint32_t a_hi = Hhi, a_lo = Hlo;
        if (seg > 0) {
          // s_b[v] = sum over type-b bonds of v of h[neighbour], edge order
          const int b = seg - 1;
          for (int i = tid; i < kTileAtoms * 16; i += kMpnnThreads) {
            const int v = i >> 4, ch = i & 15;
            float sacc[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) sacc[j] = 0.f;
            if (v < na) {
              for (int q = nbr_off[v]; q < nbr_off[v + 1]; ++q) {
                const int nb = nbr[q];
                if ((nb & 3) != b) continue;
                const int other = nb >> 2;
                const uint32_t off = (uint32_t)(other * 256 + ((ch ^ (other & 7)) << 4));
                const uint4 hh = *reinterpret_cast<const uint4*>(smem_raw + kOffHhi + off);
                const uint4 hl = *reinterpret_cast<const uint4*>(smem_raw + kOffHlo + off);
                float fh[8], fl[8];
                unpack8(hh, fh);
                unpack8(hl, fl);
#pragma unroll
                for (int j = 0; j < 8; ++j) sacc[j] += fh[j] + fl[j];
              }
            }
            uint16_t sh[8], sl[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) split_bf16(sacc[j], sh[j], sl[j]);
            const uint32_t off = (uint32_t)(v * 256 + ((ch ^ (v & 7)) << 4));
            uint4 ph, pl;
            ph.x = sh[0] | ((uint32_t)sh[1] << 16); ph.y = sh[2] | ((uint32_t)sh[3] << 16);
            ph.z = sh[4] | ((uint32_t)sh[5] << 16); ph.w = sh[6] | ((uint32_t)sh[7] << 16);
            pl.x = sl[0] | ((uint32_t)sl[1] << 16); pl.y = sl[2] | ((uint32_t)sl[3] << 16);
            pl.z = sl[4] | ((uint32_t)sl[5] << 16); pl.w = sl[6] | ((uint32_t)sl[7] << 16);
            *reinterpret_cast<uint4*>(smem_raw + kOffShi + off) = ph;
            *reinterpret_cast<uint4*>(smem_raw + kOffSlo + off) = pl;
          }
          a_hi = Shi;
          a_lo = Slo;
        }
        cp_async_wait_all();
        __syncthreads();                       // weights + S visible; previous W buffer free
        if (nxt) load_matrix_async(Wbuf[wi ^ 1], nxt, tid);
        mma_segment(acc, a_hi, a_lo, Wbuf[wi], warp, lane);
        wi ^= 1;
        __syncthreads();                       // S / W consumed before they are rewritten
      }
      // h = ReLU(acc + c) -> hi/lo (padded rows stay 0)
#pragma unroll
      for (int nt = 0; nt < 16; ++nt) {
        const int col = nt * 8 + 2 * t4;
        const float c0 = bf16_bits_to_f32(p.c[col]), c1 = bf16_bits_to_f32(p.c[col + 1]);
#pragma unroll
        for (int hr = 0; hr < 2; ++hr) {
          const int row = warp * 16 + g + hr * 8;
          float v0 = fmaxf(acc[nt][2 * hr] + c0, 0.f), v1 = fmaxf(acc[nt][2 * hr + 1] + c1, 0.f);
          if (row >= na) v0 = v1 = 0.f;
          uint16_t h0, l0, h1, l1;
          split_bf16(v0, h0, l0);
          split_bf16(v1, h1, l1);
          const uint32_t off = sw_off(row, col);
          *reinterpret_cast<uint32_t*>(smem_raw + kOffHhi + off) = h0 | ((uint32_t)h1 << 16);
          *reinterpret_cast<uint32_t*>(smem_raw + kOffHlo + off) = l0 | ((uint32_t)l1 << 16);
        }
      }
      __syncthreads();
    }
    // readout: r_m = sum_v h_v (atom order); z_m = ReLU(W1 r_m + c1); y_m = w2 . z_m + c2,
    // W1 staged (swizzled) in a free weight buffer, molecules in batches of kReadoutMols
    cp_async_wait_all();
    __syncthreads();
    load_matrix_async(Wbuf[0], p.w1, tid);
    cp_async_wait_all();
    __syncthreads();
    for (int mb = m0; mb < m1; mb += kReadoutMols) {
      const int nm = min(kReadoutMols, m1 - mb);
      for (int i = tid; i < nm * kF; i += kMpnnThreads) {
        const int mm = i / kF, f = i - mm * kF;
        const int ab = p.atom_off[mb + mm] - a0, ae = p.atom_off[mb + mm + 1] - a0;
        float t = 0.f;
        for (int v = ab; v < ae; ++v) {
          const uint32_t off = sw_off(v, f);
          t += bf16_bits_to_f32(*reinterpret_cast<const uint16_t*>(smem_raw + kOffHhi + off)) +
               bf16_bits_to_f32(*reinterpret_cast<const uint16_t*>(smem_raw + kOffHlo + off));
        }
        rz[mm * 2 * kF + f] = t;
      }
      __syncthreads();
      for (int i = tid; i < nm * kF; i += kMpnnThreads) {
        const int mm = i / kF, f = i - mm * kF;
        const float* r = rz + mm * 2 * kF;
        float t = bf16_bits_to_f32(p.c1[f]);
        for (int k = 0; k < kF; k += 8) {
          const uint4 wv = *reinterpret_cast<const uint4*>(smem_raw + kOffW0 + sw_off(f, k));
          float wf[8];
          unpack8(wv, wf);
#pragma unroll
          for (int j = 0; j < 8; ++j) t = fmaf(wf[j], r[k + j], t);
        }
        rz[mm * 2 * kF + kF + f] = fmaxf(t, 0.f);
      }
      __syncthreads();
      // one warp per molecule: y = w2 . z + c2 (fixed shuffle tree)
      if (warp < nm) {
        const float* z = rz + warp * 2 * kF + kF;
        float part = 0.f;
        for (int f = lane; f < kF; f += 32) part = fmaf(bf16_bits_to_f32(p.w2[f]), z[f], part);
        part = warp_sum(part);
        if (lane == 0) {
          p.out[mb + warp] = part + bf16_bits_to_f32(p.c2[0]);
          __threadfence_system();   // ordered before the completion flag
        }
      }
      __syncthreads();
    }
  }
  __syncthreads();
  if (tid == 0) {
    atomicMax(&p.stamps[1], (unsigned long long)globaltimer());
    if (p.h_stamps) {
      __threadfence_system();
      // the last CTA to finish publishes the completion record
      if (atomicAdd(&p.stamps[4], 1ull) == (unsigned long long)(gridDim.x - 1)) {
        __threadfence();
        volatile unsigned long long* st = p.stamps;
        volatile unsigned long long* h = p.h_stamps;
        h[0] = st[0];
        h[1] = st[1];
        h[2] = 0;
        p.stamps[4] = 0;
        __threadfence_system();
        h[3] = p.done_tag;
      }
    }
  }
}

int launch_mpnn(const MpnnParams& p, void* stream) {
  MpnnParams pc = p;
  void* args[] = {&pc};
  return launch_kernel(mpnn_kernel, dim3(p.n_ctas), dim3(kMpnnThreads), (unsigned)mpnn_smem_bytes(),
                       stream, args);
}

int mpnn_set_attrs(int device) { return set_max_smem(mpnn_kernel, mpnn_smem_bytes(), device); }

// Deterministic greedy packing of molecules into tiles of <= 128 atoms and
// <= 512 bonds (host side, runs at launch). Returns the number of tiles.
int mpnn_pack_tiles(const int* atom_off, const int* edge_off, int n_mol, int* tile_off) {
  int nt = 0;
  tile_off[0] = 0;
  int a = 0, e = 0;
  for (int m = 0; m < n_mol; ++m) {
    const int na = atom_off[m + 1] - atom_off[m], ne = edge_off[m + 1] - edge_off[m];
    if ((a + na > kTileAtoms || e + ne > kTileEdges) && a > 0) {
      tile_off[++nt] = m;
      a = e = 0;
    }
    a += na;
    e += ne;
  }
  tile_off[++nt] = n_mol;
  return nt;
}

}  // namespace mxk
