// Microbenchmark: issue-to-completion cost of skinny tcgen05 MMAs (the decode
// GEMV shape) on one SM. One thread issues `iters` MMAs (bf16, K = 16 each,
// both operands K-major SWIZZLE_128B in shared memory), commits, waits, and
// reports cycles per MMA for several (M, N, A-stream) configurations.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tcb tools/tc_bench.cu && /tmp/tcb
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__host__ __device__ constexpr uint32_t idesc(int M, int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

// mode 0: A streams through `a_boxes` 16 KiB boxes (4 MMAs per box, K advanced by 32 B)
// mode 1: A fixed (same 4 MMAs repeated)
__global__ void bench(int M, int N, int iters, int a_boxes, int accs, int warp_wide, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint8_t* base = smem + ((1024 - (su32(smem) & 1023)) & 1023);
  __shared__ uint64_t bar;
  __shared__ uint32_t tmem;
  for (int i = threadIdx.x; i < 160 * 1024 / 16; i += blockDim.x)
    reinterpret_cast<uint4*>(base)[i] = make_uint4(0x3f803f80u, 0, 0x3f803f80u, 0);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&tmem)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t t = tmem;
  if (threadIdx.x < 32 && warp_wide == 1) {
    // the whole warp runs the loop (descriptors are warp-uniform -> uniform
    // registers); one elected lane issues each MMA
    const uint32_t id = idesc(M, N);
    const uint32_t a0 = su32(base), b0 = su32(base + 128 * 1024);
    long long c0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const int box = (i >> 2) % a_boxes, j = i & 3;
      const uint64_t ad = desc_sw128(a0 + box * 16384 + j * 32, 1024);
      const uint64_t bd = desc_sw128(b0 + (box % 4) * 2048 + j * 32, 1024);
      const uint32_t dd = t + (uint32_t)((i % accs) * (N < 32 ? 32 : N));
      asm volatile("{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                   "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(dd),
                   "l"(ad), "l"(bd), "r"(id), "r"(i >= accs ? 1 : 0));
    }
    long long c1 = clock64();
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                 "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar)));
    uint32_t ok = 0;
    while (!ok)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(ok) : "r"(su32(&bar)));
    long long c2 = clock64();
    if (threadIdx.x == 0) {
      out[0] = c1 - c0;
      out[1] = c2 - c0;
    }
  } else if (threadIdx.x < 32 && warp_wide == 2) {
    // uniform: TMEM base broadcast by a shuffle, descriptors precomputed and
    // advanced by integer adds, 4 MMAs per box unrolled
    const uint32_t id = idesc(M, N);
    const uint32_t tu = __shfl_sync(0xffffffffu, t, 0);
    const uint64_t ad0 = desc_sw128(su32(base), 1024), bd0 = desc_sw128(su32(base + 128 * 1024), 1024);
    long long c0 = clock64();
    for (int i = 0; i < iters / 4; ++i) {
      const int box = i % a_boxes;
      const uint64_t ad = ad0 + (uint64_t)(box * 1024), bd = bd0 + (uint64_t)((box & 3) * 128);
#pragma unroll
      for (int j = 0; j < 4; ++j)
        asm volatile("{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tu),
                     "l"(ad + 2 * j), "l"(bd + 2 * j), "r"(id), "r"((i | j) ? 1 : 0));
    }
    long long c1 = clock64();
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                 "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar)));
    uint32_t ok = 0;
    while (!ok)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(ok) : "r"(su32(&bar)));
    long long c2 = clock64();
    if (threadIdx.x == 0) {
      out[0] = c1 - c0;
      out[1] = c2 - c0;
    }
  } else if (warp_wide == 3 && threadIdx.x < 64) {
    // two warps issue concurrently into disjoint accumulators (uniform descriptors)
    const int w = threadIdx.x >> 5;
    const uint32_t id = idesc(M, N);
    const uint32_t tu = __shfl_sync(0xffffffffu, t, 0) + (uint32_t)(w * 128);
    const uint64_t ad0 = desc_sw128(su32(base) + w * 65536, 1024), bd0 = desc_sw128(su32(base + 128 * 1024), 1024);
    __syncwarp();
    long long c0 = clock64();
    for (int i = 0; i < iters / 8; ++i) {
      const int box = i % 4;
      const uint64_t ad = ad0 + (uint64_t)(box * 1024), bd = bd0 + (uint64_t)((box & 3) * 128);
#pragma unroll
      for (int j = 0; j < 4; ++j)
        asm volatile("{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tu),
                     "l"(ad + 2 * j), "l"(bd + 2 * j), "r"(id), "r"((i | j) ? 1 : 0));
    }
    long long c1 = clock64();
    if (w == 0) {
      asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                   "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar)));
      uint32_t ok = 0;
      while (!ok)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok) : "r"(su32(&bar)));
      long long c2 = clock64();
      if (threadIdx.x == 0) {
        out[0] = c1 - c0;
        out[1] = c2 - c0;
      }
    }
  } else if ((warp_wide == 4 || warp_wide == 5) && threadIdx.x < 32) {
    // per-box mbarrier wait inside the loop (the barrier is already complete):
    // 4 = C++ polling loop + __syncwarp (as the decode kernel), 5 = spin loop inside PTX
    const uint32_t id = idesc(M, N);
    const uint32_t tu = __shfl_sync(0xffffffffu, t, 0);
    const uint32_t a0 = su32(base), b0 = su32(base + 128 * 1024);
    const uint32_t wb = su32(&bar);
    long long c0 = clock64();
    uint32_t stage = 0;
    for (int i = 0; i < iters / 4; ++i) {
      if (warp_wide == 4) {
        uint32_t ok = 0;
        while (!ok)
          asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 1;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                       : "=r"(ok) : "r"(wb));
        __syncwarp();
      } else {
        asm volatile("{\n\t.reg .pred p;\n\tWAIT_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 1;\n\t@!p bra WAIT_%=;\n\t}" ::"r"(wb) : "memory");
      }
      const uint32_t sa = a0 + stage * 16384u;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint64_t ad = desc_sw128(sa + j * 32, 1024), bd = desc_sw128(b0 + j * 32, 1024);
        asm volatile("{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tu),
                     "l"(ad), "l"(bd), "r"(id), "r"((i | j) ? 1 : 0));
      }
      if (++stage == (uint32_t)a_boxes) stage = 0;
    }
    long long c1 = clock64();
    if (threadIdx.x == 0) {
      out[0] = c1 - c0;
      out[1] = c1 - c0;
    }
  } else if (threadIdx.x == 0 && !warp_wide) {
    const uint32_t id = idesc(M, N);
    const uint32_t a0 = su32(base), b0 = su32(base + 128 * 1024);
    const uint32_t sbo_b = 1024;
    long long c0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const int box = (i >> 2) % a_boxes, j = i & 3;
      const uint64_t ad = desc_sw128(a0 + box * 16384 + j * 32, 1024);
      const uint64_t bd = desc_sw128(b0 + (box % 4) * 2048 + j * 32, sbo_b);
      const uint32_t d = t + (uint32_t)((i % accs) * (N < 32 ? 32 : N));
      asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                   "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
                   "l"(ad), "l"(bd), "r"(id), "r"(i >= accs ? 1 : 0));
    }
    long long c1 = clock64();
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)));
    uint32_t ok = 0;
    while (!ok)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(ok) : "r"(su32(&bar)));
    long long c2 = clock64();
    out[0] = c1 - c0;
    out[1] = c2 - c0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(t));
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 16);
  cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  struct Cfg { int M, N, boxes, accs, ww; const char* what; } cfgs[] = {
      {128, 16, 8, 1, 0, "1 thread: M128 N16 (decode GEMV as built)"},
      {128, 16, 8, 1, 1, "warp+elect: M128 N16"},
      {128, 16, 8, 4, 1, "warp+elect: M128 N16 4 accs"},
      {128, 32, 8, 1, 1, "warp+elect: M128 N32"},
      {128, 64, 8, 1, 1, "warp+elect: M128 N64"},
      {128, 128, 8, 1, 1, "warp+elect: M128 N128"},
      {128, 256, 8, 1, 1, "warp+elect: M128 N256"},
      {64, 16, 8, 1, 1, "warp+elect: M64 N16"},
      {128, 16, 8, 1, 2, "uniform descs: M128 N16"},
      {128, 64, 8, 1, 2, "uniform descs: M128 N64"},
      {128, 256, 8, 1, 2, "uniform descs: M128 N256"},
      {64, 16, 8, 1, 2, "uniform descs: M64 N16"},
      {128, 16, 8, 1, 3, "2 warps concurrently, M128 N16 (per MMA of all)"},
      {128, 16, 8, 1, 4, "per-box C++ mbarrier poll + syncwarp, M128 N16"},
      {128, 16, 8, 1, 5, "per-box PTX spin-loop wait, M128 N16"},
      {64, 16, 8, 1, 3, "2 warps concurrently, M64 N16 (per MMA of all)"},
  };
  for (auto& c : cfgs) {
    const int iters = 4096;
    unsigned long long h[2];
    bench<<<1, 128, 200 * 1024>>>(c.M, c.N, iters, c.boxes, c.accs, c.ww, d);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("%s: error %s\n", c.what, cudaGetErrorString(e)); return 1; }
    bench<<<1, 128, 200 * 1024>>>(c.M, c.N, iters, c.boxes, c.accs, c.ww, d);
    cudaDeviceSynchronize();
    cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
    printf("%-60s issue %6.1f cyc/MMA, complete %6.1f cyc/MMA\n", c.what, (double)h[0] / iters,
           (double)h[1] / iters);
  }
  return 0;
}
