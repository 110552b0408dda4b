// Grid-barrier microbenchmark (tools only, not product): latency of one
// device-wide barrier among C persistent CTAs, with and without a concurrent
// TMA weight stream on every SM (the decode megakernel's situation).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/bb tools/barrier_bench.cu
//   /tmp/bb
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int kThreads = 416, kStages = 6, kStage = 32768;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t gtime() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ uint64_t ld_relaxed(const unsigned long long* p) {
  uint64_t v; asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ uint64_t ld_acquire(const unsigned long long* p) {
  uint64_t v; asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }

__global__ void __launch_bounds__(kThreads, 1) bench(unsigned long long* bar, unsigned long long* flags,
                                                    const uint8_t* stream_src, size_t stream_bytes,
                                                    int variant, int iters, int do_stream,
                                                    unsigned long long* out_ns, unsigned long long base) {
  extern __shared__ __align__(128) uint8_t sm[];
  uint64_t* full = reinterpret_cast<uint64_t*>(sm + kStages * kStage);
  volatile int* stop = reinterpret_cast<volatile int*>(full + kStages);
  const int tid = threadIdx.x, warp = tid >> 5, C = gridDim.x;
  if (tid == 0) {
    for (int i = 0; i < kStages; ++i)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[i])));
    asm volatile("fence.mbarrier_init.release.cluster;");
    *stop = 0;
  }
  __syncthreads();
  if (warp == 0) {
    if (tid == 0 && do_stream) {
      size_t off = (size_t)blockIdx.x * kStage * 64;
      uint32_t ph[kStages] = {0};
      for (int i = 0;; ++i) {
        const int s = i % kStages;
        if (i >= kStages) {   // wait for this slot's previous copy
          uint32_t ok = 0;
          while (!ok) {
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                         : "=r"(ok) : "r"(su32(&full[s])), "r"(ph[s]) : "memory");
          }
          ph[s] ^= 1;
        }
        if (*stop) break;
        if (off + kStage > stream_bytes) off = 0;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(kStage) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(su32(sm + s * kStage)), "l"(stream_src + off), "r"(kStage), "r"(su32(&full[s])) : "memory");
        off += (size_t)C * kStage;
      }
      // drain
      for (int s = 0; s < kStages; ++s) {
        uint32_t ok = 0;
        for (int k = 0; k < 100000 && !ok; ++k)
          asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                       : "=r"(ok) : "r"(su32(&full[s])), "r"(ph[s]) : "memory");
      }
    }
    return;
  }
  const int tc = tid - 32, nct = kThreads - 32;
  unsigned long long target = base;
  const uint64_t t0 = gtime();
  for (int it = 0; it < iters; ++it) {
    target += C;
    asm volatile("bar.sync 1, %0;" ::"r"(nct) : "memory");
    if (variant == 0) {            // current: red.release + relaxed spin + acquire load
      if (tc == 0) {
        asm volatile("red.release.gpu.global.add.u64 [%0], 1;" ::"l"(bar) : "memory");
        while (ld_relaxed(bar) < target) {}
        (void)ld_acquire(bar);
      }
    } else if (variant == 1) {     // no fence (NOT a correct barrier; fence cost reference)
      if (tc == 0) {
        asm volatile("red.relaxed.gpu.global.add.u64 [%0], 1;" ::"l"(bar) : "memory");
        while (ld_relaxed(bar) < target) {}
      }
    } else if (variant == 2) {     // per-CTA flags: st.release own flag, C threads poll one flag each
      const unsigned long long epoch = (target - base) / C + (base / C) ;
      if (tc == 0) asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(flags + blockIdx.x * 8), "l"(epoch) : "memory");
      if (tc < C) {
        while (ld_relaxed(flags + tc * 8) < epoch) {}
        (void)ld_acquire(flags + tc * 8);
      }
    } else if (variant == 3) {     // fence + relaxed red, spin with acquire loads
      if (tc == 0) {
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        asm volatile("red.relaxed.gpu.global.add.u64 [%0], 1;" ::"l"(bar) : "memory");
        while (ld_acquire(bar) < target) {}
      }
    } else if (variant == 4) {     // atom.add.release returns old; spin
      if (tc == 0) {
        unsigned long long old;
        asm volatile("atom.release.gpu.global.add.u64 %0, [%1], 1;" : "=l"(old) : "l"(bar), "l"(1ull) : "memory");
        if (old + 1 < target) while (ld_relaxed(bar) < target) {}
        (void)ld_acquire(bar);
      }
    }
    asm volatile("bar.sync 1, %0;" ::"r"(nct) : "memory");
  }
  const uint64_t t1 = gtime();
  if (tc == 0) { *stop = 1; if (blockIdx.x == 0) out_ns[0] = t1 - t0; }
}

int main() {
  const size_t sb = (size_t)2 << 30;
  uint8_t* src; cudaMalloc(&src, sb); cudaMemset(src, 1, sb);
  unsigned long long *bar, *flags, *out;
  cudaMalloc(&bar, 8); cudaMalloc(&flags, 8 * 8 * 256); cudaMalloc(&out, 8);
  const int smem = kStages * kStage + kStages * 8 + 16;
  cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 2000;
  const char* names[] = {"red.release+spin", "relaxed(no fence)", "flags st.release", "fence+red+acq spin", "atom.release"};
  int grids[] = {4, 36, 74, 148};
  for (int gi = 0; gi < 4; ++gi)
    for (int stream = 0; stream < 2; ++stream)
      for (int v = 0; v < 5; ++v) {
        cudaMemset(bar, 0, 8); cudaMemset(flags, 0, 8 * 8 * 256);
        bench<<<grids[gi], kThreads, smem>>>(bar, flags, src, sb, v, iters, stream, out, 0);
        cudaError_t e = cudaDeviceSynchronize();
        unsigned long long ns = 0; cudaMemcpy(&ns, out, 8, cudaMemcpyDeviceToHost);
        printf("ctas %3d stream %d %-20s %7.3f us/barrier %s\n", grids[gi], stream, names[v],
               ns / 1000.0 / iters, e == cudaSuccess ? "" : cudaGetErrorString(e));
      }
  return 0;
}
