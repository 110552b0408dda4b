// Correctness probe for the decode GEMV's MMA issue styles: D[128][16] = A[128][64] . B[16][64]^T
// (bf16, K-major SWIZZLE_128B, 4 MMAs of K = 16) issued (0) by one thread, (1) by a warp with
// elect.sync inside the asm, (2) by a warp under if (lane == 0); D read back with tcgen05.ld.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tcc tools/tc_check.cu && /tmp/tcc
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cuda_runtime.h>
#include <cuda_bf16.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(16 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
constexpr uint32_t kIdesc64 = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(16 >> 3) << 17) | ((uint32_t)(64 >> 4) << 24);

// element (row, k) of a [rows][64] K-major SW128 operand
__device__ __forceinline__ uint32_t off(int row, int k) {
  const int ch = k >> 3, r = row & 7;
  return (uint32_t)((row >> 3) * 1024 + r * 128 + ((ch ^ r) << 4) + (k & 7) * 2);
}

__global__ void check(const float* A, const float* Bm, float* D, int mode, uint32_t sbo_b) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint8_t* base = smem + ((1024 - (su32(smem) & 1023)) & 1023);
  uint8_t* sa = base;            // 16 KiB
  uint8_t* sb = base + 16384;    // 2 KiB (16 rows) or 1 KiB (8 rows, read twice)
  __shared__ uint64_t bar;
  __shared__ uint32_t tmem;
  const int tid = threadIdx.x;
  for (int i = tid; i < 128 * 64; i += blockDim.x)
    *reinterpret_cast<__nv_bfloat16*>(sa + off(i / 64, i % 64)) = __float2bfloat16(A[i]);
  for (int i = tid; i < 16 * 64; i += blockDim.x)
    *reinterpret_cast<__nv_bfloat16*>(sb + off(i / 64, i % 64)) = __float2bfloat16(Bm[i]);
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (tid < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(su32(&tmem)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t t = tmem;
  const uint64_t ad = desc_sw128(su32(sa), 1024), bd = desc_sw128(su32(sb), sbo_b);
  if (mode == 0 && tid == 0) {
    for (int j = 0; j < 4; ++j)
      asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                   "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(t),
                   "l"(ad + 2 * j), "l"(bd + 2 * j), "r"(kIdesc), "r"(j > 0 ? 1 : 0));
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)));
  } else if (mode == 1 && tid < 32) {
    for (int j = 0; j < 4; ++j)
      asm volatile("{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                   "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(t),
                   "l"(ad + 2 * j), "l"(bd + 2 * j), "r"(kIdesc), "r"(j > 0 ? 1 : 0));
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                 "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar)));
  } else if (mode == 3 && tid == 0) {
    // M = 64: where do the 64 rows of D land in TMEM?
    for (int j = 0; j < 4; ++j)
      asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                   "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(t),
                   "l"(ad + 2 * j), "l"(bd + 2 * j), "r"(kIdesc64), "r"(j > 0 ? 1 : 0));
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)));
  } else if (mode == 2 && tid < 32) {
    const uint32_t tu = __shfl_sync(0xffffffffu, t, 0);
    for (int j = 0; j < 4; ++j)
      asm volatile("{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                   "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tu),
                   "l"(ad + 2 * j), "l"(bd + 2 * j), "r"(kIdesc), "r"((j > 0) ? 1 : 0));
    __syncwarp();
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                 "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar)));
  }
  uint32_t ok = 0;
  while (!ok)
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(su32(&bar)));
  asm volatile("tcgen05.fence::after_thread_sync;");
  uint32_t r[16];
  const int w = tid >> 5, lane = tid & 31;
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15}, [%16];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                 "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
               : "r"(t + ((uint32_t)(32 * w) << 16)));
  asm volatile("tcgen05.wait::ld.sync.aligned;");
  for (int n = 0; n < 16; ++n) D[(32 * w + lane) * 16 + n] = __uint_as_float(r[n]);
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(t));
}

int main() {
  float hA[128 * 64], hB[16 * 64], hD[128 * 16];
  for (int i = 0; i < 128 * 64; ++i) hA[i] = (float)((i * 37 % 17) - 8) / 8.f;
  for (int i = 0; i < 16 * 64; ++i) hB[i] = (float)((i * 11 % 13) - 6) / 4.f;
  float *A, *Bm, *D;
  cudaMalloc(&A, sizeof hA); cudaMalloc(&Bm, sizeof hB); cudaMalloc(&D, sizeof hD);
  cudaMemcpy(A, hA, sizeof hA, cudaMemcpyHostToDevice);
  cudaMemcpy(Bm, hB, sizeof hB, cudaMemcpyHostToDevice);
  cudaFuncSetAttribute(check, cudaFuncAttributeMaxDynamicSharedMemorySize, 40 * 1024);
  {
    // M = 64 layout probe: for each TMEM lane, which row m of D (if any) it holds
    cudaMemset(D, 0, sizeof hD);
    check<<<1, 128, 40 * 1024>>>(A, Bm, D, 3, 1024);
    cudaDeviceSynchronize();
    cudaMemcpy(hD, D, sizeof hD, cudaMemcpyDeviceToHost);
    printf("M=64 lane -> row:");
    for (int lane = 0; lane < 128; ++lane) {
      int found = -1;
      for (int m = 0; m < 64 && found < 0; ++m) {
        bool ok = true;
        for (int n = 0; n < 16 && ok; ++n) {
          double ref = 0;
          for (int k = 0; k < 64; ++k) ref += (double)hA[m * 64 + k] * hB[n * 64 + k];
          ok = fabs(ref - hD[lane * 16 + n]) < 1e-3;
        }
        if (ok) found = m;
      }
      printf(" %d:%d", lane, found);
    }
    printf("\n");
  }
  for (int sbo = 0; sbo <= 1024; sbo += 1024)
    for (int mode = 0; mode < 3; ++mode) {
      cudaMemset(D, 0, sizeof hD);
      check<<<1, 128, 40 * 1024>>>(A, Bm, D, mode, sbo);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("mode %d: %s\n", mode, cudaGetErrorString(e)); return 1; }
      cudaMemcpy(hD, D, sizeof hD, cudaMemcpyDeviceToHost);
      double maxerr = 0;
      for (int m = 0; m < 128; ++m)
        for (int n = 0; n < 16; ++n) {
          const int nb = (sbo == 0) ? (n & 7) : n;   // SBO 0: rows 8-15 repeat rows 0-7
          double ref = 0;
          for (int k = 0; k < 64; ++k) ref += (double)hA[m * 64 + k] * hB[nb * 64 + k];
          maxerr = fmax(maxerr, fabs(ref - hD[m * 16 + n]));
        }
      printf("sbo %4d mode %d (%s): max |D - ref| = %g\n", sbo, mode,
             mode == 0 ? "one thread" : mode == 1 ? "warp, elect in asm" : "warp, shfl base + syncwarp", maxerr);
    }
  return 0;
}
