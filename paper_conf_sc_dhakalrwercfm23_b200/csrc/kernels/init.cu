// Cold-start kernels (§6 P:240 "loading AI model
// into video memory"): seeded bf16 weight generation directly in the
// partition's arena, the RoPE table, and the %smid probe (K9).
//
// Device implementation of the counter-based generator of SURVEY.md §8(c) C1
// (written independently of workloads/prng.py; a GPU test checks the two agree
// bit for bit):
//   f(z): z ^= z>>30; z *= 0xBF58476D1CE4E5B9; z ^= z>>27; z *= 0x94D049BB133111EB; z ^= z>>31
//   draw(s, i) = f(s + (i+1) * 0x9E3779B97F4A7C15);  key(s, st) = draw(s ^ draw(st, 0), 0)
//   weight:  ((draw(key(seed, tid), i) >> 56) - 128) * 2^-12
//   gain:    1 + ((draw(key(seed, tid), i) >> 60) - 8) * 2^-6
#include "common.cuh"
#include "kernels.h"
#include "launch.cuh"

namespace mxk {

__host__ __device__ __forceinline__ uint64_t sm64_mix(uint64_t z) {
  z ^= z >> 30;
  z *= 0xBF58476D1CE4E5B9ull;
  z ^= z >> 27;
  z *= 0x94D049BB133111EBull;
  z ^= z >> 31;
  return z;
}

__host__ __device__ __forceinline__ uint64_t sm64_draw(uint64_t s, uint64_t i) {
  return sm64_mix(s + (i + 1ull) * 0x9E3779B97F4A7C15ull);
}

__host__ __device__ __forceinline__ uint64_t sm64_key(uint64_t s, uint64_t st) {
  return sm64_draw(s ^ sm64_draw(st, 0), 0);
}

__global__ void fill_weights_kernel(uint16_t* dst, uint64_t n, uint64_t key, int is_gain) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x * 8;
  for (uint64_t i0 = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8; i0 < n; i0 += stride) {
    uint16_t v[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint64_t r = sm64_draw(key, i0 + q);
      float f;
      if (is_gain)
        f = 1.0f + (float)((int)(r >> 60) - 8) * 0.015625f;
      else
        f = (float)((int)(r >> 56) - 128) * 0.000244140625f;
      v[q] = (uint16_t)(__float_as_uint(f) >> 16);   // exact: value has <= 8 significant bits
    }
    if (i0 + 8 <= n && ((reinterpret_cast<uintptr_t>(dst + i0) & 15) == 0)) {
      uint4 pk;
      pk.x = v[0] | ((uint32_t)v[1] << 16);
      pk.y = v[2] | ((uint32_t)v[3] << 16);
      pk.z = v[4] | ((uint32_t)v[5] << 16);
      pk.w = v[6] | ((uint32_t)v[7] << 16);
      *reinterpret_cast<uint4*>(dst + i0) = pk;
    } else {
      for (int q = 0; q < 8 && i0 + q < n; ++q) dst[i0 + q] = v[q];
    }
  }
}

int launch_fill_weights(uint16_t* dst, uint64_t n, uint64_t seed, uint32_t tid, int is_gain,
                        int n_ctas, void* stream) {
  uint64_t key = sm64_key(seed, tid);
  uint64_t blocks = (n + 8 * 256 - 1) / (8 * 256);
  uint64_t cap = (uint64_t)n_ctas * 8;
  if (blocks > cap) blocks = cap;
  if (blocks < 1) blocks = 1;
  void* args[] = {&dst, &n, &key, &is_gain};
  return launch_kernel(fill_weights_kernel, dim3((unsigned)blocks), dim3(256), 0, stream, args);
}

// RoPE table [max_seq][hd/2] of (cos a, sin a), a = fl32(t * inv_freq_i),
// inv_freq_i = fl32(1 / theta^(fl32(2i/hd))) (A11, HF's fp32 convention).
__global__ void rope_table_kernel(float* dst, int max_seq, int hd, float theta) {
  const int half = hd / 2;
  const int n = max_seq * half;
  for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < n; idx += gridDim.x * blockDim.x) {
    const int t = idx / half, i = idx - t * half;
    const float expo = (float)(2 * i) / (float)hd;
    const float inv_freq = 1.0f / powf(theta, expo);
    const float a = (float)t * inv_freq;
    float s, c;
    sincosf(a, &s, &c);
    dst[2 * idx] = c;
    dst[2 * idx + 1] = s;
  }
}

int launch_rope_table(float* dst, int max_seq, int hd, float theta, void* stream) {
  void* args[] = {&dst, &max_seq, &hd, &theta};
  return launch_kernel(rope_table_kernel, dim3(16), dim3(256), 0, stream, args);
}

// K9: each CTA records the SM it ran on, after spinning for spin_ns so that
// concurrently launched probes overlap in time.
__global__ void probe_kernel(uint32_t* smids, uint64_t spin_ns) {
  if (threadIdx.x == 0) {
    const uint64_t t0 = globaltimer();
    while (globaltimer() - t0 < spin_ns) {
    }
    smids[blockIdx.x] = smid();
  }
}

int launch_probe(uint32_t* smids, int n_ctas, uint64_t spin_ns, void* stream) {
  void* args[] = {&smids, &spin_ns};
  return launch_kernel(probe_kernel, dim3(n_ctas), dim3(32), 0, stream, args);
}

DriverLaunch& driver_launch() {
  static DriverLaunch d;
  return d;
}

std::atomic<uint64_t>& launch_count_ref() {
  static std::atomic<uint64_t> c{0};
  return c;
}

uint64_t launch_counter() { return launch_count_ref().load(); }

}  // namespace mxk

namespace mxk {

__global__ void clock_kernel(unsigned long long* out) {
  if (threadIdx.x == 0) out[0] = globaltimer();
}

int launch_clock(unsigned long long* out, void* stream) {
  void* args[] = {&out};
  return launch_kernel(clock_kernel, dim3(1), dim3(32), 0, stream, args);
}

}  // namespace mxk
