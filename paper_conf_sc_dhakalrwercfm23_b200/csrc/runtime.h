// Host runtime internals: devices, partitions (green contexts + arenas),
// function instances, task slots, tasks and the per-GPU dispatcher.
#pragma once

#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include <cuda.h>

#include "../../include/mx.h"
#include "arena.h"
#include "kernels/kernels.h"
#include "placement.h"

namespace mx {

uint64_t now_ns();
void set_error(const char* fmt, ...);

struct Gpu;
struct Partition;
struct FnInst;

// One execution context of a partition: a green context over its SM groups
// and one non-blocking stream (all of the partition's work is FIFO on it).
struct Exec {
  CUgreenCtx gctx = nullptr;
  CUcontext ctx = nullptr;
  CUstream stream = nullptr;
  int n_ctas = 0;          // SMs provisioned (persistent grid size)
  bool shared = false;     // whole-device stream, no SM restriction (N1); cooperative launches
  uint32_t epoch = 0;
  CUevent ev[2][3] = {};   // per in-flight lane: kernel start, kernel end, done
  int inflight = 0;
  uint64_t key = 0;        // SM-group mask | whole << 63 (green-context pool key)
};

struct Task {
  uint64_t id = 0;
  int fn = 0;
  int kind = 0;
  int gpu = 0, part = 0;
  uint64_t seq = 0;
  uint32_t epoch = 0;
  uint64_t cost = 0;
  // decode
  int B = 0, P = 0, G = 0;
  std::vector<int32_t> prompt;
  int32_t* out_tokens = nullptr;
  float* out_logits = nullptr;
  // mpnn: the task's inputs packed at submit time in their device image (one
  // H2D copy at launch): atom_off | edge_off | tile_off | targets (training) |
  // atom_type | edges, each 64-byte aligned (offsets below, bytes).
  int n_mol = 0, n_atoms = 0, n_edges = 0;
  std::vector<uint8_t> blob;
  uint32_t off_ao = 0, off_eo = 0, off_tile = 0, off_tg = 0, off_at = 0, off_ed = 0;
  int n_tiles = 0;
  int tile_ctas = -1;         // CTA count the inference tiling was balanced for
  float* out_ip = nullptr;
  // mpnn training step (N4)
  float lr = 0.f;
  float* out_loss = nullptr;
  // execution
  bool ready = false;
  FnInst* inst = nullptr;
  int slot = -1;
  Exec* exec = nullptr;
  int lane = 0;
  bool use_flag = false;      // completion = kernel-written host flag (no stream events)
  uint32_t polls = 0;
  // completion
  mx_status status = MX_OK;
  bool done = false;
  bool collected = false;
  uint64_t t_submit = 0, t_start = 0, t_end = 0, kernel_ns = 0;
};

// Device + pinned-host buffers of one task slot of a function instance.
struct Slot {
  bool busy = false;
  // decode
  CUdeviceptr x = 0, qkv = 0, o = 0, a = 0, cand = 0, kpart = 0, pflag = 0, kc = 0, vc = 0, prompt = 0, tokens = 0,
              logits = 0, img_x = 0, img_o = 0, img_a = 0, ssq = 0;
  // mpnn: device image of a task's packed inputs (Task::blob)
  CUdeviceptr in_blob = 0;
  // mpnn training (N4)
  CUdeviceptr y = 0, partials = 0, hsave = 0, wimg = 0;
  // common
  CUdeviceptr bar = 0, stamps = 0, err = 0;
  uint64_t bar_count = 0;
  bool need_reset = false;
  // pinned host staging
  void* h_in = nullptr;
  size_t h_in_bytes = 0;
  void* h_out = nullptr;
  size_t h_out_bytes = 0;
  uint64_t* h_stamps = nullptr;   // [0] start, [1] end, [2] err, [3] done tag (host-mapped)
  // device views of the host-mapped buffers (kernels write results and the
  // completion flag there directly; no copy-engine work in the stream)
  CUdeviceptr d_in = 0, d_out = 0, d_stamps = 0;
};

struct Fn {
  int id = 0;
  mx_fn_desc desc{};
};

struct FnInst {
  Fn* fn = nullptr;
  Partition* part = nullptr;
  CUdeviceptr weights = 0;
  uint64_t weight_bytes = 0;
  CUdeviceptr rope = 0;
  CUdeviceptr tmaps = 0;         // decode: mxk::kDecodeMaps CUtensorMap over the weights
  // decode layout (elements)
  uint64_t layer_stride = 0, off_wqkv = 0, off_wo = 0, off_wgate = 0, off_wup = 0, off_wdown = 0,
           off_gattn = 0, off_gmlp = 0, off_gfinal = 0, off_lm = 0, off_embed = 0;
  // mpnn layout (elements)
  uint64_t m_off[11] = {};
  Slot slots[2];
  bool loaded = false;
  bool shared_weights = false;   // weights/rope point into the GPU's weight pool (N3)
  CUdeviceptr params = 0;        // MX_FN_MPNN_TRAIN: fp32 training state (N4)
  uint64_t n_params = 0;
};

// One function's read-only weights in a GPU's shared pool (N3).
struct SharedWeights {
  CUdeviceptr weights = 0, rope = 0;
  uint64_t bytes = 0;
  int refs = 0;   // partition instances referencing them
};

struct Partition {
  int id = 0;
  int gpu = 0;
  bool live = true;
  Arena arena;
  CUdeviceptr sys = 0;     // small scratch (probe output)
  std::unique_ptr<Exec> cur;
  std::vector<std::unique_ptr<Exec>> draining;
  std::deque<Task*> fifo;       // placed, not yet launched (seq order)
  std::deque<Task*> inflight;   // launched, in order
  std::map<int, std::unique_ptr<FnInst>> insts;
  std::mutex load_mu;
  uint64_t launches = 0;
  std::atomic<int> inject_err{0};   // mx_debug_inject_error: next launched task reports it
};

struct Gpu {
  int idx = 0, ordinal = 0;
  CUdevice dev = 0;
  CUcontext primary = nullptr;
  int sm_total = 0, n_groups = 0, group_size = 8, remainder = 0, cc_major = 0, cc_minor = 0;
  uint64_t mem_bytes = 0;
  CUdevResource whole{};
  // A green context over the whole device: hosts the unpartitioned (N1) streams
  // and the clock calibration, so that no kernel of the library ever runs in
  // the primary context (an ncu launch list cannot follow a switch from a
  // primary-context kernel to a green-context one: "Failed to prepare kernel",
  // profiles/r2_ncu_green_ctx_probe.txt).
  CUgreenCtx whole_gctx = nullptr;
  CUcontext whole_ctx = nullptr;
  std::vector<CUdevResource> groups;
  int64_t clock_offset = 0;     // host_ns = device_ns + offset
  std::thread thr;
  std::mutex mu;                // guards partitions' queues / exec state on this GPU
  std::condition_variable cv;
  bool stop = false;
  std::vector<Partition*> parts;
  // Idle green contexts (+ stream + events) by SM-group set. Creating a green
  // context takes 1-200 ms on a busy device (measured), so part_resize and
  // part_destroy return execs here and make_exec reuses them.
  std::mutex pool_mu;
  std::multimap<uint64_t, std::unique_ptr<Exec>> exec_pool;
  // Shared read-only weight pool (MX_FN_SHARED_WEIGHTS, N3): one VMM arena per
  // GPU, created on first use, quota = device memory; fn id -> its weights.
  std::mutex wpool_mu;
  Arena wpool;
  bool wpool_ready = false;
  std::map<int, SharedWeights> shared_w;
};

}  // namespace mx
