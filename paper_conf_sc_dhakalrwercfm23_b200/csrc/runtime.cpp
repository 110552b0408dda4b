// Host runtime of the multiplexed small-function library and its C ABI.
//
// Paper mapping (PAPER.md, Dhakal et al. SC-W 2023):
//  * partitions = the MPS GPU% / MIG analog (§4.1, §4.2):
//    green contexts over 8-SM groups of one driver split + a VMM quota arena;
//  * one dispatcher thread per GPU replaces Parsl's HTEX pilot-job workers
//    (§2.2.1): per-partition FIFO, two tasks in flight per partition;
//  * placement decided at submit time from static costs (Fig. 4 P:195 "work
//    was divided equally"), so traces are deterministic;
//  * part_resize re-partitions live without reloading weights — the paper's
//    future work (§6 P:242 restart costs 10-20 s, §7).
#include "runtime.h"

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <set>

#include <cuda_runtime.h>

#include "drv.h"
#include "kernels/launch.cuh"

namespace mx {

// ---------------------------------------------------------------------------
// Utilities
// ---------------------------------------------------------------------------
uint64_t now_ns() {
  return (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
             std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

static thread_local char t_err[512] = "";

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(t_err, sizeof(t_err), fmt, ap);
  va_end(ap);
}

static const char* cu_str(CUresult r) {
  const char* s = nullptr;
  if (drv().cuGetErrorString) drv().cuGetErrorString(r, &s);
  return s ? s : "unknown CUDA error";
}

#define CU_TRY(call)                                                     \
  do {                                                                   \
    CUresult _r = (call);                                                \
    if (_r != CUDA_SUCCESS) {                                            \
      set_error("%s failed: %s (%d)", #call, cu_str(_r), (int)_r);       \
      return MX_EDEVICE;                                                 \
    }                                                                    \
  } while (0)

struct CtxGuard {
  bool pushed = false;
  explicit CtxGuard(CUcontext c) {
    if (c && drv().cuCtxPushCurrent(c) == CUDA_SUCCESS) pushed = true;
  }
  ~CtxGuard() {
    if (pushed) {
      CUcontext o;
      drv().cuCtxPopCurrent(&o);
    }
  }
};

static uint64_t align_up(uint64_t v, uint64_t a) { return (v + a - 1) / a * a; }

struct TimingRec {
  uint64_t task;
  int fn, gpu, part;
  uint64_t seq;
  uint32_t epoch;
  int status;
  uint64_t t_submit, t_start, t_end, kernel_ns;
};

struct Lib {
  std::mutex mu;
  std::condition_variable done_cv;
  std::vector<std::unique_ptr<Gpu>> gpus;
  std::unique_ptr<Sched> sched;
  std::vector<std::unique_ptr<Partition>> parts;
  std::vector<std::unique_ptr<Fn>> fns;
  std::map<uint64_t, std::unique_ptr<Task>> tasks;
  std::vector<TimingRec> timing;
};

static std::mutex g_init_mu;
static bool g_decode_prof = false;
static bool g_trace_resize = false;   // MX_TRACE_RESIZE=1: per-resize timing on stderr
static Lib* g_lib = nullptr;

// ---------------------------------------------------------------------------
// Shapes and costs — mirror of oracle/cost.py
// written independently from the same definitions.
// ---------------------------------------------------------------------------
static uint64_t decode_layer_weight_bytes(const mx_decode_cfg& c) {
  const uint64_t d = c.d_model, q = (uint64_t)c.n_heads * c.head_dim,
                 kv = (uint64_t)c.n_kv_heads * c.head_dim, ff = c.d_ff;
  return 2 * (d * q + 2 * d * kv + q * d + 3 * d * ff) + 2 * (2 * d);
}

static uint64_t decode_task_bytes(const mx_decode_cfg& c, uint64_t B, uint64_t P, uint64_t G) {
  const uint64_t S = P + G - 1, L = c.n_layers;
  const uint64_t kvpos = L * 2 * ((uint64_t)c.n_kv_heads * c.head_dim) * 2;
  const uint64_t head = 2ull * c.vocab * c.d_model + 2ull * c.d_model;
  return S * L * decode_layer_weight_bytes(c) + G * head + S * B * 2 * (uint64_t)c.d_model +
         B * kvpos * (S * (S + 1) / 2) + S * B * kvpos;
}

// D_ub = distinct (atom, incident bond type) pairs: one 32-bit atom mask per
// bond type (molecules have <= 32 atoms, <= 4 bond types; validated first).
static uint64_t mpnn_mol_flops(int n, const mx_bond* e, int ne, uint64_t F, uint64_t T) {
  uint32_t mask[4] = {0, 0, 0, 0};
  for (int i = 0; i < ne; ++i) mask[e[i].bond & 3] |= (1u << e[i].u) | (1u << e[i].v);
  const uint64_t D = (uint64_t)(__builtin_popcount(mask[0]) + __builtin_popcount(mask[1]) +
                                __builtin_popcount(mask[2]) + __builtin_popcount(mask[3]));
  const uint64_t edir = 2ull * ne, nn = (uint64_t)n;
  return T * (2 * F * F * (nn + D) + edir * F + 2 * nn * F) + nn * F + 2 * F * F + 4 * F;
}

static uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

// ---------------------------------------------------------------------------
// Validation
// ---------------------------------------------------------------------------
static int validate_fn(const mx_fn_desc& d) {
  if (d.flags & ~(uint32_t)MX_FN_SHARED_WEIGHTS) {
    set_error("fn_register: unknown flags 0x%x", d.flags);
    return MX_EINVAL;
  }
  if (d.kind == MX_FN_MPNN_TRAIN && (d.flags & MX_FN_SHARED_WEIGHTS)) {
    set_error("fn_register: a training function's parameters are per-instance state");
    return MX_EINVAL;
  }
  if (d.kind == MX_FN_DECODE) {
    const mx_decode_cfg& c = d.dec;
    const int q = c.n_heads * c.head_dim;
    if (c.n_layers < 1 || c.d_model < 8 || c.n_heads < 1 || c.n_kv_heads < 1 || c.d_ff < 8 ||
        c.vocab < 2 || c.max_seq < 2) {
      set_error("decode cfg: non-positive dimension");
      return MX_EINVAL;
    }
    if (c.head_dim != 32 && c.head_dim != 64 && c.head_dim != 128) {
      set_error("decode cfg: head_dim must be 32, 64 or 128");
      return MX_EINVAL;
    }
    if (c.d_model % 8 || q % 8 || c.d_ff % 8 || c.n_heads % c.n_kv_heads) {
      set_error("decode cfg: d_model, q_dim, d_ff must be multiples of 8; n_heads %% n_kv_heads == 0");
      return MX_EINVAL;
    }
    if (c.max_seq > mxk::kMaxSeqCap || c.max_batch < 1 || c.max_batch > 8) {
      set_error("decode cfg: max_seq <= %d and 1 <= max_batch <= 8", mxk::kMaxSeqCap);
      return MX_EINVAL;
    }
    if (c.d_model > 8192 || c.d_ff > 16384 || q > 16384 || c.vocab > (1 << 20)) {
      set_error("decode cfg: d_model <= 8192, q_dim and d_ff <= 16384, vocab <= 2^20");
      return MX_EINVAL;
    }
    const int kmax = std::max(std::max(c.d_model, q), c.d_ff);
    if (mxk::decode_smem_bytes(c.max_batch, kmax, nullptr) < 0) {
      set_error("decode cfg: shared-memory plan does not fit (max_batch %d, K %d)", c.max_batch,
                kmax);
      return MX_EINVAL;
    }
    if (!(c.rms_eps >= 0.f) || !(c.rope_theta > 0.f)) {
      set_error("decode cfg: bad eps/theta");
      return MX_EINVAL;
    }
    return MX_OK;
  }
  if (d.kind == MX_FN_MPNN || d.kind == MX_FN_MPNN_TRAIN) {
    const mx_mpnn_cfg& m = d.mpnn;
    if (m.hidden != 128 || m.steps < 1 || m.n_bond_types < 1 || m.n_bond_types > 4 ||
        m.n_atom_types < 1 || m.n_atom_types > 256 || m.max_mols < 1 || m.max_atoms < 1 ||
        m.max_edges < 0) {
      set_error("mpnn cfg: hidden must be 128, bond types 1..4, atom types 1..256");
      return MX_EINVAL;
    }
    return MX_OK;
  }
  set_error("unknown fn kind %d", d.kind);
  return MX_EINVAL;
}

static int validate_task(const mx_fn_desc& d, const mx_task_desc& t) {
  if (d.kind == MX_FN_DECODE) {
    const mx_decode_cfg& c = d.dec;
    if (t.batch < 1 || t.batch > c.max_batch || t.prompt_len < 1 || t.gen_len < 1 ||
        t.prompt_len + t.gen_len - 1 > c.max_seq || !t.prompt || !t.out_tokens) {
      set_error("decode task: need 1<=batch<=max_batch, P>=1, G>=1, P+G-1<=max_seq, buffers");
      return MX_EINVAL;
    }
    for (int i = 0; i < t.batch * t.prompt_len; ++i)
      if (t.prompt[i] < 0 || t.prompt[i] >= c.vocab) {
        set_error("decode task: prompt token %d out of range", t.prompt[i]);
        return MX_EINVAL;
      }
    return MX_OK;
  }
  const mx_mpnn_cfg& m = d.mpnn;
  if (t.n_mol < 1 || t.n_mol > m.max_mols || !t.atom_off || !t.atom_type || !t.edge_off ||
      (t.n_edges > 0 && !t.edges) || !t.out_ip) {
    set_error("mpnn task: bad sizes or null buffers");
    return MX_EINVAL;
  }
  if (d.kind == MX_FN_MPNN_TRAIN && (!t.targets || !t.out_loss || !(t.lr == t.lr))) {
    set_error("mpnn training task: needs targets, out_loss and a finite lr");
    return MX_EINVAL;
  }
  if (t.atom_off[0] != 0 || t.edge_off[0] != 0 || t.atom_off[t.n_mol] != t.n_atoms ||
      t.edge_off[t.n_mol] != t.n_edges || t.n_atoms > m.max_atoms || t.n_edges > m.max_edges) {
    set_error("mpnn task: CSR offsets inconsistent or over the fn's max sizes");
    return MX_EINVAL;
  }
  for (int i = 0; i < t.n_mol; ++i) {
    const int n = t.atom_off[i + 1] - t.atom_off[i], ne = t.edge_off[i + 1] - t.edge_off[i];
    if (n < 1 || n > 32 || ne < 0 || ne > 64) {
      set_error("mpnn task: molecule %d has %d atoms / %d bonds (limits 1..32, 0..64)", i, n, ne);
      return MX_EINVAL;
    }
    for (int e = t.edge_off[i]; e < t.edge_off[i + 1]; ++e) {
      const mx_bond& b = t.edges[e];
      if (b.u < 0 || b.u >= n || b.v < 0 || b.v >= n || b.bond >= m.n_bond_types) {
        set_error("mpnn task: bond %d of molecule %d out of range", e, i);
        return MX_EINVAL;
      }
      if (b.u == b.v) {   // reading R12: a bond joins two distinct atoms
        set_error("mpnn task: bond %d of molecule %d is a self-loop", e, i);
        return MX_EINVAL;
      }
    }
  }
  for (int i = 0; i < t.n_atoms; ++i)
    if (t.atom_type[i] >= m.n_atom_types) {
      set_error("mpnn task: atom type out of range");
      return MX_EINVAL;
    }
  return MX_OK;
}

static uint64_t default_cost(const mx_fn_desc& d, const mx_task_desc& t) {
  if (d.kind == MX_FN_DECODE)
    return ceil_div(decode_task_bytes(d.dec, t.batch, t.prompt_len, t.gen_len), 8000);
  uint64_t fl = 0;
  for (int i = 0; i < t.n_mol; ++i) {
    const int n = t.atom_off[i + 1] - t.atom_off[i];
    const int ne = t.edge_off[i + 1] - t.edge_off[i];
    fl += mpnn_mol_flops(n, t.edges + t.edge_off[i], ne, (uint64_t)d.mpnn.hidden,
                         (uint64_t)d.mpnn.steps);
  }
  // training: forward + backward ~ 3x the forward contractions (N4)
  return ceil_div(d.kind == MX_FN_MPNN_TRAIN ? 3 * fl : fl, 75000);
}

// ---------------------------------------------------------------------------
// Exec (green context + stream)
// ---------------------------------------------------------------------------
static void destroy_exec(Exec* e) {
  if (!e) return;
  if (e->ctx) {
    CtxGuard g(e->ctx);
    for (auto& lane : e->ev)
      for (auto& ev : lane)
        if (ev) drv().cuEventDestroy(ev);
  }
  if (e->stream) drv().cuStreamDestroy(e->stream);
  if (e->gctx) drv().cuGreenCtxDestroy(e->gctx);
}

// Unpartitioned exec (N1): a non-blocking stream of the GPU's whole-device
// green context (every shared partition's stream lives in that one context,
// like N processes' streams under the default MPS server).
static int make_shared_exec(Gpu& gpu, int n_ctas, uint32_t epoch, std::unique_ptr<Exec>* out) {
  auto e = std::make_unique<Exec>();
  e->epoch = epoch;
  e->shared = true;
  e->ctx = gpu.whole_ctx;
  e->n_ctas = n_ctas < gpu.sm_total ? n_ctas : gpu.sm_total;
  CtxGuard g(gpu.whole_ctx);
  CU_TRY(drv().cuGreenCtxStreamCreate(&e->stream, gpu.whole_gctx, CU_STREAM_NON_BLOCKING, 0));
  for (auto& lane : e->ev)
    for (auto& ev : lane)
      if (drv().cuEventCreate(&ev, CU_EVENT_DEFAULT) != CUDA_SUCCESS) {
        set_error("cuEventCreate failed");
        return MX_EDEVICE;
      }
  *out = std::move(e);
  return MX_OK;
}

static uint64_t exec_key(const std::vector<int>& groups, bool whole) {
  uint64_t m = whole ? (1ull << 63) : 0ull;
  for (int g : groups) m |= 1ull << g;
  return m;
}

// Return an idle green-context exec to the GPU's pool (shared execs are destroyed).
static void release_exec(Gpu& gpu, std::unique_ptr<Exec> e) {
  if (!e) return;
  if (e->shared || !e->gctx) {
    destroy_exec(e.get());
    return;
  }
  std::lock_guard<std::mutex> lk(gpu.pool_mu);
  const uint64_t k = e->key;
  gpu.exec_pool.emplace(k, std::move(e));
}

static int make_exec(Gpu& gpu, const std::vector<int>& groups, bool whole, uint32_t epoch,
                     std::unique_ptr<Exec>* out) {
  const uint64_t key = exec_key(groups, whole);
  {
    std::lock_guard<std::mutex> lk(gpu.pool_mu);
    auto it = gpu.exec_pool.find(key);
    if (it != gpu.exec_pool.end()) {
      *out = std::move(it->second);
      gpu.exec_pool.erase(it);
      (*out)->epoch = epoch;
      (*out)->inflight = 0;
      return MX_OK;
    }
  }
  auto e = std::make_unique<Exec>();
  e->key = key;
  e->epoch = epoch;
  CUdevResourceDesc desc;
  if (whole) {
    CU_TRY(drv().cuDevResourceGenerateDesc(&desc, &gpu.whole, 1));
  } else {
    std::vector<CUdevResource> rs;
    for (int g : groups) rs.push_back(gpu.groups[g]);
    CU_TRY(drv().cuDevResourceGenerateDesc(&desc, rs.data(), (unsigned)rs.size()));
  }
  CU_TRY(drv().cuGreenCtxCreate(&e->gctx, desc, gpu.dev, CU_GREEN_CTX_DEFAULT_STREAM));
  CUdevResource res;
  if (drv().cuGreenCtxGetDevResource(e->gctx, &res, CU_DEV_RESOURCE_TYPE_SM) != CUDA_SUCCESS) {
    destroy_exec(e.get());
    set_error("cuGreenCtxGetDevResource failed");
    return MX_EDEVICE;
  }
  e->n_ctas = (int)res.sm.smCount;
  if (drv().cuGreenCtxStreamCreate(&e->stream, e->gctx, CU_STREAM_NON_BLOCKING, 0) != CUDA_SUCCESS ||
      drv().cuCtxFromGreenCtx(&e->ctx, e->gctx) != CUDA_SUCCESS) {
    destroy_exec(e.get());
    set_error("green context stream creation failed");
    return MX_EDEVICE;
  }
  {
    CtxGuard g(e->ctx);
    for (auto& lane : e->ev)
      for (auto& ev : lane)
        if (drv().cuEventCreate(&ev, CU_EVENT_DEFAULT) != CUDA_SUCCESS) {
          set_error("cuEventCreate in green context failed");
          return MX_EDEVICE;
        }
  }
  *out = std::move(e);
  return MX_OK;
}

// ---------------------------------------------------------------------------
// Function instances (cold start, a2)
// ---------------------------------------------------------------------------
static int alloc_ptr(Partition& p, uint64_t bytes, CUdeviceptr* out) {
  int rc = p.arena.alloc(bytes, 256, out);
  if (rc == MX_ENOMEM)
    set_error("partition %d: HBM quota %llu exceeded (used %llu, need %llu more)", p.id,
              (unsigned long long)p.arena.quota(), (unsigned long long)p.arena.used(),
              (unsigned long long)bytes);
  return rc;
}

// Pinned, portable, device-mapped host memory; *dev = its device address.
static int host_alloc(size_t bytes, void** out, CUdeviceptr* dev = nullptr) {
  if (bytes == 0) bytes = 64;
  if (drv().cuMemHostAlloc(out, bytes, CU_MEMHOSTALLOC_PORTABLE | CU_MEMHOSTALLOC_DEVICEMAP) !=
      CUDA_SUCCESS) {
    set_error("pinned host allocation of %zu bytes failed", bytes);
    return MX_ENOMEM;
  }
  memset(*out, 0, bytes);
  if (dev && drv().cuMemHostGetDevicePointer(dev, *out, 0) != CUDA_SUCCESS) {
    set_error("mapping pinned host memory into the device address space failed");
    return MX_EDEVICE;
  }
  return MX_OK;
}

static int decode_layout(FnInst& fi) {
  const mx_decode_cfg& c = fi.fn->desc.dec;
  const uint64_t A = 128;
  const uint64_t d = c.d_model, q = (uint64_t)c.n_heads * c.head_dim,
                 kv = (uint64_t)c.n_kv_heads * c.head_dim, ff = c.d_ff, V = c.vocab;
  fi.off_wqkv = 0;
  fi.off_wo = align_up((q + 2 * kv) * d, A);
  fi.off_wgate = align_up(fi.off_wo + d * q, A);
  fi.off_wup = align_up(fi.off_wgate + ff * d, A);
  fi.off_wdown = align_up(fi.off_wup + ff * d, A);
  fi.off_gattn = align_up(fi.off_wdown + d * ff, A);
  fi.off_gmlp = align_up(fi.off_gattn + d, A);
  fi.layer_stride = align_up(fi.off_gmlp + d, A);
  fi.off_gfinal = fi.layer_stride * (uint64_t)c.n_layers;
  fi.off_lm = align_up(fi.off_gfinal + d, A);
  fi.off_embed = align_up(fi.off_lm + V * d, A);
  fi.weight_bytes = align_up(fi.off_embed + V * d, A) * 2;
  return MX_OK;
}

static void mpnn_layout(FnInst& fi) {
  const mx_mpnn_cfg& m = fi.fn->desc.mpnn;
  const uint64_t F = m.hidden, A = 128;
  const uint64_t sizes[11] = {(uint64_t)m.n_atom_types * F, F * F, F * F, F * F, F * F, F * F, F,
                              F * F, F, F, 1};
  uint64_t off = 0;
  for (int i = 0; i < 11; ++i) {
    fi.m_off[i] = off;
    off = align_up(off + sizes[i], (i >= 1 && i <= 3) ? 1 : A);   // W_0..W_3 contiguous
  }
  fi.weight_bytes = align_up(off, A) * 2;
}

// (tensor id) -> (element offset, count, is_gain) for fills and read-back.
static bool tensor_span(const FnInst& fi, int tid, uint64_t* off, uint64_t* n, int* is_gain) {
  const mx_fn_desc& d = fi.fn->desc;
  *is_gain = 0;
  if (d.kind == MX_FN_MPNN || d.kind == MX_FN_MPNN_TRAIN) {
    const uint64_t F = d.mpnn.hidden;
    const uint64_t sizes[11] = {(uint64_t)d.mpnn.n_atom_types * F, F * F, F * F, F * F, F * F,
                                F * F, F, F * F, F, F, 1};
    if (tid < 0 || tid > 10) return false;
    if (tid >= 1 && tid <= 4 && tid - 1 >= d.mpnn.n_bond_types) return false;
    *off = fi.m_off[tid];
    *n = sizes[tid];
    return true;
  }
  const mx_decode_cfg& c = d.dec;
  const uint64_t dd = c.d_model, q = (uint64_t)c.n_heads * c.head_dim,
                 kv = (uint64_t)c.n_kv_heads * c.head_dim, ff = c.d_ff, V = c.vocab;
  const int L = c.n_layers;
  if (tid == 0) {
    *off = fi.off_embed;
    *n = V * dd;
    return true;
  }
  if (tid == 16 * (L + 1)) {
    *off = fi.off_gfinal;
    *n = dd;
    *is_gain = 1;
    return true;
  }
  if (tid == 16 * (L + 1) + 1) {
    *off = fi.off_lm;
    *n = V * dd;
    return true;
  }
  const int l = tid / 16 - 1, w = tid % 16;
  if (l < 0 || l >= L || w > 8) return false;
  const uint64_t base = fi.layer_stride * (uint64_t)l;
  switch (w) {
    case 0: *off = base + fi.off_wqkv; *n = q * dd; break;
    case 1: *off = base + fi.off_wqkv + q * dd; *n = kv * dd; break;
    case 2: *off = base + fi.off_wqkv + (q + kv) * dd; *n = kv * dd; break;
    case 3: *off = base + fi.off_wo; *n = dd * q; break;
    case 4: *off = base + fi.off_wgate; *n = ff * dd; break;
    case 5: *off = base + fi.off_wup; *n = ff * dd; break;
    case 6: *off = base + fi.off_wdown; *n = dd * ff; break;
    case 7: *off = base + fi.off_gattn; *n = dd; *is_gain = 1; break;
    case 8: *off = base + fi.off_gmlp; *n = dd; *is_gain = 1; break;
    default: return false;
  }
  return true;
}

static int alloc_decode_slot(Partition& p, FnInst& fi, Slot& s) {
  const mx_decode_cfg& c = fi.fn->desc.dec;
  const uint64_t B = c.max_batch, d = c.d_model, q = (uint64_t)c.n_heads * c.head_dim,
                 kv = (uint64_t)c.n_kv_heads * c.head_dim, ff = c.d_ff, V = c.vocab,
                 T = c.max_seq, L = c.n_layers;
  int rc;
  if ((rc = alloc_ptr(p, B * d * 4, &s.x))) return rc;
  if ((rc = alloc_ptr(p, B * (q + 2 * kv) * 4, &s.qkv))) return rc;
  if ((rc = alloc_ptr(p, B * q * 4, &s.o))) return rc;
  if ((rc = alloc_ptr(p, B * ff * 4, &s.a))) return rc;
  // operand images sized for the widest layout (16 operand rows, B > 4)
  if ((rc = alloc_ptr(p, mxk::decode_img_bytes(8, (int)d), &s.img_x))) return rc;
  if ((rc = alloc_ptr(p, mxk::decode_img_bytes(8, (int)q), &s.img_o))) return rc;
  if ((rc = alloc_ptr(p, mxk::decode_img_bytes(8, (int)ff), &s.img_a))) return rc;
  if ((rc = alloc_ptr(p, B * (d / 8) * 4, &s.ssq))) return rc;
  if ((rc = alloc_ptr(p, (uint64_t)mxk::kMaxCtas * B * 8, &s.cand))) return rc;
  // segment partials of multi-segment phases (any batch up to max_batch) and
  // the row-block arrival counters that finish them
  uint64_t kpart = 0;
  for (uint64_t b = 1; b <= B; ++b)
    kpart = std::max(kpart, mxk::decode_kpart_floats((int)b, (int)d, (int)q, (int)(q + 2 * kv),
                                                     (int)ff, (int)V, 0));
  if ((rc = alloc_ptr(p, std::max<uint64_t>(kpart, 64) * 4, &s.kpart))) return rc;
  if ((rc = alloc_ptr(p, (uint64_t)mxk::kMaxCtas * 8, &s.pflag))) return rc;
  if ((rc = alloc_ptr(p, L * B * kv * T * 2, &s.kc))) return rc;
  if ((rc = alloc_ptr(p, L * B * kv * T * 2, &s.vc))) return rc;
  if ((rc = alloc_ptr(p, B * T * 4, &s.prompt))) return rc;
  if ((rc = alloc_ptr(p, B * T * 4, &s.tokens))) return rc;
  if ((rc = alloc_ptr(p, T * B * V * 4, &s.logits))) return rc;
  if ((rc = alloc_ptr(p, 64, &s.bar))) return rc;
  if ((rc = alloc_ptr(p, 64, &s.stamps))) return rc;
  s.err = s.stamps + 16;
  s.h_in_bytes = B * T * 4;
  s.h_out_bytes = B * T * 4 + T * B * V * 4;
  if ((rc = host_alloc(s.h_in_bytes, &s.h_in, &s.d_in))) return rc;
  if ((rc = host_alloc(s.h_out_bytes, &s.h_out, &s.d_out))) return rc;
  if ((rc = host_alloc(64, reinterpret_cast<void**>(&s.h_stamps), &s.d_stamps))) return rc;
  return MX_OK;
}

// Byte layout of a MPNN task's packed inputs (Task::blob, Slot::in_blob).
static size_t mpnn_blob_layout(Task& t, bool train, int n_mol, int n_atoms, int n_edges) {
  const size_t offs = align_up((uint64_t)(n_mol + 1) * 4, 64);
  t.off_ao = 0;
  t.off_eo = (uint32_t)offs;
  t.off_tile = (uint32_t)(2 * offs);
  t.off_tg = (uint32_t)(3 * offs);
  t.off_at = (uint32_t)(t.off_tg + (train ? align_up((uint64_t)n_mol * 4, 64) : 0));
  t.off_ed = (uint32_t)(t.off_at + align_up((uint64_t)n_atoms, 64));
  return t.off_ed + align_up((uint64_t)n_edges * 6, 64);
}

static int alloc_mpnn_slot(Partition& p, FnInst& fi, Slot& s) {
  const mx_mpnn_cfg& m = fi.fn->desc.mpnn;
  const bool train = fi.fn->desc.kind == MX_FN_MPNN_TRAIN;
  const uint64_t M = m.max_mols;
  int rc;
  Task probe;
  s.h_in_bytes = mpnn_blob_layout(probe, train, m.max_mols, m.max_atoms, std::max(1, m.max_edges));
  if ((rc = alloc_ptr(p, s.h_in_bytes, &s.in_blob))) return rc;
  if ((rc = alloc_ptr(p, 64, &s.stamps))) return rc;
  s.err = s.stamps + 16;
  s.h_out_bytes = M * 4;
  if (train) {
    // training tiles hold >= 4 molecules (<= 32 atoms each) except the last
    const uint64_t tiles = (M + 3) / 4 + 1;
    if ((rc = alloc_ptr(p, M * 4, &s.y))) return rc;
    if ((rc = alloc_ptr(p, tiles * fi.n_params * 4, &s.partials))) return rc;
    if ((rc = alloc_ptr(p, tiles * mxk::mpnn_train_tile_scratch_floats(m.steps) * 4, &s.hsave)))
      return rc;
    if ((rc = alloc_ptr(p, mxk::mpnn_train_img_bytes(), &s.wimg))) return rc;
    s.h_out_bytes = (M + 1) * 4;
  }
  if ((rc = host_alloc(s.h_in_bytes, &s.h_in, &s.d_in))) return rc;
  if ((rc = host_alloc(s.h_out_bytes, &s.h_out, &s.d_out))) return rc;
  if ((rc = host_alloc(64, reinterpret_cast<void**>(&s.h_stamps), &s.d_stamps))) return rc;
  return MX_OK;
}

// Seeded bf16 weights (C1) and the RoPE table, generated on device into the
// instance's weight block (enqueued on `st`, grid of `nct` CTAs).
static int generate_weights(FnInst& fi, CUstream st, int nct) {
  const mx_fn_desc& d = fi.fn->desc;
  uint16_t* w = reinterpret_cast<uint16_t*>(fi.weights);
  std::vector<int> tids;
  if (d.kind == MX_FN_DECODE) {
    const int L = d.dec.n_layers;
    tids.push_back(0);
    for (int l = 0; l < L; ++l)
      for (int k = 0; k <= 8; ++k) tids.push_back(16 * (l + 1) + k);
    tids.push_back(16 * (L + 1));
    tids.push_back(16 * (L + 1) + 1);
  } else {
    for (int k = 0; k <= 10; ++k)
      if (!(k >= 1 && k <= 4 && k - 1 >= d.mpnn.n_bond_types)) tids.push_back(k);
  }
  // alignment padding between tensors reads as 0 (decode TMA boxes may touch it)
  if (drv().cuMemsetD8Async(fi.weights, 0, fi.weight_bytes, st) != CUDA_SUCCESS) {
    set_error("weight block clear failed");
    return MX_EDEVICE;
  }
  for (int tid : tids) {
    uint64_t off, n;
    int gain;
    if (!tensor_span(fi, tid, &off, &n, &gain)) continue;
    if (mxk::launch_fill_weights(w + off, n, d.weight_seed, (uint32_t)tid, gain, nct, st)) {
      set_error("weight fill launch failed");
      return MX_EDEVICE;
    }
  }
  if (d.kind == MX_FN_DECODE) {
    if (mxk::launch_rope_table(reinterpret_cast<float*>(fi.rope), d.dec.max_seq, d.dec.head_dim,
                               d.dec.rope_theta, st)) {
      set_error("rope table launch failed");
      return MX_EDEVICE;
    }
  }
  return MX_OK;
}

static void free_slot_host(Slot& s) {
  if (s.h_in) drv().cuMemFreeHost(s.h_in);
  if (s.h_out) drv().cuMemFreeHost(s.h_out);
  if (s.h_stamps) drv().cuMemFreeHost(s.h_stamps);
  s.h_in = s.h_out = nullptr;
  s.h_stamps = nullptr;
}

// Drop one partition instance's reference to shared weights (N3); once no
// instance on the GPU references any shared weights, the pool is unmapped.
static void release_shared_ref(Gpu& gpu, int fn_id) {
  std::lock_guard<std::mutex> wl(gpu.wpool_mu);
  auto it = gpu.shared_w.find(fn_id);
  if (it == gpu.shared_w.end()) return;
  it->second.refs--;
  for (auto& kv : gpu.shared_w)
    if (kv.second.refs > 0) return;
  if (gpu.wpool_ready) gpu.wpool.release();
  gpu.wpool_ready = false;
  gpu.shared_w.clear();
}

// 4-D tiled TMA descriptors of a decode instance's weights (kernels.h
// kDecodeMaps): per matrix kind (QKV, O, GATE, UP, DOWN, LM) and per box
// height h = 8, 16, ..., 128 rows, the tensor {64 columns, R rows,
// ceil(K/64) column blocks, L layers} bf16 with strides {2K, 128, layer
// block} bytes and a box of {64, h, decode_box_blocks(h), 1}: one request
// fetches h rows x (blocks x 128 B) contiguous bytes per row, landing as
// [blocks][h rows][128 B] in K-major SWIZZLE_128B (the UMMA A-operand layout).
// Rows >= R and blocks >= ceil(K/64) are zero-filled; a last block that is
// partly past K reads the following (finite, zero-padded) weight elements,
// which meet zero activations.
static int encode_decode_maps(const FnInst& fi, std::vector<CUtensorMap>& maps) {
  const mx_decode_cfg& c = fi.fn->desc.dec;
  const uint64_t d = c.d_model, q = (uint64_t)c.n_heads * c.head_dim,
                 kv = (uint64_t)c.n_kv_heads * c.head_dim, ff = c.d_ff, V = c.vocab;
  struct Mat {
    uint64_t off, K, R;
    bool layered;
  } mats[mxk::kDecodeMats] = {{fi.off_wqkv, d, q + 2 * kv, true}, {fi.off_wo, q, d, true},
                              {fi.off_wgate, d, ff, true},         {fi.off_wup, d, ff, true},
                              {fi.off_wdown, ff, d, true},         {fi.off_lm, d, V, false}};
  maps.resize(mxk::kDecodeMaps);
  uint16_t* w = reinterpret_cast<uint16_t*>(fi.weights);
  for (int m = 0; m < mxk::kDecodeMats; ++m) {
    const Mat& M = mats[m];
    const cuuint64_t dims[4] = {(cuuint64_t)mxk::kBlkK, M.R, (M.K + mxk::kBlkK - 1) / mxk::kBlkK,
                                M.layered ? (cuuint64_t)c.n_layers : 1};
    const cuuint64_t strides[3] = {M.K * 2, 128,
                                   M.layered ? fi.layer_stride * 2 : align_up(M.K * M.R * 2, 256)};
    const cuuint32_t estr[4] = {1, 1, 1, 1};
    for (int h = 0; h < mxk::kDecodeBoxH; ++h) {
      const int rows = 8 * (h + 1);
      const cuuint32_t box[4] = {(cuuint32_t)mxk::kBlkK, (cuuint32_t)rows,
                                 (cuuint32_t)mxk::decode_box_blocks(rows), 1};
      CUresult r = drv().cuTensorMapEncodeTiled(
          &maps[m * mxk::kDecodeBoxH + h], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, w + M.off, dims,
          strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
          CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) {
        set_error("cuTensorMapEncodeTiled (matrix %d, box %d rows) failed: %s", m, rows,
                  cu_str(r));
        return MX_EDEVICE;
      }
    }
  }
  return MX_OK;
}

// Caller holds p.load_mu (part_resize / part_destroy take it too, so p.cur and
// its stream stay fixed while the load runs). Synchronous cold start on the
// partition's stream.
static int load_instance(Gpu& gpu, Partition& p, Fn& fn, FnInst** out) {
  auto it = p.insts.find(fn.id);
  if (it != p.insts.end() && it->second->loaded) {
    *out = it->second.get();
    return MX_OK;
  }
  CtxGuard cg(gpu.primary);
  auto fi = std::make_unique<FnInst>();
  fi->fn = &fn;
  fi->part = &p;
  const mx_fn_desc& d = fn.desc;
  if (d.kind == MX_FN_DECODE)
    decode_layout(*fi);
  else
    mpnn_layout(*fi);
  int rc = MX_OK;
  CUstream st = p.cur->stream;
  const int nct = p.cur->n_ctas;
  if (d.flags & MX_FN_SHARED_WEIGHTS) {
    // N3: one copy per GPU in the read-only weight pool, generated by the first
    // load on this GPU (on the loading partition's SMs) and referenced after.
    std::lock_guard<std::mutex> wl(gpu.wpool_mu);
    SharedWeights& sw = gpu.shared_w[fn.id];
    if (!sw.weights) {
      if (!gpu.wpool_ready) {
        if ((rc = gpu.wpool.init(gpu.ordinal, gpu.mem_bytes, gpu.mem_bytes))) {
          set_error("shared weight pool reservation failed");
          return rc;
        }
        gpu.wpool_ready = true;
      }
      CUdeviceptr w = 0, rope = 0;
      rc = gpu.wpool.alloc(fi->weight_bytes, 256, &w);
      if (!rc && d.kind == MX_FN_DECODE)
        rc = gpu.wpool.alloc((uint64_t)d.dec.max_seq * d.dec.head_dim * 4, 256, &rope);
      if (rc) {
        set_error("shared weight pool: device memory cannot back %llu more bytes",
                  (unsigned long long)fi->weight_bytes);
        return rc;
      }
      fi->weights = w;
      fi->rope = rope;
      if ((rc = generate_weights(*fi, st, nct))) return rc;
      CU_TRY(drv().cuStreamSynchronize(st));
      sw.weights = w;
      sw.rope = rope;
      sw.bytes = fi->weight_bytes;
    }
    fi->weights = sw.weights;
    fi->rope = sw.rope;
    fi->shared_weights = true;
    ++sw.refs;
  } else {
    if ((rc = alloc_ptr(p, fi->weight_bytes, &fi->weights))) return rc;
    if (d.kind == MX_FN_MPNN_TRAIN) {
      fi->n_params = fi->weight_bytes / 2;
      if ((rc = alloc_ptr(p, fi->n_params * 4, &fi->params))) return rc;
    }
    if (d.kind == MX_FN_DECODE) {
      const mx_decode_cfg& c = d.dec;
      if ((rc = alloc_ptr(p, (uint64_t)c.max_seq * c.head_dim * 4, &fi->rope))) return rc;
    }
  }
  // from here on a failure releases the pinned host staging already allocated
  // (arena bytes stay used: bump allocator; reported by part_query)
  auto fail = [&](int code) {
    for (Slot& s : fi->slots) free_slot_host(s);
    if (fi->shared_weights) {
      std::lock_guard<std::mutex> wl(gpu.wpool_mu);
      gpu.shared_w[fn.id].refs--;
    }
    return code;
  };
  for (Slot& s : fi->slots) {
    rc = (d.kind == MX_FN_DECODE) ? alloc_decode_slot(p, *fi, s) : alloc_mpnn_slot(p, *fi, s);
    if (rc) return fail(rc);
  }
  if (!fi->shared_weights && (rc = generate_weights(*fi, st, nct))) return fail(rc);
  std::vector<CUtensorMap> maps;
  if (d.kind == MX_FN_DECODE) {
    if ((rc = encode_decode_maps(*fi, maps))) return fail(rc);
    const uint64_t mb = maps.size() * sizeof(CUtensorMap);
    if ((rc = alloc_ptr(p, mb, &fi->tmaps))) return fail(rc);
    if (drv().cuMemcpyHtoDAsync(fi->tmaps, maps.data(), mb, st) != CUDA_SUCCESS) {
      set_error("tensor map upload failed");
      return fail(MX_EDEVICE);
    }
  }
  if (d.kind == MX_FN_MPNN_TRAIN) {
    // fp32 training state, widened exactly from the seeded bf16 values (N4)
    if (mxk::launch_widen_bf16(reinterpret_cast<float*>(fi->params),
                               reinterpret_cast<const uint16_t*>(fi->weights), fi->n_params, nct,
                               st)) {
      set_error("parameter widening launch failed");
      return fail(MX_EDEVICE);
    }
  }
  for (Slot& s : fi->slots) {
    if ((s.bar && drv().cuMemsetD8Async(s.bar, 0, 64, st) != CUDA_SUCCESS) ||
        drv().cuMemsetD8Async(s.stamps, 0, 64, st) != CUDA_SUCCESS) {
      set_error("slot reset failed");
      return fail(MX_EDEVICE);
    }
    if (d.kind == MX_FN_DECODE) {
      // operand images: columns past the input width and rows of absent
      // sequences are never written by the kernel and must read as zero
      const mx_decode_cfg& c = d.dec;
      const int q = c.n_heads * c.head_dim;
      if (drv().cuMemsetD8Async(s.pflag, 0, (size_t)mxk::kMaxCtas * 8, st) != CUDA_SUCCESS ||
          drv().cuMemsetD8Async(s.img_x, 0, mxk::decode_img_bytes(8, c.d_model), st) != CUDA_SUCCESS ||
          drv().cuMemsetD8Async(s.img_o, 0, mxk::decode_img_bytes(8, q), st) != CUDA_SUCCESS ||
          drv().cuMemsetD8Async(s.img_a, 0, mxk::decode_img_bytes(8, c.d_ff), st) != CUDA_SUCCESS) {
        set_error("slot reset failed");
        return fail(MX_EDEVICE);
      }
    }
  }
  if (drv().cuStreamSynchronize(st) != CUDA_SUCCESS) {
    set_error("cold start on partition %d failed on the device", p.id);
    return fail(MX_EDEVICE);
  }
  fi->loaded = true;
  *out = fi.get();
  p.insts[fn.id] = std::move(fi);
  return MX_OK;
}

// ---------------------------------------------------------------------------
// Dispatcher
// ---------------------------------------------------------------------------

// Inference tiling for a partition of n_ctas CTAs: the 128-atom next-fit
// packing, unless its last round of tiles would leave CTAs idle — then the
// smallest atom cap (start + 2k, < 128) whose packing has at most
// rounds * n_ctas tiles, so every CTA of the last round gets a (smaller) tile.
// Next-fit tile counts do not increase with the cap, so a binary search finds
// the same cap as a linear scan. Results are per molecule and do not depend on
// the tiling (tested bit-identical across partition sizes).
static int balanced_tiles(const int* ao, const int* eo, int n_mol, int n_ctas, int* tile_off) {
  const int nt = mxk::mpnn_pack_tiles(ao, eo, n_mol, tile_off);
  if (n_ctas <= 0) return nt;
  const int rounds = (nt + n_ctas - 1) / n_ctas;
  const int want = std::min(rounds * n_ctas, n_mol);
  if (nt >= want) return nt;
  const int total = ao[n_mol] - ao[0];
  const int start = std::max(1, (total + want - 1) / want);
  const int K = start < 128 ? (128 - start + 1) / 2 : 0;
  int lo = 0, hi = K;
  while (lo < hi) {
    const int mid = (lo + hi) / 2;
    if (mxk::mpnn_pack_tiles_cap(ao, eo, n_mol, start + 2 * mid, tile_off) <= want)
      hi = mid;
    else
      lo = mid + 1;
  }
  if (lo < K) return mxk::mpnn_pack_tiles_cap(ao, eo, n_mol, start + 2 * lo, tile_off);
  return mxk::mpnn_pack_tiles(ao, eo, n_mol, tile_off);
}

static int launch_task(Gpu& gpu, Partition& p, Task* t) {
  Exec* e = p.cur.get();
  t->exec = e;
  t->lane = (int)(p.launches++ & 1);
  FnInst* fi = t->inst;
  int si = fi->slots[0].busy ? 1 : 0;
  Slot& s = fi->slots[si];
  s.busy = true;
  t->slot = si;
  CUstream st = e->stream;
  CUevent* ev = e->ev[t->lane];
  if (s.need_reset) {
    if (s.bar) CU_TRY(drv().cuMemsetD8Async(s.bar, 0, 8, st));
    if (s.pflag) CU_TRY(drv().cuMemsetD8Async(s.pflag, 0, (size_t)mxk::kMaxCtas * 8, st));
    CU_TRY(drv().cuMemsetD8Async(s.stamps, 0, 64, st));
    s.bar_count = 0;
    s.need_reset = false;
  }
  const mx_fn_desc& d = fi->fn->desc;
  const int inject = p.inject_err.exchange(0);
  // Completion: the kernel writes its results and a done tag into host-mapped
  // memory, so a task is ONE kernel launch in the stream with nothing queued
  // behind it (copies / event records after a kernel would block unrelated
  // partitions' streams that share its hardware channel). Parity mode
  // (logits requested) keeps a D2H copy and an event.
  t->use_flag = !(t->kind == MX_FN_DECODE && t->out_logits);
  t->polls = 0;
  volatile uint64_t* hst = s.h_stamps;
  hst[3] = 0;
  if (t->kind == MX_FN_DECODE) {
    const mx_decode_cfg& c = d.dec;
    const size_t pb = (size_t)t->B * t->P * 4;
    memcpy(s.h_in, t->prompt.data(), pb);   // read by the kernel through the mapping
    mxk::DecodeParams k{};
    k.L = c.n_layers;
    k.d = c.d_model;
    k.H = c.n_heads;
    k.Hkv = c.n_kv_heads;
    k.hd = c.head_dim;
    k.ff = c.d_ff;
    k.V = c.vocab;
    k.q_dim = c.n_heads * c.head_dim;
    k.kv_dim = c.n_kv_heads * c.head_dim;
    k.qkv_rows = k.q_dim + 2 * k.kv_dim;
    k.max_seq = c.max_seq;
    k.B = t->B;
    k.P = t->P;
    k.G = t->G;
    k.eps = c.rms_eps;
    k.n_ctas = e->n_ctas;
    k.fuse_att = mxk::decode_fuse_attention(k.B, k.H, k.hd, k.n_ctas);
    const uint16_t* wb = reinterpret_cast<const uint16_t*>(fi->weights);
    k.w_layers = wb;
    k.layer_stride = fi->layer_stride;
    k.off_wqkv = fi->off_wqkv;
    k.off_wo = fi->off_wo;
    k.off_wgate = fi->off_wgate;
    k.off_wup = fi->off_wup;
    k.off_wdown = fi->off_wdown;
    k.off_gattn = fi->off_gattn;
    k.off_gmlp = fi->off_gmlp;
    k.g_final = wb + fi->off_gfinal;
    k.lm_head = wb + fi->off_lm;
    k.embed = wb + fi->off_embed;
    k.rope_cs = reinterpret_cast<const float*>(fi->rope);
    k.x = reinterpret_cast<float*>(s.x);
    k.qkv = reinterpret_cast<float*>(s.qkv);
    k.o = reinterpret_cast<float*>(s.o);
    k.a = reinterpret_cast<float*>(s.a);
    k.img_x = reinterpret_cast<uint8_t*>(s.img_x);
    k.img_o = reinterpret_cast<uint8_t*>(s.img_o);
    k.img_a = reinterpret_cast<uint8_t*>(s.img_a);
    k.ssq = reinterpret_cast<float*>(s.ssq);
    k.cand = reinterpret_cast<unsigned long long*>(s.cand);
    k.kpart = reinterpret_cast<float*>(s.kpart);
    k.pflag = reinterpret_cast<unsigned long long*>(s.pflag);
    k.kc = reinterpret_cast<uint16_t*>(s.kc);
    k.vc = reinterpret_cast<uint16_t*>(s.vc);
    k.prompt = reinterpret_cast<const int*>(s.d_in);
    k.tokens = reinterpret_cast<int*>(s.d_out);
    k.h_stamps = reinterpret_cast<unsigned long long*>(s.d_stamps);
    k.done_tag = t->id;
    k.inject_err = inject;
    k.logits = t->out_logits ? reinterpret_cast<float*>(s.logits) : nullptr;
    k.bar = reinterpret_cast<unsigned long long*>(s.bar);
    k.bar_base = s.bar_count;
    k.stamps = reinterpret_cast<unsigned long long*>(s.stamps);
    k.err = reinterpret_cast<int*>(s.err);
    k.prof = g_decode_prof ? reinterpret_cast<unsigned long long*>(p.sys + 65536) : nullptr;
    k.tmaps = reinterpret_cast<const void*>(fi->tmaps);
    if (!t->use_flag) CU_TRY(drv().cuEventRecord(ev[0], st));
    int rc = mxk::launch_decode(k, st, e->shared ? 1 : 0);
    if (rc) {
      set_error("decode launch failed (%d)", rc);
      return MX_EDEVICE;
    }
    s.bar_count += mxk::decode_barriers(k.L, k.P, k.G, k.fuse_att) * (uint64_t)k.n_ctas;
    if (!t->use_flag) {
      CU_TRY(drv().cuEventRecord(ev[1], st));
      CU_TRY(drv().cuMemcpyDtoHAsync(static_cast<uint8_t*>(s.h_out) + (size_t)t->B * c.max_seq * 4,
                                     s.logits, (size_t)t->G * t->B * c.vocab * 4, st));
    }
  } else {
    // the inputs were packed at submit in their device image: one H2D copy
    if (t->kind == MX_FN_MPNN && t->tile_ctas != e->n_ctas) {
      // the partition was resized after submit: re-balance the tiles for its CTA count
      const int* ao = reinterpret_cast<const int*>(t->blob.data() + t->off_ao);
      const int* eo = reinterpret_cast<const int*>(t->blob.data() + t->off_eo);
      t->n_tiles = balanced_tiles(ao, eo, t->n_mol, e->n_ctas,
                                  reinterpret_cast<int*>(t->blob.data() + t->off_tile));
      t->tile_ctas = e->n_ctas;
    }
    memcpy(s.h_in, t->blob.data(), t->blob.size());
    CU_TRY(drv().cuMemcpyHtoDAsync(s.in_blob, s.h_in, t->blob.size(), st));
    const int n_tiles = t->n_tiles;
    const mx_mpnn_cfg& m = d.mpnn;
    const uint16_t* wb = reinterpret_cast<const uint16_t*>(fi->weights);
    mxk::MpnnParams k{};
    k.F = m.hidden;
    k.T = m.steps;
    k.n_types = m.n_atom_types;
    k.n_bonds = m.n_bond_types;
    k.n_mol = t->n_mol;
    k.e_atom = wb + fi->m_off[0];
    k.w_b = wb + fi->m_off[1];
    k.u = wb + fi->m_off[5];
    k.c = wb + fi->m_off[6];
    k.w1 = wb + fi->m_off[7];
    k.c1 = wb + fi->m_off[8];
    k.w2 = wb + fi->m_off[9];
    k.c2 = wb + fi->m_off[10];
    k.atom_off = reinterpret_cast<const int*>(s.in_blob + t->off_ao);
    k.atom_type = reinterpret_cast<const uint8_t*>(s.in_blob + t->off_at);
    k.edge_off = reinterpret_cast<const int*>(s.in_blob + t->off_eo);
    k.edges = reinterpret_cast<const uint32_t*>(s.in_blob + t->off_ed);
    k.out = reinterpret_cast<float*>(s.d_out);
    k.stamps = reinterpret_cast<unsigned long long*>(s.stamps);
    k.h_stamps = reinterpret_cast<unsigned long long*>(s.d_stamps);
    k.done_tag = t->id;
    k.inject_err = inject;
    k.n_ctas = e->n_ctas;
    k.tile_off = reinterpret_cast<const int*>(s.in_blob + t->off_tile);
    k.n_tiles = n_tiles;
    if (t->kind == MX_FN_MPNN_TRAIN) {
      mxk::MpnnTrainParams q{};
      q.T = m.steps;
      q.n_bonds = m.n_bond_types;
      q.n_mol = t->n_mol;
      q.n_params = (int)fi->n_params;
      q.n_tiles = n_tiles;
      q.n_ctas = e->n_ctas;
      for (int i = 0; i < 11; ++i) q.off[i] = (uint32_t)fi->m_off[i];
      q.params = reinterpret_cast<float*>(fi->params);
      q.partials = reinterpret_cast<float*>(s.partials);
      q.hsave = reinterpret_cast<float*>(s.hsave);
      q.wimg = reinterpret_cast<uint8_t*>(s.wimg);
      q.atom_off = k.atom_off;
      q.atom_type = k.atom_type;
      q.edge_off = k.edge_off;
      q.edges = k.edges;
      q.tile_off = k.tile_off;
      q.targets = reinterpret_cast<const float*>(s.in_blob + t->off_tg);
      q.y = reinterpret_cast<float*>(s.y);
      q.out = reinterpret_cast<float*>(s.d_out);
      q.lr = t->lr;
      q.stamps = k.stamps;
      q.h_stamps = k.h_stamps;
      q.done_tag = t->id;
      q.inject_err = inject;
      if (mxk::launch_mpnn_train(q, st)) {
        set_error("mpnn training launch failed");
        return MX_EDEVICE;
      }
    } else if (mxk::launch_mpnn(k, st)) {
      set_error("mpnn launch failed");
      return MX_EDEVICE;
    }
  }
  if (!t->use_flag) {
    CU_TRY(drv().cuMemcpyDtoHAsync(s.h_stamps, s.stamps, 24, st));
    CU_TRY(drv().cuEventRecord(ev[2], st));
  }
  e->inflight++;
  return MX_OK;
}

static bool task_flag_seen(const Task* t) {
  const volatile uint64_t* st = t->inst->slots[t->slot].h_stamps;
  if (st[3] != t->id) return false;
  std::atomic_thread_fence(std::memory_order_acquire);
  return true;
}

static void finish_task(Gpu& gpu, Task* t, bool dev_ok) {
  Slot& s = t->inst->slots[t->slot];
  Exec* e = t->exec;
  const volatile uint64_t* st = s.h_stamps;
  float ms = 0.f;
  if (!t->use_flag) {
    if (dev_ok && drv().cuEventElapsedTime(&ms, e->ev[t->lane][0], e->ev[t->lane][1]) == CUDA_SUCCESS)
      t->kernel_ns = (uint64_t)((double)ms * 1e6);
  } else if (dev_ok && st[1] >= st[0]) {
    t->kernel_ns = st[1] - st[0];   // device %globaltimer span of the launch
  }
  const int err = dev_ok ? (int)(st[2] & 0xffffffffu) : 1;
  t->status = (!dev_ok || err) ? MX_EDEVICE : MX_OK;
  if (t->kind == MX_FN_DECODE) {
    memcpy(t->out_tokens, s.h_out, (size_t)t->B * t->G * 4);
    if (t->out_logits) {
      const mx_decode_cfg& c = t->inst->fn->desc.dec;
      memcpy(t->out_logits, static_cast<uint8_t*>(s.h_out) + (size_t)t->B * c.max_seq * 4,
             (size_t)t->G * t->B * c.vocab * 4);
    }
  } else {
    memcpy(t->out_ip, s.h_out, (size_t)t->n_mol * 4);
    if (t->kind == MX_FN_MPNN_TRAIN)
      memcpy(t->out_loss, static_cast<uint8_t*>(s.h_out) + (size_t)t->n_mol * 4, 4);
  }
  t->t_start = (uint64_t)((int64_t)st[0] + gpu.clock_offset);
  t->t_end = (uint64_t)((int64_t)st[1] + gpu.clock_offset);
  if (err || !dev_ok) s.need_reset = true;
  s.busy = false;
  e->inflight--;
}

// Tasks kept in flight per partition. Two (double-buffered task slots) hide
// the host reaction time between consecutive tasks, but every queued-behind
// kernel occupies its hardware channel: once a GPU has more partition streams
// than CUDA_DEVICE_MAX_CONNECTIONS (32) can give their own channel, a second
// queued task blocks the unrelated streams sharing that channel until the
// first one ends (measured: 37 partitions, busy fraction 0.78 -> one-task
// gaps). So more than kDeepPartsMax partitions per GPU run one task at a
// time (the host reaction, ~10s of us, is < 0.1% of a decode task).
// MX_INFLIGHT=1|2 overrides.
static constexpr size_t kDeepPartsMax = 16;
static size_t g_inflight_override = 0;

static size_t inflight_depth(const Gpu& gpu) {
  if (g_inflight_override) return g_inflight_override;
  size_t live = 0;
  for (const Partition* p : gpu.parts)
    if (p->live) ++live;
  return live > kDeepPartsMax ? 1 : 2;
}

static void dispatcher_main(Lib* L, Gpu* gpu) {
  drv().cuCtxSetCurrent(gpu->primary);
  std::vector<Task*> completed;
  for (;;) {
    completed.clear();
    bool any_inflight = false;
    {
      std::unique_lock<std::mutex> lk(gpu->mu);
      bool progress = false;
      const size_t depth = inflight_depth(*gpu);
      for (Partition* p : gpu->parts) {
        while (!p->inflight.empty()) {
          Task* t = p->inflight.front();
          bool ok = true;
          if (t->use_flag) {
            if (!task_flag_seen(t)) {
              // no flag yet: every 256th poll ask the driver whether the stream
              // faulted (or drained without the kernel signalling)
              if ((++t->polls & 255u) != 0) break;
              CUresult r = drv().cuStreamQuery(t->exec->stream);
              if (r == CUDA_ERROR_NOT_READY) break;
              if (r == CUDA_SUCCESS && !task_flag_seen(t)) {
                // the stream is idle only after the kernel ended: its flag must be there
                if ((t->polls >> 8) < 4) break;   // allow the PCIe write to land
                set_error("task %llu: kernel ended without its completion flag",
                          (unsigned long long)t->id);
              }
              ok = (r == CUDA_SUCCESS) && task_flag_seen(t);
            }
          } else {
            CUresult r = drv().cuEventQuery(t->exec->ev[t->lane][2]);
            if (r == CUDA_ERROR_NOT_READY) break;
            ok = (r == CUDA_SUCCESS);
          }
          finish_task(*gpu, t, ok);
          p->inflight.pop_front();
          completed.push_back(t);
          progress = true;
        }
        while (p->inflight.size() < depth && !p->fifo.empty() && p->fifo.front()->ready) {
          Task* t = p->fifo.front();
          p->fifo.pop_front();
          if (launch_task(*gpu, *p, t) != MX_OK) {
            t->status = MX_EDEVICE;
            if (t->slot >= 0) t->inst->slots[t->slot].busy = false;
            completed.push_back(t);
          } else {
            p->inflight.push_back(t);
          }
          progress = true;
        }
        for (size_t i = 0; i < p->draining.size();) {
          if (p->draining[i]->inflight == 0) {
            release_exec(*gpu, std::move(p->draining[i]));
            p->draining.erase(p->draining.begin() + i);
          } else {
            ++i;
          }
        }
        if (!p->inflight.empty()) any_inflight = true;
      }
      if (!progress) {
        bool queued = false;
        for (Partition* p : gpu->parts)
          if (!p->fifo.empty() && p->fifo.front()->ready) queued = true;
        if (gpu->stop && !any_inflight && !queued) break;
        if (!any_inflight && !queued)
          gpu->cv.wait_for(lk, std::chrono::milliseconds(2));
      }
    }
    if (!completed.empty()) {
      std::lock_guard<std::mutex> lk(L->mu);
      for (Task* t : completed) t->done = true;
      L->done_cv.notify_all();
    } else if (any_inflight) {
      std::this_thread::sleep_for(std::chrono::microseconds(5));
    }
  }
}

// ---------------------------------------------------------------------------
// Init / shutdown
// ---------------------------------------------------------------------------
static int calibrate_clock(Gpu& gpu) {
  CtxGuard cg(gpu.primary);
  CUstream st;
  CU_TRY(drv().cuGreenCtxStreamCreate(&st, gpu.whole_gctx, CU_STREAM_NON_BLOCKING, 0));
  CUdeviceptr dbuf = 0;
  Arena tmp;
  int rc = tmp.init(gpu.ordinal, 1 << 21, 1 << 21);
  if (rc) return rc;
  if ((rc = tmp.alloc(64, 64, &dbuf))) return rc;
  int64_t best_lat = INT64_MAX, best_off = 0;
  for (int i = 0; i < 8; ++i) {
    uint64_t h0 = now_ns();
    if (mxk::launch_clock(reinterpret_cast<unsigned long long*>(dbuf), st)) {
      set_error("clock kernel launch failed");
      return MX_EDEVICE;
    }
    CU_TRY(drv().cuStreamSynchronize(st));
    uint64_t h1 = now_ns();
    uint64_t dv = 0;
    CU_TRY(drv().cuMemcpyDtoH(&dv, dbuf, 8));
    const int64_t lat = (int64_t)(h1 - h0);
    if (lat < best_lat) {
      best_lat = lat;
      best_off = (int64_t)((h0 + h1) / 2) - (int64_t)dv;
    }
  }
  gpu.clock_offset = best_off;
  drv().cuStreamDestroy(st);
  tmp.release();
  return MX_OK;
}

static int init_gpu(Gpu& gpu) {
  CU_TRY(drv().cuDeviceGet(&gpu.dev, gpu.ordinal));
  CU_TRY(drv().cuDeviceGetAttribute(&gpu.cc_major, CU_DEVICE_ATTRIBUTE_COMPUTE_CAPABILITY_MAJOR, gpu.dev));
  CU_TRY(drv().cuDeviceGetAttribute(&gpu.cc_minor, CU_DEVICE_ATTRIBUTE_COMPUTE_CAPABILITY_MINOR, gpu.dev));
  if (gpu.cc_major != 10) {
    set_error("device %d is compute capability %d.%d; this library is built for sm_100a only",
              gpu.ordinal, gpu.cc_major, gpu.cc_minor);
    return MX_ENODEV;
  }
  CU_TRY(drv().cuDevicePrimaryCtxRetain(&gpu.primary, gpu.dev));
  CtxGuard cg(gpu.primary);
  size_t mem = 0;
  CU_TRY(drv().cuDeviceTotalMem(&mem, gpu.dev));
  gpu.mem_bytes = mem;
  CU_TRY(drv().cuDeviceGetDevResource(gpu.dev, &gpu.whole, CU_DEV_RESOURCE_TYPE_SM));
  gpu.sm_total = (int)gpu.whole.sm.smCount;
  // One split of the device into equal SM groups. The default (co-scheduling
  // aware) split of a B200 into 8-SM groups only yields 15 groups (120 SMs) plus
  // a 28-SM remainder, so by default the split ignores SM co-scheduling (none of
  // the kernels uses thread-block clusters) and uses 4-SM groups: 37 x 4 = 148.
  // MX_SM_GROUP=8 selects the co-scheduling-aware 8-SM split instead.
  int want = 4;
  if (const char* e = getenv("MX_SM_GROUP")) want = atoi(e);
  unsigned flags = (want == 8) ? 0u : (unsigned)CU_DEV_SM_RESOURCE_SPLIT_IGNORE_SM_COSCHEDULING;
  if (want < 1) want = 4;
  unsigned nb = 0;
  CUdevResource rem{};
  if (drv().cuDevSmResourceSplitByCount(nullptr, &nb, &gpu.whole, nullptr, flags, want) !=
          CUDA_SUCCESS ||
      nb == 0 || nb > 64) {
    flags = 0;
    want = 8;
    nb = 0;
    CU_TRY(drv().cuDevSmResourceSplitByCount(nullptr, &nb, &gpu.whole, nullptr, 0, 8));
  }
  gpu.groups.resize(nb);
  CU_TRY(drv().cuDevSmResourceSplitByCount(gpu.groups.data(), &nb, &gpu.whole, &rem, flags, want));
  gpu.groups.resize(nb);
  gpu.n_groups = (int)nb;
  if (nb == 0 || nb > 64) {
    set_error("unexpected SM split: %u groups", nb);
    return MX_EDEVICE;
  }
  gpu.group_size = (int)gpu.groups[0].sm.smCount;
  for (auto& g : gpu.groups)
    if ((int)g.sm.smCount != gpu.group_size) {
      set_error("non-uniform SM groups from cuDevSmResourceSplitByCount");
      return MX_EDEVICE;
    }
  gpu.remainder = gpu.sm_total - gpu.n_groups * gpu.group_size;
  {
    CUdevResourceDesc wd;
    CU_TRY(drv().cuDevResourceGenerateDesc(&wd, &gpu.whole, 1));
    CU_TRY(drv().cuGreenCtxCreate(&gpu.whole_gctx, wd, gpu.dev, CU_GREEN_CTX_DEFAULT_STREAM));
    CU_TRY(drv().cuCtxFromGreenCtx(&gpu.whole_ctx, gpu.whole_gctx));
  }
  if (mxk::decode_set_attrs(gpu.dev) || mxk::mpnn_set_attrs(gpu.dev) ||
      mxk::mpnn_train_set_attrs(gpu.dev)) {
    set_error("setting kernel shared-memory attributes failed");
    return MX_EDEVICE;
  }
  return calibrate_clock(gpu);
}

static int init_impl(const std::vector<int>& ordinals) {
  std::lock_guard<std::mutex> lk(g_init_mu);
  if (g_lib) return MX_OK;
  setenv("CUDA_DEVICE_MAX_CONNECTIONS", "32", 0);
  g_decode_prof = getenv("MX_DECODE_PROF") && atoi(getenv("MX_DECODE_PROF")) == 1;
  g_trace_resize = getenv("MX_TRACE_RESIZE") && atoi(getenv("MX_TRACE_RESIZE")) == 1;
  if (g_decode_prof && !mxk::decode_prof_buckets())
    fprintf(stderr, "[mx] MX_DECODE_PROF=1 needs a build with MX_DEFS=-DMX_PROF_BUCKETS; "
                    "the cycle buckets will read 0\n");
  if (const char* e = getenv("MX_INFLIGHT")) {
    const int v = atoi(e);
    g_inflight_override = (v == 1 || v == 2) ? (size_t)v : 0;
  }
  const char* why = nullptr;
  if (!drv().load(&why)) {
    set_error("%s (no CUDA driver?)", why ? why : "driver load failed");
    return MX_ENODEV;
  }
  mxk::driver_launch().launch = drv().cuLaunchKernel;
  mxk::driver_launch().launch_coop = drv().cuLaunchCooperativeKernel;
  mxk::driver_launch().kernel_set_attr = drv().cuKernelSetAttribute;
  if (drv().cuInit(0) != CUDA_SUCCESS) {
    set_error("cuInit failed: no usable GPU");
    return MX_ENODEV;
  }
  int count = 0;
  if (drv().cuDeviceGetCount(&count) != CUDA_SUCCESS || count == 0) {
    set_error("no CUDA device visible");
    return MX_ENODEV;
  }
  std::vector<int> ords = ordinals;
  if (ords.empty())
    for (int i = 0; i < count; ++i) ords.push_back(i);
  auto L = std::make_unique<Lib>();
  for (int o : ords) {
    if (o < 0 || o >= count) {
      set_error("device ordinal %d out of range (%d visible)", o, count);
      return MX_ENODEV;
    }
    auto g = std::make_unique<Gpu>();
    g->idx = (int)L->gpus.size();
    g->ordinal = o;
    int rc = init_gpu(*g);
    if (rc) return rc;
    L->gpus.push_back(std::move(g));
  }
  int ng = INT32_MAX;
  uint64_t mem = UINT64_MAX;
  for (auto& g : L->gpus) {
    ng = std::min(ng, g->n_groups);
    mem = std::min(mem, g->mem_bytes);
  }
  L->sched = std::make_unique<Sched>((int)L->gpus.size(), ng, L->gpus[0]->group_size,
                                     L->gpus[0]->sm_total, mem);
  Lib* raw = L.release();
  for (auto& g : raw->gpus) g->thr = std::thread(dispatcher_main, raw, g.get());
  g_lib = raw;
  return MX_OK;
}

}  // namespace mx

// ===========================================================================
// C ABI
// ===========================================================================
using namespace mx;

#define MX_REQUIRE_INIT()                   \
  Lib* L = g_lib;                           \
  if (!L) {                                 \
    set_error("mx_init has not been called"); \
    return MX_ESTATE;                       \
  }

extern "C" {

mx_status mx_init(uint32_t flags) {
  (void)flags;
  try {
    return init_impl({});
  } catch (...) {
    set_error("exception in mx_init");
    return MX_EDEVICE;
  }
}

mx_status mx_init_devices(const int32_t* ordinals, int32_t n, uint32_t flags) {
  (void)flags;
  if (n < 0 || (n > 0 && !ordinals)) return MX_EINVAL;
  try {
    return init_impl(std::vector<int>(ordinals, ordinals + n));
  } catch (...) {
    set_error("exception in mx_init_devices");
    return MX_EDEVICE;
  }
}

mx_status mx_shutdown(void) {
  std::lock_guard<std::mutex> ilk(g_init_mu);
  Lib* L = g_lib;
  if (!L) return MX_OK;
  for (auto& g : L->gpus) {
    {
      std::lock_guard<std::mutex> lk(g->mu);
      g->stop = true;
    }
    g->cv.notify_all();
  }
  for (auto& g : L->gpus)
    if (g->thr.joinable()) g->thr.join();
  for (auto& p : L->parts) {
    if (!p->live) continue;
    CtxGuard cg(L->gpus[p->gpu]->primary);
    if (p->cur) drv().cuStreamSynchronize(p->cur->stream);
    for (auto& kv : p->insts)
      for (Slot& s : kv.second->slots) free_slot_host(s);
    for (auto& e : p->draining) destroy_exec(e.get());
    destroy_exec(p->cur.get());
    p->arena.release();
  }
  for (auto& g : L->gpus) {
    CtxGuard cg(g->primary);
    for (auto& kv : g->exec_pool) {
      drv().cuStreamSynchronize(kv.second->stream);
      destroy_exec(kv.second.get());
    }
    g->exec_pool.clear();
  }
  for (auto& g : L->gpus) {
    CtxGuard cg(g->primary);
    if (g->wpool_ready) g->wpool.release();
    g->shared_w.clear();
  }
  for (auto& g : L->gpus) {
    if (g->whole_gctx) drv().cuGreenCtxDestroy(g->whole_gctx);
    drv().cuDevicePrimaryCtxRelease(g->dev);
  }
  g_lib = nullptr;
  delete L;
  return MX_OK;
}

mx_status mx_gpu_count(int32_t* n) {
  MX_REQUIRE_INIT();
  if (!n) return MX_EINVAL;
  *n = (int32_t)L->gpus.size();
  return MX_OK;
}

mx_status mx_gpu_query(int32_t gpu, mx_gpu_info* out) {
  MX_REQUIRE_INIT();
  if (!out) return MX_EINVAL;
  if (gpu < 0 || gpu >= (int)L->gpus.size()) return MX_ENODEV;
  const Gpu& g = *L->gpus[gpu];
  out->ordinal = g.ordinal;
  out->sm_total = g.sm_total;
  out->n_groups = g.n_groups;
  out->group_size = g.group_size;
  out->remainder_sms = g.remainder;
  out->cc_major = g.cc_major;
  out->cc_minor = g.cc_minor;
  out->reserved = 0;
  out->mem_bytes = g.mem_bytes;
  return MX_OK;
}

const char* mx_strerror(mx_status s) {
  switch (s) {
    case MX_OK: return "ok";
    case MX_ENOENT: return "no such task (unknown or already collected)";
    case MX_EDEVICE: return "device error";
    case MX_ENOMEM: return "partition HBM quota or device memory exhausted";
    case MX_EBUSY: return "busy (pending work or quota below usage)";
    case MX_ENODEV: return "no such device / device not compute capability 10.x";
    case MX_EINVAL: return "invalid argument";
    case MX_ENOSM: return "not enough free SM groups";
    case MX_ETIMEDOUT: return "timed out";
    case MX_ESTATE: return "library not initialised";
    default: return "unknown status";
  }
}

const char* mx_last_error(void) { return t_err; }

mx_status part_create(int32_t gpu, int32_t sm_count, uint64_t hbm_bytes, int32_t* out_part) {
  MX_REQUIRE_INIT();
  if (!out_part) return MX_EINVAL;
  std::lock_guard<std::mutex> lk(L->mu);
  std::vector<int> groups;
  int smc = 0;
  bool whole = false;
  int rc = L->sched->plan_create(gpu, sm_count, hbm_bytes, &groups, &smc, &whole);
  if (rc) {
    set_error("part_create(gpu=%d, sm=%d, hbm=%llu): %s", gpu, sm_count,
              (unsigned long long)hbm_bytes, mx_strerror(rc));
    return rc;
  }
  Gpu& g = *L->gpus[gpu];
  CtxGuard cg(g.primary);
  auto p = std::make_unique<Partition>();
  p->gpu = gpu;
  rc = make_exec(g, groups, whole, 0, &p->cur);
  if (rc) return rc;
  rc = p->arena.init(g.ordinal, hbm_bytes, g.mem_bytes);
  if (rc) {
    destroy_exec(p->cur.get());
    set_error("arena reservation failed");
    return rc;
  }
  rc = p->arena.alloc(128 * 1024, 256, &p->sys);
  if (rc) {
    destroy_exec(p->cur.get());
    p->arena.release();
    set_error("partition quota below the 64 KiB system scratch");
    return MX_ENOMEM;
  }
  int id = -1;
  rc = L->sched->create(gpu, sm_count, hbm_bytes, &id);
  if (rc || id != (int)L->parts.size()) {
    destroy_exec(p->cur.get());
    p->arena.release();
    set_error("internal: scheduler/partition table mismatch");
    return rc ? rc : MX_EDEVICE;
  }
  p->id = id;
  Partition* raw = p.get();
  L->parts.push_back(std::move(p));
  {
    std::lock_guard<std::mutex> glk(g.mu);
    g.parts.push_back(raw);
  }
  *out_part = id;
  return MX_OK;
}

mx_status part_create_shared(int32_t gpu, int32_t n_ctas, uint64_t hbm_bytes, int32_t* out_part) {
  MX_REQUIRE_INIT();
  if (!out_part) return MX_EINVAL;
  std::lock_guard<std::mutex> lk(L->mu);
  int rc = L->sched->plan_create_shared(gpu, n_ctas, hbm_bytes);
  if (rc) {
    set_error("part_create_shared(gpu=%d, n_ctas=%d, hbm=%llu): %s", gpu, n_ctas,
              (unsigned long long)hbm_bytes, mx_strerror(rc));
    return rc;
  }
  Gpu& g = *L->gpus[gpu];
  CtxGuard cg(g.primary);
  auto p = std::make_unique<Partition>();
  p->gpu = gpu;
  rc = make_shared_exec(g, n_ctas, 0, &p->cur);
  if (rc) return rc;
  rc = p->arena.init(g.ordinal, hbm_bytes, g.mem_bytes);
  if (rc == MX_OK) rc = p->arena.alloc(128 * 1024, 256, &p->sys);
  int id = -1;
  if (rc == MX_OK) rc = L->sched->create_shared(gpu, n_ctas, hbm_bytes, &id);
  if (rc || id != (int)L->parts.size()) {
    destroy_exec(p->cur.get());
    p->arena.release();
    set_error("part_create_shared: arena or scheduler failure");
    return rc ? rc : MX_EDEVICE;
  }
  p->id = id;
  Partition* raw = p.get();
  L->parts.push_back(std::move(p));
  {
    std::lock_guard<std::mutex> glk(g.mu);
    g.parts.push_back(raw);
  }
  *out_part = id;
  return MX_OK;
}

mx_status part_resize(int32_t part, int32_t sm_count, uint64_t hbm_bytes) {
  MX_REQUIRE_INIT();
  std::lock_guard<std::mutex> lk(L->mu);
  if (!L->sched->is_live(part)) {
    set_error("part_resize: unknown partition %d", part);
    return MX_EINVAL;
  }
  Partition& p = *L->parts[part];
  Gpu& g = *L->gpus[p.gpu];
  std::lock_guard<std::mutex> llk(p.load_mu);   // a cold start keeps p.cur until it ends
  std::vector<int> groups;
  int smc = 0;
  bool whole = false;
  uint64_t quota = 0;
  int rc = L->sched->plan_resize(part, sm_count, hbm_bytes, &groups, &smc, &whole, &quota);
  if (rc) {
    set_error("part_resize(%d, sm=%d): %s", part, sm_count, mx_strerror(rc));
    return rc;
  }
  if (p.arena.used() > quota) {
    set_error("part_resize: quota %llu below used %llu", (unsigned long long)quota,
              (unsigned long long)p.arena.used());
    return MX_EBUSY;
  }
  CtxGuard cg(g.primary);
  const SchedPart& sp = L->sched->part(part);
  const bool same_sms = sp.shared || (groups == sp.groups && whole == sp.whole);
  std::unique_ptr<Exec> ne;
  const uint64_t t0 = now_ns();
  if (!same_sms) {
    rc = make_exec(g, groups, whole, sp.epoch + 1, &ne);
    if (rc) return rc;
  }
  const uint64_t t1 = now_ns();
  uint64_t t2 = 0;
  {
    std::lock_guard<std::mutex> glk(g.mu);
    t2 = now_ns();
    if (ne) {
      // FIFO across the switch: the new stream starts after the old one's last work.
      Exec* old = p.cur.get();
      {
        CtxGuard og(old->ctx);
        CUevent fence_ev = nullptr;
        if (drv().cuEventCreate(&fence_ev, CU_EVENT_DISABLE_TIMING) == CUDA_SUCCESS) {
          drv().cuEventRecord(fence_ev, old->stream);
          drv().cuStreamWaitEvent(ne->stream, fence_ev, 0);
          drv().cuEventDestroy(fence_ev);   // released once it completes
        }
      }
      p.draining.push_back(std::move(p.cur));
      p.cur = std::move(ne);
    } else {
      p.cur->epoch = sp.epoch + 1;
      if (sp.shared) p.cur->n_ctas = smc;   // unpartitioned: only the grid size changes
    }
    p.arena.set_quota(quota);
  }
  if (g_trace_resize)
    fprintf(stderr, "[mx] part_resize(%d -> %d SMs): new exec %.3f ms, dispatcher lock %.3f ms, "
            "switch %.3f ms\n", part, smc, (t1 - t0) * 1e-6, (t2 - t1) * 1e-6,
            (now_ns() - t2) * 1e-6);
  rc = L->sched->resize(part, sm_count, hbm_bytes);
  return rc;
}

mx_status part_destroy(int32_t part) {
  MX_REQUIRE_INIT();
  std::lock_guard<std::mutex> lk(L->mu);
  if (!L->sched->is_live(part)) {
    set_error("part_destroy: unknown partition %d", part);
    return MX_EINVAL;
  }
  Partition& p = *L->parts[part];
  Gpu& g = *L->gpus[p.gpu];
  std::lock_guard<std::mutex> llk(p.load_mu);   // no cold start in progress
  {
    std::lock_guard<std::mutex> glk(g.mu);
    if (!p.fifo.empty() || !p.inflight.empty() || !p.draining.empty()) {
      set_error("part_destroy: partition %d has pending work", part);
      return MX_EBUSY;
    }
    g.parts.erase(std::remove(g.parts.begin(), g.parts.end(), &p), g.parts.end());
  }
  CtxGuard cg(g.primary);
  drv().cuStreamSynchronize(p.cur->stream);
  for (auto& kv : p.insts) {
    for (Slot& s : kv.second->slots) free_slot_host(s);
    if (kv.second->shared_weights) release_shared_ref(g, kv.first);
  }
  p.insts.clear();
  release_exec(g, std::move(p.cur));
  p.arena.release();
  p.live = false;
  return L->sched->destroy(part);
}

mx_status part_query(int32_t part, mx_part_info* out) {
  MX_REQUIRE_INIT();
  if (!out) return MX_EINVAL;
  std::lock_guard<std::mutex> lk(L->mu);
  if (!L->sched->is_live(part)) return MX_EINVAL;
  const SchedPart& sp = L->sched->part(part);
  Partition& p = *L->parts[part];
  out->gpu = sp.gpu;
  out->sm_count = sp.sm_count;
  out->n_ctas = p.cur ? p.cur->n_ctas : 0;
  out->whole = sp.whole ? 1 : 0;
  out->group_mask = sp.mask();
  out->hbm_quota = p.arena.quota();
  out->hbm_used = p.arena.used();
  out->hbm_peak = p.arena.peak();
  out->epoch = sp.epoch;
  out->shared = sp.shared ? 1u : 0u;
  return MX_OK;
}

mx_status fn_register(const mx_fn_desc* desc, int32_t* out_fn) {
  MX_REQUIRE_INIT();
  if (!desc || !out_fn) return MX_EINVAL;
  int rc = validate_fn(*desc);
  if (rc) return rc;
  std::lock_guard<std::mutex> lk(L->mu);
  auto f = std::make_unique<Fn>();
  f->id = (int)L->fns.size() + 1;
  f->desc = *desc;
  *out_fn = f->id;
  L->fns.push_back(std::move(f));
  return MX_OK;
}

static Fn* find_fn(Lib* L, int fn) {
  if (fn < 1 || fn > (int)L->fns.size()) return nullptr;
  return L->fns[fn - 1].get();
}

mx_status fn_load(int32_t fn, int32_t part) {
  MX_REQUIRE_INIT();
  Partition* p = nullptr;
  Fn* f = nullptr;
  Gpu* g = nullptr;
  {
    std::lock_guard<std::mutex> lk(L->mu);
    f = find_fn(L, fn);
    if (!f || !L->sched->is_live(part)) {
      set_error("fn_load: unknown fn %d or partition %d", fn, part);
      return MX_EINVAL;
    }
    p = L->parts[part].get();
    g = L->gpus[p->gpu].get();
  }
  std::lock_guard<std::mutex> llk(p->load_mu);
  FnInst* fi = nullptr;
  return load_instance(*g, *p, *f, &fi);
}

mx_status mx_weight_pool_query(int32_t gpu, uint64_t* used_bytes, int32_t* n_fns) {
  MX_REQUIRE_INIT();
  if (!used_bytes || !n_fns) return MX_EINVAL;
  if (gpu < 0 || gpu >= (int)L->gpus.size()) return MX_ENODEV;
  Gpu& g = *L->gpus[gpu];
  std::lock_guard<std::mutex> wl(g.wpool_mu);
  *used_bytes = g.wpool_ready ? g.wpool.used() : 0;
  int n = 0;
  for (auto& kv : g.shared_w)
    if (kv.second.weights) ++n;
  *n_fns = n;
  return MX_OK;
}

mx_status mx_task_default_cost(const mx_fn_desc* desc, const mx_task_desc* task, uint64_t* out) {
  if (!desc || !task || !out) return MX_EINVAL;
  int rc = validate_fn(*desc);
  if (rc) return rc;
  rc = validate_task(*desc, *task);
  if (rc) return rc;
  *out = default_cost(*desc, *task);
  return MX_OK;
}

mx_status fn_submit(int32_t part, const mx_task_desc* task, uint64_t* out_task) {
  MX_REQUIRE_INIT();
  if (!task || !out_task) return MX_EINVAL;
  Fn* f;
  {
    std::lock_guard<std::mutex> lk(L->mu);
    f = find_fn(L, task->fn);
  }
  if (!f) {
    set_error("fn_submit: unknown fn %d", task->fn);
    return MX_EINVAL;
  }
  int rc = validate_task(f->desc, *task);
  if (rc) return rc;
  auto t = std::make_unique<Task>();
  t->fn = f->id;
  t->kind = f->desc.kind;
  t->cost = task->cost ? task->cost : default_cost(f->desc, *task);
  if (t->kind == MX_FN_DECODE) {
    t->B = task->batch;
    t->P = task->prompt_len;
    t->G = task->gen_len;
    t->prompt.assign(task->prompt, task->prompt + (size_t)t->B * t->P);
    t->out_tokens = task->out_tokens;
    t->out_logits = task->out_logits;
  } else {
    // copy the inputs once, straight into their device image (caller may free on return)
    const bool train = t->kind == MX_FN_MPNN_TRAIN;
    t->n_mol = task->n_mol;
    t->n_atoms = task->n_atoms;
    t->n_edges = task->n_edges;
    t->blob.resize(mpnn_blob_layout(*t, train, t->n_mol, t->n_atoms, t->n_edges));
    uint8_t* b = t->blob.data();
    memcpy(b + t->off_ao, task->atom_off, (size_t)(t->n_mol + 1) * 4);
    memcpy(b + t->off_eo, task->edge_off, (size_t)(t->n_mol + 1) * 4);
    memcpy(b + t->off_at, task->atom_type, (size_t)t->n_atoms);
    if (t->n_edges > 0) memcpy(b + t->off_ed, task->edges, (size_t)t->n_edges * 6);
    t->out_ip = task->out_ip;
    if (train) {
      memcpy(b + t->off_tg, task->targets, (size_t)t->n_mol * 4);
      t->lr = task->lr;
      t->out_loss = task->out_loss;
      // training tiles are full 128-atom tiles, independent of the partition
      // (per-tile gradient partials are summed in tile order). A 64-atom cap
      // was 0.50 -> 0.42 ms at 148 SMs but 1.42 -> 1.99 ms at 20 SMs; not kept.
      t->n_tiles = mxk::mpnn_pack_tiles(task->atom_off, task->edge_off, t->n_mol,
                                        reinterpret_cast<int*>(b + t->off_tile));
      t->tile_ctas = -2;
    }
  }
  Task* raw = t.get();
  Partition* p = nullptr;
  Gpu* g = nullptr;
  {
    std::lock_guard<std::mutex> lk(L->mu);
    Placement pl{};
    rc = L->sched->submit(f->id, part, t->cost, &pl);
    if (rc) {
      set_error("fn_submit: partition %d not live", part);
      return rc;
    }
    t->id = pl.task;
    t->gpu = pl.gpu;
    t->part = pl.part;
    t->seq = pl.seq;
    t->epoch = pl.epoch;
    t->t_submit = now_ns();
    p = L->parts[pl.part].get();
    g = L->gpus[pl.gpu].get();
    L->tasks[t->id] = std::move(t);
    std::lock_guard<std::mutex> glk(g->mu);
    p->fifo.push_back(raw);
    if (raw->kind == MX_FN_MPNN) raw->tile_ctas = p->cur->n_ctas;   // balance for this size
  }
  if (raw->kind == MX_FN_MPNN) {
    // inference tiling, outside every lock (the task is not `ready` yet); the
    // dispatcher re-balances only if the partition is resized before launch
    uint8_t* b = raw->blob.data();
    raw->n_tiles = balanced_tiles(reinterpret_cast<const int*>(b + raw->off_ao),
                                  reinterpret_cast<const int*>(b + raw->off_eo), raw->n_mol,
                                  raw->tile_ctas, reinterpret_cast<int*>(b + raw->off_tile));
  }
  // cold start on first use (outside the global lock; FIFO order is kept by `ready`)
  FnInst* fi = nullptr;
  {
    std::lock_guard<std::mutex> llk(p->load_mu);
    rc = load_instance(*g, *p, *f, &fi);
  }
  {
    std::lock_guard<std::mutex> glk(g->mu);
    if (rc) {
      // the task completes (exactly once) with the load error
      p->fifo.erase(std::remove(p->fifo.begin(), p->fifo.end(), raw), p->fifo.end());
    } else {
      raw->inst = fi;
      raw->ready = true;
    }
  }
  if (rc) {
    std::lock_guard<std::mutex> lk(L->mu);
    raw->status = rc;
    raw->done = true;
    L->done_cv.notify_all();
  } else {
    g->cv.notify_all();
  }
  *out_task = raw->id;
  return MX_OK;
}

mx_status fn_wait(uint64_t task, int64_t timeout_ns, mx_result* out) {
  MX_REQUIRE_INIT();
  std::unique_lock<std::mutex> lk(L->mu);
  auto it = L->tasks.find(task);
  if (it == L->tasks.end() || it->second->collected) {
    set_error("fn_wait: task %llu unknown or already collected", (unsigned long long)task);
    return MX_ENOENT;
  }
  Task* t = it->second.get();
  if (timeout_ns < 0) {
    L->done_cv.wait(lk, [&] { return t->done; });
  } else if (!L->done_cv.wait_for(lk, std::chrono::nanoseconds(timeout_ns), [&] { return t->done; })) {
    return MX_ETIMEDOUT;
  }
  if (out) {
    out->status = t->status;
    out->gpu = t->gpu;
    out->part = t->part;
    out->epoch = t->epoch;
    out->seq_in_part = t->seq;
    out->t_submit_ns = t->t_submit;
    out->t_start_ns = t->t_start;
    out->t_end_ns = t->t_end;
    out->kernel_ns = t->kernel_ns;
  }
  L->timing.push_back({t->id, t->fn, t->gpu, t->part, t->seq, t->epoch, t->status, t->t_submit,
                       t->t_start, t->t_end, t->kernel_ns});
  t->collected = true;
  L->tasks.erase(it);
  return MX_OK;
}

mx_status mx_trace_write(const char* path) {
  MX_REQUIRE_INIT();
  if (!path) return MX_EINVAL;
  std::lock_guard<std::mutex> lk(L->mu);
  std::vector<uint8_t> b = L->sched->trace_bytes();
  FILE* f = fopen(path, "wb");
  if (!f) {
    set_error("cannot open %s", path);
    return MX_EINVAL;
  }
  fwrite(b.data(), 1, b.size(), f);
  fclose(f);
  std::string tp = std::string(path) + ".timing";
  FILE* ft = fopen(tp.c_str(), "w");
  if (ft) {
    fprintf(ft, "task,fn,gpu,part,seq,epoch,status,t_submit_ns,t_start_ns,t_end_ns,kernel_ns\n");
    for (const TimingRec& r : L->timing)
      fprintf(ft, "%llu,%d,%d,%d,%llu,%u,%d,%llu,%llu,%llu,%llu\n", (unsigned long long)r.task, r.fn,
              r.gpu, r.part, (unsigned long long)r.seq, r.epoch, r.status,
              (unsigned long long)r.t_submit, (unsigned long long)r.t_start,
              (unsigned long long)r.t_end, (unsigned long long)r.kernel_ns);
    fclose(ft);
  }
  return MX_OK;
}

mx_status fn_read_tensor(int32_t fn, int32_t part, int32_t tensor_id, void* host, uint64_t bytes) {
  MX_REQUIRE_INIT();
  if (!host) return MX_EINVAL;
  Partition* p;
  Gpu* g;
  {
    std::lock_guard<std::mutex> lk(L->mu);
    if (!L->sched->is_live(part)) return MX_EINVAL;
    p = L->parts[part].get();
    g = L->gpus[p->gpu].get();
  }
  std::lock_guard<std::mutex> llk(p->load_mu);
  auto it = p->insts.find(fn);
  if (it == p->insts.end() || !it->second->loaded) {
    set_error("fn %d not loaded on partition %d", fn, part);
    return MX_EINVAL;
  }
  uint64_t off, n;
  int gain;
  const bool f32 = it->second->fn->desc.kind == MX_FN_MPNN_TRAIN;   // fp32 training state
  if (!tensor_span(*it->second, tensor_id, &off, &n, &gain) || bytes > n * (f32 ? 4 : 2)) {
    set_error("bad tensor id %d or size", tensor_id);
    return MX_EINVAL;
  }
  CtxGuard cg(g->primary);
  if (f32)
    CU_TRY(drv().cuMemcpyDtoH(host, it->second->params + off * 4, bytes));
  else
    CU_TRY(drv().cuMemcpyDtoH(host, it->second->weights + off * 2, bytes));
  return MX_OK;
}

static int probe_many(Lib* L, const int32_t* parts, int n_parts, int n_ctas, uint64_t spin_ns,
                      uint32_t* smids) {
  if (n_ctas < 1 || n_ctas > 16384 || n_parts < 1 || !smids) return MX_EINVAL;
  std::vector<Partition*> ps;
  {
    std::lock_guard<std::mutex> lk(L->mu);
    for (int i = 0; i < n_parts; ++i) {
      if (!L->sched->is_live(parts[i])) return MX_EINVAL;
      ps.push_back(L->parts[parts[i]].get());
    }
  }
  for (Partition* p : ps) {
    Gpu& g = *L->gpus[p->gpu];
    std::lock_guard<std::mutex> glk(g.mu);
    if (mxk::launch_probe(reinterpret_cast<uint32_t*>(p->sys), n_ctas, spin_ns, p->cur->stream)) {
      set_error("probe launch failed");
      return MX_EDEVICE;
    }
  }
  for (int i = 0; i < n_parts; ++i) {
    Partition* p = ps[i];
    CtxGuard cg(L->gpus[p->gpu]->primary);
    CU_TRY(drv().cuStreamSynchronize(p->cur->stream));
    CU_TRY(drv().cuMemcpyDtoH(smids + (size_t)i * n_ctas, p->sys, (size_t)n_ctas * 4));
  }
  return MX_OK;
}

mx_status mx_probe_smids(int32_t part, int32_t n_ctas, uint64_t spin_ns, uint32_t* smids) {
  MX_REQUIRE_INIT();
  return probe_many(L, &part, 1, n_ctas, spin_ns, smids);
}

mx_status mx_probe_smids_concurrent(const int32_t* parts, int32_t n_parts, int32_t n_ctas,
                                    uint64_t spin_ns, uint32_t* smids) {
  MX_REQUIRE_INIT();
  if (!parts) return MX_EINVAL;
  return probe_many(L, parts, n_parts, n_ctas, spin_ns, smids);
}

mx_status mx_decode_profile(int32_t part, uint64_t* out, int32_t n_words) {
  MX_REQUIRE_INIT();
  if (!out || n_words < 0 || n_words > 8192) return MX_EINVAL;
  Partition* p;
  {
    std::lock_guard<std::mutex> lk(L->mu);
    if (!L->sched->is_live(part)) return MX_EINVAL;
    p = L->parts[part].get();
  }
  CtxGuard cg(L->gpus[p->gpu]->primary);
  CU_TRY(drv().cuStreamSynchronize(p->cur->stream));
  CU_TRY(drv().cuMemcpyDtoH(out, p->sys + 65536, (size_t)n_words * 8));
  return MX_OK;
}

mx_status mx_debug_inject_error(int32_t part, int32_t code) {
  MX_REQUIRE_INIT();
  if (code <= 0) return MX_EINVAL;
  std::lock_guard<std::mutex> lk(L->mu);
  if (!L->sched->is_live(part)) return MX_EINVAL;
  L->parts[part]->inject_err.store(code);
  return MX_OK;
}

mx_status mx_launch_count(uint64_t* out) {
  if (!out) return MX_EINVAL;
  *out = mxk::launch_counter();
  return MX_OK;
}

// ---- host-only placement engine --------------------------------------------
struct mx_sched {
  mx::Sched s;
  mx_sched(int a, int b, int c, int d, uint64_t e) : s(a, b, c, d, e) {}
};

mx_sched* mx_sched_new(int32_t n_gpus, int32_t n_groups, int32_t group_size, int32_t total_sms,
                       uint64_t mem_bytes) {
  if (n_gpus < 1 || n_groups < 1 || n_groups > 64 || group_size < 1 || total_sms < 1) return nullptr;
  return new mx_sched(n_gpus, n_groups, group_size, total_sms, mem_bytes);
}

void mx_sched_free(mx_sched* s) { delete s; }

mx_status mx_sched_create(mx_sched* s, int32_t gpu, int32_t sm_count, uint64_t hbm, int32_t* out_part) {
  if (!s || !out_part) return MX_EINVAL;
  return s->s.create(gpu, sm_count, hbm, out_part);
}

mx_status mx_sched_create_shared(mx_sched* s, int32_t gpu, int32_t n_ctas, uint64_t hbm,
                                 int32_t* out_part) {
  if (!s || !out_part) return MX_EINVAL;
  return s->s.create_shared(gpu, n_ctas, hbm, out_part);
}

mx_status mx_sched_resize(mx_sched* s, int32_t part, int32_t sm_count, uint64_t hbm) {
  if (!s) return MX_EINVAL;
  return s->s.resize(part, sm_count, hbm);
}

mx_status mx_sched_destroy(mx_sched* s, int32_t part) {
  if (!s) return MX_EINVAL;
  return s->s.destroy(part);
}

mx_status mx_sched_submit(mx_sched* s, int32_t fn, int32_t part, uint64_t cost, uint64_t* out_task,
                          int32_t* out_part, uint64_t* out_seq) {
  if (!s) return MX_EINVAL;
  Placement pl{};
  int rc = s->s.submit(fn, part, cost, &pl);
  if (rc) return rc;
  if (out_task) *out_task = pl.task;
  if (out_part) *out_part = pl.part;
  if (out_seq) *out_seq = pl.seq;
  return MX_OK;
}

mx_status mx_sched_trace(const mx_sched* s, void* buf, uint64_t cap, uint64_t* len) {
  if (!s || !len) return MX_EINVAL;
  std::vector<uint8_t> b = s->s.trace_bytes();
  *len = b.size();
  if (buf && cap >= b.size()) memcpy(buf, b.data(), b.size());
  return MX_OK;
}

// N2: measure a function's single-instance service time on partitions of the
// candidate sizes (one warm-up + `reps` timed runs of `sample` each, alone on
// the GPU), then apply the right-sizing rule (mx_rightsize) to the measured
// curve. Uses only this ABI (part_create / fn_load / fn_submit / fn_wait /
// part_destroy), so the calibration tasks are ordinary tasks of the trace.
mx_status fn_rightsize(int32_t fn, int32_t gpu, const mx_task_desc* sample, uint64_t hbm_bytes,
                       const int32_t* cand_sms, int32_t n_cand, int32_t reps, int32_t objective,
                       double slack, int32_t* out_sm, int32_t* out_parts, double* out_rate,
                       double* out_t_ns) {
  MX_REQUIRE_INIT();
  if (!sample || !cand_sms || n_cand < 1 || n_cand > 64 || reps < 1 || !out_sm || !out_parts ||
      sample->fn != fn)
    return MX_EINVAL;
  int sm_total = 0;
  {
    std::lock_guard<std::mutex> lk(L->mu);
    if (!find_fn(L, fn)) {
      set_error("fn_rightsize: unknown fn %d", fn);
      return MX_EINVAL;
    }
    if (gpu < 0 || gpu >= (int)L->gpus.size()) return MX_ENODEV;
    sm_total = L->gpus[gpu]->sm_total;
  }
  std::vector<int32_t> sms;
  std::vector<double> t;
  for (int i = 0; i < n_cand; ++i) {
    if (cand_sms[i] <= 0 || (i > 0 && cand_sms[i] <= cand_sms[i - 1])) return MX_EINVAL;
    int32_t part = -1;
    int rc = part_create(gpu, cand_sms[i], hbm_bytes, &part);
    if (rc) return rc;
    mx_part_info info{};
    part_query(part, &info);
    if (!sms.empty() && info.sm_count <= sms.back()) {   // rounds to the same group count
      part_destroy(part);
      continue;
    }
    double best = 0.0;
    for (int r = 0; r <= reps && rc == MX_OK; ++r) {
      uint64_t id = 0;
      mx_result res{};
      rc = fn_submit(part, sample, &id);
      if (rc == MX_OK) rc = fn_wait(id, -1, &res);
      if (rc == MX_OK && res.status != MX_OK) rc = res.status;
      const double ns = (double)(res.t_end_ns - res.t_start_ns);
      if (rc == MX_OK && r > 0 && (best == 0.0 || ns < best)) best = ns;   // r = 0: warm-up
    }
    part_destroy(part);
    if (rc) return rc;
    sms.push_back(info.sm_count);
    t.push_back(best);
    if (out_t_ns) out_t_ns[i] = best;
  }
  return mx_rightsize(sms.data(), t.data(), (int32_t)sms.size(), sm_total, 64, objective, slack,
                      out_sm, out_parts, out_rate);
}

mx_status mx_rightsize(const int32_t* sms, const double* t, int32_t n_points, int32_t total_sms,
                       int32_t max_parts, int32_t objective, double slack, int32_t* out_sm,
                       int32_t* out_parts, double* out_rate) {
  if (!sms || !t || !out_sm || !out_parts || n_points < 1 || total_sms < 1 || max_parts < 1 ||
      !(slack >= 0.0) || (objective != 0 && objective != 1))
    return MX_EINVAL;
  double tmin = 0.0;
  for (int i = 0; i < n_points; ++i) {
    if (sms[i] <= 0 || !(t[i] > 0.0) || (i > 0 && sms[i] <= sms[i - 1])) return MX_EINVAL;
    if (i == 0 || t[i] < tmin) tmin = t[i];
  }
  int best = -1;
  int best_parts = 0;
  for (int i = 0; i < n_points; ++i) {
    if (sms[i] > total_sms) break;
    const int parts = std::min(max_parts, total_sms / sms[i]);
    if (objective == 0) {
      if (t[i] <= (1.0 + slack) * tmin) {
        best = i;
        best_parts = parts;
        break;
      }
    } else if (best < 0 || (double)parts * t[best] >= (double)best_parts * t[i]) {
      // parts / t[i] >= best_parts / t[best]; ascending sms -> ties go to the larger size
      best = i;
      best_parts = parts;
    }
  }
  if (best < 0) return MX_EINVAL;
  *out_sm = sms[best];
  *out_parts = best_parts;
  if (out_rate) *out_rate = (double)best_parts / t[best];
  return MX_OK;
}

}  // extern "C"
