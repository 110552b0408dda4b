/*
 * mx.h — C ABI of the B200-native multiplexed small-function runtime.
 *
 * What it does: runs many independent small function invocations ("tasks")
 * concurrently on fine-grained spatial partitions of each GPU instead of
 * time-sharing the whole device — Dhakal et al., "Fine-grained accelerator
 * partitioning for Machine Learning and Scientific Computing in Function as a
 * Service Platform", SC-W 2023. Citations: P:NNN = PAPER.md line
 * (section in brackets); C1..C7, A1..A27 = SURVEY.md §8(c) items.
 *
 *   paper (Parsl + MPS/MIG on A100)              this ABI (B200)
 *   ---------------------------------------------------------------------------
 *   GPU% per listed accelerator [P:171-173 §4.1]  part_create(gpu, sm_count, ...)
 *   same GPU listed twice         [P:173 §4.1]    several part_create on one gpu
 *   MIG slice: SMs + memory       [P:181 §4.2]    sm_count + hbm_bytes quota
 *   restart to re-partition       [P:242 §6]      part_resize (live, weights stay)
 *   register app, get future      [P:55,59,63]    fn_register, fn_submit -> id
 *   future.result()               [P:63 §2.2.1]   fn_wait
 *
 * Threading: every call is thread-safe. No C++ exception crosses the ABI.
 * Errors: every call returns an mx_status (0 = MX_OK, negative = error);
 * mx_last_error() gives a human-readable detail for the calling thread.
 * There is no CPU fallback: without a CC 10.x device, mx_init returns
 * MX_ENODEV and every device call returns MX_ESTATE.
 */
#ifndef MX_H_
#define MX_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t mx_status;
enum {
  MX_OK = 0,
  MX_ENOENT = -2,      /* unknown or already-collected task                           */
  MX_EDEVICE = -5,     /* asynchronous device fault; the task still completes once   */
  MX_ENOMEM = -12,     /* weights/slots exceed the partition quota, or no HBM         */
  MX_EBUSY = -16,      /* resize shrink below used; destroy with pending work         */
  MX_ENODEV = -19,     /* gpu out of range, or device is not compute capability 10.x */
  MX_EINVAL = -22,     /* null/unknown handle, bad shape, sm_count <= 0 at create     */
  MX_ENOSM = -28,      /* not enough free SM groups (keeps sum of SMs <= device)      */
  MX_ETIMEDOUT = -110, /* fn_wait timed out; the task stays waitable                  */
  MX_ESTATE = -125     /* library not initialised (or already shut down)              */
};
enum { MX_PART_ANY = -1 };           /* fn_submit: let the placement policy choose (C5) */
enum { MX_FN_DECODE = 1, MX_FN_MPNN = 2, MX_FN_MPNN_TRAIN = 3 };
/* MX_FN_MPNN_TRAIN (§3.1 P:109 steps (3)/(7)
 * "train an ML model that acts as an emulator", §3.4): one SGD step of
 * the IP emulator per task on the MSE loss over the task's molecules
 * (reading R10). The instance holds fp32 parameters, initialised from the same
 * seeded values as MX_FN_MPNN, updated in place; tasks on one partition apply
 * their steps in seq_in_part order. Uses mx_fn_desc.mpnn; task inputs are the
 * MPNN CSR arrays plus targets[n_mol] and lr; outputs out_ip[n_mol] = the
 * predictions BEFORE the update and *out_loss = the loss. fn_read_tensor
 * returns fp32 values (4 bytes per element) for this kind. Not combinable
 * with MX_FN_SHARED_WEIGHTS (training state is per instance).             */
/* mx_fn_desc.flags */
enum { MX_FN_SHARED_WEIGHTS = 1 };   /* one read-only weight copy per GPU (N3)  */
enum { MX_INIT_DEFAULT = 0 };

/* ---------------------------------------------------------------------------
 * Function descriptors (fn_register).
 * ------------------------------------------------------------------------- */

/* Llama-style greedy decoder shape (the paper's LLaMa-2 text completion,
 * P:113-115 §3.2, §3.4, Fig. 4; block conventions C2/A8).
 * Constraints: d_model, q_dim = n_heads*head_dim and d_ff multiples of 8;
 * head_dim in {32, 64, 128}; n_heads % n_kv_heads == 0; 1 <= max_batch <= 8;
 * d_model <= 8192, q_dim and d_ff <= 16384, vocab <= 2^20. GEMVs run on the tensor cores
 * (tcgen05); phases whose input is wider than 64 KiB of bf16 hi/lo operand
 * (4096 columns at batch <= 4, 2048 above) run as K segments (split-K).    */
typedef struct {
  int32_t n_layers, d_model, n_heads, n_kv_heads, head_dim, d_ff, vocab;
  int32_t max_seq;   /* KV positions per sequence (>= prompt_len + gen_len - 1) */
  int32_t max_batch; /* sequences per task (B)                                  */
  float rms_eps, rope_theta;
} mx_decode_cfg;

/* IP-emulator message-passing network (molecular design, §3.1 step (4);
 * architecture is reading A22 / C4). Constraints: hidden == 128, steps >= 1,
 * n_atom_types <= 256, n_bond_types <= 4; per task at most max_mols
 * molecules, each with <= 32 atoms. */
typedef struct {
  int32_t n_atom_types, n_bond_types, hidden, steps;
  int32_t max_mols;  /* molecules per task                        */
  int32_t max_atoms; /* total atoms per task (sizes the slot)     */
  int32_t max_edges; /* total bonds per task                      */
} mx_mpnn_cfg;

typedef struct {
  int32_t kind;           /* MX_FN_DECODE or MX_FN_MPNN                              */
  /* MX_FN_SHARED_WEIGHTS (the paper's future work "share the
   * model weights" across instances, §7, and the cold-start cost
   * of loading them, §6): the weights (and RoPE table) live ONCE per GPU
   * in the GPU's read-only weight pool, generated by the first fn_load on that
   * GPU and referenced by every partition's instance. Partition quotas then
   * hold only the task slots (KV cache, activations). The pool is outside the
   * partition quotas; it is bounded by device memory (MX_ENOMEM when physical
   * memory cannot back it) and freed at mx_shutdown.                        */
  uint32_t flags;
  uint64_t weight_seed;   /* weights are generated on device from this seed (C1)     */
  mx_decode_cfg dec;
  mx_mpnn_cfg mpnn;
} mx_fn_desc;

/* One bond of a molecule: atoms u, v are local indices within the molecule,
 * u != v (a self-loop is MX_EINVAL at fn_submit, reading R12). The same pair
 * may be listed more than once; each listing is a bond of C4's sum.         */
typedef struct {
  int16_t u, v;
  uint8_t bond, pad;
} mx_bond;

/* One invocation. Inputs are COPIED during fn_submit (the caller may free them
 * on return). Output buffers are caller-owned host memory and must stay valid
 * until fn_wait returns for this task.                                        */
typedef struct {
  int32_t fn;
  /* decode (a6): steps s = 0..P+G-2 at positions t = s; outputs G tokens     */
  int32_t batch, prompt_len, gen_len;
  const int32_t* prompt;  /* [batch][prompt_len] token ids in [0, vocab)        */
  int32_t* out_tokens;    /* [batch][gen_len]                                   */
  float* out_logits;      /* [gen_len][batch][vocab] fp32, or NULL (parity mode) */
  /* mpnn (a7): CSR molecules; outputs one IP estimate per molecule            */
  int32_t n_mol, n_atoms, n_edges, reserved;
  const int32_t* atom_off;  /* [n_mol+1], atom_off[0] = 0, atom_off[n_mol] = n_atoms */
  const uint8_t* atom_type; /* [n_atoms]                                            */
  const int32_t* edge_off;  /* [n_mol+1], edge_off[n_mol] = n_edges                  */
  const mx_bond* edges;     /* [n_edges], u, v local to their molecule               */
  float* out_ip;            /* [n_mol]                                              */
  uint64_t cost;            /* placement cost units (C5); 0 = library default       */
  /* MX_FN_MPNN_TRAIN only                                                     */
  const float* targets;     /* [n_mol] training targets (the simulated IPs)         */
  float* out_loss;          /* [1] loss of the step (before the update)             */
  float lr;                 /* SGD learning rate                                    */
  int32_t reserved2;
} mx_task_desc;

typedef struct {
  mx_status status;       /* MX_OK or MX_EDEVICE                                       */
  int32_t gpu, part;
  uint32_t epoch;         /* partition epoch at submit (bumped by part_resize)         */
  uint64_t seq_in_part;   /* FIFO position in the partition (0-based)                  */
  uint64_t t_submit_ns;   /* host steady clock                                         */
  uint64_t t_start_ns;    /* device %globaltimer at kernel start, mapped to host clock */
  uint64_t t_end_ns;      /* device %globaltimer at kernel end, mapped to host clock   */
  uint64_t kernel_ns;     /* CUDA-event duration of the task's kernel on its stream    */
} mx_result;

typedef struct {
  int32_t gpu, sm_count;  /* sm_count: SMs actually provisioned (whole SM groups, R8)  */
  int32_t n_ctas;         /* persistent grid size used for this partition              */
  int32_t whole;          /* 1 = the whole device (all groups + remainder)            */
  uint64_t group_mask;    /* bit g = SM group g of the device split                    */
  uint64_t hbm_quota, hbm_used, hbm_peak;
  uint32_t epoch;
  uint32_t shared;        /* 1 = unpartitioned stream (part_create_shared, N1)        */
} mx_part_info;

typedef struct {
  int32_t ordinal, sm_total, n_groups, group_size, remainder_sms, cc_major, cc_minor, reserved;
  uint64_t mem_bytes;
} mx_gpu_info;

/* ---------------------------------------------------------------------------
 * Lifecycle.
 * ------------------------------------------------------------------------- */

/* Initialise on every visible GPU of compute capability 10.x. Sets
 * CUDA_DEVICE_MAX_CONNECTIONS=32 if unset (only effective before the first
 * CUDA call of the process), retains each primary context, splits each
 * device's SMs once into equal SM groups (cuDevSmResourceSplitByCount; on a
 * B200 37 groups of 4 SMs, reading R8 in DESIGN.md; MX_SM_GROUP=8 selects the
 * co-scheduling-aware 8-SM split), creates one whole-device green context
 * (clock calibration, unpartitioned N1 streams: no library kernel runs in the
 * primary context) and starts one dispatcher thread per GPU. MX_ENODEV if no
 * suitable GPU.                                                            */
mx_status mx_init(uint32_t flags);
/* Same, restricted to the listed device ordinals (e.g. one per torchrun rank). */
mx_status mx_init_devices(const int32_t* ordinals, int32_t n, uint32_t flags);
/* Waits for in-flight work, destroys partitions and releases everything.   */
mx_status mx_shutdown(void);
mx_status mx_gpu_count(int32_t* n);
mx_status mx_gpu_query(int32_t gpu, mx_gpu_info* out);
const char* mx_strerror(mx_status s);
const char* mx_last_error(void);   /* thread-local detail of the last failure   */

/* ---------------------------------------------------------------------------
 * Partitions (a1, a9).
 * ------------------------------------------------------------------------- */

/* Create a partition of `gpu` with at least `sm_count` SMs (rounded up to whole
 * SM groups, lowest free groups first; sm_count >= the device's SM count asks
 * for the whole device) and an HBM quota of `hbm_bytes` enforced by the
 * partition's allocator arena (A23: a capacity limit, not bandwidth or fault
 * isolation). Errors: MX_ENODEV, MX_EINVAL, MX_ENOSM, MX_ENOMEM (sum of quotas
 * would exceed device memory, I5).                                         */
mx_status part_create(int32_t gpu, int32_t sm_count, uint64_t hbm_bytes, int32_t* out_part);
/* Unpartitioned comparison mode (Table 1
 * and §5.2: time-sharing vs MPS vs MIG). The partition is a plain
 * stream of the GPU's whole-device green context: it owns NO SM groups (not counted in the
 * 148-SM budget, I2), its kernels may run on any SM, and decode grids are
 * `n_ctas` CTAs launched cooperatively (all CTAs co-resident or none).
 *   n_ctas = SM count  -> every task wants the whole GPU: tasks of different
 *                          shared partitions take turns (time-sharing analog);
 *   n_ctas = SMs / N   -> N partitions run side by side on hardware-chosen SMs
 *                          (default-MPS analog, no isolation).
 * `n_ctas` (clamped to the SM count) is also the partition's WLAW weight. The
 * HBM quota is enforced as for part_create. part_resize(part, n, 0) changes
 * the grid size; the partition stays shared. Errors as part_create, except
 * MX_ENOSM (no groups are taken).                                           */
mx_status part_create_shared(int32_t gpu, int32_t n_ctas, uint64_t hbm_bytes, int32_t* out_part);
/* Live re-partition (the paper's future work, §7): new SM group set (own
 * groups released first) -> new green context + stream; queued tasks go to the
 * new stream, in-flight ones finish on the old. Weights never move or reload.
 * sm_count <= 0 keeps the SMs, hbm_bytes == 0 keeps the quota. MX_EBUSY if the
 * new quota is below the bytes already used, MX_ENOSM if groups run out.   */
mx_status part_resize(int32_t part, int32_t sm_count, uint64_t hbm_bytes);
/* MX_EBUSY while the partition has queued or in-flight tasks.              */
mx_status part_destroy(int32_t part);
mx_status part_query(int32_t part, mx_part_info* out);

/* ---------------------------------------------------------------------------
 * Functions and tasks (a2-a8).
 * ------------------------------------------------------------------------- */

/* Register a function shape. Nothing is allocated until it is loaded.      */
mx_status fn_register(const mx_fn_desc* desc, int32_t* out_fn);
/* Cold start (§6): carve the weights and two task slots from the
 * partition arena (MX_ENOMEM if over quota) and generate the seeded bf16
 * weights on the partition's SMs. Synchronous. Implicit on first submit.   */
mx_status fn_load(int32_t fn, int32_t part);
/* Bytes held by `gpu`'s shared read-only weight pool and the number of
 * MX_FN_SHARED_WEIGHTS functions with weights in it (N3).                   */
mx_status mx_weight_pool_query(int32_t gpu, uint64_t* used_bytes, int32_t* n_fns);
/* Submit one task to `part` or MX_PART_ANY. Task ids are 1, 2, 3, ... in
 * submission order across the library. Placement is decided here, from
 * static costs only (deterministic, C5).                                   */
mx_status fn_submit(int32_t part, const mx_task_desc* task, uint64_t* out_task);
/* Block until the task completes (timeout_ns < 0: forever). Succeeds exactly
 * once per task (then MX_ENOENT). MX_ETIMEDOUT leaves the task waitable.
 * On return the caller's output buffers hold the results.                  */
mx_status fn_wait(uint64_t task, int64_t timeout_ns, mx_result* out);
/* Default placement cost of a task (C5): decode ceil(bytes/8000), MPNN
 * ceil(flops/75000). Pure host arithmetic.                                 */
mx_status mx_task_default_cost(const mx_fn_desc* desc, const mx_task_desc* task, uint64_t* out);

/* Canonical deterministic trace (C5): little-endian records of 8 x uint64,
 * timestamps excluded; a "<path>.timing" CSV sidecar holds the per-task times. */
mx_status mx_trace_write(const char* path);

/* ---------------------------------------------------------------------------
 * Inspection (tests and benches).
 * ------------------------------------------------------------------------- */

/* Copy `bytes` of weight tensor `tensor_id` (C1 ids; logical row-major bf16)
 * of fn's instance in `part` to host memory.                               */
mx_status fn_read_tensor(int32_t fn, int32_t part, int32_t tensor_id, void* host, uint64_t bytes);
/* Launch the %smid probe (K9) with `n_ctas` CTAs on the partition; each CTA
 * spins for `spin_ns` and writes its SM id to smids[cta]. Synchronous.     */
mx_status mx_probe_smids(int32_t part, int32_t n_ctas, uint64_t spin_ns, uint32_t* smids);
/* Launch probes on several partitions at once (all in flight together) and
 * collect every CTA's SM id: smids[i*n_ctas + c] for parts[i].              */
mx_status mx_probe_smids_concurrent(const int32_t* parts, int32_t n_parts, int32_t n_ctas,
                                    uint64_t spin_ns, uint32_t* smids);
/* Per-CTA cycle buckets of the last decode launch on `part` when the library
 * was initialised with MX_DECODE_PROF=1: [cta][8] = total, grid barrier,
 * input staging, TMA-ring wait, GEMV, attention, producer wait, 0.       */
mx_status mx_decode_profile(int32_t part, uint64_t* out, int32_t n_words);
/* Number of kernels this library launched since init (all GPUs).          */
mx_status mx_launch_count(uint64_t* out);
/* Fault-path test hook: the next task LAUNCHED on `part` runs normally but its
 * kernel reports device error `code` (> 0) in its completion record, exactly
 * as a bounded-wait timeout would (SURVEY.md §8(b) MX_EDEVICE row: "the task
 * still completes exactly once, with this status"). The slot is reset before
 * its next use. MX_EINVAL for an unknown partition or code <= 0.           */
mx_status mx_debug_inject_error(int32_t part, int32_t code);

/* ---------------------------------------------------------------------------
 * Host-only placement engine (no device needed): the same C++ object the
 * runtime uses for every placement, exposed so the policy can be checked
 * against the oracle's simulator on any machine.
 * ------------------------------------------------------------------------- */
typedef struct mx_sched mx_sched;
mx_sched* mx_sched_new(int32_t n_gpus, int32_t n_groups, int32_t group_size, int32_t total_sms,
                       uint64_t mem_bytes);
void mx_sched_free(mx_sched* s);
mx_status mx_sched_create(mx_sched* s, int32_t gpu, int32_t sm_count, uint64_t hbm, int32_t* out_part);
mx_status mx_sched_create_shared(mx_sched* s, int32_t gpu, int32_t n_ctas, uint64_t hbm,
                                 int32_t* out_part);
mx_status mx_sched_resize(mx_sched* s, int32_t part, int32_t sm_count, uint64_t hbm);
mx_status mx_sched_destroy(mx_sched* s, int32_t part);
mx_status mx_sched_submit(mx_sched* s, int32_t fn, int32_t part, uint64_t cost,
                          uint64_t* out_task, int32_t* out_part, uint64_t* out_seq);
/* Serialise the canonical trace into buf (cap bytes); *len = bytes needed. */
mx_status mx_sched_trace(const mx_sched* s, void* buf, uint64_t cap, uint64_t* len);

/* ---------------------------------------------------------------------------
 * Right-sizing policy (Fig. 2
 * "LLaMa2 can only properly utilize about 20 SMs", future work P:252). Host
 * only. Input: a function's single-instance service time t[i] (any time unit)
 * measured alone on sms[i] SMs (the D2b sweep; n_points >= 1, sms ascending,
 * each > 0). Output: a partition size *out_sm (one of sms[]) and a count
 * *out_parts of equal partitions for a device of total_sms SMs (<= max_parts),
 * with the predicted throughput *out_rate = parts / t (tasks per time unit):
 *   objective 0 (latency knee): the smallest sms[i] with
 *                t[i] <= (1 + slack) * min_j t[j];
 *   objective 1 (throughput):   argmax_i floor(total_sms / sms[i]) / t[i]
 *                (exact ties -> the larger partition, i.e. lower latency).
 * Errors: MX_EINVAL on null pointers, n_points < 1, non-positive or
 * non-ascending sms, non-positive t, slack < 0, or no size fitting total_sms. */
mx_status mx_rightsize(const int32_t* sms, const double* t, int32_t n_points, int32_t total_sms,
                       int32_t max_parts, int32_t objective, double slack, int32_t* out_sm,
                       int32_t* out_parts, double* out_rate);

/* Right-sizing from a measured sweep (N2: "the dispatcher sizes partitions
 * automatically"). For each candidate SM count cand_sms[i] (ascending; a
 * count that rounds to an already measured group count is skipped and its
 * out_t_ns entry left untouched) a partition of that size and `hbm_bytes`
 * is created on `gpu`, `fn` is loaded, `sample` (a task of `fn`; its output
 * buffers receive the results) runs once to warm up and `reps` more times,
 * and the best device service time (t_end - t_start) is kept in out_t_ns[i]
 * (may be NULL). The partition is destroyed before the next size, so the
 * function runs alone (the paper's Fig. 2 SM sweep). The
 * measured curve then goes through mx_rightsize(objective, slack) over the
 * GPU's SM count with at most 64 partitions: *out_sm per partition,
 * *out_parts partitions, *out_rate = out_parts / t (tasks per ns). The
 * calibration tasks are ordinary tasks (they appear in the trace). Errors
 * of the underlying calls are returned as is; MX_EINVAL for bad arguments. */
mx_status fn_rightsize(int32_t fn, int32_t gpu, const mx_task_desc* sample, uint64_t hbm_bytes,
                       const int32_t* cand_sms, int32_t n_cand, int32_t reps, int32_t objective,
                       double slack, int32_t* out_sm, int32_t* out_parts, double* out_rate,
                       double* out_t_ns);

#ifdef __cplusplus
}
#endif
#endif /* MX_H_ */
