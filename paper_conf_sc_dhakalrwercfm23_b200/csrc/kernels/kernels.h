// Host-visible kernel parameter blocks and launch helpers (no CUDA types in
// the signatures beyond the opaque stream handle).
#pragma once

#include <cstdint>

namespace mxk {

#ifdef __CUDACC__
#define MX_HD __host__ __device__
#else
#define MX_HD
#endif
#define MX_HD_FWD MX_HD
#ifndef MX_CONSUMER_WARPS
#define MX_CONSUMER_WARPS 11
#endif
#ifndef MX_MAX_STAGES
#define MX_MAX_STAGES 12
#endif
// Decode GEMVs run on the 5th-generation tensor cores (tcgen05): D[rows][16] =
// W[rows][K] . X[16][K]^T with W (bf16 weights, the A operand, M = 128 rows
// per MMA) streamed by 3-D tiled TMA in K-major SWIZZLE_128B boxes of
// [128 rows][64 columns] (16 KiB = one ring stage) and X (the activations as
// a bf16 hi/lo pair per sequence, the B operand) staged in shared memory.
constexpr int kTileM = 128;             // weight rows per MMA tile (UMMA M)
constexpr int kBlkK = 64;               // K columns per swizzle-atom row (128 bytes)
constexpr int kStageBytes = 32 * 1024;  // one ring stage: a tile's rows x up to 8 column blocks
// Column blocks per TMA box for a tile of h8 rows (h8 a multiple of 8): the
// box is [blocks][h8 rows][64 columns], so each row's nk*128 contiguous bytes
// are fetched by one request.
// (a power of two <= 8 dividing the 512-column segment grain).
MX_HD_FWD constexpr int decode_box_blocks(int h8) {
  return h8 <= 32 ? 8 : h8 <= 64 ? 4 : h8 <= 128 ? 2 : 1;
}
constexpr int kConsumerWarps = MX_CONSUMER_WARPS;   // staging / attention / MMA / epilogue warps
constexpr int kDecodeThreads = 32 * (kConsumerWarps + 1);  // + 1 producer (TMA) warp
constexpr int kAttHd = 128;             // max attention head_dim
constexpr int kMaxCtas = 160;           // >= 148 SMs
constexpr int kMaxSeqCap = 512;         // attention keeps <= 16 scores per lane
// Tensor maps of one decode function instance (device global memory, 64-byte
// aligned CUtensorMap objects): 6 matrices (QKV, O, GATE, UP, DOWN, LM) x 16
// box heights (8..128 rows): 4-D {64 columns, rows, column blocks, layers}.
constexpr int kDecodeMats = 6;
constexpr int kDecodeBoxH = 16;
constexpr int kDecodeMaps = kDecodeMats * kDecodeBoxH;
// Activation operand: B <= 4 -> one 8-row swizzle atom per 64 columns (hi of
// sequence b in row b, lo in row 4 + b; the N = 16 MMA reads the atom twice,
// stride byte offset 0); B > 4 -> two atoms (hi rows 0-7, lo rows 8-15).
MX_HD constexpr int decode_act_rows(int B) { return B <= 4 ? 8 : 16; }
MX_HD constexpr int decode_act_lo(int B) { return B <= 4 ? 4 : 8; }
MX_HD constexpr int decode_act_blk_bytes(int B) { return decode_act_rows(B) * 128; }
// Columns of one K segment: phases whose input is wider than 64 KiB of operand
// run as several K segments (split-K inside the owning CTA).
MX_HD constexpr int decode_seg_cols(int B) { return (64 * 1024 / decode_act_blk_bytes(B)) * kBlkK; }
constexpr int kSegGrain = 8 * kBlkK;   // K segment widths are multiples of 512 columns
MX_HD constexpr int decode_act_bytes(int B, int kmax) {
  return ((((kmax + kBlkK - 1) / kBlkK) * kBlkK < decode_seg_cols(B)
               ? ((kmax + kBlkK - 1) / kBlkK) * kBlkK
               : decode_seg_cols(B)) /
          kBlkK) *
         decode_act_blk_bytes(B);
}
// K segments of one GEMV phase (R output rows, KF input columns), a function
// of the shape only, so results stay bit-identical for any partition size:
// one segment when the input fits the operand region, else segments of at
// most half of it (the operand of segment s + 1 is copied into one half while
// the MMAs of segment s read the other). Large matrices (R x KF >= 2^24, e.g.
// every 7B phase) are split into half-region segments even when the input
// fits: their (segment, row-group) pieces are spread over the CTAs, so a CTA
// issues each M = 128 MMA on ~2x more of its own rows than a pure row split
// would give it (a skinny MMA costs the same issue time for 8 or 128 rows).
MX_HD constexpr int decode_nseg(int B, long long R, int KF, int splittable) {
  return KF > decode_seg_cols(B)
             ? (KF + decode_seg_cols(B) / 2 - 1) / (decode_seg_cols(B) / 2)
         : (splittable && R * KF >= (1ll << 24) && KF > decode_seg_cols(B) / 2)
             ? (KF + decode_seg_cols(B) / 2 - 1) / (decode_seg_cols(B) / 2)
             : 1;
}
// Rows per finalisation block of a distributed multi-segment phase: one CTA
// (assigned statically) sums the block's segment partials in segment order
// and applies the phase's epilogue.
constexpr int kFinRows = 128;
// Bytes of a global image of the activation operand over `cols` input columns
// (the shared-memory layout above, every 64-column block): the phase that
// produces an input writes it in this form, the consuming phase copies each
// K segment into shared memory with one bulk copy.
MX_HD constexpr int decode_img_bytes(int B, int cols) {
  return ((cols + kBlkK - 1) / kBlkK) * decode_act_blk_bytes(B);
}

// One decode task on one partition: all P+G-1 steps in ONE persistent launch
// (grid = the partition's SMs, one CTA per SM), phases separated by a
// device-wide barrier on a per-slot counter.
struct DecodeParams {
  int L, d, H, Hkv, hd, ff, V, q_dim, kv_dim, qkv_rows, max_seq;
  int B, P, G;
  float eps;
  int n_ctas;
  int fuse_att;              // attention computed per CTA inside the O phase
  // weights (bf16 bits)
  const uint16_t* w_layers;  // layer 0 block
  uint64_t layer_stride;     // elements between layer blocks
  uint64_t off_wqkv, off_wo, off_wgate, off_wup, off_wdown, off_gattn, off_gmlp;
  const uint16_t* g_final;
  const uint16_t* lm_head;
  const uint16_t* embed;
  const float* rope_cs;      // [max_seq][hd/2][2] (cos, sin)
  // per-slot activations (fp32) and state
  float* x;                  // [B][d] residual stream
  float* qkv;                // [B][qkv_rows]
  float* o;                  // [B][q_dim]
  float* a;                  // [B][ff]
  // operand images (decode_img_bytes): x * gain of the next normed phase (GU,
  // QKV of the next layer, LM head), attention output o, MLP activation a
  uint8_t* img_x;
  uint8_t* img_o;
  uint8_t* img_a;
  float* ssq;                // [B][d / 8] sums of squares of x over 8-row groups
  unsigned long long* cand;  // [kMaxCtas][B] per-CTA argmax keys
  float* kpart;              // segment partial sums [nseg][B][R (x2 for gate/up)] (decode_kpart_floats)
  unsigned long long* pflag; // [kMaxCtas] per-CTA "partials stored" flags (monotone: barrier targets)
  uint16_t* kc;              // [L][B][Hkv][max_seq][hd] bf16
  uint16_t* vc;
  const int* prompt;         // [B][P] (host-mapped)
  int* tokens;               // [B][G] (host-mapped)
  float* logits;             // [G][B][V] or nullptr
  unsigned long long* bar;   // grid barrier counter (monotone across launches)
  unsigned long long bar_base;
  unsigned long long* stamps;  // [2] globaltimer start / end
  int* err;                  // 0 ok, 1 barrier timeout
  unsigned long long* prof;  // [n_ctas][16] cycle buckets (MX_DECODE_PROF=1) or nullptr
  const void* tmaps;         // kDecodeMaps CUtensorMap (device memory): [matrix][box height]
  // host-mapped completion record: [0] start, [1] end, [2] err, [3] = done_tag,
  // written last (after a system-scope fence) by CTA 0
  unsigned long long* h_stamps;
  unsigned long long done_tag;
  int inject_err;            // test hook (mx_debug_inject_error): reported as the task's device error
};

// Floats of the segment-partial buffer for a shape (max over the phases).
uint64_t decode_kpart_floats(int B, int d, int q_dim, int qkv_rows, int ff, int V, int fuse_att);
// 1 if every CTA computes the whole attention itself (B*H*hd <= 1024, grid small enough).
int decode_fuse_attention(int B, int H, int hd, int n_ctas);
// 1 if this build records the per-CTA cycle buckets (-DMX_PROF_BUCKETS).
int decode_prof_buckets();
// Number of grid barriers one decode launch performs (host bookkeeping of bar_base).
uint64_t decode_barriers(int L, int P, int G, int fuse_att);

// Shared-memory bytes of the decode kernel for a given shape (-1: does not fit);
// fuse_att = 0 (separate attention phase) lets the attention scratch share the
// activation operand, leaving more of the 227 KiB to the weight ring.
int decode_smem_bytes(int B, int kmax, int* n_stages, int fuse_att = 1);
MX_HD constexpr bool decode_att_in_act(int B, int kmax, int fuse_att) {
  return !fuse_att && decode_act_bytes(B, kmax) >= kConsumerWarps * 3 * kAttHd * 4;
}

// cooperative != 0: cuLaunchCooperativeKernel (all CTAs co-resident; used on
// unpartitioned streams where other kernels compete for the same SMs).
int launch_decode(const DecodeParams& p, void* stream, int cooperative = 0);
int launch_fill_weights(uint16_t* dst, uint64_t n, uint64_t seed, uint32_t tid, int is_gain,
                        int n_ctas, void* stream);
int launch_rope_table(float* dst, int max_seq, int hd, float theta, void* stream);
int launch_probe(uint32_t* smids, int n_ctas, uint64_t spin_ns, void* stream);

// IP-emulator MPNN (C4): grid = partition SMs, molecules strided over CTAs.
struct MpnnParams {
  int F, T, n_types, n_bonds;
  int n_mol;
  const uint16_t* e_atom;    // [n_types][F]
  const uint16_t* w_b;       // [4][F][F]
  const uint16_t* u;         // [F][F]
  const uint16_t* c;         // [F]
  const uint16_t* w1;        // [F][F]
  const uint16_t* c1;        // [F]
  const uint16_t* w2;        // [F]
  const uint16_t* c2;        // [1]
  const int* atom_off;       // [n_mol+1]
  const uint8_t* atom_type;  // [n_atoms]
  const int* edge_off;       // [n_mol+1]
  const uint32_t* edges;     // packed mx_bond (6 B each) as raw bytes
  float* out;                // [n_mol] (host-mapped)
  unsigned long long* stamps;
  int n_ctas;
  const int* tile_off;       // [n_tiles+1] first molecule of each <=128-atom tile
  int n_tiles;
  // host-mapped completion record (as DecodeParams), written by the last CTA to
  // finish; stamps[4] is the CTA-completion counter (reset by that CTA)
  unsigned long long* h_stamps;
  unsigned long long done_tag;
  int inject_err;            // test hook (mx_debug_inject_error): reported as the task's device error
};
int mpnn_smem_bytes();
// Greedy, deterministic packing of molecules into <=128-atom / <=512-bond tiles.
int mpnn_pack_tiles(const int* atom_off, const int* edge_off, int n_mol, int* tile_off);
// Same packing with a smaller atom cap per tile (<= 128): used to spread an
// inference task over every CTA of the partition when the 128-atom packing
// leaves part of the last round of tiles idle.
int mpnn_pack_tiles_cap(const int* atom_off, const int* edge_off, int n_mol, int cap_atoms,
                        int* tile_off);
int launch_mpnn(const MpnnParams& p, void* stream);

// IP-emulator training step (N4): tile forward/backward + SGD apply.
struct MpnnTrainParams {
  int T, n_bonds, n_mol, n_params, n_tiles, n_ctas;
  uint32_t off[11];          // element offsets of the 11 tensors in params (C1 ids)
  float* params;             // fp32 training state [n_params]
  float* partials;           // [n_tiles][n_params] per-tile gradients
  float* hsave;              // [n_tiles][T+5][128][128] saved h^t (feature-major) + backward scratch
  uint8_t* wimg;             // mpnn_train_img_bytes(): tensor-core operand images of U, W_b
  const int* atom_off;
  const uint8_t* atom_type;
  const int* edge_off;
  const uint32_t* edges;
  const int* tile_off;
  const float* targets;      // [n_mol]
  float* y;                  // [n_mol] device copy of the predictions
  float* out;                // host-mapped [n_mol + 1]: predictions, loss
  float lr;
  unsigned long long* stamps;
  unsigned long long* h_stamps;
  unsigned long long done_tag;
  int inject_err;            // test hook (mx_debug_inject_error): reported as the task's device error
};
int mpnn_train_smem_bytes();
uint64_t mpnn_train_tile_scratch_floats(int T);
uint64_t mpnn_train_img_bytes();
int launch_mpnn_train(const MpnnTrainParams& p, void* stream);
int launch_widen_bf16(float* dst, const uint16_t* src, uint64_t n, int n_ctas, void* stream);
int mpnn_train_set_attrs(int device);

uint64_t launch_counter();

}  // namespace mxk

namespace mxk {
int launch_clock(unsigned long long* out, void* stream);
int decode_set_attrs(int device);
int mpnn_set_attrs(int device);
}  // namespace mxk
