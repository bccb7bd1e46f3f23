// Internal structures of libdyo (not part of the ABI). See include/dyo.h and DESIGN.md.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/dyo.h"

namespace dyo {

// Current CUDA device (0..63): one-time per-kernel attributes and caches are kept per device,
// since a process may drive several GPUs (one ctx each).
inline int current_device() {
  int d = 0;
  cudaGetDevice(&d);
  return d & 63;
}

constexpr int kSat = (1 << 24) - 1;       // R1(iii)
constexpr int kMaxSites = 4096;
constexpr int kEntCap = 1024;             // tensor-set entries per group (records before dedupe)
constexpr int kPlanThreads = 1024;

enum OpClass : int8_t { C_KEEP = 0, C_CARRY = 1, C_ALLOC = 2, C_FETCH = 3, C_SHARE = 4 };   // C_SHARE: R20

// ---- pilot --------------------------------------------------------------------------
constexpr int kMaxLayers = 16;
struct LayerDev {
  const float* W;    // out x in_pad: [w_0..w_{in-1}, bias, 0...] padded to a multiple of 4 floats
  const float* b;    // out
  int in_off;        // offset of this layer's input in the stage input vector
  int in_len;
  int in_pad;
  int out_off;       // offset in the stage output vector
  int out_len;
};
struct StageDev {
  int first_layer, n_layers;
  int in_width, out_width;   // widths of the stage input / output vectors
  int act;                   // 1: LeakyReLU
  int rows;                  // total output rows of the stage
};
struct PilotDev {
  int F, O;
  int n_stages;
  int max_width;            // largest stage in/out width (smem sizing)
  double slope;
  StageDev st[4 + kMaxLayers];
  LayerDev ly[3 * kMaxLayers + 8];
};

// ---- K1-TC: tensor-core batch pilot plan (pilot_tc.cu; built by dyo_load_pilot) --------
constexpr int kTcCtas = 16;           // CTAs per cluster
constexpr int kTcBatch = 64;          // predictions per cluster (MMA N)
constexpr int kTcMaxStages = 8;
constexpr int kTcSlots = 4;           // weight-chunk ring
constexpr int kTcSlotBytes = 24 * 1024;   // 128 rows x <= 24 K x (hi + lo) x 4 B
constexpr int kTcMaxKc = 24;
constexpr int kTcMaxKsl = 128;        // K-slice of one CTA (X buffer: 64 x 128 x (hi + lo))
constexpr int kTcMinBatch = 16;       // smaller batches take the cluster GEMV kernel
struct TcStage {
  int n_out, K, n_m, n_ks, ksl, act;
  const float* bias;                  // device, n_out
};
struct TcChunk {                      // one weight chunk: rows m*128.. of tile m, K [k0, k0+kc) of the slice
  int64_t off;                        // float offset into the blob (hi block, then lo block)
  int32_t bytes, stage, job, k0, kc, pad;
};
struct TcPlan {
  int n_stages, n_feat;
  TcStage st[kTcMaxStages];
  int chunk_ptr[kTcCtas + 1];
  const TcChunk* chunks;
  const float* blob;
};

// ---- arch on the device -------------------------------------------------------------
// 64-bit key hash of the memo: a sum of splitmix64-mixed (position, value) words, so one warp
// reduces it in any order; host (insert) and device (lookup) share it.
__host__ __device__ inline uint64_t memo_mix(uint64_t pos, int32_t v) {
  uint64_t z = pos * 0x9E3779B97F4A7C15ull ^ (uint64_t)(uint32_t)v;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

struct ArchDev {
  int T, n_ops, n_sites, n_pieces, n_arms, nn_type, S_max, D_s, h, K_max, F, O, n_branch_logits;
  int L_max;
  int64_t H, align;
  // tensors
  const int64_t* t_bytes;
  const int64_t* t_abytes;   // aligned
  const int64_t* t_host;
  const int32_t* t_flags;
  // operators
  const int32_t* op_sig;     // n_ops x 9 (saturated)
  const int32_t* acc_ptr;    // n_ops + 1
  const int32_t* acc_t;
  const int32_t* acc_m;
  const int32_t* acc_s;      // stride per access (R13): tensor = acc_t + acc_s * iteration
  const int32_t* acc_sb;     //   + acc_sb * (prediction index in the batch)
  // sites (preorder IF/LOOP)
  const int32_t* site_kind;  // 1 IF, 2 LOOP
  const int32_t* site_nch;   // choices
  const int32_t* site_lo;
  const int32_t* site_tie;
  const int32_t* site_logit; // logit offset (absolute in the O vector) or -1 (tied)
  const int32_t* site_arm_ptr;   // IF: site -> first arm index; arms give (first op, n ops)
  const int32_t* site_rev;   // LOOP: 1 = iteration index counts down (R13)
  const int32_t* arm_first_op;
  const int32_t* arm_nops;
  // top-level pieces: kind 0 static run (a = first op, b = n ops), 1 IF (a = site),
  // 2 LOOP (a = site, b = body first op, c = body n ops)
  const int32_t* piece_kind;
  const int32_t* piece_a;
  const int32_t* piece_b;
  const int32_t* piece_c;
  const int32_t* seg_table;  // S_max x 10
  int branch_head;           // 0: choices come from the host traversal (forced, R4)
  // nested sites (R16): the host resolves every prediction's path (rows + iteration indices);
  // the decode kernels read it instead of expanding top-level pieces (null otherwise)
  const int32_t* hp_op;      // max_batch x L_max: operator of each row (-1 control)
  const int32_t* hp_it;      // max_batch x L_max: iteration index of the row's loop (R13)
  const int32_t* hp_len;     // max_batch: path length
  const int32_t* forced;     // max_batch x n_sites choices written by the traversal, or null
  // exact-match mis-prediction memo (R15; memo.cpp): live entries > 0 enables the
  // lookup in the head decode. index: open-addressing slots (entry id, -1 empty, -2 deleted)
  int memo_live, memo_mask;
  const int32_t* memo_index;     // memo_mask + 1
  const uint64_t* memo_hash;     // capacity
  const int32_t* memo_key;       // capacity x (10 K_max + n_sites): raw block head, raw choices
  const int32_t* memo_val;       // capacity x n_sites: the actual choices
  unsigned long long* memo_hits; // device counter
};

// ---- prediction storage -------------------------------------------------------------
struct PredDev {
  int B;
  int32_t* K;         // B
  int32_t* L;         // B
  int32_t* choices;   // B x n_sites (after a memo hit: the memoised actual choices)
  int32_t* rchoices;  // B x n_sites: the pilot's own (raw) choices, the memo key's half
  int32_t* slots;     // B x K_max x 10 (decoded block head)
  int32_t* path;      // B x L_max (operator index, -1 control)
  int32_t* path_it;   // B x L_max iteration index (nested arches: written by the host)
  int32_t* grp;       // B x K_max x 2 (start, end rows)
  int32_t* blocks;    // B x K_max x 10 executed block vectors
  int32_t* ent_n;     // B x K_max entry counts
  int2* ent;          // B x K_max x kEntCap (t, mode | needs_fetch << 2)
  int32_t* status;    // decode status word (0 ok, else DYO_E_*), [1] = detail
  int32_t* head;      // B x head_stride: decoded heads for the two-phase batch decode (decode.cu)
  int head_stride;    // 3 + n_sites + (n_pieces + 1) + (K_max + 1) + K_max
};

// ---- planner state (device) -----------------------------------------------------------
// Resident records (one int4 per tensor valid in a half, the half's list in ascending offset):
//   x = offset / ALIGN, y = aligned size / ALIGN, z = t | flags << 20, w = next-use group index
//   within the current plan (-1: none). flags: kRecTransient, kRecNxRd (the next use reads
//   first), kRecDirty, kRecTomb (carried to the other half: dropped at the next rebuild).
constexpr int kRecTransient = 1 << 20, kRecNxRd = 1 << 21, kRecDirty = 1 << 22, kRecTomb = 1 << 23;
constexpr int kRecIdMask = (1 << 20) - 1;
struct PlanState {
  int8_t* loc;        // T: -1 host, 0/1 half
  int64_t* off;       // T: offset within the half
  uint8_t* dirty;     // T
  uint8_t* pw;        // T: written by the previous group
  int32_t* prev;      // T: entries of the previous group (ids)
  int32_t* prev_n;    // 1
  int64_t* G;         // 1
  int4* rl[2][2];     // [half][buffer]: resident records (capacity T each)
  int32_t* rl_meta;   // [0..1] records per half (tombstones included), [2..3] buffer selector
  int32_t* pos;       // T: index of a valid tensor's record in its half's current list
};
struct PlanHdr {      // per transition (device + pinned mirror)
  int32_t half, n_ent, n_evict, n_move, n_carry, n_alloc, n_fetch, flags;   // flags: bit 0 late_all, >> 1 n_share (R20)
  int64_t need, h2d, d2h, d2d;
  int64_t o_ent, o_evict, o_move, o_carry, o_alloc, o_fetch;  // record offsets
};

struct PlanOut {
  PlanHdr* hdr;          // max_groups
  dyo_entry_rec* ent;
  dyo_evict_rec* ev;
  dyo_move_rec* mv;
  dyo_carry_rec* ca;
  dyo_alloc_rec* al;
  dyo_fetch_rec* fe;
  int64_t cap_ent, cap_rec;
  int32_t* status;       // [0] status, [1] failing transition, [2] needed capacity
  int32_t* counts;       // [0..5] total records written per list
};

struct PlanScratch {
  // group list of the plan (plan_prep_kernel)
  int32_t* grp_b;       // max_groups: prediction of each planned group
  int32_t* grp_k;
  int64_t* ebase;       // max_groups: first entry record of each planned group
  int32_t* Kt;          // 1: groups in the plan
  // next occurrences (bucket kernels): every entry's next group holding its tensor
  int32_t* bcnt;        // T + 1: entries per tensor -> bucket bases
  int32_t* bfill;       // T
  int32_t* bkey;        // cap_ent: (group << 10 | entry) per bucket slot
  int32_t* bsort;       // cap_ent: the same, sorted per bucket
  int32_t* nxt;         // cap_ent: next group index of the entry's tensor (-1: none)
  uint8_t* nxt_rd;      // cap_ent: that occurrence reads first
  int32_t* first;       // T: first group of each tensor in the plan (-1)
  uint8_t* first_rd;    // T
  int32_t* au;          // T: aligned size / ALIGN
  // sequential planner
  uint32_t* inw;        // (T + 31) / 32: membership bitmap of W_j (global fallback of the smem copy)
  int32_t* wnx;         // T: next use of a W_j member (valid while it is in W_j)
  uint8_t* wfl;         // T: flags of a W_j member (bit 0 needs_fetch, 1 written)
  uint64_t* keys;       // 2 T + 2048: live candidate keys / EVICT sort keys (global when large)
  int4* kept;           // T: kept records of the half, ascending offset
  int32_t* gap_s;       // T + 2: free gaps (ALIGN units)
  int32_t* gap_e;
  int32_t* newoff;      // T: new offsets (ALIGN units) of placed / compacted tensors
};
// ---- host traversal decode (traverse.cpp, R4) ------------------------------
struct TravArch {
  std::vector<int32_t> sig;   // n_ops x 9 saturated signatures
  std::vector<int32_t> site_kind, site_nch, site_lo, site_tie, site_arm_ptr, arm_first, arm_n;
  std::vector<int32_t> piece_kind, piece_a, piece_b, piece_c;
};
// slots: K_max x 10 decoded block head of one prediction; choices: n_sites out; *matched = 1
// when an exact match was found (else the closest-count fallback of P:L147).
dyo_status traverse_decode(const TravArch& A, const int32_t* slots, int K_max, int32_t* choices, int* matched,
                           std::string& err);

// ---- host nested-site decode (nested.cpp, R16) -----------------------------
// Program tree of an arch with nested sites: every nested site is an If directly inside a
// top-level Loop body or If arm whose own arms hold operators only.
struct NestArch {
  std::vector<int32_t> kind, a, b, span, flags, site_of;   // per node (site_of: site index or -1)
  std::vector<int32_t> sig;                                // n_ops x 9 saturated signatures
  std::vector<int32_t> site_lo, site_tie, top;             // per site; top = 1 for top-level sites
};
// top_choices: n_sites ints (nested sites ignored). Outputs the path (operator per row, -1 for
// control rows; iteration index per row), the nested executions' choices in execution order and
// *matched (1 exact, 0 closest-count fallback).
dyo_status nested_decode(const NestArch& N, const int32_t* slots, int K_max, const int32_t* top_choices,
                         std::vector<int32_t>& path_op, std::vector<int32_t>& path_it, std::vector<int32_t>& nested,
                         int* matched, std::string& err);

// The path of given top-level choices and nested executions' choices (execution order).
dyo_status trace_path(const NestArch& N, const int32_t* choices, const int32_t* nested, int n_nested,
                      std::vector<int32_t>& path_op, std::vector<int32_t>& path_it, std::string& err);

// ---- launchers (implemented in the .cu files) ------------------------------------------
cudaError_t launch_encode(const ArchDev& a, const int64_t* desc, const int32_t* hist,
                          const int32_t* hist_tab, const int32_t* hist_K, int hist_B, int B, float* feat,
                          cudaStream_t s);
// Fused encode + pilot (+ decode epilogue when *fused is set on return; otherwise the caller
// launches the decode kernel).
cudaError_t launch_pilot(const ArchDev& a, const PilotDev& p, const PilotDev* p_dev, const float* feat_or_null,
                         const int64_t* desc, const int32_t* hist, const int32_t* hist_tab,
                         const int32_t* hist_K, int hist_B, int B, double* logits64, float* logits32,
                         PredDev& pd, int32_t* hist_tab_out, int32_t* hist_K_out, int* fused,
                         cudaStream_t s);
cudaError_t debug_stamps(int on, unsigned long long* out);
cudaError_t launch_floor(int C, int n_barriers, cudaStream_t s);
cudaError_t tc_debug_stamps(int on, unsigned long long* out);   // K1-TC: globaltimer ns of CTA 0
// K1-TC: batch pilot on tensor cores (logits only; the caller launches the decode kernel).
cudaError_t launch_pilot_tc(const ArchDev& a, const PilotDev* p_dev, const TcPlan* plan_dev, const float* feat,
                            const int64_t* desc, const int32_t* hist, const int32_t* hist_tab, const int32_t* hist_K,
                            int hist_B, int B, double* logits64, float* logits32, cudaStream_t s);
cudaError_t plan_debug_stamps(int j, unsigned long long* out);
// Copies a finished plan's headers and EVICT/MOVE/CARRY/ALLOC/FETCH records from the planner's
// device arrays (d) into the pinned mapped mirrors (h: device-side aliases) by the counts in
// d.counts; nothing when d.status[0] != 0. Entry records are not copied.
cudaError_t launch_plan_export(const PlanOut& d, const PlanOut& h, cudaStream_t s);
cudaError_t launch_partition(const ArchDev& a, const int32_t* ops, const int32_t* its, int L, int b,
                             const long long* op_ns, int K, int method, long long H, long long bw, long long* need,
                             long long* fetch, long long* comp, long long* f, int32_t* cuts, long long* result,
                             int* overflow, cudaStream_t s);
cudaError_t launch_fault_drop(const ArchDev& a, const PredDev& pd, int b0, int nb, double p, uint64_t seed,
                              cudaStream_t s);
cudaError_t launch_decode(const ArchDev& a, const double* logits, PredDev& pd, int B,
                          int32_t* hist_tab_out, int32_t* hist_K_out, cudaStream_t s);
cudaError_t launch_plan(const ArchDev& a, const PredDev& pd, int b0, int nb, int policy,
                        PlanState& in, PlanState& work, PlanScratch& sc, PlanOut& out,
                        int max_groups, cudaStream_t s);
struct CopySeg { const char* src; char* dst; int64_t bytes; };
cudaError_t launch_copy_segments(const CopySeg* segs_dev_or_mapped, int n, int64_t chunk,
                                 int grid, cudaStream_t s);
// Record-driven device<->device copy (TMA bulk; copy.cu): records rec[i*stride ..] (int64
// fields) in DEVICE memory, i < n, filtered by rec[f_late] == late_val when f_late >= 0, copy
// rec[f_bytes] bytes from src_base + rec[f_src] to dst_base + rec[f_dst] - dst_bias.
// rec == nullptr: one range of `total` bytes from src_base to dst_base. total = sum over the
// selected records of their 16-byte-aligned bodies (bytes & ~15, or 0 when src or dst is not
// 16-byte aligned): the host computes it with rec_body() below.
constexpr int kMaxWaves = 24;    // compaction waves per record-copy launch (grid barrier between)
struct RecCopyArgs {
  const int64_t* rec;
  int32_t stride, n, f_src, f_dst, f_bytes, f_late;
  int64_t late_val;
  const char* src_base;
  char* dst_base;
  int64_t dst_bias;
  int64_t total;
  unsigned long long* stamps;  // measurement aid (DYO_COPY_STAMPS): 4 x u64 per CTA, or null
  int64_t launch;              // launch index for the stamps
  // n_waves > 1: the records are processed as consecutive waves [wave_end[w-1], wave_end[w])
  // (relative to rec) of wave_total[w] body bytes each, every CTA arriving at a grid barrier
  // (counter gbar, target gbar_base + (w+1) * grid) between waves; cooperative launch
  int32_t n_waves;
  int32_t wave_end[kMaxWaves];
  int64_t wave_total[kMaxWaves];
  unsigned int* gbar;
  unsigned int gbar_base;
};
int64_t copy_stamps_read(unsigned long long* host, int64_t cap);
inline int64_t rec_body(const char* src, const char* dst, int64_t bytes) {
  return ((((uintptr_t)src) | ((uintptr_t)dst)) & 15) == 0 ? (bytes & ~(int64_t)15) : 0;
}
cudaError_t launch_copy_records(const RecCopyArgs& a, int grid, cudaStream_t s, int* grid_used = nullptr);

}  // namespace dyo
