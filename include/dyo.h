/*
 * dyo.h — C ABI of the B200-native DyNN-Offload hot path (libdyo.so).
 *
 * Paper: Ren et al., "Enabling Large Dynamic Neural Network Training with Learning-based
 * Memory Management", HPCA 2024 (PAPER.md; "P:Lnnn" = line nnn). Readings R1-R12 of the
 * paper's silent/garbled points are in DESIGN.md §2 and are referenced below.
 *
 * Per training step the caller runs
 *     dyo_pilot_predict  (encode + pilot MLP + decode; on device)
 *     dyo_plan           (double-buffered evict/prefetch plan; on device, then
 *                         one synchronisation that hands the DMA sizes to the host)
 *     dyo_migrate(j)     for j = 0..K-1 (evict -> compact/carry -> fetch)
 *
 * Conventions (all entry points):
 *   - return a dyo_status (0 = OK, negative = error); nothing throws or aborts;
 *     dyo_strerror() names a status, dyo_last_error() describes the last failure of a ctx.
 *   - "device" pointers are CUDA device (or managed) memory; "host" pointers are CPU memory;
 *     arguments documented "host or device" are detected with cudaPointerGetAttributes and
 *     host data is staged to the device on the call's stream (the end-to-end path).
 *   - streams/events are cudaStream_t / cudaEvent_t passed as void*; NULL stream = legacy
 *     default stream. Calls are stream-ordered and asynchronous unless stated otherwise.
 *   - a dyo_ctx is bound to one GPU and is not thread-safe (one manager per GPU, §8(e)).
 *   - integer limits (validated at load, DYO_E_INVAL otherwise): tensors < 2^20, aligned
 *     tensor size / ALIGN < 2^28, groups per dyo_plan < 2^16, operators < 2^24.
 */
#ifndef DYO_H
#define DYO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  DYO_OK = 0,
  DYO_E_INVAL = -1,       /* bad argument / malformed arch or pilot */
  DYO_E_NOMEM = -2,       /* device or pinned host allocation failed */
  DYO_E_BUDGET = -3,      /* some W_j needs more than half the budget (R7) */
  DYO_E_CUDA = -4,        /* a CUDA runtime call failed (dyo_last_error has the text) */
  DYO_E_STATE = -5,       /* calls out of order (e.g. migrate before plan, j out of order) */
  DYO_E_CAPACITY = -6,    /* a fixed-capacity buffer overflowed (needed size in last_error) */
  DYO_E_UNSUPPORTED = -7  /* program shape not supported by this decode mode */
} dyo_status;

typedef struct dyo_ctx dyo_ctx;

/* Runtime configuration (host struct, copied by dyo_create). */
typedef struct {
  int64_t budget;         /* B: device arena bytes, split in two equal halves (R7) */
  int32_t align;          /* ALIGN in bytes (power of two >= 16; 256 in all configs) */
  int32_t policy;         /* bit 0: 0 = PAPER (evict every unused tensor), 1 = RETAIN (R10);
                             bit 1: SHARE (R20): a W_j tensor valid in the other half that
                             W_{j+1} also holds stays in place (no D2D carry) */
  int32_t max_batch;      /* max predictions per dyo_pilot_predict call (1..1024) */
  int32_t max_groups;     /* max groups per dyo_plan (sum over its predictions), <= 65535 */
  int32_t max_entries;    /* capacity of tensor-set entries per dyo_plan (0 = 512 per group) */
  int32_t max_records;    /* capacity of plan records per dyo_plan (0 = auto) */
  int64_t staging_bytes;  /* device staging for pack/unpack/compaction (outside B; 0 = 64 MiB) */
  int64_t dma_min_bytes;  /* host runs >= this move by DMA, smaller by zero-copy kernel (0 = 2 MiB) */
  int32_t flags;          /* DYO_F_* */
} dyo_config;

#define DYO_F_NO_ZEROCOPY 1   /* move every run by DMA (measurement switch) */
#define DYO_F_NO_PACK 2       /* never pack scattered writebacks into one DMA */
#define DYO_F_NO_HOST_POOL 4  /* plan-only ctx: no pinned host pool (dyo_migrate -> DYO_E_STATE) */
#define DYO_F_TIMING 8        /* record CUDA events around every internal launch (dyo_get_timings) */
#define DYO_F_SM_COPY 16      /* device<->device moves by the SM vector-copy kernel instead of TMA bulk copies */
#define DYO_F_PILOT_TC 32     /* batches >= 16 on K1-TC (tcgen05 kind::tf32, 3xTF32, fp32 accumulation; reading
                               * R14's componentwise tolerance) instead of the default K1 batch path (fp64
                               * DMMA tensor-core tiles, fp64 accumulation: the north_star gate) */
#define DYO_F_STRICT_ORDER 64 /* R12's strict phase order in dyo_migrate: every FETCH waits for the whole EVICT
                               * phase (default: reading R21, a FETCH DMA waits only for block j-2 and the
                               * write-backs whose device range it overwrites) */

/* Static architecture: the DyNN program in preorder, its operators and the
 * tensor table. All arrays are HOST memory; dyo_load_arch copies what it needs. */
typedef struct {
  int32_t nn_type;        /* 0 CNN, 1 LSTM, 2 transformer: selects the MLP */
  int32_t S_max;          /* AFM segments fed to the pilot (R3) */
  int32_t D_s;            /* input-shape descriptors per sample (R3) */
  int32_t h;              /* history groups per sample (R3) */
  int32_t K_max;          /* block-head slots (R4) */
  int32_t branch_head;    /* 1: logits carry a branch head (R4); 0: the paper's traversal decode
                           * (P:L145-L147): dyo_pilot_predict copies the logits to the host,
                           * synchronises its stream once and searches the program's paths
                           * there (top-level sites only, like the device decode) */
  /* program nodes in preorder; node kinds: 0 OP, 1 IF, 2 LOOP, 3 BRANCH (start of an If arm).
   * IF: a = number of branches, followed by that many BRANCH nodes each followed by its body;
   * LOOP: a = lo, b = hi trip count, followed by its body; OP: a = operator index (operators
   * are numbered in preorder). span = number of descendant nodes. tie = index (in preorder
   * among IF/LOOP nodes) of the site whose choice this site replays, or -1 (R6). */
  int32_t n_nodes;
  const int32_t* node_kind;
  const int32_t* node_a;
  const int32_t* node_b;
  const int32_t* node_span;
  const int32_t* node_tie;
  /* operators: six idiom counts (order of P:L135) and input shapes (CSR: op ->
   * inputs -> dims); signature = idioms ++ [sum of shape[k] over inputs, k < 3] (Fig. 3, R1) */
  int32_t n_ops;
  const int32_t* op_idioms;     /* n_ops x 6 */
  const int32_t* op_in_ptr;     /* n_ops + 1 */
  const int32_t* in_dim_ptr;    /* n_inputs + 1 */
  const int64_t* in_dims;
  const int32_t* op_acc_ptr;    /* n_ops + 1: tensor accesses of each operator */
  const int32_t* acc_tensor;    /* ascending tensor id within an operator, unique */
  const int32_t* acc_mode;      /* 1 read, 2 write (full overwrite), 3 read-write */
  /* tensor table */
  int32_t n_tensors;
  const int64_t* t_bytes;       /* > 0 */
  const int64_t* t_host_off;    /* home offset in the ctx's pinned host pool, ALIGN-aligned */
  const int32_t* t_flags;       /* bit 0: transient (contents end with the step, R9) */
  /* per-iteration and per-sample tensors (R13; each may be NULL = all zero): access q of an
   * operator names tensor acc_tensor[q] + acc_stride[q] * k + acc_bstride[q] * b, where k is
   * the iteration index of its LOOP (0..n-1, or n-1..0 when the LOOP node's flags bit 0 is
   * set: a backward pass over a forward loop's tensors) and b the prediction's index in its
   * dyo_pilot_predict batch (e.g. the minibatch row whose input sequence it reads). The named
   * ids must stay in [0, n_tensors) and ascending within the operator for every k < hi and
   * b < max_batch (linear, so checked at the corners; DYO_E_INVAL otherwise); operators outside
   * loops must have acc_stride 0. */
  const int32_t* acc_stride;
  const int32_t* node_flags;
  const int32_t* acc_bstride;
} dyo_arch;

/* Pilot weights (host fp32, row-major W[out][in]); topology R5. n_feature = 0 means an
 * identity feature stage (the MLP reads the F features); otherwise feature layer i maps
 * features [feat_off[i], feat_off[i]+feat_len[i]) to feat_out[i] outputs, concatenated.
 * The three MLPs share layer dims; mlp_W[k*n_mlp + l] is layer l of MLP k. */
typedef struct {
  int32_t F, O;
  int32_t n_feature;
  const int32_t* feat_off;
  const int32_t* feat_len;
  const int32_t* feat_out;
  const float* const* feat_W;
  const float* const* feat_b;
  int32_t n_mlp;
  const int32_t* mlp_in;
  const int32_t* mlp_out;
  const float* const* mlp_W;
  const float* const* mlp_b;
  int32_t out_in;
  const float* out_W;           /* O x out_in */
  const float* out_b;           /* O */
  double slope;                 /* LeakyReLU negative slope (0.01, R5) */
} dyo_pilot_desc;

/* One batch of samples. desc: B x D_s int64 shape descriptors; hist_ids: B x h int32 history
 * group ids (>= 0 index the history table, < 0 count from its end, R3) or NULL (no history).
 * Either pointer may be host or device memory. */
typedef struct {
  const int64_t* desc;
  const int32_t* hist_ids;
} dyo_sample;

/* Host-visible summary of one transition of the current plan (valid after dyo_plan). */
typedef struct {
  int32_t half;                 /* m = (G + j) mod 2 */
  int32_t n_entries;            /* |W_j| */
  int32_t n_evict, n_move, n_carry, n_alloc, n_fetch;
  int64_t need;                 /* aligned bytes of W_j */
  int64_t h2d, d2h, d2d;        /* algorithmic bytes (FETCH; written-back EVICT; MOVE + CARRY) */
  int32_t n_share;              /* R20: W_j tensors left in half 1-m (their entry records' dst) */
  int32_t late_all;             /* R20: 1 if MOVE / CARRY / FETCH wait for block j-1 (compaction of a
                                   half holding tensors block j-1 SHARE'd); dyo_migrate honours it */
} dyo_transition_info;

/* Plan records as stored by libdyo (little-endian int64 fields, absolute device offsets into
 * the arena, host offsets into the host pool). */
typedef struct { int64_t t, src, host_off, bytes, writeback; } dyo_evict_rec;
typedef struct { int64_t t, src, dst, bytes; } dyo_move_rec;
typedef struct { int64_t t, src, dst, bytes, late; } dyo_carry_rec;
typedef struct { int64_t t, dst, bytes; } dyo_alloc_rec;
typedef struct { int64_t t, host_off, dst, bytes; } dyo_fetch_rec;
typedef struct { int64_t t, mode, needs_fetch, dst; } dyo_entry_rec;  /* W_j entry + placement */

const char* dyo_strerror(dyo_status s);
const char* dyo_last_error(const dyo_ctx* ctx);
int32_t dyo_version(void);

/* Create a manager on `device`: allocates the device arena (cfg->budget), staging, status
 * words. Ownership: ctx owns every buffer it allocates; free with dyo_destroy. */
dyo_status dyo_create(const dyo_config* cfg, int32_t device, dyo_ctx** out);
dyo_status dyo_destroy(dyo_ctx* ctx);

/* Load the static architecture (copies it; builds the AFM segment table (R3), operator
 * signatures, site table and tensor table on the device; allocates the pinned, mapped host
 * pool sized to max(host_off + bytes), bound to the GPU's NUMA node - DYO_Q_HOST_NUMA). Resets
 * residency: all tensors on the host. DYO_E_NOMEM if the pool exceeds ~94% of the node's
 * MemAvailable (one manager per GPU pins from the same host RAM), DYO_E_INVAL for a malformed
 * program, DYO_E_UNSUPPORTED for a Loop nested in a dynamic site. */
dyo_status dyo_load_arch(dyo_ctx* ctx, const dyo_arch* arch);

/* Host-only check of an arch (no GPU needed; used by the CPU test suite): runs the same parse
 * as dyo_load_arch and returns its summary, the S_max x 10 AFM segment table (R3) and the
 * n_ops x 9 operator signatures (R1). seg_table / op_sig may be NULL; err (errlen bytes) gets
 * the failure text. */
typedef struct {
  int32_t n_sites, n_branch_logits, n_pieces, F;
  int64_t L_max, host_pool_bytes;
} dyo_arch_summary;
dyo_status dyo_arch_check(const dyo_arch* arch, int32_t align, dyo_arch_summary* out, int32_t* seg_table,
                          int32_t* op_sig, char* err, int32_t errlen);

/* Host-only run of the traversal decode (R4) that dyo_pilot_predict uses when the
 * arch has no branch head (no GPU needed; used by the CPU test suite). slots: K_max x 10 decoded
 * block-head vectors (a slot with count 0 is empty); choices (n_sites int32 out): the choice of
 * every site, preorder; *matched = 1 for an exact match, 0 for the closest-count fallback.
 * DYO_E_UNSUPPORTED for nested control flow (R16 needs a branch head), DYO_E_CAPACITY if the
 * search exceeds its budget. */
dyo_status dyo_traverse_check(const dyo_arch* arch, const int32_t* slots, int32_t* choices, int32_t* matched,
                              char* err, int32_t errlen);

/* Host-only run of the nested-site decode (R16) that dyo_pilot_predict uses for arches with
 * nested sites (no GPU needed; used by the CPU test suite): slots = K_max x 10 decoded block-head
 * vectors, top_choices = the choice of every site in preorder (nested sites ignored). Outputs the
 * nested executions' choices (cap ints; *n_nested), the path's operator per row (path_ops may be
 * NULL; -1 for control rows; *path_len rows) and *matched. DYO_E_STATE if the arch has no nested
 * sites, DYO_E_CAPACITY if an output is too small. */
dyo_status dyo_nested_check(const dyo_arch* arch, const int32_t* slots, const int32_t* top_choices, int32_t* nested,
                            int32_t cap, int32_t* n_nested, int32_t* path_ops, int32_t path_cap, int32_t* path_len,
                            int32_t* matched, char* err, int32_t errlen);

/* Load pilot weights (copied to the device, rows padded to 16 bytes). F and O must match the
 * arch: F = pad16(3 + D_s + 10*S_max + 10*h); O >= 10*K_max + branch logits. */
dyo_status dyo_load_pilot(dyo_ctx* ctx, const dyo_pilot_desc* w);

/* The ctx-owned pinned host pool holding every tensor's home ("initially allocates all
 * tensors on CPU memory"); the caller fills initial contents. Valid until dyo_destroy or the
 * next dyo_load_arch. */
dyo_status dyo_host_pool(dyo_ctx* ctx, void** host_base, int64_t* bytes);
/* Device arena base (2 halves of H bytes each) and H. */
dyo_status dyo_arena(dyo_ctx* ctx, void** dev_base, int64_t* half_bytes);

/* A1: feature vectors of B samples (R3) into feat (device, B x F fp32). Uses the history
 * table of the previous dyo_pilot_predict. */
dyo_status dyo_encode_features(dyo_ctx* ctx, const dyo_sample* s, int32_t B, float* feat,
                               void* stream);

/* A2 + A3: pilot forward for B samples (feat = NULL: fused encode from s; else device B x F
 * features) and decode (R4) into ctx-owned device storage; logits (device B x O fp32 copy of the fp64 logits the decode uses) may be
 * NULL. Asynchronous; decode errors surface at dyo_plan. After the call the history table is
 * the executed block vectors of these predictions (in sample order). */
dyo_status dyo_pilot_predict(dyo_ctx* ctx, const float* feat, const dyo_sample* s, int32_t B,
                             float* logits, void* stream);

/* Copy prediction b of the last dyo_pilot_predict to host arrays (synchronises `stream`).
 * K (groups), blocks (K_max x 10 int32, first K rows valid), choices (n_sites int32),
 * group_rows (2*K_max int32 [start, end) pairs). Any output pointer may be NULL. */
dyo_status dyo_prediction_get(dyo_ctx* ctx, int32_t b, int32_t* K, int32_t* blocks,
                              int32_t* choices, int32_t* group_rows, void* stream);
/* Traversal decode only (arch without a branch head): *matched = 1 if prediction b
 * of the last dyo_pilot_predict matched a path exactly, 0 if the closest-operator-count
 * fallback of P:L147 was taken. DYO_E_STATE with a branch head. Host-side; no sync. */
dyo_status dyo_prediction_matched(dyo_ctx* ctx, int32_t b, int32_t* matched);
/* Nested sites (reading R16: a site inside a top-level loop body or If arm executes once per
 * iteration / arm execution with its own choice; only Ifs with operator-only arms may nest, and
 * only with a branch head - DYO_E_UNSUPPORTED at load otherwise): the choices of prediction b's
 * nested executions in execution order, resolved on the host against the block head by the
 * paper's traversal (exact match, else the closest operator count) - which is also
 * why dyo_pilot_predict synchronises its stream once for such arches. out (host, cap ints) may
 * be NULL to query *n; DYO_E_CAPACITY if cap < *n. *n = 0 for arches without nested sites. The
 * prediction's `choices` (dyo_prediction_get) hold -1 for nested sites; dyo_prediction_matched
 * reports whether the nested resolution matched exactly. */
dyo_status dyo_prediction_nested(dyo_ctx* ctx, int32_t b, int32_t* out, int32_t cap, int32_t* n);

/* Tensor-set entries of group g of prediction b (host out, capacity cap entries of 3 int32:
 * tensor, mode, needs_fetch); *n receives the count (DYO_E_CAPACITY if cap < n). */
dyo_status dyo_group_entries(dyo_ctx* ctx, int32_t b, int32_t g, int32_t* out, int32_t cap,
                             int32_t* n, void* stream);

/* A4: plan every transition of the predictions [b0, b0 + n) of the last predict, concatenated
 * in sample order (n = -1: all). Runs the planner kernel on `stream`, then synchronises once
 * and copies the plan lists to pinned host memory (the DMA issue needs host-visible sizes).
 * On DYO_E_BUDGET / DYO_E_CAPACITY the residency state is unchanged. *K_out = transitions.
 * Plans are double-buffered (plan lookahead): the next step may be predicted and planned while
 * the previous plan's transitions are still migrating - the planned state does not depend on the
 * migrations' progress - so the pilot runs ahead of the batch as in the paper. At most
 * two plans may be outstanding (DYO_E_STATE otherwise); a new plan waits (host) for the
 * migrations of the plan two generations back to finish. In a plan-only ctx
 * (DYO_F_NO_HOST_POOL) each plan supersedes the previous ones. */
dyo_status dyo_plan(dyo_ctx* ctx, int32_t b0, int32_t n, int32_t* K_out, void* stream);
/* dyo_plan in two halves, so the host can enqueue the previous plan's transitions while this
 * plan's kernels run: dyo_plan_async launches the planner (same arguments and checks as dyo_plan,
 * no synchronisation); dyo_plan_wait takes the one synchronisation and commits the plan (K_out,
 * DYO_E_BUDGET / DYO_E_CAPACITY as dyo_plan, state unchanged on error). Between the two only
 * dyo_migrate (of older plans), dyo_fault_* and the read-only queries of the previous plan are
 * allowed; dyo_pilot_predict, dyo_residency and dyo_load_* return DYO_E_STATE, as does a second
 * dyo_plan_async or a dyo_plan_wait without a pending plan. */
dyo_status dyo_plan_async(dyo_ctx* ctx, int32_t b0, int32_t n, void* stream);
dyo_status dyo_plan_wait(dyo_ctx* ctx, int32_t* K_out);

/* Host copies of the most recent plan (valid until the dyo_plan after next). */
dyo_status dyo_plan_info(dyo_ctx* ctx, int32_t j, dyo_transition_info* info);
/* list: 0 evict, 1 move, 2 carry, 3 alloc, 4 fetch, 5 entries (with placement); returns a
 * pointer to the transition's records (host memory owned by the ctx) and their count. */
dyo_status dyo_plan_records(dyo_ctx* ctx, int32_t j, int32_t list, const void** recs,
                            int32_t* n);

/* A5: execute transition j of the OLDEST plan that still has transitions to enqueue (plans
 * migrate in FIFO order; j = 0, 1, ... in order; DYO_E_STATE otherwise):
 *   EVICT writebacks (D2H: DMA per host run, K3 pack + DMA for scattered sources, K5 zero-copy
 *   for small runs) on a ctx-owned D2H stream, after ev_half_free = the end of block j-2, the
 *   last user of half m (NULL: after everything already enqueued on copy_stream); then on
 *   copy_stream: MOVE (compaction through staging), early CARRY (D2D), FETCH (H2D: DMA per host
 *   run or one K5 zero-copy gather), late CARRY after ev_prev_done (end of block j-1; may be
 *   NULL), and finally ev_ready (may be NULL), which block j must wait on.
 * Because EVICT_j only waits for block j-2, it overlaps transition j-1's fetches (P:L176's
 * double buffer; PCIe is full duplex). Reading R21 (default; DYO_F_STRICT_ORDER restores R12's
 * phase order): in a transition without compaction MOVEs and with at most 64 write-backs, each
 * FETCH DMA waits only for ev_half_free and for the write-backs whose device range it overwrites,
 * so the H2D link starts while later write-backs still run D2H; CARRYs, zero-copy fetches and
 * ev_ready still follow the whole EVICT phase. The plan (layout, records, bytes) is unchanged.
 * A late_all transition (R20) runs MOVE / CARRY / FETCH after ev_prev_done.
 * Host-non-blocking; all transitions of a plan may be enqueued at once. */
dyo_status dyo_migrate(dyo_ctx* ctx, int32_t j, void* copy_stream, void* ev_half_free,
                       void* ev_prev_done, void* ev_ready);

/* ---- On-demand fetch of mis-predicted tensors ("checks whether the tensor
 * is in GPU memory ... migrates the tensors on demand", P:L197 tensor fault handler; DESIGN.md
 * reading R17) --------------------------------------------------------------------------------
 * When the pilot mis-predicts, block j (the rows [C_j, C_j+1) of the ACTUAL path, cut at the
 * predicted counts: the operator counter of P:L178) touches tensors the plan did not make
 * ready. Before block j runs, the runtime passes the actual accesses that may be missing.
 * dyo_fault_config: allocates the device fault area (outside B; two halves used by alternate
 *   blocks); 0 frees it. Synchronises the device.
 * dyo_fault_fetch: j = the transition last enqueued by dyo_migrate (block j is next to run;
 *   DYO_E_STATE otherwise - with faults the runtime enqueues transitions one block ahead).
 *   For each id (modes: 1 read, 2 write, 3 read-write), dev_ptrs[i] (host array) receives:
 *     - the tensor's planned slot if it is in the planned W_j and that entry is valid for the
 *       access (read-first in the plan or a write-first access, and a write only where the plan
 *       writes): the residency check;
 *     - else a fault-area copy: read-first accesses copy the tensor's latest bytes - from its
 *       valid device copy after transition j (for a tensor the plan ALLOCs in this transition,
 *       its copy before it), else from its host home - on `stream`, after transition j's
 *       migrations; ev_done (may be NULL) is recorded after the copies: block j waits on it.
 *   `ids` must list every access of the actual block (not only the suspected misses): a tensor
 *   the plan ALLOCs at transition j (slot not filled, treated as dirty afterwards) that the
 *   actual block does not write through its slot gets its latest bytes copied into that slot
 *   (the repair), so no later write-back publishes stale bytes.
 *   Written faulted tensors are written back after block j ends, by the next dyo_migrate
 *   (after its ev_prev_done): to the host home and to the tensor's valid device copy, before
 *   that transition's EVICT and carries. The plan's residency is never changed, so plans
 *   computed ahead stay valid. DYO_E_CAPACITY if a block's faults exceed half the area.
 * dyo_fault_stats: faults served from the fault area, their bytes copied in, and accesses
 *   found resident (any pointer may be NULL). */
dyo_status dyo_fault_config(dyo_ctx* ctx, int64_t area_bytes);
dyo_status dyo_fault_fetch(dyo_ctx* ctx, int32_t j, const int32_t* ids, const int32_t* modes, int32_t n,
                           void** dev_ptrs, void* stream, void* ev_done);
dyo_status dyo_fault_stats(dyo_ctx* ctx, int64_t* faults, int64_t* bytes, int64_t* resident);
/* Enqueues the pending write-backs of the last block's written faulted tensors on `stream`
 * after ev_block_end (may be NULL) - what the next dyo_migrate would do; for the last block of
 * a run. No-op without pending write-backs. */
dyo_status dyo_fault_flush(dyo_ctx* ctx, void* stream, void* ev_block_end);
/* Fault injection (tests / measurement): from the next dyo_plan on, every read-first entry of the
 * planned predictions whose splitmix64 hash of (seed, prediction, group slot, tensor) is below
 * p x 2^64 is dropped before planning (workloads.drop_prefetch is the test side's twin), so the
 * runtime faults it in. p < 0 restores the DYO_FAULT=drop_prefetch:p[:seed] environment
 * setting (default off); p = 0 disables. DYO_E_INVAL for p > 1. */
dyo_status dyo_fault_inject(dyo_ctx* ctx, double p, uint64_t seed);

/* ---- Partition labels (§IV-D: Sentinel-style labels that "maximize the
 * overlap between tensor migration and training computation without violating the GPU memory
 * capacity"; §V L203-L205 the partition simulator; §VI-G L275 the heuristics; R18) ----
 * One sample's execution trace: L rows of the loaded arch (path_ops: operator per row, -1 for a
 * control row; path_it: the row's iteration index, R13; b: the per-sample binding), compute time
 * per operator op_time_ns (n_ops int64, host). Block j = rows [c_j, c_j+1) needs the aligned bytes
 * of its tensor set (<= H), migrates the bytes of the tensors it reads first, and hides that
 * migration (ceil(bytes * 1000 / bw) ns, bw in bytes per microsecond) behind block j-1's compute;
 * exposed = sum over j >= 1 of max(0, migration_j - compute_j-1).
 * method 0: the overlap partition - minimum exposed time over K-block partitions within the
 *   capacity, the lexicographically smallest cut vector among the minimisers (GPU dynamic
 *   programming over (block, previous block start, block end));
 * method 1 / 2 / 3: even operators / even compute time / even accessed bytes (cut j after the
 *   longest prefix holding at most j/K of the total, kept non-empty).
 * cuts (host, K+1 ints) receives 0 = c_0 < ... < c_K = L, *exposed the ns, *feasible (may be
 * NULL) whether every block fits H (method 0: 0 and *exposed = -1 when none does). L <= 4096;
 * synchronises `stream`. DYO_E_CAPACITY if a block start meets more than 4096 distinct tensors. */
dyo_status dyo_partition(dyo_ctx* ctx, const int32_t* path_ops, const int32_t* path_it, int32_t L, int32_t b,
                         const int64_t* op_time_ns, int32_t K, int32_t method, int64_t H, int64_t bw, int32_t* cuts,
                         int64_t* exposed, int32_t* feasible, void* stream);

/* ---- Pilot training (§IV-D, §V: LeakyReLU, SGD, learning rate 0.01;
 * DESIGN.md reading R19) ------------------------------------------------------------------
 * A trainer holds an fp64 copy of a pilot (the weights of w, widened exactly) and trains the
 * feature layers, the MLP of nn_type (the only one that runs) and the output layer.
 * dyo_trainer_step: one SGD step on a minibatch - feat (device, B x F fp32: dyo_encode_features
 *   output) and target (device, B x O fp32: label block vectors in R4 block-head units and
 *   one-hot branch choices) - on L = (1/(B O)) sum (y - t)^2, on `stream`; *loss (may be NULL)
 *   receives the loss before the step (synchronises the stream). B <= max_batch.
 * dyo_trainer_export: every weight array of the pilot in dyo_pilot_desc order (feature layers
 *   W then b; MLP k = 0..2, layer l: W then b; out W then b) into blob (host fp64, cap doubles;
 *   NULL to query *n); the untrained MLPs keep their weights. Synchronises the device.
 * Deterministic: every sum runs in a fixed order. */
typedef struct dyo_trainer dyo_trainer;
dyo_status dyo_trainer_create(const dyo_pilot_desc* w, int32_t nn_type, int32_t max_batch, int32_t device,
                              dyo_trainer** out);
dyo_status dyo_trainer_step(dyo_trainer* tr, const float* feat, const float* target, int32_t B, double lr,
                            double* loss, void* stream);
dyo_status dyo_trainer_export(dyo_trainer* tr, double* blob, int64_t cap, int64_t* n);
dyo_status dyo_trainer_destroy(dyo_trainer* tr);

/* The resolved path (R2 rows: operator per row, -1 for a control row; iteration index per row,
 * R13) of the loaded arch for the given site choices (n_sites ints, preorder; nested sites
 * ignored) and nested executions' choices (R16, execution order) - the execution trace of a
 * sample whose control flow is known (partition labels, R18). Host-only; DYO_E_CAPACITY with the
 * needed length in *L if cap is too small. */
dyo_status dyo_trace_path(dyo_ctx* ctx, const int32_t* choices, const int32_t* nested, int32_t n_nested, int32_t* ops,
                          int32_t* its, int32_t cap, int32_t* L);

/* Device address of tensor t after the last planned transition that placed it (NULL if it is
 * on the host). Valid until the next dyo_migrate that moves it. */
dyo_status dyo_residency(dyo_ctx* ctx, int32_t t, void** dev_ptr);

/* Introspection of the last calls (tests and measurement; host-only, no synchronisation).
 *   DYO_Q_PILOT_KERNEL: kernel the last dyo_pilot_predict ran: 0 = K1 (cluster GEMV at batch < 8,
 *     fp64 DMMA tensor-core tiles at batch >= 8; fp64 accumulation), 1 = K1-TC (tcgen05 3xTF32,
 *     opt-in DYO_F_PILOT_TC, batch >= 16).
 *   DYO_Q_DECODE_FUSED: 1 if the last dyo_pilot_predict decoded in K1's epilogue, 0 if it
 *     launched the stand-alone decode kernels.
 *   DYO_Q_PLAN_SYNCS: host synchronisations taken by the last successful dyo_plan (1, §8(b)).
 *   DYO_Q_HOST_DECODE: 1 if the loaded arch's decode runs on the host (no branch head, or nested
 *     sites: dyo_pilot_predict synchronises its stream once, so it cannot be graph-captured).
 *   DYO_Q_HOST_NUMA: NUMA node the pinned host pool is bound to (survey §8(e): each GPU's
 *     manager uses its own host link): the node sysfs reports for the device's PCI address (or
 *     $DYO_HOST_NUMA), pages bound with mbind before cudaHostRegister; -1 if the platform reports
 *     no node or binding failed, in which case the pool is a plain cudaHostAlloc.
 * DYO_E_INVAL for a NULL ctx / value or an unknown `what`. */
/* Measurement switch at run time: sets or clears DYO_F_TIMING (the only flag that may change
 * after dyo_create; DYO_E_INVAL for any other bit). With it clear no timing events are recorded,
 * so a headline measurement runs uninstrumented and a second pass gets the breakdown. */
dyo_status dyo_set_timing(dyo_ctx* ctx, int32_t on);

#define DYO_Q_PILOT_KERNEL 0
#define DYO_Q_DECODE_FUSED 1
#define DYO_Q_PLAN_SYNCS 2
#define DYO_Q_HOST_DECODE 3
#define DYO_Q_HOST_NUMA 4
dyo_status dyo_query(dyo_ctx* ctx, int32_t what, int64_t* value);

/* Per-ctx counters of the last dyo_plan / dyo_migrate calls (bytes by mechanism, launches). */
typedef struct {
  int64_t h2d_dma, h2d_zc, d2h_dma, d2h_zc, d2h_packed, d2d;
  int64_t n_dma, n_kernels;
} dyo_counters;
dyo_status dyo_get_counters(dyo_ctx* ctx, dyo_counters* c, int32_t reset);

/* With DYO_F_TIMING: device time (CUDA events on the launching stream) summed over the launches
 * of one kind since the last reset: 0 pilot kernel (K1), 1 decode kernels, 2 planner kernel (K2),
 * 3 device copy kernel (pack / unpack / carry / compaction), 4 zero-copy kernel (K5),
 * 5 DMA H2D, 6 DMA D2H. bytes = algorithmic bytes moved by those launches; busy_ms = length of
 * the union of their [start, end] intervals (launches of one kind on different streams overlap).
 * Any output may be NULL. reset also records the reference event the intervals are measured
 * from. Synchronises on the recorded events. */
#define DYO_T_KINDS 7
dyo_status dyo_get_timings(dyo_ctx* ctx, int32_t kind, double* ms, int64_t* launches, int64_t* bytes,
                           double* busy_ms, int32_t reset);

/* Debugging / measurement aid: copy `bytes` device->device (or through mapped host memory) with
 * the library's segment-copy kernel: mode 0 = SM vector copies (K5 path), 1 = TMA bulk copies
 * (K3/K4 path). Synchronises `stream`. */
dyo_status dyo_debug_copy(dyo_ctx* ctx, const void* src, void* dst, int64_t bytes, int32_t mode, void* stream);

/* Debugging aid: enable (1) / disable (0) phase stamps of the pilot kernel and read the 32
 * stamps of the last launch (out32 may be NULL): SM clock cycles for the cluster GEMV kernel,
 * %globaltimer ns for the tensor-core batch kernel (K1-TC). Synchronises the device. */
dyo_status dyo_debug_pilot_stamps(dyo_ctx* ctx, int32_t enable, uint64_t* out32);
/* Debugging aid: clock64 stamps of the planner's phases for transition j of the next dyo_plan
 * (j = -1 disables); out64 (64 entries, may be NULL) receives the stamps of the last plan. */
dyo_status dyo_debug_plan_stamps(dyo_ctx* ctx, int32_t j, uint64_t* out64);
/* ---- Mis-prediction handling (§IV-E "Handling mis-prediction", §VI-H
 * P:L280; reading R15) ------------------------------------------------------------
 * The pilot may mis-predict the control flow. After a sample has executed, the runtime reports
 * the control flow that actually ran; the library records the mis-prediction (the paper's
 * training record: a count here) and memoises it: "the output of the pilot model is compared
 * with the output where there is mis-prediction. If the two outputs are exactly the same, then
 * the correct execution block in the mis-prediction case is used to resolve the control flows"
 * (P:L186-L187). The compared output is the decoded integer pilot output of a prediction: its
 * raw block head (K_max x 10 ints, reading R4) and its own branch-head choices. A later
 * prediction with exactly that output is decoded with the memoised actual choices (inside the
 * decode kernels: a 64-bit key hash probes a device open-addressing table, then the full key is
 * compared); its groups are cut from the actual path at the predicted counts.
 *
 * dyo_memo_config: (re)allocates the memo for `capacity` entries (0 disables it; default
 *   disabled). FIFO replacement of the oldest key when full; a re-reported key keeps its most
 *   recent value. Requires dyo_load_arch (DYO_E_STATE); reset by it. Synchronises the device.
 * dyo_report: `actual` (host, n_sites ints, site order of the branch head; a tied site must
 *   replay its target, R6) is compared with the FINAL choices of prediction b (0 <= b < the B of
 *   the last dyo_pilot_predict). *mispredicted (may be NULL) = 1 if they differ. On a
 *   mis-prediction the count is incremented and, with the memo enabled, the prediction's raw
 *   output -> actual choices is memoised (host mirror + device table). DYO_E_INVAL on a bad b or
 *   an invalid choice vector. Stream-ordered: waits (host) only for the end of the last
 *   dyo_pilot_predict (the prediction being reported), reads it back on a ctx-owned stream, and
 *   uploads a new memo entry on that stream; the next dyo_pilot_predict waits for the upload on
 *   the device (no device-wide synchronisation). Branch-head arches only (with the traversal decode the memo is not consulted).
 * dyo_memo_stats: mis-predictions reported so far (since dyo_load_arch), live memo entries, and
 *   memo hits taken by the decode kernels (device counter). Any pointer may be NULL. */
dyo_status dyo_memo_config(dyo_ctx* ctx, int32_t capacity);
dyo_status dyo_report(dyo_ctx* ctx, int32_t b, const int32_t* actual, int32_t* mispredicted);
dyo_status dyo_memo_stats(dyo_ctx* ctx, int64_t* mispredictions, int32_t* live, int64_t* hits);

/* Measurement aid for the batch-1 pilot's latency floor (survey section 8(d)): launches, on
 * `stream`, an otherwise empty kernel with the pilot's launch shape (one cluster of `cluster`
 * CTAs x 512 threads, the pilot's dynamic shared memory) that performs `n_barriers`
 * cluster-wide barriers (one per dependent layer stage). Asynchronous; capturable in a CUDA
 * graph. DYO_E_INVAL if cluster is not 1..16 or n_barriers < 0. */
dyo_status dyo_debug_floor(dyo_ctx* ctx, int32_t cluster, int32_t n_barriers, void* stream);

/* Measurement aid for the live rate of the record-copy kernel (survey section 8(d), migrate row):
 * with DYO_COPY_STAMPS=1 in the environment (read at the first copy launch of the process) every
 * CTA of copy_records_tma_kernel appends 4 x u64 {launch << 32 | cta << 8 | smid, globaltimer at
 * entry, after its record scan, at exit} to a device log of up to 2^22 - 1 entries. This call
 * synchronises the device and copies min(count, cap) entries (4 x u64 each, caller-owned host
 * buffer `out`) and stores that number in *n (0 when stamps are off); out == NULL with cap == 0
 * empties the log instead (*n = 0).
 * DYO_E_INVAL on NULL ctx / n or cap < 0; DYO_E_CUDA if the readback fails. */
dyo_status dyo_debug_copy_stamps(dyo_ctx* ctx, uint64_t* out, int64_t cap, int64_t* n);

#ifdef __cplusplus
}
#endif
#endif /* DYO_H */
