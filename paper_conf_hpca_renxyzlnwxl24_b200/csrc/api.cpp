// libdyo C ABI: context, loaders, the four hot-path calls and the migration engine.
// See include/dyo.h for the contract and DESIGN.md for the readings R1-R12.
#include <cuda_runtime.h>

#include <algorithm>
#include <array>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <unordered_map>
#include <vector>

#include <cctype>
#include <sys/mman.h>
#include <sys/syscall.h>
#include <unistd.h>

#include "dyo_internal.h"

using namespace dyo;

constexpr int64_t kChunk = 256 << 10;   // copy-kernel work item

struct dyo_ctx {
  dyo_config cfg{};
  int device = 0;
  std::string err;
  bool arch_ok = false, pilot_ok = false;
  // host copy of the arch
  int T = 0, n_ops = 0, n_sites = 0, K_max = 0, F = 0, O_min = 0, n_branch_logits = 0;
  std::vector<int64_t> t_bytes, t_abytes, t_host;
  std::vector<int32_t> t_flags;
  int64_t H = 0;
  ArchDev ad{};
  std::vector<void*> arch_dev;     // device buffers of the arch / prediction / plan
  struct Slab { std::vector<void*>* owner = nullptr; char* p = nullptr; size_t left = 0; } slab[2];
  PilotDev pdv{};
  const PilotDev* pdv_dev = nullptr;    // device copy of pdv
  std::vector<void*> pilot_dev;
  // memory
  char* arena = nullptr;
  char* staging = nullptr;
  int64_t staging_bytes = 0;
  char* host_pool = nullptr;
  int64_t host_bytes = 0;
  int host_numa = -1;              // NUMA node the pool was bound to (-1: unbound, cudaHostAlloc)
  bool host_registered = false;    // pool = mmap + mbind + cudaHostRegister (free with munmap)
  // prediction
  PredDev pd{};
  double* logits64 = nullptr;      // fp64 logits (decode decisions, R4)
  // traversal decode (no branch head): host copy of the program tables, pinned
  // logits / choices staging and the device choices the decode kernel replays
  int branch_head = 1;
  TravArch trav;
  // nested sites (R16): the host resolves every prediction's path after the pilot
  int nested = 0;
  NestArch nest;
  std::vector<int32_t> site_logit;            // host copy: logit offset of each site (-1: none)
  int32_t* h_path = nullptr;                  // pinned: B x L_max ops | B x L_max iterations | B lengths
  std::vector<std::vector<int32_t>> last_nested;   // nested executions' choices of each prediction
  // exact-match mis-prediction memo (R15): host mirror of the device table (ad.memo_*)
  struct Memo {
    int cap = 0, kw = 0, ns = 0, mask = 0, live = 0, tomb = 0;
    std::vector<uint64_t> hash;
    std::vector<int32_t> key, val, index, id_slot;
    std::vector<int> fifo;            // live entry ids, oldest first
    std::vector<int> free_ids;
    int64_t mispredictions = 0;
    std::vector<void*> dev;           // index, hash, key, val, hits
  } memo;
  double* h_logits = nullptr;      // pinned, max_batch x O
  int32_t* h_forced[2] = {nullptr, nullptr};   // pinned, max_batch x n_sites (alternating)
  int32_t* d_forced = nullptr;
  int32_t* h_matched = nullptr;    // per prediction of the last traversal: 1 exact match
  // K1-TC (tensor-core batch pilot): device plan, or null when the pilot's shape does not fit it
  const TcPlan* tc_dev = nullptr;
  int tc_flag_off = 0;             // DYO_PILOT_TC=0 in the environment disables it (measurement)
  int last_tc = 0;                 // the last dyo_pilot_predict ran K1-TC
  int last_fused = 0;              // the last dyo_pilot_predict decoded in K1's epilogue
  int64_t last_plan_syncs = 0;     // host synchronisations taken by the last dyo_plan
  // stream-ordered mis-prediction reports (R15): the report / stats readbacks and the memo
  // uploads run on `aux`; ev_pred marks the end of the last dyo_pilot_predict, ev_memo the last
  // memo upload (the next predict waits on it)
  cudaStream_t aux = nullptr;
  cudaEvent_t ev_pred = nullptr, ev_memo = nullptr;
  bool memo_pending = false;
  int32_t* h_rep = nullptr;        // pinned readback of a report (status, choices, key)
  char* h_memo_stage = nullptr;    // pinned staging of a memo upload (entry + index)
  size_t h_memo_stage_bytes = 0;
  int64_t* desc_dev = nullptr;
  int32_t* hist_dev = nullptr;
  int32_t* hist_tab[2] = {nullptr, nullptr};
  int32_t* hist_K[2] = {nullptr, nullptr};   // groups per prediction of each history table
  int hist_B[2] = {0, 0};                    // predictions in each history table
  int hist_cur = 0;
  int last_B = 0;
  // plan
  int max_groups = 0;
  PlanState state[2]{};
  int committed = 0;
  PlanScratch sc{};
  // Two plan slots: dyo_plan fills slot (plan_seq & 1) while the previous plan may still be
  // migrating (plan lookahead); dyo_migrate continues the oldest plan with transitions left.
  struct PlanSlot {
    PlanOut out{};                 // host (pinned) mirrors of the plan records + headers
    PlanOut dout{};                // device record arrays the planner kernel writes
    PlanOut hout{};                // device-side aliases of the pinned mirrors (export kernel)
    CopySeg* h_segs = nullptr;     // pinned mapped work items for the copy kernels
    int64_t seg_cap = 0, seg_used = 0;
    int K = 0, next_j = 0;
    bool valid = false;
    cudaEvent_t ev_last = nullptr; // recorded after every migrate of this plan
    bool ev_pending = false;
    bool ent_host = false;         // entry records copied to out.ent (lazily, dyo_plan_records)
    int64_t n_ent = 0;
  };
  PlanSlot slot[2];
  int64_t plan_seq = 0, mig_seq = 0;
  int32_t* h_status = nullptr;     // pinned mapped
  int32_t* h_counts = nullptr;
  int8_t* h_loc = nullptr;         // pinned mirrors of the committed residency
  int64_t* h_off = nullptr;

  // on-demand fetch of mis-predicted tensors (reading R17)
  char* fault_area = nullptr;
  int64_t fault_cap = 0, fault_used = 0;
  int fault_j = -1;                          // block whose faults occupy the area
  struct FaultWb { int32_t t; char* src; };
  std::vector<FaultWb> fault_wb;             // written faulted tensors of the last block
  cudaEvent_t ev_fault_wb = nullptr;
  int64_t n_faults = 0, fault_bytes = 0, n_fault_resident = 0, n_fault_repair = 0;
  // copy descriptors of the fault copies: two halves alternating between blocks like the fault
  // area; the host rewrites a half only after the launch that read it (ev_fseg) has run
  CopySeg* fault_segs = nullptr;
  int64_t fseg_cap = 0, fseg_used = 0;
  cudaEvent_t ev_fseg[2] = {nullptr, nullptr};
  double drop_p = -1.0;                      // dyo_fault_inject (< 0: DYO_FAULT environment)
  unsigned long long drop_seed = 0;
  // host replay of the residency after every migrated transition (FIFO over plans)
  std::vector<int8_t> mig_loc;
  std::vector<int64_t> mig_off;
  std::vector<std::pair<int32_t, std::pair<int8_t, int64_t>>> mig_prev_alloc;   // ALLOC'd in the last transition
  PlanSlot* last_mig_slot = nullptr;
  int last_mig_j = -1;
  int64_t last_mig_seq = -1;
  // partition labels (R18): device scratch grown on demand
  void* part_buf = nullptr;
  size_t part_bytes = 0;
  // migration
  cudaStream_t d2h = nullptr;      // ctx-owned stream for the EVICT (D2H) phase
  cudaStream_t side = nullptr;     // ctx-owned stream for early CARRY (overlaps FETCH)
  cudaEvent_t ev_entry = nullptr, ev_evict = nullptr, ev_moves = nullptr, ev_carry = nullptr;
  std::vector<cudaEvent_t> ev_wb;   // R21: one per write-back copy group of a transition (D2H stream order)
  cudaStream_t join = nullptr;      // R21: ready[j] = FETCH_j + EVICT_j joined off the copy stream
  bool plan_pending = false;        // dyo_plan_async issued, dyo_plan_wait not yet called
  cudaStream_t plan_stream = nullptr;
  unsigned int* gbar = nullptr;     // grid-barrier counter of the multi-wave compaction launches
  unsigned int gbar_issued = 0;     // arrivals the launches enqueued so far (stream order on copy_stream)
  cudaEvent_t ev_tail = nullptr;
  dyo_counters ctr{};
  int sm_count = 148;
  // DYO_F_TIMING: event pairs per launch kind
  struct Tm { int kind; cudaEvent_t a, b; int64_t bytes; };
  std::vector<Tm> tm;
  std::vector<cudaEvent_t> ev_pool;
  double tm_ms[DYO_T_KINDS] = {};
  int64_t tm_n[DYO_T_KINDS] = {}, tm_bytes[DYO_T_KINDS] = {};
  cudaEvent_t ev_ref = nullptr;                           // timing reference (recorded at reset)
  std::vector<std::pair<double, double>> tm_iv[DYO_T_KINDS];  // [start, end] ms after ev_ref
};

namespace {

dyo_status fail(dyo_ctx* c, dyo_status s, const char* fmt, ...) {
  if (c) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    c->err = buf;
  }
  return s;
}

#define CK(call)                                                                          \
  do {                                                                                    \
    cudaError_t e_ = (call);                                                              \
    if (e_ != cudaSuccess)                                                                \
      return fail(ctx, e_ == cudaErrorMemoryAllocation ? DYO_E_NOMEM : DYO_E_CUDA,        \
                  "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__);   \
  } while (0)

template <class T>
dyo_status dalloc(dyo_ctx* ctx, std::vector<void*>& owner, T** p, size_t n) {
  // Small buffers are carved (256-byte aligned) from 16 MiB slabs owned by `owner`, so the
  // kernels' many small tables share a handful of pages (fewer TLB misses on the dependent
  // lookups of the decode and planner); large buffers get their own allocation.
  constexpr size_t kSlab = 16u << 20, kSmall = 2u << 20;
  size_t bytes = std::max<size_t>(n * sizeof(T), 16);
  void* v = nullptr;
  if (bytes <= kSmall) {
    dyo_ctx::Slab* sl = nullptr;
    for (auto& c : ctx->slab)
      if (c.owner == &owner) sl = &c;
    if (!sl) {
      sl = ctx->slab[0].owner == nullptr || ctx->slab[0].owner == &owner ? &ctx->slab[0] : &ctx->slab[1];
      *sl = dyo_ctx::Slab{};
      sl->owner = &owner;
    }
    bytes = (bytes + 255) / 256 * 256;
    if (sl->left < bytes) {
      void* blk = nullptr;
      CK(cudaMalloc(&blk, kSlab));
      owner.push_back(blk);
      sl->p = static_cast<char*>(blk);
      sl->left = kSlab;
    }
    v = sl->p;
    sl->p += bytes;
    sl->left -= bytes;
  } else {
    CK(cudaMalloc(&v, bytes));
    owner.push_back(v);
  }
  CK(cudaMemset(v, 0, bytes));
  *p = static_cast<T*>(v);
  return DYO_OK;
}

template <class T>
dyo_status dupload(dyo_ctx* ctx, std::vector<void*>& owner, const T** p, const std::vector<T>& h) {
  T* d = nullptr;
  dyo_status s = dalloc(ctx, owner, &d, h.size());
  if (s) return s;
  if (!h.empty()) CK(cudaMemcpy(d, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice));
  *p = d;
  return DYO_OK;
}

void free_list(std::vector<void*>& v) {
  for (void* p : v) cudaFree(p);
  v.clear();
}
// free an owner's buffers and forget its slab (the next small allocation starts a new one)
void free_owned(dyo_ctx* ctx, std::vector<void*>& v) {
  free_list(v);
  for (auto& c : ctx->slab)
    if (c.owner == &v) c = dyo_ctx::Slab{};
}

int64_t align_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

// DYO_TRACE=1: one line per migration operation on stderr (debugging hangs / ordering)
bool trace_on() {
  static int v = -1;
  if (v < 0) { const char* e = getenv("DYO_TRACE"); v = (e && *e == '1') ? 1 : 0; }
  return v == 1;
}
#define TRACE(...) do { if (trace_on()) { fprintf(stderr, "[dyo] " __VA_ARGS__); fputc('\n', stderr); fflush(stderr); } } while (0)

bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes at{};
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

void free_plan_host(dyo_ctx* c) {
  auto fh = [](void* p) { if (p) cudaFreeHost(p); };
  for (auto& P : c->slot) {
    fh(P.out.hdr); fh(P.out.ent); fh(P.out.ev); fh(P.out.mv); fh(P.out.ca); fh(P.out.al); fh(P.out.fe);
    fh(P.h_segs);
    P.out = PlanOut{};
    P.dout = PlanOut{};
    P.h_segs = nullptr;
    P.valid = false;
    P.K = P.next_j = 0;
    P.seg_used = 0;
  }
  fh(c->h_status); fh(c->h_counts); fh(c->h_loc); fh(c->h_off);
  fh(c->h_forced[0]); fh(c->h_forced[1]); fh(c->h_matched); fh(c->h_rep); fh(c->h_path);
  c->h_rep = nullptr;
  c->h_path = nullptr;
  c->h_forced[0] = c->h_forced[1] = c->h_matched = nullptr;
  c->h_status = c->h_counts = nullptr;
  c->h_loc = nullptr;
  c->h_off = nullptr;
  c->plan_seq = c->mig_seq = 0;
}

// timing helpers (no-ops unless DYO_F_TIMING)
cudaEvent_t pool_event(dyo_ctx* c) {
  if (!c->ev_pool.empty()) { cudaEvent_t e = c->ev_pool.back(); c->ev_pool.pop_back(); return e; }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}
struct TScope {
  dyo_ctx* c; int kind; cudaStream_t s; int64_t bytes; cudaEvent_t a = nullptr;
  TScope(dyo_ctx* c_, int k, cudaStream_t s_, int64_t b = 0) : c(c_), kind(k), s(s_), bytes(b) {
    if (c->cfg.flags & DYO_F_TIMING) { a = pool_event(c); cudaEventRecord(a, s); }
  }
  ~TScope() {
    if (a) {
      cudaEvent_t b = pool_event(c);
      cudaEventRecord(b, s);
      c->tm.push_back({kind, a, b, bytes});
    }
  }
};

void drain_timings(dyo_ctx* c) {
  for (auto& t : c->tm) {
    cudaEventSynchronize(t.b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, t.a, t.b);
    if (c->ev_ref) {
      float t0 = 0.f, t1 = 0.f;
      if (cudaEventElapsedTime(&t0, c->ev_ref, t.a) == cudaSuccess &&
          cudaEventElapsedTime(&t1, c->ev_ref, t.b) == cudaSuccess)
        c->tm_iv[t.kind].push_back({t0, t1});
      cudaGetLastError();
    }
    c->tm_ms[t.kind] += ms;
    c->tm_n[t.kind] += 1;
    c->tm_bytes[t.kind] += t.bytes;
    c->ev_pool.push_back(t.a);
    c->ev_pool.push_back(t.b);
  }
  c->tm.clear();
}

// Host-side parse of a dyo_arch (no CUDA): signatures (Fig. 3, R1), AFM segment table (R3),
// sites / arms / top-level pieces (R2, R4, R6), tensor table. Shared by dyo_load_arch and
// dyo_arch_check.
struct ArchHost {
  int T = 0, n_sites = 0, n_branch_logits = 0;
  int64_t L_max = 0, pool = 0;
  std::vector<int64_t> t_bytes, t_abytes, t_host;
  std::vector<int32_t> t_flags, sig, acc_ptr, acc_t, acc_m, acc_s, acc_sb, site_rev;
  std::vector<int32_t> site_kind, site_nch, site_lo, site_tie, site_logit, site_arm_ptr, arm_first, arm_n;
  std::vector<int32_t> piece_kind, piece_a, piece_b, piece_c, seg_table;
  int nested = 0;            // 1: some sites are nested (R16): the host resolves the paths
  NestArch nest;
};

dyo_status hfail(std::string& err, dyo_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  err = buf;
  return s;
}

dyo_status parse_arch(const dyo_arch* A, int64_t AL, int max_b, ArchHost& h, std::string& err) {
  if (A->nn_type < 0 || A->nn_type > 2 || A->S_max < 0 || A->D_s < 0 || A->h < 0 || A->K_max < 1 ||
      A->K_max > 256 || A->n_tensors < 1 || A->n_tensors >= (1 << 20) || A->n_ops < 0 ||
      A->n_ops >= (1 << 24) || A->n_nodes < 0)
    return hfail(err, DYO_E_INVAL, "arch: bad sizes");
  const int T = A->n_tensors, n_ops = A->n_ops, N = A->n_nodes;
  // ---- tensors ----
  h.T = T;
  h.t_bytes.assign(A->t_bytes, A->t_bytes + T);
  h.t_host.assign(A->t_host_off, A->t_host_off + T);
  h.t_flags.assign(A->t_flags, A->t_flags + T);
  h.t_abytes.resize(T);
  int64_t& pool = h.pool;
  pool = 0;
  for (int t = 0; t < T; ++t) {
    if (h.t_bytes[t] <= 0 || h.t_host[t] < 0 || h.t_host[t] % AL)
      return hfail(err, DYO_E_INVAL, "arch: tensor %d bytes/host_off invalid", t);
    h.t_abytes[t] = align_up(h.t_bytes[t], AL);
    if (h.t_abytes[t] / AL >= (1ll << 28)) return hfail(err, DYO_E_INVAL, "arch: tensor %d too large", t);
    pool = std::max(pool, h.t_host[t] + h.t_abytes[t]);
  }
  if (pool / AL >= (1ll << 42)) return hfail(err, DYO_E_INVAL, "arch: host pool too large");
  // ---- operators: signatures (Fig. 3 / R1) and accesses ----
  auto& sig = h.sig; auto& acc_ptr = h.acc_ptr; auto& acc_t = h.acc_t; auto& acc_m = h.acc_m;
  sig.assign((size_t)n_ops * 9, 0);
  acc_ptr.assign(n_ops + 1, 0);
  for (int o = 0; o < n_ops; ++o) {
    for (int k = 0; k < 6; ++k) {
      int64_t v = A->op_idioms[o * 6 + k];
      sig[o * 9 + k] = (int32_t)std::min<int64_t>(std::max<int64_t>(v, 0), kSat);
    }
    for (int k = 0; k < 3; ++k) {
      int64_t s = 0;
      for (int i = A->op_in_ptr[o]; i < A->op_in_ptr[o + 1]; ++i) {
        const int rank = A->in_dim_ptr[i + 1] - A->in_dim_ptr[i];
        if (rank > k) s += A->in_dims[A->in_dim_ptr[i] + k];
      }
      sig[o * 9 + 6 + k] = (int32_t)std::min<int64_t>(std::max<int64_t>(s, 0), kSat);
    }
    acc_ptr[o] = (int32_t)acc_t.size();
    int prev = -1;
    for (int q = A->op_acc_ptr[o]; q < A->op_acc_ptr[o + 1]; ++q) {
      const int t = A->acc_tensor[q], md = A->acc_mode[q];
      if (t < 0 || t >= T || t <= prev || md < 1 || md > 3)
        return hfail(err, DYO_E_INVAL, "arch: op %d accesses must be ascending unique tensor ids with mode 1..3", o);
      prev = t;
      acc_t.push_back(t);
      acc_m.push_back(md);
      h.acc_s.push_back(A->acc_stride ? A->acc_stride[q] : 0);
      h.acc_sb.push_back(A->acc_bstride ? A->acc_bstride[q] : 0);
    }
  }
  acc_ptr[n_ops] = (int32_t)acc_t.size();
  // ---- program: sites, arms, top-level pieces, AFM segments (R2, R3, R4, R6) ----
  auto& site_kind = h.site_kind; auto& site_nch = h.site_nch; auto& site_lo = h.site_lo;
  auto& site_tie = h.site_tie; auto& site_logit = h.site_logit; auto& site_arm_ptr = h.site_arm_ptr;
  auto& arm_first = h.arm_first; auto& arm_n = h.arm_n;
  std::vector<int32_t> site_node;                   // node index of each site
  auto& piece_kind = h.piece_kind; auto& piece_a = h.piece_a; auto& piece_b = h.piece_b; auto& piece_c = h.piece_c;
  std::vector<std::array<int64_t, 10>> segs;
  std::array<int64_t, 10> cur{};
  bool cur_open = false;
  int expect_op = 0;
  auto close_seg = [&]() { if (cur_open) segs.push_back(cur); cur = {}; cur_open = false; };
  for (int i = 0; i < N; ++i) {
    const int k = A->node_kind[i];
    if (k == 0) {
      const int o = A->node_a[i];
      if (o != expect_op) return hfail(err, DYO_E_INVAL, "arch: operators must be numbered in preorder");
      ++expect_op;
      cur[0] += 1;
      for (int q = 0; q < 9; ++q) cur[1 + q] += sig[o * 9 + q];
      cur_open = true;
    } else if (k == 1 || k == 2) {
      close_seg();
      cur[0] = 1;              // the control row starts the new segment (R3)
      cur_open = true;
      site_node.push_back(i);
    } else if (k != 3) {
      return hfail(err, DYO_E_INVAL, "arch: node kind %d", k);
    }
  }
  close_seg();
  if (expect_op != n_ops) return hfail(err, DYO_E_INVAL, "arch: %d ops in nodes, %d declared", expect_op, n_ops);
  const int n_sites = (int)site_node.size();
  if (n_sites > kMaxSites) return hfail(err, DYO_E_CAPACITY, "arch: too many sites");
  // nesting (R16): a site inside another site's span executes per iteration / arm execution
  std::vector<int> depth(n_sites, 0);
  for (int s2 = 0; s2 < n_sites; ++s2)
    for (int s1 = 0; s1 < s2; ++s1)
      if (site_node[s2] <= site_node[s1] + A->node_span[site_node[s1]]) ++depth[s2];
  std::vector<int> tied_to(n_sites, 0);
  for (int s2 = 0; s2 < n_sites; ++s2)
    if (A->node_tie[site_node[s2]] >= 0 && A->node_tie[site_node[s2]] < n_sites) tied_to[A->node_tie[site_node[s2]]] = 1;
  for (int s2 = 0; s2 < n_sites; ++s2) {
    if (!depth[s2]) continue;
    const int i = site_node[s2];
    if (A->node_kind[i] != 1 || depth[s2] > 1)
      return hfail(err, DYO_E_UNSUPPORTED, "arch: site %d: only Ifs directly inside a top-level site may nest (R16)", s2);
    for (int q = i + 1; q <= i + A->node_span[i]; ++q)
      if (A->node_kind[q] == 1 || A->node_kind[q] == 2)
        return hfail(err, DYO_E_UNSUPPORTED, "arch: nested site %d: its arms must hold operators only (R16)", s2);
    if (A->node_tie[i] >= 0 || tied_to[s2])
      return hfail(err, DYO_E_INVAL, "arch: nested site %d cannot replay or be replayed (R6, R16)", s2);
    if (!A->branch_head)
      return hfail(err, DYO_E_UNSUPPORTED, "arch: nested sites need a branch head (the traversal over nested sites is not built)");
    h.nested = 1;
  }
  int logit = 10 * A->K_max;
  int64_t L_max = 0;
  // walk the top level
  auto count_ops = [&](int first_node, int span, int* first_op, bool* has_site) {
    int n = 0;
    *first_op = -1;
    *has_site = false;
    for (int q = first_node; q < first_node + span; ++q) {
      if (A->node_kind[q] == 0) { if (*first_op < 0) *first_op = A->node_a[q]; ++n; }
      else if (A->node_kind[q] != 3) *has_site = true;
    }
    if (*first_op < 0) *first_op = 0;
    return n;
  };
  std::vector<int> node_site(N, -1);
  for (int s = 0; s < n_sites; ++s) node_site[site_node[s]] = s;
  for (int s = 0; s < n_sites; ++s) {
    const int i = site_node[s];
    const int k = A->node_kind[i];
    site_kind.push_back(k);
    const int tie = A->node_tie[i];
    if (tie >= s) return hfail(err, DYO_E_INVAL, "arch: site %d ties to a later site", s);
    if (tie >= 0 && depth[tie]) return hfail(err, DYO_E_INVAL, "arch: site %d ties to a nested site", s);
    site_tie.push_back(tie);
    if (k == 1) {
      site_nch.push_back(A->node_a[i]);
      site_lo.push_back(0);
    } else {
      if (A->node_b[i] < A->node_a[i] || A->node_a[i] < 0) return hfail(err, DYO_E_INVAL, "arch: loop bounds");
      site_nch.push_back(A->node_b[i] - A->node_a[i] + 1);
      site_lo.push_back(A->node_a[i]);
    }
    h.site_rev.push_back(k == 2 && A->node_flags && (A->node_flags[i] & 1) ? 1 : 0);
    if (tie >= 0) {
      if (site_tie[tie] >= 0 || site_nch[tie] != site_nch[s] || site_kind[tie] != k)
        return hfail(err, DYO_E_INVAL, "arch: site %d tie target must be a free site of the same shape", s);
      site_logit.push_back(-1);
    } else if (!A->branch_head || depth[s]) {
      site_logit.push_back(-1);          // traversal decode / nested site: choices from the host (R4, R16)
    } else {
      site_logit.push_back(logit);
      logit += site_nch[s];
    }
    site_arm_ptr.push_back((int)arm_first.size());
    if (k == 1) {
      int q = i + 1;
      for (int br = 0; br < A->node_a[i]; ++br) {
        if (A->node_kind[q] != 3) return hfail(err, DYO_E_INVAL, "arch: IF node %d arm %d", i, br);
        int fo; bool hs;
        const int n = count_ops(q + 1, A->node_span[q], &fo, &hs);
        arm_first.push_back(fo);
        arm_n.push_back(n);
        q += 1 + A->node_span[q];
      }
    }
  }
  h.n_branch_logits = logit - 10 * A->K_max;
  // longest row count of a node range (nested Ifs: control row + their longest arm)
  auto range_maxlen = [&](int first, int last) {
    int64_t L = 0;
    for (int q = first; q < last;) {
      const int kq = A->node_kind[q];
      if (kq == 0) { ++L; ++q; }
      else if (kq == 1) {
        int64_t mx = 0;
        int r = q + 1;
        for (int br = 0; br < A->node_a[q]; ++br) { mx = std::max<int64_t>(mx, A->node_span[r]); r += 1 + A->node_span[r]; }
        L += 1 + mx;
        q += 1 + A->node_span[q];
      } else {
        ++q;
      }
    }
    return L;
  };
  for (int i = 0; i < N;) {
    const int k = A->node_kind[i];
    if (k == 0) {
      const int first = A->node_a[i];
      int n = 0;
      while (i < N && A->node_kind[i] == 0) { ++n; ++i; }
      piece_kind.push_back(0); piece_a.push_back(first); piece_b.push_back(n); piece_c.push_back(0);
      L_max += n;
    } else if (k == 1 || k == 2) {
      const int s = node_site[i];
      int fo; bool hs;
      const int n = count_ops(i + 1, A->node_span[i], &fo, &hs);
      (void)hs;                          // nested sites were validated above (R16)
      if (k == 1) {
        int64_t mx = 0;
        int r = i + 1;
        for (int br = 0; br < site_nch[s]; ++br) {
          mx = std::max<int64_t>(mx, range_maxlen(r + 1, r + 1 + A->node_span[r]));
          r += 1 + A->node_span[r];
        }
        piece_kind.push_back(1); piece_a.push_back(s); piece_b.push_back(0); piece_c.push_back(0);
        L_max += 1 + mx;
      } else {
        piece_kind.push_back(2); piece_a.push_back(s); piece_b.push_back(fo); piece_c.push_back(n);
        L_max += (int64_t)(site_lo[s] + site_nch[s] - 1) * (1 + range_maxlen(i + 1, i + 1 + A->node_span[i])) + 1;
      }
      i += 1 + A->node_span[i];
    } else {
      return hfail(err, DYO_E_INVAL, "arch: stray BRANCH node %d", i);
    }
  }
  if ((int)piece_kind.size() > 1024) return hfail(err, DYO_E_CAPACITY, "arch: more than 1024 top-level pieces");
  // per-iteration tensors (R13): strides only in loop bodies; named ids in range and ascending
  // within the operator at k = 0 (checked above) and k = hi - 1 (linear in k, so everywhere)
  {
    std::vector<int> op_hi(n_ops, -1);   // trip bound of the operator's loop, -1 outside loops
    for (size_t p = 0; p < piece_kind.size(); ++p)
      if (piece_kind[p] == 2) {
        const int s = piece_a[p];
        for (int o = piece_b[p]; o < piece_b[p] + piece_c[p]; ++o) op_hi[o] = site_lo[s] + site_nch[s] - 1;
      }
    for (int o = 0; o < n_ops; ++o) {
      for (int q = acc_ptr[o]; q < acc_ptr[o + 1]; ++q)
        if (h.acc_s[q] != 0 && op_hi[o] < 0)
          return hfail(err, DYO_E_INVAL, "arch: op %d has a strided access outside a loop", o);
      // corners (k, b) in {0, hi-1} x {0, max_b-1}; (0, 0) was checked with the accesses
      const int kmax = std::max(op_hi[o] - 1, 0), bmax = std::max(max_b - 1, 0);
      for (int corner = 1; corner < 4; ++corner) {
        const int k = (corner & 1) ? kmax : 0, b = (corner & 2) ? bmax : 0;
        int64_t prev_id = -1;
        for (int q = acc_ptr[o]; q < acc_ptr[o + 1]; ++q) {
          const int64_t t = (int64_t)acc_t[q] + (int64_t)h.acc_s[q] * k + (int64_t)h.acc_sb[q] * b;
          if (t < 0 || t >= T || t <= prev_id)
            return hfail(err, DYO_E_INVAL, "arch: op %d strided accesses leave [0, T) or lose ascending order", o);
          prev_id = t;
        }
      }
    }
  }
  if (L_max >= (1 << 30)) return hfail(err, DYO_E_CAPACITY, "arch: path too long");
  auto& seg_table = h.seg_table;
  seg_table.assign((size_t)A->S_max * 10, 0);
  for (int s = 0; s < A->S_max && s < (int)segs.size(); ++s)
    for (int e = 0; e < 10; ++e) seg_table[s * 10 + e] = (int32_t)std::min<int64_t>(segs[s][e], kSat);

  h.n_sites = n_sites;
  h.L_max = L_max;
  {                                      // the program tree (nested decode, dyo_trace_path)
    NestArch& na = h.nest;
    na.kind.assign(A->node_kind, A->node_kind + N);
    na.a.assign(A->node_a, A->node_a + N);
    na.b.assign(A->node_b, A->node_b + N);
    na.span.assign(A->node_span, A->node_span + N);
    na.flags.assign(N, 0);
    if (A->node_flags) na.flags.assign(A->node_flags, A->node_flags + N);
    na.site_of.assign(N, -1);
    for (int s2 = 0; s2 < n_sites; ++s2) na.site_of[site_node[s2]] = s2;
    na.sig = sig;
    na.site_lo = site_lo;
    na.site_tie = site_tie;
    na.top.assign(n_sites, 0);
    for (int s2 = 0; s2 < n_sites; ++s2) na.top[s2] = depth[s2] ? 0 : 1;
  }
  return DYO_OK;
}

}  // namespace

extern "C" {

const char* dyo_strerror(dyo_status s) {
  switch (s) {
    case DYO_OK: return "ok";
    case DYO_E_INVAL: return "invalid argument";
    case DYO_E_NOMEM: return "out of memory";
    case DYO_E_BUDGET: return "a tensor set does not fit half the budget";
    case DYO_E_CUDA: return "CUDA error";
    case DYO_E_STATE: return "call out of order";
    case DYO_E_CAPACITY: return "buffer capacity exceeded";
    case DYO_E_UNSUPPORTED: return "unsupported program shape";
  }
  return "unknown status";
}

const char* dyo_last_error(const dyo_ctx* ctx) { return ctx ? ctx->err.c_str() : ""; }

int32_t dyo_version(void) { return 1; }

dyo_status dyo_create(const dyo_config* cfg, int32_t device, dyo_ctx** outp) {
  if (!cfg || !outp) return DYO_E_INVAL;
  dyo_ctx* ctx = new dyo_ctx();
  ctx->cfg = *cfg;
  ctx->device = device;
  dyo_config& c = ctx->cfg;
  if (c.align <= 0 || (c.align & (c.align - 1)) || c.align < 16 || c.budget < 2 * c.align ||
      c.max_batch < 1 || c.max_batch > 1024 || c.policy < 0 || c.policy > 3) {
    delete ctx;
    return DYO_E_INVAL;
  }
  if (c.staging_bytes <= 0) c.staging_bytes = 64ll << 20;
  // compaction stages self-overlapping moves through two staging halves of >= max(256, ALIGN)
  // bytes each (a smaller staging would never advance)
  c.staging_bytes = std::max<int64_t>(c.staging_bytes, 2 * std::max<int64_t>(256, c.align));
  if (c.dma_min_bytes <= 0) c.dma_min_bytes = 2ll << 20;
  ctx->H = c.budget / 2 / c.align * c.align;
  if (ctx->H / c.align >= (1ll << 28)) { delete ctx; return DYO_E_INVAL; }
  cudaError_t e = cudaSetDevice(device);
  if (e == cudaSuccess) e = cudaMalloc(&ctx->arena, 2 * ctx->H);
  if (e == cudaSuccess) e = cudaMalloc(&ctx->staging, c.staging_bytes);
  for (auto& P : ctx->slot)
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&P.ev_last, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_entry, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_evict, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->d2h, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->side, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_moves, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_carry, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&ctx->sm_count, cudaDevAttrMultiProcessorCount, device);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->aux, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_pred, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_memo, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_fault_wb, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->join, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaMalloc((void**)&ctx->gbar, 64);
  if (e == cudaSuccess) e = cudaMemset(ctx->gbar, 0, 64);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_tail, cudaEventDisableTiming);
  if (e != cudaSuccess) {
    dyo_destroy(ctx);
    return e == cudaErrorMemoryAllocation ? DYO_E_NOMEM : DYO_E_CUDA;
  }
  ctx->staging_bytes = c.staging_bytes;
  *outp = ctx;
  return DYO_OK;
}

void memo_free(dyo_ctx* ctx) {
  for (void* p : ctx->memo.dev) cudaFree(p);
  const int64_t mp = ctx->memo.mispredictions;
  ctx->memo = dyo_ctx::Memo{};
  ctx->memo.mispredictions = mp;
  ctx->ad.memo_live = 0;
  ctx->ad.memo_mask = 0;
  ctx->ad.memo_index = nullptr;
  ctx->ad.memo_hash = nullptr;
  ctx->ad.memo_key = nullptr;
  ctx->ad.memo_val = nullptr;
  ctx->ad.memo_hits = nullptr;
}

// ---- NUMA-local pinned host pool (survey §8(e): each GPU's manager migrates over its own
// host link, so its tensor homes belong on the GPU's NUMA node). The node comes from sysfs for the
// device's PCI address; the pages are bound there (mbind, preferred) before cudaHostRegister faults
// them in. Without a node (or if any step fails) the pool falls back to cudaHostAlloc.
static int device_numa_node(int device) {
  if (const char* e = getenv("DYO_HOST_NUMA")) return atoi(e);   // -1 disables binding
  char bus[32] = {0};
  if (cudaDeviceGetPCIBusId(bus, sizeof bus, device) != cudaSuccess) return -1;
  for (char* c = bus; *c; ++c) *c = (char)tolower(*c);
  char path[96];
  snprintf(path, sizeof path, "/sys/bus/pci/devices/%s/numa_node", bus);
  FILE* f = fopen(path, "r");
  if (!f) return -1;
  int node = -1;
  if (fscanf(f, "%d", &node) != 1) node = -1;
  fclose(f);
  return node;
}

static void host_pool_free(dyo_ctx* ctx) {
  if (!ctx->host_pool) return;
  if (ctx->host_registered) {
    cudaHostUnregister(ctx->host_pool);
    munmap(ctx->host_pool, (size_t)std::max<int64_t>(ctx->host_bytes, 64));
  } else {
    cudaFreeHost(ctx->host_pool);
  }
  ctx->host_pool = nullptr;
  ctx->host_registered = false;
}

// MemAvailable of /proc/meminfo in bytes (-1 if unreadable): several managers on one node pin
// their pools from the same RAM (one per GPU), so a pool that cannot fit is refused up front
// (DYO_E_NOMEM) instead of letting pinning drive the host into the OOM killer.
static int64_t host_mem_available() {
  FILE* f = fopen("/proc/meminfo", "r");
  if (!f) return -1;
  char line[256];
  int64_t kb = -1;
  while (fgets(line, sizeof line, f))
    if (sscanf(line, "MemAvailable: %lld kB", (long long*)&kb) == 1) break;
  fclose(f);
  return kb < 0 ? -1 : kb * 1024;
}

static dyo_status host_pool_alloc(dyo_ctx* ctx, int64_t bytes) {
  const size_t n = (size_t)std::max<int64_t>(bytes, 64);
  const int64_t avail = host_mem_available();
  if (avail > 0 && (int64_t)n > avail - (avail >> 4))
    return fail(ctx, DYO_E_NOMEM, "host pool of %lld MiB exceeds the node's available memory (%lld MiB)",
                (long long)(n >> 20), (long long)(avail >> 20));
  ctx->host_numa = -1;
  ctx->host_registered = false;
  const int node = device_numa_node(ctx->device);
  if (node >= 0 && node < 64) {
    void* p = mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    if (p != MAP_FAILED) {
      unsigned long mask = 1UL << node;
      const int MPOL_PREFERRED_ = 1;
      bool ok = syscall(SYS_mbind, p, n, MPOL_PREFERRED_, &mask, 64UL, 0U) == 0;
      if (ok && cudaHostRegister(p, n, cudaHostRegisterMapped | cudaHostRegisterPortable) == cudaSuccess) {
        ctx->host_pool = (char*)p;
        ctx->host_registered = true;
        ctx->host_numa = node;
        return DYO_OK;
      }
      cudaGetLastError();
      munmap(p, n);
    }
  }
  CK(cudaHostAlloc((void**)&ctx->host_pool, n, cudaHostAllocMapped | cudaHostAllocPortable));
  return DYO_OK;
}

dyo_status dyo_destroy(dyo_ctx* ctx) {
  if (!ctx) return DYO_E_INVAL;
  cudaSetDevice(ctx->device);
  cudaDeviceSynchronize();
  free_owned(ctx, ctx->arch_dev);
  free_owned(ctx, ctx->pilot_dev);
  memo_free(ctx);
  free_plan_host(ctx);
  host_pool_free(ctx);
  if (ctx->h_logits) cudaFreeHost(ctx->h_logits);
  if (ctx->arena) cudaFree(ctx->arena);
  if (ctx->staging) cudaFree(ctx->staging);
  for (auto& P : ctx->slot)
    if (P.ev_last) cudaEventDestroy(P.ev_last);
  if (ctx->ev_entry) cudaEventDestroy(ctx->ev_entry);
  if (ctx->ev_evict) cudaEventDestroy(ctx->ev_evict);
  if (ctx->join) cudaStreamDestroy(ctx->join);
  if (ctx->gbar) cudaFree(ctx->gbar);
  if (ctx->ev_tail) cudaEventDestroy(ctx->ev_tail);
  if (ctx->d2h) cudaStreamDestroy(ctx->d2h);
  if (ctx->side) cudaStreamDestroy(ctx->side);
  if (ctx->ev_moves) cudaEventDestroy(ctx->ev_moves);
  if (ctx->ev_carry) cudaEventDestroy(ctx->ev_carry);
  if (ctx->aux) cudaStreamDestroy(ctx->aux);
  if (ctx->ev_pred) cudaEventDestroy(ctx->ev_pred);
  if (ctx->ev_memo) cudaEventDestroy(ctx->ev_memo);
  if (ctx->ev_fault_wb) cudaEventDestroy(ctx->ev_fault_wb);
  if (ctx->fault_area) cudaFree(ctx->fault_area);
  if (ctx->fault_segs) cudaFreeHost(ctx->fault_segs);
  for (auto e : ctx->ev_fseg) if (e) cudaEventDestroy(e);
  if (ctx->part_buf) cudaFree(ctx->part_buf);
  if (ctx->h_rep) cudaFreeHost(ctx->h_rep);
  if (ctx->h_memo_stage) cudaFreeHost(ctx->h_memo_stage);
  for (auto& t : ctx->tm) { cudaEventDestroy(t.a); cudaEventDestroy(t.b); }
  for (auto e : ctx->ev_pool) cudaEventDestroy(e);
  for (auto e : ctx->ev_wb) cudaEventDestroy(e);
  if (ctx->ev_ref) cudaEventDestroy(ctx->ev_ref);
  delete ctx;
  return DYO_OK;
}

dyo_status dyo_load_arch(dyo_ctx* ctx, const dyo_arch* A) {
  if (ctx && ctx->plan_pending) return fail(ctx, DYO_E_STATE, "dyo_load_arch: a plan is pending (dyo_plan_wait first)");
  if (!ctx || !A) return DYO_E_INVAL;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  free_owned(ctx, ctx->arch_dev);
  memo_free(ctx);
  ctx->memo.mispredictions = 0;
  free_plan_host(ctx);
  host_pool_free(ctx);
  ctx->arch_ok = false;
  const int64_t AL = ctx->cfg.align;
  ArchHost h;
  dyo_status pst = parse_arch(A, AL, ctx->cfg.max_batch, h, ctx->err);
  if (pst) return pst;
  const int T = h.T, n_ops = A->n_ops, n_sites = h.n_sites;
  ctx->T = T;
  ctx->t_bytes = h.t_bytes; ctx->t_abytes = h.t_abytes; ctx->t_host = h.t_host; ctx->t_flags = h.t_flags;
  ctx->n_branch_logits = h.n_branch_logits;
  const int64_t pool = h.pool, L_max = h.L_max;
  auto& sig = h.sig; auto& acc_ptr = h.acc_ptr; auto& acc_t = h.acc_t; auto& acc_m = h.acc_m;
  auto& site_kind = h.site_kind; auto& site_nch = h.site_nch; auto& site_lo = h.site_lo;
  auto& site_tie = h.site_tie; auto& site_logit = h.site_logit; auto& site_arm_ptr = h.site_arm_ptr;
  auto& arm_first = h.arm_first; auto& arm_n = h.arm_n;
  auto& piece_kind = h.piece_kind; auto& piece_a = h.piece_a; auto& piece_b = h.piece_b; auto& piece_c = h.piece_c;
  auto& seg_table = h.seg_table;
  // ---- device copies ----
  ArchDev& ad = ctx->ad;
  ad = ArchDev{};
  ad.T = T; ad.n_ops = n_ops; ad.n_sites = n_sites; ad.n_pieces = (int)piece_kind.size();
  ad.n_arms = (int)arm_first.size();
  ad.nn_type = A->nn_type; ad.S_max = A->S_max; ad.D_s = A->D_s; ad.h = A->h; ad.K_max = A->K_max;
  ad.F = (3 + A->D_s + 10 * A->S_max + 10 * A->h + 15) / 16 * 16;
  ad.O = 0;
  ad.n_branch_logits = ctx->n_branch_logits;
  ad.L_max = (int)std::max<int64_t>(L_max, 1);
  ad.H = ctx->H;
  ad.align = AL;
  std::vector<void*>& own = ctx->arch_dev;
  dyo_status st;
#define UP(field, vec) if ((st = dupload(ctx, own, &ad.field, vec))) return st
  UP(t_bytes, ctx->t_bytes); UP(t_abytes, ctx->t_abytes); UP(t_host, ctx->t_host); UP(t_flags, ctx->t_flags);
  UP(op_sig, sig); UP(acc_ptr, acc_ptr); UP(acc_t, acc_t); UP(acc_m, acc_m); UP(acc_s, h.acc_s); UP(acc_sb, h.acc_sb);
  UP(site_rev, h.site_rev);
  UP(site_kind, site_kind); UP(site_nch, site_nch); UP(site_lo, site_lo); UP(site_tie, site_tie);
  UP(site_logit, site_logit); UP(site_arm_ptr, site_arm_ptr); UP(arm_first_op, arm_first); UP(arm_nops, arm_n);
  UP(piece_kind, piece_kind); UP(piece_a, piece_a); UP(piece_b, piece_b); UP(piece_c, piece_c);
  UP(seg_table, seg_table);
#undef UP
  ctx->n_ops = n_ops; ctx->n_sites = n_sites; ctx->K_max = A->K_max; ctx->F = ad.F;
  ctx->branch_head = A->branch_head ? 1 : 0;
  ad.branch_head = ctx->branch_head;
  ctx->nested = h.nested;
  ctx->nest = h.nest;
  ctx->site_logit = site_logit;
  ctx->last_nested.clear();
  ctx->trav = TravArch{h.sig, site_kind, site_nch, site_lo, site_tie, site_arm_ptr, arm_first, arm_n,
                       piece_kind, piece_a, piece_b, piece_c};
  ctx->O_min = 10 * A->K_max + ctx->n_branch_logits;

  // ---- prediction storage ----
  const int B = ctx->cfg.max_batch, K = A->K_max;
  PredDev& pd = ctx->pd;
  pd = PredDev{};
  pd.B = B;
#define DA(p, n) if ((st = dalloc(ctx, own, &p, (size_t)(n)))) return st
  DA(pd.K, B); DA(pd.L, B); DA(pd.choices, (size_t)B * std::max(n_sites, 1)); DA(pd.rchoices, (size_t)B * std::max(n_sites, 1)); DA(pd.slots, (size_t)B * K * 10);
  DA(pd.path, (size_t)B * ad.L_max); DA(pd.path_it, (size_t)B * ad.L_max); DA(pd.grp, (size_t)B * K * 2);
  DA(pd.blocks, (size_t)B * K * 10);
  DA(pd.ent_n, (size_t)B * K); DA(pd.ent, (size_t)B * K * kEntCap); DA(pd.status, 4);
  pd.head_stride = 3 + n_sites + ((int)piece_kind.size() + 1) + (K + 1) + K;
  DA(pd.head, (size_t)B * pd.head_stride);
  DA(ctx->desc_dev, (size_t)B * std::max(A->D_s, 1)); DA(ctx->hist_dev, (size_t)B * std::max(A->h, 1));
  DA(ctx->hist_tab[0], (size_t)B * K * 10); DA(ctx->hist_tab[1], (size_t)B * K * 10);
  DA(ctx->hist_K[0], B); DA(ctx->hist_K[1], B);
  if (!ctx->branch_head || ctx->nested) {
    int32_t* f = nullptr;
    DA(f, (size_t)B * std::max(n_sites, 1));
    ad.forced = ctx->d_forced = f;
  }
  if (ctx->nested) {                    // the decode kernels read the host-resolved paths (R16)
    ad.hp_op = pd.path;
    ad.hp_it = pd.path_it;
    ad.hp_len = pd.L;
  }
  ctx->hist_B[0] = ctx->hist_B[1] = 0;
  ctx->hist_cur = 0;
  ctx->last_B = 0;
  // ---- planner state, scratch and outputs ----
  int mg = ctx->cfg.max_groups > 0 ? ctx->cfg.max_groups : B * K;
  mg = std::min(mg, 65535);
  ctx->max_groups = mg;
  for (int s2 = 0; s2 < 2; ++s2) {
    PlanState& ps = ctx->state[s2];
    DA(ps.loc, T); DA(ps.off, T); DA(ps.dirty, T); DA(ps.pw, T);
    DA(ps.prev, T); DA(ps.prev_n, 1); DA(ps.G, 1); DA(ps.rl_meta, 4); DA(ps.pos, T);
    for (int h = 0; h < 2; ++h)
      for (int q = 0; q < 2; ++q) DA(ps.rl[h][q], T);
    CK(cudaMemset(ps.loc, 0xff, T));   // -1: every tensor starts on the host
  }
  ctx->committed = 0;
  int64_t cap_ent = ctx->cfg.max_entries > 0 ? ctx->cfg.max_entries : (int64_t)mg * 512;
  int64_t cap_rec = ctx->cfg.max_records > 0 ? ctx->cfg.max_records : 4 * ((int64_t)T + cap_ent);
  PlanScratch& sc = ctx->sc;
  DA(sc.grp_b, mg); DA(sc.grp_k, mg); DA(sc.ebase, mg); DA(sc.Kt, 1);
  DA(sc.bcnt, T + 1); DA(sc.bfill, T); DA(sc.bkey, cap_ent); DA(sc.bsort, cap_ent);
  DA(sc.nxt, cap_ent); DA(sc.nxt_rd, cap_ent); DA(sc.first, T); DA(sc.first_rd, T); DA(sc.au, T);
  DA(sc.inw, (T + 31) / 32); DA(sc.wnx, T); DA(sc.wfl, T); DA(sc.keys, 2 * (size_t)T + 2048);
  DA(sc.kept, T); DA(sc.gap_s, T + 2); DA(sc.gap_e, T + 2); DA(sc.newoff, T);
  auto hmap = [&](void** p, size_t bytes) -> dyo_status {
    CK(cudaHostAlloc(p, std::max<size_t>(bytes, 64), cudaHostAllocMapped | cudaHostAllocPortable));
    memset(*p, 0, std::max<size_t>(bytes, 64));
    return DYO_OK;
  };
  if ((st = hmap((void**)&ctx->h_status, 16 * sizeof(int32_t)))) return st;
  if ((st = hmap((void**)&ctx->h_counts, 16 * sizeof(int32_t)))) return st;
  if ((st = hmap((void**)&ctx->h_loc, T))) return st;
  if ((st = hmap((void**)&ctx->h_off, sizeof(int64_t) * T))) return st;
  if ((st = hmap((void**)&ctx->h_rep, sizeof(int32_t) * (4 + 10 * (size_t)K + 2 * (size_t)std::max(n_sites, 1))))) return st;
  if (!ctx->branch_head || ctx->nested) {
    for (int i = 0; i < 2; ++i)
      if ((st = hmap((void**)&ctx->h_forced[i], sizeof(int32_t) * B * std::max(n_sites, 1)))) return st;
    if ((st = hmap((void**)&ctx->h_matched, sizeof(int32_t) * B))) return st;
  }
  if (ctx->nested && (st = hmap((void**)&ctx->h_path, sizeof(int32_t) * ((size_t)2 * B * ad.L_max + B)))) return st;
  memset(ctx->h_loc, 0xff, T);
  int32_t* d_status = nullptr;
  int32_t* d_counts = nullptr;
  CK(cudaHostGetDevicePointer((void**)&d_status, ctx->h_status, 0));
  CK(cudaHostGetDevicePointer((void**)&d_counts, ctx->h_counts, 0));
  for (auto& P : ctx->slot) {
    PlanOut& o = P.out;
    o = PlanOut{};
    o.cap_ent = cap_ent;
    o.cap_rec = cap_rec;
    if ((st = hmap((void**)&o.hdr, sizeof(PlanHdr) * mg))) return st;
    if ((st = hmap((void**)&o.ent, sizeof(dyo_entry_rec) * cap_ent))) return st;
    if ((st = hmap((void**)&o.ev, sizeof(dyo_evict_rec) * cap_rec))) return st;
    if ((st = hmap((void**)&o.mv, sizeof(dyo_move_rec) * cap_rec))) return st;
    if ((st = hmap((void**)&o.ca, sizeof(dyo_carry_rec) * cap_rec))) return st;
    if ((st = hmap((void**)&o.al, sizeof(dyo_alloc_rec) * cap_rec))) return st;
    if ((st = hmap((void**)&o.fe, sizeof(dyo_fetch_rec) * cap_rec))) return st;
    // the planner writes its records to device memory (writes to pinned host memory from a
    // latency-bound single-CTA kernel are avoided); dyo_plan copies them back by count
    PlanOut& dO = P.dout;
    dO = PlanOut{};
    dO.cap_ent = cap_ent;
    dO.cap_rec = cap_rec;
    PlanHdr* h1; dyo_entry_rec* e1; dyo_evict_rec* v1; dyo_move_rec* m1; dyo_carry_rec* c1; dyo_alloc_rec* a1; dyo_fetch_rec* f1;
    DA(h1, mg); DA(e1, cap_ent); DA(v1, cap_rec); DA(m1, cap_rec); DA(c1, cap_rec); DA(a1, cap_rec); DA(f1, cap_rec);
    dO.hdr = h1; dO.ent = e1; dO.ev = v1; dO.mv = m1; dO.ca = c1; dO.al = a1; dO.fe = f1;
    PlanOut& hO = P.hout;
    hO = o;
    CK(cudaHostGetDevicePointer((void**)&hO.hdr, o.hdr, 0));
    CK(cudaHostGetDevicePointer((void**)&hO.ev, o.ev, 0));
    CK(cudaHostGetDevicePointer((void**)&hO.mv, o.mv, 0));
    CK(cudaHostGetDevicePointer((void**)&hO.ca, o.ca, 0));
    CK(cudaHostGetDevicePointer((void**)&hO.al, o.al, 0));
    CK(cudaHostGetDevicePointer((void**)&hO.fe, o.fe, 0));
    hO.ent = nullptr;
    P.seg_cap = 8 * cap_rec + 65536;
    if ((st = hmap((void**)&P.h_segs, sizeof(CopySeg) * P.seg_cap))) return st;
    o.status = dO.status = hO.status = d_status;
    o.counts = dO.counts = hO.counts = d_counts;
    P.valid = false;
    P.K = P.next_j = 0;
    P.seg_used = 0;
    P.ev_pending = false;
  }
  ctx->plan_seq = ctx->mig_seq = 0;
  ctx->mig_loc.assign(T, -1);            // every tensor starts on the host
  ctx->mig_off.assign(T, 0);
  ctx->mig_prev_alloc.clear();
  ctx->last_mig_slot = nullptr;
  ctx->last_mig_j = -1;
  ctx->fault_wb.clear();
  ctx->fault_j = -1;
  ctx->n_faults = ctx->fault_bytes = ctx->n_fault_resident = ctx->n_fault_repair = 0;
#undef DA
  // ---- host pool (pinned, mapped: DMA and zero-copy kernels) ----
  ctx->host_bytes = pool;
  if (!(ctx->cfg.flags & DYO_F_NO_HOST_POOL)) {
    dyo_status hst = host_pool_alloc(ctx, pool);
    if (hst) return hst;
  }
  ctx->arch_ok = true;
  ctx->pilot_ok = false;
  return DYO_OK;
}

dyo_status dyo_traverse_check(const dyo_arch* A, const int32_t* slots, int32_t* choices, int32_t* matched,
                              char* err, int32_t errlen) {
  if (!A || !slots || !choices || !matched) return DYO_E_INVAL;
  ArchHost h;
  std::string e;
  dyo_status st = parse_arch(A, 256, 1, h, e);
  if (!st) {
    TravArch t{h.sig, h.site_kind, h.site_nch, h.site_lo, h.site_tie, h.site_arm_ptr, h.arm_first, h.arm_n,
               h.piece_kind, h.piece_a, h.piece_b, h.piece_c};
    int m = 0;
    st = traverse_decode(t, slots, A->K_max, choices, &m, e);
    *matched = m;
  }
  if (err && errlen > 0) { strncpy(err, e.c_str(), errlen - 1); err[errlen - 1] = 0; }
  return st;
}

dyo_status dyo_nested_check(const dyo_arch* A, const int32_t* slots, const int32_t* top_choices, int32_t* nested,
                            int32_t cap, int32_t* n_nested, int32_t* path_ops, int32_t path_cap, int32_t* path_len,
                            int32_t* matched, char* err, int32_t errlen) {
  if (!A || !slots || !top_choices || !n_nested || !path_len || !matched) return DYO_E_INVAL;
  ArchHost h;
  std::string e;
  dyo_status st = parse_arch(A, 256, 1, h, e);
  if (!st && !h.nested) { e = "arch has no nested sites"; st = DYO_E_STATE; }
  if (!st) {
    std::vector<int32_t> pop, pit, nest;
    int m = 0;
    st = nested_decode(h.nest, slots, A->K_max, top_choices, pop, pit, nest, &m, e);
    if (!st) {
      *matched = m;
      *n_nested = (int32_t)nest.size();
      *path_len = (int32_t)pop.size();
      if ((int32_t)nest.size() > cap || (path_ops && (int32_t)pop.size() > path_cap)) st = DYO_E_CAPACITY;
      else {
        if (nested) std::copy(nest.begin(), nest.end(), nested);
        if (path_ops) std::copy(pop.begin(), pop.end(), path_ops);
      }
    }
  }
  if (err && errlen > 0) { strncpy(err, e.c_str(), errlen - 1); err[errlen - 1] = 0; }
  return st;
}

dyo_status dyo_arch_check(const dyo_arch* A, int32_t align, dyo_arch_summary* out, int32_t* seg_table,
                          int32_t* op_sig, char* err, int32_t errlen) {
  if (!A || align < 16 || (align & (align - 1))) return DYO_E_INVAL;
  ArchHost h;
  std::string e;
  dyo_status st = parse_arch(A, align, 1, h, e);
  if (err && errlen > 0) { strncpy(err, e.c_str(), errlen - 1); err[errlen - 1] = 0; }
  if (st) return st;
  if (out) {
    out->n_sites = h.n_sites;
    out->n_branch_logits = h.n_branch_logits;
    out->n_pieces = (int32_t)h.piece_kind.size();
    out->L_max = h.L_max;
    out->F = (3 + A->D_s + 10 * A->S_max + 10 * A->h + 15) / 16 * 16;
    out->host_pool_bytes = h.pool;
  }
  if (seg_table) std::copy(h.seg_table.begin(), h.seg_table.end(), seg_table);
  if (op_sig) std::copy(h.sig.begin(), h.sig.end(), op_sig);
  return DYO_OK;
}

// cvt.rna.tf32.f32 on the host: round to nearest (ties away) to 10 mantissa bits
static float tf32_rna_host(float x) {
  uint32_t u;
  memcpy(&u, &x, 4);
  if ((u & 0x7f800000u) == 0x7f800000u) return x;
  u = (u + 0x1000u) & ~0x1fffu;
  float y;
  memcpy(&y, &u, 4);
  return y;
}

// K1-TC plan (pilot_tc.cu): stages = the selected MLP's layers + the output layer; stage s has
// n_m = ceil(out/128) tiles and its K split n_ks ways (n_m * n_ks <= 16 CTAs; K-slices multiple
// of 8 and <= 128); weights pre-split into TF32 hi/lo and laid out per (CTA, chunk) in the UMMA
// K-major no-swizzle core-matrix layout ([k/4][row/8][row%8][k%4]) so one cp.async.bulk moves a
// chunk. Only for the P-type topology (three feature layers); otherwise tc_dev stays null.
static dyo_status build_tc_plan(dyo_ctx* ctx, const dyo_pilot_desc* w) {
  // K1-TC is opt-in (DYO_F_PILOT_TC, or DYO_PILOT_TC=1 for measurement): the default batch path
  // is K1's fp64 DMMA tiles, which meet the north_star gate exactly like batch 1
  ctx->tc_flag_off = (ctx->cfg.flags & DYO_F_PILOT_TC) ? 0 : 1;
  if (const char* e = getenv("DYO_PILOT_TC")) ctx->tc_flag_off = (e[0] == '0');
  if (w->n_feature != 3 || ctx->F > 256 || ctx->cfg.max_batch < kTcMinBatch) return DYO_OK;
  const int k = ctx->ad.nn_type;
  int n_feat = 0;
  for (int i = 0; i < 3; ++i) n_feat += w->feat_out[i];
  struct L { const float* W; const float* b; int out, in, act; };
  std::vector<L> layers;
  // stage 0: the three feature layers as one block-diagonal [n_feat x F_pad] layer (F padded to
  // a multiple of 64 so its K splits over many CTAs; the padded inputs are zero)
  const int Fp = (ctx->F + 63) / 64 * 64;
  std::vector<float> fW((size_t)n_feat * Fp, 0.f), fb(n_feat, 0.f);
  {
    int o = 0;
    for (int i = 0; i < 3; ++i) {
      if (w->feat_off[i] < 0 || w->feat_off[i] + w->feat_len[i] > ctx->F) return DYO_OK;
      for (int rr = 0; rr < w->feat_out[i]; ++rr) {
        for (int c = 0; c < w->feat_len[i]; ++c)
          fW[(size_t)(o + rr) * Fp + w->feat_off[i] + c] = w->feat_W[i][(size_t)rr * w->feat_len[i] + c];
        fb[o + rr] = w->feat_b[i][rr];
      }
      o += w->feat_out[i];
    }
  }
  layers.push_back({fW.data(), fb.data(), n_feat, Fp, 1});
  for (int l = 0; l < w->n_mlp; ++l)
    layers.push_back({w->mlp_W[k * w->n_mlp + l], w->mlp_b[k * w->n_mlp + l], w->mlp_out[l], w->mlp_in[l], 1});
  layers.push_back({w->out_W, w->out_b, w->O, w->out_in, 0});
  if ((int)layers.size() > kTcMaxStages || layers[1].in != n_feat) return DYO_OK;
  TcPlan P{};
  P.n_stages = (int)layers.size();
  P.n_feat = n_feat;
  std::vector<std::vector<TcChunk>> per(kTcCtas);
  std::vector<float> blob;
  for (int s = 0; s < P.n_stages; ++s) {
    const L& ly = layers[s];
    TcStage& S = P.st[s];
    S.n_out = ly.out; S.K = ly.in; S.act = ly.act;
    S.n_m = (ly.out + 127) / 128;
    if (ly.in % 8) return DYO_OK;
    if (S.n_m > kTcCtas) {
      if (s != P.n_stages - 1 || S.n_m > 2 * kTcCtas || ly.in > kTcMaxKsl) return DYO_OK;
      S.n_ks = 1;
    } else {
      // n_ks <= 8 (an owner's w = 64 / n_ks samples form whole 8-sample groups); hidden stages
      // need n_ks >= 4 (w <= 16: the owner's staging buffer)
      S.n_ks = 0;
      for (int p = 8; p >= 1; p >>= 1)
        if (S.n_m * p <= kTcCtas && ly.in % (8 * p) == 0 && ly.in / p <= kTcMaxKsl) { S.n_ks = p; break; }
      if (!S.n_ks) return DYO_OK;
      if (s != P.n_stages - 1 && S.n_ks < 4) return DYO_OK;
    }
    S.ksl = ly.in / S.n_ks;
    std::vector<float> bias(ly.b, ly.b + ly.out);
    const float* db = nullptr;
    dyo_status st = dupload(ctx, ctx->pilot_dev, &db, bias);
    if (st) return st;
    S.bias = db;
    // jobs of every CTA (same rule as jobs_of() in the kernel), chunked along K
    for (int r = 0; r < kTcCtas; ++r) {
      std::vector<std::pair<int, int>> jobs;   // (m, ks)
      if (S.n_m * S.n_ks <= kTcCtas) {
        if (r < S.n_m * S.n_ks) jobs.push_back({r / S.n_ks, r % S.n_ks});
      } else {
        for (int m = r; m < S.n_m && (int)jobs.size() < 2; m += kTcCtas) jobs.push_back({m, 0});
      }
      for (size_t jj = 0; jj < jobs.size(); ++jj) {
        const int m = jobs[jj].first, ks = jobs[jj].second;
        for (int k0 = 0; k0 < S.ksl; k0 += kTcMaxKc) {
          const int kc = std::min(kTcMaxKc, S.ksl - k0);
          TcChunk ch{};
          ch.off = (int64_t)blob.size();
          ch.bytes = 128 * kc * 8;
          ch.stage = s; ch.job = (int)jj; ch.k0 = k0; ch.kc = kc;
          blob.resize(blob.size() + (size_t)128 * kc * 2, 0.f);
          float* hi = blob.data() + ch.off;
          float* lo = hi + 128 * kc;
          for (int row = 0; row < 128; ++row) {
            const int R = m * 128 + row;
            if (R >= ly.out) continue;
            for (int kk = 0; kk < kc; ++kk) {
              const int K = ks * S.ksl + k0 + kk;
              const float v = ly.W[(size_t)R * ly.in + K];
              if (!std::isfinite(v)) return DYO_E_INVAL;
              const float h = tf32_rna_host(v);
              const float l = tf32_rna_host(v - h);
              const size_t o = (size_t)(kk >> 2) * (16 * 32) + (size_t)(row >> 3) * 32 + (size_t)(row & 7) * 4 + (kk & 3);
              hi[o] = h;
              lo[o] = l;
            }
          }
          per[r].push_back(ch);
        }
      }
    }
  }
  // an owner's tile rows split into whole K-slices of the next stage
  for (int s2 = 0; s2 + 1 < P.n_stages; ++s2)
    if (P.st[s2].n_m > 1 && 128 % P.st[s2 + 1].ksl) return DYO_OK;
  std::vector<TcChunk> all;
  for (int r = 0; r < kTcCtas; ++r) {
    P.chunk_ptr[r] = (int)all.size();
    all.insert(all.end(), per[r].begin(), per[r].end());
  }
  P.chunk_ptr[kTcCtas] = (int)all.size();
  const float* dblob = nullptr;
  const TcChunk* dch = nullptr;
  dyo_status st = dupload(ctx, ctx->pilot_dev, &dblob, blob);
  if (st) return st;
  st = dupload(ctx, ctx->pilot_dev, &dch, all);
  if (st) return st;
  P.blob = dblob;
  P.chunks = dch;
  std::vector<TcPlan> one(1, P);
  const TcPlan* dp = nullptr;
  st = dupload(ctx, ctx->pilot_dev, &dp, one);
  if (st) return st;
  ctx->tc_dev = dp;
  return DYO_OK;
}

dyo_status dyo_load_pilot(dyo_ctx* ctx, const dyo_pilot_desc* w) {
  if (ctx && ctx->plan_pending) return fail(ctx, DYO_E_STATE, "dyo_load_pilot: a plan is pending (dyo_plan_wait first)");
  if (!ctx || !w) return DYO_E_INVAL;
  if (!ctx->arch_ok) return fail(ctx, DYO_E_STATE, "load the arch first");
  CK(cudaSetDevice(ctx->device));
  if (w->F != ctx->F) return fail(ctx, DYO_E_INVAL, "pilot F=%d, arch needs %d", w->F, ctx->F);
  if (w->O < ctx->O_min) return fail(ctx, DYO_E_INVAL, "pilot O=%d < %d", w->O, ctx->O_min);
  if (w->n_mlp < 1 || w->n_mlp > kMaxLayers || w->n_feature < 0 || w->n_feature > 8)
    return fail(ctx, DYO_E_INVAL, "pilot: layer counts");
  free_owned(ctx, ctx->pilot_dev);
  PilotDev& p = ctx->pdv;
  p = PilotDev{};
  p.F = w->F;
  p.O = w->O;
  p.slope = w->slope;
  int nl = 0, ns = 0, width = w->F;
  int maxw = w->F;
  auto add_layer = [&](const float* W, const float* b, int in_off, int in_len, int out_len, int out_off) -> dyo_status {
    LayerDev& L = p.ly[nl++];
    // row layout [w_0 .. w_{in-1}, bias, 0 pad] padded to 16 bytes: the bias rides with the
    // weights in the same TMA bulk copy and is applied as the weight of a constant-1 input
    const int in_pad = (in_len + 1 + 3) / 4 * 4;
    std::vector<float> wp((size_t)out_len * in_pad, 0.f), bp(b, b + out_len);
    // device copy: subnormal weights flushed to zero (the kernel widens fp32 -> fp64 by
    // exponent rebias, exact for normals and zero); non-finite weights are rejected
    auto keep = [](float v) { return std::fpclassify(v) == FP_SUBNORMAL ? 0.0f : v; };
    for (int r = 0; r < out_len; ++r) {
      for (int c = 0; c < in_len; ++c) {
        const float v = W[(size_t)r * in_len + c];
        if (!std::isfinite(v)) return DYO_E_INVAL;
        wp[(size_t)r * in_pad + c] = keep(v);
      }
      if (!std::isfinite(b[r])) return DYO_E_INVAL;
      wp[(size_t)r * in_pad + in_len] = keep(b[r]);
    }
    const float* dw = nullptr;
    const float* db = nullptr;
    dyo_status s = dupload(ctx, ctx->pilot_dev, &dw, wp);
    if (s) return s;
    s = dupload(ctx, ctx->pilot_dev, &db, bp);
    if (s) return s;
    L.W = dw; L.b = db; L.in_off = in_off; L.in_len = in_len; L.in_pad = in_pad; L.out_off = out_off; L.out_len = out_len;
    return DYO_OK;
  };
  dyo_status s;
  if (w->n_feature > 0) {
    StageDev& S = p.st[ns++];
    S.first_layer = nl; S.n_layers = w->n_feature; S.in_width = w->F; S.act = 1;
    int o = 0;
    for (int i = 0; i < w->n_feature; ++i) {
      if (w->feat_off[i] < 0 || w->feat_off[i] + w->feat_len[i] > w->F) return fail(ctx, DYO_E_INVAL, "pilot: feature slice");
      if ((s = add_layer(w->feat_W[i], w->feat_b[i], w->feat_off[i], w->feat_len[i], w->feat_out[i], o))) return s;
      o += w->feat_out[i];
    }
    S.out_width = S.rows = o;
    width = o;
    maxw = std::max(maxw, o);
  }
  const int k = ctx->ad.nn_type;   // only the MLP of the arch's NN type runs
  for (int l = 0; l < w->n_mlp; ++l) {
    if (w->mlp_in[l] != width) return fail(ctx, DYO_E_INVAL, "pilot: MLP layer %d input %d != %d", l, w->mlp_in[l], width);
    StageDev& S = p.st[ns++];
    S.first_layer = nl; S.n_layers = 1; S.in_width = width; S.act = 1;
    if ((s = add_layer(w->mlp_W[k * w->n_mlp + l], w->mlp_b[k * w->n_mlp + l], 0, w->mlp_in[l], w->mlp_out[l], 0))) return s;
    width = S.out_width = S.rows = w->mlp_out[l];
    maxw = std::max(maxw, width);
  }
  if (w->out_in != width) return fail(ctx, DYO_E_INVAL, "pilot: output layer input %d != %d", w->out_in, width);
  StageDev& S = p.st[ns++];
  S.first_layer = nl; S.n_layers = 1; S.in_width = width; S.act = 0;
  if ((s = add_layer(w->out_W, w->out_b, 0, width, w->O, 0))) return s;
  S.out_width = S.rows = w->O;
  p.n_stages = ns;
  p.max_width = (maxw + 3) / 4 * 4;
  {
    // device copy of the descriptor block: the kernel loads it with 16-byte loads in one round trip
    std::vector<PilotDev> one(1, p);
    const PilotDev* dp = nullptr;
    dyo_status s2 = dupload(ctx, ctx->pilot_dev, &dp, one);
    if (s2) return s2;
    ctx->pdv_dev = dp;
  }
  ctx->ad.O = w->O;
  CK(cudaFree(nullptr));
  double* lg = nullptr;
  if ((s = dalloc(ctx, ctx->pilot_dev, &lg, (size_t)ctx->cfg.max_batch * w->O))) return s;
  ctx->logits64 = lg;
  ctx->tc_dev = nullptr;
  if ((s = build_tc_plan(ctx, w))) return s;
  if (ctx->h_logits) { cudaFreeHost(ctx->h_logits); ctx->h_logits = nullptr; }
  if (!ctx->branch_head || ctx->nested)
    CK(cudaHostAlloc((void**)&ctx->h_logits, sizeof(double) * ctx->cfg.max_batch * w->O, cudaHostAllocPortable));
  ctx->pilot_ok = true;
  return DYO_OK;
}

dyo_status dyo_host_pool(dyo_ctx* ctx, void** base, int64_t* bytes) {
  if (!ctx || !ctx->arch_ok || !ctx->host_pool) return DYO_E_STATE;
  if (base) *base = ctx->host_pool;
  if (bytes) *bytes = ctx->host_bytes;
  return DYO_OK;
}

dyo_status dyo_arena(dyo_ctx* ctx, void** base, int64_t* half) {
  if (!ctx) return DYO_E_INVAL;
  if (base) *base = ctx->arena;
  if (half) *half = ctx->H;
  return DYO_OK;
}

static dyo_status stage_samples(dyo_ctx* ctx, const dyo_sample* s, int B, cudaStream_t st,
                                const int64_t** desc, const int32_t** hist) {
  const ArchDev& a = ctx->ad;
  *desc = nullptr;
  *hist = nullptr;
  if (a.D_s > 0) {
    if (!s || !s->desc) return fail(ctx, DYO_E_INVAL, "sample descriptors missing");
    if (is_device_ptr(s->desc)) *desc = s->desc;
    else {
      CK(cudaMemcpyAsync(ctx->desc_dev, s->desc, sizeof(int64_t) * B * a.D_s, cudaMemcpyHostToDevice, st));
      *desc = ctx->desc_dev;
    }
  } else {
    *desc = ctx->desc_dev;
  }
  if (a.h > 0 && s && s->hist_ids) {
    if (is_device_ptr(s->hist_ids)) *hist = s->hist_ids;
    else {
      CK(cudaMemcpyAsync(ctx->hist_dev, s->hist_ids, sizeof(int32_t) * B * a.h, cudaMemcpyHostToDevice, st));
      *hist = ctx->hist_dev;
    }
  }
  return DYO_OK;
}

dyo_status dyo_encode_features(dyo_ctx* ctx, const dyo_sample* s, int32_t B, float* feat, void* stream) {
  if (!ctx || !feat) return DYO_E_INVAL;
  if (!ctx->arch_ok) return fail(ctx, DYO_E_STATE, "load the arch first");
  if (B < 1 || B > ctx->cfg.max_batch) return fail(ctx, DYO_E_INVAL, "B=%d out of [1, max_batch]", B);
  CK(cudaSetDevice(ctx->device));
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t* desc;
  const int32_t* hist;
  dyo_status r = stage_samples(ctx, s, B, st, &desc, &hist);
  if (r) return r;
  CK(launch_encode(ctx->ad, desc, hist, ctx->hist_tab[ctx->hist_cur], ctx->hist_K[ctx->hist_cur],
                   ctx->hist_B[ctx->hist_cur], B, feat, st));
  return DYO_OK;
}

dyo_status dyo_pilot_predict(dyo_ctx* ctx, const float* feat, const dyo_sample* s, int32_t B,
                             float* logits, void* stream) {
  if (ctx && ctx->plan_pending) return fail(ctx, DYO_E_STATE, "dyo_pilot_predict: a plan is pending (dyo_plan_wait first)");
  if (!ctx) return DYO_E_INVAL;
  if (!ctx->arch_ok || !ctx->pilot_ok) return fail(ctx, DYO_E_STATE, "load arch and pilot first");
  if (B < 1 || B > ctx->cfg.max_batch) return fail(ctx, DYO_E_INVAL, "B=%d out of [1, max_batch]", B);
  CK(cudaSetDevice(ctx->device));
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t* desc = nullptr;
  const int32_t* hist = nullptr;
  if (!feat) {
    dyo_status r = stage_samples(ctx, s, B, st, &desc, &hist);
    if (r) return r;
  } else if (!is_device_ptr(feat)) {
    return fail(ctx, DYO_E_INVAL, "feat must be device memory");
  }
  if (ctx->memo_pending) {
    // decode kernels read the memo table: order them after the last upload (dyo_report)
    if (cudaEventQuery(ctx->ev_memo) == cudaSuccess) ctx->memo_pending = false;
    else CK(cudaStreamWaitEvent(st, ctx->ev_memo, 0));
    cudaGetLastError();
  }
  const int cur = ctx->hist_cur;
  int fused = 0;
  {
    TScope ts(ctx, 0, st);
    if (ctx->tc_dev && !ctx->tc_flag_off && B >= kTcMinBatch) {
      // K1-TC: batch large enough for the layers to be real dense contractions (3xTF32)
      CK(launch_pilot_tc(ctx->ad, ctx->pdv_dev, ctx->tc_dev, feat, desc, hist, ctx->hist_tab[cur], ctx->hist_K[cur],
                         ctx->hist_B[cur], B, ctx->logits64, logits, st));
      fused = 0;
      ctx->last_tc = 1;
    } else {
      ctx->last_tc = 0;
      CK(launch_pilot(ctx->ad, ctx->pdv, ctx->pdv_dev, feat, desc, hist, ctx->hist_tab[cur], ctx->hist_K[cur],
                      ctx->hist_B[cur], B, ctx->logits64, logits, ctx->pd, ctx->hist_tab[1 - cur], ctx->hist_K[1 - cur],
                      &fused, st));
    }
  }
  if (!ctx->branch_head || ctx->nested) {
    // host decode: logits to the host, one sync, block head -> slots (R4: rint
    // half-even of y * 2^sigma, clamped); traversal over the top-level sites (no branch head)
    // or, with nested sites (R16), the branch-head argmax (lowest index on ties) and the nested
    // executions resolved against the block head; choices (and paths) back to the device
    const int O = ctx->ad.O, K = ctx->K_max, ns = ctx->n_sites;
    CK(cudaMemcpyAsync(ctx->h_logits, ctx->logits64, sizeof(double) * B * O, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    int32_t* hf = ctx->h_forced[cur];
    std::vector<int32_t> slots((size_t)K * 10);
    if (ctx->nested) ctx->last_nested.assign(B, {});
    const int64_t Lm = ctx->ad.L_max;
    for (int b = 0; b < B; ++b) {
      const double* y = ctx->h_logits + (size_t)b * O;
      for (int i = 0; i < K * 10; ++i) {
        const double t = std::fmin(std::fmax(y[i] * ((i % 10) < 7 ? 16.0 : 1024.0), 0.0), (double)kSat);
        slots[i] = (int32_t)std::nearbyint(t);
      }
      int matched = 0;
      int32_t* chb = hf + (size_t)b * std::max(ns, 1);
      if (!ctx->nested) {
        dyo_status r = traverse_decode(ctx->trav, slots.data(), K, chb, &matched, ctx->err);
        if (r) return r;
      } else {
        for (int s2 = 0; s2 < ns; ++s2) {
          const int off = ctx->site_logit[s2];
          if (off < 0) { chb[s2] = -1; continue; }
          int best = 0;
          for (int c = 1; c < ctx->trav.site_nch[s2]; ++c)
            if (y[off + c] > y[off + best]) best = c;
          chb[s2] = best;
        }
        for (int s2 = 0; s2 < ns; ++s2)
          if (ctx->trav.site_tie[s2] >= 0) chb[s2] = chb[ctx->trav.site_tie[s2]];
        std::vector<int32_t> pop, pit;
        dyo_status r = nested_decode(ctx->nest, slots.data(), K, chb, pop, pit, ctx->last_nested[b], &matched, ctx->err);
        if (r) return r;
        if ((int64_t)pop.size() > Lm) return fail(ctx, DYO_E_CAPACITY, "nested path of %zu rows > L_max", pop.size());
        std::copy(pop.begin(), pop.end(), ctx->h_path + (size_t)b * Lm);
        std::copy(pit.begin(), pit.end(), ctx->h_path + (size_t)B * Lm + (size_t)b * Lm);
        ctx->h_path[(size_t)2 * B * Lm + b] = (int32_t)pop.size();
      }
      ctx->h_matched[b] = matched;
    }
    if (ns > 0) CK(cudaMemcpyAsync(ctx->d_forced, hf, sizeof(int32_t) * B * ns, cudaMemcpyHostToDevice, st));
    if (ctx->nested) {
      CK(cudaMemcpyAsync(ctx->pd.path, ctx->h_path, sizeof(int32_t) * B * Lm, cudaMemcpyHostToDevice, st));
      CK(cudaMemcpyAsync(ctx->pd.path_it, ctx->h_path + (size_t)B * Lm, sizeof(int32_t) * B * Lm, cudaMemcpyHostToDevice, st));
      CK(cudaMemcpyAsync(ctx->pd.L, ctx->h_path + (size_t)2 * B * Lm, sizeof(int32_t) * B, cudaMemcpyHostToDevice, st));
    }
  }
  if (!fused) {
    TScope ts(ctx, 1, st);
    CK(launch_decode(ctx->ad, ctx->logits64, ctx->pd, B, ctx->hist_tab[1 - cur], ctx->hist_K[1 - cur], st));
  }
  ctx->hist_B[1 - cur] = B;
  ctx->hist_cur = 1 - cur;
  ctx->last_B = B;
  ctx->last_fused = fused;
  CK(cudaEventRecord(ctx->ev_pred, st));
  return DYO_OK;
}

dyo_status dyo_prediction_get(dyo_ctx* ctx, int32_t b, int32_t* K, int32_t* blocks, int32_t* choices,
                              int32_t* group_rows, void* stream) {
  if (!ctx || b < 0 || b >= ctx->last_B) return DYO_E_INVAL;
  cudaStream_t st = (cudaStream_t)stream;
  CK(cudaStreamSynchronize(st));
  int32_t status = 0;
  CK(cudaMemcpy(&status, ctx->pd.status, sizeof status, cudaMemcpyDeviceToHost));
  if (status) return fail(ctx, (dyo_status)status, "decode failed (status %d)", status);
  const int Km = ctx->K_max;
  if (K) CK(cudaMemcpy(K, ctx->pd.K + b, sizeof(int32_t), cudaMemcpyDeviceToHost));
  if (blocks) CK(cudaMemcpy(blocks, ctx->pd.blocks + (size_t)b * Km * 10, sizeof(int32_t) * Km * 10, cudaMemcpyDeviceToHost));
  if (choices && ctx->n_sites)
    CK(cudaMemcpy(choices, ctx->pd.choices + (size_t)b * ctx->n_sites, sizeof(int32_t) * ctx->n_sites, cudaMemcpyDeviceToHost));
  if (group_rows) CK(cudaMemcpy(group_rows, ctx->pd.grp + (size_t)b * Km * 2, sizeof(int32_t) * Km * 2, cudaMemcpyDeviceToHost));
  return DYO_OK;
}

// ---- mis-prediction record + exact-match memo (R15) --------------
namespace {
uint64_t memo_hash_of(const int32_t* key, int kw_total) {
  uint64_t h = 0;
  for (int i = 0; i < kw_total; ++i) h += dyo::memo_mix((uint64_t)i, key[i]);
  return h ? h : 1;
}
// Upload entry `id` (and the index when with_index) of the host mirror to the device table:
// staged in pinned memory, copied on the ctx's aux stream, ordered before the next
// dyo_pilot_predict by ev_memo (no device-wide synchronisation).
dyo_status memo_upload(dyo_ctx* ctx, int id, bool with_index) {
  auto& M = ctx->memo;
  const int kt = M.kw + M.ns;
  const size_t need = 8 + 4 * (size_t)kt + 4 * (size_t)std::max(M.ns, 1) + 4 * M.index.size();
  if (ctx->memo_pending) CK(cudaEventSynchronize(ctx->ev_memo));   // the staging is reused
  ctx->memo_pending = false;
  if (ctx->h_memo_stage_bytes < need) {
    if (ctx->h_memo_stage) cudaFreeHost(ctx->h_memo_stage);
    ctx->h_memo_stage = nullptr;
    ctx->h_memo_stage_bytes = 0;
    CK(cudaHostAlloc((void**)&ctx->h_memo_stage, need, cudaHostAllocPortable));
    ctx->h_memo_stage_bytes = need;
  }
  char* q = ctx->h_memo_stage;
  memcpy(q, &M.hash[id], 8);
  memcpy(q + 8, &M.key[(size_t)id * kt], 4 * (size_t)kt);
  char* qv = q + 8 + 4 * (size_t)kt;
  if (M.ns) memcpy(qv, &M.val[(size_t)id * M.ns], 4 * (size_t)M.ns);
  char* qi = qv + 4 * (size_t)std::max(M.ns, 1);
  CK(cudaMemcpyAsync(static_cast<uint64_t*>(M.dev[1]) + id, q, 8, cudaMemcpyHostToDevice, ctx->aux));
  CK(cudaMemcpyAsync(static_cast<int32_t*>(M.dev[2]) + (size_t)id * kt, q + 8, 4 * (size_t)kt, cudaMemcpyHostToDevice,
                     ctx->aux));
  if (M.ns)
    CK(cudaMemcpyAsync(static_cast<int32_t*>(M.dev[3]) + (size_t)id * M.ns, qv, 4 * (size_t)M.ns,
                       cudaMemcpyHostToDevice, ctx->aux));
  if (with_index) {
    memcpy(qi, M.index.data(), 4 * M.index.size());
    CK(cudaMemcpyAsync(M.dev[0], qi, 4 * M.index.size(), cudaMemcpyHostToDevice, ctx->aux));
  }
  CK(cudaEventRecord(ctx->ev_memo, ctx->aux));
  ctx->memo_pending = true;
  return DYO_OK;
}
// slot of entry `id` (or of key `key` when id < 0) in the index; -1 if absent
int memo_find(const dyo_ctx::Memo& M, uint64_t h, const int32_t* key, int id) {
  const int kt = M.kw + M.ns;
  int slot = (int)(h & (uint64_t)M.mask);
  for (int probe = 0; probe <= M.mask; ++probe) {
    const int e = M.index[slot];
    if (e == -1) return -1;
    if (e >= 0 && M.hash[e] == h) {
      if (id >= 0 ? e == id : std::equal(key, key + kt, &M.key[(size_t)e * kt])) return slot;
    }
    slot = (slot + 1) & M.mask;
  }
  return -1;
}
void memo_rebuild(dyo_ctx::Memo& M) {
  std::fill(M.index.begin(), M.index.end(), -1);
  for (int id : M.fifo) {
    int slot = (int)(M.hash[id] & (uint64_t)M.mask);
    while (M.index[slot] != -1) slot = (slot + 1) & M.mask;
    M.index[slot] = id;
  }
  M.tomb = 0;
}
}  // namespace

dyo_status dyo_memo_config(dyo_ctx* ctx, int32_t capacity) {
  if (!ctx || capacity < 0 || capacity > (1 << 20)) return DYO_E_INVAL;
  if (!ctx->arch_ok) return fail(ctx, DYO_E_STATE, "dyo_memo_config before dyo_load_arch");
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  memo_free(ctx);
  ctx->memo_pending = false;
  if (capacity == 0) return DYO_OK;
  auto& M = ctx->memo;
  M.cap = capacity;
  M.kw = 10 * ctx->K_max;
  M.ns = ctx->n_sites;
  int slots = 1;
  while (slots < 2 * capacity) slots <<= 1;
  M.mask = slots - 1;
  const int kt = M.kw + M.ns;
  M.hash.assign(capacity, 0);
  M.key.assign((size_t)capacity * kt, 0);
  M.val.assign((size_t)capacity * std::max(M.ns, 1), 0);
  M.index.assign(slots, -1);
  M.free_ids.clear();
  for (int i = capacity - 1; i >= 0; --i) M.free_ids.push_back(i);
  const size_t bytes[5] = {4u * (size_t)slots, 8u * (size_t)capacity, 4u * (size_t)capacity * kt,
                           4u * (size_t)capacity * std::max(M.ns, 1), 8};
  for (size_t b : bytes) {
    void* p = nullptr;
    CK(cudaMalloc(&p, b));
    CK(cudaMemset(p, 0, b));
    M.dev.push_back(p);
  }
  CK(cudaMemcpy(M.dev[0], M.index.data(), 4 * M.index.size(), cudaMemcpyHostToDevice));
  ctx->ad.memo_mask = M.mask;
  ctx->ad.memo_live = 0;
  ctx->ad.memo_index = static_cast<const int32_t*>(M.dev[0]);
  ctx->ad.memo_hash = static_cast<const uint64_t*>(M.dev[1]);
  ctx->ad.memo_key = static_cast<const int32_t*>(M.dev[2]);
  ctx->ad.memo_val = static_cast<const int32_t*>(M.dev[3]);
  ctx->ad.memo_hits = static_cast<unsigned long long*>(M.dev[4]);
  return DYO_OK;
}

dyo_status dyo_report(dyo_ctx* ctx, int32_t b, const int32_t* actual, int32_t* mispredicted) {
  if (!ctx || !actual || b < 0 || b >= ctx->last_B) return DYO_E_INVAL;
  const int ns = ctx->n_sites;
  const TravArch& T = ctx->trav;
  for (int i = 0; i < ns; ++i) {
    if (actual[i] < 0 || actual[i] >= T.site_nch[i]) return fail(ctx, DYO_E_INVAL, "actual choice %d of site %d out of range", actual[i], i);
    if (T.site_tie[i] >= 0 && actual[i] != actual[T.site_tie[i]])
      return fail(ctx, DYO_E_INVAL, "site %d must replay site %d (R6)", i, T.site_tie[i]);
  }
  CK(cudaSetDevice(ctx->device));
  // stream-ordered readback: the aux stream waits for the end of the last dyo_pilot_predict
  // (its decode) and copies the status, the final choices and the memo key of prediction b to
  // pinned memory; the host waits for that stream only
  const int Km = ctx->K_max;
  int32_t* hr = ctx->h_rep;
  int32_t* h_fin = hr + 4;
  int32_t* h_key = h_fin + std::max(ns, 1);
  CK(cudaStreamWaitEvent(ctx->aux, ctx->ev_pred, 0));
  CK(cudaMemcpyAsync(hr, ctx->pd.status, sizeof(int32_t), cudaMemcpyDeviceToHost, ctx->aux));
  if (ns) CK(cudaMemcpyAsync(h_fin, ctx->pd.choices + (size_t)b * ns, 4 * (size_t)ns, cudaMemcpyDeviceToHost, ctx->aux));
  CK(cudaMemcpyAsync(h_key, ctx->pd.slots + (size_t)b * Km * 10, 4 * (size_t)Km * 10, cudaMemcpyDeviceToHost, ctx->aux));
  if (ns) CK(cudaMemcpyAsync(h_key + 10 * Km, ctx->pd.rchoices + (size_t)b * ns, 4 * (size_t)ns, cudaMemcpyDeviceToHost,
                             ctx->aux));
  CK(cudaStreamSynchronize(ctx->aux));
  const int32_t status = hr[0];
  if (status) return fail(ctx, (dyo_status)status, "decode failed (status %d)", status);
  const bool miss = !std::equal(actual, actual + ns, h_fin);
  if (mispredicted) *mispredicted = miss ? 1 : 0;
  if (!miss) return DYO_OK;
  ctx->memo.mispredictions++;
  auto& M = ctx->memo;
  if (M.cap == 0) return DYO_OK;                   // recorded (counted), memo disabled
  std::vector<int32_t> key(h_key, h_key + (size_t)10 * Km + ns);
  const int kt = M.kw + M.ns;
  const uint64_t h = memo_hash_of(key.data(), kt);
  const int slot_old = memo_find(M, h, key.data(), -1);
  dyo_status st;
  if (slot_old >= 0) {                              // same output reported again: most recent wins
    const int id = M.index[slot_old];
    std::copy(actual, actual + ns, &M.val[(size_t)id * ns]);
    M.fifo.erase(std::find(M.fifo.begin(), M.fifo.end(), id));
    M.fifo.push_back(id);
    return memo_upload(ctx, id, false);
  }
  if (M.live == M.cap) {                            // FIFO replacement of the oldest key
    const int old = M.fifo.front();
    M.fifo.erase(M.fifo.begin());
    const int sl = memo_find(M, M.hash[old], nullptr, old);
    if (sl >= 0) { M.index[sl] = -2; ++M.tomb; }
    M.free_ids.push_back(old);
    --M.live;
  }
  const int id = M.free_ids.back();
  M.free_ids.pop_back();
  M.hash[id] = h;
  std::copy(key.begin(), key.end(), &M.key[(size_t)id * kt]);
  std::copy(actual, actual + ns, &M.val[(size_t)id * ns]);
  M.fifo.push_back(id);
  ++M.live;
  if (M.tomb > M.cap / 2) {
    memo_rebuild(M);
  } else {
    int slot = (int)(h & (uint64_t)M.mask);
    while (M.index[slot] >= 0) slot = (slot + 1) & M.mask;
    if (M.index[slot] == -2) --M.tomb;
    M.index[slot] = id;
  }
  if ((st = memo_upload(ctx, id, true))) return st;
  ctx->ad.memo_live = M.live;
  return DYO_OK;
}

dyo_status dyo_memo_stats(dyo_ctx* ctx, int64_t* mispredictions, int32_t* live, int64_t* hits) {
  if (!ctx) return DYO_E_INVAL;
  if (mispredictions) *mispredictions = ctx->memo.mispredictions;
  if (live) *live = ctx->memo.live;
  if (hits) {
    *hits = 0;
    if (!ctx->memo.dev.empty()) {
      // hits counted by the decode kernels of every prediction so far (stream-ordered readback)
      CK(cudaStreamWaitEvent(ctx->aux, ctx->ev_pred, 0));
      CK(cudaMemcpyAsync(ctx->h_rep, ctx->memo.dev[4], 8, cudaMemcpyDeviceToHost, ctx->aux));
      CK(cudaStreamSynchronize(ctx->aux));
      unsigned long long v = 0;
      memcpy(&v, ctx->h_rep, 8);
      *hits = (int64_t)v;
    }
  }
  return DYO_OK;
}

dyo_status dyo_prediction_matched(dyo_ctx* ctx, int32_t b, int32_t* matched) {
  if (!ctx || !matched || b < 0 || b >= ctx->last_B) return DYO_E_INVAL;
  if ((ctx->branch_head && !ctx->nested) || !ctx->h_matched) return fail(ctx, DYO_E_STATE, "no traversal decode in this arch");
  *matched = ctx->h_matched[b];
  return DYO_OK;
}

dyo_status dyo_trace_path(dyo_ctx* ctx, const int32_t* choices, const int32_t* nested, int32_t n_nested, int32_t* ops,
                          int32_t* its, int32_t cap, int32_t* L) {
  if (!ctx || !choices || !L || (n_nested > 0 && !nested)) return DYO_E_INVAL;
  if (!ctx->arch_ok) return fail(ctx, DYO_E_STATE, "load the arch first");
  for (int s2 = 0; s2 < ctx->n_sites; ++s2)
    if (ctx->nest.top[s2] && (choices[s2] < 0 || choices[s2] >= ctx->trav.site_nch[s2]))
      return fail(ctx, DYO_E_INVAL, "choice %d of site %d", choices[s2], s2);
  std::vector<int32_t> pop, pit;
  std::string e;
  dyo_status st = trace_path(ctx->nest, choices, nested, n_nested, pop, pit, e);
  if (st) return fail(ctx, st, "%s", e.c_str());
  *L = (int32_t)pop.size();
  if ((int32_t)pop.size() > cap) return fail(ctx, DYO_E_CAPACITY, "need %zu rows", pop.size());
  if (ops) std::copy(pop.begin(), pop.end(), ops);
  if (its) std::copy(pit.begin(), pit.end(), its);
  return DYO_OK;
}

dyo_status dyo_prediction_nested(dyo_ctx* ctx, int32_t b, int32_t* out, int32_t cap, int32_t* n) {
  if (!ctx || !n || b < 0 || b >= ctx->last_B) return DYO_E_INVAL;
  if (!ctx->nested) { *n = 0; return DYO_OK; }
  if (b >= (int)ctx->last_nested.size()) return fail(ctx, DYO_E_STATE, "no prediction");
  const auto& v = ctx->last_nested[b];
  *n = (int32_t)v.size();
  if ((int32_t)v.size() > cap) return fail(ctx, DYO_E_CAPACITY, "need %zu", v.size());
  if (out) std::copy(v.begin(), v.end(), out);
  return DYO_OK;
}

dyo_status dyo_group_entries(dyo_ctx* ctx, int32_t b, int32_t g, int32_t* outp, int32_t cap, int32_t* n,
                             void* stream) {
  if (!ctx || b < 0 || b >= ctx->last_B || g < 0 || g >= ctx->K_max || !n) return DYO_E_INVAL;
  CK(cudaStreamSynchronize((cudaStream_t)stream));
  int32_t cnt = 0;
  CK(cudaMemcpy(&cnt, ctx->pd.ent_n + (size_t)b * ctx->K_max + g, sizeof cnt, cudaMemcpyDeviceToHost));
  *n = cnt;
  if (cnt > cap) return fail(ctx, DYO_E_CAPACITY, "need %d entries", cnt);
  std::vector<int2> tmp(cnt);
  if (cnt) CK(cudaMemcpy(tmp.data(), ctx->pd.ent + ((size_t)b * ctx->K_max + g) * kEntCap, sizeof(int2) * cnt, cudaMemcpyDeviceToHost));
  for (int i = 0; i < cnt; ++i) {
    outp[3 * i] = tmp[i].x;
    outp[3 * i + 1] = tmp[i].y & 3;
    outp[3 * i + 2] = (tmp[i].y >> 2) & 1;
  }
  return DYO_OK;
}

static dyo_status plan_complete(dyo_ctx* ctx, int32_t* K_out);

dyo_status dyo_plan_async(dyo_ctx* ctx, int32_t b0, int32_t n, void* stream) {
  if (!ctx) return DYO_E_INVAL;
  if (ctx->plan_pending) return fail(ctx, DYO_E_STATE, "a plan is pending: dyo_plan_wait first");
  if (!ctx->arch_ok || ctx->last_B <= 0) return fail(ctx, DYO_E_STATE, "no prediction to plan");
  if (n < 0) { b0 = 0; n = ctx->last_B; }
  if (b0 < 0 || n < 1 || b0 + n > ctx->last_B) return fail(ctx, DYO_E_INVAL, "prediction range");
  CK(cudaSetDevice(ctx->device));
  cudaStream_t st = (cudaStream_t)stream;
  // plan slot (plan_seq & 1): its previous plan (two generations back) must be fully enqueued
  // and its migrations must have consumed the pinned lists and copy descriptors
  // advance the migration cursor past fully enqueued plans BEFORE a slot is reused (a plan-only
  // ctx, DYO_F_NO_HOST_POOL, never migrates: its earlier plans are simply superseded)
  if (!ctx->host_pool) ctx->mig_seq = ctx->plan_seq;
  while (ctx->mig_seq < ctx->plan_seq) {
    const dyo_ctx::PlanSlot& Q = ctx->slot[ctx->mig_seq & 1];
    if (Q.valid && Q.next_j < Q.K) break;
    ctx->mig_seq += 1;
  }
  dyo_ctx::PlanSlot& P = ctx->slot[ctx->plan_seq & 1];
  if (ctx->plan_seq - ctx->mig_seq >= 2)
    return fail(ctx, DYO_E_STATE, "two plans are outstanding: migrate the older one first");
  if (P.ev_pending) { CK(cudaEventSynchronize(P.ev_last)); P.ev_pending = false; }
  P.valid = false;
  ctx->h_status[0] = -100;
  PlanState& in = ctx->state[ctx->committed];
  PlanState& wk = ctx->state[1 - ctx->committed];
  {
    // DYO_FAULT=drop_prefetch:p[:seed] - fault injection: read-first entries of the prediction
    // dropped before planning (the runtime's accesses then fault them in, R17)
    static int parsed = 0;
    static double env_p = 0.0;
    static unsigned long long env_seed = 0;
    if (!parsed) {
      parsed = 1;
      if (const char* e = getenv("DYO_FAULT"))
        if (strncmp(e, "drop_prefetch:", 14) == 0) {
          char* q = nullptr;
          env_p = strtod(e + 14, &q);
          if (q && *q == ':') env_seed = strtoull(q + 1, nullptr, 10);
        }
    }
    const double drop_p = ctx->drop_p >= 0.0 ? ctx->drop_p : env_p;
    const unsigned long long drop_seed = ctx->drop_p >= 0.0 ? ctx->drop_seed : env_seed;
    if (drop_p > 0.0) CK(launch_fault_drop(ctx->ad, ctx->pd, b0, n, drop_p, drop_seed, st));
  }
  {
    TScope ts(ctx, 2, st);
    CK(launch_plan(ctx->ad, ctx->pd, b0, n, ctx->cfg.policy, in, wk, ctx->sc, P.dout, ctx->max_groups, st));
  }
  // the export kernel copies the headers and the EVICT/MOVE/CARRY/ALLOC/FETCH records (the DMA
  // issue needs them on the host) into the pinned mirrors by the counts the planner left in
  // mapped memory; entry records stay on the device until dyo_plan_records asks for them
  CK(launch_plan_export(P.dout, P.hout, st));
  CK(cudaMemcpyAsync(ctx->h_loc, wk.loc, ctx->T, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(ctx->h_off, wk.off, sizeof(int64_t) * ctx->T, cudaMemcpyDeviceToHost, st));
  ctx->plan_pending = true;
  ctx->plan_stream = st;
  return DYO_OK;
}

dyo_status dyo_plan_wait(dyo_ctx* ctx, int32_t* K_out) {
  if (!ctx) return DYO_E_INVAL;
  if (!ctx->plan_pending) return fail(ctx, DYO_E_STATE, "no pending plan");
  return plan_complete(ctx, K_out);
}

dyo_status dyo_plan(dyo_ctx* ctx, int32_t b0, int32_t n, int32_t* K_out, void* stream) {
  dyo_status s0 = dyo_plan_async(ctx, b0, n, stream);
  if (s0) return s0;
  return plan_complete(ctx, K_out);
}

static dyo_status plan_complete(dyo_ctx* ctx, int32_t* K_out) {
  ctx->plan_pending = false;
  CK(cudaSetDevice(ctx->device));
  cudaStream_t st = ctx->plan_stream;
  dyo_ctx::PlanSlot& P = ctx->slot[ctx->plan_seq & 1];
  PlanState& in = ctx->state[ctx->committed];
  CK(cudaStreamSynchronize(st));     // the one synchronisation of the hot path (DMA sizes to host)
  ctx->last_plan_syncs = 1;
  const int32_t status = ctx->h_status[0];
  if (status != 0) {
    // restore the residency mirror of the committed state
    cudaMemcpy(ctx->h_loc, in.loc, ctx->T, cudaMemcpyDeviceToHost);
    cudaMemcpy(ctx->h_off, in.off, sizeof(int64_t) * ctx->T, cudaMemcpyDeviceToHost);
    if (status == DYO_E_BUDGET) return fail(ctx, DYO_E_BUDGET, "transition %d: W_j exceeds half the budget", ctx->h_status[1]);
    if (status == DYO_E_CAPACITY) return fail(ctx, DYO_E_CAPACITY, "capacity exceeded (needed %d)", ctx->h_status[2]);
    return fail(ctx, (dyo_status)(status < 0 ? status : DYO_E_CUDA), "planner status %d", status);
  }
  {
    const int K = ctx->h_counts[0];
    P.n_ent = K > 0 ? P.out.hdr[K - 1].o_ent + P.out.hdr[K - 1].n_ent : 0;
    P.ent_host = false;
  }
  ctx->committed = 1 - ctx->committed;
  P.K = ctx->h_counts[0];
  P.next_j = 0;
  P.seg_used = 0;
  P.valid = true;
  ctx->plan_seq += 1;
  if (K_out) *K_out = P.K;
  return DYO_OK;
}

dyo_status dyo_plan_info(dyo_ctx* ctx, int32_t j, dyo_transition_info* info) {
  if (!ctx || !info) return DYO_E_INVAL;
  if (ctx->plan_seq == 0 || !ctx->slot[(ctx->plan_seq - 1) & 1].valid) return fail(ctx, DYO_E_STATE, "no valid plan");
  const dyo_ctx::PlanSlot& P = ctx->slot[(ctx->plan_seq - 1) & 1];
  if (j < 0 || j >= P.K) return DYO_E_INVAL;
  const PlanHdr& h = P.out.hdr[j];
  info->half = h.half; info->n_entries = h.n_ent; info->n_evict = h.n_evict; info->n_move = h.n_move;
  info->n_carry = h.n_carry; info->n_alloc = h.n_alloc; info->n_fetch = h.n_fetch;
  info->need = h.need; info->h2d = h.h2d; info->d2h = h.d2h; info->d2d = h.d2d;
  info->n_share = h.flags >> 1;
  info->late_all = h.flags & 1;
  return DYO_OK;
}

dyo_status dyo_plan_records(dyo_ctx* ctx, int32_t j, int32_t list, const void** recs, int32_t* n) {
  if (!ctx || !recs || !n) return DYO_E_INVAL;
  if (ctx->plan_seq == 0 || !ctx->slot[(ctx->plan_seq - 1) & 1].valid) return fail(ctx, DYO_E_STATE, "no valid plan");
  const dyo_ctx::PlanSlot& P = ctx->slot[(ctx->plan_seq - 1) & 1];
  if (j < 0 || j >= P.K) return DYO_E_INVAL;
  const PlanHdr& h = P.out.hdr[j];
  switch (list) {
    case 0: *recs = P.out.ev + h.o_evict; *n = h.n_evict; break;
    case 1: *recs = P.out.mv + h.o_move; *n = h.n_move; break;
    case 2: *recs = P.out.ca + h.o_carry; *n = h.n_carry; break;
    case 3: *recs = P.out.al + h.o_alloc; *n = h.n_alloc; break;
    case 4: *recs = P.out.fe + h.o_fetch; *n = h.n_fetch; break;
    case 5:
      if (!P.ent_host) {            // lazily: the migration engine never reads the entries
        if (P.n_ent) CK(cudaMemcpy(P.out.ent, P.dout.ent, sizeof(dyo_entry_rec) * P.n_ent, cudaMemcpyDeviceToHost));
        const_cast<dyo_ctx::PlanSlot&>(P).ent_host = true;
      }
      *recs = P.out.ent + h.o_ent; *n = h.n_ent; break;
    default: return DYO_E_INVAL;
  }
  return DYO_OK;
}

// ---- migration engine -----------------------------------------------------------------
namespace {

struct Run { int64_t host_off, dev_off, bytes; bool dev_contig; int first, count; };


// push (src, dst, bytes) split into work items; returns false on capacity
// the slot being migrated (set by dyo_migrate before it pushes descriptors)
thread_local dyo_ctx::PlanSlot* g_mslot = nullptr;

bool push_seg(dyo_ctx* ctx, const char* src, char* dst, int64_t bytes) {
  dyo_ctx::PlanSlot& P = *g_mslot;
  (void)ctx;
  for (int64_t o = 0; o < bytes; o += kChunk) {
    if (P.seg_used >= P.seg_cap) return false;
    P.h_segs[P.seg_used++] = CopySeg{src + o, dst + o, std::min(kChunk, bytes - o)};
  }
  return true;
}

dyo_status launch_segs(dyo_ctx* ctx, int64_t first, cudaStream_t s, int grid, int kind = 3) {
  dyo_ctx::PlanSlot& P = *g_mslot;
  const int64_t n = P.seg_used - first;
  if (n <= 0) return DYO_OK;
  CopySeg* dptr = nullptr;
  CK(cudaHostGetDevicePointer((void**)&dptr, P.h_segs + first, 0));
  int64_t bytes = 0;
  for (int64_t i = first; i < P.seg_used; ++i) bytes += P.h_segs[i].bytes;
  TScope ts(ctx, kind, s, bytes);
  CK(launch_copy_segments(dptr, (int)n, kChunk, grid, s));
  ctx->ctr.n_kernels++;
  return DYO_OK;
}

// DYO_COPY_LOG=<path>: one line per TMA copy launch with its algorithmic bytes (bytes moved);
// tools/ncu_traffic.py pairs these with an ncu capture's per-launch DRAM bytes (same order).
void log_copy_bytes(int64_t bytes) {
  static FILE* f = nullptr;
  static int init = 0;
  if (!init) {
    init = 1;
    if (const char* e = getenv("DYO_COPY_LOG")) f = fopen(e, "w");
  }
  if (f) { fprintf(f, "%lld\n", (long long)bytes); fflush(f); }
}

// Device<->device copies of plan records [i0, i1) (R = one of the all-int64 record types):
// record k copies rec.bytes from src_base + rec.<f_src> to dst_base + rec.<f_dst> - dst_bias;
// f_late >= 0 selects the records with rec.late == late_val. The TMA copy kernel reads the
// records from the plan's device copy (P.dout); the pinned host copy (P.out) only sizes the
// launch. With DYO_F_SM_COPY the host builds work items for the SM vector-copy kernel instead.
extern "C++" template <class R>
dyo_status d2d_records(dyo_ctx* ctx, const R* hrec, const R* drec, int i0, int i1, int f_src, int f_dst,
                       int f_bytes, int f_late, int64_t late_val, const char* src_base, char* dst_base,
                       int64_t dst_bias, cudaStream_t s, int grid) {
  static_assert(sizeof(R) % sizeof(int64_t) == 0, "records are int64 fields");
  const int stride = (int)(sizeof(R) / sizeof(int64_t));
  int64_t total = 0, bytes = 0;
  for (int k = i0; k < i1; ++k) {
    const int64_t* r = reinterpret_cast<const int64_t*>(hrec + k);
    if (f_late >= 0 && r[f_late] != late_val) continue;
    total += rec_body(src_base + r[f_src], dst_base + (r[f_dst] - dst_bias), r[f_bytes]);
    bytes += r[f_bytes];
  }
  if (bytes == 0) return DYO_OK;
  if (ctx->cfg.flags & DYO_F_SM_COPY) {
    dyo_ctx::PlanSlot& P = *g_mslot;
    const int64_t g0 = P.seg_used;
    for (int k = i0; k < i1; ++k) {
      const int64_t* r = reinterpret_cast<const int64_t*>(hrec + k);
      if (f_late >= 0 && r[f_late] != late_val) continue;
      if (!push_seg(ctx, src_base + r[f_src], dst_base + (r[f_dst] - dst_bias), r[f_bytes]))
        return fail(ctx, DYO_E_CAPACITY, "copy descriptors");
    }
    return launch_segs(ctx, g0, s, grid);
  }
  RecCopyArgs a{};
  a.rec = reinterpret_cast<const int64_t*>(drec + i0);
  a.stride = stride;
  a.n = i1 - i0;
  a.f_src = f_src; a.f_dst = f_dst; a.f_bytes = f_bytes; a.f_late = f_late;
  a.late_val = late_val;
  a.src_base = src_base; a.dst_base = dst_base; a.dst_bias = dst_bias;
  a.total = total;
  TScope ts(ctx, 3, s, bytes);
  log_copy_bytes(bytes);
  CK(launch_copy_records(a, ctx->sm_count, s));
  ctx->ctr.n_kernels++;
  return DYO_OK;
}

// Compaction waves [wv[k].first, wv[k].second) of MOVE records as ONE cooperative launch with a
// grid barrier between consecutive waves (instead of one launch per wave: each launch boundary
// costs ~13 us on a busy stream). Falls back to a launch per wave with DYO_F_SM_COPY, a single
// wave, or DYO_COPY_WAVES=0.
dyo_status d2d_move_waves(dyo_ctx* ctx, const dyo_move_rec* hrec, const dyo_move_rec* drec,
                          const std::vector<std::pair<int, int>>& wv, char* arena, cudaStream_t s, int grid) {
  static int waves_on = -1;
  if (waves_on < 0) { const char* e = getenv("DYO_COPY_WAVES"); waves_on = (e && e[0] == '0') ? 0 : 1; }
  if (wv.empty()) return DYO_OK;
  if (wv.size() == 1 || !waves_on || (ctx->cfg.flags & DYO_F_SM_COPY)) {
    for (const auto& w : wv) {
      dyo_status s1 = d2d_records(ctx, hrec, drec, w.first, w.second, 1, 2, 3, -1, 0, arena, arena, 0, s, grid);
      if (s1) return s1;
    }
    return DYO_OK;
  }
  for (size_t g0 = 0; g0 < wv.size(); g0 += kMaxWaves) {
    const size_t g1 = std::min(wv.size(), g0 + (size_t)kMaxWaves);
    const int i0 = wv[g0].first;
    RecCopyArgs a{};
    a.rec = reinterpret_cast<const int64_t*>(drec + i0);
    a.stride = (int)(sizeof(dyo_move_rec) / sizeof(int64_t));
    a.n = wv[g1 - 1].second - i0;
    a.f_src = 1; a.f_dst = 2; a.f_bytes = 3; a.f_late = -1;
    a.src_base = arena; a.dst_base = arena; a.dst_bias = 0;
    int64_t bytes = 0;
    for (size_t k = g0; k < g1; ++k) {
      int64_t tot = 0;
      for (int q = wv[k].first; q < wv[k].second; ++q) {
        tot += rec_body(arena + hrec[q].src, arena + hrec[q].dst, hrec[q].bytes);
        bytes += hrec[q].bytes;
      }
      a.wave_end[k - g0] = wv[k].second - i0;
      a.wave_total[k - g0] = tot;
      a.total += tot;
    }
    a.n_waves = (int)(g1 - g0);
    a.gbar = ctx->gbar;
    a.gbar_base = ctx->gbar_issued;
    int used = 0;
    {
      TScope ts(ctx, 3, s, bytes);
      log_copy_bytes(bytes);
      CK(launch_copy_records(a, ctx->sm_count, s, &used));
    }
    ctx->gbar_issued += (unsigned)(a.n_waves - 1) * (unsigned)used;
    ctx->ctr.n_kernels++;
  }
  return DYO_OK;
}

// One device<->device range (staged pieces of a self-overlapping move).
dyo_status d2d_range(dyo_ctx* ctx, const char* src, char* dst, int64_t bytes, cudaStream_t s, int grid) {
  if (bytes <= 0) return DYO_OK;
  if (ctx->cfg.flags & DYO_F_SM_COPY) {
    dyo_ctx::PlanSlot& P = *g_mslot;
    const int64_t g0 = P.seg_used;
    if (!push_seg(ctx, src, dst, bytes)) return fail(ctx, DYO_E_CAPACITY, "copy descriptors");
    return launch_segs(ctx, g0, s, grid);
  }
  RecCopyArgs a{};
  a.src_base = src; a.dst_base = dst; a.total = bytes;
  TScope ts(ctx, 3, s, bytes);
  log_copy_bytes(bytes);
  CK(launch_copy_records(a, ctx->sm_count, s));
  ctx->ctr.n_kernels++;
  return DYO_OK;
}

}  // namespace

dyo_status dyo_migrate(dyo_ctx* ctx, int32_t j, void* copy_stream, void* ev_half_free, void* ev_prev_done,
                       void* ev_ready) {
  if (!ctx) return DYO_E_INVAL;
  // the oldest plan with transitions left (plans migrate in FIFO order, at most two outstanding)
  while (ctx->mig_seq < ctx->plan_seq) {
    dyo_ctx::PlanSlot& Q = ctx->slot[ctx->mig_seq & 1];
    if (Q.valid && Q.next_j < Q.K) break;
    ctx->mig_seq += 1;
  }
  if (ctx->mig_seq >= ctx->plan_seq) return fail(ctx, DYO_E_STATE, "dyo_migrate without a pending plan");
  dyo_ctx::PlanSlot& P = ctx->slot[ctx->mig_seq & 1];
  if (j != P.next_j || j >= P.K) return fail(ctx, DYO_E_STATE, "transition %d out of order (next %d)", j, P.next_j);
  if (!ctx->host_pool) return fail(ctx, DYO_E_STATE, "plan-only ctx (DYO_F_NO_HOST_POOL) cannot migrate");
  CK(cudaSetDevice(ctx->device));
  g_mslot = &P;
  cudaStream_t s = (cudaStream_t)copy_stream;
  const PlanHdr& h = P.out.hdr[j];
  char* arena = ctx->arena;
  char* host = ctx->host_pool;
  const int64_t AL = ctx->cfg.align;
  const int64_t dma_min = (ctx->cfg.flags & DYO_F_NO_ZEROCOPY) ? 0 : ctx->cfg.dma_min_bytes;
  const int zc_grid = 16;
  const int d2d_grid = 4 * ctx->sm_count;
  // The EVICT phase runs on the ctx's D2H stream: it only needs the last user of half m (block
  // j-2) to be done, so it overlaps the previous transition's H2D fetches (full-duplex PCIe).
  // Without ev_half_free every prior operation on copy_stream counts as that user.
  cudaStream_t sd = ctx->d2h;
  TRACE("migrate j=%d evict=%d move=%d carry=%d fetch=%d", j, h.n_evict, h.n_move, h.n_carry, h.n_fetch);
  if (ev_half_free) {
    CK(cudaStreamWaitEvent(sd, (cudaEvent_t)ev_half_free, 0));
  } else {
    CK(cudaEventRecord(ctx->ev_entry, s));
    CK(cudaStreamWaitEvent(sd, ctx->ev_entry, 0));
  }
  // 0. write-backs of the faulted tensors block j-1 wrote (R17): after block j-1 ends, the
  //    fault area's bytes go to the tensor's host home and to its valid device copy; this
  //    transition's EVICT (D2H stream) and carries (after ev_moves) are ordered after them
  if (!ctx->fault_wb.empty()) {
    if (ev_prev_done) CK(cudaStreamWaitEvent(s, (cudaEvent_t)ev_prev_done, 0));
    const int64_t seg0 = P.seg_used;                 // one segment-copy launch for all of them
    for (const auto& w : ctx->fault_wb) {
      const int64_t nb = ctx->t_bytes[w.t];
      if (!push_seg(ctx, w.src, host + ctx->t_host[w.t], nb)) return fail(ctx, DYO_E_CAPACITY, "copy descriptors (fault write-backs)");
      if (ctx->mig_loc[w.t] >= 0 &&
          !push_seg(ctx, w.src, arena + ctx->mig_loc[w.t] * ctx->H + ctx->mig_off[w.t], nb))
        return fail(ctx, DYO_E_CAPACITY, "copy descriptors (fault write-backs)");
    }
    if (dyo_status s1 = launch_segs(ctx, seg0, s, 16, 4)) return s1;
    ctx->fault_wb.clear();
    CK(cudaEventRecord(ctx->ev_fault_wb, s));
    CK(cudaStreamWaitEvent(sd, ctx->ev_fault_wb, 0));
  }
  const int64_t stage_half = ctx->staging_bytes / 2 / 256 * 256;
  char* stage_pack = ctx->staging;                 // D2H stream
  char* stage_move = ctx->staging + stage_half;    // copy stream

  // R21: FETCH DMAs wait only for the write-backs whose device range they overwrite (and for
  //      block j-2, the last user of half m), not for the whole EVICT phase. Applies when the
  //      transition has no compaction MOVEs and a bounded number of write-backs; otherwise the
  //      phase order is strict (R12). wb_iv: (src range, index of its copy group's event).
  int n_wb = 0;
  for (int i = 0; i < h.n_evict; ++i) n_wb += P.out.ev[h.o_evict + i].writeback ? 1 : 0;
  const bool relaxed = h.n_move == 0 && ev_half_free && n_wb > 0 && n_wb <= 64 &&
                       !(ctx->cfg.flags & DYO_F_STRICT_ORDER) && !(h.flags & 1);
  struct WbIv { int64_t lo, hi; int ev; };
  std::vector<WbIv> wb_iv;
  int n_wb_ev = 0;
  auto wb_mark = [&](const dyo_evict_rec* ev0, int a0, int a1, bool only_wb) -> dyo_status {
    if (!relaxed) return DYO_OK;
    if (n_wb_ev == (int)ctx->ev_wb.size()) {
      cudaEvent_t e;
      CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
      ctx->ev_wb.push_back(e);
    }
    CK(cudaEventRecord(ctx->ev_wb[n_wb_ev], sd));
    for (int q = a0; q < a1; ++q)
      if (!only_wb || ev0[q].writeback) wb_iv.push_back({ev0[q].src, ev0[q].src + ev0[q].bytes, n_wb_ev});
    ++n_wb_ev;
    return DYO_OK;
  };
  // 1. EVICT writebacks (D2H): host runs (ascending host offset) -> DMA (direct, or K3 packed
  //    through staging when the device sources are scattered), or one zero-copy scatter launch
  //    (K5) for the runs below dma_min
  {
    const dyo_evict_rec* ev = P.out.ev + h.o_evict;
    const dyo_evict_rec* dev_ev = P.dout.ev + h.o_evict;
    std::vector<int> small;
    int i = 0;
    while (i < h.n_evict) {
      if (!ev[i].writeback) { ++i; continue; }
      Run r{ev[i].host_off, ev[i].src, ev[i].bytes, true, i, 1};
      int64_t hend = ev[i].host_off + align_up(ev[i].bytes, AL);
      int64_t dend = ev[i].src + align_up(ev[i].bytes, AL);
      int k = i + 1;
      while (k < h.n_evict && ev[k].writeback && ev[k].host_off == hend) {
        if (ev[k].src != dend) r.dev_contig = false;
        hend = ev[k].host_off + align_up(ev[k].bytes, AL);
        dend = ev[k].src + align_up(ev[k].bytes, AL);
        r.bytes = ev[k].host_off + ev[k].bytes - r.host_off;
        ++k;
        ++r.count;
      }
      if (r.bytes >= dma_min && r.dev_contig) {
        TRACE("  d2h dma host_off=%lld dev=%lld bytes=%lld", (long long)r.host_off, (long long)r.dev_off, (long long)r.bytes);
        { TScope ts(ctx, 6, sd, r.bytes);
          CK(cudaMemcpyAsync(host + r.host_off, arena + r.dev_off, r.bytes, cudaMemcpyDeviceToHost, sd)); }
        ctx->ctr.d2h_dma += r.bytes;
        ctx->ctr.n_dma++;
        if (dyo_status s1 = wb_mark(ev, r.first, r.first + r.count, true)) return s1;
      } else if (r.bytes >= dma_min && !(ctx->cfg.flags & DYO_F_NO_PACK)) {
        int q = r.first;
        while (q < r.first + r.count) {
          const int64_t base = ev[q].host_off;
          int q2 = q;
          while (q2 < r.first + r.count && ev[q2].host_off + ev[q2].bytes - base <= stage_half) ++q2;
          if (q2 == q) {   // a tensor larger than the staging buffer: its own DMA
            { TScope ts(ctx, 6, sd, ev[q].bytes);
              CK(cudaMemcpyAsync(host + ev[q].host_off, arena + ev[q].src, ev[q].bytes, cudaMemcpyDeviceToHost, sd)); }
            ctx->ctr.d2h_dma += ev[q].bytes;
            ctx->ctr.n_dma++;
            if (dyo_status s1 = wb_mark(ev, q, q + 1, true)) return s1;
            ++q;
            continue;
          }
          TRACE("  pack %d tensors", q2 - q);
          dyo_status s1 = d2d_records(ctx, ev, dev_ev, q, q2, 1, 2, 3, -1, 0, arena, stage_pack, base, sd, d2d_grid);
          if (s1) return s1;
          const int64_t len = ev[q2 - 1].host_off + ev[q2 - 1].bytes - base;
          { TScope ts(ctx, 6, sd, len);
            CK(cudaMemcpyAsync(host + base, stage_pack, len, cudaMemcpyDeviceToHost, sd)); }
          ctx->ctr.d2h_packed += len;
          ctx->ctr.n_dma++;
          // the pack kernel read the sources: their ranges are free once it has run, but the
          // staging buffer is reused by the next pack only after this DMA - mark after the DMA
          if (dyo_status s1 = wb_mark(ev, q, q2, true)) return s1;
          q = q2;
        }
      } else {
        for (int q = r.first; q < r.first + r.count; ++q) small.push_back(q);
      }
      i = k;
    }
    if (!small.empty()) {
      const int64_t g0 = P.seg_used;
      for (int q : small) {
        if (!push_seg(ctx, arena + ev[q].src, host + ev[q].host_off, ev[q].bytes))
          return fail(ctx, DYO_E_CAPACITY, "copy descriptors");
        ctx->ctr.d2h_zc += ev[q].bytes;
      }
      dyo_status s1 = launch_segs(ctx, g0, sd, zc_grid, 4);
      if (s1) return s1;
      if (relaxed) {
        if (n_wb_ev == (int)ctx->ev_wb.size()) {
          cudaEvent_t e;
          CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
          ctx->ev_wb.push_back(e);
        }
        CK(cudaEventRecord(ctx->ev_wb[n_wb_ev], sd));
        for (int q : small) wb_iv.push_back({ev[q].src, ev[q].src + ev[q].bytes, n_wb_ev});
        ++n_wb_ev;
      }
    }
  }
  TRACE("  evict phase issued");
  CK(cudaEventRecord(ctx->ev_evict, sd));
  if (relaxed) {
    CK(cudaStreamWaitEvent(s, (cudaEvent_t)ev_half_free, 0));   // block j-2 done: half m is ours
    std::sort(wb_iv.begin(), wb_iv.end(), [](const WbIv& x, const WbIv& y) { return x.lo < y.lo; });
  } else {
    CK(cudaStreamWaitEvent(s, ctx->ev_evict, 0));
  }
  int wb_waited = -1;   // s has waited the copy groups [0, wb_waited] (they complete in order on sd)
  auto wait_wb = [&](int64_t lo, int64_t hi) -> dyo_status {
    if (!relaxed) return DYO_OK;
    int need = -1;
    auto it = std::upper_bound(wb_iv.begin(), wb_iv.end(), lo, [](int64_t v, const WbIv& x) { return v < x.lo; });
    if (it != wb_iv.begin()) --it;   // the interval starting at or before lo may reach into [lo, hi)
    for (; it != wb_iv.end() && it->lo < hi; ++it)
      if (it->hi > lo) need = std::max(need, it->ev);
    if (need > wb_waited) {
      CK(cudaStreamWaitEvent(s, ctx->ev_wb[need], 0));
      wb_waited = need;
    }
    return DYO_OK;
  };
  // R20: this transition compacts a half that holds tensors the running block j-1 SHARE'd, so
  //      its MOVE / CARRY / FETCH wait for block j-1 to end (the EVICTs above never touch them)
  if ((h.flags & 1) && ev_prev_done) CK(cudaStreamWaitEvent(s, (cudaEvent_t)ev_prev_done, 0));

  // 2. MOVE (compaction, R11/R12), ascending destination. Processed in order, moves are safe
  //    (new <= old and every destination ends below the later sources), but run in parallel a
  //    move may overwrite an earlier move's source: group them into waves of mutually
  //    non-overlapping (destination vs source) moves, one copy-kernel launch per wave. A move
  //    overlapping its own source goes through the staging buffer in pieces.
  {
    const dyo_move_rec* mv = P.out.mv + h.o_move;
    const dyo_move_rec* dev_mv = P.dout.mv + h.o_move;
    int wave0 = -1, wave1 = -1;                           // the open wave: records [wave0, wave1)
    std::vector<std::pair<int64_t, int64_t>> wave_src;    // its source ranges
    std::vector<std::pair<int, int>> waves;               // closed waves, launched together
    auto flush = [&]() -> dyo_status {                    // close the open wave
      if (wave0 >= 0) waves.push_back({wave0, wave1});
      wave0 = wave1 = -1;
      wave_src.clear();
      return DYO_OK;
    };
    auto launch_waves = [&]() -> dyo_status {
      dyo_status s1 = flush();
      if (s1) return s1;
      s1 = d2d_move_waves(ctx, mv, dev_mv, waves, arena, s, d2d_grid);
      waves.clear();
      return s1;
    };
    // Many small moves (fragmented halves of small tensors) would make many waves of one or
    // two records: move them in rounds through the staging buffer instead - records -> staging
    // (one launch), staging -> the round's contiguous destination range (one launch). In
    // ascending destination order a round never overwrites a later round's sources (the
    // destinations are prefix sums below every later source), and a round's destination range
    // holds exactly its moves (with their alignment padding).
    int64_t mv_bytes = 0;
    for (int i = 0; i < h.n_move; ++i) mv_bytes += mv[i].bytes;
    bool staged_rounds = h.n_move >= 8 && mv_bytes / h.n_move <= (1 << 20);   // many small moves only
    for (int i = 0; i < h.n_move && staged_rounds; ++i)
      if (align_up(mv[i].bytes, AL) > stage_half) staged_rounds = false;
    for (int i = 0; staged_rounds && i < h.n_move;) {
      const int64_t d0 = mv[i].dst;
      int k = i;
      while (k < h.n_move && mv[k].dst + mv[k].bytes - d0 <= stage_half) ctx->ctr.d2d += mv[k++].bytes;
      dyo_status s1 = d2d_records(ctx, mv, dev_mv, i, k, 1, 2, 3, -1, 0, arena, stage_move, d0, s, d2d_grid);
      if (s1) return s1;
      s1 = d2d_range(ctx, stage_move, arena + d0, mv[k - 1].dst + mv[k - 1].bytes - d0, s, d2d_grid);
      if (s1) return s1;
      i = k;
    }
    for (int i = 0; i < h.n_move && !staged_rounds; ++i) {
      const int64_t src = mv[i].src, dst = mv[i].dst, nbytes = mv[i].bytes;
      ctx->ctr.d2d += nbytes;
      if (dst + nbytes > src) {                     // self-overlap: staged pieces, after the waves
        dyo_status s1 = launch_waves();
        if (s1) return s1;
        for (int64_t o = 0; o < nbytes; o += stage_half) {
          const int64_t n = std::min(stage_half, nbytes - o);
          s1 = d2d_range(ctx, arena + src + o, stage_move, n, s, d2d_grid);
          if (s1) return s1;
          s1 = d2d_range(ctx, stage_move, arena + dst + o, n, s, d2d_grid);
          if (s1) return s1;
        }
        continue;
      }
      bool clash = false;
      for (auto& w : wave_src)
        if (dst < w.second && dst + nbytes > w.first) { clash = true; break; }
      if (clash) {
        dyo_status s1 = flush();
        if (s1) return s1;
      }
      if (wave0 < 0) wave0 = i;
      wave1 = i + 1;
      wave_src.push_back({src, src + nbytes});
    }
    dyo_status s1 = launch_waves();
    if (s1) return s1;
  }
  // 3. early CARRY (D2D, one launch) and FETCH (H2D: DMA per host run, zero-copy gather for
  //    the small runs, one launch)
  //    early CARRYs run on the side stream, concurrently with the FETCH DMAs: their
  //    destinations are disjoint from the fetch destinations and their sources lie in the
  //    other half (read-only here)
  bool carry_side = false;
  {
    const dyo_carry_rec* ca = P.out.ca + h.o_carry;
    int64_t early = 0;
    for (int i = 0; i < h.n_carry; ++i)
      if (!ca[i].late) early += ca[i].bytes;
    ctx->ctr.d2d += early;
    if (early > 0) {
      CK(cudaEventRecord(ctx->ev_moves, s));
      CK(cudaStreamWaitEvent(ctx->side, ctx->ev_moves, 0));
      if (relaxed) CK(cudaStreamWaitEvent(ctx->side, ctx->ev_evict, 0));   // carry destinations: every write-back done
      dyo_status s1 = d2d_records(ctx, ca, P.dout.ca + h.o_carry, 0, h.n_carry, 1, 2, 3, 4, 0, arena, arena, 0,
                                  ctx->side, d2d_grid);
      if (s1) return s1;
      CK(cudaEventRecord(ctx->ev_carry, ctx->side));
      carry_side = true;
    }
  }
  {
    const dyo_fetch_rec* fe = P.out.fe + h.o_fetch;
    const int64_t g0 = P.seg_used;
    int i = 0;
    while (i < h.n_fetch) {
      int64_t hend = fe[i].host_off + align_up(fe[i].bytes, AL);
      int64_t dend = fe[i].dst + align_up(fe[i].bytes, AL);
      int k = i + 1;
      while (k < h.n_fetch && fe[k].host_off == hend && fe[k].dst == dend) {
        hend = fe[k].host_off + align_up(fe[k].bytes, AL);
        dend = fe[k].dst + align_up(fe[k].bytes, AL);
        ++k;
      }
      const int64_t bytes = fe[k - 1].host_off + fe[k - 1].bytes - fe[i].host_off;
      if (bytes >= dma_min) {
        if (dyo_status s1 = wait_wb(fe[i].dst, fe[i].dst + bytes)) return s1;
        TRACE("  h2d dma host_off=%lld dst=%lld bytes=%lld", (long long)fe[i].host_off, (long long)fe[i].dst, (long long)bytes);
        { TScope ts(ctx, 5, s, bytes);
          CK(cudaMemcpyAsync(arena + fe[i].dst, host + fe[i].host_off, bytes, cudaMemcpyHostToDevice, s)); }
        ctx->ctr.h2d_dma += bytes;
        ctx->ctr.n_dma++;
      } else {
        for (int q = i; q < k; ++q) {
          if (!push_seg(ctx, host + fe[q].host_off, arena + fe[q].dst, fe[q].bytes))
            return fail(ctx, DYO_E_CAPACITY, "copy descriptors");
          ctx->ctr.h2d_zc += fe[q].bytes;
        }
      }
      i = k;
    }
    if (relaxed && P.seg_used > g0) CK(cudaStreamWaitEvent(s, ctx->ev_evict, 0));   // small fetches: after all
    dyo_status s1 = launch_segs(ctx, g0, s, zc_grid, 4);
    if (s1) return s1;
  }
  if (carry_side) CK(cudaStreamWaitEvent(s, ctx->ev_carry, 0));
  // R21: late carries and block j (ALLOC'd tensors it writes, CARRY destinations) need every
  //      write-back of this transition done. Without late carries the copy stream does not wait:
  //      ready[j] joins FETCH_j and EVICT_j on the join stream, so FETCH_{j+1} (the other half)
  //      may start while EVICT_j's write-backs still run
  bool any_late = false;
  for (int i = 0; i < h.n_carry; ++i) any_late |= P.out.ca[h.o_carry + i].late != 0;
  const bool join = relaxed && !any_late;
  if (relaxed && any_late) CK(cudaStreamWaitEvent(s, ctx->ev_evict, 0));
  // 4. late CARRY: block j-1 writes them, so they wait for its end
  {
    const dyo_carry_rec* ca = P.out.ca + h.o_carry;
    const bool any = any_late;
    if (any) {
      if (ev_prev_done) CK(cudaStreamWaitEvent(s, (cudaEvent_t)ev_prev_done, 0));
      for (int i = 0; i < h.n_carry; ++i)
        if (ca[i].late) ctx->ctr.d2d += ca[i].bytes;
      dyo_status s1 = d2d_records(ctx, ca, P.dout.ca + h.o_carry, 0, h.n_carry, 1, 2, 3, 4, 1, arena, arena, 0, s,
                                  d2d_grid);
      if (s1) return s1;
    }
  }
  TRACE("  transition %d issued", j);
  if (join) {
    CK(cudaEventRecord(ctx->ev_tail, s));
    CK(cudaStreamWaitEvent(ctx->join, ctx->ev_tail, 0));
    CK(cudaStreamWaitEvent(ctx->join, ctx->ev_evict, 0));
    if (ev_ready) CK(cudaEventRecord((cudaEvent_t)ev_ready, ctx->join));
    CK(cudaEventRecord(P.ev_last, ctx->join));
  } else {
    if (ev_ready) CK(cudaEventRecord((cudaEvent_t)ev_ready, s));
    CK(cudaEventRecord(P.ev_last, s));
  }
  // host replay of the residency after transition j (the fault path's residency check, R17)
  {
    const int m = h.half;
    const int64_t mb = (int64_t)m * ctx->H;
    ctx->mig_prev_alloc.clear();
    for (int i = 0; i < h.n_evict; ++i) ctx->mig_loc[P.out.ev[h.o_evict + i].t] = -1;
    for (int i = 0; i < h.n_move; ++i) ctx->mig_off[P.out.mv[h.o_move + i].t] = P.out.mv[h.o_move + i].dst - mb;
    for (int i = 0; i < h.n_carry; ++i) {
      const auto& r = P.out.ca[h.o_carry + i];
      ctx->mig_loc[r.t] = (int8_t)m; ctx->mig_off[r.t] = r.dst - mb;
    }
    for (int i = 0; i < h.n_alloc; ++i) {
      const auto& r = P.out.al[h.o_alloc + i];
      ctx->mig_prev_alloc.push_back({(int32_t)r.t, {ctx->mig_loc[r.t], ctx->mig_off[r.t]}});
      ctx->mig_loc[r.t] = (int8_t)m; ctx->mig_off[r.t] = r.dst - mb;
    }
    for (int i = 0; i < h.n_fetch; ++i) {
      const auto& r = P.out.fe[h.o_fetch + i];
      ctx->mig_loc[r.t] = (int8_t)m; ctx->mig_off[r.t] = r.dst - mb;
    }
    ctx->last_mig_slot = &P;
    ctx->last_mig_j = j;
    ctx->last_mig_seq = ctx->mig_seq;
  }
  P.ev_pending = true;
  P.next_j = j + 1;
  return DYO_OK;
}

// ---- partition labels (R18) ----------------------
dyo_status dyo_partition(dyo_ctx* ctx, const int32_t* path_ops, const int32_t* path_it, int32_t L, int32_t b,
                         const int64_t* op_time_ns, int32_t K, int32_t method, int64_t H, int64_t bw, int32_t* cuts,
                         int64_t* exposed, int32_t* feasible, void* stream) {
  if (!ctx || !path_ops || !path_it || !op_time_ns || !cuts || !exposed) return DYO_E_INVAL;
  if (!ctx->arch_ok) return fail(ctx, DYO_E_STATE, "load the arch first");
  if (L < 1 || K < 1 || K > L || L > 4096 || method < 0 || method > 3 || bw < 1 || H < 0 || b < 0 ||
      b >= ctx->cfg.max_batch)
    return fail(ctx, DYO_E_INVAL, "partition: L=%d K=%d method=%d", L, K, method);
  for (int r = 0; r < L; ++r)
    if (path_ops[r] < -1 || path_ops[r] >= ctx->n_ops) return fail(ctx, DYO_E_INVAL, "row %d: operator %d", r, path_ops[r]);
  CK(cudaSetDevice(ctx->device));
  cudaStream_t s = (cudaStream_t)stream;
  const size_t lay = (size_t)L * (L + 1);
  const size_t need_b = 3 * lay * 8 + (method == 0 ? (size_t)K * lay * 8 : 0) + (size_t)L * 8 + (size_t)ctx->n_ops * 8 +
                        (size_t)(K + 1) * 4 + 64 + 16;
  if (need_b > ctx->part_bytes) {
    if (ctx->part_buf) { CK(cudaStreamSynchronize(s)); cudaFree(ctx->part_buf); ctx->part_buf = nullptr; ctx->part_bytes = 0; }
    CK(cudaMalloc(&ctx->part_buf, need_b));
    ctx->part_bytes = need_b;
  }
  char* q = static_cast<char*>(ctx->part_buf);
  long long* need = reinterpret_cast<long long*>(q); q += lay * 8;
  long long* fetch = reinterpret_cast<long long*>(q); q += lay * 8;
  long long* comp = reinterpret_cast<long long*>(q); q += lay * 8;
  long long* f = reinterpret_cast<long long*>(q); if (method == 0) q += (size_t)K * lay * 8;
  long long* ons = reinterpret_cast<long long*>(q); q += (size_t)ctx->n_ops * 8;
  int32_t* ops = reinterpret_cast<int32_t*>(q); q += (size_t)L * 4;
  int32_t* its = reinterpret_cast<int32_t*>(q); q += (size_t)L * 4;
  long long* res = reinterpret_cast<long long*>(q); q += 16;
  int* ovf = reinterpret_cast<int*>(q); q += 16;
  int32_t* dcuts = reinterpret_cast<int32_t*>(q);
  CK(cudaMemcpyAsync(ops, path_ops, (size_t)L * 4, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(its, path_it, (size_t)L * 4, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(ons, op_time_ns, (size_t)ctx->n_ops * 8, cudaMemcpyHostToDevice, s));
  CK(cudaMemsetAsync(ovf, 0, 4, s));
  CK(cudaMemsetAsync(res, 0, 16, s));
  CK(launch_partition(ctx->ad, ops, its, L, b, ons, K, method, H, bw, need, fetch, comp, f, dcuts, res, ovf, s));
  long long hres[2] = {0, 0};
  int hovf = 0;
  CK(cudaMemcpyAsync(hres, res, 16, cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(&hovf, ovf, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(cuts, dcuts, (size_t)(K + 1) * 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (hovf) return fail(ctx, DYO_E_CAPACITY, "partition: more distinct tensors per block start than the hash holds");
  if (method == 0) {
    *exposed = hres[0];
    if (feasible) *feasible = hres[0] >= 0 ? 1 : 0;
  } else {
    *exposed = hres[0];
    if (feasible) *feasible = (int32_t)hres[1];
  }
  return DYO_OK;
}

// ---- on-demand fetch of mis-predicted tensors (R17) -------------
dyo_status dyo_fault_config(dyo_ctx* ctx, int64_t area_bytes) {
  if (!ctx || area_bytes < 0) return DYO_E_INVAL;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  if (ctx->fault_area) { cudaFree(ctx->fault_area); ctx->fault_area = nullptr; }
  ctx->fault_cap = ctx->fault_used = 0;
  ctx->fault_wb.clear();
  ctx->fault_j = -1;
  if (area_bytes == 0) return DYO_OK;
  CK(cudaMalloc(&ctx->fault_area, area_bytes));
  ctx->fault_cap = area_bytes;
  if (!ctx->fault_segs) {
    ctx->fseg_cap = 1 << 16;                     // per half
    CK(cudaHostAlloc((void**)&ctx->fault_segs, sizeof(CopySeg) * 2 * ctx->fseg_cap, cudaHostAllocMapped | cudaHostAllocPortable));
    for (auto& e : ctx->ev_fseg) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  return DYO_OK;
}

dyo_status dyo_fault_fetch(dyo_ctx* ctx, int32_t j, const int32_t* ids, const int32_t* modes, int32_t n,
                           void** dev_ptrs, void* stream, void* ev_done) {
  if (!ctx || (n > 0 && (!ids || !modes || !dev_ptrs)) || n < 0) return DYO_E_INVAL;
  if (!ctx->fault_area) return fail(ctx, DYO_E_STATE, "dyo_fault_config first");
  dyo_ctx::PlanSlot* P = ctx->last_mig_slot;
  if (!P || j != ctx->last_mig_j || !P->valid || ctx->last_mig_seq != ctx->mig_seq)
    return fail(ctx, DYO_E_STATE, "block %d is not the last migrated transition", j);
  CK(cudaSetDevice(ctx->device));
  cudaStream_t s = (cudaStream_t)stream;
  const PlanHdr& h = P->out.hdr[j];
  // the planned W_j with its placement: the plan's entry records, copied to the host once per
  // plan (the first fault fetch or dyo_plan_records), then a tensor -> entry index for block j
  if (!P->ent_host) {
    if (P->n_ent) CK(cudaMemcpy(P->out.ent, P->dout.ent, sizeof(dyo_entry_rec) * P->n_ent, cudaMemcpyDeviceToHost));
    P->ent_host = true;
  }
  const dyo_entry_rec* ent = P->out.ent + h.o_ent;
  std::unordered_map<int32_t, int32_t> ent_of;
  ent_of.reserve((size_t)h.n_ent * 2);
  for (int q = 0; q < h.n_ent; ++q) ent_of.emplace((int32_t)ent[q].t, q);
  auto find_ent = [&](int t) -> const dyo_entry_rec* {
    auto it = ent_of.find(t);
    return it == ent_of.end() ? nullptr : ent + it->second;
  };
  if (ctx->fault_j != j) {
    ctx->fault_used = 0;
    ctx->fault_j = j;
    CK(cudaEventSynchronize(ctx->ev_fseg[j & 1]));    // block j-2's fault copies have run
    ctx->fseg_used = 0;
  }
  // copies after transition j's migrations (stream order with the ctx's last migrate); the
  // fault copies of the call go to the SM copy kernel as one launch (device and mapped pinned
  // host sources alike) instead of one cudaMemcpyAsync per tensor
  CK(cudaStreamWaitEvent(s, P->ev_last, 0));
  CopySeg* fsegs = ctx->fault_segs + (int64_t)(j & 1) * ctx->fseg_cap;
  const int64_t seg0 = ctx->fseg_used;
  auto push_fault = [&](const char* src, char* dst, int64_t bytes) -> bool {
    for (int64_t o = 0; o < bytes; o += kChunk) {
      if (ctx->fseg_used >= ctx->fseg_cap) return false;
      fsegs[ctx->fseg_used++] = CopySeg{src + o, dst + o, std::min(kChunk, bytes - o)};
    }
    return true;
  };
  const int64_t AL = ctx->cfg.align;
  for (int i = 0; i < n; ++i) {
    const int t = ids[i], md = modes[i];
    if (t < 0 || t >= ctx->T || md < 1 || md > 3) return fail(ctx, DYO_E_INVAL, "fault %d: tensor %d mode %d", i, t, md);
    const dyo_entry_rec* e = find_ent(t);
    // residency check: planned and valid for this access -> its slot. Valid: the
    // plan fetched it (or the access writes first), and a write is one the plan knows about
    // (a write the plan does not expect would leave a device copy it treats as clean)
    if (e && (e->needs_fetch || !(md & 1)) && (!(md & 2) || (e->mode & 2))) {
      dev_ptrs[i] = ctx->arena + e->dst;
      ++ctx->n_fault_resident;
      continue;
    }
    // miss: a fault-area copy from the tensor's latest bytes - its valid device copy after
    // transition j (or, for a tensor the plan ALLOCs in this transition, its copy before it),
    // else its host home
    // the area's halves alternate between blocks: block j's half is still read by block j and
    // by the write-backs migrate(j+1) enqueues; block j+2 reuses it after its EVICT waited for
    // block j's end
    const int64_t nb = ctx->t_bytes[t], ab = align_up(nb, AL);
    const int64_t half = ctx->fault_cap / 2 / AL * AL;
    if (ctx->fault_used + ab > half)
      return fail(ctx, DYO_E_CAPACITY, "fault area: need %lld bytes per block", (long long)(ctx->fault_used + ab));
    char* dst = ctx->fault_area + (j & 1) * half + ctx->fault_used;
    ctx->fault_used += ab;
    int8_t loc = ctx->mig_loc[t];
    int64_t off = ctx->mig_off[t];
    for (const auto& pa : ctx->mig_prev_alloc)       // ALLOC'd at j: its slot holds no bytes yet
      if (pa.first == t) { loc = pa.second.first; off = pa.second.second; }
    if (md & 1) {
      const char* src = loc >= 0 ? ctx->arena + loc * ctx->H + off : ctx->host_pool + ctx->t_host[t];
      if (!push_fault(src, dst, nb)) return fail(ctx, DYO_E_CAPACITY, "copy descriptors (faults)");
      ctx->fault_bytes += nb;
    }
    if (md & 2) ctx->fault_wb.push_back({t, dst});
    dev_ptrs[i] = dst;
    ++ctx->n_faults;
  }
  // repair: a tensor the plan ALLOCs at transition j (its slot holds no bytes; the plan expects
  // block j to write it and treats it as dirty afterwards) that the actual block does not write
  // through that slot would later be written back with the slot's stale bytes: its latest bytes
  // are copied into the slot now (from its previous device copy, else its host home)
  for (const auto& pa : ctx->mig_prev_alloc) {
    const int t = pa.first;
    const dyo_entry_rec* e = find_ent(t);
    if (!e) continue;
    bool written = false;
    for (int i = 0; i < n && !written; ++i)
      written = ids[i] == t && (modes[i] & 2) && dev_ptrs[i] == ctx->arena + e->dst;
    if (written) continue;
    const int8_t loc = pa.second.first;
    const int64_t off = pa.second.second, nb = ctx->t_bytes[t];
    const char* src = loc >= 0 ? ctx->arena + loc * ctx->H + off : ctx->host_pool + ctx->t_host[t];
    if (!push_fault(src, ctx->arena + e->dst, nb)) return fail(ctx, DYO_E_CAPACITY, "copy descriptors (faults)");
    ++ctx->n_fault_repair;
  }
  if (ctx->fseg_used > seg0) {
    CopySeg* dptr = nullptr;
    CK(cudaHostGetDevicePointer((void**)&dptr, fsegs + seg0, 0));
    TScope ts(ctx, 4, s, 0);
    CK(launch_copy_segments(dptr, (int)(ctx->fseg_used - seg0), kChunk, 16, s));
    ctx->ctr.n_kernels++;
  }
  CK(cudaEventRecord(ctx->ev_fseg[j & 1], s));
  if (ev_done) CK(cudaEventRecord((cudaEvent_t)ev_done, s));
  return DYO_OK;
}

dyo_status dyo_fault_inject(dyo_ctx* ctx, double p, uint64_t seed) {
  if (!ctx || !(p <= 1.0)) return DYO_E_INVAL;
  ctx->drop_p = p;
  ctx->drop_seed = seed;
  return DYO_OK;
}

dyo_status dyo_fault_flush(dyo_ctx* ctx, void* stream, void* ev_block_end) {
  if (!ctx) return DYO_E_INVAL;
  if (ctx->fault_wb.empty()) return DYO_OK;
  CK(cudaSetDevice(ctx->device));
  cudaStream_t s = (cudaStream_t)stream;
  if (ev_block_end) CK(cudaStreamWaitEvent(s, (cudaEvent_t)ev_block_end, 0));
  for (const auto& w : ctx->fault_wb) {
    const int64_t nb = ctx->t_bytes[w.t];
    CK(cudaMemcpyAsync(ctx->host_pool + ctx->t_host[w.t], w.src, nb, cudaMemcpyDeviceToHost, s));
    if (ctx->mig_loc[w.t] >= 0)
      CK(cudaMemcpyAsync(ctx->arena + ctx->mig_loc[w.t] * ctx->H + ctx->mig_off[w.t], w.src, nb, cudaMemcpyDeviceToDevice, s));
  }
  ctx->fault_wb.clear();
  return DYO_OK;
}

dyo_status dyo_fault_stats(dyo_ctx* ctx, int64_t* faults, int64_t* bytes, int64_t* resident) {
  if (!ctx) return DYO_E_INVAL;
  if (faults) *faults = ctx->n_faults;
  if (bytes) *bytes = ctx->fault_bytes;
  if (resident) *resident = ctx->n_fault_resident;
  return DYO_OK;
}

dyo_status dyo_residency(dyo_ctx* ctx, int32_t t, void** dev_ptr) {
  if (ctx && ctx->plan_pending) return fail(ctx, DYO_E_STATE, "dyo_residency: a plan is pending (dyo_plan_wait first)");
  if (!ctx || !dev_ptr || t < 0 || t >= ctx->T) return DYO_E_INVAL;
  const int8_t l = ctx->h_loc[t];
  *dev_ptr = l < 0 ? nullptr : ctx->arena + (int64_t)l * ctx->H + ctx->h_off[t];
  return DYO_OK;
}

dyo_status dyo_get_timings(dyo_ctx* ctx, int32_t kind, double* ms, int64_t* launches, int64_t* bytes,
                           double* busy_ms, int32_t reset) {
  if (!ctx || kind < 0 || kind >= DYO_T_KINDS) return DYO_E_INVAL;
  drain_timings(ctx);
  if (ms) *ms = ctx->tm_ms[kind];
  if (launches) *launches = ctx->tm_n[kind];
  if (bytes) *bytes = ctx->tm_bytes[kind];
  if (busy_ms) {
    // length of the union of this kind's [start, end] intervals: launches of one kind that run
    // concurrently on different streams share the hardware, so their summed durations overstate
    // the time the kind kept the GPU busy
    auto iv = ctx->tm_iv[kind];
    std::sort(iv.begin(), iv.end());
    double tot = 0, cs = -1, ce = -1;
    for (auto& p : iv) {
      if (p.first > ce) { if (ce > cs) tot += ce - cs; cs = p.first; ce = p.second; }
      else if (p.second > ce) ce = p.second;
    }
    if (ce > cs) tot += ce - cs;
    *busy_ms = tot;
  }
  if (reset) {
    for (int k = 0; k < DYO_T_KINDS; ++k) { ctx->tm_ms[k] = 0; ctx->tm_n[k] = 0; ctx->tm_bytes[k] = 0; ctx->tm_iv[k].clear(); }
    if (!ctx->ev_ref) cudaEventCreate(&ctx->ev_ref);
    cudaEventRecord(ctx->ev_ref, 0);
  }
  return DYO_OK;
}

dyo_status dyo_debug_copy(dyo_ctx* ctx, const void* src, void* dst, int64_t bytes, int32_t mode, void* stream) {
  if (!ctx || !src || !dst || bytes < 0) return DYO_E_INVAL;
  CK(cudaSetDevice(ctx->device));
  // descriptors in a temporary device buffer (work items of kChunk bytes)
  std::vector<CopySeg> segs;
  for (int64_t o = 0; o < bytes; o += kChunk)
    segs.push_back(CopySeg{(const char*)src + o, (char*)dst + o, std::min(kChunk, bytes - o)});
  if (segs.empty()) return DYO_OK;
  CopySeg* d = nullptr;
  CK(cudaMallocAsync((void**)&d, sizeof(CopySeg) * segs.size(), (cudaStream_t)stream));
  CK(cudaMemcpyAsync(d, segs.data(), sizeof(CopySeg) * segs.size(), cudaMemcpyHostToDevice, (cudaStream_t)stream));
  if (mode == 1) {
    RecCopyArgs a{};
    a.src_base = (const char*)src; a.dst_base = (char*)dst; a.total = bytes;
    CK(launch_copy_records(a, ctx->sm_count, (cudaStream_t)stream));
  }
  else CK(launch_copy_segments(d, (int)segs.size(), kChunk, 4 * ctx->sm_count, (cudaStream_t)stream));
  CK(cudaFreeAsync(d, (cudaStream_t)stream));
  CK(cudaStreamSynchronize((cudaStream_t)stream));
  return DYO_OK;
}

dyo_status dyo_debug_floor(dyo_ctx* ctx, int32_t cluster, int32_t n_barriers, void* stream) {
  if (!ctx || cluster < 1 || cluster > 16 || n_barriers < 0) return DYO_E_INVAL;
  CK(cudaSetDevice(ctx->device));
  CK(launch_floor(cluster, n_barriers, (cudaStream_t)stream));
  return DYO_OK;
}

dyo_status dyo_debug_copy_stamps(dyo_ctx* ctx, uint64_t* out, int64_t cap, int64_t* n) {
  if (!ctx || cap < 0 || !n) return DYO_E_INVAL;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  const int64_t k = copy_stamps_read(reinterpret_cast<unsigned long long*>(out), cap);
  if (k < 0) return fail(ctx, DYO_E_CUDA, "copy stamps readback");
  *n = k;
  return DYO_OK;
}

dyo_status dyo_debug_pilot_stamps(dyo_ctx* ctx, int32_t enable, uint64_t* out32) {
  if (!ctx) return DYO_E_INVAL;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  CK(debug_stamps(enable, reinterpret_cast<unsigned long long*>(out32)));
  CK(tc_debug_stamps(enable, ctx->last_tc ? reinterpret_cast<unsigned long long*>(out32) : nullptr));
  return DYO_OK;
}

dyo_status dyo_debug_plan_stamps(dyo_ctx* ctx, int32_t j, uint64_t* out64) {
  if (!ctx) return DYO_E_INVAL;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  CK(plan_debug_stamps(j, reinterpret_cast<unsigned long long*>(out64)));
  return DYO_OK;
}

dyo_status dyo_set_timing(dyo_ctx* ctx, int32_t on) {
  if (!ctx || on < 0 || on > 1) return DYO_E_INVAL;
  if (on) ctx->cfg.flags |= DYO_F_TIMING;
  else ctx->cfg.flags &= ~DYO_F_TIMING;
  return DYO_OK;
}

dyo_status dyo_query(dyo_ctx* ctx, int32_t what, int64_t* value) {
  if (!ctx || !value) return DYO_E_INVAL;
  switch (what) {
    case DYO_Q_PILOT_KERNEL: *value = ctx->last_tc; return DYO_OK;
    case DYO_Q_DECODE_FUSED: *value = ctx->last_fused; return DYO_OK;
    case DYO_Q_PLAN_SYNCS: *value = ctx->last_plan_syncs; return DYO_OK;
    case DYO_Q_HOST_DECODE: *value = (!ctx->branch_head || ctx->nested) ? 1 : 0; return DYO_OK;
    case DYO_Q_HOST_NUMA: *value = ctx->host_numa; return DYO_OK;
  }
  return DYO_E_INVAL;
}

dyo_status dyo_get_counters(dyo_ctx* ctx, dyo_counters* c, int32_t reset) {
  if (!ctx || !c) return DYO_E_INVAL;
  *c = ctx->ctr;
  if (reset) ctx->ctr = dyo_counters{};
  return DYO_OK;
}

}  // extern "C"
